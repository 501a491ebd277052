"""Partitioning overhead of the distributed path on ONE GPU: config-5-shaped problems (7-point,
2x2x2 aggregation) split over G = 1 / 2 / 4 / 8 virtual ranks (loopback transport, one host
thread + stream per rank).  The total work is the same for every G, so the time above G = 1 is
what the partition costs: halo exchanges, boundary-row launches, the agglomerated tail's
all-gather, host rendezvous.  Prints one JSON line per G.

  python tools/dist_overhead.py [--n 512] [--nlev 7] [--cycles 10] [--G 1,2,4,8]
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402
from paper_conf_sc_luzwflcy0c024_b200.dist import DistHierarchy, run_loopback  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--nlev", type=int, default=7)
    ap.add_argument("--cycles", type=int, default=10)
    ap.add_argument("--G", default="1,2,4,8")
    ap.add_argument("--agg-rows", type=int, default=32768)
    ap.add_argument("--prec", default="f64,f32,f16,f16,f16,f16,f16")
    a = ap.parse_args()
    dims = (a.n, a.n, a.n)
    lp = tuple(a.prec.split(","))[:a.nlev]
    n = a.n ** 3
    bglob = gen.uniform_vector(n, 5)
    base = None
    for G in [int(g) for g in a.G.split(",")]:
        rows = gen.partition.slab_ranges(a.n, a.n * a.n, G)

        def fn(r, comm, st):
            A, rws, nn, Ps = gen.partition.slab_inputs("7pt", dims, a.nlev, r, G, device="cuda")
            b = bglob[rws[0]:rws[1]].cuda()
            x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
            torch.cuda.synchronize()
            out = {}
            for rep in range(2):  # second repetition timed (warm allocator, NCCL-free)
                e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                t0 = time.perf_counter()
                e0.record(st)
                MA = amgt.from_csr(A)
                MPs = [amgt.from_csr(P) for P in Ps]
                H = DistHierarchy(comm, MA, MPs, level_prec=lp, agg_rows=a.agg_rows)
                e1.record(st)
                t1 = time.perf_counter()
                H.vcycle(b, x, 1)
                e2_ = torch.cuda.Event(enable_timing=True)
                e2_.record(st)
                res, calls = H.vcycle(b, x, a.cycles)
                e2.record(st)
                st.synchronize()
                out = {"setup_ms": e0.elapsed_time(e1), "setup_host_ms": (t1 - t0) * 1e3,
                       "cycle_ms": e2_.elapsed_time(e2) / a.cycles, "calls": calls, "info": H.info(),
                       "rel_res": res[-1] / res[0]}
                H.close()
                MA.free()
                for M in MPs:
                    M.free()
            return out

        outs = run_loopback(G, lambda r: rows[r], fn)
        cyc = max(o["cycle_ms"] for o in outs)
        setup = max(o["setup_ms"] for o in outs)
        if base is None:
            base = (cyc, setup)
        print(json.dumps({"G": G, "grid": f"{a.n}^3", "nlev": a.nlev, "cycle_ms": round(cyc, 4),
                          "setup_ms": round(setup, 3), "cycle_overhead": round(cyc / base[0] - 1, 4),
                          "setup_overhead": round(setup / base[1] - 1, 4),
                          "agg_level": outs[0]["info"]["agg_level"], "calls": outs[0]["calls"],
                          "rel_res": outs[0]["rel_res"],
                          "per_rank_cycle_ms": [round(o["cycle_ms"], 4) for o in outs]}), flush=True)


if __name__ == "__main__":
    main()
