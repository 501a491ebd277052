"""Fused-sweep microbenchmark on config 2's level-1 operator (FP64 7-point 128^3): the
three-stage sweep {Jacobi, Jacobi + residual norm, residual} of amgt_spmv_sweeps against the
same three steps as separate kernels, L2 flushed before each repetition, CUDA events on the
launching stream.  Wavefront knobs per setting: AMGT_SWEEP_CTAS (CTAs per SM) and
AMGT_SWEEP_LAG (extra lag in chunks beyond the bandwidth), read at plan creation.

usage: python tools/sweep_bench.py [N] [reps] [ctas:lag,ctas:lag,...]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 128
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
settings = [tuple(int(v) for v in s.split(":")) for s in (sys.argv[3] if len(sys.argv) > 3 else
                                                          "4:-1,4:0,4:128,4:296,2:-1,2:0,1:-1,1:0,4:100000").split(",")]
impls = (sys.argv[4] if len(sys.argv) > 4 else "tma").split(",")
A = gen.laplacian_7pt(N, device="cuda")
M = amgt.from_csr(A).analyze()
n = 4 * M.blc_row
x = gen.uniform_vector(n, 1).cuda()
b = gen.uniform_vector(n, 2).cuda()
d = torch.full((n,), 1.0 / 6.0, dtype=torch.float64, device="cuda")
v = [torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(4)]
nrm = torch.zeros(1, dtype=torch.float64, device="cuda")
flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
a_bytes = M.blc_num * (16 * 8 + 6) + (M.blc_row + 1) * 8
pass_bytes = a_bytes + 8 * n * (3 + 3)
s = torch.cuda.current_stream()


def timed(fn):
    ts = []
    for i in range(reps + 2):
        flush.fill_(float(i))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2] * 1e3


def separate():
    amgt.spmv_fused(M, x, v[0], "jacobi", b=b, dinv=d)
    amgt.spmv_jacobi_res(M, v[0], v[1], b, d, v[3])
    amgt.spmv_fused(M, v[1], v[2], "residual", b=b)


out = {"lib": os.path.basename(amgt.LIB_PATH), "N": N, "tiles": M.blc_num, "A_bytes": a_bytes, "pass_bytes": pass_bytes,
       "separate_us": round(timed(separate), 1),
       "single_jacobi_us": round(timed(lambda: amgt.spmv_fused(M, x, v[0], "jacobi", b=b, dinv=d)), 1)}
for impl, (ctas, lag) in [(i, st_) for i in impls for st_ in settings]:
    os.environ["AMGT_SWEEP_IMPL"] = impl
    os.environ["AMGT_SWEEP_CTAS"] = str(ctas)
    if lag >= 0:
        os.environ["AMGT_SWEEP_LAG"] = str(lag)
    else:
        os.environ.pop("AMGT_SWEEP_LAG", None)
    plan = amgt.SweepPlan(M)
    st = [("jacobi", x, v[0]), ("jacobi_res", v[0], v[1]), ("residual", v[1], v[2])]
    us = timed(lambda: plan.run(st, b, d, norm=nrm))
    out[f"{impl}_c{ctas}_l{lag}"] = {"us": round(us, 1), "GBps_pass": round(pass_bytes / (us * 1e-6) / 1e9, 1)}
    plan.stats()
    plan.run(st, b, d, norm=nrm)
    stt = plan.stats()
    if impl == "tma" and stt["n_later"]:
        items = max(stt["polls"], 1)  # stats[5] = consumer items
        out[f"{impl}_stats_c{ctas}_l{lag}"] = {k_: round(v_ / 1.9e3 / 148, 1) for k_, v_ in
                                               zip(("prod_issue_us", "prod_empty_wait_us", "prod_dep_wait_us",
                                                    "cons_full_wait_us_4groups", "cons_compute_us_4groups",
                                                    "prod_total_us"),
                                                   [stt["cyc_s0"], stt["n_s0"], stt["cyc_later"], stt["n_later"],
                                                    stt["cyc_wait"], stt["polls"]])}
    elif stt["n_s0"]:
        out[f"{impl}_stats_c{ctas}_l{lag}"] = {"us_s0": round(stt["cyc_s0"] / stt["n_s0"] / 1.9e3, 2),
                                       "us_later": round(stt["cyc_later"] / max(stt["n_later"], 1) / 1.9e3, 2),
                                       "us_wait": round(stt["cyc_wait"] / max(stt["n_later"], 1) / 1.9e3, 2),
                                       "polls_per_later": round(stt["polls"] / max(stt["n_later"], 1), 2)}
    if lag < 0:  # one and two stages (persistent-loop overhead without / with one wait level)
        out[f"{impl}_1stage_c{ctas}"] = round(timed(lambda: plan.run(st[:1], b, d)), 1)
        out[f"{impl}_2stage_c{ctas}"] = round(timed(lambda: plan.run(st[:2], b, d, norm=nrm)), 1)
    plan.close()
print(json.dumps(out))
