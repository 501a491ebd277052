"""Small loopback V-cycle (debug aid): python tools/dist_repro.py [G] [n] [nlev] [agg_rows] [prec]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402
from paper_conf_sc_luzwflcy0c024_b200.dist import DistHierarchy, run_loopback  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 2
n = int(sys.argv[2]) if len(sys.argv) > 2 else 32
nlev = int(sys.argv[3]) if len(sys.argv) > 3 else 4
agg = int(sys.argv[4]) if len(sys.argv) > 4 else 32768
prec = tuple((sys.argv[5] if len(sys.argv) > 5 else "f64,f64,f64,f64,f64,f64,f64").split(","))[:nlev]
dims = (n, n, n)
rows = gen.partition.slab_ranges(n, n * n, G)
bglob = gen.uniform_vector(n ** 3, 3)


def fn(r, comm, st):
    A, rws, nn, Ps = gen.partition.slab_inputs("7pt", dims, nlev, r, G, device="cuda")
    MA = amgt.from_csr(A)
    MPs = [amgt.from_csr(P) for P in Ps]
    H = DistHierarchy(comm, MA, MPs, level_prec=prec, agg_rows=agg)
    print(r, H.info(), flush=True)
    b = bglob[rws[0]:rws[1]].cuda()
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res, calls = H.vcycle(b, x, 3)
    return res, calls


print(run_loopback(G, lambda r: rows[r], fn))
