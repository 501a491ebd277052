"""Run the hot kernels on a config a few times (for ncu captures; not a benchmark).

usage: python tools/profile_kernels.py [spmv|spgemm|all] [reps] [N] [7pt|27pt]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

what = sys.argv[1] if len(sys.argv) > 1 else "all"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
N = int(sys.argv[3]) if len(sys.argv) > 3 else 128
kind = sys.argv[4] if len(sys.argv) > 4 else "7pt"
A = (gen.laplacian_7pt if kind == "7pt" else gen.laplacian_27pt)(N, device="cuda")
P = gen.aggregation_P((N, N, N), 0.5, device="cuda")
R = gen.aggregation_R((N, N, N), 0.5, device="cuda")
for _ in range(reps):
    MA = amgt.from_csr(A)
    if what in ("spmv", "all"):
        MA.analyze()
        x = gen.uniform_vector(A.n, 1).cuda()
        y = torch.empty(A.m, dtype=torch.float64, device="cuda")
        for _ in range(reps):
            amgt.spmv(MA, x, y)
        MA32 = MA.cast("f32")
        amgt.spmv(MA32, x.float(), torch.empty(A.m, dtype=torch.float32, device="cuda"))
    if what in ("spgemm", "all"):
        MP, MR = amgt.from_csr(P), amgt.from_csr(R)
        AP = amgt.spgemm(MA, MP)
        Ac = amgt.spgemm(MR, AP)
torch.cuda.synchronize()
print("done")
