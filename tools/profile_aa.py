"""A*A SpGEMM on a stencil (numeric repeated; for ncu captures of the warp numeric kernel).
usage: python tools/profile_aa.py [7pt|27pt] [N] [prec] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

kind = sys.argv[1] if len(sys.argv) > 1 else "7pt"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 128
prec = sys.argv[3] if len(sys.argv) > 3 else "f64"
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
A = (gen.laplacian_7pt if kind == "7pt" else gen.laplacian_27pt)(N, device="cuda")
M = amgt.from_csr(A, prec=prec)
C, info = amgt.spgemm_symbolic(M, M, info=True)
for _ in range(reps):
    amgt.spgemm_numeric(M, M, C)
torch.cuda.synchronize()
nC = torch.diff(C.blc_ptr).cpu()
print(info, "C tiles", C.blc_num, "max row", int(nC.max()), "rows>8", int((nC > 8).sum()))
