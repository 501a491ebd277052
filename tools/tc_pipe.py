"""One numeric SpGEMM (27-point 64^3 A*A, FP64) and one SpMV per tensor-core threshold, for an
ncu capture of the tensor / FP64 pipe activity of the DMMA routes (tensor-pipe
utilisation of the numeric SpGEMM tiles as evidence).  Order: thresholds 10 (paper), 0 (all
tiles), 17 (none); ncu -k regex:"k_numeric|k_spmv_rows".

usage: python tools/tc_pipe.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

X = gen.laplacian_27pt(64, device="cuda")
M = amgt.from_csr(X)
C = amgt.spgemm_symbolic(M, M)
x = torch.rand(4 * M.blc_col, dtype=torch.float64, device="cuda")
for thr in (10, 0, 17):
    amgt.set_tc_threshold(thr, thr)
    amgt.spgemm_numeric(M, M, C)
    amgt.spmv(M, x)
    torch.cuda.synchronize()
amgt.set_tc_threshold(17, 17)
print("ok")
