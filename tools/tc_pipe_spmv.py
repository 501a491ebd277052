"""SpMV tensor-core routes vs CUDA cores for an ncu capture (tensor-pipe activity, DRAM bytes):
27-point 128^3 and config 4 (2^18 block rows, 44% of tiles with popcount >= 10), FP64 and FP16,
thresholds 17 (CUDA cores), 10 (paper's rule per tile), 0 (every tile).
  ncu --set full -k regex:"k_spmv" python tools/tc_pipe_spmv.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

for mk in (lambda: gen.laplacian_27pt(128, device="cuda"), lambda: gen.irregular_block_sparse(1 << 18).to("cuda")):
    M = amgt.from_csr(mk()).analyze()
    M16 = M.cast("f16").analyze()
    x = torch.rand(4 * M.blc_col, dtype=torch.float64, device="cuda")
    x32 = x.float()
    y32 = torch.empty(4 * M.blc_row, dtype=torch.float32, device="cuda")
    for thr in (17, 10, 0):
        amgt.set_tc_threshold(17, thr)
        amgt.spmv(M, x)
        amgt.spmv(M16, x32, y32)
        torch.cuda.synchronize()
amgt.set_tc_threshold(17, 17)
print("ok")
