"""Config 4 (irregular 2^18 block rows) A*A SpGEMM once (for ncu launch lists)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

A = gen.configs.build_matrix(gen.configs.CONFIGS["cfg4"], device="cuda")
M = amgt.from_csr(A)
for _ in range(int(sys.argv[1]) if len(sys.argv) > 1 else 1):
    C, info = amgt.spgemm(M, M, info=True)
    torch.cuda.synchronize()
print(info)
