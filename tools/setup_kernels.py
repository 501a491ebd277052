"""One hierarchy setup of a config (after a warm-up setup) inside an NVTX range "setup", for an ncu
launch list of the setup kernels: python tools/setup_kernels.py [config]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

cfg = gen.configs.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "cfg3"]
A = gen.configs.build_matrix(cfg, device="cuda")
PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device="cuda")
Ps = [P for P, _ in PR]
for rep in range(2):
    torch.cuda.synchronize()
    if rep:
        torch.cuda.nvtx.range_push("setup")
    M = amgt.from_csr(A)
    MPs = [amgt.from_csr(P) for P in Ps]
    H = amgt.Hierarchy(M, MPs, level_prec=cfg.level_prec[:cfg.nlev])
    torch.cuda.synchronize()
    if rep:
        torch.cuda.nvtx.range_pop()
    H.close()
    M.free()
    for P in MPs:
        P.free()
print("ok")
