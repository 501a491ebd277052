"""Hierarchy + a few V-cycles of a config (for ncu launch lists of the solve phase):
python tools/profile_vcycle.py [cycles] [config]  (config default cfg2)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

cycles = int(sys.argv[1]) if len(sys.argv) > 1 else 2
cfg = gen.configs.CONFIGS[sys.argv[2] if len(sys.argv) > 2 else "cfg2"]
A = gen.configs.build_matrix(cfg, device="cuda")
PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device="cuda")
H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=cfg.level_prec[:cfg.nlev])
b = gen.uniform_vector(A.m, cfg.seed).cuda()
x = torch.zeros(4 * ((A.m + 3) // 4), dtype=torch.float64, device="cuda")
torch.cuda.synchronize()
H.vcycle(b, x, 1)  # graph capture and first-use effects before the profiled cycles
torch.cuda.synchronize()
torch.cuda.nvtx.range_push("solve")
print("MARK-SOLVE", flush=True)
res, calls = H.vcycle(b, x, cycles)
torch.cuda.synchronize()
torch.cuda.nvtx.range_pop()
print("done", calls, res[-1] / res[0])
