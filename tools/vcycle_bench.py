"""Solve-phase timing: config-2 (or config-3) hierarchy, amgt_vcycle with 50 cycles timed with
CUDA events (median of reps), printed as ms per cycle.  Launch-mode knobs are read from the
environment by the library (AMGT_COARSE, AMGT_PDL, AMGT_TAIL_BLOCKROWS, ...), so variants are
compared by running this tool once per setting.

usage: python tools/vcycle_bench.py [cfg2|cfg3] [cycles] [reps]
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "cfg2"
cycles = int(sys.argv[2]) if len(sys.argv) > 2 else 50
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
cfg = gen.configs.CONFIGS[name]
A = gen.configs.build_matrix(cfg, device="cuda")
PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device="cuda")
H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=cfg.level_prec[:cfg.nlev])
del PR
b = gen.uniform_vector(A.m, cfg.seed).cuda()
x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
s = torch.cuda.current_stream()
H.vcycle(b, x, 3)
ts = []
for _ in range(reps):
    x.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    res, calls = H.vcycle(b, x, cycles)
    e1.record(s)
    e1.synchronize()
    ts.append(e0.elapsed_time(e1))
env = {k: v for k, v in os.environ.items() if k.startswith("AMGT_")}
print(json.dumps({"cfg": name, "env": env, "cycles": cycles, "ms": statistics.median(ts),
                  "us_per_cycle": 1000 * statistics.median(ts) / cycles, "calls": calls,
                  "rel_res": res[-1] / res[0]}))
H.close()
