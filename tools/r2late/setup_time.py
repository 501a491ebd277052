"""Config-3 (or other) hierarchy setup: wall time (CUDA events) of several setups after a warm-up,
and the per-class device timers of the last one.  usage: python tools/r2late/setup_time.py [cfg3] [reps]"""
import json, os, sys, statistics
sys.path.insert(0, os.getcwd())
import torch
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
name = sys.argv[1] if len(sys.argv) > 1 else "cfg3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
cfg = gen.configs.CONFIGS[name]
A = gen.configs.build_matrix(cfg, device="cuda")
PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device="cuda")
Ps = [P for P, _ in PR]
s = torch.cuda.current_stream()
ts = []
for rep in range(reps + 1):
    torch.cuda.synchronize()
    if rep == reps:
        amgt.timing_enable(True); amgt.timing_reset()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    M = amgt.from_csr(A)
    MPs = [amgt.from_csr(P) for P in Ps]
    H = amgt.Hierarchy(M, MPs, level_prec=cfg.level_prec[:cfg.nlev])
    e1.record(s); e1.synchronize()
    if 0 < rep < reps: ts.append(e0.elapsed_time(e1))
    H.close(); M.free()
    for P in MPs: P.free()
prof = amgt.timing_read()
amgt.timing_enable(False)
print(json.dumps({"cfg": name, "setup_ms": ts, "median": statistics.median(ts) if ts else None,
                  "classes": {k: round(v["ms"], 3) for k, v in prof.items() if isinstance(v, dict) and "ms" in v}}))
