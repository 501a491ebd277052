"""Break the bench step (cfg2) into conversion / hierarchy setup / V-cycles, device events
and host wall time side by side (host-bound phases show wall >> device)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

cfg = gen.configs.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "cfg2"]
A, Ps, b, PR, N = bench.make_inputs(cfg, "cuda")
x = torch.zeros(4 * ((A.m + 3) // 4), dtype=torch.float64, device="cuda")
s = torch.cuda.current_stream()
rows = []
for it in range(6):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    torch.cuda.synchronize()
    t = [time.perf_counter()]
    ev[0].record(s)
    MA = amgt.from_csr(A)
    MPs = [amgt.from_csr(P) for P in Ps]
    ev[1].record(s)
    t.append(time.perf_counter())
    H = amgt.Hierarchy(MA, MPs, level_prec=bench.LEVEL_PREC[:len(Ps) + 1])
    ev[2].record(s)
    t.append(time.perf_counter())
    x.zero_()
    res, calls = H.vcycle(b, x, 50)
    ev[3].record(s)
    t.append(time.perf_counter())
    torch.cuda.synchronize()
    t.append(time.perf_counter())
    H.close()
    MA.free()
    for M in MPs:
        M.free()
    dev = [ev[i].elapsed_time(ev[i + 1]) for i in range(3)]
    wall = [(t[i + 1] - t[i]) * 1e3 for i in range(3)]
    rows.append((dev, wall, (t[4] - t[0]) * 1e3, ev[0].elapsed_time(ev[3])))
for dev, wall, tot, dtot in rows[2:]:
    print("convert dev %.2f wall %.2f | setup dev %.2f wall %.2f | vcycle dev %.2f wall %.2f | total dev %.2f wall %.2f"
          % (dev[0], wall[0], dev[1], wall[1], dev[2], wall[2], dtot, tot))
