"""Break one partitioned (row-slab) bench step into hierarchy setup and native V-cycles, device
events and host wall time side by side (run single-rank: python tools/dist_breakdown.py)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", "29533")
os.environ.setdefault("RANK", "0")
os.environ.setdefault("WORLD_SIZE", "1")
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import bench  # noqa: E402
import gen  # noqa: E402
from paper_conf_sc_luzwflcy0c024_b200.dist import Comm, DistHierarchy, NativeComm  # noqa: E402

torch.cuda.set_device(0)
dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
comm = Comm()
cfg = gen.configs.CONFIGS["cfg2"]
dims = (cfg.N, cfg.N, cfg.N)
A, rows, n, Ps = gen.partition.slab_inputs("7pt", dims, cfg.nlev, 0, 1, alpha=cfg.alpha, device="cuda")
b = gen.uniform_vector(n, cfg.seed)[rows[0]:rows[1]].cuda()
x = torch.zeros(rows[1] - rows[0], dtype=torch.float64, device="cuda")
native = NativeComm(comm)
s = torch.cuda.current_stream()
for it in range(5):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ev[0].record(s)
    H = DistHierarchy(comm, A, rows, n, Ps, level_prec=bench.LEVEL_PREC[:cfg.nlev])
    ev[1].record(s)
    t1 = time.perf_counter()
    x.zero_()
    res, calls = H.native_vcycle(native, b, x, 50)
    ev[2].record(s)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    print("setup dev %.2f wall %.2f | vcycle dev %.2f wall %.2f" % (ev[0].elapsed_time(ev[1]), (t1 - t0) * 1e3,
                                                                   ev[1].elapsed_time(ev[2]), (t2 - t1) * 1e3))
dist.destroy_process_group()
