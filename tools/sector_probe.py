"""Level-1 FP64 SpMV with / without sector skipping (AMGT_SPMV_VARIANT=4: a lane skips the 16-B
value half whose bitmap bits are clear) and under an L2 fetch granularity (AMGT_L2_FETCH).
Plain y = A x, CUDA events, inputs larger than L2 (config 3) or L2 flushed (config 2).
Prints one JSON line: ms per launch, full-tile bytes and sector bytes (32-B sectors holding a set bit).

usage: AMGT_SPMV_VARIANT=4 AMGT_L2_FETCH=32 python tools/sector_probe.py cfg3 [reps]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "cfg3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
cfg = gen.configs.CONFIGS[name]
A = gen.configs.build_matrix(cfg, device="cuda")
M = amgt.from_csr(A)
del A
mp = M.map_u16().to(torch.int32) & 0xFFFF
rows_nz = sum(((mp >> (4 * r)) & 0xF) != 0 for r in range(4)).to(torch.int64)
sectors = int(rows_nz.sum())  # FP64: one 32-B sector per tile row
T, BR, BC = M.blc_num, M.blc_row, M.blc_col
vec = (BR + 1) * 8 + 4 * BC * 8 + 4 * BR * 8
full = T * (16 * 8 + 6) + vec
sect = T * 6 + sectors * 32 + vec
x = gen.uniform_vector(4 * BC, 1).cuda()
y = torch.empty(4 * BR, dtype=torch.float64, device="cuda")
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
s = torch.cuda.current_stream()
for _ in range(3):
    amgt.spmv(M, x, y)
torch.cuda.synchronize()
ts = []
for _ in range(reps):
    flush.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    amgt.spmv(M, x, y)
    e1.record(s)
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
ts.sort()
ms = ts[len(ts) // 2]
print(json.dumps({"config": name, "variant": os.environ.get("AMGT_SPMV_VARIANT", "0"),
                  "l2_fetch": os.environ.get("AMGT_L2_FETCH", "default"), "ms": round(ms, 4), "tiles": T,
                  "sectors": sectors, "full_bytes": full, "sector_bytes": sect,
                  "gbs_full": round(full / ms / 1e6, 1), "gbs_sector": round(sect / ms / 1e6, 1),
                  "ysum": float(y.sum())}))
