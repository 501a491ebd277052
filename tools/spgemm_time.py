"""SpGEMM C = A*A timing on config 1 / config 4 (irregular power-law block rows): symbolic and
numeric phases with CUDA events after an L2 flush (median of reps), GFLOP/s (2 x scalar
products) and the fraction of the copy bandwidth for the algorithmic bytes of SURVEY §8(d).

usage: python tools/spgemm_time.py [cfg4|cfg1] [reps]
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json"))).get("hbm_gbs", 6460.9)
A = gen.configs.build_matrix(gen.configs.CONFIGS[name], device="cuda")
M = amgt.from_csr(A)
del A
s = torch.cuda.current_stream()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def tmed(fn):
    ts, res = [], None
    for i in range(reps + 1):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        res = fn()
        e1.record(s)
        e1.synchronize()
        if i:
            ts.append(e0.elapsed_time(e1))
    return statistics.median(ts), res


_, info = amgt.spgemm_symbolic(M, M, info=True)
t_sym, C = tmed(lambda: amgt.spgemm_symbolic(M, M))
t_num, _ = tmed(lambda: amgt.spgemm_numeric(M, M, C))
fl = 2 * info["scalar_products"]
nb = (2 * M.blc_num + C.blc_num) * (16 * 8 + 6) + (2 * M.blc_row + C.blc_row + 3) * 8
out = {"cfg": name, "tiles_A": M.blc_num, "tiles_C": C.blc_num, "bins": info["bin_rows"], "sym_ms": t_sym,
       "num_ms": t_num, "flops": fl, "gflops": fl / ((t_sym + t_num) * 1e-3) / 1e9,
       "num_gflops": fl / (t_num * 1e-3) / 1e9, "bytes": nb,
       "frac": nb / ((t_sym + t_num) * 1e-3) / 1e9 / peak, "num_frac": nb / (t_num * 1e-3) / 1e9 / peak}
print(json.dumps(out))
