"""Level-1 Galerkin RAP timing (SURVEY §8(a) a3-a7, §8(d) roofline): A_c = R*(A*P) on the
config-2 (7-point 128^3) or config-3 (27-point 256^3) operator with the 2x2x2 aggregation P,
every SpGEMM phase timed separately with CUDA events after an L2 flush (median of reps).

usage: python tools/rap_bench.py [cfg2|cfg3] [reps] [--out file.json]
Prints one JSON object: per-phase ms, GFLOP/s (2 x scalar products), algorithmic bytes
((T_A + T_B + T_C)(16s + 6) + pointers, §8(d)) and the fraction of the copy bandwidth.
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

out_path = None
argv = sys.argv[1:]
if "--out" in argv:
    k = argv.index("--out")
    out_path = argv[k + 1]
    argv = argv[:k] + argv[k + 2:]
cfg = argv[0] if argv else "cfg2"
reps = int(argv[1]) if len(argv) > 1 else 5
peaks = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))
bw = float(peaks.get("hbm_gbs", 0)) or None
bw = bw or 6460.9

if cfg == "cfg2":
    N = 128
    Acsr = gen.laplacian_7pt(N, device="cuda")
else:
    N = 256
    Acsr = gen.laplacian_27pt(N, device="cuda")
Pcsr = gen.aggregation_P((N, N, N), 0.5, device="cuda")
A = amgt.from_csr(Acsr)
P = amgt.from_csr(Pcsr)
R = P.transpose()
del Acsr, Pcsr
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


def sbytes(X, Y, C, s_):
    return (X.blc_num + Y.blc_num + C.blc_num) * (16 * s_ + 6) + (X.blc_row + Y.blc_row + C.blc_row + 3) * 8


out = {"cfg": cfg, "reps": reps, "peak_gbs": bw}
APs, info1 = amgt.spgemm_symbolic(A, P, info=True)
t_sym1, AP = tmed(lambda: amgt.spgemm_symbolic(A, P))
t_num1, _ = tmed(lambda: amgt.spgemm_numeric(A, P, AP))
Acs, info2 = amgt.spgemm_symbolic(R, AP, info=True)
t_sym2, Ac = tmed(lambda: amgt.spgemm_symbolic(R, AP))
t_num2, _ = tmed(lambda: amgt.spgemm_numeric(R, AP, Ac))
t_rap, _ = tmed(lambda: amgt.rap(R, A, P))
fl1, fl2 = 2 * info1["scalar_products"], 2 * info2["scalar_products"]
b1, b2 = sbytes(A, P, AP, 8), sbytes(R, AP, Ac, 8)
sb1 = (A.blc_num + P.blc_num) * 12 + AP.blc_num * 6
sb2 = (R.blc_num + AP.blc_num) * 12 + Ac.blc_num * 6
out.update({
    "tiles": {"A": A.blc_num, "P": P.blc_num, "AP": AP.blc_num, "Ac": Ac.blc_num},
    "ap": {"sym_ms": t_sym1, "num_ms": t_num1, "flops": fl1, "num_bytes": b1,
           "num_gbs": b1 / t_num1 / 1e6, "num_frac": b1 / t_num1 / 1e6 / bw, "sym_struct_bytes": sb1},
    "rap2": {"sym_ms": t_sym2, "num_ms": t_num2, "flops": fl2, "num_bytes": b2,
             "num_gbs": b2 / t_num2 / 1e6, "num_frac": b2 / t_num2 / 1e6 / bw, "sym_struct_bytes": sb2},
    "rap_ms": t_rap, "rap_gflops": (fl1 + fl2) / t_rap / 1e6,
    "rap_bytes": b1 + b2, "rap_roofline_ms": (b1 + b2) / bw / 1e6,
    "rap_frac": (b1 + b2) / bw / 1e6 / t_rap,
})
print(json.dumps(out))
if out_path:
    with open(out_path, "w") as f:
        json.dump(out, f, indent=1)
