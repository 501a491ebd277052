"""Tensor-core route vs CUDA-core route on B200 (the default-threshold decision, DESIGN §4 R9/R10).
SpMV (L2 flushed between launches) and numeric SpGEMM at thresholds 17 (no tile), 10 (paper),
0 (every tile); median of reps, CUDA events.  Prints one JSON object."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def med(fn, cold):
    ts = []
    for i in range(reps + 2):
        if cold:
            flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return round(ts[len(ts) // 2], 1)


out = {}
mats = {"cfg2_7pt_128": lambda: gen.laplacian_7pt(128, device="cuda"),
        "27pt_64": lambda: gen.laplacian_27pt(64, device="cuda"),
        "cfg4_small_2^16": lambda: gen.irregular_block_sparse(1 << 16).to("cuda")}
for name, mk in mats.items():
    A = mk()
    M = amgt.from_csr(A).analyze()
    x = gen.uniform_vector(A.n, 1).cuda()
    y = torch.empty(4 * M.blc_row, dtype=torch.float64, device="cuda")
    r = {}
    for thr in (17, 10, 0):
        amgt.set_tc_threshold(17, thr)
        r[f"spmv_thr{thr}_us"] = med(lambda: amgt.spmv(M, x, y), True)
    C = amgt.spgemm_symbolic(M, M)
    for prec in ("f64", "f16"):
        Mp = M if prec == "f64" else M.cast("f16") if name != "cfg4_small_2^16" else None
        if Mp is None:
            continue
        Cp = C if prec == "f64" else amgt.spgemm_symbolic(Mp, Mp)
        for thr in (17, 10, 0):
            amgt.set_tc_threshold(thr, 17)
            r[f"spgemm_{prec}_thr{thr}_us"] = med(lambda: amgt.spgemm_numeric(Mp, Mp, Cp), False)
    out[name] = r
amgt.set_tc_threshold(17, 17)
print(json.dumps(out))
