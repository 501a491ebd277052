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
        "27pt_128": lambda: gen.laplacian_27pt(128, device="cuda"),
        "cfg4_2^18": lambda: gen.irregular_block_sparse(1 << 18).to("cuda")}
if len(sys.argv) > 2 and sys.argv[2] == "spmv":
    SPGEMM = False
else:
    SPGEMM = True
for name, mk in mats.items():
    A = mk()
    M = amgt.from_csr(A).analyze()
    x = gen.uniform_vector(A.n, 1).cuda()
    y = torch.empty(4 * M.blc_row, dtype=torch.float64, device="cuda")
    r = {}
    st = M.spmv_stats()
    r["avg_nnz_blc"] = round(st["avg_nnz_blc"], 3)
    for thr in (17, 10, 0):
        amgt.set_tc_threshold(17, thr)
        r[f"spmv_f64_thr{thr}_us"] = med(lambda: amgt.spmv(M, x, y), True)
    M16 = M.cast("f16").analyze() if name != "cfg4_2^18" else None  # cfg4 values fit FP16 too
    if M16 is None:
        M16 = M.cast("f16").analyze()
    x32 = x.float()
    y32 = torch.empty(4 * M.blc_row, dtype=torch.float32, device="cuda")
    for thr in (17, 10, 0):
        amgt.set_tc_threshold(17, thr)
        r[f"spmv_f16_thr{thr}_us"] = med(lambda: amgt.spmv(M16, x32, y32), True)
    tb = M.blc_num * (16 * 8 + 6) + (M.blc_row + 1) * 8 + 8 * 4 * (M.blc_col + M.blc_row)
    r["spmv_f64_bytes"] = tb
    r["spmv_f16_bytes"] = M.blc_num * (16 * 2 + 6) + (M.blc_row + 1) * 8 + 4 * 4 * (M.blc_col + M.blc_row)
    amgt.set_tc_threshold(17, 17)
    if not SPGEMM:
        out[name] = r
        continue
    C = amgt.spgemm_symbolic(M, M)
    for prec in ("f64", "f16"):
        Mp = M if prec == "f64" else M.cast("f16") if name != "cfg4_2^18" else None
        if Mp is None:
            continue
        Cp = C if prec == "f64" else amgt.spgemm_symbolic(Mp, Mp)
        for thr in (17, 10, 0):
            amgt.set_tc_threshold(thr, 17)
            r[f"spgemm_{prec}_thr{thr}_us"] = med(lambda: amgt.spgemm_numeric(Mp, Mp, Cp), False)
    out[name] = r
amgt.set_tc_threshold(17, 17)
print(json.dumps(out))
