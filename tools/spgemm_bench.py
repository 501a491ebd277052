"""Numeric SpGEMM timing vs the tensor-core threshold (CUDA events, median of reps).

usage: python tools/spgemm_bench.py [which] [reps]
  which: ap7   (7-point 128^3 A * P, FP64 and FP16)
         aa27  (27-point 64^3 A * A: dense tiles, FP64 and FP16)
         irr   (irregular 2^16 block rows A * A)
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "ap7"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
if which == "ap7":
    X, Y = gen.laplacian_7pt(128, device="cuda"), gen.aggregation_P((128, 128, 128), 0.5, device="cuda")
elif which == "aa27":
    X = Y = gen.laplacian_27pt(64, device="cuda")
else:
    X = Y = gen.irregular_block_sparse(1 << 16).to("cuda")
s = torch.cuda.current_stream()
out = {"case": which}
for prec in ("f64", "f16"):
    MX, MY = amgt.from_csr(X, prec=prec), amgt.from_csr(Y, prec=prec)
    C, info = amgt.spgemm_symbolic(MX, MY, info=True)
    for thr in (10, 17, 0):
        amgt.set_tc_threshold(thr, 17)
        ts = []
        for i in range(reps + 2):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            amgt.spgemm_numeric(MX, MY, C)
            e1.record(s)
            e1.synchronize()
            if i >= 2:
                ts.append(e0.elapsed_time(e1))
        ts.sort()
        out[f"{prec}_thr{thr}_us"] = round(ts[len(ts) // 2] * 1e3, 1)
    out[f"{prec}_pairs"] = info["pairs_nonzero"]
    out[f"{prec}_tc_pairs_at10"] = info["pairs_tc"]
amgt.set_tc_threshold(17, 17)
print(json.dumps(out))
