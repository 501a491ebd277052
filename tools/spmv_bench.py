"""SpMV microbenchmark on config 2's level-1 operator (FP64 7-point 128^3): plain SpMV with
L2 flushed between launches (cold), back-to-back (warm), and the fused Jacobi epilogue.
CUDA events on the launching stream; prints one JSON line.  The kernel variant comes from
the AMGT_SPMV_VARIANT environment variable (read once by libamgt).

usage: AMGT_SPMV_VARIANT=v python tools/spmv_bench.py [N] [reps]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 128
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
A = gen.laplacian_7pt(N, device="cuda")
M = amgt.from_csr(A).analyze()
n = A.m
x = gen.uniform_vector(n, 1).cuda()
b = gen.uniform_vector(n, 2).cuda()
d = torch.full((n,), 1.0 / 6.0, dtype=torch.float64, device="cuda")
y = torch.empty(n, dtype=torch.float64, device="cuda")
flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
bytes_spmv = M.blc_num * (16 * 8 + 6) + (M.blc_row + 1) * 8 + 8 * 4 * M.blc_col + 8 * 4 * M.blc_row
s = torch.cuda.current_stream()


def timed(fn, cold):
    ts = []
    for i in range(reps + 3):
        if cold:
            flush.fill_(float(i))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        if i >= 3:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


plain = lambda: amgt.spmv(M, x, y)
jac = lambda: amgt.spmv_fused(M, x, y, "jacobi", b=b, dinv=d)
out = {"variant": os.environ.get("AMGT_SPMV_VARIANT", "0"), "N": N, "bytes": bytes_spmv}
for name, fn, cold, by in (("plain_cold", plain, True, bytes_spmv), ("plain_warm", plain, False, bytes_spmv),
                           ("jacobi_cold", jac, True, bytes_spmv + 16 * n), ("jacobi_warm", jac, False, bytes_spmv + 16 * n)):
    ms = timed(fn, cold)
    out[name] = {"us": round(ms * 1e3, 2), "GBps": round(by / (ms * 1e-3) / 1e9, 1)}
print(json.dumps(out))
