"""Fused level-1 sweeps on a bench config's A_1 (config 3: 27-point 256^3, A_1 = 14.9 GB): two
(Jacobi, Jacobi + residual norm) or three stages of amgt_spmv_sweeps against the same steps as
separate kernels; CUDA events, inputs larger than L2.  Knobs per setting: AMGT_SWEEP_IMPL
(ldg | tma), AMGT_SWEEP_CTAS, AMGT_SWEEP_LAG.

usage: python tools/sweep_cfg.py cfg3 [reps] [impl:ctas:lag,...]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "cfg3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
settings = [s.split(":") for s in (sys.argv[3] if len(sys.argv) > 3 else "ldg:4:-1,ldg:2:-1,tma:1:-1").split(",")]
cfg = gen.configs.CONFIGS[name]
A = gen.configs.build_matrix(cfg, device="cuda")
M = amgt.from_csr(A).analyze()
del A
n = 4 * M.blc_row
x = gen.uniform_vector(n, 1).cuda()
b = gen.uniform_vector(n, 2).cuda()
d = torch.full((n,), 1.0 / 26.0, dtype=torch.float64, device="cuda")
v = [torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(4)]
nrm = torch.zeros(1, dtype=torch.float64, device="cuda")
s = torch.cuda.current_stream()


def timed(fn):
    ts = []
    for i in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        if i >= 1:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    return round(ts[len(ts) // 2], 3)


def sep2():
    amgt.spmv_fused(M, x, v[0], "jacobi", b=b, dinv=d)
    amgt.spmv_jacobi_res(M, v[0], v[1], b, d, v[3])


def sep3():
    sep2()
    amgt.spmv_fused(M, v[1], v[2], "residual", b=b)


out = {"config": name, "tiles": M.blc_num, "sep2_ms": timed(sep2), "sep3_ms": timed(sep3)}
ref = v[1].clone(), v[2].clone()
for impl, ctas, lag in settings:
    os.environ["AMGT_SWEEP_IMPL"] = impl
    os.environ["AMGT_SWEEP_CTAS"] = ctas
    if int(lag) >= 0:
        os.environ["AMGT_SWEEP_LAG"] = lag
    else:
        os.environ.pop("AMGT_SWEEP_LAG", None)
    plan = amgt.SweepPlan(M)
    st = [("jacobi", x, v[0]), ("jacobi_res", v[0], v[1]), ("residual", v[1], v[2])]
    k = f"{impl}_c{ctas}_l{lag}"
    out[k + "_2st_ms"] = timed(lambda: plan.run(st[:2], b, d, norm=nrm))
    same2 = bool(torch.equal(v[1], ref[0]))
    out[k + "_3st_ms"] = timed(lambda: plan.run(st, b, d, norm=nrm))
    out[k + "_bitexact"] = same2 and bool(torch.equal(v[2], ref[1]))
    out[k + "_maxrel"] = float(((v[2] - ref[1]).abs().max() / ref[1].abs().max()).item())
    plan.close()
    print(json.dumps(out), flush=True)
