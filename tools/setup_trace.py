"""Single-GPU hierarchy setup of a 7-point grid, timed twice (second = warm allocator/pools);
AMGT_TRACE=1 prints the per-step host/device trace.  python tools/setup_trace.py [N] [nlev]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 512
nlev = int(sys.argv[2]) if len(sys.argv) > 2 else 7
A = gen.laplacian_7pt(N, device="cuda")
PR = gen.aggregation_hierarchy((N, N, N), nlev, device="cuda")
Ps = [P for P, _ in PR]
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    MA = amgt.from_csr(A)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    MPs = [amgt.from_csr(P) for P in Ps]
    H = amgt.Hierarchy(MA, MPs, level_prec=("f64", "f32", "f16", "f16", "f16", "f16", "f16")[:nlev])
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    print(f"rep {rep}: convert {1e3 * (t1 - t0):.1f} ms, hierarchy {1e3 * (t2 - t1):.1f} ms", flush=True)
    H.close()
    MA.free()
    for M in MPs:
        M.free()
