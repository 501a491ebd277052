import sys, time, torch
sys.path.insert(0, "/root/repo")
import bench, gen
import paper_conf_sc_luzwflcy0c024_b200 as amgt
cfg = gen.configs.CONFIGS["cfg2"]
A, Ps, b, PR, N = bench.make_inputs(cfg, "cuda")
x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
hA = type(A)(A.m, A.n, A.row_ptr.cpu().pin_memory(), A.col.cpu().pin_memory(), A.val.cpu().pin_memory())
hPs = [type(P)(P.m, P.n, P.row_ptr.cpu().pin_memory(), P.col.cpu().pin_memory(), P.val.cpu().pin_memory()) for P in Ps]
hb = b.cpu().pin_memory()
def to_dev(t):
    d = torch.empty(t.shape, dtype=t.dtype, device="cuda"); d.copy_(t, non_blocking=True); return d
for i in range(6):
    torch.cuda.synchronize(); t0 = time.time()
    dA = type(A)(A.m, A.n, to_dev(hA.row_ptr), to_dev(hA.col), to_dev(hA.val))
    dPs = [type(P)(P.m, P.n, to_dev(P.row_ptr), to_dev(P.col), to_dev(P.val)) for P in hPs]
    db = to_dev(hb)
    torch.cuda.synchronize(); t1 = time.time()
    bench.gpu_step(amgt, dA, dPs, db, x, 50, torch)
    torch.cuda.synchronize(); t2 = time.time()
    bench.gpu_step(amgt, A, Ps, b, x, 50, torch)
    torch.cuda.synchronize(); t3 = time.time()
    print(f"h2d {1e3*(t1-t0):.1f} ms  step(copied) {1e3*(t2-t1):.1f} ms  step(resident) {1e3*(t3-t2):.1f} ms")
