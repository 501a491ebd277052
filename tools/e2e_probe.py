import os, sys, time
sys.path.insert(0, "/root/repo")
import torch, bench, gen
import paper_conf_sc_luzwflcy0c024_b200 as amgt
cfg = gen.configs.CONFIGS["cfg2"]
A, Ps, b, PR, N = bench.make_inputs(cfg, "cuda")
x = torch.zeros(4 * ((A.m + 3) // 4), dtype=torch.float64, device="cuda")
host_in = [A.row_ptr, A.col, A.val] + [t for P in Ps for t in (P.row_ptr, P.col, P.val)] + [b]
host_in = [t.cpu().pin_memory() for t in host_in]
dev_in = [torch.empty(t.shape, dtype=t.dtype, device="cuda") for t in host_in]
s = torch.cuda.current_stream()
cs = torch.cuda.Stream()
def tm(fn, n=5):
    torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s); t0=time.perf_counter()
    for _ in range(n): fn()
    e1.record(s); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n, (time.perf_counter()-t0)*1e3/n
def upload():
    for d, h in zip(dev_in, host_in): d.copy_(h, non_blocking=True)
print("upload only (ms dev, wall):", tm(upload))
print("bytes", sum(t.numel()*t.element_size() for t in host_in)/1e6, "MB")
def step(): bench.gpu_step(amgt, A, Ps, b, x, 50, torch)
for _ in range(3): step()
print("step only:", tm(step))
def step_up():
    with torch.cuda.stream(cs): upload()
    step()
    torch.cuda.current_stream().wait_stream(cs)
print("step + concurrent upload:", tm(step_up))
