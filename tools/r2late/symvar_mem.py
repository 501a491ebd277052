"""sym_var after the process has filled device memory (the bench's config-3 state): is the
config-4 symbolic time sensitive to allocator state?"""
import sys, os, time, torch
sys.path.insert(0, os.getcwd())
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
hog_gb = float(sys.argv[1]) if len(sys.argv) > 1 else 0
hogs = [torch.empty(1 << 30, dtype=torch.uint8, device="cuda") for _ in range(int(hog_gb))]
A = gen.configs.build_matrix(gen.configs.CONFIGS["cfg4"], device="cuda")
M = amgt.from_csr(A); del A
s = torch.cuda.current_stream()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for i in range(8):
    flush.zero_()
    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    t0 = time.perf_counter()
    e0.record(s); C = amgt.spgemm_symbolic(M, M); e1.record(s)
    t1 = time.perf_counter()
    amgt.spgemm_numeric(M, M, C); e2.record(s); e2.synchronize()
    print(f"hog {hog_gb} rep {i}: sym {e0.elapsed_time(e1):.3f} ms (host {1e3*(t1-t0):.3f}) num {e1.elapsed_time(e2):.3f} ms", flush=True)
    C.free()
