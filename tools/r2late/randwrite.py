"""Micro-benchmark: 128-B rows scattered to random positions (the record pass's store pattern) vs a
contiguous copy of the same bytes (torch kernels; CUDA events, median of 5)."""
import torch, statistics
N = 16_000_000
src = torch.randn(N, 16, dtype=torch.float64, device="cuda")
dst = torch.empty_like(src)
perm = torch.randperm(N, device="cuda")
blk = torch.randperm(N // 1024, device="cuda")
perm_blk = (blk[:, None] * 1024 + torch.arange(1024, device="cuda")[None, :]).reshape(-1)
def t(fn):
    ts = []
    for i in range(6):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); e1.synchronize()
        if i: ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)
by = N * 128 * 2
for name, fn in [("copy", lambda: dst.copy_(src)), ("scatter_random", lambda: dst.index_copy_(0, perm, src)),
                 ("scatter_1024run", lambda: dst.index_copy_(0, perm_blk, src)), ("gather_random", lambda: torch.index_select(src, 0, perm, out=dst))]:
    ms = t(fn); print(f"{name:18s} {ms:.3f} ms  {by / ms / 1e6:.0f} GB/s (read+write bytes)")
