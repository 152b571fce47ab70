"""Pinned host buffer H2D rate per allocation (diagnosing bimodal e2e times)."""
import time
import torch

def h2d_rate(h, d, n=20):
    d.copy_(h, non_blocking=True); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n):
        d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    return h.numel() * n / (time.perf_counter() - t0) / 1e9

d = torch.empty(5 << 20, dtype=torch.uint8, device="cuda")
for i in range(8):
    h = torch.empty(5 << 20, dtype=torch.uint8).pin_memory()
    print("alloc", i, "GB/s %.1f" % h2d_rate(h, d), "ptr %x" % h.data_ptr(), flush=True)
    del h
hs = [torch.empty(5 << 20, dtype=torch.uint8).pin_memory() for _ in range(6)]
for i, h in enumerate(hs):
    print("live", i, "GB/s %.1f" % h2d_rate(h, d), "ptr %x" % h.data_ptr(), flush=True)
big = torch.empty(64 << 20, dtype=torch.uint8).pin_memory()
print("64MB GB/s %.1f" % h2d_rate(big, torch.empty(64 << 20, dtype=torch.uint8, device='cuda'), 5))
