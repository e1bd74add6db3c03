#!/usr/bin/env python
"""Device->host copy bandwidth into pinned memory (the e2e leg's ceiling)."""
import torch, time
for mb in (134, 1024):
    d = torch.empty(mb * 2**20 // 8, dtype=torch.int64, device="cuda")
    h = torch.empty_like(d, device="cpu").pin_memory()
    for _ in range(2): h.copy_(d, non_blocking=True); torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(10): h.copy_(d, non_blocking=True)
    torch.cuda.synchronize(); dt = time.perf_counter() - t
    print(f"D2H {mb} MB pinned: {10 * mb * 2**20 / dt / 1e9:.1f} GB/s")
s2 = torch.cuda.Stream()
d = torch.empty(134 * 2**20 // 8, dtype=torch.int64, device="cuda")
hs = [torch.empty_like(d, device="cpu").pin_memory() for _ in range(2)]
torch.cuda.synchronize()
t = time.perf_counter()
for i in range(10):
    with torch.cuda.stream(s2 if i % 2 else torch.cuda.current_stream()):
        hs[i % 2].copy_(d, non_blocking=True)
torch.cuda.synchronize(); dt = time.perf_counter() - t
print(f"D2H 134 MB x 10 on two streams: {10 * 134 * 2**20 / dt / 1e9:.1f} GB/s")
