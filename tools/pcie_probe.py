#!/usr/bin/env python
"""PCIe probe: bare pinned 4 GiB H2D, D2H and both concurrently (the e2e roof)."""
import torch, time
N = 1 << 30  # 4 GiB fp32
h = torch.empty(N, dtype=torch.float32).pin_memory()
h2 = torch.empty(N, dtype=torch.float32).pin_memory()
d = torch.empty(N, dtype=torch.float32, device="cuda")
d2 = torch.empty(N, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for _ in range(2):
    d.copy_(h, non_blocking=True); torch.cuda.synchronize()
def t(fn):
    torch.cuda.synchronize(); t0 = time.perf_counter(); fn(); torch.cuda.synchronize(); return time.perf_counter() - t0
a = t(lambda: d.copy_(h, non_blocking=True))
b = t(lambda: h2.copy_(d, non_blocking=True))
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
c = t(both)
print(f"H2D {4.295/a:.1f} GB/s  D2H {4.295/b:.1f} GB/s  both {2*4.295/c:.1f} GB/s total ({c*1e3:.1f} ms for 4+4 GiB)")
