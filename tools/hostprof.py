#!/usr/bin/env python
"""Host-side cost of one binding call (ctypes + argument checks + C-side launch), cProfile."""
import time, torch, sys, cProfile, pstats
sys.path.insert(0, '.')
import paper_conf_ipps_tanitni14_b200 as bo
c = bo.generate_tri(16, 65536, 3, torch.int32, 1)
out = torch.empty(65536, dtype=torch.int32, device="cuda")
x = bo.generate_prefix(32, 1024, 1, torch.int32, 0)
y = torch.empty_like(x)
for _ in range(10): bo.triangulation(c, 1, 0, out=out); bo.prefix_sums(x, 0, out=y)
torch.cuda.synchronize()
def loop():
    for _ in range(500):
        bo.prefix_sums(x, 0, out=y)
t = time.perf_counter(); loop(); dt = (time.perf_counter() - t) / 500
print(f"prefix_sums host {dt*1e6:.2f} us/call")
torch.cuda.synchronize()
pr = cProfile.Profile(); pr.enable(); loop(); pr.disable()
pstats.Stats(pr).sort_stats("tottime").print_stats(12)
