#!/usr/bin/env python
"""Host-side cost of one binding call (ctypes + argument checks + C-side launch):
us per call for triangulation (both layouts) and prefix sums, then a cProfile of
the prefix-sum call.  python tools/hostprof.py"""
import cProfile
import os
import pstats
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
    ct = bo.generate_tri(16, 65536, 3, torch.int32, layout)
    ot = torch.empty(65536, dtype=torch.int32, device="cuda")
    for _ in range(10):
        bo.triangulation(ct, layout, out=ot)
    torch.cuda.synchronize()
    torch.cuda._sleep(int(0.2 * 2e9))
    t0 = time.perf_counter()
    for _ in range(200):
        bo.triangulation(ct, layout, out=ot)
    print(f"triangulation layout {layout}: host {(time.perf_counter() - t0) / 200 * 1e6:.2f} us/call")
    torch.cuda.synchronize()
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
# the same call recorded once as a CUDA graph (bo.Captured): host time per replay of 8 calls
ys = [torch.empty_like(x) for _ in range(8)]
cap = bo.Captured(lambda s: [bo.prefix_sums(x, 0, out=yy, stream=s) for yy in ys])
torch.cuda.synchronize()
torch.cuda._sleep(int(0.2 * 2e9))
t = time.perf_counter()
for _ in range(200):
    cap.replay()
dt = (time.perf_counter() - t) / 200
print(f"Captured replay of 8 prefix_sums calls: host {dt*1e6:.2f} us/replay ({dt*1e6/8:.2f} us per call)")
torch.cuda.synchronize()
torch.cuda.synchronize()
pr = cProfile.Profile(); pr.enable(); loop(); pr.disable()
pstats.Stats(pr).sort_stats("tottime").print_stats(12)
# device time per call inside the replayed graph (events around 200 replays)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda._sleep(int(0.05 * 2e9))
e0.record()
for _ in range(200):
    cap.replay()
e1.record()
torch.cuda.synchronize()
print(f"Captured replay: device {e0.elapsed_time(e1) * 1e3 / 200 / 8:.2f} us per prefix_sums call (n=32 p=1024 int32)")
