#!/usr/bin/env python
"""Back-to-back timing of small triangulation / prefix configs the way bench.py
does it (inputs rotate over enough copies to exceed 2x L2, CUDA events around K
steps).  python tools/small_time.py tri|prefix n p dtype layout variant [K]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

algo, n, p, dt, layout, variant = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), getattr(torch, sys.argv[4]), \
    int(sys.argv[5]), int(sys.argv[6])
K = int(sys.argv[7]) if len(sys.argv) > 7 else 50
L2 = 126 * 2 ** 20
if algo == "tri":
    x = bo.generate_tri(n, p, 3, dt, layout)
    out = torch.empty(p, dtype=dt, device="cuda")
else:
    x = bo.generate_prefix(n, p, 1, dt, layout, "uniform")
    out = torch.empty_like(x)
copies = max(1, -(-2 * L2 // (x.numel() * 4)) + 1)
xs = [x] + [x.clone() for _ in range(copies - 1)]
ref = None


def step(i):
    if algo == "tri":
        return bo.triangulation(xs[i % copies], layout, variant, out=out)
    return bo.prefix_sums(xs[i % copies], layout, variant, out=out)


ref = step(0).clone()
for i in range(5):
    step(i)
torch.cuda.synchronize()
torch.cuda._sleep(int(0.02 * 2e9))
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for i in range(K):
    step(i)
b.record()
torch.cuda.synchronize()
print(f"{algo} n={n} p={p} {sys.argv[4]} layout={layout} variant={variant}: {a.elapsed_time(b) / K * 1e3:.2f} us/step "
      f"({copies} copies), same result: {bool(torch.equal(out.view(torch.int32), ref.view(torch.int32)))}")
