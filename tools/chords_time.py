#!/usr/bin/env python
"""Time bulk_triangulation_chords (TR-2 shape) back to back, CUDA events.
python tools/chords_time.py [n] [p] [K]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 64
p = int(sys.argv[2]) if len(sys.argv) > 2 else 65536
K = int(sys.argv[3]) if len(sys.argv) > 3 else 20
c = bo.generate_tri(n, p, 4, torch.float32, bo.ROW_WISE)
out = torch.empty(p, dtype=torch.float32, device="cuda")
ch = torch.empty((p, n - 3, 2), dtype=torch.int16, device="cuda")
for _ in range(3):
    bo.triangulation_chords(c, bo.ROW_WISE, out=out, chords=ch)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda._sleep(40_000_000)
a.record()
for _ in range(K):
    bo.triangulation_chords(c, bo.ROW_WISE, out=out, chords=ch)
b.record()
torch.cuda.synchronize()
print(f"chords n={n} p={p}: {a.elapsed_time(b) / K:.4f} ms")
