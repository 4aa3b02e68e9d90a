#!/usr/bin/env python
"""Small inputs through every kernel, for compute-sanitizer (memcheck /
racecheck / synccheck).  Run: compute-sanitizer --tool racecheck python tools/sanitize.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
    for n, p in ((64, 300), (33, 129), (1024, 260), (300, 100)):   # (300, 100) column-wise: the 32-wide TMA ring
        x = bo.generate_prefix(n, p, 1, torch.float32, layout)
        vs = [bo.AUTO, bo.PS_NAIVE] + ([bo.PS_FUSED_ROW, bo.PS_WARPSCAN, bo.PS_TRANSPOSED] if layout == 0 else
                                       [bo.PS_ACROSS])
        for v in vs:
            bo.prefix_sums(x, layout, v)
    for n, p in ((16, 70), (24, 40), (64, 40)):
        c = bo.generate_tri(n, p, 1, torch.float32, layout)
        for v in (bo.AUTO, bo.TRI_SMEM_WARP, bo.TRI_TILED, bo.TRI_TILED_HALF, bo.TRI_TILED_QUARTER, bo.TRI_UMM_GLOBAL) + \
                ((bo.TRI_THREAD_REG,) if n <= 18 else ()):
            bo.triangulation(c, layout, v)
        bo.triangulation_chords(c, layout)
for layout in (bo.PACKED_ROW, bo.PACKED_COLUMN):
    for n, p in ((16, 70), (40, 40), (64, 40)):
        c = bo.generate_tri(n, p, 1, torch.float32, layout)
        bo.triangulation(c, layout)
        bo.triangulation_chords(c, layout)
c = bo.generate_tri(80, 3, 1, torch.float32, bo.ROW_WISE)
bo.triangulation(c, bo.ROW_WISE, bo.TRI_TILED_GLOBAL)
bo.triangulation(c, bo.ROW_WISE, bo.TRI_TILED_GLOBAL8)
for layout in (bo.COLUMN_WISE, bo.PACKED_ROW):
    bo.triangulation(bo.generate_tri(37, 5, 1, torch.int32, layout), layout, bo.TRI_TILED_GLOBAL8)
from paper_conf_ipps_tanitni14_b200 import programs  # noqa: E402
for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
    m = bo.generate_prefix(16, 70, 1, torch.float32, layout)
    bo.execute(programs.bitonic_sort(16), m, layout)
x = torch.zeros((300, 260), dtype=torch.int32, device="cuda")
bo.transpose(x)
torch.cuda.synchronize()
print("sanitize run complete")
