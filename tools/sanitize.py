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
# the CTA-cooperative column-wise preload over several batches per CTA (+ a per-warp tail batch)
for layout in (bo.COLUMN_WISE, bo.PACKED_COLUMN):
    for n, p, v in ((16, 7112, bo.TRI_TILED_HALF), (24, 7112, bo.TRI_TILED_QUARTER)):
        bo.triangulation(bo.generate_tri(n, p, 1, torch.float32, layout), layout, v)
c = bo.generate_tri(80, 3, 1, torch.float32, bo.ROW_WISE)
bo.triangulation(c, bo.ROW_WISE, bo.TRI_TILED_GLOBAL)
bo.triangulation(c, bo.ROW_WISE, bo.TRI_TILED_GLOBAL8)
for layout in (bo.COLUMN_WISE, bo.PACKED_ROW):
    bo.triangulation(bo.generate_tri(37, 5, 1, torch.int32, layout), layout, bo.TRI_TILED_GLOBAL8)
from paper_conf_ipps_tanitni14_b200 import programs  # noqa: E402
for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
    m = bo.generate_prefix(16, 70, 1, torch.float32, layout)
    bo.execute(programs.bitonic_sort(16), m, layout)                     # staged in shared memory
    bo.execute(programs.prefix_sums(300, "float32"), bo.generate_prefix(300, 130, 2, torch.float32, layout),
               layout)                                                    # direct (msize too large to stage)
# a program that reads registers before writing them (the kernel zeroes its register file)
import numpy as np  # noqa: E402
bo.execute(np.array([[2, 0, 1, 2], [1, 0, 0, 0]], dtype=np.int32), torch.zeros((64, 4), dtype=torch.int32,
                                                                                 device="cuda"), bo.ROW_WISE)
# graph capture: the queue kernels stride statically, eager launches on another stream beside it
xg = bo.generate_prefix(1024, 40000, 3, torch.float32, bo.ROW_WISE)
og = torch.empty_like(xg)
sc = torch.cuda.Stream()
with torch.cuda.stream(sc):
    bo.prefix_sums(xg, bo.ROW_WISE, out=og, stream=sc)
sc.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=sc):
    bo.prefix_sums(xg, bo.ROW_WISE, out=og, stream=sc)
g.replay()
bo.prefix_sums(xg, bo.ROW_WISE)
x = torch.zeros((300, 260), dtype=torch.int32, device="cuda")
bo.transpose(x)
torch.cuda.synchronize()
print("sanitize run complete")
