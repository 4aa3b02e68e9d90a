#!/usr/bin/env python
"""Run one op a few times (for ncu).
    python tools/prof_one.py prefix|tri|transpose|exec_prefix|exec_bitonic n p dtype layout variant [reps]
(exec_*: variant 1 = compiled program)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

algo, n, p, dt, layout, variant = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), sys.argv[4], int(sys.argv[5]), int(sys.argv[6])
reps = int(sys.argv[7]) if len(sys.argv) > 7 else 3
dt = getattr(torch, dt)
if algo == "prefix":
    x = bo.generate_prefix(n, p, 2, dt, layout)
    y = torch.empty_like(x)
    need = bo.prefix_sums_workspace(n, p, 0, layout, variant)
    ws = torch.empty(max(need, 1), dtype=torch.uint8, device="cuda")
    for _ in range(reps):
        bo.prefix_sums(x, layout, variant, out=y, workspace=ws)
elif algo == "tri":
    c = bo.generate_tri(n, p, 4, dt, layout)
    o = torch.empty(p, dtype=dt, device="cuda")
    need = bo.triangulation_workspace(n, p, 0, layout, variant)
    ws = torch.empty(max(need, 1), dtype=torch.uint8, device="cuda")
    for _ in range(reps):
        bo.triangulation(c, layout, variant, out=o, workspace=ws)
elif algo.startswith("exec_"):
    from paper_conf_ipps_tanitni14_b200 import programs
    P = programs.prefix_sums(n, sys.argv[4]) if algo == "exec_prefix" else programs.bitonic_sort(n)
    x = bo.generate_prefix(n, p, 2, dt, layout)
    if variant == 1:                       # variant 1: the compiled program (bulk_program_compile)
        P = bo.prepare(P, n)
        assert P.compile(dt, layout)
    for _ in range(reps):
        bo.execute(P, x, layout)
else:
    x = torch.empty((p, n), dtype=dt, device="cuda")
    for _ in range(reps):
        bo.transpose(x)
torch.cuda.synchronize()
print("done")
