#!/usr/bin/env python
"""Development sweep: time every variant on the configs (device-resident
inputs, CUDA events, warm-up 3, median of N).  Not the contract bench; see
bench.py.  Usage: python tools/sweep.py [prefix|tri|transpose|all] [--reps N]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

L2 = torch.empty(256 * 2 ** 20 // 4, dtype=torch.int32, device="cuda")


def t_ms(fn, reps=20, flush=False):
    for _ in range(3):
        fn()
    times = []
    for _ in range(reps):
        if flush:
            L2.fill_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        times.append(a.elapsed_time(b))
    return statistics.median(times)


def prefix(reps):
    out = []
    for (n, p, dt) in [(1024, 2 ** 20, torch.float32), (32, 2 ** 22, torch.float32), (32, 1024, torch.int32),
                       (32768, 2 ** 13, torch.float32), (1024, 2 ** 14, torch.float32)]:
        for layout, variants in ((bo.ROW_WISE, [bo.PS_FUSED_ROW, bo.PS_WARPSCAN, bo.PS_TRANSPOSED, bo.PS_NAIVE]),
                                 (bo.COLUMN_WISE, [bo.PS_ACROSS, bo.PS_NAIVE])):
            x = bo.generate_prefix(n, p, 2, dt, layout)
            y = torch.empty_like(x)
            ws = torch.empty(n * p * 4, dtype=torch.uint8, device="cuda")
            for v in variants:
                ms = t_ms(lambda: bo.prefix_sums(x, layout, v, out=y, workspace=ws), reps, flush=n * p * 4 < 2 ** 28)
                gbs = 2 * n * p * 4 / ms / 1e6
                out.append(dict(algo="prefix", n=n, p=p, layout=layout, variant=bo.VARIANT_NAMES[v], ms=ms,
                                gbs=gbs, inst_s=p / ms * 1e3))
                print(json.dumps(out[-1]), flush=True)
            del x, y, ws
    return out


def tri(reps):
    out = []
    for (n, p, dt) in [(16, 65536, torch.int32), (64, 65536, torch.float32), (64, 65536, torch.int32),
                       (8, 2 ** 22, torch.int32), (32, 65536, torch.float32)]:
        for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
            c = bo.generate_tri(n, p, 4, dt, layout)
            o = torch.empty(p, dtype=dt, device="cuda")
            vs = [bo.TRI_SMEM_WARP, bo.TRI_TILED, bo.TRI_TILED_HALF]
            if n <= 18:
                vs = [bo.TRI_THREAD_REG] + vs
            if n <= 16 or (n == 64 and layout == bo.COLUMN_WISE):
                vs.append(bo.TRI_UMM_GLOBAL)
            for v in vs:
                need = bo.triangulation_workspace(n, p, 0, layout, v)
                ws = torch.empty(max(need, 1), dtype=torch.uint8, device="cuda")
                try:
                    ms = t_ms(lambda: bo.triangulation(c, layout, v, out=o, workspace=ws), reps,
                              flush=n * n * p * 4 < 2 ** 28)
                except bo.BulkError as e:
                    print("skip", n, v, e)
                    continue
                ops = n * (n - 1) * (n - 2) // 6 * p
                out.append(dict(algo="tri", n=n, p=p, dtype=str(dt), layout=layout, variant=bo.VARIANT_NAMES[v],
                                ms=ms, inst_s=p / ms * 1e3, taddmin=ops / ms / 1e9))
                print(json.dumps(out[-1]), flush=True)
                del ws
            del c
    return out


def transpose(reps):
    out = []
    for rows, cols in [(2 ** 20, 1024), (1024, 2 ** 20), (2 ** 16, 4096), (2 ** 22, 32)]:
        x = torch.empty((rows, cols), dtype=torch.int32, device="cuda")
        y = torch.empty((cols, rows), dtype=torch.int32, device="cuda")
        ms = t_ms(lambda: bo.transpose(x, out=y), reps)
        out.append(dict(algo="transpose", rows=rows, cols=cols, ms=ms, gbs=2 * rows * cols * 4 / ms / 1e6))
        print(json.dumps(out[-1]), flush=True)
    return out


if __name__ == "__main__":
    what = sys.argv[1] if len(sys.argv) > 1 else "all"
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 20
    res = []
    if what in ("prefix", "all"):
        res += prefix(reps)
    if what in ("tri", "all"):
        res += tri(reps)
    if what in ("transpose", "all"):
        res += transpose(reps)
