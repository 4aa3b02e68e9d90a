#!/usr/bin/env python
"""Development timer for the tiled triangulation kernels: TR-2 shapes in every
layout and dtype, CUDA events, L2 flushed, median of N, plus an oracle check
of 64 sampled instances per config.  Usage: python tools/tri_time.py [--reps N]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bulkgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

L2 = torch.empty(256 * 2 ** 20 // 4, dtype=torch.int32, device="cuda")


def t_ms(fn, reps):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        L2.fill_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 20
    small = [(16, 65536, "int32", bo.ROW_WISE, bo.AUTO), (16, 65536, "int32", bo.COLUMN_WISE, bo.AUTO),
             (16, 65536, "int32", bo.PACKED_ROW, bo.AUTO), (16, 65536, "float32", bo.ROW_WISE, bo.AUTO),
             (12, 65536, "int32", bo.ROW_WISE, bo.AUTO), (16, 1 << 20, "int32", bo.ROW_WISE, bo.AUTO)]
    if "--cmp" in sys.argv:     # --cmp n,dtype,layout,v1/v2/...  (variant numbers)
        n_, dt_, lay_, vs_ = sys.argv[sys.argv.index("--cmp") + 1].split(",")
        small = [(int(n_), 65536, dt_, int(lay_), int(v)) for v in vs_.split("/")]
    cfgs = small if ("--small" in sys.argv or "--cmp" in sys.argv) else [(64, 65536, "float32", bo.ROW_WISE, bo.AUTO), (64, 65536, "int32", bo.ROW_WISE, bo.AUTO),
            (64, 65536, "float32", bo.COLUMN_WISE, bo.AUTO), (64, 65536, "float32", bo.PACKED_ROW, bo.AUTO),
            (64, 65536, "float32", bo.ROW_WISE, bo.TRI_TILED), (40, 65536, "float32", bo.ROW_WISE, bo.AUTO),
            (33, 65536, "int32", bo.ROW_WISE, bo.AUTO), (64, 65536, "float32", bo.ROW_WISE, "chords")]
    for n, p, dt, layout, v in cfgs:
        ids = np.unique(np.linspace(0, p - 1, 64).astype(np.int64))
        c = bo.generate_tri(n, p, 4, getattr(torch, dt), layout)
        if v == "chords":
            fn = lambda: bo.triangulation_chords(c, layout)
            val, ch = fn()
        else:
            out = torch.empty(p, dtype=c.dtype, device="cuda")
            fn = lambda: bo.triangulation(c, layout, v, out=out)
            val = fn()
        ms = t_ms(fn, reps)
        ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 4, dt), oracle.ROW_WISE)
        got = val.cpu().numpy()[ids]
        ok = bool(np.array_equal(got.view(np.uint32), ref.view(np.uint32)))
        if v == "chords":
            _, rc = oracle.bulk_opt_chords(bulkgen.tri_instances(n, ids[:8], 4, dt), oracle.ROW_WISE)
            ok = ok and bool(np.array_equal(ch.cpu().numpy()[ids[:8]], rc))
        adds = (n - 2) * (n - 1) * n // 6
        print(json.dumps(dict(n=n, p=p, dtype=dt, layout=layout, variant=v if v == "chords" else bo.VARIANT_NAMES[
            bo.triangulation_variant(n, p, bo.F32 if dt == "float32" else bo.I32, layout, v)],
            ms=round(ms, 4), tadd_min_s=round(adds * p / ms / 1e9, 3), ok=ok)), flush=True)


if __name__ == "__main__":
    main()
