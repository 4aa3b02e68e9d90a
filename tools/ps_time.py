#!/usr/bin/env python
"""Development timer for the prefix-sum kernels (CUDA events, inputs > L2 or
flushed, median of N) with an oracle check on sampled instances.
Usage: python tools/ps_time.py [--reps N]"""
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


def t_ms(fn, reps, flush):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        if flush:
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
    cfgs = [(1024, 1 << 20, "float32", bo.COLUMN_WISE), (1024, 1 << 20, "int32", bo.COLUMN_WISE),
            (32, 1 << 22, "int32", bo.COLUMN_WISE), (1024, 1 << 16, "float32", bo.COLUMN_WISE),
            (1000, (1 << 20) + 4, "float32", bo.COLUMN_WISE), (1024, 1 << 20, "float32", bo.ROW_WISE)]
    for n, p, dt, layout in cfgs:
        x = bo.generate_prefix(n, p, 2, getattr(torch, dt), layout)
        y = torch.empty_like(x)
        fn = lambda: bo.prefix_sums(x, layout, out=y)
        ms = t_ms(fn, reps, flush=n * p * 4 < 2 * 126 * 2 ** 20)
        fn()
        ids = np.unique(np.linspace(0, p - 1, 24).astype(np.int64))
        ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(n, ids, 2, dt), oracle.ROW_WISE)
        t = torch.from_numpy(ids).cuda()
        got = (y[t] if layout == bo.ROW_WISE else y[:, t].T).contiguous().cpu().numpy()
        ok = bool(np.array_equal(got.view(np.uint32), ref.view(np.uint32)))
        v = bo.VARIANT_NAMES[bo.prefix_sums_variant(n, p, bo.F32 if dt == "float32" else bo.I32, layout)]
        print(json.dumps(dict(n=n, p=p, dtype=dt, layout=layout, variant=v, ms=round(ms, 4),
                              tbs=round(2 * n * p * 4 / ms / 1e9, 3), ok=ok)), flush=True)


if __name__ == "__main__":
    main()
