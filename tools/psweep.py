#!/usr/bin/env python
"""configs[4]: p-sweep 2^10..2^22 for both algorithms on one GPU (AUTO variants,
device-resident inputs, CUDA events, 3 warm-ups, median of 10, L2 flushed when
the input is smaller than 2x L2).  Each point also checks a handful of sampled
instances against the oracle (this is a dev tool; it may use oracle/).
Prints one JSON line per point.   python tools/psweep.py [--max-log2 22]"""
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

FLUSH = torch.empty(256 * 2 ** 20 // 4, dtype=torch.int32, device="cuda")


def med_ms(fn, flush, reps=10):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        if flush:
            FLUSH.fill_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    hi = int(sys.argv[sys.argv.index("--max-log2") + 1]) if "--max-log2" in sys.argv else 22
    cases = [("prefix", 32, "int32"), ("prefix", 1024, "float32"), ("tri", 16, "int32"), ("tri", 64, "float32")]
    for algo, n, dt in cases:
        for lg in range(10, hi + 1, 2):
            p = 2 ** lg
            tdt = getattr(torch, dt)
            rng = np.random.default_rng(lg)
            ids = np.unique(np.r_[rng.integers(0, p, 6), 0, p - 1])
            if algo == "prefix":
                x = bo.generate_prefix(n, p, 5, tdt, bo.ROW_WISE)
                y = torch.empty_like(x)
                ms = med_ms(lambda: bo.prefix_sums(x, bo.ROW_WISE, out=y), n * p * 4 < 2 ** 28)
                got = y[torch.from_numpy(ids).cuda()].cpu().numpy()
                ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(n, ids, 5, dt), oracle.ROW_WISE)
                bytes_ = 2 * n * p * 4
                variant = bo.VARIANT_NAMES[bo.prefix_sums_variant(n, p, bo.I32 if dt == "int32" else bo.F32, 0)]
                extra = {"GBps": bytes_ / ms / 1e6}
                del x, y
            else:
                c = bo.generate_tri(n, p, 5, tdt, bo.ROW_WISE)
                out = torch.empty(p, dtype=tdt, device="cuda")
                ms = med_ms(lambda: bo.triangulation(c, bo.ROW_WISE, out=out), n * n * p * 4 < 2 ** 28)
                got = out[torch.from_numpy(ids).cuda()].cpu().numpy()
                ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 5, dt), oracle.ROW_WISE)
                variant = bo.VARIANT_NAMES[bo.triangulation_variant(n, p, bo.I32 if dt == "int32" else bo.F32, 0)]
                extra = {"T_addmin_s": n * (n - 1) * (n - 2) // 6 * p / ms / 1e9}
                del c, out
            ok = bool(np.array_equal(np.ascontiguousarray(got).view(np.uint32), ref.view(np.uint32)))
            torch.cuda.empty_cache()
            print(json.dumps(dict(algo=algo, n=n, dtype=dt, p=p, variant=variant, ms=ms, inst_per_s=p / ms * 1e3,
                                  sampled_parity=ok, **extra)), flush=True)


if __name__ == "__main__":
    main()
