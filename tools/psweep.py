#!/usr/bin/env python
"""configs[4]: p-sweep 2^10..2^22 for both algorithms on one GPU (AUTO variants,
device-resident inputs, timed like bench.py: inputs smaller than 2x L2 rotate
over copies that together exceed it, 20 steps back to back between two events).  Each point also checks a handful of sampled
instances against the oracle (this is a dev tool; it may use oracle/).
Prints one JSON line per point.   python tools/psweep.py [--max-log2 22]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bulkgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_tanitni14_b200 as bo  # noqa: E402

L2 = 126 * 2 ** 20


def rot_ms(step, in_bytes, steps=20):
    """Per-step ms the way bench.py times it: the step rotates over enough
    input copies to exceed 2x L2 (step(i) uses copy i mod copies) and K steps
    run back to back between two events."""
    for i in range(3):
        step(i)
    torch.cuda.synchronize()
    torch.cuda._sleep(int(0.01 * 2e9))
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for i in range(steps):
        step(i)
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / steps


def copies(in_bytes):
    return 1 if in_bytes >= 2 * L2 else -(-2 * L2 // in_bytes) + 1


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
                xs = [x] + [x.clone() for _ in range(copies(n * p * 4) - 1)]
                ms = rot_ms(lambda i: bo.prefix_sums(xs[i % len(xs)], bo.ROW_WISE, out=y), n * p * 4)
                got = y[torch.from_numpy(ids).cuda()].cpu().numpy()
                ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(n, ids, 5, dt), oracle.ROW_WISE)
                bytes_ = 2 * n * p * 4
                variant = bo.VARIANT_NAMES[bo.prefix_sums_variant(n, p, bo.I32 if dt == "int32" else bo.F32, 0)]
                extra = {"GBps": bytes_ / ms / 1e6}
                del x, y, xs
            else:
                c = bo.generate_tri(n, p, 5, tdt, bo.ROW_WISE)
                out = torch.empty(p, dtype=tdt, device="cuda")
                cs = [c] + [c.clone() for _ in range(copies(n * n * p * 4) - 1)]
                ms = rot_ms(lambda i: bo.triangulation(cs[i % len(cs)], bo.ROW_WISE, out=out), n * n * p * 4)
                got = out[torch.from_numpy(ids).cuda()].cpu().numpy()
                ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 5, dt), oracle.ROW_WISE)
                variant = bo.VARIANT_NAMES[bo.triangulation_variant(n, p, bo.I32 if dt == "int32" else bo.F32, 0)]
                extra = {"T_addmin_s": n * (n - 1) * (n - 2) // 6 * p / ms / 1e9}
                del c, out, cs
            ok = bool(np.array_equal(np.ascontiguousarray(got).view(np.uint32), ref.view(np.uint32)))
            torch.cuda.empty_cache()
            print(json.dumps(dict(algo=algo, n=n, dtype=dt, p=p, variant=variant, ms=ms, inst_per_s=p / ms * 1e3,
                                  sampled_parity=ok, **extra)), flush=True)


if __name__ == "__main__":
    main()
