#!/usr/bin/env python
"""Development A/B timer: time bench.py workloads exactly as bench.py does
(rotating input copies, spin kernel ahead of the events, K steps back to back)
for the library BULKOBL_LIB points at.  One JSON line per workload.
    BULKOBL_LIB=ab/NAME/libbulkobl.so python tools/abtime.py ps2col tr2 prefix:1024:16384:float32:0 [--steps 20] [--reps 3]
(ad-hoc executor specs: exec_prefix:n:p:dtype:layout, exec_bitonic:n:p:dtype:layout)"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    steps = int(sys.argv[sys.argv.index("--steps") + 1]) if "--steps" in sys.argv else 20
    reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 3
    args = [a for a in args if not a.isdigit()]
    ctx = bench.Ctx()
    stream = torch.cuda.Stream()
    lib = os.environ.get("BULKOBL_LIB", "in-tree")
    for name in args:
        if ":" in name:          # ad-hoc spec algo:n:p:dtype:layout[:variant], e.g. prefix:1024:16384:float32:0
            f = name.split(":")
            wl = dict(seed=5, algo=f[0], n=int(f[1]), p=int(f[2]), dtype=f[3], layout=int(f[4]),
                      variant=int(f[5]) if len(f) > 5 else 0, desc=name)
            if f[0].startswith("exec_"):              # exec_prefix:... / exec_bitonic:...
                wl.update(algo="exec", prog=f[0][5:])
        else:
            wl = bench.WORKLOADS[name]
        st = bench.setup_workload(wl, 0, bench.copies_for(wl))
        ms = min(bench.timed(ctx, st["fn"], steps, 3, stream)[0] for _ in range(reps))
        print(json.dumps({"lib": lib, "workload": name, "variant": st["variant"], "ms": round(ms, 5),
                          "minst_per_s": round(wl["p"] / ms / 1e3, 2)}), flush=True)
        del st
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
