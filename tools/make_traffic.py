#!/usr/bin/env python
"""profiles/traffic.json (bench.py's roofline.traffic) from the per-capture
traffic.json that tools/ncu_summarize.py writes: workload -> DRAM bytes per
launch of its dominant kernel.

    python tools/make_traffic.py profiles/r01/traffic.json r01
"""
import json
import os
import sys

# bench workload -> capture name in tools/gpu_profile.sh
MAP = {"ps2": "ps2_fused", "ps2col": "ps2_across", "tr2": "tr2_tiled", "tr1": "tr1_reg", "tr_transpose": "transpose",
       "tr1col": "tr1col_reg", "tr2col": "tr2col_tiled", "tr2chords": "chords", "ps32k": "ps32k_row",
       "ps32k_col": "ps32k_col", "exec_bitonic_col": "exec_bitonic_col", "exec_prefix_col": "exec_prefix_col",
       "exec_prefix_row": "exec_prefix_row",
       "exec_bitonic_col_jit": "exec_bitonic_col_jit", "exec_bitonic_row_jit": "exec_bitonic_row_jit",
       "exec_prefix_col_jit": "exec_prefix_col_jit", "tr2packed": "tr2prow_tiled"}


def main():
    src, rnd = sys.argv[1], sys.argv[2]
    caps = json.load(open(src))
    out = {}
    for wl, cap in MAP.items():
        if cap in caps:
            d = dict(caps[cap])
            d["capture"] = f"profiles/{rnd}/ncu_summary.md ({cap})"
            d["round"] = rnd
            out[wl] = d
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    with open(os.path.join(root, "profiles", "traffic.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps({k: v["dram_bytes_per_launch"] for k, v in out.items()}))


if __name__ == "__main__":
    main()
