#!/usr/bin/env python
"""Per-CUDA-source-line stall attribution from an ncu report:
  ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > X.csv
  python tools/ncu_lines.py X.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1], errors="replace")))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
hdr, fname, out = None, "?", []
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r or not r[0].isdigit():
        continue
    d = dict(zip(hdr[4:], r[4:]))
    def f(k):
        try:
            return float(d.get(k, "0").replace(",", ""))
        except ValueError:
            return 0.0
    reasons = {k[6:]: f(k) for k in hdr if k.startswith("stall_") and "Not Issued" not in k}
    out.append((f("Warp Stall Sampling (All Samples)"), f("Instructions Executed"), fname, r[0], r[1].strip()[:70],
                reasons, f("L1 Wavefronts Shared")))
tot = sum(o[0] for o in out) or 1
tot_i = sum(o[1] for o in out) or 1
tot_w = sum(o[6] for o in out) or 1
print(f"samples {tot:.0f}  instructions {tot_i:.4g}  smem wavefronts {tot_w:.4g}")
for s, i, fn, ln, src, rs, w in sorted(out, key=lambda o: -o[0])[:top]:
    rtop = ", ".join(f"{k} {v / max(s, 1) * 100:.0f}%" for k, v in sorted(rs.items(), key=lambda kv: -kv[1])[:3] if v)
    print(f"{s / tot * 100:5.1f}% samp {i / tot_i * 100:5.1f}% inst {w / tot_w * 100:5.1f}% wf  {fn}:{ln}  {src}  [{rtop}]")
