#!/usr/bin/env python
"""Summarise an `ncu --page source --print-source sass --csv` dump: top
instructions by executed count and by stall samples, stall-reason totals."""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
def f(x):
    try:
        return float(x.replace(",", ""))
    except Exception:
        return 0.0
tot_exec = sum(f(d["Instructions Executed"]) for d in data)
tot_samp = sum(f(d["Warp Stall Sampling (All Samples)"]) for d in data)
print(f"instructions executed {tot_exec:.4g}, stall samples {tot_samp:.4g}")
op = Counter()
for d in data:
    o = d["Source"].split()[0] if d["Source"].split() else "?"
    if o.startswith("@"):
        o = d["Source"].split()[1]
    op[o.split(".")[0]] += f(d["Instructions Executed"])
print("by opcode:", ", ".join(f"{k}:{v/tot_exec*100:.1f}%" for k, v in op.most_common(18)))
stalls = Counter()
for d in data:
    for k in hdr:
        if k.startswith("stall_") and "Not Issued" not in k:
            stalls[k] += f(d[k])
print("stalls:", ", ".join(f"{k[6:]}:{v/tot_samp*100:.1f}%" for k, v in stalls.most_common(10)))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
print("\ntop by samples:")
for d in sorted(data, key=lambda d: -f(d["Warp Stall Sampling (All Samples)"]))[:n]:
    print(f'{d["Address"]:>6} {f(d["Warp Stall Sampling (All Samples)"]):8.0f} {f(d["Instructions Executed"]):12.0f}  {d["Source"][:90]}')
