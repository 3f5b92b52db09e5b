#!/usr/bin/env python3
"""Top SASS instructions by warp-stall samples from an `ncu -i rep --page source
--csv --print-source sass` dump.  Usage: sass_hot.py dump.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
idx = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
S = idx["Warp Stall Sampling (All Samples)"]
tot = sum(float(r[S] or 0) for r in data)
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
top = sorted(data, key=lambda r: -float(r[S] or 0))[: int(sys.argv[2]) if len(sys.argv) > 2 else 30]
print(f"total samples {tot:.0f}")
for r in top:
    v = float(r[S] or 0)
    st = sorted(((float(r[idx[h]] or 0), h) for h in stalls), reverse=True)[:2]
    print(f"{v / tot * 100:5.1f}%  {r[idx['Address']]:>6}  {r[idx['Source']][:60]:60s}  " +
          " ".join(f"{h[6:]}={x:.0f}" for x, h in st if x > 0))
