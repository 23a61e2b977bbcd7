#!/usr/bin/env python
"""Top SASS lines by warp-stall samples from `ncu -i X --page source --csv --print-source sass`.

usage: python scripts/sass_hot.py file.csv [top]
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top_n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
kernels = []
for i, r in enumerate(rows):
    if r and r[0] == "Kernel Name":
        kernels.append((r[1], i))
for kname, start in kernels[:1]:
    hdr = rows[start + 1]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    data = []
    for r in rows[start + 2:]:
        if r and r[0] == "Kernel Name":
            break
        try:
            data.append((float(r[si] or 0), r))
        except (ValueError, IndexError):
            pass
    tot = sum(x for x, _ in data) or 1
    print(kname, "samples", tot)
    for x, r in sorted(data, key=lambda t: -t[0])[:top_n]:
        print(f"{x:8.0f} {100 * x / tot:5.1f}%  {r[0]}  {r[1][:90]}")
