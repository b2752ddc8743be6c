#!/usr/bin/env python
"""Per-CUDA-source-line instruction counts / stall samples from
`ncu -i rep --page source --csv --print-source cuda,sass`.  Usage: cuda_lines.py csv [norm] [top]"""
import csv
import sys

path = sys.argv[1]
norm = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 50
fname = "?"
out = []
tot = 0
for r in csv.reader(open(path)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] in ("Function Name", "Line No") or r[0] == "":
        continue
    try:
        n = int(r[7] or 0)
        s = int(r[4] or 0)
    except (ValueError, IndexError):
        continue
    tot += n
    out.append((n, s, f"{fname}:{r[0]}", r[1][:80]))
print(f"total {tot} ({tot / norm:.1f} per unit)")
for n, s, loc, src in sorted(out, reverse=True)[:top]:
    print(f"{n / norm:8.1f} {s:7d} {loc:22s} {src}")
