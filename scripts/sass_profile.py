#!/usr/bin/env python
"""Summarise an ncu --page source --print-source sass CSV: executed instructions per opcode
and the hottest stall locations.  Usage: sass_profile.py file.csv [top]"""
import collections
import csv
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
rows = list(csv.reader(open(path)))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
ops = collections.Counter()
stall = []
total = 0
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    src = r[ix["Source"]].strip()
    n = int(r[ix["Instructions Executed"]] or 0)
    s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    ops[op.split(".")[0]] += n
    total += n
    stall.append((s, r[ix["Address"]][-5:], src[:70], n))
print(f"total warp instructions executed: {total}")
for op, n in ops.most_common(top):
    print(f"{op:12s} {n:12d} {100*n/total:5.1f}%")
print("--- top stall locations")
tot_s = sum(s for s, *_ in stall)
for s, a, src, n in sorted(stall, reverse=True)[:top]:
    print(f"{100*s/max(tot_s,1):5.1f}% {a} {src:70s} {n}")
