#!/usr/bin/env python
"""Top SASS lines by one stall reason from `ncu --page source --csv --print-source sass`.
Usage: stall_lines.py csv [reason=stall_long_sb] [top=25]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
reason = sys.argv[2] if len(sys.argv) > 2 else "stall_long_sb"
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
lines = []
for n, r in enumerate(rows[2:]):
    if len(r) < len(hdr):
        continue
    lines.append((int(r[ix[reason]] or 0), n, r[ix["Address"]][-5:], r[ix["Source"]].strip()[:80]))
tot = sum(l[0] for l in lines)
print(f"{reason}: total {tot}")
for s, n, a, src in sorted(lines, reverse=True)[:top]:
    print(f"{100 * s / max(tot, 1):5.1f}% #{n:5d} {a} {src}")
