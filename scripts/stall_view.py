#!/usr/bin/env python
"""Per-instruction stall view of an ncu report (source page, SASS): address, executions per
32-det-sample step, stall_wait / short_sb / long_sb / branch samples, source.
Usage: stall_view.py report.ncu-rep det_samples [min_ratio] [top]"""
import csv
import io
import subprocess
import sys

rep, det = sys.argv[1], float(sys.argv[2])
lo = float(sys.argv[3]) if len(sys.argv) > 3 else 0.3
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
steps = det / 32
tot = {k: 0 for k in ("stall_wait", "stall_short_sb", "stall_long_sb", "stall_branch_resolving", "stall_math",
                      "stall_no_inst", "stall_not_selected", "stall_selected")}
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    for k in tot:
        tot[k] += int(r[ix[k]] or 0)
print("totals:", tot)
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    n = int(r[ix["Instructions Executed"]] or 0) / steps
    if n < lo:
        continue
    w = int(r[ix["stall_wait"]] or 0)
    ss = int(r[ix["stall_short_sb"]] or 0)
    ls = int(r[ix["stall_long_sb"]] or 0)
    br = int(r[ix["stall_branch_resolving"]] or 0)
    print(f"{r[ix['Address']][-4:]} {n:5.2f} w{w:5d} ss{ss:5d} ls{ls:5d} br{br:4d}  {r[ix['Source']].strip()[:70]}")
