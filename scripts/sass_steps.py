#!/usr/bin/env python
"""Per-step SASS view of an ncu report: each instruction's execution count divided by the number
of 32-det-sample steps (det_samples / 32), in address order, plus totals by frequency class.
Usage: sass_steps.py report.ncu-rep det_samples [min_ratio]"""
import csv
import io
import subprocess
import sys

rep, det_samples = sys.argv[1], float(sys.argv[2])
lo = float(sys.argv[3]) if len(sys.argv) > 3 else 0.02
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
steps = det_samples / 32
tot = 0.0
acc = 0.0
lines = []
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    n = int(r[ix["Instructions Executed"]] or 0)
    tot += n / steps
    st = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    ratio = n / steps
    if ratio > lo:
        acc += ratio
        lines.append(f"{r[ix['Address']][-4:]} {ratio:6.3f} {acc:7.2f} {st:6d} {float(r[ix['Avg. Threads Executed']] or 0):5.1f} "
                     f"{r[ix['Source']].strip()[:90]}")
print(f"total warp instructions per 32 det-samples: {tot:.1f}")
print("\n".join(lines))
