#!/usr/bin/env python
"""Instruction count (and local-memory ops) per kernel / device function in a .so's SASS.
Usage: sass_sizes.py lib.so [substring]"""
import re
import subprocess
import sys

out = subprocess.run(["cuobjdump", "-sass", sys.argv[1]], capture_output=True, text=True).stdout
pat = sys.argv[2] if len(sys.argv) > 2 else ""
name, n, ll = None, 0, 0
rows = []
for line in out.splitlines():
    m = re.match(r"\s+Function : (\S+)", line)
    if m:
        if name:
            rows.append((name, n, ll))
        name, n, ll = m.group(1), 0, 0
        continue
    if re.match(r"\s+/\*[0-9a-f]{4}\*/", line):
        n += 1
        if re.search(r"\b(STL|LDL)\b", line):
            ll += 1
if name:
    rows.append((name, n, ll))
for name, n, ll in rows:
    if pat in name:
        t = re.search(r"kernelIL(.*?)EEEv", name)
        print(f"{n:6d} instr {ll:3d} local  {('p2m ' + t.group(1)) if t else name[:100]}")
