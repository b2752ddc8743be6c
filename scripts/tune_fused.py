#!/usr/bin/env python
"""Time toast_pointing_to_map for several library variants (tuning aid, GPU box).

    python scripts/tune_fused.py [--workload c2] lib1.so lib2.so ...

Each library is timed in its own subprocess (TOASTB200_LIB=...) on the same seeded
workload: 3 warm-ups, then the median of 20 CUDA-event-timed calls.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, os, sys, statistics
sys.path.insert(0, os.environ["ROOT"])
import torch
from paper_conf_sc_demeurekktbb23_b200 import binding, synth
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload
w = synth.make_workload(os.environ["WL"], **json.loads(os.environ.get("WLARGS", "{}")))
dw = DeviceWorkload.upload(w, "cuda")
raw = dw.raw_args()
lib = binding.load()
ts = []
for i in range(23):
    dw.zmap.zero_()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    rc = lib.toast_pointing_to_map(*raw)
    b.record()
    torch.cuda.synchronize()
    assert rc == 0, lib.toast_last_error()
    if i >= 3:
        ts.append(a.elapsed_time(b))
ms = statistics.median(ts)
print(json.dumps({"lib": os.environ.get("TOASTB200_LIB", "default"), "ms": ms,
                  "det_samples_per_s": w.det_samples / (ms / 1e3),
                  "zsum": float(dw.zmap.sum())}))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--wlargs", default="{}", help="JSON overrides for synth.make_workload (nside, nest, n_det, ...)")
    ap.add_argument("libs", nargs="*")
    args = ap.parse_args()
    libs = args.libs or [None]
    for lib in libs:
        env = dict(os.environ, ROOT=ROOT, WL=args.workload, WLARGS=args.wlargs)
        if lib:
            env["TOASTB200_LIB"] = os.path.abspath(lib)
        r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True)
        line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else json.dumps({"lib": lib, "error": r.stderr[-800:]})
        print(line.rstrip("}") + f', "wl": "{args.workload}", "wlargs": {args.wlargs}}}', flush=True)


if __name__ == "__main__":
    main()
