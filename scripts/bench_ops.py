#!/usr/bin/env python
"""Per-entry timing of every C-ABI entry on one workload (GPU box), for DESIGN.md / profiles.

    python scripts/bench_ops.py [--workload c2] [--reps 10]

Prints one JSON line per entry: CUDA-event time per call (median of 3 batches of `reps`
back-to-back calls, after 3 warm-ups),
det-samples/s, and for the HBM-bound entries the algorithmic bytes and the fraction of the
measured copy bandwidth (MEASURED_PEAKS.json)."""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_demeurekktbb23_b200 import binding, synth  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload  # noqa: E402


def timed(fn, reps):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    # `reps` calls back to back between two events: the host-side marshalling of call i+1
    # overlaps kernel i, so the time is the device time per call (median of 3 batches)
    ts = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(reps):
            fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / reps)
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--only", default="", help="comma-separated substrings of entry names to time")
    args = ap.parse_args()
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        pass
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    w = synth.make_workload(args.workload)
    dw = DeviceWorkload.upload(w, "cuda")
    nds = w.det_samples
    n_det, n_samp, ivs = w.n_det, w.n_samp, w.intervals
    dev = "cuda"
    only = [x for x in args.only.split(",") if x]
    fused_only = bool(only) and all("fused" in o or "pointing_to_" in o for o in only)
    # unfused intermediates (32 + 8 + 24 B per det-sample) only when an unfused entry is timed
    shp = (1, 1) if fused_only else (n_det, n_samp)
    quats = torch.zeros((*shp, 4), dtype=torch.float64, device=dev)
    pix = torch.zeros(shp, dtype=torch.int64, device=dev)
    wts = torch.zeros((*shp, 3), dtype=torch.float64, device=dev)
    tod2 = dw.det_data.clone()
    rng = np.random.default_rng(0)
    m = torch.from_numpy(rng.normal(size=(w.n_submap, w.n_pix_submap, 3))).to(dev)
    out = []


    def timed_if(name, fn):
        return timed(fn, args.reps) if not only or any(o in name for o in only) else None

    def rep(name, ms, bytes_per=None):
        if ms is None:
            return
        d = {"workload": args.workload, "entry": name, "ms": ms, "det_samples_per_s": nds / (ms / 1e3)}
        if "pointing_to_map" in name:
            d["staging"] = binding.last_fused_path()
        if bytes_per is not None:
            gbs = bytes_per * nds / (ms / 1e3) / 1e9
            d.update(alg_bytes_per_det_sample=bytes_per, achieved_gbs=gbs, hbm_frac=gbs / hbm)
        out.append(d)
        print(json.dumps(d), flush=True)

    sf = dict(shared_flags=dw.shared_flags, shared_flag_mask=w.shared_flag_mask)
    # the unfused chain's intermediates, computed once untimed so any --only subset sees real data
    if not fused_only:
        binding.pointing_detector(dw.fp_quats, dw.boresight, ivs, quats, **sf)
        binding.pixels_healpix(quats, ivs, w.nside, w.nest, w.n_pix_submap, pix, **sf)
        binding.stokes_weights_iqu(quats, ivs, dw.epsilon, w.cal, wts, hwp=dw.hwp)
    rep("pointing_to_map (fused A1-A4)", timed_if("pointing_to_map (fused A1-A4)", lambda: dw.pointing_to_map()))
    rep("pointing_to_tod (fused A1-A3+A5)", timed_if("pointing_to_tod (fused A1-A3+A5)", lambda: binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, ivs, w.nside, w.nest, 3,
                                              dw.global2local, w.n_pix_submap, m, tod2, hwp=dw.hwp, **sf)), 16)
    rep("pointing_detector (A1)", timed_if("pointing_detector (A1)", lambda: binding.pointing_detector(dw.fp_quats, dw.boresight, ivs, quats, **sf)),
        32 + 32.0 / n_det)
    rep("pixels_healpix (A2)", timed_if("pixels_healpix (A2)", lambda: binding.pixels_healpix(quats, ivs, w.nside, w.nest, w.n_pix_submap, pix, **sf)),
        32 + 8)
    rep("stokes_weights_iqu (A3)", timed_if("stokes_weights_iqu (A3)", lambda: binding.stokes_weights_iqu(quats, ivs, dw.epsilon, w.cal, wts, hwp=dw.hwp)),
        32 + 24)
    zg = torch.zeros_like(dw.zmap)
    rep("build_noise_weighted (A4)", timed_if("build_noise_weighted (A4)", lambda: binding.build_noise_weighted(zg, dw.global2local, w.n_pix_submap, pix, wts, dw.det_data,
                                                   dw.det_scale, ivs, det_flags=dw.det_flags,
                                                   det_flag_mask=w.det_flag_mask, **sf)),
        8 + 24 + 8 + (1 if w.det_flags is not None else 0))
    rep("scan_map (A5)", timed_if("scan_map (A5)", lambda: binding.scan_map(m, dw.global2local, w.n_pix_submap, pix, wts, tod2, ivs)),
        8 + 24 + 16)
    step = 100
    amp_off = torch.arange(n_det, dtype=torch.int64, device=dev) * sum(
        (l - f + 1 + step - 1) // step for f, l in ivs)
    amps = torch.zeros(int(amp_off[-1].item()) + sum((l - f + 1 + step - 1) // step for f, l in ivs),
                       dtype=torch.float64, device=dev)
    rep("template_offset_add_to_signal (f2)", timed_if("template_offset_add_to_signal (f2)", lambda: binding.template_offset_add_to_signal(step, amp_off, amps, tod2, ivs)), 16)
    rep("template_offset_project_signal (f2)", timed_if("template_offset_project_signal (f2)", lambda: binding.template_offset_project_signal(step, amp_off, amps, dw.det_data, ivs,
                                                             det_flags=dw.det_flags,
                                                             det_flag_mask=w.det_flag_mask)),
        8 + (1 if w.det_flags is not None else 0))
    rep("noise_weight (f4)", timed_if("noise_weight (f4)", lambda: binding.noise_weight(tod2, dw.det_scale, ivs)), 16)
    rep("stokes_weights_i (f4)", timed_if("stokes_weights_i (f4)", lambda: binding.stokes_weights_i(pix.view(torch.float64), 1.0, ivs)), 8)


if __name__ == "__main__":
    main()
