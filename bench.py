#!/usr/bin/env python
"""Benchmark of the fused pointing->map hot path (BASELINE.json metric) on N B200s.

Default workload: C4, "large satellite: 2048 detectors x 3.2M samples (1 day @ 37 Hz), nside
2048, sharded over 8 GPUs with map allreduce" — the largest BASELINE.json config that fits one
GPU (52 GB of TOD).  One step = zero the map + toast_pointing_to_map over the whole observation
(all of SURVEY 8(a) A1-A4 in one kernel) + (N > 1) the map reduction.

N > 1 (torchrun, one rank per GPU, NCCL): C4 is sharded by DETECTOR BLOCKS (rank r
takes detectors [r 2048/N, (r+1) 2048/N)), the total work is fixed ("scaling": "strong"), and
the partial maps are summed by one packed all-reduce over the union of hit submaps.  C5m (18
observations) is sharded by LPT over (observation, 256-detector block) units.  The small
configs run one observation per rank (weak scaling).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c4] [--impl ours|reference]

Workloads: c1..c5 (BASELINE.json configs; one observation), c3rt (C3's "IQU + scan_map round
trip": f1 pointing_to_tod of a smooth map, then A6), c5m (C5 "medium-shaped": 18 observations x
2048 detectors x 133200 samples, scan_map + build_noise_weighted per observation).  Inputs are
HBM-resident (C4 / C5 TOD generated on the device by the seeded counter hash, bit-identical to
synth.py) and larger than L2; no flush.  Prints ONE JSON line on rank 0.  `--impl reference`
times the CPU oracle (OpenMP timing mode) on a bounded sample of the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "detector-samples/sec pointing→map (fused) at 1/2/4/8 B200; % of HBM/fp64 roofline"
UNIT = "det-samples/s"

# Algorithmic fp64 work per det-sample (FMA = 2 flops): quaternion
# product 28, dir 13, orient 10, bx/by 13, cos/sin 2psi 15, HWP rotation 6, eta*cal 2,
# HEALPix ~10 + atan2 30 + 1/3 sqrt 6, noise weighting 4  ->  ~133.
F_ALG = 133.0
SMS = 148
DFMA_PER_SM_PER_CLK = 64  # B200 fp64 pipe, nominal (the measured peak is preferred, see fp64_peak)

WORKLOAD_DESC = {
    "c1": "tiny satellite scan: 4 dets x 100k samples, nside 64 RING, IQU, no HWP",
    "c2": "small ground scan: 64 dets x 1M samples, nside 256 NESTED, HWP + flags",
    "c3": "medium ground scan: 1024 dets x 60k samples, nside 1024, IQU",
    "c3rt": "medium ground scan: 1024 dets x 60k samples, nside 1024, IQU + scan_map round trip "
            "(pointing_to_tod of a smooth map, then pointing_to_map)",
    "c4": "large satellite: 2048 dets x 3.2M samples (1 day @ 37 Hz), nside 2048 NESTED, map allreduce",
    "c5": "TOAST-benchmark-shaped observation: 2048 dets x 133200 samples, 60 intervals, nside 4096 NESTED",
    "c5m": "TOAST-benchmark-shaped medium workflow: 18 observations x 2048 dets x 133200 samples (4.9e9 "
           "det-samples), nside 4096 NESTED, scan_map + build_noise_weighted per observation",
}
DEVICE_TOD = {"c4", "c5", "c5m"}  # TOD generated in HBM (toast_synth_tod)
C5M_OBS = 18


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="c4", choices=sorted(WORKLOAD_DESC))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--soak", type=float, default=1.0, help="seconds of untimed steps before timing (clocks)")
    ap.add_argument("--shard", default="auto", choices=["auto", "det", "obs"],
                    help="N>1: detector blocks of one observation (strong scaling; auto for c4, c5m) or one "
                         "observation per rank (weak scaling; auto for the small configs)")
    ap.add_argument("--graph", type=int, default=0,
                    help="launch-bound configs (C1, SURVEY 8(d)): one step = a CUDA graph of G back-to-back "
                         "(zero map + fused call)s, captured once and replayed")
    ap.add_argument("--reduce", default="auto", choices=["auto", "dense", "packed", "scatter", "nvls"],
                    help="N>1 map reduction: dense all_reduce, all_reduce of the union of hit submaps (packed), "
                         "or the sparse distributed map domain (compact map + reduce_scatter, SURVEY 8(f) f3)")
    return ap.parse_args()


# ----------------------------------------------------------------------------- clocks

class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled every 100 ms (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = None

    def start(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        q = ("timestamp,index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except (FileNotFoundError, OSError):
            self.proc = None
            return
        # nvidia-smi can take a second to print its first sample: the timed region starts after it
        t0 = time.time()
        while time.time() - t0 < 5.0 and os.path.getsize(self.path) == 0:
            time.sleep(0.05)

    def stop(self):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self, t_start: float, t_end: float):
        if self.proc is None or not self.path:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        rows = []
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 10:
                continue
            try:
                ts = time.mktime(time.strptime(parts[0].split(".")[0], "%Y/%m/%d %H:%M:%S"))
                rows.append((ts, float(parts[2]), float(parts[3]), parts[6:10]))
            except ValueError:
                continue
        os.unlink(self.path)
        win = [r for r in rows if t_start - 1.0 <= r[0] <= t_end + 1.0]
        if len(win) < 3:
            win = rows
        if not win:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in win for i, v in enumerate(r[3]) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(r[1] for r in win), "sm_max_mhz": max(r[2] for r in win),
                "reasons": reasons, "samples": len(win)}


# ----------------------------------------------------------------------------- helpers

def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def base_name(name: str) -> str:
    return {"c3rt": "c3", "c5m": "c5"}.get(name, name)


def fp64_peak():
    """The MEASURED fp64 (DFMA) peak of this pool's B200s (scripts/fp64_peak.cu, committed under
    profiles/): the sustained figure for a kernel timed inside a long step."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "fp64_peak.json")))
        return float(d["fp64_tflops_sustained"]), d.get("source", "profiles/fp64_peak.json")
    except (OSError, ValueError, KeyError):
        return None, None


def algorithmic_bytes(n_det, det_samples, n_samp_in, has_flags, has_hwp, has_sflags, touched_pixels, nnz):
    """HBM bytes one launch of the fused kernel must move (SURVEY 8(d) B_alg):
    TOD + det flags per det-sample, boresight/HWP/shared flags per sample, and one read + one
    write-back of the map pixels the launch touches."""
    b = det_samples * (8 + (1 if has_flags else 0))
    b += n_samp_in * (32 + (8 if has_hwp else 0) + (1 if has_sflags else 0))
    b += 2 * touched_pixels * nnz * 8
    return float(b)


# ----------------------------------------------------------------------------- cpu baseline / reference arm

def cpu_sample_workload(name: str, target_det_samples: float, obs: int = 0):
    """A bounded sample of the workload: all detectors of the first samples of observation `obs`
    (host-generated, synth.py)."""
    from paper_conf_sc_demeurekktbb23_b200 import synth
    full = synth.CONFIGS[base_name(name)]
    n_det, n_samp = full[1], full[2]
    ns = int(min(n_samp, max(1000, target_det_samples / n_det)))
    ns -= ns % 16
    return synth.make_workload(base_name(name), n_samp=ns, obs=obs)


def time_oracle(w, threads: int):
    import oracle
    zmap = np.zeros((w.n_submap, w.n_pix_submap, w.nnz))
    t0 = time.perf_counter()
    used = oracle.pointing_to_map_omp(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals,
                                      w.nside, w.nest, w.nnz, w.global2local, w.n_pix_submap, zmap, hwp=w.hwp,
                                      det_flags=w.det_flags, det_flag_mask=w.det_flag_mask,
                                      shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask,
                                      n_threads=threads)
    return time.perf_counter() - t0, used


def cpu_baseline(name: str, seconds_target: float = 8.0):
    cores = cpu_cores()
    probe = cpu_sample_workload(name, 2e6)
    dt, used = time_oracle(probe, cores)
    rate = probe.det_samples / max(dt, 1e-9)
    w = cpu_sample_workload(name, rate * seconds_target)
    dt, used = time_oracle(w, cores)
    return {"value": w.det_samples / dt, "unit": UNIT, "cores": used, "kind": "oracle",
            "sample": f"{w.n_det} dets x first {w.n_samp} samples of observation 0 of {base_name(name)} "
                      f"({w.det_samples} det-samples), oracle OpenMP timing mode (omp atomic map updates), "
                      f"{dt:.1f} s"}


def run_reference(args):
    world, rank, local = dist_env()
    if rank != 0:
        return
    cores = cpu_cores()
    probe = cpu_sample_workload(args.workload, 1e6)
    dt, used = time_oracle(probe, cores)
    rate = probe.det_samples / max(dt, 1e-9)
    # each step: a sample sized to ~1.5 s so the whole run stays within a few minutes
    w = cpu_sample_workload(args.workload, rate * 1.5)
    for _ in range(args.warmup):
        time_oracle(w, cores)
    times = []
    for _ in range(args.steps):
        dt, used = time_oracle(w, cores)
        times.append(dt)
    tot = sum(times)
    value = w.det_samples * args.steps / tot
    sample = (f"per step {w.n_det} dets x first {w.n_samp} samples ({w.det_samples} det-samples) of "
              f"{base_name(args.workload)}, oracle OpenMP timing mode")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
            "higher_is_better": True, "scaling": "strong" if args.workload in ("c4", "c5m") else "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.workload}: {WORKLOAD_DESC[args.workload]}", "oracle_sample": sample},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": used, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- inputs

class Obs:
    """One observation (or a detector block of one) resident on the device."""

    def __init__(self, name, obs, det_range, device):
        import torch
        from paper_conf_sc_demeurekktbb23_b200 import binding, synth
        from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload
        bn = base_name(name)
        on_dev = name in DEVICE_TOD
        w = synth.make_workload(bn, obs=obs, det_range=det_range, with_tod=not on_dev)
        tod = None
        if on_dev:
            w.gen_det_flags()
            tod = torch.empty((w.n_det, w.n_samp), dtype=torch.float64, device=device)
            binding.synth_tod(tod, torch.from_numpy(w.sigma).to(device), torch.from_numpy(w.det_ids).to(device),
                              w.seed)
        self.w = w
        self.dw = DeviceWorkload.upload(w, device, det_data=tod, alloc_map=False)
        self.det_samples = w.det_samples
        self.n_in = w.det_samples // max(w.n_det, 1)


def smooth_map(w, device):
    """I = cos 3theta, Q = sin 2phi sin theta, U = cos phi sin theta on the RING pixel centres
    (Gorski's inverse formulas, the scan input of c3rt), in w's (identity) map layout."""
    import torch
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    from independent import ring_centres
    z, ph = ring_centres(w.nside)
    st = np.sqrt(1 - z * z)
    m = np.stack([np.cos(3 * np.arccos(z)), np.sin(2 * ph) * st, np.cos(ph) * st], -1)
    return torch.from_numpy(np.ascontiguousarray(m.reshape(w.n_submap, w.n_pix_submap, 3))).to(device)


# ----------------------------------------------------------------------------- ours

def main():
    args = parse()
    world, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist
    from paper_conf_sc_demeurekktbb23_b200 import binding
    from paper_conf_sc_demeurekktbb23_b200 import dist as tdist

    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (there is no CPU fallback)")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    binding.load()
    name = args.workload
    shard = args.shard if args.shard != "auto" else ("det" if name in ("c4", "c5m") else "obs")

    # ---- this rank's work: (observation, detector range) units (dist.work_plan)
    from paper_conf_sc_demeurekktbb23_b200 import synth
    full_det = synth.CONFIGS[base_name(name)][1]
    work = tdist.work_plan(C5M_OBS if name == "c5m" else 1, full_det, world, rank, shard)
    obs = [Obs(name, o, dr, dev) for o, dr in work]
    w0 = obs[0].w
    n_submap, nps, nnz = w0.n_submap, w0.n_pix_submap, w0.nnz
    zmap = torch.zeros((n_submap, nps, nnz), dtype=torch.float64, device=dev)
    hits = torch.zeros(n_submap, dtype=torch.uint8, device=dev)
    g2l = obs[0].dw.global2local
    scan_map_in = None
    if name == "c3rt":
        scan_map_in = smooth_map(w0, dev)
    elif name == "c5m":
        scan_map_in = torch.randn((n_submap, nps, nnz), dtype=torch.float64, device=dev,
                                  generator=torch.Generator(dev).manual_seed(20231112))
    det_samples = sum(o.det_samples for o in obs)  # this rank's, per step
    stream = torch.cuda.current_stream()
    lib = binding.load()
    # pre-marshalled C-ABI arguments (one map and one hit-submap buffer for all of this rank's units)
    raws = [o.dw.raw_args(stream, zmap=zmap) for o in obs]
    raws = [tuple(list(r[:19]) + [hits.data_ptr()] + list(r[20:])) for r in raws]

    # f3 sparse map domain (--reduce scatter): one pointing pass marks the hit submaps (TOAST computes
    # its pixel distribution once per data set), the map then holds storage for the union of hit
    # submaps only; N > 1 reduce-scatters it (each rank keeps its owned block)
    own = None
    if args.reduce == "scatter":
        for raw in raws:
            if lib.toast_pointing_to_map(*raw) != 0:
                raise binding.ToastError(lib.toast_last_error().decode())
        hits_all = tdist.union_hit_submaps(hits) if world > 1 else hits
        g2l, n_hit = tdist.compact_global2local(hits_all)
        own = tdist.MapOwnership.make(n_hit, world)
        zmap = tdist.alloc_compact_map(own, nps, nnz, dev)
        raws = [o.dw.raw_args(stream, zmap=zmap, global2local=g2l) for o in obs]
        raws = [tuple(list(r[:19]) + [hits.data_ptr()] + list(r[20:])) for r in raws]
        torch.cuda.synchronize()

    packed = own is None and world > 1 and (args.reduce in ("packed", "nvls") or
                                            (args.reduce == "auto" and zmap.numel() * 8 > (256 << 20)))
    # --reduce nvls: the packed union summed in the switch by toast_map_allreduce_nvls (f3)
    nvls_red = tdist.NvlsReducer(zmap.numel(), dev) if (world > 1 and args.reduce == "nvls") else None
    reduced = {"bytes": 0}
    kern_events = []  # (start, end) of every fused map launch in the timed region

    def scan(o):
        binding.pointing_to_tod(o.dw.fp_quats, o.dw.boresight, o.dw.epsilon, o.w.cal, o.dw.intervals, o.w.nside,
                                o.w.nest, nnz, g2l, nps, scan_map_in, o.dw.det_data, should_zero=True, hwp=o.dw.hwp,
                                shared_flags=o.dw.shared_flags, shared_flag_mask=o.w.shared_flag_mask, stream=stream)

    def step(timed=False):
        zmap.zero_()
        hits.zero_()
        for o, raw in zip(obs, raws):
            if scan_map_in is not None:
                scan(o)
            if timed:
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
            rc = lib.toast_pointing_to_map(*raw)
            if rc != 0:
                raise binding.ToastError(lib.toast_last_error().decode())
            if timed:
                b.record(stream)
                kern_events.append((a, b))
        if world > 1:
            if own is not None:
                _, reduced["bytes"] = tdist.reduce_scatter_map(zmap, own)
            elif packed:
                tdist.union_hit_submaps(hits)
                _, reduced["bytes"] = tdist.reduce_map(zmap, hit_submaps=hits, global2local=g2l, nvls=nvls_red)
            else:
                _, reduced["bytes"] = tdist.reduce_map(zmap)

    graph = None
    if args.graph > 0:
        if world > 1 or scan_map_in is not None:
            raise SystemExit("--graph: single-GPU map workloads only")
        step()  # the work list is cached before capture
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            cs = torch.cuda.current_stream()
            graws = [tuple(list(r[:-1]) + [cs.cuda_stream]) for r in raws]
            for _ in range(args.graph):
                zmap.zero_()
                hits.zero_()
                for raw in graws:
                    if lib.toast_pointing_to_map(*raw) != 0:
                        raise binding.ToastError(lib.toast_last_error().decode())
        plain_step = step

        def step(timed=False):  # noqa: F811  (one step = one replay of G calls)
            if timed:
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
            graph.replay()
            if timed:
                b.record(stream)
                kern_events.append((a, b))
        del plain_step

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    # soak: keep the GPU busy so clocks settle before the timed region
    t_end_soak = time.time() + args.soak
    while time.time() < t_end_soak:
        step()
        torch.cuda.synchronize()

    # one separately timed reduction (reported in config; the timed steps include it)
    ar_ms = 0.0
    if world > 1:
        dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        if own is not None:
            tdist.reduce_scatter_map(zmap, own)
        elif packed:
            tdist.union_hit_submaps(hits)
            tdist.reduce_map(zmap, hit_submaps=hits, global2local=g2l, nvls=nvls_red)
        else:
            tdist.reduce_map(zmap)
        b.record(stream)
        torch.cuda.synchronize()
        ar_ms = a.elapsed_time(b)

    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_wall0 = time.time()
    e0.record(stream)
    for _ in range(args.steps):
        step(timed=True)
    e1.record(stream)
    torch.cuda.synchronize()
    t_wall1 = time.time()
    if world > 1:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    kern_ms = statistics.mean(a.elapsed_time(b) for a, b in kern_events)  # per launch
    launches_per_step = len(obs) * (2 if scan_map_in is not None else 1)
    if graph is not None:  # a replay holds G (zero + fused call)s: per call
        kern_ms /= args.graph
        det_samples *= args.graph
        launches_per_step *= args.graph
    time.sleep(0.2)
    sampler.stop()
    clocks = sampler.summary(t_wall0, t_wall1)

    ms_t = torch.tensor([ms, kern_ms], dtype=torch.float64, device=dev)
    tot_t = torch.tensor([float(det_samples)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
        dist.all_reduce(tot_t, op=dist.ReduceOp.SUM)
    ms, kern_ms = float(ms_t[0]), float(ms_t[1])
    total_det_samples = float(tot_t[0])  # all ranks, per step
    value = total_det_samples * args.steps / (ms / 1e3)

    # ---- end to end through the public API, host (pinned) buffers, copies in the timed region
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, obs, zmap, hits, g2l, world, stream, packed,
                      total_det_samples / (args.graph if graph is not None else 1), scan_map_in, own, nvls_red)

    # ---- roofline of the dominant kernel (the fused pointing->map kernel), per launch
    det_per_launch = det_samples / len(obs) / (args.graph if graph is not None else 1)
    peak_meas, peak_src = fp64_peak()
    clk = clocks.get("sm_max_mhz") or 1965.0
    peak_nominal = SMS * DFMA_PER_SM_PER_CLK * 2 * clk * 1e6 / 1e12
    peak = peak_meas or peak_nominal
    ach_tflops = F_ALG * det_per_launch / (kern_ms / 1e3) / 1e12
    touched = int(torch.count_nonzero(zmap.reshape(-1, nnz).abs().sum(dim=1))) // max(len(obs), 1)
    b_alg = algorithmic_bytes(w0.n_det, det_per_launch, obs[0].n_in, w0.det_flags is not None, w0.hwp is not None,
                              w0.shared_flags is not None, touched, nnz)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    # DRAM traffic of one launch of the fused kernel, from the committed ncu --set full capture of
    # this workload (profiles/traffic.json; ncu never runs inside the bench), else null
    traffic, traffic_src = None, None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "traffic.json"))).get(base_name(name))
        if tr:
            traffic, traffic_src = float(tr["dram_bytes_per_launch"]), tr["source"]
    except (OSError, ValueError, KeyError):
        pass
    roofline = {"bound": "alu", "achieved": ach_tflops, "peak": peak, "unit": "TFLOP/s", "frac": ach_tflops / peak,
                "traffic": traffic, "traffic_unit": "B/launch", "traffic_source": traffic_src,
                "kernel": "pointing_to_map_kernel (fused A1-A4)", "kernel_ms": kern_ms,
                "det_samples_per_launch": det_per_launch, "f_alg_per_det_sample": F_ALG,
                "peak_note": (f"of measured: sustained DFMA peak of this pool's B200 ({peak_src}); nominal "
                              f"{SMS} SM x {DFMA_PER_SM_PER_CLK} DFMA/clk x 2 x {clk:.0f} MHz = {peak_nominal:.1f}")
                if peak_meas else f"derived (no measured peak): {SMS} x {DFMA_PER_SM_PER_CLK} x 2 x {clk:.0f} MHz",
                "frac_of_nominal": ach_tflops / peak_nominal,
                "hbm": {"achieved_gbs": b_alg / (kern_ms / 1e3) / 1e9, "peak_gbs": hbm_peak,
                        "frac": b_alg / (kern_ms / 1e3) / 1e9 / hbm_peak, "alg_bytes_per_launch": b_alg,
                        "touched_pixels": touched,
                        "peak_note": "MEASURED_PEAKS.json hbm_gbs (measured)" if "hbm_gbs" in peaks
                        else "fallback 6650 GB/s"}}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(name)

    if rank == 0:
        strong = shard == "det" and world > 1 or name == "c5m"
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
                "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": f"{name}: {WORKLOAD_DESC[name]}",
                           "det_samples_per_step": total_det_samples, "n_det": int(synth.CONFIGS[base_name(name)][1]),
                           "n_samp": w0.n_samp, "n_intervals": len(w0.intervals), "nside": w0.nside,
                           "nest": w0.nest, "nnz": nnz, "observations_per_rank": len(obs),
                           "l2": "inputs larger than L2 (TOD %.0f MB per rank), no flush" %
                                 (sum(o.w.n_det * o.w.n_samp * 8 for o in obs) / 1e6),
                           "parallelism": (f"dp{world}: " + ("detector blocks of one observation" if shard == "det"
                                                             else "one observation per rank") +
                                           (" + NVLS multimem all-reduce (toast_map_allreduce_nvls) of the union of "
                                            "hit submaps" if nvls_red is not None else
                                            " + NCCL " + ("packed all_reduce (union of hit submaps)" if packed
                                                          else "all_reduce") + " of the map")) if world > 1
                           else "single GPU",
                           "step": "zero map + " + ("(pointing_to_tod + pointing_to_map) per observation"
                                                    if scan_map_in is not None else "toast_pointing_to_map") +
                                   (" + map reduction" if world > 1 else ""),
                           "map_domain": (f"compact: {own.n_hit} hit submaps of {n_submap} (dist.compact_global2local)"
                                          + (", NCCL reduce_scatter" if world > 1 else "")) if own is not None
                           else "dense",
                           "allreduce_bytes_per_step": reduced["bytes"], "allreduce_ms": ar_ms,
                           "staging": binding.last_fused_path(),
                           "cuda_graph": (f"one step = one replay of a CUDA graph of {args.graph} x (zero map + "
                                          "toast_pointing_to_map); roofline.kernel_ms per call includes the zeroing")
                           if graph is not None else None,
                           "tod_source": "device counter hash (toast_synth_tod, bit-identical to synth.py)"
                           if name in DEVICE_TOD else "host synth.py"},
                "clocks": clocks, "gpu_launches": args.steps * launches_per_step, "roofline": roofline}
        if e2e is not None:
            line["e2e"] = e2e
        if cpu is not None:
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_e2e(args, obs, zmap, hits, g2l, world, stream, packed, total_det_samples, with_scan, own=None,
            nvls_red=None):
    """Same metric through the public API with host buffers: every step copies the step's inputs
    from pinned host memory (the TOD in 256-detector blocks through two device staging buffers,
    overlapped with the fused kernel: streaming.Streamer) and reads the map back."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_demeurekktbb23_b200 import dist as tdist
    from paper_conf_sc_demeurekktbb23_b200.streaming import HostInputs, Streamer
    if with_scan is not None:
        return run_e2e_round_trip(args, obs, zmap, hits, g2l, world, stream, packed, total_det_samples, own, with_scan,
                                  nvls_red)
    hosts, streamers = [], []
    try:
        for o in obs:
            def pin(t):
                if t is None:
                    return None
                h = torch.empty(t.shape, dtype=t.dtype, pin_memory=True)
                h.copy_(t)
                return h
            hosts.append(HostInputs(pin(o.dw.fp_quats), pin(o.dw.boresight), pin(o.dw.epsilon), pin(o.dw.det_scale),
                                    pin(o.dw.det_data), pin(o.dw.hwp), pin(o.dw.det_flags), pin(o.dw.shared_flags)))
        for o in obs:
            streamers.append(Streamer(o.w.n_det, o.w.n_samp, 256, zmap.device, o.dw.hwp is not None,
                                      o.dw.det_flags is not None, o.dw.shared_flags is not None))
    except RuntimeError as e:  # pinned host memory exhausted
        return {"value": None, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0,
                "note": f"pinned host buffers unavailable: {str(e)[:120]}"}
    host_map = torch.empty(zmap.shape, dtype=torch.float64).pin_memory()
    h2d = sum(h.nbytes() for h in hosts)
    d2h = host_map.numel() * 8
    steps = max(2, min(args.steps, 5 if h2d > (8 << 30) else 20))

    def e2e_step():
        zmap.zero_()
        hits.zero_()
        for o, h, sr in zip(obs, hosts, streamers):
            sr.pointing_to_map(h, o.dw.intervals, o.w.nside, o.w.nest, o.w.nnz, g2l, o.w.n_pix_submap, zmap, o.w.cal,
                               det_flag_mask=o.w.det_flag_mask, shared_flag_mask=o.w.shared_flag_mask,
                               hit_submaps=hits, stream=stream)
        if world > 1:
            if own is not None:
                tdist.reduce_scatter_map(zmap, own)
            elif packed:
                tdist.union_hit_submaps(hits)
                tdist.reduce_map(zmap, hit_submaps=hits, global2local=g2l, nvls=nvls_red)
            else:
                tdist.reduce_map(zmap)
        host_map.copy_(zmap, non_blocking=True)

    e2e_step()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    a.record(stream)
    for _ in range(steps):
        e2e_step()
    b.record(stream)
    torch.cuda.synchronize()
    ms = torch.tensor([a.elapsed_time(b)], dtype=torch.float64, device=zmap.device)
    if world > 1:
        dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms = float(ms[0])
    return {"value": total_det_samples * steps / (ms / 1e3), "unit": UNIT, "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": d2h, "steps": steps,
            "path": "streaming.Streamer -> binding.pointing_to_map (ctypes -> toast_pointing_to_map), TOD in "
                    "256-detector blocks from pinned host memory, copy of block b+1 overlapping the kernel on b"}


def run_e2e_round_trip(args, obs, zmap, hits, g2l, world, stream, packed, total_det_samples, own, scan_map_in,
                       nvls_red=None):
    """e2e of the round-trip workloads (c3rt, c5m): every step copies the input map and each
    observation's pointing inputs (focal plane, boresight, HWP, flags; the TOD is the scan's
    output and never leaves the device) from pinned host memory, scans and accumulates through
    the public API, and reads the map back."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_demeurekktbb23_b200 import binding
    from paper_conf_sc_demeurekktbb23_b200 import dist as tdist

    def pin(t):
        if t is None:
            return None
        h = torch.empty(t.shape, dtype=t.dtype, pin_memory=True)
        h.copy_(t)
        return h
    try:
        names = ("fp_quats", "boresight", "epsilon", "det_scale", "hwp", "det_flags", "shared_flags")
        hosts = [{k: pin(getattr(o.dw, k)) for k in names} for o in obs]
        host_in = pin(scan_map_in)
        host_map = torch.empty(zmap.shape, dtype=torch.float64).pin_memory()
    except RuntimeError as e:  # pinned host memory exhausted
        return {"value": None, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0,
                "note": f"pinned host buffers unavailable: {str(e)[:120]}"}
    dev_in = torch.empty_like(scan_map_in)
    h2d = host_in.numel() * 8 + sum(t.numel() * t.element_size() for h in hosts for t in h.values() if t is not None)
    d2h = host_map.numel() * 8

    def e2e_step():
        dev_in.copy_(host_in, non_blocking=True)
        zmap.zero_()
        hits.zero_()
        for o, h in zip(obs, hosts):
            for k, t in h.items():
                if t is not None:
                    getattr(o.dw, k).copy_(t, non_blocking=True)
            w, dw = o.w, o.dw
            binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, dw.intervals, w.nside, w.nest, w.nnz,
                                    g2l, w.n_pix_submap, dev_in, dw.det_data, should_zero=True, hwp=dw.hwp,
                                    shared_flags=dw.shared_flags, shared_flag_mask=w.shared_flag_mask, stream=stream)
            binding.pointing_to_map(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, dw.det_scale, dw.det_data,
                                    dw.intervals, w.nside, w.nest, w.nnz, g2l, w.n_pix_submap, zmap, hwp=dw.hwp,
                                    det_flags=dw.det_flags, det_flag_mask=w.det_flag_mask,
                                    shared_flags=dw.shared_flags, shared_flag_mask=w.shared_flag_mask,
                                    hit_submaps=hits, stream=stream)
        if world > 1:
            if own is not None:
                tdist.reduce_scatter_map(zmap, own)
            elif packed:
                tdist.union_hit_submaps(hits)
                tdist.reduce_map(zmap, hit_submaps=hits, global2local=g2l, nvls=nvls_red)
            else:
                tdist.reduce_map(zmap)
        host_map.copy_(zmap, non_blocking=True)

    e2e_step()
    torch.cuda.synchronize()
    steps = max(2, min(args.steps, 5))
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    a.record(stream)
    for _ in range(steps):
        e2e_step()
    b.record(stream)
    torch.cuda.synchronize()
    ms = torch.tensor([a.elapsed_time(b)], dtype=torch.float64, device=zmap.device)
    if world > 1:
        dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms = float(ms[0])
    return {"value": total_det_samples * steps / (ms / 1e3), "unit": UNIT, "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": d2h, "steps": steps,
            "path": "binding.pointing_to_tod -> binding.pointing_to_map per observation (ctypes -> C-ABI), the input "
                    "map and every observation's pointing inputs copied from pinned host memory each step, the "
                    "map read back"}


if __name__ == "__main__":
    main()
