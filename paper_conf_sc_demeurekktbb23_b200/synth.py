"""Seeded synthetic inputs for the pointing->map path (SURVEY.md Sec. 8(d) recipe).

This module is the ONE piece shared by the oracle side (tests, cpu_baseline)
and the CUDA side (bench, tests).  It holds none of the method's arithmetic:
  * quaternions are built from rotation MATRICES (products of axis rotations)
    converted with Shepperd's method — never with the Hamilton product or the
    vector rotation the method computes (A1/A2/A3);
  * no HEALPix, no Stokes weights, no map arithmetic;
  * the timestream is a counter-based SplitMix64 hash of
    (seed, stream, det, sample) turned into an exact dyadic in [-1, 1), scaled
    by a per-detector sigma, so any subset can be regenerated bit-identically.

Shapes follow the paper's workloads: a satellite scan (PAPER.md:193-196,
"satellite-telescope simulation" with "a couple thousand detectors", :51) and
a ground constant-elevation scan; detectors x intervals x samples with
intervals of varying length.  Config sizes are BASELINE.json's
configs C1-C5.
"""
from __future__ import annotations

import dataclasses
import math
from typing import Optional

import numpy as np

MASTER_SEED = 20231112
STREAM_TOD = 1
STREAM_FP = 2
STREAM_INTERVALS = 3
STREAM_FLAGS = 4
STREAM_DETFLAGS = 5

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


# --------------------------------------------------------------------------- counter-based RNG

def splitmix64_mix(z):
    """SplitMix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def counter_hash(seed: int, stream: int, det, sample):
    """h = mix(mix(mix(seed + G(stream+1)) + G(det+1)) + G(sample+1)), all mod 2^64."""
    with np.errstate(over="ignore"):
        k = splitmix64_mix(np.uint64(seed) + _GOLDEN * np.uint64(stream + 1))
        k = splitmix64_mix(k + _GOLDEN * (np.asarray(det, dtype=np.uint64) + np.uint64(1)))
        return splitmix64_mix(k + _GOLDEN * (np.asarray(sample, dtype=np.uint64) + np.uint64(1)))


def hash_to_unit(h):
    """Exact dyadic in [-1, 1): (h >> 11) * 2^-52 - 1."""
    return (np.asarray(h) >> np.uint64(11)).astype(np.float64) * (2.0 ** -52) - 1.0


def hash_to_u01(h):
    """Exact dyadic in [0, 1)."""
    return (np.asarray(h) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def tod_rows(seed: int, sigma: np.ndarray, det_ids: np.ndarray, n_samp: int, s0: int = 0, s1: Optional[int] = None):
    """TOD[d, s] = sigma_d * u(seed, TOD, det, s) for the given detector ids."""
    s1 = n_samp if s1 is None else s1
    samples = np.arange(s0, s1, dtype=np.uint64)
    out = np.empty((len(det_ids), s1 - s0))
    for i, d in enumerate(det_ids):
        out[i] = sigma[i] * hash_to_unit(counter_hash(seed, STREAM_TOD, int(d), samples))
    return out


# --------------------------------------------------------------------------- rotations (matrices)

def rot_axis(axis: str, angle):
    """Stack of 3x3 right-handed rotation matrices about a coordinate axis."""
    a = np.atleast_1d(np.asarray(angle, dtype=np.float64))
    c, s = np.cos(a), np.sin(a)
    m = np.zeros(a.shape + (3, 3))
    i, j = {"x": (1, 2), "y": (2, 0), "z": (0, 1)}[axis]
    k = 3 - i - j
    m[..., k, k] = 1.0
    m[..., i, i] = c
    m[..., j, j] = c
    m[..., i, j] = -s
    m[..., j, i] = s
    return m


def matmul_chain(*mats):
    out = mats[0]
    for m in mats[1:]:
        out = np.einsum("...ij,...jk->...ik", out, m)
    return out


def matrix_to_quat(m):
    """Shepperd's method: rotation matrix -> unit quaternion [x, y, z, w] (w >= 0),
    renormalised in fp64 (reading S7)."""
    m = np.asarray(m, dtype=np.float64)
    shp = m.shape[:-2]
    m = m.reshape(-1, 3, 3)
    tr = m[:, 0, 0] + m[:, 1, 1] + m[:, 2, 2]
    cand = np.stack([tr, m[:, 0, 0], m[:, 1, 1], m[:, 2, 2]], axis=1)
    which = np.argmax(cand, axis=1)
    q = np.empty((m.shape[0], 4))
    for k in range(4):
        sel = which == k
        if not np.any(sel):
            continue
        mm = m[sel]
        if k == 0:
            r = np.sqrt(1.0 + tr[sel]) * 2.0
            q[sel, 3] = 0.25 * r
            q[sel, 0] = (mm[:, 2, 1] - mm[:, 1, 2]) / r
            q[sel, 1] = (mm[:, 0, 2] - mm[:, 2, 0]) / r
            q[sel, 2] = (mm[:, 1, 0] - mm[:, 0, 1]) / r
        elif k == 1:
            r = np.sqrt(1.0 + mm[:, 0, 0] - mm[:, 1, 1] - mm[:, 2, 2]) * 2.0
            q[sel, 3] = (mm[:, 2, 1] - mm[:, 1, 2]) / r
            q[sel, 0] = 0.25 * r
            q[sel, 1] = (mm[:, 0, 1] + mm[:, 1, 0]) / r
            q[sel, 2] = (mm[:, 0, 2] + mm[:, 2, 0]) / r
        elif k == 2:
            r = np.sqrt(1.0 + mm[:, 1, 1] - mm[:, 0, 0] - mm[:, 2, 2]) * 2.0
            q[sel, 3] = (mm[:, 0, 2] - mm[:, 2, 0]) / r
            q[sel, 0] = (mm[:, 0, 1] + mm[:, 1, 0]) / r
            q[sel, 1] = 0.25 * r
            q[sel, 2] = (mm[:, 1, 2] + mm[:, 2, 1]) / r
        else:
            r = np.sqrt(1.0 + mm[:, 2, 2] - mm[:, 0, 0] - mm[:, 1, 1]) * 2.0
            q[sel, 3] = (mm[:, 1, 0] - mm[:, 0, 1]) / r
            q[sel, 0] = (mm[:, 0, 2] + mm[:, 2, 0]) / r
            q[sel, 1] = (mm[:, 1, 2] + mm[:, 2, 1]) / r
            q[sel, 2] = 0.25 * r
    q[q[:, 3] < 0] *= -1.0
    q /= np.sqrt(np.sum(q * q, axis=1))[:, None]
    return q.reshape(shp + (4,))


# --------------------------------------------------------------------------- focal plane

def hex_positions(n_pos: int):
    """n_pos points of a hexagonal lattice closest to the centre (unit spacing)."""
    r = int(math.ceil(math.sqrt(n_pos))) + 2
    pts = []
    for i in range(-r, r + 1):
        for j in range(-r, r + 1):
            x = i + 0.5 * j
            y = j * math.sqrt(3.0) / 2.0
            pts.append((x * x + y * y, math.atan2(y, x), x, y))
    pts.sort()
    return np.array([(p[2], p[3]) for p in pts[:n_pos]])


def focal_plane(n_det: int, radius_deg: float, seed: int):
    """fp[d] = Rz(phi_d) Ry(rho_d) Rz(-phi_d) Rz(gamma_d): n_det/2 hex positions,
    2 orthogonal detectors per position, alternate positions rotated by 45 deg.
    Returns (fp_quats[n_det][4], epsilon[n_det], sigma[n_det])."""
    n_pos = max(1, (n_det + 1) // 2)
    xy = hex_positions(n_pos)
    rmax = np.max(np.hypot(xy[:, 0], xy[:, 1]))
    scale = (math.radians(radius_deg) / rmax) if rmax > 0 else 0.0
    mats = []
    for d in range(n_det):
        p = d // 2
        x, y = xy[p] * scale
        rho = math.hypot(x, y)
        phi = math.atan2(y, x)
        gamma = (0.0 if d % 2 == 0 else math.pi / 2) + (math.pi / 4 if p % 2 else 0.0)
        mats.append(matmul_chain(rot_axis("z", phi), rot_axis("y", rho), rot_axis("z", -phi),
                                 rot_axis("z", gamma))[0])
    fp = matrix_to_quat(np.array(mats))
    u = hash_to_u01(counter_hash(seed, STREAM_FP, np.arange(n_det), 0))
    v = hash_to_u01(counter_hash(seed, STREAM_FP, np.arange(n_det), 1))
    epsilon = 0.01 * u
    sigma = 0.8 + 0.4 * v
    return fp, epsilon, sigma


# --------------------------------------------------------------------------- scans

def satellite_boresight(n_samp: int, rate: float, t0: float = 0.0):
    """LiteBIRD-like: Rz(2pi t/yr) Ry(pi/2) Rz(2pi t/T_p) Ry(alpha) Rz(2pi t/T_s) Ry(beta),
    alpha = 45 deg, beta = 50 deg, T_p = 192.348 min, T_s = 20 min."""
    t = t0 + np.arange(n_samp) / rate
    yr = 365.25 * 86400.0
    m = matmul_chain(rot_axis("z", 2 * np.pi * t / yr), rot_axis("y", np.pi / 2),
                     rot_axis("z", 2 * np.pi * t / (192.348 * 60.0)), rot_axis("y", np.radians(45.0)),
                     rot_axis("z", 2 * np.pi * t / (20.0 * 60.0)), rot_axis("y", np.radians(50.0)))
    return matrix_to_quat(m)


def satellite_intervals(n_samp: int, rate: float, seed: int, obs: int = 0):
    """Spans of U[0.5, 1.5] spin periods separated by gaps of U{0..50} samples."""
    spin = 20.0 * 60.0 * rate
    out = []
    s = 0
    k = 0
    while s < n_samp:
        h = counter_hash(seed, STREAM_INTERVALS, obs, np.array([2 * k, 2 * k + 1], dtype=np.uint64))
        length = max(1, int((0.5 + hash_to_u01(h[0])) * spin))
        gap = int(h[1] % np.uint64(51))
        last = min(n_samp - 1, s + length - 1)
        out.append((s, last))
        s = last + 1 + gap
        k += 1
    return out


def ground_boresight(n_samp: int, rate: float, az_center_deg: float = 120.0, az_throw_deg: float = 40.0,
                     speed_deg: float = 1.0, lat_deg: float = -22.96, el_deg: float = 50.0, t0: float = 0.0):
    """CES: Rz(w_E t) Ry(pi/2 - lat) Rz(pi - az(t)) Ry(pi/2 - el); az a triangle wave.
    Returns (quats, az_deg)."""
    t = t0 + np.arange(n_samp) / rate
    period = 2.0 * az_throw_deg / speed_deg
    ph = np.mod(t, period) * speed_deg
    tri = np.where(ph < az_throw_deg, ph, 2 * az_throw_deg - ph)
    az = az_center_deg - az_throw_deg / 2 + tri
    w_e = 2 * np.pi / 86164.0905
    m = matmul_chain(rot_axis("z", w_e * t), rot_axis("y", np.pi / 2 - np.radians(lat_deg)),
                     rot_axis("z", np.pi - np.radians(az)), rot_axis("y", np.pi / 2 - np.radians(el_deg)))
    return matrix_to_quat(m), az


def ground_intervals_and_flags(az_deg, az_center_deg=120.0, az_throw_deg=40.0, margin_deg=0.5, seed=0,
                               obs=0):
    """Intervals = constant-speed half scans (turnarounds +-0.5 deg excluded);
    shared flags: 0x01 at turnarounds, 0x02 in 0.1% bursts."""
    lo = az_center_deg - az_throw_deg / 2 + margin_deg
    hi = az_center_deg + az_throw_deg / 2 - margin_deg
    good = (az_deg > lo) & (az_deg < hi)
    flags = np.where(good, 0, 1).astype(np.uint8)
    n = len(az_deg)
    # bursts of 100 samples starting at ~1e-5 of samples -> ~0.1% flagged with 0x02
    starts = np.nonzero(hash_to_u01(counter_hash(seed, STREAM_FLAGS, obs, np.arange(n, dtype=np.uint64)))
                        < 1e-5)[0]
    for s in starts:
        flags[s:s + 100] |= 2
    edges = np.diff(np.concatenate([[0], good.astype(np.int8), [0]]))
    firsts = np.nonzero(edges == 1)[0]
    lasts = np.nonzero(edges == -1)[0] - 1
    return list(zip(firsts.tolist(), lasts.tolist())), flags


def det_flags_for(seed: int, det_ids, n_samp: int, frac: float = 0.01, obs: int = 0):
    """1% of samples flagged with bit 0x01 (masked) per detector."""
    out = np.zeros((len(det_ids), n_samp), np.uint8)
    s = np.arange(n_samp, dtype=np.uint64)
    for i, d in enumerate(det_ids):
        u = hash_to_u01(counter_hash(seed + 7919 * obs, STREAM_DETFLAGS, int(d), s))
        out[i] = (u < frac).astype(np.uint8)
    return out


def hwp_angle(n_samp: int, rate: float, freq_hz: float = 2.0, t0: float = 0.0):
    """chi = 2 pi f t wrapped into [0, 2 pi) (keeps 2 psi + 4 chi well conditioned)."""
    t = t0 + np.arange(n_samp) / rate
    return np.mod(2 * np.pi * freq_hz * t, 2 * np.pi)


# --------------------------------------------------------------------------- workloads

@dataclasses.dataclass
class Workload:
    name: str
    nside: int
    nest: bool
    nnz: int
    n_pix_submap: int
    fp_quats: np.ndarray          # [n_det][4]
    boresight: np.ndarray         # [n_samp][4]
    hwp: Optional[np.ndarray]     # [n_samp] or None
    epsilon: np.ndarray           # [n_det]
    sigma: np.ndarray             # [n_det]
    det_scale: np.ndarray         # [n_det] = 1/sigma^2
    cal: float
    intervals: list               # [(first, last)] inclusive
    shared_flags: Optional[np.ndarray]
    shared_flag_mask: int
    det_flag_frac: float
    det_flag_mask: int
    seed: int
    det_ids: np.ndarray           # global detector ids (for the hash)
    det_data: Optional[np.ndarray] = None
    det_flags: Optional[np.ndarray] = None

    @property
    def n_det(self):
        return self.fp_quats.shape[0]

    @property
    def n_samp(self):
        return self.boresight.shape[0]

    @property
    def npix(self):
        return 12 * self.nside * self.nside

    @property
    def n_submap(self):
        return self.npix // self.n_pix_submap

    @property
    def global2local(self):
        return np.arange(self.n_submap, dtype=np.int64)

    @property
    def det_samples(self):
        return self.n_det * sum(l - f + 1 for f, l in self.intervals)

    def gen_tod(self):
        self.det_data = tod_rows(self.seed, self.sigma, self.det_ids, self.n_samp)
        return self.det_data

    def gen_det_flags(self):
        if self.det_flag_frac > 0:
            self.det_flags = det_flags_for(self.seed, self.det_ids, self.n_samp, self.det_flag_frac)
        return self.det_flags


def submap_pixels(nside: int) -> int:
    ns = min(16, nside)
    return (nside // ns) ** 2


CONFIGS = {
    # name: (kind, n_det, n_samp, rate, nside, nest, hwp, flags)
    "c1": ("satellite", 4, 100_000, 37.0, 64, False, False, False),
    "c2": ("ground", 64, 1_000_000, 100.0, 256, True, True, True),
    "c3": ("ground", 1024, 60_000, 100.0, 1024, False, False, True),
    "c4": ("satellite", 2048, 3_196_800, 37.0, 2048, True, False, False),
    "c5": ("satellite", 2048, 133_200, 37.0, 4096, True, False, False),  # one of 18 observations
}


def make_workload(name: str = "c1", seed: int = MASTER_SEED, n_det: Optional[int] = None,
                  n_samp: Optional[int] = None, nside: Optional[int] = None, nest: Optional[bool] = None,
                  det_range: Optional[tuple] = None, obs: int = 0, with_tod: bool = True,
                  single_interval: Optional[bool] = None, nnz: int = 3) -> Workload:
    """Build a seeded workload.  Overrides shrink a config for tests.
    ``det_range=(d0, d1)`` keeps only those detectors of the full focal plane
    (same ids, same TOD) — used for sharding and bounded CPU samples."""
    kind, nd, ns, rate, nsd, nst, use_hwp, use_flags = CONFIGS[name]
    nd = n_det or nd
    ns = n_samp or ns
    nsd = nside or nsd
    nst = nst if nest is None else nest
    fp, eps, sigma = focal_plane(nd, 5.0 if kind == "satellite" else 2.0, seed)
    det_ids = np.arange(nd, dtype=np.int64)
    if det_range is not None:
        d0, d1 = det_range
        fp, eps, sigma, det_ids = fp[d0:d1], eps[d0:d1], sigma[d0:d1], det_ids[d0:d1]
    t0 = obs * ns / rate
    if kind == "satellite":
        bore = satellite_boresight(ns, rate, t0=t0)
        if single_interval is None:
            single_interval = name == "c1"
        intervals = [(0, ns - 1)] if single_interval else satellite_intervals(ns, rate, seed, obs)
        if name == "c5" and not single_interval:
            # ~60 intervals per 1 h observation: spans of ~1 min
            intervals = _even_intervals(ns, 60, seed, obs)
        shared = None
    else:
        bore, az = ground_boresight(ns, rate, t0=t0)
        intervals, shared = ground_intervals_and_flags(az, seed=seed, obs=obs)
        if not use_flags:
            shared = None
    hwp = hwp_angle(ns, rate, t0=t0) if use_hwp else None
    w = Workload(name=name, nside=nsd, nest=bool(nst), nnz=nnz, n_pix_submap=submap_pixels(nsd), fp_quats=fp,
                 boresight=bore, hwp=hwp, epsilon=eps, sigma=sigma, det_scale=1.0 / sigma ** 2, cal=1.0,
                 intervals=intervals, shared_flags=shared, shared_flag_mask=1 if shared is not None else 0,
                 det_flag_frac=0.01 if use_flags else 0.0, det_flag_mask=1 if use_flags else 0,
                 seed=seed + 104729 * obs, det_ids=det_ids)
    if with_tod:
        w.gen_tod()
        w.gen_det_flags()
    return w


def _even_intervals(n_samp: int, n_iv: int, seed: int, obs: int):
    span = n_samp // n_iv
    out = []
    for k in range(n_iv):
        h = counter_hash(seed, STREAM_INTERVALS, obs, np.array([k], dtype=np.uint64))
        gap = int(h[0] % np.uint64(51))
        first = k * span + gap
        last = min(n_samp - 1, (k + 1) * span - 1)
        if last >= first:
            out.append((first, last))
    return out
