"""Parity comparison rules T1-T4 — tests only.

T1 pixels: equal, except mismatches whose ORACLE direction is within 1e-12 rad of a
   pixel boundary (oracle classifier, run on mismatches only); such mismatches must be
   <= 1e-6 of the compared samples.  Flagged samples must be exactly -1.
T2 weights: |dI| <= 1e-12 |cal|; |dQ|, |dU| <= |eta cal| max(1e-12, 1e-15 / sin(theta)).
T3 timestreams: |dtod| <= 1e-12 B (+ weight tolerance propagated through the map values).
T4 maps: |dzmap| <= 1e-10 A, A = sum |terms|; A = 0 -> exactly 0.  For Q and U of the fused
   path the T2 weight tolerance of each term propagates: + sum |det_scale tod| |eta cal|
   max(1e-12, 1e-15 / sin(theta)) (the oracle's t2map).
"""
from __future__ import annotations

import numpy as np

import oracle

NEAR_DELTA = 1.1e-12


def classify_pixel_mismatches(gpu_pix, ora_pix, probe, nside, nest, n_compared):
    """Returns the (d, s) index arrays of mismatches.  `probe(d, s)` -> oracle direction.
    Asserts every mismatch is near a boundary and the count is <= 1e-6 of n_compared."""
    bad = np.nonzero(gpu_pix != ora_pix)
    n_bad = len(bad[0])
    for d, s in zip(*bad):
        assert ora_pix[d, s] >= 0 and gpu_pix[d, s] >= 0, f"flag mismatch at det {d} sample {s}"
        v = probe(int(d), int(s))
        assert oracle.near_boundary(nside, nest, v, NEAR_DELTA), (
            f"pixel mismatch away from a boundary: det {d} sample {s} gpu {gpu_pix[d, s]} oracle {ora_pix[d, s]}")
    assert n_bad <= 1e-6 * n_compared, f"{n_bad} near-boundary mismatches > 1e-6 of {n_compared}"
    return bad


def t2_weight_tol(sin_theta, eta_cal):
    """T2 bound of |dQ|, |dU| for one det-sample."""
    return np.abs(eta_cal) * np.maximum(1e-12, 1e-15 / np.maximum(sin_theta, 1e-300))


def check_weights(gpu_w, ora_w, sin_theta, eta_cal, cal, mask):
    """T2 on the masked (in-interval) det-samples. eta_cal: [n_det]."""
    gi, oi = gpu_w[..., 0][mask], ora_w[..., 0][mask]
    assert np.all(np.abs(gi - oi) <= 1e-12 * abs(cal))
    if gpu_w.shape[-1] == 3:
        tol = t2_weight_tol(sin_theta, np.asarray(eta_cal)[:, None])[mask]
        for k in (1, 2):
            dk = np.abs(gpu_w[..., k][mask] - ora_w[..., k][mask])
            worst = np.argmax(dk - tol) if dk.size else 0
            assert np.all(dk <= tol), f"weight {k}: max excess {(dk - tol).max()} at {worst}"


def check_map(gpu_map, ora_map, absmap, t2map=None, rel=1e-10, extra=None):
    """T4: |d| <= rel A (+ t2map: the propagated T2 tolerance of Q/U terms) (+ extra)."""
    zero = absmap[..., :1] == 0 if absmap.shape[-1] == 3 else absmap == 0
    zero = np.broadcast_to(zero, absmap.shape)
    assert np.all(gpu_map[zero] == 0.0), "map element with no contribution is not exactly 0"
    diff = np.abs(gpu_map - ora_map)
    tol = rel * absmap
    if t2map is not None:
        tol = tol + t2map
    if extra is not None:
        tol = tol + extra
    bad = diff > tol
    assert not np.any(bad), f"{int(bad.sum())} map elements beyond T4; worst excess {(diff - tol).max()}"


def reconcile_map(ora_map, absmap, mism, gpu_pix, ora_pix, ora_w, w, g2l, nps, t2map=None, sin_theta=None):
    """Move the contributions of near-boundary mismatched samples to the GPU's pixel, so the
    map comparison checks the arithmetic and not the (allowed) boundary decisions.  The moved
    sample's tolerance terms go with it."""
    for d, s in zip(*mism):
        if w.det_flags is not None and (w.det_flags[d, s] & w.det_flag_mask):
            continue
        val = w.det_scale[d] * w.det_data[d, s]
        i_from = (g2l[ora_pix[d, s] // nps], ora_pix[d, s] % nps)
        i_to = (g2l[gpu_pix[d, s] // nps], gpu_pix[d, s] % nps)
        terms = val * ora_w[d, s]
        ora_map[i_from] -= terms
        ora_map[i_to] += terms
        absmap[i_to] += np.abs(terms)
        if t2map is not None:
            eta_cal = (1 - w.epsilon[d]) / (1 + w.epsilon[d]) * w.cal
            t2map[i_to][1:] += abs(val) * t2_weight_tol(sin_theta(int(d), int(s)), eta_cal)
    return ora_map, absmap
