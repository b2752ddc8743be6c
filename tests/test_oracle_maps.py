"""Pins for oracle A1-A6 entry points (loops, indexing, flags, accumulation), CPU only.

The accumulation is pinned by an independent numpy formulation (np.add.at over
a boolean selection), integer inputs (hit counts, bit-exact), the global-sum
identity, constant-map scans and the scan/accumulate adjoint identity
(SURVEY 8(c) O5, O6).  Loops over intervals are pinned by 'out-of-interval
samples untouched'.
"""
import math

import numpy as np
import pytest

import oracle
from independent import rodrigues
from paper_conf_sc_demeurekktbb23_b200 import synth


def _mask_intervals(intervals, n_samp):
    m = np.zeros(n_samp, bool)
    for f, l in intervals:
        m[f:l + 1] = True
    return m


@pytest.fixture(scope="module")
def small():
    w = synth.make_workload("c2", n_det=6, n_samp=9000, nside=32)
    return w


def test_pointing_detector_composes_and_skips_gaps(small):
    w = small
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    inside = _mask_intervals(w.intervals, w.n_samp)
    assert np.all(quats[:, ~inside] == 0.0)  # untouched
    # direction of detector d = R(bore) R(fp) z, via rotation matrices from synth's Shepperd inverse
    rng = np.random.default_rng(0)
    for _ in range(50):
        d = int(rng.integers(w.n_det)); s = int(rng.choice(np.nonzero(inside)[0]))
        flagged = w.shared_flags[s] & w.shared_flag_mask
        rb = np.eye(3) if flagged else _quat_matrix_ref(w.boresight[s])
        ref = rb @ _quat_matrix_ref(w.fp_quats[d]) @ np.array([0, 0, 1.0])
        np.testing.assert_allclose(oracle.quat_rotate(quats[d, s], [0, 0, 1.0]), ref, atol=1e-14)


def _quat_matrix_ref(q):
    """Rotation matrix of a unit quaternion via its axis-angle (Rodrigues), independent path."""
    x, y, z, wq = q
    s = math.sqrt(x * x + y * y + z * z)
    if s == 0:
        return np.eye(3)
    return rodrigues([x / s, y / s, z / s], 2 * math.atan2(s, wq))


def test_pixels_flags_and_hit_submaps(small):
    w = small
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals)
    pix, hits = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                      w.shared_flag_mask)
    inside = _mask_intervals(w.intervals, w.n_samp)
    assert np.all(pix[:, ~inside] == -7)  # untouched sentinel
    flagged = (w.shared_flags & w.shared_flag_mask) != 0
    assert np.all(pix[:, inside & flagged] == -1)
    good = pix[:, inside & ~flagged]
    assert good.min() >= 0 and good.max() < w.npix
    ref_hits = np.zeros(w.n_submap, np.uint8)
    ref_hits[np.unique(good // w.n_pix_submap)] = 1
    np.testing.assert_array_equal(hits, ref_hits)


def _random_inputs(rng, n_det, n_samp, npix, nnz):
    pixels = rng.integers(-1, npix, size=(n_det, n_samp)).astype(np.int64)
    weights = rng.normal(size=(n_det, n_samp, nnz))
    tod = rng.normal(size=(n_det, n_samp))
    det_flags = (rng.random((n_det, n_samp)) < 0.1).astype(np.uint8) * rng.integers(1, 4, size=(n_det, n_samp)).astype(np.uint8)
    shared = (rng.random(n_samp) < 0.1).astype(np.uint8) * 2
    scale = rng.uniform(0.5, 2, size=n_det)
    return pixels, weights, tod, det_flags, shared, scale


@pytest.mark.parametrize("nnz", [1, 3])
def test_build_noise_weighted_vs_add_at(nnz):
    rng = np.random.default_rng(21)
    n_det, n_samp, nside = 5, 3000, 8
    npix = 12 * nside * nside
    nps = 16
    pixels, weights, tod, dflags, shared, scale = _random_inputs(rng, n_det, n_samp, npix, nnz)
    intervals = [(10, 900), (1000, 1000), (1200, 2999)]
    # permuted submap storage: global2local is a permutation
    g2l = rng.permutation(npix // nps).astype(np.int64)
    zmap = np.zeros((npix // nps, nps, nnz))
    oracle.build_noise_weighted(zmap, g2l, nps, pixels, weights, tod, scale, intervals, det_flags=dflags,
                                det_flag_mask=1, shared_flags=shared, shared_flag_mask=2)
    sel = np.zeros((n_det, n_samp), bool)
    for f, l in intervals:
        sel[:, f:l + 1] = True
    sel &= pixels >= 0
    sel &= (dflags & 1) == 0
    sel &= ((shared & 2) == 0)[None, :]
    ref = np.zeros((npix // nps, nps, nnz))
    dd, ss = np.nonzero(sel)
    p = pixels[dd, ss]
    np.add.at(ref, (g2l[p // nps], p % nps), (scale[dd] * tod[dd, ss])[:, None] * weights[dd, ss])
    np.testing.assert_allclose(zmap, ref, rtol=0, atol=1e-12)


def test_integer_inputs_give_hit_counts_exactly():
    rng = np.random.default_rng(22)
    n_det, n_samp, npix = 4, 5000, 192
    pixels = rng.integers(-1, npix, size=(n_det, n_samp)).astype(np.int64)
    weights = np.ones((n_det, n_samp, 1))
    zmap = np.zeros((12, 16, 1))
    oracle.build_noise_weighted(zmap, np.arange(12), 16, pixels, weights, np.ones((n_det, n_samp)), np.ones(n_det),
                                [(0, n_samp - 1)])
    counts = np.bincount(pixels[pixels >= 0], minlength=npix)
    np.testing.assert_array_equal(zmap.reshape(-1), counts.astype(float))


def test_scan_map_constant_map_and_modes():
    rng = np.random.default_rng(23)
    n_det, n_samp, nside = 3, 2000, 4
    npix = 12 * nside * nside
    pixels = rng.integers(-1, npix, size=(n_det, n_samp)).astype(np.int64)
    w = np.stack([np.full((n_det, n_samp), 1.3), rng.normal(size=(n_det, n_samp)), rng.normal(size=(n_det, n_samp))], -1)
    m = np.zeros((12, 16, 3)); m[..., 0] = 2.0
    intervals = [(5, 1500), (1600, 1999)]
    tod = np.full((n_det, n_samp), 7.0)
    oracle.scan_map(m, np.arange(12), 16, pixels, w, tod, intervals, data_scale=0.5, should_zero=True)
    inside = _mask_intervals(intervals, n_samp)[None, :] & (pixels >= 0)
    assert np.all(tod[inside] == 0.5 * 2.0 * 1.3)  # exact
    assert np.all(tod[~inside] == 7.0)            # untouched
    tod2 = np.full((n_det, n_samp), 1.0)
    oracle.scan_map(m, np.arange(12), 16, pixels, w, tod2, intervals, data_scale=1.0, should_subtract=True)
    assert np.all(tod2[inside] == 1.0 - 2.6)
    # map (0, 1, 0) scans the Q weight
    m2 = np.zeros((12, 16, 3)); m2[..., 1] = 1.0
    tod3 = np.zeros((n_det, n_samp))
    oracle.scan_map(m2, np.arange(12), 16, pixels, w, tod3, intervals)
    np.testing.assert_array_equal(tod3[inside], w[..., 1][inside])


def test_adjoint_identity():
    """<scan_map(m), t> = <m, build_noise_weighted(t; det_scale = 1)>."""
    rng = np.random.default_rng(24)
    n_det, n_samp, nside = 4, 4000, 8
    npix = 12 * nside * nside
    pixels = rng.integers(-1, npix, size=(n_det, n_samp)).astype(np.int64)
    w = rng.normal(size=(n_det, n_samp, 3))
    m = rng.normal(size=(48, 16, 3))
    t = rng.normal(size=(n_det, n_samp))
    intervals = [(0, 1999), (2500, 3999)]
    scanned = np.zeros((n_det, n_samp))
    oracle.scan_map(m, np.arange(48), 16, pixels, w, scanned, intervals)
    z = np.zeros_like(m)
    oracle.build_noise_weighted(z, np.arange(48), 16, pixels, w, t, np.ones(n_det), intervals)
    lhs = float(np.sum(scanned * t))
    rhs = float(np.sum(z * m))
    assert abs(lhs - rhs) <= 1e-12 * float(np.sum(np.abs(scanned * t)) + 1)


def test_fused_equals_composition(small):
    w = small
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    pix, hits = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                      w.shared_flag_mask)
    wts = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp)
    z1 = np.zeros((w.n_submap, w.n_pix_submap, 3))
    oracle.build_noise_weighted(z1, w.global2local, w.n_pix_submap, pix, wts, w.det_data, w.det_scale, w.intervals,
                                det_flags=w.det_flags, det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                                shared_flag_mask=w.shared_flag_mask)
    z2 = np.zeros_like(z1)
    hits2 = np.zeros(w.n_submap, np.uint8)
    pix2 = np.full((w.n_det, w.n_samp), -7, np.int64)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, zmap=z2, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, hit_submaps=hits2, pixels_out=pix2)
    np.testing.assert_array_equal(pix2, pix)
    np.testing.assert_array_equal(hits2, hits)
    np.testing.assert_array_equal(z2, z1)
    # global sum identity: sum of I map = cal * sum over good samples of det_scale * tod
    good = (pix >= 0) & ((w.det_flags & w.det_flag_mask) == 0)
    tot = np.sum((w.det_scale[:, None] * w.det_data)[good])
    assert abs(z2[..., 0].sum() - w.cal * tot) <= 1e-12 * np.sum(np.abs(w.det_scale[:, None] * w.det_data)[good])


def test_omp_mode_matches_sequential(small):
    w = small
    z1 = np.zeros((w.n_submap, w.n_pix_submap, 3))
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, zmap=z1, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask)
    z2 = np.zeros_like(z1)
    used = oracle.pointing_to_map_omp(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals,
                                      w.nside, w.nest, 3, w.global2local, w.n_pix_submap, z2, hwp=w.hwp,
                                      det_flags=w.det_flags, det_flag_mask=w.det_flag_mask,
                                      shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask, n_threads=2)
    assert used >= 1
    np.testing.assert_allclose(z2, z1, rtol=1e-12, atol=1e-12)


def test_pointing_to_tod_equals_composition_and_modes(small):
    """f1 pointing_to_tod == A1 -> A2 -> A3 -> A5 (oracle entries), for each tod mode."""
    w = small
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    pix, _ = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                   w.shared_flag_mask)
    wts = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp)
    rng = np.random.default_rng(71)
    m = rng.normal(size=(w.n_submap, w.n_pix_submap, 3))
    for zero, sub in ((False, False), (True, False), (False, True)):
        t1 = w.det_data.copy()
        oracle.scan_map(m, w.global2local, w.n_pix_submap, pix, wts, t1, w.intervals, data_scale=0.3,
                        should_zero=zero, should_subtract=sub)
        t2 = w.det_data.copy()
        oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                               w.global2local, w.n_pix_submap, m, t2, data_scale=0.3, should_zero=zero,
                               should_subtract=sub, hwp=w.hwp, shared_flags=w.shared_flags,
                               shared_flag_mask=w.shared_flag_mask)
        np.testing.assert_array_equal(t2, t1)


def test_pointing_to_tod_constant_map_and_adjoint(small):
    """Constant I map scans to data_scale * c * cal exactly; <scan(m), t> = <m, accumulate(t)>
    with det_scale = 1 and no det flags."""
    w = small
    m = np.zeros((w.n_submap, w.n_pix_submap, 3)); m[..., 0] = 1.75
    tod = np.full((w.n_det, w.n_samp), 9.0)
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                           w.global2local, w.n_pix_submap, m, tod, data_scale=2.0, should_zero=True, hwp=w.hwp,
                           shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask)
    inside = _mask_intervals(w.intervals, w.n_samp) & ((w.shared_flags & w.shared_flag_mask) == 0)
    assert np.all(tod[:, inside] == 2.0 * 1.75 * w.cal)
    assert np.all(tod[:, ~inside] == 9.0)
    rng = np.random.default_rng(72)
    m = rng.normal(size=(w.n_submap, w.n_pix_submap, 3))
    t = rng.normal(size=(w.n_det, w.n_samp))
    scanned = np.zeros((w.n_det, w.n_samp))
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                           w.global2local, w.n_pix_submap, m, scanned, hwp=w.hwp, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask)
    z = np.zeros_like(m)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, np.ones(w.n_det), t, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, zmap=z, hwp=w.hwp, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask)
    lhs, rhs = float(np.sum(scanned * t)), float(np.sum(z * m))
    assert abs(lhs - rhs) <= 1e-12 * (float(np.sum(np.abs(scanned * t))) + 1.0)


@pytest.mark.parametrize("variant", ["plain", "gamma_iau"])
def test_det_sample_probe_equals_fused_outputs(variant):
    """oracle.det_sample_probe (the one-by-one expectation of the full-size parity tests and the
    direction fed to the T1 classifier) is pinned to the fused oracle's debug outputs and to the
    A1 composition: pixel and weights element by element, direction == R(q_det) z with q_det
    from oracle.pointing_detector; shared-flagged samples give pixel -1."""
    w = synth.make_workload("c2", n_det=4, n_samp=300_000, nside=64)  # long enough for the 0x02 bursts
    gamma = np.linspace(-1.0, 1.0, w.n_det) if variant == "gamma_iau" else None
    iau = variant == "gamma_iau"
    smask = w.shared_flag_mask | 2  # the 0x02 bursts lie inside intervals: flagged in-interval samples
    pix = np.full((w.n_det, w.n_samp), -7, np.int64)
    wts = np.zeros((w.n_det, w.n_samp, 3))
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=smask, pixels_out=pix, weights_out=wts, gamma=gamma, iau=iau)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, smask)
    rng = np.random.default_rng(7)
    inside = np.nonzero(_mask_intervals(w.intervals, w.n_samp))[0]
    flagged_in = inside[(w.shared_flags[inside] & smask) != 0]
    samples = np.concatenate([rng.choice(inside, 400), flagged_in[:50]])
    n_flagged = 0
    for s in samples:
        d = int(rng.integers(w.n_det))
        fl = bool(w.shared_flags[s] & smask)
        p, wt, v = oracle.det_sample_probe(w.fp_quats[d], w.boresight[s], w.hwp[s], w.epsilon[d], w.cal, fl, w.nside,
                                           w.nest, gamma=0.0 if gamma is None else gamma[d], iau=iau)
        assert p == pix[d, s]
        np.testing.assert_array_equal(wt, wts[d, s])
        np.testing.assert_array_equal(v, oracle.quat_rotate(quats[d, s], [0.0, 0.0, 1.0]))
        if fl:
            assert p == -1
            n_flagged += 1
        else:
            assert p == oracle.vec2pix(w.nside, w.nest, v)
    assert n_flagged > 10


def test_fused_gamma_iau_equals_composition(small):
    """The fused oracle with the reading-R3 variant equals A1 -> A2 -> A3(gamma, IAU) -> A4."""
    w = small
    gamma = np.linspace(-0.7, 0.9, w.n_det)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    pix, _ = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                   w.shared_flag_mask)
    wts = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp, gamma=gamma, iau=True)
    wts_plain = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp)
    m = _mask_intervals(w.intervals, w.n_samp)
    assert np.abs(wts[:, m, 1:] - wts_plain[:, m, 1:]).max() > 0.1  # the variant changes Q/U
    z1 = np.zeros((w.n_submap, w.n_pix_submap, 3))
    oracle.build_noise_weighted(z1, w.global2local, w.n_pix_submap, pix, wts, w.det_data, w.det_scale, w.intervals,
                                det_flags=w.det_flags, det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                                shared_flag_mask=w.shared_flag_mask)
    z2 = oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals,
                                w.nside, w.nest, 3, w.global2local, w.n_pix_submap, hwp=w.hwp, det_flags=w.det_flags,
                                det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                                shared_flag_mask=w.shared_flag_mask, gamma=gamma, iau=True)
    np.testing.assert_array_equal(z2, z1)
