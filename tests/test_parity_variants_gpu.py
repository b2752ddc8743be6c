"""GPU parity, round 2: the fused round trip at full C3 size, map storage on the 64-bit key path
(nside > 4096) and with a non-power-of-two submap, the f4 variants (reading R3 gamma / IAU, fp32
maps), unwrapped HWP angles (reading R1), the dropped-sample counter and the
scan direction's should_zero on a NaN-filled timestream.  Every expectation comes from oracle/
on the same seeded inputs (rules T1-T4, tests/parity.py)."""
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from parity import check_map, check_weights, classify_pixel_mismatches, reconcile_map, t2_weight_tol  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200 import binding, synth  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload  # noqa: E402

pytestmark = pytest.mark.gpu

DEV = "cuda"


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    binding.load()


def _cuda(a, dtype):
    return torch.from_numpy(np.ascontiguousarray(a)).to(dtype).to(DEV)


def _in_mask(w):
    m = np.zeros(w.n_samp, bool)
    for f, l in w.intervals:
        m[f:l + 1] = True
    return m


def _probe_fn(w, gamma=None, iau=False):
    def probe(d, s):
        fl = w.shared_flags is not None and bool(w.shared_flags[s] & w.shared_flag_mask)
        return oracle.det_sample_probe(w.fp_quats[d], w.boresight[s], None if w.hwp is None else w.hwp[s],
                                       w.epsilon[d], w.cal, fl, w.nside, w.nest,
                                       gamma=0.0 if gamma is None else gamma[d], iau=iau)
    return probe


def _oracle_map(w, g2l=None, gamma=None, iau=False, tod=None):
    g2l = w.global2local if g2l is None else g2l
    n_loc = int(g2l.max()) + 1
    zo = np.zeros((n_loc, w.n_pix_submap, w.nnz)); am = np.zeros_like(zo); t2 = np.zeros_like(zo)
    po = np.full((w.n_det, w.n_samp), -7, np.int64)
    wo = np.zeros((w.n_det, w.n_samp, w.nnz))
    ho = np.zeros(w.n_submap, np.uint8)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale,
                           w.det_data if tod is None else tod, w.intervals, w.nside, w.nest, w.nnz, g2l,
                           w.n_pix_submap, zmap=zo, hwp=w.hwp, det_flags=w.det_flags, det_flag_mask=w.det_flag_mask,
                           shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask, hit_submaps=ho,
                           pixels_out=po, weights_out=wo, absmap=am, gamma=gamma, iau=iau, t2map=t2)
    return zo, am, t2, po, wo, ho


def _reconciled_check(gpu_map, ref, mism, pg, w, g2l, gamma=None, iau=False, rel=1e-10, extra=None):
    zo, am, t2, po, wo, _ = ref
    zo, am, t2 = zo.copy(), am.copy(), t2.copy()
    probe = _probe_fn(w, gamma, iau)
    reconcile_map(zo, am, mism, pg, po, wo, w, g2l, w.n_pix_submap, t2map=t2,
                  sin_theta=lambda d, s: float(np.hypot(*probe(d, s)[2][:2])))
    check_map(gpu_map, zo, am, t2, rel=rel, extra=extra)


def _compact_g2l(hits):
    g2l = np.full(len(hits), -1, np.int64)
    idx = np.nonzero(hits)[0]
    g2l[idx] = np.arange(len(idx))
    return g2l


# ----------------------------------------------------------------------------- map storage

@pytest.mark.parametrize("nside,nest,nps,n_samp", [(1 << 13, True, 512 * 512, 2000), (1 << 14, False, 4096, 2000),
                                                   (1 << 16, True, 4096, 400)])
def test_fused_storage_on_the_wide_key_path(nside, nest, nps, n_samp):
    """nside > 4096 (64-bit keys): real map storage over a compact global2local of the oracle's
    hit submaps (the cached global2local at 3072 submaps, the uncached one beyond 4096);
    production and debug instantiations, map T4, hit submaps exact."""
    w = synth.make_workload("c4", n_det=40, n_samp=n_samp, nside=nside, nest=nest)
    w.n_pix_submap = nps
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals)
    _, hits = oracle.pixels_healpix(quats, w.intervals, nside, nest, w.n_pix_submap)
    g2l = _compact_g2l(hits)
    assert 0 < int(hits.sum()) * nps * 24 < 1 << 30, int(hits.sum())  # a small compact map
    ref = _oracle_map(w, g2l)
    dw = DeviceWorkload.upload(w, DEV, alloc_map=False)
    dw.global2local = _cuda(g2l, torch.int64)
    dw.zmap = torch.zeros(ref[0].shape, dtype=torch.float64, device=DEV)
    dw.hit_submaps = torch.zeros(w.n_submap, dtype=torch.uint8, device=DEV)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g)
    torch.cuda.synchronize()
    pg = pix_g.cpu().numpy()
    n_in = int(_in_mask(w).sum()) * w.n_det
    mism = classify_pixel_mismatches(pg, ref[3], lambda d, s: _probe_fn(w)(d, s)[2], nside, nest, n_in)
    _reconciled_check(dw.zmap.cpu().numpy(), ref, mism, pg, w, g2l)
    dw.zmap.zero_(); dw.hit_submaps.zero_()
    dw.pointing_to_map()
    torch.cuda.synchronize()
    _reconciled_check(dw.zmap.cpu().numpy(), ref, mism, pg, w, g2l)
    if len(mism[0]) == 0:
        np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits)


@pytest.mark.parametrize("name,nside,nps", [("c2", 64, 768), ("c3", 256, 3 * 4096), ("c5", 1024, 3 * 256)])
def test_fused_non_power_of_two_submap(name, nside, nps):
    """n_pix_submap not a power of two: the division paths of the submap / pixel split."""
    w = synth.make_workload(name, n_det=40, n_samp=30_000, nside=nside)
    w.n_pix_submap = nps
    assert (12 * nside * nside) % nps == 0 and nps & (nps - 1) != 0
    ref = _oracle_map(w)
    dw = DeviceWorkload.upload(w, DEV)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g)
    torch.cuda.synchronize()
    pg = pix_g.cpu().numpy()
    mism = classify_pixel_mismatches(pg, ref[3], lambda d, s: _probe_fn(w)(d, s)[2], w.nside, w.nest,
                                     int(_in_mask(w).sum()) * w.n_det)
    _reconciled_check(dw.zmap.cpu().numpy(), ref, mism, pg, w, w.global2local)
    dw.zmap.zero_(); dw.hit_submaps.zero_()
    dw.pointing_to_map()
    torch.cuda.synchronize()
    _reconciled_check(dw.zmap.cpu().numpy(), ref, mism, pg, w, w.global2local)
    if len(mism[0]) == 0:
        np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), ref[5])


def test_dropped_sample_counter():
    """Hit submaps without storage (global2local = -1): their samples are skipped and counted
    (unflagged in-interval det-samples); everything else matches the oracle."""
    w = synth.make_workload("c2", n_det=24, n_samp=60_000, nside=128)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    po, hits = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                     w.shared_flag_mask)
    hit_idx = np.nonzero(hits)[0]
    assert len(hit_idx) >= 4
    g2l = np.arange(w.n_submap, dtype=np.int64)
    dropped_sm = hit_idx[::3]
    g2l[dropped_sm] = -1
    inside = _in_mask(w)[None, :]
    good = (po >= 0) & inside & ((w.det_flags & w.det_flag_mask) == 0)
    expect_dropped = int(np.isin(po // w.n_pix_submap, dropped_sm)[good].sum())
    assert expect_dropped > 0
    # oracle map on the kept submaps only: zero the TOD of the dropped samples (they add nothing)
    tod = w.det_data.copy()
    tod[np.isin(po // w.n_pix_submap, dropped_sm) & (po >= 0)] = 0.0
    g2l_full = np.arange(w.n_submap, dtype=np.int64)
    ref = _oracle_map(w, g2l_full, tod=tod)
    dw = DeviceWorkload.upload(w, DEV)
    dw.global2local = _cuda(g2l, torch.int64)
    cnt = torch.zeros(1, dtype=torch.int64, device=DEV)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g, dropped=cnt)
    torch.cuda.synchronize()
    pg = pix_g.cpu().numpy()
    if np.array_equal(pg, po):
        assert int(cnt.item()) == expect_dropped
    else:  # a near-boundary decision may move a sample across a dropped submap's edge
        classify_pixel_mismatches(pg, po, lambda d, s: _probe_fn(w)(d, s)[2], w.nside, w.nest, po.size)
        assert abs(int(cnt.item()) - expect_dropped) <= int((pg != po).sum())
    zg = dw.zmap.cpu().numpy()
    keep = g2l >= 0
    assert np.all(zg[~keep] == 0.0)
    mism = np.nonzero(pg != po)
    _reconciled_check(zg, ref, mism, pg, w, g2l_full)
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits)  # dropped submaps are still marked


# ----------------------------------------------------------------------------- f4 variants

@pytest.mark.parametrize("iau", [False, True])
def test_fused_gamma_iau(iau):
    """Reading R3: detector angle gamma with an HWP, and the IAU sign of U: debug weights (T2),
    the production map (T4), the scan direction (T3) and the unfused A3 entry."""
    w = synth.make_workload("c2", n_det=40, n_samp=80_000)
    gamma = np.linspace(-1.3, 1.1, w.n_det)
    ref = _oracle_map(w, gamma=gamma, iau=iau)
    zo, am, t2, po, wo, ho = ref
    dw = DeviceWorkload.upload(w, DEV)
    gg = _cuda(gamma, torch.float64)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    wts_g = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g, weights_out=wts_g, gamma=gg, iau=iau)
    torch.cuda.synchronize()
    pg = pix_g.cpu().numpy()
    mism = classify_pixel_mismatches(pg, po, lambda d, s: _probe_fn(w, gamma, iau)(d, s)[2], w.nside, w.nest,
                                     int(_in_mask(w).sum()) * w.n_det)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    sth = np.hypot(*_dirs_xy(quats))
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    mask = np.broadcast_to(_in_mask(w), (w.n_det, w.n_samp))
    check_weights(wts_g.cpu().numpy(), wo, sth, eta_cal, w.cal, mask)
    _reconciled_check(dw.zmap.cpu().numpy(), ref, mism, pg, w, w.global2local, gamma, iau)
    dw.zmap.zero_()
    dw.pointing_to_map(gamma=gg, iau=iau)
    torch.cuda.synchronize()
    _reconciled_check(dw.zmap.cpu().numpy(), ref, mism, pg, w, w.global2local, gamma, iau)
    # unfused A3 _ex
    wa = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    binding.stokes_weights_iqu(_cuda(quats, torch.float64), w.intervals, dw.epsilon, w.cal, wa, hwp=dw.hwp, gamma=gg,
                               iau=iau)
    wref = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp, gamma=gamma, iau=iau)
    check_weights(wa.cpu().numpy(), wref, sth, eta_cal, w.cal, mask)
    # scan direction
    rng = np.random.default_rng(5)
    m = rng.normal(size=(w.n_submap, w.n_pix_submap, 3))
    ref_tod = w.det_data.copy(); b = np.zeros_like(ref_tod)
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                           w.global2local, w.n_pix_submap, m, ref_tod, hwp=w.hwp, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, bscale=b, gamma=gamma, iau=iau)
    tg = dw.det_data.clone()
    binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                            dw.global2local, w.n_pix_submap, _cuda(m, torch.float64), tg, hwp=dw.hwp,
                            shared_flags=dw.shared_flags, shared_flag_mask=w.shared_flag_mask, gamma=gg, iau=iau)
    got = tg.cpu().numpy()
    tol = 1e-12 * b + 2 * np.abs(m).max() * t2_weight_tol(sth, eta_cal[:, None]) + 4e-16 * np.abs(ref_tod)
    bad = np.nonzero(np.abs(got - ref_tod) > tol)
    for d, s in zip(*bad):
        assert oracle.near_boundary(w.nside, w.nest, _probe_fn(w, gamma, iau)(int(d), int(s))[2])
    assert len(bad[0]) <= 1e-6 * got.size + 2


def _dirs_xy(quats):
    """(x, y) of R(q) z for an array of quaternions (the sin(theta) of each det-sample)."""
    x, y, z, ww = quats[..., 0], quats[..., 1], quats[..., 2], quats[..., 3]
    return 2.0 * (x * z + y * ww), 2.0 * (y * z - x * ww)


def test_unwrapped_hwp_angle():
    """Reading R1: an unwrapped HWP angle (chi ~ 1e6 - 1e7 rad: a 2 Hz HWP over days) gives the
    oracle's weights to T2 (the oracle evaluates the exact angle) in the fused kernel (both
    sincos paths of the per-sample state) and in the unfused A3."""
    w = synth.make_workload("c2", n_det=12, n_samp=40_000)
    w.hwp = w.hwp + 2 * np.pi * np.where(np.arange(w.n_samp) < w.n_samp // 2, 1.7e5, 1.9e6)  # both reduction paths
    ref = _oracle_map(w)
    dw = DeviceWorkload.upload(w, DEV)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    wts_g = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g, weights_out=wts_g)
    torch.cuda.synchronize()
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    sth = np.hypot(*_dirs_xy(quats))
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    mask = np.broadcast_to(_in_mask(w), (w.n_det, w.n_samp))
    check_weights(wts_g.cpu().numpy(), ref[4], sth, eta_cal, w.cal, mask)
    wa = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    binding.stokes_weights_iqu(_cuda(quats, torch.float64), w.intervals, dw.epsilon, w.cal, wa, hwp=dw.hwp)
    check_weights(wa.cpu().numpy(), ref[4], sth, eta_cal, w.cal, mask)


def test_fused_fp32_map():
    """map_f32: fp64 arithmetic, run sums rounded to fp32 once and accumulated with fp32 atomics.
    Bound: each of the n (<= hits) fp32 additions into an element errs by <= 2^-24 of the
    running |sum| <= A, and each run sum by 2^-24 of itself: |d| <= (2 n + 1) 2^-24 A + T4.
    The scan direction reads the fp32 map exactly (T3 against the oracle fed the same fp32
    values widened to fp64)."""
    w = synth.make_workload("c3", n_det=64, n_samp=30_000)
    ref = _oracle_map(w)
    zo, am, t2, po, wo, ho = ref
    dw = DeviceWorkload.upload(w, DEV)
    z32 = torch.zeros(zo.shape, dtype=torch.float32, device=DEV)
    dw.pointing_to_map(zmap=z32)
    torch.cuda.synchronize()
    good = (po >= 0) & _in_mask(w)[None, :]
    hits = np.bincount(po[good], minlength=w.npix).reshape(zo.shape[:2])[..., None].astype(np.float64)
    extra = (2 * hits + 1) * 2.0 ** -24 * am
    check_map(z32.cpu().numpy().astype(np.float64), zo, am, t2, extra=extra)
    # scan from the fp32 map
    m32 = torch.randn(zo.shape, dtype=torch.float32, device=DEV, generator=torch.Generator(DEV).manual_seed(3))
    m64 = m32.cpu().numpy().astype(np.float64)
    ref_tod = np.zeros((w.n_det, w.n_samp)); b = np.zeros_like(ref_tod)
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                           w.global2local, w.n_pix_submap, m64, ref_tod, should_zero=True,
                           shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask, bscale=b)
    tg = torch.zeros((w.n_det, w.n_samp), dtype=torch.float64, device=DEV)
    binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                            dw.global2local, w.n_pix_submap, m32, tg, should_zero=True, shared_flags=dw.shared_flags,
                            shared_flag_mask=w.shared_flag_mask)
    got = tg.cpu().numpy()
    tol = 1e-12 * b + 2 * float(np.abs(m64).max()) * 1e-12 + 4e-16 * np.abs(ref_tod)
    bad = np.nonzero(np.abs(got - ref_tod) > tol)
    for d, s in zip(*bad):
        assert oracle.near_boundary(w.nside, w.nest, _probe_fn(w)(int(d), int(s))[2])
    assert len(bad[0]) <= 1e-6 * got.size + 2


# ----------------------------------------------------------------------------- scan direction

def test_scan_should_zero_overwrites_nan():
    """should_zero overwrites the old value (never reads it): a NaN-filled timestream gives the
    oracle's scan on every scanned sample and stays NaN elsewhere."""
    w = synth.make_workload("c2", n_det=40, n_samp=40_000)
    rng = np.random.default_rng(9)
    m = rng.normal(size=(w.n_submap, w.n_pix_submap, 3))
    ref = np.full((w.n_det, w.n_samp), np.nan); b = np.zeros_like(ref)
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                           w.global2local, w.n_pix_submap, m, ref, should_zero=True, hwp=w.hwp,
                           shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask, bscale=b)
    dw = DeviceWorkload.upload(w, DEV)
    tg = torch.full((w.n_det, w.n_samp), float("nan"), dtype=torch.float64, device=DEV)
    binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                            dw.global2local, w.n_pix_submap, _cuda(m, torch.float64), tg, should_zero=True,
                            hwp=dw.hwp, shared_flags=dw.shared_flags, shared_flag_mask=w.shared_flag_mask)
    got = tg.cpu().numpy()
    np.testing.assert_array_equal(np.isnan(got), np.isnan(ref))
    fin = ~np.isnan(ref)
    assert fin.sum() > 0.5 * got.size
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    tol = 1e-12 * b + 2 * np.abs(m).max() * t2_weight_tol(np.hypot(*_dirs_xy(quats)), eta_cal[:, None])
    bad = np.nonzero(fin & (np.abs(got - ref) > tol))
    for d, s in zip(*bad):
        assert oracle.near_boundary(w.nside, w.nest, _probe_fn(w)(int(d), int(s))[2])
    assert len(bad[0]) <= 1e-6 * got.size + 2


# ----------------------------------------------------------------------------- fused round trip, full C3

@pytest.mark.slow
def test_fused_round_trip_full_c3():
    """C3 at full size (1024 dets x 60k samples, nside 1024 RING): f1 pointing_to_tod scans a
    smooth map into a timestream, A6 pointing_to_map (production instantiation) accumulates it
    back — against oracle.pointing_to_tod -> oracle.pointing_to_map on the same inputs."""
    from independent import ring_centres
    w = synth.make_workload("c3", with_tod=False)
    w.gen_det_flags()
    z, ph = ring_centres(w.nside)
    st = np.sqrt(1 - z * z)
    m = np.stack([np.cos(3 * np.arccos(z)), np.sin(2 * ph) * st, np.cos(ph) * st], -1)
    m = np.ascontiguousarray(m.reshape(w.n_submap, w.n_pix_submap, 3))
    # oracle: scan then accumulate
    tod = np.zeros((w.n_det, w.n_samp)); bsc = np.zeros_like(tod)
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                           w.global2local, w.n_pix_submap, m, tod, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, bscale=bsc)
    w.det_data = tod
    ref = _oracle_map(w)
    zo, am, t2, po, wo, ho = ref
    # GPU: the same two fused calls
    dw = DeviceWorkload.upload(w, DEV, det_data=torch.zeros((w.n_det, w.n_samp), dtype=torch.float64, device=DEV))
    binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, w.intervals, w.nside, w.nest, 3,
                            dw.global2local, w.n_pix_submap, _cuda(m, torch.float64), dw.det_data,
                            shared_flags=dw.shared_flags, shared_flag_mask=w.shared_flag_mask)
    dw.pointing_to_map()
    torch.cuda.synchronize()
    assert binding.last_fused_path() == "tma"
    got_tod = dw.det_data.cpu().numpy()
    # pixel decisions of this kernel (debug instantiation, same arithmetic)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    dw.pointing_to_map(zmap=torch.zeros_like(dw.zmap), pixels_out=pix_g)
    torch.cuda.synchronize()
    pg = pix_g.cpu().numpy()
    del pix_g
    n_in = int(_in_mask(w).sum()) * w.n_det
    mism = classify_pixel_mismatches(pg, po, lambda d, s: _probe_fn(w)(d, s)[2], w.nside, w.nest, n_in)
    # timestream: T3 (+ the T2 weight tolerance through |m_Q|, |m_U| <= 1); the scan at a
    # reconciled sample uses the GPU's (admissible) pixel
    eta_max = float(np.max((1 - w.epsilon) / (1 + w.epsilon))) * w.cal
    z_max = np.max(np.abs(z[np.unique(po[po >= 0])]))
    t2 = eta_max * max(1e-12, 1e-15 / math.sqrt(1 - z_max * z_max))
    tod_r = tod.copy()
    for d, s in zip(*mism):
        p = pg[d, s]
        tod_r[d, s] = float(np.dot(m[p // w.n_pix_submap, p % w.n_pix_submap], wo[d, s]))
    tol_tod = 1e-12 * np.maximum(bsc, np.abs(tod_r)) + 2 * t2 + 4e-16 * np.abs(tod_r)
    assert np.all(np.abs(got_tod - tod_r) <= tol_tod), float(np.max(np.abs(got_tod - tod_r) - tol_tod))
    # map: T4 + what the tolerated timestream differences carry (|w_k| <= cal)
    good = (po >= 0) & _in_mask(w)[None, :]
    if w.det_flags is not None:
        good &= (w.det_flags & w.det_flag_mask) == 0
    extra = np.zeros(w.npix)
    np.add.at(extra, po[good], (w.det_scale[:, None] * tol_tod)[good] * abs(w.cal))
    extra = np.repeat(extra.reshape(w.n_submap, w.n_pix_submap, 1), 3, axis=2)
    w.det_data = tod_r
    ref_r = _oracle_map(w)
    for d, s in zip(*mism):  # the tolerance of a moved sample follows it
        extra[pg[d, s] // w.n_pix_submap, pg[d, s] % w.n_pix_submap] += w.det_scale[d] * tol_tod[d, s] * abs(w.cal)
    _reconciled_check(dw.zmap.cpu().numpy(), ref_r, mism, pg, w, w.global2local, extra=extra)
