"""GPU parity: every C-ABI entry vs the CPU oracle on the same seeded inputs (rules T1-T4).

Runs on a B200 through paper_conf_sc_demeurekktbb23_b200.binding (ctypes -> libtoastb200.so).
Sizes span many 256-sample chunks, ragged interval tails, ragged detector blocks (n_det not a
multiple of 32), both orderings, nnz 1 and 3, HWP, flags, index arrays and extreme nside.
"""
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from parity import check_map, check_weights, classify_pixel_mismatches, reconcile_map  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200 import binding, synth  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload  # noqa: E402

pytestmark = pytest.mark.gpu

DEV = "cuda"


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    binding.load()


def _in_mask(intervals, n_det, n_samp):
    m = np.zeros(n_samp, bool)
    for f, l in intervals:
        m[f:l + 1] = True
    return np.broadcast_to(m, (n_det, n_samp))


def _sin_theta(quats):
    x, y = quats[..., 0], quats[..., 1]
    a = x * x + y * y
    return 2.0 * np.sqrt(np.clip(a * (1.0 - a), 0, None))


def _oracle_fused(w, gamma=None, iau=False):
    zmap = np.zeros((w.n_submap, w.n_pix_submap, w.nnz))
    absmap = np.zeros_like(zmap)
    t2map = np.zeros_like(zmap)
    hits = np.zeros(w.n_submap, np.uint8)
    pix = np.full((w.n_det, w.n_samp), -7, np.int64)
    wts = np.zeros((w.n_det, w.n_samp, w.nnz))
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, w.nnz, w.global2local, w.n_pix_submap, zmap=zmap, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, hit_submaps=hits, pixels_out=pix, weights_out=wts,
                           absmap=absmap, gamma=gamma, iau=iau, t2map=t2map)
    return zmap, absmap, hits, pix, wts, t2map


def _probe(w, gamma=None, iau=False):
    def probe(d, s):
        flagged = w.shared_flags is not None and bool(w.shared_flags[s] & w.shared_flag_mask)
        _, _, v = oracle.det_sample_probe(w.fp_quats[d], w.boresight[s], None if w.hwp is None else w.hwp[s],
                                          w.epsilon[d], w.cal, flagged, w.nside, w.nest,
                                          gamma=0.0 if gamma is None else gamma[d], iau=iau)
        return v
    return probe


def _sin_theta_of(w):
    probe = _probe(w)

    def sth(d, s):
        v = probe(d, s)
        return float(np.hypot(v[0], v[1]))
    return sth


def _check_fused_map(gpu_map, ref, mism, pg, w):
    """T4 of a fused map against the oracle's, the near-boundary decisions reconciled."""
    zo, absmap, _, po, wo, t2map = ref
    zo_r, abs_r = zo.copy(), absmap.copy()
    t2_r = t2map.copy()
    reconcile_map(zo_r, abs_r, mism, pg, po, wo, w, w.global2local, w.n_pix_submap, t2map=t2_r,
                  sin_theta=_sin_theta_of(w))
    check_map(gpu_map, zo_r, abs_r, t2_r)


FUSED_CASES = {
    "c1_full": dict(name="c1"),
    "c2_hwp_flags_nest": dict(name="c2", n_det=16, n_samp=200_000),
    "c2_nnz1": dict(name="c2", n_det=8, n_samp=120_000, nnz=1),
    "c3_ring_ragged_dets": dict(name="c3", n_det=40, n_samp=60_000),
    "c4_sat_nest_2048": dict(name="c4", n_det=36, n_samp=40_000),
    "c5_nest_4096": dict(name="c5", n_det=24, n_samp=133_200),
    "c1_ring_nest_swap": dict(name="c1", n_samp=50_000, nest=True, nside=128),
    # n_samp % 16 != 0: the cp.async staging path instead of the TMA path
    "c2_cp_async_path": dict(name="c2", n_det=40, n_samp=100_003),
}


@pytest.mark.parametrize("case", list(FUSED_CASES))
def test_fused_pointing_to_map(case):
    w = synth.make_workload(**FUSED_CASES[case])
    ref = _oracle_fused(w)
    zo, absmap, ho, po, wo, t2map = ref
    dw = DeviceWorkload.upload(w, DEV)
    n_in = int(_in_mask(w.intervals, 1, w.n_samp).sum()) * w.n_det

    # debug variant: materialised pixels / weights
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    wts_g = torch.zeros((w.n_det, w.n_samp, w.nnz), dtype=torch.float64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g, weights_out=wts_g)
    torch.cuda.synchronize()
    pg, wg = pix_g.cpu().numpy(), wts_g.cpu().numpy()
    mism = classify_pixel_mismatches(pg, po, _probe(w), w.nside, w.nest, n_in)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    mask = np.array(_in_mask(w.intervals, w.n_det, w.n_samp))
    check_weights(wg, wo, _sin_theta(quats), eta_cal, w.cal, mask)
    _check_fused_map(dw.zmap.cpu().numpy(), ref, mism, pg, w)
    hits_expect = np.zeros(w.n_submap, np.uint8)
    good = pg[pg >= 0]
    hits_expect[np.unique(good // w.n_pix_submap)] = 1
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits_expect)
    if len(mism[0]) == 0:
        np.testing.assert_array_equal(hits_expect, ho)

    # production variant (no debug outputs): the instantiation bench.py times
    dw.zmap.zero_()
    dw.hit_submaps.zero_()
    dw.pointing_to_map()
    torch.cuda.synchronize()
    _check_fused_map(dw.zmap.cpu().numpy(), ref, mism, pg, w)
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits_expect)


def test_fused_tma_and_cp_async_paths():
    """The same workload staged by TMA (aligned TOD) and by cp.async (TOD base only 8-byte
    aligned, so the TMA constraints fail) gives the oracle's map either way."""
    w = synth.make_workload("c2", n_det=36, n_samp=64_000)
    ref = _oracle_fused(w)
    po = ref[3]
    buf = torch.empty(w.n_det * w.n_samp + 1, dtype=torch.float64, device=DEV)
    odd = buf[1:].view(w.n_det, w.n_samp)
    odd.copy_(torch.from_numpy(np.ascontiguousarray(w.det_data)))
    assert odd.data_ptr() % 16 == 8
    for det_data, path in ((None, "tma"), (odd, "cp.async")):
        dw = DeviceWorkload.upload(w, DEV, det_data=det_data)
        pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
        dw.pointing_to_map(pixels_out=pix_g)
        torch.cuda.synchronize()
        assert binding.last_fused_path().startswith(path), binding.last_fused_path()
        pg = pix_g.cpu().numpy()
        n_in = int(_in_mask(w.intervals, 1, w.n_samp).sum()) * w.n_det
        mism = classify_pixel_mismatches(pg, po, _probe(w), w.nside, w.nest, n_in)
        _check_fused_map(dw.zmap.cpu().numpy(), ref, mism, pg, w)
        # production instantiation on the same staging path
        dw.zmap.zero_()
        dw.pointing_to_map()
        torch.cuda.synchronize()
        assert binding.last_fused_path().startswith(path), binding.last_fused_path()
        _check_fused_map(dw.zmap.cpu().numpy(), ref, mism, pg, w)


def test_fused_integer_inputs_give_exact_hit_counts():
    """tod = 1, det_scale = 1, cal = 1, nnz = 1: the I map is the hit count, bit-exact under
    any atomic order."""
    w = synth.make_workload("c2", n_det=20, n_samp=150_000, nnz=1)
    w.det_data = np.ones_like(w.det_data)
    w.det_scale = np.ones_like(w.det_scale)
    zo, absmap, ho, po, wo, _ = _oracle_fused(w)
    dw = DeviceWorkload.upload(w, DEV)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g)
    pg = pix_g.cpu().numpy()
    good = (pg >= 0) & ((w.det_flags & w.det_flag_mask) == 0)
    counts = np.bincount(pg[good], minlength=w.npix).astype(np.float64)
    np.testing.assert_array_equal(dw.zmap.cpu().numpy().reshape(-1), counts)
    if np.array_equal(pg, po):
        np.testing.assert_array_equal(dw.zmap.cpu().numpy(), zo)


@pytest.mark.parametrize("nside,nest", [(1, False), (1, True), (2, True), (1 << 16, False), (1 << 29, True),
                                        (1 << 29, False)])
def test_fused_extreme_nside(nside, nest):
    w = synth.make_workload("c1", n_samp=20_000, nside=nside, nest=nest, nnz=1)
    w.n_pix_submap = 1 if nside <= 16 else (nside // 16) ** 2
    n_in = int(_in_mask(w.intervals, 1, w.n_samp).sum()) * w.n_det
    dw = DeviceWorkload.upload(w, DEV, alloc_map=False)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    if nside >= (1 << 16):
        # a full-sky map is too large: no submap has storage (global2local = -1), so only
        # pixels and hit submaps are produced and checked
        quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals)
        po, hits = oracle.pixels_healpix(quats, w.intervals, nside, nest, w.n_pix_submap)
        dw.global2local = torch.full((w.n_submap,), -1, dtype=torch.int64, device=DEV)
        dw.zmap = torch.zeros((1, 1, 1), dtype=torch.float64, device=DEV)
        dw.pointing_to_map(pixels_out=pix_g)
        classify_pixel_mismatches(pix_g.cpu().numpy(), po, _probe(w), nside, nest, n_in)
        np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits)
        assert np.all(dw.zmap.cpu().numpy() == 0)
        return
    ref = _oracle_fused(w)
    dw.zmap = torch.zeros(ref[0].shape, dtype=torch.float64, device=DEV)
    dw.hit_submaps = torch.zeros(w.n_submap, dtype=torch.uint8, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g)
    pg = pix_g.cpu().numpy()
    mism = classify_pixel_mismatches(pg, ref[3], _probe(w), nside, nest, n_in)
    _check_fused_map(dw.zmap.cpu().numpy(), ref, mism, pg, w)


@pytest.mark.parametrize("name,n_det", [("c1", 4), ("c2", 40)])  # thread path and warp path
def test_fused_production_wide_and_many_submaps(name, n_det):
    """Production calls (no debug outputs) on the paths the tests above reach only with debug
    outputs: 64-bit keys (nside 2^16, hit submaps only) and more than 8192 submaps (the hit flags
    then go straight to global memory instead of the CTA's shared copy)."""
    # nside 2^16: no storage, the hit submaps against the oracle's A2
    w = synth.make_workload(name, n_det=n_det, n_samp=20_000, nside=1 << 16, nest=True)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    _, hits = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                    w.shared_flag_mask)
    dw = DeviceWorkload.upload(w, DEV, alloc_map=False)
    dw.global2local = torch.full((w.n_submap,), -1, dtype=torch.int64, device=DEV)
    dw.pointing_to_map()
    torch.cuda.synchronize()
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits)
    # nside 64 with 4-pixel submaps: 12288 submaps
    w = synth.make_workload(name, n_det=n_det, n_samp=20_000, nside=64)
    w.n_pix_submap = 4
    zo, absmap, ho, po, wo, t2map = _oracle_fused(w)
    dw = DeviceWorkload.upload(w, DEV, alloc_map=False)
    dw.zmap = torch.zeros(zo.shape, dtype=torch.float64, device=DEV)
    dw.hit_submaps = torch.zeros(w.n_submap, dtype=torch.uint8, device=DEV)
    assert w.n_submap > 8192
    dw.pointing_to_map()
    torch.cuda.synchronize()
    check_map(dw.zmap.cpu().numpy(), zo, absmap, t2map)
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), ho)


@pytest.mark.parametrize("n_samp", [5000, 5008])  # cp.async path (n_samp % 16 != 0) and TMA path
def test_fused_edge_intervals(n_samp):
    """Empty interval list, single-sample intervals, chunk-boundary lengths (255/256/257),
    odd first samples (the TMA box then starts one sample earlier), the last sample."""
    w = synth.make_workload("c1", n_samp=n_samp)
    last = n_samp - 1
    for ivs in ([], [(0, 0)], [(0, 254), (300, 555), (600, 856), (last, last)], [(10, 10), (11, 11), (12, 4000)],
                [(1, 1), (3, 17), (33, 160), (161, 290), (4001, last)], [(last - 16, last)]):
        w.intervals = ivs
        zo, absmap, ho, po, wo, t2map = _oracle_fused(w)
        dw = DeviceWorkload.upload(w, DEV)
        pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
        dw.pointing_to_map(pixels_out=pix_g)
        np.testing.assert_array_equal(pix_g.cpu().numpy(), po)  # includes untouched -7 outside intervals
        check_map(dw.zmap.cpu().numpy(), zo, absmap, t2map)
        np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), ho)


def test_fused_global2local_permuted():
    w = synth.make_workload("c1", n_samp=30_000)
    rng = np.random.default_rng(3)
    perm = rng.permutation(w.n_submap).astype(np.int64)
    zo = np.zeros((w.n_submap, w.n_pix_submap, 3)); absmap = np.zeros_like(zo); t2map = np.zeros_like(zo)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, perm, w.n_pix_submap, zmap=zo, absmap=absmap, t2map=t2map)
    dw = DeviceWorkload.upload(w, DEV)
    dw.global2local = torch.from_numpy(perm).to(DEV)
    dw.pointing_to_map()
    check_map(dw.zmap.cpu().numpy(), zo, absmap, t2map)


def test_fused_compact_map_domain():
    """f3 on the GPU: the hit submaps of a first pass define a compact (hit-submap-only)
    global2local; the fused kernel accumulating into the compact map gives the oracle's dense
    map on every hit submap (bench.py --reduce scatter runs exactly this)."""
    from paper_conf_sc_demeurekktbb23_b200 import dist as tdist
    w = synth.make_workload("c5", n_det=40, n_samp=40_000)
    zo, absmap, ho, po, wo, t2map = _oracle_fused(w)
    dw = DeviceWorkload.upload(w, DEV)
    dw.pointing_to_map()
    g2l, n_hit = tdist.compact_global2local(dw.hit_submaps)
    assert 0 < n_hit < w.n_submap
    own = tdist.MapOwnership.make(n_hit, 1)
    zc = tdist.alloc_compact_map(own, w.n_pix_submap, w.nnz, DEV)
    dw.global2local = g2l
    dw.hit_submaps.zero_()
    dw.pointing_to_map(zmap=zc)
    torch.cuda.synchronize()
    hit = np.nonzero(ho)[0]
    np.testing.assert_array_equal(np.nonzero(dw.hit_submaps.cpu().numpy())[0], hit)
    check_map(zc[:n_hit].cpu().numpy(), zo[hit], absmap[hit], t2map[hit])
    full = tdist.gather_map(zc[:own.per_rank], own, g2l, w.n_submap)
    check_map(full.cpu().numpy(), zo, absmap, t2map)


@pytest.mark.parametrize("dets", [(0, 0), (5, 6), (0, 7), (0, 8), (0, 33)])
def test_fused_detector_counts(dets):
    """No detector (a no-op), one and seven detectors (the thread-per-(chunk, detector) path), eight
    (the warp path with 24 idle lanes), one full warp group plus a one-detector group."""
    w = synth.make_workload("c2", n_det=64, n_samp=30_000, det_range=dets)
    zo, absmap, ho, po, wo, t2map = _oracle_fused(w)
    dw = DeviceWorkload.upload(w, DEV)
    dw.pointing_to_map()
    torch.cuda.synchronize()
    check_map(dw.zmap.cpu().numpy(), zo, absmap, t2map)
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), ho)


# ----------------------------------------------------------------------------- unfused entries

@pytest.fixture(scope="module")
def chain():
    """Oracle A1 -> A2 -> A3 intermediates on a ground scan with HWP and flags."""
    w = synth.make_workload("c2", n_det=12, n_samp=80_000, nside=512)
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    pix, hits = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                      w.shared_flag_mask)
    wts = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp)
    return w, quats, pix, hits, wts


def _cuda(a, dtype):
    return torch.from_numpy(np.ascontiguousarray(a)).to(dtype).to(DEV)


def test_pointing_detector(chain):
    w, quats, *_ = chain
    q = torch.zeros((w.n_det, w.n_samp, 4), dtype=torch.float64, device=DEV)
    binding.pointing_detector(_cuda(w.fp_quats, torch.float64), _cuda(w.boresight, torch.float64), w.intervals, q,
                              shared_flags=_cuda(w.shared_flags, torch.uint8), shared_flag_mask=w.shared_flag_mask)
    np.testing.assert_allclose(q.cpu().numpy(), quats, rtol=0, atol=4e-16)


def test_pointing_detector_quat_index():
    w = synth.make_workload("c1", n_det=4, n_samp=3000)
    qi = np.array([5, 0, 3, 1], np.int32)
    ref = np.zeros((6, w.n_samp, 4))
    oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, quat_index=qi, quats=ref)
    q = torch.zeros((6, w.n_samp, 4), dtype=torch.float64, device=DEV)
    binding.pointing_detector(_cuda(w.fp_quats, torch.float64), _cuda(w.boresight, torch.float64), w.intervals, q,
                              quat_index=_cuda(qi, torch.int32))
    np.testing.assert_allclose(q.cpu().numpy(), ref, rtol=0, atol=4e-16)


def test_pixels_healpix(chain):
    w, quats, pix, hits, _ = chain
    pg = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    hg = torch.zeros(w.n_submap, dtype=torch.uint8, device=DEV)
    binding.pixels_healpix(_cuda(quats, torch.float64), w.intervals, w.nside, w.nest, w.n_pix_submap, pg,
                           hit_submaps=hg, shared_flags=_cuda(w.shared_flags, torch.uint8),
                           shared_flag_mask=w.shared_flag_mask)
    n_in = int(_in_mask(w.intervals, 1, w.n_samp).sum()) * w.n_det

    def probe(d, s):
        return oracle.quat_rotate(quats[d, s], [0, 0, 1.0])
    mism = classify_pixel_mismatches(pg.cpu().numpy(), pix, probe, w.nside, w.nest, n_in)
    if len(mism[0]) == 0:
        np.testing.assert_array_equal(hg.cpu().numpy(), hits)


@pytest.mark.parametrize("nest", [False, True])
def test_pixels_healpix_random_directions_and_index(nest):
    """Uniform random unit quaternions at several nside, written through a pixel_index map."""
    rng = np.random.default_rng(31 + nest)
    n_det, n_samp = 3, 40_000
    q = rng.normal(size=(n_det, n_samp, 4))
    q /= np.linalg.norm(q, axis=-1, keepdims=True)
    ivs = [(0, n_samp - 1)]
    pidx = np.array([2, 0, 1], np.int32)
    for nside in (1, 8, 1024, 1 << 13, 1 << 20):
        nps = 1 if nside < 16 else (nside // 16) ** 2
        ref = np.full((n_det, n_samp), -7, np.int64)
        oracle.pixels_healpix(q, ivs, nside, nest, nps, pixel_index=pidx, pixels=ref)
        pg = torch.full((n_det, n_samp), -7, dtype=torch.int64, device=DEV)
        binding.pixels_healpix(_cuda(q, torch.float64), ivs, nside, nest, nps, pg,
                               pixel_index=_cuda(pidx, torch.int32))
        inv = np.argsort(pidx)

        def probe(r, s, inv=inv):
            return oracle.quat_rotate(q[inv[r], s], [0, 0, 1.0])
        classify_pixel_mismatches(pg.cpu().numpy(), ref, probe, nside, nest, n_det * n_samp)


def test_stokes_weights(chain):
    w, quats, _, _, wts = chain
    wg = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    binding.stokes_weights_iqu(_cuda(quats, torch.float64), w.intervals, _cuda(w.epsilon, torch.float64), w.cal, wg,
                               hwp=_cuda(w.hwp, torch.float64))
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    check_weights(wg.cpu().numpy(), wts, _sin_theta(quats), eta_cal, w.cal,
                  np.array(_in_mask(w.intervals, w.n_det, w.n_samp)))
    out = ~np.array(_in_mask(w.intervals, w.n_det, w.n_samp))
    assert np.all(wg.cpu().numpy()[out] == 0.0)


def test_stokes_weights_random_quats_no_hwp():
    rng = np.random.default_rng(41)
    q = rng.normal(size=(2, 30_000, 4))
    q /= np.linalg.norm(q, axis=-1, keepdims=True)
    eps = np.array([0.0, 0.2])
    ref = oracle.stokes_weights_iqu(q, [(0, 29_999)], eps, 1.3)
    wg = torch.zeros((2, 30_000, 3), dtype=torch.float64, device=DEV)
    binding.stokes_weights_iqu(_cuda(q, torch.float64), [(0, 29_999)], _cuda(eps, torch.float64), 1.3, wg)
    check_weights(wg.cpu().numpy(), ref, _sin_theta(q), (1 - eps) / (1 + eps) * 1.3, 1.3, np.ones((2, 30_000), bool))


@pytest.mark.parametrize("nnz", [1, 3])
def test_build_noise_weighted(chain, nnz):
    w, quats, pix, hits, wts = chain
    wn = np.ascontiguousarray(wts[..., :nnz])
    ref = np.zeros((w.n_submap, w.n_pix_submap, nnz)); absmap = np.zeros_like(ref)
    oracle.build_noise_weighted(ref, w.global2local, w.n_pix_submap, pix, wn, w.det_data, w.det_scale, w.intervals,
                                det_flags=w.det_flags, det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                                shared_flag_mask=w.shared_flag_mask, absmap=absmap)
    zg = torch.zeros(ref.shape, dtype=torch.float64, device=DEV)
    binding.build_noise_weighted(zg, _cuda(w.global2local, torch.int64), w.n_pix_submap, _cuda(pix, torch.int64),
                                 _cuda(wn, torch.float64), _cuda(w.det_data, torch.float64),
                                 _cuda(w.det_scale, torch.float64), w.intervals,
                                 det_flags=_cuda(w.det_flags, torch.uint8), det_flag_mask=w.det_flag_mask,
                                 shared_flags=_cuda(w.shared_flags, torch.uint8), shared_flag_mask=w.shared_flag_mask)
    check_map(zg.cpu().numpy(), ref, absmap)


def test_build_noise_weighted_index_arrays_and_random_pixels():
    rng = np.random.default_rng(51)
    n_det, n_samp, npix, nps = 5, 20_000, 12 * 64 * 64, 256
    pixels = rng.integers(-1, npix, size=(7, n_samp)).astype(np.int64)
    weights = rng.normal(size=(6, n_samp, 3))
    tod = rng.normal(size=(8, n_samp))
    flags = (rng.random((5, n_samp)) < 0.05).astype(np.uint8) * 4
    scale = rng.uniform(0.5, 2, n_det)
    pidx, widx, didx, fidx = (np.array(a, np.int32) for a in ([6, 0, 2, 3, 1], [5, 4, 0, 1, 2], [7, 1, 2, 0, 4],
                                                              [4, 3, 2, 1, 0]))
    ivs = [(3, 9000), (9500, 19_999)]
    g2l = rng.permutation(npix // nps).astype(np.int64)
    ref = np.zeros((npix // nps, nps, 3)); absmap = np.zeros_like(ref)
    oracle.build_noise_weighted(ref, g2l, nps, pixels, weights, tod, scale, ivs, det_flags=flags, det_flag_mask=4,
                                pixel_index=pidx, weight_index=widx, data_index=didx, flag_index=fidx, n_det=n_det,
                                absmap=absmap)
    zg = torch.zeros(ref.shape, dtype=torch.float64, device=DEV)
    binding.build_noise_weighted(zg, _cuda(g2l, torch.int64), nps, _cuda(pixels, torch.int64),
                                 _cuda(weights, torch.float64), _cuda(tod, torch.float64), _cuda(scale, torch.float64),
                                 ivs, det_flags=_cuda(flags, torch.uint8), det_flag_mask=4,
                                 pixel_index=_cuda(pidx, torch.int32), weight_index=_cuda(widx, torch.int32),
                                 data_index=_cuda(didx, torch.int32), flag_index=_cuda(fidx, torch.int32), n_det=n_det)
    check_map(zg.cpu().numpy(), ref, absmap)


@pytest.mark.parametrize("zero,subtract", [(False, False), (True, False), (False, True)])
def test_scan_map(chain, zero, subtract):
    w, quats, pix, hits, wts = chain
    rng = np.random.default_rng(61)
    m = rng.normal(size=(w.n_submap, w.n_pix_submap, 3))
    tod0 = rng.normal(size=(w.n_det, w.n_samp))
    ref = tod0.copy(); b = np.zeros_like(tod0)
    oracle.scan_map(m, w.global2local, w.n_pix_submap, pix, wts, ref, w.intervals, data_scale=0.7,
                    should_zero=zero, should_subtract=subtract, bscale=b)
    tg = _cuda(tod0, torch.float64)
    binding.scan_map(_cuda(m, torch.float64), _cuda(w.global2local, torch.int64), w.n_pix_submap,
                     _cuda(pix, torch.int64), _cuda(wts, torch.float64), tg, w.intervals, data_scale=0.7,
                     should_zero=zero, should_subtract=subtract)
    got = tg.cpu().numpy()
    tol = 1e-12 * b + 4e-16 * np.abs(ref)
    assert np.all(np.abs(got - ref) <= tol)


def test_round_trip_scan_then_accumulate():
    """C3-shaped round trip on the GPU chain (A1 -> A2 -> A3 -> A5 -> A4) vs the oracle chain;
    smooth map I = cos 3theta, Q = sin 2phi sin theta, U = cos phi sin theta.  Near-boundary
    pixel decisions (rule T1) are reconciled: the oracle chain is re-run with the GPU's pixel at
    exactly the samples the oracle classifier proves to lie within 1e-12 rad of a boundary."""
    w = synth.make_workload("c3", n_det=20, n_samp=30_000, nside=256)
    from independent import ring_centres
    z, ph = ring_centres(w.nside)
    st = np.sqrt(1 - z * z)
    th = np.arccos(z)
    m_ring = np.stack([np.cos(3 * th), np.sin(2 * ph) * st, np.cos(ph) * st], -1)
    m = m_ring.reshape(w.n_submap, w.n_pix_submap, 3)  # RING ordering, identity global2local
    # GPU chain
    qg = torch.zeros((w.n_det, w.n_samp, 4), dtype=torch.float64, device=DEV)
    sf = _cuda(w.shared_flags, torch.uint8)
    binding.pointing_detector(_cuda(w.fp_quats, torch.float64), _cuda(w.boresight, torch.float64), w.intervals, qg,
                              shared_flags=sf, shared_flag_mask=w.shared_flag_mask)
    pg = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)  # -7: untouched, as the oracle's
    binding.pixels_healpix(qg, w.intervals, w.nside, w.nest, w.n_pix_submap, pg, shared_flags=sf,
                           shared_flag_mask=w.shared_flag_mask)
    wg = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    binding.stokes_weights_iqu(qg, w.intervals, _cuda(w.epsilon, torch.float64), w.cal, wg)
    tg = torch.zeros((w.n_det, w.n_samp), dtype=torch.float64, device=DEV)
    g2l = _cuda(w.global2local, torch.int64)
    binding.scan_map(_cuda(m, torch.float64), g2l, w.n_pix_submap, pg, wg, tg, w.intervals)
    zg = torch.zeros(m.shape, dtype=torch.float64, device=DEV)
    binding.build_noise_weighted(zg, g2l, w.n_pix_submap, pg, wg, tg, _cuda(w.det_scale, torch.float64), w.intervals,
                                 shared_flags=sf, shared_flag_mask=w.shared_flag_mask)
    # oracle chain
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    pix, _ = oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags,
                                   w.shared_flag_mask)
    wts = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal)
    pgn = pg.cpu().numpy()
    n_in = int(_in_mask(w.intervals, 1, w.n_samp).sum()) * w.n_det
    mism = classify_pixel_mismatches(pgn, pix, lambda d, s: oracle.quat_rotate(quats[d, s], [0, 0, 1.0]), w.nside,
                                     w.nest, n_in)
    pix_r = pix.copy()
    pix_r[mism] = pgn[mism]  # admissible decisions (T1), proven near a boundary above
    tod = np.zeros((w.n_det, w.n_samp)); bsc = np.zeros_like(tod)
    oracle.scan_map(m, w.global2local, w.n_pix_submap, pix_r, wts, tod, w.intervals, bscale=bsc)
    ref = np.zeros_like(m); absmap = np.zeros_like(m)
    oracle.build_noise_weighted(ref, w.global2local, w.n_pix_submap, pix_r, wts, tod, w.det_scale, w.intervals,
                                shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask, absmap=absmap)
    # T3 on the timestream: 1e-12 B + the T2 weight tolerance carried by |m_Q|, |m_U| (<= 1)
    sth = _sin_theta(quats)
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    t2 = np.abs(eta_cal)[:, None] * np.maximum(1e-12, 1e-15 / np.maximum(sth, 1e-300))
    tol_tod = 1e-12 * bsc + 2 * t2 + 4e-16 * np.abs(tod)
    got = tg.cpu().numpy()
    assert np.all(np.abs(got - tod) <= tol_tod)
    # T4 on the map, plus what the tolerated tod and weight differences carry into it
    good = (pix_r >= 0) & np.array(_in_mask(w.intervals, w.n_det, w.n_samp))
    d_idx = np.nonzero(good)
    flat = pix_r[good]
    extra = np.zeros((m.shape[0] * m.shape[1], 3))
    scale = w.det_scale[d_idx[0]]
    for k in range(3):
        e = scale * tol_tod[good] * np.abs(wts[..., k][good])
        if k > 0:
            e = e + scale * np.abs(tod[good]) * t2[good]
        np.add.at(extra[:, k], flat, e)
    check_map(zg.cpu().numpy(), ref, absmap, extra=extra.reshape(m.shape))


def test_invalid_arguments_are_rejected():
    w = synth.make_workload("c1", n_samp=1000)
    dw = DeviceWorkload.upload(w, DEV)
    with pytest.raises(binding.ToastError, match="power of two"):
        binding.pointing_to_map(dw.fp_quats, dw.boresight, dw.epsilon, 1.0, dw.det_scale, dw.det_data, w.intervals,
                                3, False, 3, dw.global2local, w.n_pix_submap, dw.zmap)
    with pytest.raises(binding.ToastError, match="overlap"):
        binding.pointing_to_map(dw.fp_quats, dw.boresight, dw.epsilon, 1.0, dw.det_scale, dw.det_data,
                                [(0, 10), (5, 20)], w.nside, False, 3, dw.global2local, w.n_pix_submap, dw.zmap)
    with pytest.raises(binding.ToastError, match="CUDA tensor"):
        binding.pointing_to_map(dw.fp_quats.cpu(), dw.boresight, dw.epsilon, 1.0, dw.det_scale, dw.det_data,
                                w.intervals, w.nside, False, 3, dw.global2local, w.n_pix_submap, dw.zmap)


# ----------------------------------------------------------------------------- f1 pointing_to_tod

SCAN_CASES = {
    "c1_ring": dict(name="c1", n_samp=60_000),
    "c2_nest_hwp_flags": dict(name="c2", n_det=40, n_samp=120_000),
    "c2_nnz1": dict(name="c2", n_det=12, n_samp=60_000, nnz=1),
    "c3_ring_flags": dict(name="c3", n_det=36, n_samp=30_000),
    "c5_nest_4096": dict(name="c5", n_det=20, n_samp=60_000),
    # n_samp % 16 != 0: the cp.async staging path instead of the TMA path
    "c2_cp_async_path": dict(name="c2", n_det=36, n_samp=60_003),
}


@pytest.mark.parametrize("case", list(SCAN_CASES))
@pytest.mark.parametrize("mode", ["add", "zero", "subtract"])
def test_fused_pointing_to_tod(case, mode):
    w = synth.make_workload(**SCAN_CASES[case])
    rng = np.random.default_rng(81)
    m = rng.normal(size=(w.n_submap, w.n_pix_submap, w.nnz))
    zero, sub = mode == "zero", mode == "subtract"
    ref = w.det_data.copy()
    b = np.zeros_like(ref)
    oracle.pointing_to_tod(w.fp_quats, w.boresight, w.epsilon, w.cal, w.intervals, w.nside, w.nest, w.nnz,
                           w.global2local, w.n_pix_submap, m, ref, data_scale=0.8, should_zero=zero,
                           should_subtract=sub, hwp=w.hwp, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, bscale=b)
    dw = DeviceWorkload.upload(w, DEV)
    tg = dw.det_data.clone()
    binding.pointing_to_tod(dw.fp_quats, dw.boresight, dw.epsilon, w.cal, w.intervals, w.nside, w.nest, w.nnz,
                            dw.global2local, w.n_pix_submap, _cuda(m, torch.float64), tg, data_scale=0.8,
                            should_zero=zero, should_subtract=sub, hwp=dw.hwp, shared_flags=dw.shared_flags,
                            shared_flag_mask=w.shared_flag_mask)
    got = tg.cpu().numpy()
    # T3: 1e-12 of the scanned magnitude, plus the T2 weight tolerance carried by the map values
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    wtol = np.abs(eta_cal)[:, None] * np.maximum(1e-12, 1e-15 / np.maximum(_sin_theta(quats), 1e-300))
    mabs = float(np.abs(m).max())
    tol = 1e-12 * b + 0.8 * mabs * 2 * wtol + 4e-16 * np.abs(ref) + 1e-300
    bad = np.nonzero(np.abs(got - ref) > tol)
    n_in = int(_in_mask(w.intervals, 1, w.n_samp).sum()) * w.n_det
    probe = _probe(w)
    for d, s in zip(*bad):
        assert oracle.near_boundary(w.nside, w.nest, probe(int(d), int(s))), f"tod mismatch at det {d} sample {s}"
    assert len(bad[0]) <= 1e-6 * n_in
    out = ~np.array(_in_mask(w.intervals, w.n_det, w.n_samp))
    np.testing.assert_array_equal(got[out], w.det_data[out])  # out-of-interval samples untouched


# ----------------------------------------------------------------------------- f2, f4

NEXT_IVS = [(3, 40_002), (40_100, 40_100), (41_000, 99_998)]


def test_stokes_weights_i_and_noise_weight_gpu():
    n_det, n_samp = 5, 100_000
    wg = torch.full((n_det, n_samp), -1.0, dtype=torch.float64, device=DEV)
    binding.stokes_weights_i(wg, 1.25, NEXT_IVS)
    ref = np.full((n_det, n_samp), -1.0)
    oracle.stokes_weights_i(ref, 1.25, NEXT_IVS, n_det)
    np.testing.assert_array_equal(wg.cpu().numpy(), ref)
    rng = np.random.default_rng(91)
    tod = rng.normal(size=(n_det, n_samp)); dwt = rng.uniform(0.1, 3, n_det)
    ref = tod.copy(); oracle.noise_weight(ref, dwt, NEXT_IVS)
    tg = _cuda(tod, torch.float64)
    binding.noise_weight(tg, _cuda(dwt, torch.float64), NEXT_IVS)
    np.testing.assert_array_equal(tg.cpu().numpy(), ref)  # one IEEE multiply: bit-exact


@pytest.mark.parametrize("step", [1, 37, 256, 1000])
def test_template_offsets_gpu(step):
    n_det, n_samp = 6, 100_000
    n_amp = oracle.offset_amplitude_counts(NEXT_IVS, step)
    amp_offset = (np.arange(n_det, dtype=np.int64) * n_amp)[::-1].copy()  # permuted detector blocks
    rng = np.random.default_rng(92 + step)
    amps = rng.normal(size=n_det * n_amp)
    tod = rng.normal(size=(n_det, n_samp))
    flags = (rng.random((n_det, n_samp)) < 0.05).astype(np.uint8) * 2
    # add_to_signal: one add per sample, bit-exact
    ref = tod.copy(); oracle.template_offset_add_to_signal(step, amp_offset, amps, ref, NEXT_IVS)
    tg = _cuda(tod, torch.float64)
    binding.template_offset_add_to_signal(step, _cuda(amp_offset, torch.int64), _cuda(amps, torch.float64), tg,
                                          NEXT_IVS)
    np.testing.assert_array_equal(tg.cpu().numpy(), ref)
    # project_signal: sums in a different order -> 1e-12 of the sum of |terms|
    refa = np.zeros(n_det * n_amp)
    oracle.template_offset_project_signal(step, amp_offset, refa, tod, NEXT_IVS, det_flags=flags, det_flag_mask=2)
    absa = np.zeros(n_det * n_amp)
    oracle.template_offset_project_signal(step, amp_offset, absa, np.abs(tod), NEXT_IVS, det_flags=flags,
                                          det_flag_mask=2)
    ag = torch.zeros(n_det * n_amp, dtype=torch.float64, device=DEV)
    binding.template_offset_project_signal(step, _cuda(amp_offset, torch.int64), ag, _cuda(tod, torch.float64),
                                           NEXT_IVS, det_flags=_cuda(flags, torch.uint8), det_flag_mask=2)
    assert np.all(np.abs(ag.cpu().numpy() - refa) <= 1e-12 * absa + (absa == 0) * 0.0)
    # diagonal preconditioner: one multiply, bit-exact
    var = rng.uniform(0.1, 2, n_det * n_amp)
    out = torch.zeros(n_det * n_amp, dtype=torch.float64, device=DEV)
    binding.template_offset_apply_diag_precond(_cuda(var, torch.float64), ag, out)
    np.testing.assert_array_equal(out.cpu().numpy(), oracle.template_offset_apply_diag_precond(var, ag.cpu().numpy()))


@pytest.mark.parametrize("nside,nest", [(1 << 13, True), (1 << 13, False), (1 << 20, True)])
def test_fused_incremental_longitude_wraps_and_poles(nside, nest):
    """The fused kernel carries the longitude incrementally along each detector's samples
    (DESIGN.md "Fused kernel"): boresights that circle the pole (the quarter-turn longitude
    wraps 4 -> 0 every ~600 samples, steps of 0.01 rad: the series path), that cross it (the
    step exceeds the series range: the full-arctangent fallback) and a slow drift (long series
    chains) give the oracle's pixels up to near-boundary samples, at fine pixelisations."""
    n_samp = 6000
    w = synth.make_workload("c1", n_samp=n_samp, nside=nside, nest=nest, nnz=3)
    t = np.arange(n_samp, dtype=np.float64)
    third = n_samp // 3
    a, b, c = t[:third], t[third:2 * third], t[2 * third:]
    mats = np.concatenate([
        # circle at colatitude 0.05 rad: phi advances 0.01 rad per sample
        synth.matmul_chain(synth.rot_axis("z", 0.01 * a), synth.rot_axis("y", np.full_like(a, 0.05))),
        # great circle through both poles, 2e-3 rad per sample
        synth.rot_axis("x", 2e-3 * (b - third) - 0.3),
        # slow drift near the equator
        synth.matmul_chain(synth.rot_axis("z", 1e-5 * c + 1.0), synth.rot_axis("y", np.full_like(c, 1.2))),
    ])
    w.boresight = synth.matrix_to_quat(mats)
    w.intervals = [(0, n_samp - 1)]
    w.n_pix_submap = (nside // 16) ** 2
    quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals)
    po, hits = oracle.pixels_healpix(quats, w.intervals, nside, nest, w.n_pix_submap)
    dw = DeviceWorkload.upload(w, DEV, alloc_map=False)
    dw.global2local = torch.full((w.n_submap,), -1, dtype=torch.int64, device=DEV)
    dw.zmap = torch.zeros((1, 1, 3), dtype=torch.float64, device=DEV)
    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    wts_g = torch.zeros((w.n_det, w.n_samp, 3), dtype=torch.float64, device=DEV)
    dw.pointing_to_map(pixels_out=pix_g, weights_out=wts_g)
    torch.cuda.synchronize()
    classify_pixel_mismatches(pix_g.cpu().numpy(), po, _probe(w), nside, nest, w.n_det * n_samp)
    np.testing.assert_array_equal(dw.hit_submaps.cpu().numpy(), hits)
    wo = oracle.stokes_weights_iqu(quats, w.intervals, w.epsilon, w.cal, hwp=w.hwp)
    eta_cal = (1 - w.epsilon) / (1 + w.epsilon) * w.cal
    check_weights(wts_g.cpu().numpy(), wo, _sin_theta(quats), eta_cal, w.cal, np.ones((w.n_det, n_samp), bool))
