"""GPU parity at BASELINE.json's FULL sizes, in the launch configuration bench.py times.

bench.py times the production instantiation of toast_pointing_to_map (no debug outputs, TMA
staging) on the whole C1-C5 workloads.  These tests run exactly that call on exactly those
shapes and check it against the oracle:

* C2, C3 (6e7 det-samples each): the whole map, element by element, against the oracle's map
  (rule T4), hit submaps exactly; the pixel decisions through the debug instantiation (T1).
* Every config, via outputs the oracle computes ONE BY ONE (task rule: "on sampled outputs the
  oracle can compute one by one"): the TOD is zero except at 2048 seeded probe det-samples, so
  every non-zero map element is the sum of a few probes' det_scale * tod * w, each from
  oracle.det_sample_probe; every other element must be exactly 0.
* Every config, via properties that hold at any size: with tod = det_scale = cal = 1 the I map
  is the hit count, integral everywhere, summing EXACTLY to the number of unflagged in-interval
  det-samples, and |Q|, |U| <= eta_max * I.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
from parity import NEAR_DELTA, check_map, classify_pixel_mismatches  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200 import binding, synth  # noqa: E402
from paper_conf_sc_demeurekktbb23_b200.staging import DeviceWorkload  # noqa: E402

pytestmark = pytest.mark.gpu

DEV = "cuda"
STREAM_PROBE = 0x5EED  # probe positions / values: a stream of their own


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    binding.load()


def _assert_bench_path(w):
    """The staging path bench.py times on this workload: TMA, or the thread-per-(chunk, detector)
    kernel below 8 detectors (C1)."""
    path = binding.last_fused_path()
    assert path == "tma" or (w.n_det < 8 and path.startswith("thin")), path


def _valid_mask_counts(w):
    """Per detector: number of in-interval samples that are neither shared- nor det-flagged."""
    inside = np.zeros(w.n_samp, bool)
    for f, l in w.intervals:
        inside[f:l + 1] = True
    if w.shared_flags is not None:
        inside &= (w.shared_flags & w.shared_flag_mask) == 0
    if w.det_flags is None:
        return np.full(w.n_det, int(inside.sum()), np.int64)
    return np.array([int((inside & ((w.det_flags[d] & w.det_flag_mask) == 0)).sum()) for d in range(w.n_det)])


def _need_bytes(nbytes):
    free, _ = torch.cuda.mem_get_info()
    if free < nbytes * 1.1:
        pytest.skip(f"needs {nbytes / 1e9:.1f} GB of device memory, {free / 1e9:.1f} GB free")


def _workload_no_tod(name):
    w = synth.make_workload(name, with_tod=False)
    w.gen_det_flags()
    return w


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4", "c5"])
def test_full_size_hit_count_property(name):
    """tod = det_scale = cal = 1: the production kernel's I map counts hits exactly."""
    w = _workload_no_tod(name)
    _need_bytes(w.n_det * w.n_samp * 8 + 2 * w.npix * w.nnz * 8)
    ones = torch.ones((w.n_det, w.n_samp), dtype=torch.float64, device=DEV)
    dw = DeviceWorkload.upload(w, DEV, det_data=ones)
    dw.det_scale.fill_(1.0)
    w.cal = 1.0
    dw.pointing_to_map()
    torch.cuda.synchronize()
    _assert_bench_path(w)
    del ones
    z = dw.zmap
    n_valid = int(_valid_mask_counts(w).sum())
    total = float(z[..., 0].sum())  # integers < 2^53: exact in any summation order
    assert total == float(n_valid), f"{name}: sum of I = {total}, unflagged in-interval det-samples = {n_valid}"
    assert bool(torch.all(z[..., 0] == torch.floor(z[..., 0]))), "I map not integral"
    assert bool(torch.all(z[..., 0] >= 0))
    if w.nnz == 3:
        eta_max = float(np.max((1 - w.epsilon) / (1 + w.epsilon)))
        bound = eta_max * z[..., 0] * (1 + 1e-12) + 1e-12
        assert bool(torch.all(z[..., 1].abs() <= bound)) and bool(torch.all(z[..., 2].abs() <= bound))
    # the hit submaps are exactly the submaps with a hit (each hit sample marks its submap)
    hit_sm = (z[..., 0].sum(dim=1) > 0).to(torch.uint8)
    # a det-flagged sample still marks its submap (reading R2), so hits may exceed the I support
    assert bool(torch.all(dw.hit_submaps >= hit_sm))


def _probes(w, k=2048):
    """Seeded probe det-samples: 85% inside intervals, the rest anywhere (out-of-interval probes
    must add nothing); distinct (d, s); exact dyadic non-zero values."""
    rng_h = synth.counter_hash(w.seed, STREAM_PROBE, 0, np.arange(4 * k, dtype=np.uint64))
    u = synth.hash_to_u01(rng_h)
    lens = np.array([l - f + 1 for f, l in w.intervals], np.int64)
    cum = np.concatenate([[0], np.cumsum(lens)])
    n_in = int(cum[-1])
    d = (u[:k] * w.n_det).astype(np.int64)
    pos = (u[k:2 * k] * n_in).astype(np.int64)
    iv = np.searchsorted(cum, pos, side="right") - 1
    s_in = np.array([w.intervals[i][0] for i in iv], np.int64) + (pos - cum[iv])
    s_any = (u[2 * k:3 * k] * w.n_samp).astype(np.int64)
    s = np.where(u[3 * k:4 * k] < 0.85, s_in, s_any)
    ds = np.unique(d * w.n_samp + s)
    d, s = ds // w.n_samp, ds % w.n_samp
    vals = synth.hash_to_unit(synth.counter_hash(w.seed, STREAM_PROBE, 1, ds.astype(np.uint64)))
    vals = np.where(vals == 0.0, 0.5, vals)
    return d, s, vals


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4", "c5"])
def test_full_size_sparse_probes(name):
    """The production call on the full workload with a TOD that is zero except at probe
    det-samples: every map element equals the oracle's one-by-one sum of its probes."""
    w = _workload_no_tod(name)
    _need_bytes(w.n_det * w.n_samp * 8 + w.npix * w.nnz * 8)
    d, s, vals = _probes(w)
    inside = np.zeros(w.n_samp, bool)
    for f, l in w.intervals:
        inside[f:l + 1] = True
    expect, absmap = {}, {}
    keep = np.ones(len(d), bool)
    n_contrib = 0
    for i in range(len(d)):
        di, si = int(d[i]), int(s[i])
        sflag = w.shared_flags is not None and bool(w.shared_flags[si] & w.shared_flag_mask)
        pix, wt, v = oracle.det_sample_probe(w.fp_quats[di], w.boresight[si], 0.0 if w.hwp is None else w.hwp[si],
                                             w.epsilon[di], w.cal, sflag, w.nside, w.nest)
        if inside[si] and not sflag and oracle.near_boundary(w.nside, w.nest, v, NEAR_DELTA):
            keep[i] = False  # boundary decisions are rule T1's business (tests/test_parity_gpu.py)
            continue
        if not inside[si] or sflag or pix < 0:
            continue
        if w.det_flags is not None and (w.det_flags[di, si] & w.det_flag_mask):
            continue
        n_contrib += 1
        terms = w.det_scale[di] * vals[i] * wt[:w.nnz]
        sm, lp = pix // w.n_pix_submap, pix % w.n_pix_submap
        key = (int(w.global2local[sm]), int(lp))
        expect[key] = expect.get(key, np.zeros(w.nnz)) + terms
        absmap[key] = absmap.get(key, np.zeros(w.nnz)) + np.abs(terms)
    d, s, vals = d[keep], s[keep], vals[keep]
    assert n_contrib > 1000, n_contrib

    tod = torch.zeros((w.n_det, w.n_samp), dtype=torch.float64, device=DEV)
    tod[torch.from_numpy(d).to(DEV), torch.from_numpy(s).to(DEV)] = torch.from_numpy(vals).to(DEV)
    dw = DeviceWorkload.upload(w, DEV, det_data=tod)
    dw.pointing_to_map()
    torch.cuda.synchronize()
    _assert_bench_path(w)
    del tod

    keys = sorted(expect)
    loc = torch.tensor([k[0] for k in keys], device=DEV)
    lp = torch.tensor([k[1] for k in keys], device=DEV)
    got = dw.zmap[loc, lp].cpu().numpy()
    ora = np.array([expect[k] for k in keys])
    am = np.array([absmap[k] for k in keys])
    check_map(got, ora, am)
    # nothing anywhere else: the element count of the support matches
    n_nonzero = int(torch.count_nonzero(dw.zmap[..., 0]))
    assert n_nonzero == len(keys), f"{n_nonzero} non-zero I elements, oracle support {len(keys)}"


@pytest.mark.parametrize("name", ["c2", "c3"])
def test_full_size_whole_map(name):
    """C2 / C3 at full size: the whole production map against the oracle's, element by
    element (T4), the hit submaps exactly, and the pixel decisions (T1) via the debug outputs."""
    w = synth.make_workload(name)
    zo = np.zeros((w.n_submap, w.n_pix_submap, w.nnz))
    absmap = np.zeros_like(zo)
    ho = np.zeros(w.n_submap, np.uint8)
    po = np.full((w.n_det, w.n_samp), -7, np.int64)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, w.nnz, w.global2local, w.n_pix_submap, zmap=zo, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, hit_submaps=ho, pixels_out=po, absmap=absmap)
    dw = DeviceWorkload.upload(w, DEV)
    dw.pointing_to_map()  # production instantiation, as bench.py times it
    torch.cuda.synchronize()
    _assert_bench_path(w)
    zg = dw.zmap.cpu().numpy()
    hg = dw.hit_submaps.cpu().numpy()

    pix_g = torch.full((w.n_det, w.n_samp), -7, dtype=torch.int64, device=DEV)
    dw.pointing_to_map(zmap=torch.zeros_like(dw.zmap), pixels_out=pix_g)
    torch.cuda.synchronize()
    pg = pix_g.cpu().numpy()
    del pix_g
    n_in = sum(l - f + 1 for f, l in w.intervals) * w.n_det

    def probe(di, si):
        flagged = w.shared_flags is not None and bool(w.shared_flags[si] & w.shared_flag_mask)
        return oracle.det_sample_probe(w.fp_quats[di], w.boresight[si], 0.0 if w.hwp is None else w.hwp[si],
                                       w.epsilon[di], w.cal, flagged, w.nside, w.nest)[2]

    mism = classify_pixel_mismatches(pg, po, probe, w.nside, w.nest, n_in)
    for di, si in zip(*mism):  # move the (allowed) near-boundary decisions to the GPU's pixel
        if w.det_flags is not None and (w.det_flags[di, si] & w.det_flag_mask):
            continue
        flagged = w.shared_flags is not None and bool(w.shared_flags[si] & w.shared_flag_mask)
        _, wt, _ = oracle.det_sample_probe(w.fp_quats[di], w.boresight[si], 0.0 if w.hwp is None else w.hwp[si],
                                           w.epsilon[di], w.cal, flagged, w.nside, w.nest)
        terms = w.det_scale[di] * w.det_data[di, si] * wt[:w.nnz]
        for p, sign in ((po[di, si], -1.0), (pg[di, si], 1.0)):
            zo[w.global2local[p // w.n_pix_submap], p % w.n_pix_submap] += sign * terms
            absmap[w.global2local[p // w.n_pix_submap], p % w.n_pix_submap] += np.abs(terms)
    check_map(zg, zo, absmap)
    expect_hits = np.zeros(w.n_submap, np.uint8)
    expect_hits[np.unique(pg[pg >= 0] // w.n_pix_submap)] = 1
    np.testing.assert_array_equal(hg, expect_hits)
    if len(mism[0]) == 0:
        np.testing.assert_array_equal(hg, ho)
