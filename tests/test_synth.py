"""The shared seeded input generator (no method arithmetic): determinism, unit
quaternions (reading S7), subset regeneration, interval validity."""
import numpy as np

from paper_conf_sc_demeurekktbb23_b200 import synth


def test_splitmix_known_values():
    # SplitMix64 reference stream from seed 0 (Vigna's splitmix64.c): first outputs
    # are mix(0x9E3779B97F4A7C15 * k) for k = 1, 2
    g = np.uint64(0x9E3779B97F4A7C15)
    with np.errstate(over="ignore"):
        out = synth.splitmix64_mix(np.array([g, g * np.uint64(2)], dtype=np.uint64))
    assert int(out[0]) == 0xE220A8397B1DCDAF
    assert int(out[1]) == 0x6E789E6AA1B965F4


def test_tod_subset_regenerates_bit_identically():
    w = synth.make_workload("c1", n_samp=5000)
    sub = synth.tod_rows(w.seed, w.sigma[2:4], w.det_ids[2:4], w.n_samp, 100, 900)
    np.testing.assert_array_equal(sub, w.det_data[2:4, 100:900])
    u = w.det_data / w.sigma[:, None]
    assert np.all(np.abs(u) <= 1.0 + 1e-15)


def test_quaternions_unit_and_intervals_valid():
    for name in ("c1", "c2", "c5"):
        w = synth.make_workload(name, n_det=8, n_samp=40000, with_tod=False)
        assert np.max(np.abs(np.linalg.norm(w.boresight, axis=1) - 1)) <= 4.5e-16
        assert np.max(np.abs(np.linalg.norm(w.fp_quats, axis=1) - 1)) <= 4.5e-16
        last = -1
        for f, l in w.intervals:
            assert 0 <= f <= l < w.n_samp and f > last
            last = l


def test_det_range_is_a_slice_of_the_full_focal_plane():
    full = synth.make_workload("c2", n_det=16, n_samp=3000)
    part = synth.make_workload("c2", n_det=16, n_samp=3000, det_range=(4, 10))
    np.testing.assert_array_equal(part.fp_quats, full.fp_quats[4:10])
    np.testing.assert_array_equal(part.det_data, full.det_data[4:10])
    np.testing.assert_array_equal(part.det_flags, full.det_flags[4:10])
