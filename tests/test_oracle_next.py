"""Pins for the NEXT-row oracle functions, CPU only:
stokes_weights_I / noise_weight closed forms, and the offset-template kernels pinned by the
project(add(a)) = (samples per step) * a identity, the add/project adjoint identity and an
independent numpy formulation of reading O1."""
import numpy as np

import oracle

IVS = [(3, 1002), (1100, 1100), (1200, 2999)]
N_SAMP = 3100


def _inside():
    m = np.zeros(N_SAMP, bool)
    for f, l in IVS:
        m[f:l + 1] = True
    return m


def test_stokes_weights_i_and_noise_weight():
    w = np.full((3, N_SAMP), -1.0)
    oracle.stokes_weights_i(w, 1.25, IVS, 3)
    ins = _inside()
    assert np.all(w[:, ins] == 1.25) and np.all(w[:, ~ins] == -1.0)
    rng = np.random.default_rng(1)
    tod = rng.normal(size=(3, N_SAMP))
    t2 = tod.copy()
    dw = np.array([0.5, 2.0, -3.0])
    oracle.noise_weight(t2, dw, IVS)
    np.testing.assert_array_equal(t2[:, ins], tod[:, ins] * dw[:, None])
    np.testing.assert_array_equal(t2[:, ~ins], tod[:, ~ins])


def _index_numpy(step, amp_offset, d, s):
    """Reading O1 written independently: enumerate the steps interval by interval."""
    base = amp_offset[d]
    for f, l in IVS:
        if f <= s <= l:
            return base + (s - f) // step
        base += -(-(l - f + 1) // step)
    return -1


def test_offset_add_matches_independent_indexing():
    step = 37
    n_det = 3
    n_amp = oracle.offset_amplitude_counts(IVS, step)
    amp_offset = np.arange(n_det, dtype=np.int64) * n_amp
    rng = np.random.default_rng(2)
    amps = rng.normal(size=n_det * n_amp)
    tod = np.zeros((n_det, N_SAMP))
    oracle.template_offset_add_to_signal(step, amp_offset, amps, tod, IVS)
    for d in range(n_det):
        for s in range(0, N_SAMP, 7):
            i = _index_numpy(step, amp_offset, d, s)
            assert tod[d, s] == (amps[i] if i >= 0 else 0.0)


def test_offset_project_of_add_counts_samples_and_adjoint():
    step = 50
    n_det = 2
    n_amp = oracle.offset_amplitude_counts(IVS, step)
    amp_offset = np.arange(n_det, dtype=np.int64) * n_amp
    a = np.random.default_rng(3).normal(size=n_det * n_amp)
    tod = np.zeros((n_det, N_SAMP))
    oracle.template_offset_add_to_signal(step, amp_offset, a, tod, IVS)
    proj = np.zeros_like(a)
    oracle.template_offset_project_signal(step, amp_offset, proj, tod, IVS)
    counts = np.zeros(n_det * n_amp)
    for d in range(n_det):
        for s in np.nonzero(_inside())[0]:
            counts[_index_numpy(step, amp_offset, d, s)] += 1
    np.testing.assert_allclose(proj, counts * a, rtol=1e-14, atol=0)
    # adjoint: <add(a), t> = <a, project(t)>
    t = np.random.default_rng(4).normal(size=(n_det, N_SAMP))
    sc = np.zeros((n_det, N_SAMP))
    oracle.template_offset_add_to_signal(step, amp_offset, a, sc, IVS)
    pr = np.zeros_like(a)
    oracle.template_offset_project_signal(step, amp_offset, pr, t, IVS)
    assert abs(float(np.sum(sc * t)) - float(np.sum(a * pr))) <= 1e-12 * float(np.sum(np.abs(sc * t)))


def test_offset_project_skips_flagged_and_precond():
    step = 10
    n_amp = oracle.offset_amplitude_counts(IVS, step)
    amp_offset = np.zeros(1, np.int64)
    tod = np.ones((1, N_SAMP))
    flags = np.zeros((1, N_SAMP), np.uint8)
    flags[0, 3:8] = 2    # masked
    flags[0, 8:13] = 4   # not masked
    proj = np.zeros(n_amp)
    oracle.template_offset_project_signal(step, amp_offset, proj, tod, IVS, det_flags=flags, det_flag_mask=2)
    assert proj[0] == 5.0   # samples 3..12 of the first step, 3..7 flagged
    assert proj[1] == 10.0
    var = np.random.default_rng(5).uniform(0.1, 2, n_amp)
    a = np.random.default_rng(6).normal(size=n_amp)
    np.testing.assert_array_equal(oracle.template_offset_apply_diag_precond(var, a), var * a)
