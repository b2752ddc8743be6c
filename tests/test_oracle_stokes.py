"""Pins for oracle O4 (stokes_weights_IQU; readings S9, S10), CPU only.

Pinned against closed forms, the geometric polarisation angle in the local
(e_theta, e_phi) frame (tests/independent.py), the roll / HWP symmetries and
the epsilon limits.
"""
import math

import numpy as np

import oracle
from independent import axis_angle_quat, psi_geometric, random_axis_angle, rodrigues


def test_identity_quaternion():
    w = oracle.stokes_iqu([0, 0, 0, 1.0], 0.0, 0.0, 2.5)
    np.testing.assert_array_equal(w, [2.5, 2.5, 0.0])  # pole, psi = 0 (S10)
    eps = 0.01
    eta = (1 - eps) / (1 + eps)
    np.testing.assert_allclose(oracle.stokes_iqu([0, 0, 0, 1.0], 0.0, eps, 1.0), [1.0, eta, 0.0], rtol=0, atol=1e-16)


def test_quarter_turn_about_y():
    s = math.sin(math.pi / 4)
    w = oracle.stokes_iqu([0, s, 0, s], 0.0, 0.0, 1.0)  # bx = -1, by = 0 -> psi = pi
    np.testing.assert_allclose(w, [1.0, 1.0, 0.0], atol=1e-15)


def test_matches_geometric_angle():
    rng = np.random.default_rng(11)
    for _ in range(500):
        n, a = random_axis_angle(rng)
        r = rodrigues(n, a)
        d, o = r[:, 2], r[:, 0]
        if math.hypot(d[0], d[1]) < 1e-3:
            continue
        psi = psi_geometric(d, o)
        chi = rng.uniform(0, 2 * math.pi)
        w = oracle.stokes_iqu(axis_angle_quat(n, a), chi, 0.0, 1.0)
        ang = 2 * psi + 4 * chi
        np.testing.assert_allclose(w, [1.0, math.cos(ang), math.sin(ang)], atol=2e-13)


def test_polarisation_amplitude():
    rng = np.random.default_rng(12)
    for _ in range(500):
        q = axis_angle_quat(*random_axis_angle(rng))
        eps = rng.uniform(0, 0.3)
        cal = rng.uniform(0.5, 2)
        w = oracle.stokes_iqu(q, rng.uniform(0, 6.28), eps, cal)
        eta = (1 - eps) / (1 + eps)
        assert abs(math.hypot(w[1], w[2]) - eta * cal) <= 1e-15 * 4
        assert w[0] == cal


def test_roll_rotates_q_u_by_twice_the_angle():
    """psi(q (x) Rz(a)) = psi(q) + a, so (Q, U) rotate by 2a."""
    rng = np.random.default_rng(13)
    for _ in range(300):
        q = axis_angle_quat(*random_axis_angle(rng))
        a = rng.uniform(-math.pi, math.pi)
        qr = oracle.quat_mul(q, axis_angle_quat([0, 0, 1], a))
        w0 = oracle.stokes_iqu(q, 0.0, 0.0, 1.0)
        w1 = oracle.stokes_iqu(qr, 0.0, 0.0, 1.0)
        c, s = math.cos(2 * a), math.sin(2 * a)
        np.testing.assert_allclose(w1[1:], [c * w0[1] - s * w0[2], s * w0[1] + c * w0[2]], atol=5e-12)


def test_hwp_symmetries():
    rng = np.random.default_rng(14)
    for _ in range(200):
        q = axis_angle_quat(*random_axis_angle(rng))
        chi = rng.uniform(0, math.pi)
        w = oracle.stokes_iqu(q, chi, 0.0, 1.0)
        np.testing.assert_allclose(oracle.stokes_iqu(q, chi + math.pi / 4, 0.0, 1.0)[1:], -w[1:], atol=1e-14)
        np.testing.assert_allclose(oracle.stokes_iqu(q, chi + math.pi / 2, 0.0, 1.0)[1:], w[1:], atol=1e-14)


def test_epsilon_limits():
    rng = np.random.default_rng(15)
    q = axis_angle_quat(*random_axis_angle(rng))
    w1 = oracle.stokes_iqu(q, 0.3, 1.0, 1.7)
    assert w1[0] == 1.7 and w1[1] == 0.0 and w1[2] == 0.0
    w0 = oracle.stokes_iqu(q, 0.3, 0.0, 1.0)
    assert abs(math.hypot(w0[1], w0[2]) - 1.0) < 1e-15


# ----------------------------------------------------------------------------- reading R3 (f4)

def _mueller_response(psi, hwp_axis):
    """Detector response row (I, Q, U) of a linear polariser at sky angle psi behind an ideal
    half-wave plate with its fast axis at sky angle hwp_axis — Mueller calculus, written
    from the textbook matrices (polariser row 1/2 [1, cos 2psi, sin 2psi]; HWP at angle a:
    [[1, 0, 0], [0, cos 4a, sin 4a], [0, sin 4a, -cos 4a]] on (I, Q, U)), normalised to I = 1."""
    pol = np.array([1.0, math.cos(2 * psi), math.sin(2 * psi)])
    if hwp_axis is None:
        return pol
    c, s = math.cos(4 * hwp_axis), math.sin(4 * hwp_axis)
    hwp = np.array([[1.0, 0.0, 0.0], [0.0, c, s], [0.0, s, -c]])
    return pol @ hwp


def test_gamma_hwp_convention_matches_mueller_calculus():
    """Reading R3: with an HWP at angle chi from the focal-plane x axis and a detector at angle
    gamma in the focal plane, the HWP fast axis lies at psi - gamma + chi on the sky; the
    Mueller response of that system is (1, cos(2 psi + 4 (chi - gamma)), sin(...))."""
    rng = np.random.default_rng(16)
    n = 0
    for _ in range(400):
        ax, a = random_axis_angle(rng)
        r = rodrigues(ax, a)
        d, o = r[:, 2], r[:, 0]
        if math.hypot(d[0], d[1]) < 1e-3:
            continue
        psi = psi_geometric(d, o)
        chi, gamma = rng.uniform(0, 2 * math.pi), rng.uniform(-math.pi, math.pi)
        eps, cal = rng.uniform(0, 0.1), rng.uniform(0.5, 2.0)
        eta = (1 - eps) / (1 + eps)
        want = _mueller_response(psi, psi - gamma + chi) * np.array([cal, eta * cal, eta * cal])
        got = oracle.stokes_iqu(axis_angle_quat(ax, a), chi, eps, cal, gamma=gamma)
        np.testing.assert_allclose(got, want, atol=2e-13)
        # without an HWP the detector angle is already inside the quaternion: gamma has no effect
        want0 = _mueller_response(psi, None) * np.array([cal, eta * cal, eta * cal])
        np.testing.assert_allclose(oracle.stokes_iqu(axis_angle_quat(ax, a), None, eps, cal, gamma=gamma), want0,
                                   atol=2e-13)
        n += 1
    assert n > 350


def test_iau_flips_u_only():
    rng = np.random.default_rng(17)
    for _ in range(200):
        q = axis_angle_quat(*random_axis_angle(rng))
        chi = rng.uniform(0, 2 * math.pi) if rng.random() < 0.5 else None
        g = rng.uniform(-1, 1)
        w = oracle.stokes_iqu(q, chi, 0.01, 1.3, gamma=g)
        wi = oracle.stokes_iqu(q, chi, 0.01, 1.3, gamma=g, iau=True)
        assert wi[0] == w[0] and wi[1] == w[1] and wi[2] == -w[2]


def test_gamma_zero_and_hwp_zero_reduce_to_plain_reading():
    """gamma = 0 is reading S9 exactly; an HWP angle of 0 equals no HWP when gamma = 0."""
    rng = np.random.default_rng(18)
    for _ in range(100):
        q = axis_angle_quat(*random_axis_angle(rng))
        chi = rng.uniform(0, 2 * math.pi)
        np.testing.assert_array_equal(oracle.stokes_iqu(q, chi, 0.02, 1.0),
                                      oracle.stokes_iqu(q, chi, 0.02, 1.0, gamma=0.0))
        np.testing.assert_array_equal(oracle.stokes_iqu(q, 0.0, 0.02, 1.0), oracle.stokes_iqu(q, None, 0.02, 1.0))


def test_unwrapped_hwp_angle_is_exact_to_the_angle():
    """Reading R1: an unwrapped HWP angle (a 2 Hz HWP over days: chi ~ 1e6 rad) still gives the
    response of the exact angle 2 psi + 4 chi (evaluated here in 60-digit arithmetic from the
    geometric psi), not that of the rounded fp64 sum, which is off by up to |4 chi| 2^-53."""
    import mpmath
    mpmath.mp.dps = 60
    rng = np.random.default_rng(19)
    worst_sum = 0.0
    for _ in range(200):
        ax, a = random_axis_angle(rng)
        r = rodrigues(ax, a)
        d, o = r[:, 2], r[:, 0]
        if math.hypot(d[0], d[1]) < 1e-2:
            continue
        psi = psi_geometric(d, o)
        chi = float(rng.uniform(1e5, 4e6))
        ang = 2 * mpmath.mpf(psi) + 4 * mpmath.mpf(chi)
        want = [1.0, float(mpmath.cos(ang)), float(mpmath.sin(ang))]
        got = oracle.stokes_iqu(axis_angle_quat(ax, a), chi, 0.0, 1.0)
        np.testing.assert_allclose(got, want, atol=2e-13)
        worst_sum = max(worst_sum, abs(math.cos(2 * psi + 4 * chi) - want[1]))
    assert worst_sum > 1e-11  # the naive fp64 sum would not pass this pin
