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
