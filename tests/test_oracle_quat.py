"""Pins for oracle O1/O2 (quaternion product and rotation), CPU only.

Pinned against Rodrigues rotation matrices and the axis-angle definition of a
rotation quaternion (tests/independent.py), never against a retyped product.
"""
import math

import numpy as np
import pytest

import oracle
from independent import axis_angle_quat, random_axis_angle, rodrigues

X, Y, Z = np.eye(3)


def test_identity_and_quarter_turn_closed_forms():
    ident = np.array([0, 0, 0, 1.0])
    np.testing.assert_array_equal(oracle.quat_rotate(ident, Z), Z)
    np.testing.assert_array_equal(oracle.quat_rotate(ident, X), X)
    s = math.sin(math.pi / 4)
    q = np.array([0, s, 0, s])  # +90 deg about y: z -> x, x -> -z (SURVEY 8(c) O1/O2 pins)
    np.testing.assert_allclose(oracle.quat_rotate(q, Z), X, atol=1e-16)
    np.testing.assert_allclose(oracle.quat_rotate(q, X), -Z, atol=1e-16)


def test_hamilton_basis_products():
    """Hamilton's rules i j = k, j i = -k, i^2 = j^2 = k^2 = ijk = -1."""
    i, j, k, one = (np.array(v, float) for v in ([1, 0, 0, 0], [0, 1, 0, 0], [0, 0, 1, 0], [0, 0, 0, 1]))
    np.testing.assert_array_equal(oracle.quat_mul(i, j), k)
    np.testing.assert_array_equal(oracle.quat_mul(j, i), -k)
    np.testing.assert_array_equal(oracle.quat_mul(j, k), i)
    np.testing.assert_array_equal(oracle.quat_mul(k, i), j)
    for e in (i, j, k):
        np.testing.assert_array_equal(oracle.quat_mul(e, e), -one)
    np.testing.assert_array_equal(oracle.quat_mul(oracle.quat_mul(i, j), k), -one)


def test_rotation_matches_rodrigues():
    rng = np.random.default_rng(1)
    for _ in range(300):
        n, a = random_axis_angle(rng)
        v = rng.normal(size=3)
        np.testing.assert_allclose(oracle.quat_rotate(axis_angle_quat(n, a), v), rodrigues(n, a) @ v,
                                   atol=4e-15 * np.linalg.norm(v))


def test_product_composes_rotations():
    """R(p (x) q) = R(p) R(q): the product order of reading S1 (q_det = q_bore (x) q_fp)."""
    rng = np.random.default_rng(2)
    for _ in range(300):
        n1, a1 = random_axis_angle(rng)
        n2, a2 = random_axis_angle(rng)
        v = rng.normal(size=3)
        pq = oracle.quat_mul(axis_angle_quat(n1, a1), axis_angle_quat(n2, a2))
        np.testing.assert_allclose(oracle.quat_rotate(pq, v), rodrigues(n1, a1) @ (rodrigues(n2, a2) @ v),
                                   atol=6e-15 * np.linalg.norm(v))


def test_same_axis_angles_add():
    rng = np.random.default_rng(3)
    for _ in range(200):
        n, a = random_axis_angle(rng)
        b = rng.uniform(-3, 3)
        np.testing.assert_allclose(oracle.quat_mul(axis_angle_quat(n, a), axis_angle_quat(n, b)),
                                   axis_angle_quat(n, a + b), atol=3e-16 * 4)


def test_unit_norm_preserved():
    rng = np.random.default_rng(4)
    worst = 0.0
    for _ in range(1000):
        p = axis_angle_quat(*random_axis_angle(rng))
        q = axis_angle_quat(*random_axis_angle(rng))
        worst = max(worst, abs(np.linalg.norm(oracle.quat_mul(p, q)) - 1.0))
    assert worst <= 6e-16
