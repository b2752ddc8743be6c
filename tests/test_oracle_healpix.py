"""Pins for oracle O3 (HEALPix vec2pix, Gorski et al. 2005 = PAPER.md ref [16]), CPU only.

Pins: closed forms at the poles and equator, published healpy ang2pix values
(tests/golden/healpy_ang2pix.txt), the nside=2 numbering (golden), pixel-centre
round trips and brute-force interior points from the INVERSE maps in
tests/independent.py, the RING<->NEST bijection, and equal area.
"""
import math
import os

import numpy as np
import pytest

import oracle
from independent import face_point, nest_index, ring_centres, zphi_to_vec

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.mark.parametrize("nside", [1, 2, 4, 64, 1024, 1 << 13, 1 << 20])
def test_poles(nside):
    npix = 12 * nside * nside
    assert oracle.vec2pix(nside, False, [0, 0, 1.0]) == 0
    assert oracle.vec2pix(nside, True, [0, 0, 1.0]) == nside * nside - 1
    assert oracle.vec2pix(nside, False, [0, 0, -1.0]) == npix - 4
    assert oracle.vec2pix(nside, True, [0, 0, -1.0]) == 8 * nside * nside


def test_pole_closed_forms_survey_examples():
    assert oracle.vec2pix(2, True, [0, 0, 1.0]) == 3
    assert oracle.vec2pix(64, True, [0, 0, 1.0]) == 4095
    assert oracle.vec2pix(1024, True, [0, 0, 1.0]) == 1048575
    assert oracle.vec2pix(2, False, [0, 0, -1.0]) == 44
    assert oracle.vec2pix(2, True, [0, 0, -1.0]) == 32
    assert oracle.vec2pix(64, False, [0, 0, -1.0]) == 49148
    assert oracle.vec2pix(64, True, [0, 0, -1.0]) == 32768


def _parse_angle(s):
    return float(eval(s, {"pi": math.pi}))


def test_published_healpy_values():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "healpy_ang2pix.txt")) if l.strip() and l[0] != "#"]
    assert len(rows) >= 9
    for nside, th, ph, pix in rows:
        assert oracle.ang2pix(int(nside), False, _parse_angle(th), _parse_angle(ph)) == int(pix), (nside, th, ph)


def test_nside1_ring_equals_nest():
    z, phi = ring_centres(1)
    for p in range(12):
        v = zphi_to_vec(z[p], phi[p])
        assert oracle.vec2pix(1, False, v) == p
        assert oracle.vec2pix(1, True, v) == p
    # (theta = pi/2, phi = 0) -> pixel 4 (SURVEY 8(c) O3 pin)
    assert oracle.ang2pix(1, False, math.pi / 2, 0.0) == 4


def _golden_ring2nest():
    lines = [l for l in open(os.path.join(GOLDEN, "ring2nest_nside2.txt")) if l.strip() and l[0] != "#"]
    return [int(x) for x in lines[0].split()], [int(x) for x in lines[1].split()]


def _independent_ring2nest(nside):
    """RING->NEST permutation from the two inverse maps only (match pixel centres)."""
    z, phi = ring_centres(nside)
    key = {}
    for p in range(len(z)):
        key[(round(z[p], 11), round(math.fmod(phi[p], 2 * math.pi), 9))] = p
    r2n = np.full(len(z), -1)
    for face in range(12):
        for ix in range(nside):
            for iy in range(nside):
                zz, pp = face_point(face, (ix + 0.5) / nside, (iy + 0.5) / nside)
                r = key[(round(zz, 11), round(math.fmod(pp, 2 * math.pi), 9))]
                r2n[r] = nest_index(nside, face, ix, iy)
    return r2n


def test_ring2nest_golden_nside2():
    g2, g16 = _golden_ring2nest()
    assert list(_independent_ring2nest(2)) == g2
    z, phi = ring_centres(2)
    assert [oracle.vec2pix(2, True, zphi_to_vec(z[p], phi[p])) for p in range(48)] == g2
    z, phi = ring_centres(16)
    assert [oracle.vec2pix(16, True, zphi_to_vec(z[p], phi[p])) for p in range(10)] == g16


@pytest.mark.parametrize("nside", [1, 2, 4, 8, 16])
def test_ring_centres_round_trip_and_bijection(nside):
    z, phi = ring_centres(nside)
    npix = 12 * nside * nside
    assert len(z) == npix
    nest = []
    for p in range(npix):
        v = zphi_to_vec(z[p], phi[p])
        assert oracle.vec2pix(nside, False, v) == p
        nest.append(oracle.vec2pix(nside, True, v))
    assert sorted(nest) == list(range(npix))  # RING -> NEST is a permutation
    assert nest == list(_independent_ring2nest(nside))


@pytest.mark.parametrize("nside", [1, 2, 4, 8, 16])
def test_brute_force_interior_points(nside):
    """7x7 interior points of every NEST pixel (from the inverse projection) map to that
    pixel in NEST and to the matching pixel in RING (SURVEY 8(c) 'O3 brute force')."""
    r2n = _independent_ring2nest(nside)
    n2r = np.empty_like(r2n)
    n2r[r2n] = np.arange(len(r2n))
    fr = np.linspace(0.03, 0.97, 7)
    for face in range(12):
        for ix in range(nside):
            for iy in range(nside):
                pn = nest_index(nside, face, ix, iy)
                for fx in fr:
                    for fy in fr:
                        v = zphi_to_vec(*face_point(face, (ix + fx) / nside, (iy + fy) / nside))
                        assert oracle.vec2pix(nside, True, v) == pn
                        assert oracle.vec2pix(nside, False, v) == n2r[pn]


def test_large_nside_centre_round_trip():
    """Random RING pixel centres at nside 4096 map back to themselves (closed-form centres)."""
    nside = 4096
    rng = np.random.default_rng(5)
    N = nside
    for _ in range(3000):
        i = int(rng.integers(1, 4 * N))
        if i < N:
            j = int(rng.integers(1, 4 * i + 1)); z = 1 - i * i / (3.0 * N * N); ph = math.pi / (2 * i) * (j - 0.5)
            p = 2 * i * (i - 1) + j - 1
        elif i <= 3 * N:
            f = 1.0 if (i + N) % 2 else 0.5
            j = int(rng.integers(1, 4 * N + 1)); z = 4.0 / 3.0 - 2.0 * i / (3.0 * N); ph = math.pi / (2 * N) * (j - f)
            p = 2 * N * (N - 1) + 4 * N * (i - N) + j - 1
        else:
            ii = 4 * N - i
            j = int(rng.integers(1, 4 * ii + 1)); z = -(1 - ii * ii / (3.0 * N * N)); ph = math.pi / (2 * ii) * (j - 0.5)
            p = 12 * N * N - 2 * ii * (ii + 1) + j - 1
        assert oracle.vec2pix(nside, False, zphi_to_vec(z, ph)) == p


def test_equal_area_and_range():
    """Uniform directions fill the 12 N^2 pixels equally (Gorski 2005: equal area)."""
    rng = np.random.default_rng(6)
    nside = 4
    npix = 12 * nside * nside
    v = rng.normal(size=(200_000, 3))
    v /= np.linalg.norm(v, axis=1)[:, None]
    for nest in (False, True):
        pix = np.array([oracle.vec2pix(nside, nest, x) for x in v])
        assert pix.min() >= 0 and pix.max() < npix
        counts = np.bincount(pix, minlength=npix)
        expect = len(v) / npix
        assert np.all(np.abs(counts - expect) < 6 * math.sqrt(expect))


def test_nest_equals_ring2nest_of_ring_random():
    rng = np.random.default_rng(7)
    nside = 16
    r2n = _independent_ring2nest(nside)
    v = rng.normal(size=(20_000, 3))
    v /= np.linalg.norm(v, axis=1)[:, None]
    for x in v:
        assert oracle.vec2pix(nside, True, x) == r2n[oracle.vec2pix(nside, False, x)]


def test_near_boundary_classifier():
    # a pixel centre is interior; the equatorial 4-pixel vertex (1,0,0) is on a boundary
    z, phi = ring_centres(64)
    for p in (0, 100, 5000, 20000, 49151):
        assert not oracle.near_boundary(64, False, zphi_to_vec(z[p], phi[p]))
        assert not oracle.near_boundary(64, True, zphi_to_vec(z[p], phi[p]))
    assert oracle.near_boundary(64, False, [1.0, 0.0, 0.0])
    assert oracle.near_boundary(64, True, [1.0, 0.0, 0.0])
    # 5e-13 rad from the vertex is still 'near'; 1e-6 rad inside a pixel is not
    v = np.array([math.cos(5e-13), 0.0, math.sin(5e-13)])
    assert oracle.near_boundary(64, True, v)
    zz, pp = face_point(4, 0.5, 0.5)
    assert not oracle.near_boundary(1, True, zphi_to_vec(zz, pp))  # face centre = pixel centre at N=1
    assert oracle.near_boundary(2, True, zphi_to_vec(zz, pp))  # ... and a 4-pixel vertex at N=2
