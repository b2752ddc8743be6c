"""Independent formulations used to PIN the oracle (tests only).

Nothing here shares arithmetic with oracle/toast_oracle.c:
  * rotations: Rodrigues' formula R = I + sin(a) K + (1 - cos(a)) K^2 from an
    axis-angle pair (not quaternion algebra);
  * HEALPix: the INVERSE maps of Gorski et al. 2005 (ref [16]):
    ring pixel centres (their Eqs. 4-9 / Sec. 4) and the continuous face
    coordinates -> (z, phi) map of the NESTED faces — no floor logic, no
    forward vec2pix;
  * Stokes angle: the geometric definition of the polarisation angle in the
    local (e_theta, e_phi) frame at the pointing direction.
"""
from __future__ import annotations

import math

import numpy as np

# ----------------------------------------------------------------------------- rotations


def rodrigues(axis, angle):
    n = np.asarray(axis, dtype=np.float64)
    n = n / np.linalg.norm(n)
    k = np.array([[0, -n[2], n[1]], [n[2], 0, -n[0]], [-n[1], n[0], 0]])
    return np.eye(3) + math.sin(angle) * k + (1 - math.cos(angle)) * (k @ k)


def axis_angle_quat(axis, angle):
    """Unit quaternion [x,y,z,w] of a rotation by `angle` about `axis` (definition)."""
    n = np.asarray(axis, dtype=np.float64)
    n = n / np.linalg.norm(n)
    return np.array([*(math.sin(angle / 2) * n), math.cos(angle / 2)])


def random_axis_angle(rng):
    v = rng.normal(size=3)
    return v / np.linalg.norm(v), rng.uniform(-math.pi, math.pi)


# ----------------------------------------------------------------------------- HEALPix inverse maps

JRLL = [2, 2, 2, 2, 3, 3, 3, 3, 4, 4, 4, 4]
JPLL = [1, 3, 5, 7, 0, 2, 4, 6, 1, 3, 5, 7]


def ring_centres(nside: int):
    """(z, phi) of every RING pixel centre, index = RING pixel number
    (Gorski et al. 2005 Sec. 4: polar caps z = 1 - i^2/(3N^2), phi = pi/(2i)(j - 1/2);
    belt z = 4/3 - 2i/(3N), phi = pi/(2N)(j - f), f = 1 if i + N is odd else 1/2,
    numbering each ring's first pixel from phi = 0 as HEALPix/healpy do)."""
    N = nside
    zs, ph = [], []
    for i in range(1, 4 * N):
        if i < N:
            for j in range(1, 4 * i + 1):
                zs.append(1 - i * i / (3.0 * N * N)); ph.append(math.pi / (2 * i) * (j - 0.5))
        elif i <= 3 * N:
            f = 1.0 if (i + N) % 2 else 0.5
            for j in range(1, 4 * N + 1):
                zs.append(4.0 / 3.0 - 2.0 * i / (3.0 * N)); ph.append(math.pi / (2 * N) * (j - f))
        else:
            ii = 4 * N - i
            for j in range(1, 4 * ii + 1):
                zs.append(-(1 - ii * ii / (3.0 * N * N))); ph.append(math.pi / (2 * ii) * (j - 0.5))
    return np.array(zs), np.array(ph)


def face_point(face: int, x: float, y: float):
    """Continuous face coordinates (x, y in [0,1]) -> (z, phi) (HEALPix inverse projection)."""
    jr = JRLL[face] - x - y
    if jr < 1:
        nr = jr; z = 1 - nr * nr / 3.0
    elif jr > 3:
        nr = 4 - jr; z = nr * nr / 3.0 - 1
    else:
        nr = 1.0; z = (2 - jr) * 2.0 / 3.0
    tmp = JPLL[face] * nr + x - y
    if tmp < 0:
        tmp += 8
    if tmp >= 8:
        tmp -= 8
    phi = 0.0 if nr < 1e-15 else (math.pi / 4) * tmp / nr
    return z, phi


def zphi_to_vec(z, phi):
    s = math.sqrt(max(0.0, (1 - z) * (1 + z)))
    return np.array([s * math.cos(phi), s * math.sin(phi), z])


def nest_index(nside: int, face: int, ix: int, iy: int) -> int:
    """NESTED index by the definition: face*N^2 + bit-interleave(ix -> even, iy -> odd)."""
    p = 0
    for b in range(int(math.log2(nside)) + 1):
        p |= ((ix >> b) & 1) << (2 * b)
        p |= ((iy >> b) & 1) << (2 * b + 1)
    return face * nside * nside + p


# ----------------------------------------------------------------------------- Stokes geometry


def psi_geometric(dir_, orient):
    """Polarisation angle of `orient` in the local frame at `dir_`:
    psi = atan2(o . e_phi, o . e_theta) + pi (the detector's 'x' axis measured
    from the meridian, reversed); returned mod 2 pi."""
    d = np.asarray(dir_); o = np.asarray(orient)
    theta = math.acos(max(-1.0, min(1.0, d[2])))
    phi = math.atan2(d[1], d[0])
    e_theta = np.array([math.cos(theta) * math.cos(phi), math.cos(theta) * math.sin(phi), -math.sin(theta)])
    e_phi = np.array([-math.sin(phi), math.cos(phi), 0.0])
    return math.atan2(float(o @ e_phi), float(o @ e_theta)) + math.pi
