"""CPU fp64 ORACLE for the TOAST pointing->map hot path — TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product path in
``paper_conf_sc_demeurekktbb23_b200`` never imports it, and it imports nothing
from there.

The arithmetic lives in ``toast_oracle.c`` (plain C, fp64, det -> interval ->
sample loops, built with ``-ffp-contract=off``); each function there cites the
PAPER.md passage it follows.  This module is argument marshalling (numpy ->
ctypes) only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "toast_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

GCC_FLAGS = ["-O2", "-fPIC", "-shared", "-std=c11", "-D_DEFAULT_SOURCE", "-ffp-contract=off",
             "-fno-fast-math", "-fopenmp", "-Wall"]

INTERVAL_DTYPE = np.dtype([("first", np.int64), ("last", np.int64)])


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (no-op when up to date)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *GCC_FLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
        _declare(_lib)
    return _lib


P = ctypes.c_void_p
I64 = ctypes.c_int64
U8 = ctypes.c_uint8
D = ctypes.c_double
INT = ctypes.c_int


def _declare(L):
    L.oracle_quat_mul.argtypes = [P, P, P]
    L.oracle_quat_rotate.argtypes = [P, P, P]
    L.oracle_loc2pix.argtypes = [I64, INT, D, D, D]
    L.oracle_loc2pix.restype = I64
    L.oracle_vec2pix.argtypes = [I64, INT, P]
    L.oracle_vec2pix.restype = I64
    L.oracle_near_boundary.argtypes = [I64, INT, P, D]
    L.oracle_near_boundary.restype = INT
    L.oracle_stokes_iqu.argtypes = [P, D, D, D, P]
    L.oracle_stokes_iqu_ex.argtypes = [P, INT, D, D, INT, D, D, P]
    L.oracle_stokes_weights_iqu_ex.argtypes = [P, P, P, P, P, P, P, INT, D, P, I64, I64, I64]
    L.oracle_pointing_detector.argtypes = [P, P, P, P, P, I64, P, U8, I64, I64]
    L.oracle_pixels_healpix.argtypes = [P, P, P, U8, P, P, P, I64, P, I64, I64, INT, I64, I64]
    L.oracle_stokes_weights_iqu.argtypes = [P, P, P, P, P, P, D, P, I64, I64, I64]
    L.oracle_build_noise_weighted.argtypes = [P, P, I64, I64, P, P, P, P, P, P, P, P, U8, P, P, U8, P, I64,
                                              I64, I64, P]
    L.oracle_scan_map.argtypes = [P, I64, P, I64, P, P, P, P, P, P, P, I64, D, INT, INT, I64, I64, P]
    L.oracle_pointing_to_map.argtypes = [P, P, P, P, D, P, P, P, U8, P, U8, P, I64, I64, INT, I64, P, I64, P, P,
                                         P, P, I64, I64, P]
    L.oracle_pointing_to_map_ex.argtypes = [P, P, P, P, D, P, P, P, U8, P, U8, P, I64, I64, INT, I64, P, I64, P,
                                            P, P, P, I64, I64, P, P, INT, P]
    L.oracle_pointing_to_map_omp.argtypes = [P, P, P, P, D, P, P, P, U8, P, U8, P, I64, I64, INT, I64, P, I64,
                                             P, I64, I64, INT]
    L.oracle_pointing_to_map_omp.restype = INT
    L.oracle_det_sample_probe.argtypes = [P, P, D, D, D, INT, I64, INT, P, P, P]
    L.oracle_det_sample_probe_ex.argtypes = [P, P, INT, D, D, INT, D, D, INT, I64, INT, P, P, P]
    L.oracle_pointing_to_tod.argtypes = [P, P, P, P, D, P, U8, P, I64, I64, INT, I64, P, I64, P, D, INT, INT, P, I64,
                                         I64, P]
    L.oracle_pointing_to_tod_ex.argtypes = [P, P, P, P, D, P, U8, P, I64, I64, INT, I64, P, I64, P, D, INT, INT, P,
                                            I64, I64, P, P, INT]


def _p(a):
    """Pointer of a C-contiguous numpy array (None -> NULL)."""
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"], "oracle inputs must be C-contiguous"
    return a.ctypes.data


def _arr(a, dtype):
    return None if a is None else np.ascontiguousarray(a, dtype=dtype)


def intervals_array(intervals) -> np.ndarray:
    """[(first, last), ...] inclusive -> structured int64 array."""
    a = np.zeros(len(intervals), dtype=INTERVAL_DTYPE)
    if len(intervals):
        arr = np.asarray(intervals, dtype=np.int64).reshape(-1, 2)
        a["first"], a["last"] = arr[:, 0], arr[:, 1]
    return a


# ----------------------------------------------------------------------------- primitives

def quat_mul(p, q):
    p = _arr(p, np.float64); q = _arr(q, np.float64); r = np.zeros(4)
    lib().oracle_quat_mul(_p(p), _p(q), _p(r))
    return r


def quat_rotate(q, v):
    q = _arr(q, np.float64); v = _arr(v, np.float64); r = np.zeros(3)
    lib().oracle_quat_rotate(_p(q), _p(v), _p(r))
    return r


def vec2pix(nside: int, nest: bool, v) -> int:
    v = _arr(v, np.float64)
    return int(lib().oracle_vec2pix(nside, int(nest), _p(v)))


def ang2pix(nside: int, nest: bool, theta: float, phi: float) -> int:
    """HEALPix ang2pix with z = cos(theta) (as healpy feeds loc2pix)."""
    z = np.cos(theta)
    sth = np.sin(theta)
    return int(lib().oracle_loc2pix(nside, int(nest), float(z), float(phi), float(sth) if abs(z) >= 0.99 else 0.0))


def near_boundary(nside: int, nest: bool, v, delta: float = 1.1e-12) -> bool:
    v = _arr(v, np.float64)
    return bool(lib().oracle_near_boundary(nside, int(nest), _p(v), delta))


def stokes_iqu(q, hwp_angle, epsilon: float, cal: float, gamma: float = 0.0, iau: bool = False):
    """Weights of one det-sample; hwp_angle None = no HWP (then gamma has no effect, reading R3)."""
    q = _arr(q, np.float64); w = np.zeros(3)
    eta = (1.0 - epsilon) / (1.0 + epsilon)
    lib().oracle_stokes_iqu_ex(_p(q), int(hwp_angle is not None), 0.0 if hwp_angle is None else float(hwp_angle),
                               float(gamma), int(bool(iau)), eta, cal, _p(w))
    return w


def det_sample_probe(fp_q, bore_q, hwp_angle, epsilon, cal, flagged, nside, nest, gamma=0.0, iau=False):
    """One det-sample through A1->A2->A3: returns (pix, weights[3], dir[3]).  hwp_angle None = no
    HWP (identical to 0.0 unless gamma != 0, reading R3)."""
    fp_q = _arr(fp_q, np.float64); bore_q = _arr(bore_q, np.float64)
    pix = np.zeros(1, np.int64); w = np.zeros(3); d = np.zeros(3)
    lib().oracle_det_sample_probe_ex(_p(fp_q), _p(bore_q), int(hwp_angle is not None),
                                     0.0 if hwp_angle is None else float(hwp_angle), float(gamma), int(bool(iau)),
                                     float(epsilon), float(cal), int(bool(flagged)), nside, int(nest), _p(pix), _p(w),
                                     _p(d))
    return int(pix[0]), w, d


# ----------------------------------------------------------------------------- the six entries

def pointing_detector(fp_quats, boresight, intervals, shared_flags=None, shared_flag_mask=0, quat_index=None,
                      quats=None, n_rows=None):
    fp = _arr(fp_quats, np.float64); bore = _arr(boresight, np.float64)
    n_det, n_samp = fp.shape[0], bore.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    qi = _arr(quat_index, np.int32)
    if quats is None:
        quats = np.zeros((n_rows or n_det, n_samp, 4))
    sf = _arr(shared_flags, np.uint8)
    lib().oracle_pointing_detector(_p(fp), _p(bore), _p(qi), _p(quats), _p(iv), len(iv), _p(sf),
                                   shared_flag_mask, n_det, n_samp)
    return quats


def pixels_healpix(quats, intervals, nside, nest, n_pix_submap, shared_flags=None, shared_flag_mask=0,
                   quat_index=None, pixel_index=None, pixels=None, hit_submaps=None, n_det=None):
    quats = _arr(quats, np.float64)
    n_samp = quats.shape[1]
    n_det = n_det if n_det is not None else quats.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    if pixels is None:
        pixels = np.full((n_det, n_samp), -7, dtype=np.int64)
    if hit_submaps is None:
        hit_submaps = np.zeros(12 * nside * nside // n_pix_submap, np.uint8)
    lib().oracle_pixels_healpix(_p(_arr(quat_index, np.int32)), _p(quats), _p(_arr(shared_flags, np.uint8)),
                                shared_flag_mask, _p(_arr(pixel_index, np.int32)), _p(pixels), _p(iv), len(iv),
                                _p(hit_submaps), n_pix_submap, nside, int(nest), n_det, n_samp)
    return pixels, hit_submaps


def stokes_weights_iqu(quats, intervals, epsilon, cal, hwp=None, quat_index=None, weight_index=None,
                       weights=None, n_det=None, gamma=None, iau=False):
    quats = _arr(quats, np.float64)
    n_samp = quats.shape[1]
    n_det = n_det if n_det is not None else quats.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    if weights is None:
        weights = np.zeros((n_det, n_samp, 3))
    lib().oracle_stokes_weights_iqu_ex(_p(_arr(quat_index, np.int32)), _p(quats), _p(_arr(weight_index, np.int32)),
                                       _p(weights), _p(_arr(hwp, np.float64)), _p(_arr(epsilon, np.float64)),
                                       _p(_arr(gamma, np.float64)), int(bool(iau)), float(cal), _p(iv), len(iv),
                                       n_det, n_samp)
    return weights


def build_noise_weighted(zmap, global2local, n_pix_submap, pixels, weights, det_data, det_scale, intervals,
                         det_flags=None, det_flag_mask=0, shared_flags=None, shared_flag_mask=0,
                         pixel_index=None, weight_index=None, data_index=None, flag_index=None, n_det=None,
                         absmap=None):
    pixels = _arr(pixels, np.int64); weights = _arr(weights, np.float64); det_data = _arr(det_data, np.float64)
    nnz = weights.shape[-1]
    n_samp = pixels.shape[1]
    n_det = n_det if n_det is not None else pixels.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    assert zmap.dtype == np.float64 and zmap.flags["C_CONTIGUOUS"]
    lib().oracle_build_noise_weighted(_p(_arr(global2local, np.int64)), _p(zmap), n_pix_submap, nnz,
                                      _p(_arr(pixel_index, np.int32)), _p(pixels), _p(_arr(weight_index, np.int32)),
                                      _p(weights), _p(_arr(data_index, np.int32)), _p(det_data),
                                      _p(_arr(flag_index, np.int32)), _p(_arr(det_flags, np.uint8)), det_flag_mask,
                                      _p(_arr(det_scale, np.float64)), _p(_arr(shared_flags, np.uint8)),
                                      shared_flag_mask, _p(iv), len(iv), n_det, n_samp, _p(absmap))
    return zmap


def scan_map(mapdata, global2local, n_pix_submap, pixels, weights, det_data, intervals, data_scale=1.0,
             should_zero=False, should_subtract=False, pixel_index=None, weight_index=None, data_index=None,
             n_det=None, bscale=None):
    pixels = _arr(pixels, np.int64); weights = _arr(weights, np.float64); mapdata = _arr(mapdata, np.float64)
    nnz = weights.shape[-1]
    n_samp = pixels.shape[1]
    n_det = n_det if n_det is not None else pixels.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    assert det_data.dtype == np.float64 and det_data.flags["C_CONTIGUOUS"]
    lib().oracle_scan_map(_p(_arr(global2local, np.int64)), n_pix_submap, _p(mapdata), nnz,
                          _p(_arr(data_index, np.int32)), _p(det_data), _p(_arr(pixel_index, np.int32)), _p(pixels),
                          _p(_arr(weight_index, np.int32)), _p(weights), _p(iv), len(iv), float(data_scale),
                          int(should_zero), int(should_subtract), n_det, n_samp, _p(bscale))
    return det_data


def pointing_to_map(fp_quats, boresight, epsilon, cal, det_scale, det_data, intervals, nside, nest, nnz,
                    global2local, n_pix_submap, zmap=None, hwp=None, det_flags=None, det_flag_mask=0,
                    shared_flags=None, shared_flag_mask=0, hit_submaps=None, pixels_out=None, weights_out=None,
                    absmap=None, gamma=None, iau=False, t2map=None):
    """A6.  absmap (optional, zmap's shape) += |terms| (T4 scale); t2map (optional) += the T2
    weight tolerance of each Q/U term propagated through |det_scale tod| (T4)."""
    fp = _arr(fp_quats, np.float64); bore = _arr(boresight, np.float64)
    det_data = _arr(det_data, np.float64)
    n_det, n_samp = fp.shape[0], bore.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    g2l = _arr(global2local, np.int64)
    if zmap is None:
        zmap = np.zeros((int(g2l.max()) + 1, n_pix_submap, nnz))
    lib().oracle_pointing_to_map_ex(_p(fp), _p(bore), _p(_arr(hwp, np.float64)), _p(_arr(epsilon, np.float64)),
                                    float(cal), _p(_arr(det_scale, np.float64)), _p(det_data),
                                    _p(_arr(det_flags, np.uint8)), det_flag_mask, _p(_arr(shared_flags, np.uint8)),
                                    shared_flag_mask, _p(iv), len(iv), nside, int(nest), nnz, _p(g2l), n_pix_submap,
                                    _p(zmap), _p(hit_submaps), _p(pixels_out), _p(weights_out), n_det, n_samp,
                                    _p(absmap), _p(_arr(gamma, np.float64)), int(bool(iau)), _p(t2map))
    return zmap


def pointing_to_map_omp(fp_quats, boresight, epsilon, cal, det_scale, det_data, intervals, nside, nest, nnz,
                        global2local, n_pix_submap, zmap, hwp=None, det_flags=None, det_flag_mask=0,
                        shared_flags=None, shared_flag_mask=0, n_threads=0, n_det=None):
    """OpenMP timing mode (CPU baseline only).  Returns the thread count used."""
    fp = _arr(fp_quats, np.float64); bore = _arr(boresight, np.float64)
    n_det = n_det if n_det is not None else fp.shape[0]
    n_samp = bore.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    return int(lib().oracle_pointing_to_map_omp(
        _p(fp), _p(bore), _p(_arr(hwp, np.float64)), _p(_arr(epsilon, np.float64)), float(cal),
        _p(_arr(det_scale, np.float64)), _p(_arr(det_data, np.float64)), _p(_arr(det_flags, np.uint8)),
        det_flag_mask, _p(_arr(shared_flags, np.uint8)), shared_flag_mask, _p(iv), len(iv), nside, int(nest), nnz,
        _p(_arr(global2local, np.int64)), n_pix_submap, _p(zmap), n_det, n_samp, int(n_threads)))


def pointing_to_tod(fp_quats, boresight, epsilon, cal, intervals, nside, nest, nnz, global2local, n_pix_submap,
                    mapdata, det_data, data_scale=1.0, should_zero=False, should_subtract=False, hwp=None,
                    shared_flags=None, shared_flag_mask=0, bscale=None, gamma=None, iau=False):
    """f1: A1 -> A2 -> A3 -> A5 per det-sample (scan a map onto the timestream in place)."""
    fp = _arr(fp_quats, np.float64); bore = _arr(boresight, np.float64)
    n_det, n_samp = fp.shape[0], bore.shape[0]
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    assert det_data.dtype == np.float64 and det_data.flags["C_CONTIGUOUS"] and det_data.shape == (n_det, n_samp)
    lib().oracle_pointing_to_tod_ex(_p(fp), _p(bore), _p(_arr(hwp, np.float64)), _p(_arr(epsilon, np.float64)),
                                    float(cal), _p(_arr(shared_flags, np.uint8)), shared_flag_mask, _p(iv), len(iv),
                                    nside, int(nest), nnz, _p(_arr(global2local, np.int64)), n_pix_submap,
                                    _p(_arr(mapdata, np.float64)), float(data_scale), int(should_zero),
                                    int(should_subtract), _p(det_data), n_det, n_samp, _p(bscale),
                                    _p(_arr(gamma, np.float64)), int(bool(iau)))
    return det_data


# ----------------------------------------------------------------------------- NEXT rows (f2, f4)

def _declare_next(L):
    L.oracle_stokes_weights_i.argtypes = [P, P, D, P, I64, I64, I64]
    L.oracle_noise_weight.argtypes = [P, P, P, P, I64, I64, I64]
    L.oracle_template_offset_add_to_signal.argtypes = [I64, P, P, P, P, P, I64, I64, I64]
    L.oracle_template_offset_project_signal.argtypes = [I64, P, P, P, P, P, P, U8, P, I64, I64, I64]
    L.oracle_template_offset_apply_diag_precond.argtypes = [P, P, P, I64]


def _lib_next():
    L = lib()
    if not getattr(L, "_next_declared", False):
        _declare_next(L)
        L._next_declared = True
    return L


def stokes_weights_i(weights, cal, intervals, n_det, weight_index=None):
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    _lib_next().oracle_stokes_weights_i(_p(_arr(weight_index, np.int32)), _p(weights), float(cal), _p(iv), len(iv),
                                        n_det, weights.shape[1])
    return weights


def noise_weight(det_data, det_weights, intervals, data_index=None, n_det=None):
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    dw = _arr(det_weights, np.float64)
    n_det = dw.shape[0] if n_det is None else n_det
    _lib_next().oracle_noise_weight(_p(_arr(data_index, np.int32)), _p(det_data), _p(dw), _p(iv), len(iv), n_det,
                                    det_data.shape[1])
    return det_data


def offset_amplitude_counts(intervals, step_length):
    """Amplitudes per detector under reading O1: sum over intervals of ceil(len / step)."""
    return int(sum((l - f + 1 + step_length - 1) // step_length for f, l in intervals))


def template_offset_add_to_signal(step_length, amp_offset, amplitudes, det_data, intervals, data_index=None,
                                  n_det=None):
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    ao = _arr(amp_offset, np.int64)
    n_det = ao.shape[0] if n_det is None else n_det
    _lib_next().oracle_template_offset_add_to_signal(step_length, _p(ao), _p(_arr(amplitudes, np.float64)),
                                                     _p(_arr(data_index, np.int32)), _p(det_data), _p(iv), len(iv),
                                                     n_det, det_data.shape[1])
    return det_data


def template_offset_project_signal(step_length, amp_offset, amplitudes, det_data, intervals, det_flags=None,
                                   det_flag_mask=0, data_index=None, flag_index=None, n_det=None):
    iv = intervals_array(intervals) if not isinstance(intervals, np.ndarray) else intervals
    ao = _arr(amp_offset, np.int64)
    n_det = ao.shape[0] if n_det is None else n_det
    dd = _arr(det_data, np.float64)
    _lib_next().oracle_template_offset_project_signal(step_length, _p(ao), _p(amplitudes),
                                                      _p(_arr(data_index, np.int32)), _p(dd),
                                                      _p(_arr(flag_index, np.int32)), _p(_arr(det_flags, np.uint8)),
                                                      det_flag_mask, _p(iv), len(iv), n_det, dd.shape[1])
    return amplitudes


def template_offset_apply_diag_precond(offset_var, amp_in):
    ov = _arr(offset_var, np.float64); ai = _arr(amp_in, np.float64)
    out = np.zeros_like(ai)
    _lib_next().oracle_template_offset_apply_diag_precond(_p(ov), _p(ai), _p(out), ai.shape[0])
    return out
