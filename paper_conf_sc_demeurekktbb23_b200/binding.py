"""Thin ctypes binding of libtoastb200.so (include/toast_b200.h), same entry-point names.

Argument marshalling only: torch CUDA tensors -> device pointers, the current torch
stream -> cudaStream_t, host intervals -> a packed int64 array.  Every step of the path
runs in the library's kernels; there is NO CPU fallback — if the library is missing or a
tensor is not on the GPU this raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np
import torch

from . import _build

_lib = None

P = ctypes.c_void_p
I64 = ctypes.c_int64
I32 = ctypes.c_int
U8 = ctypes.c_uint8
D = ctypes.c_double


class ToastError(RuntimeError):
    pass


def lib_path() -> str:
    return _build.LIB


def load():
    """Load libtoastb200.so (built by __graft_entry__.build() / _build.build())."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("TOASTB200_LIB", _build.LIB)  # tuning experiments may point at a variant build
    if not os.path.exists(path):
        raise ToastError(f"{path} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                         "(there is no CPU fallback)")
    L = ctypes.CDLL(path)
    L.toast_last_error.restype = ctypes.c_char_p
    L.toast_version.restype = ctypes.c_char_p
    L.toast_last_fused_path.restype = ctypes.c_char_p
    L.toast_release.restype = I32
    L.toast_pointing_detector.argtypes = [P, P, P, P, P, I64, P, U8, I64, I64, P]
    L.toast_pixels_healpix.argtypes = [P, P, P, U8, P, P, P, I64, P, I64, I64, I32, I64, I64, P]
    L.toast_stokes_weights_iqu.argtypes = [P, P, P, P, P, P, D, P, I64, I64, I64, P]
    L.toast_build_noise_weighted.argtypes = [P, P, I64, I64, P, P, P, P, P, P, P, P, U8, P, P, U8, P, I64, I64, I64,
                                             P]
    L.toast_scan_map.argtypes = [P, I64, P, I64, P, P, P, P, P, P, P, I64, D, I32, I32, I64, I64, P]
    L.toast_pointing_to_map.argtypes = [P, P, P, P, D, P, P, P, U8, P, U8, P, I64, I64, I32, I64, P, I64, P, P, P, P,
                                        I64, I64, P]
    L.toast_pointing_to_tod.argtypes = [P, P, P, P, D, P, U8, P, I64, I64, I32, I64, P, I64, P, D, I32, I32, P, I64,
                                        I64, P]
    L.toast_stokes_weights_i.argtypes = [P, P, D, P, I64, I64, I64, P]
    L.toast_noise_weight.argtypes = [P, P, P, P, I64, I64, I64, P]
    L.toast_template_offset_add_to_signal.argtypes = [I64, P, P, P, P, P, I64, I64, I64, P]
    L.toast_template_offset_project_signal.argtypes = [I64, P, P, P, P, P, P, U8, P, I64, I64, I64, P]
    L.toast_template_offset_apply_diag_precond.argtypes = [P, P, P, I64, P]
    for name in ("toast_pointing_detector", "toast_pixels_healpix", "toast_stokes_weights_iqu",
                 "toast_build_noise_weighted", "toast_scan_map", "toast_pointing_to_map", "toast_pointing_to_tod",
                 "toast_stokes_weights_i", "toast_noise_weight", "toast_template_offset_add_to_signal",
                 "toast_template_offset_project_signal", "toast_template_offset_apply_diag_precond"):
        getattr(L, name).restype = I32
    _lib = L
    return L


EXPORTED = ("toast_last_error", "toast_version", "toast_last_fused_path", "toast_release", "toast_pointing_detector", "toast_pixels_healpix",
            "toast_stokes_weights_iqu", "toast_build_noise_weighted", "toast_scan_map", "toast_pointing_to_map",
            "toast_pointing_to_tod", "toast_stokes_weights_i", "toast_noise_weight",
            "toast_template_offset_add_to_signal", "toast_template_offset_project_signal",
            "toast_template_offset_apply_diag_precond")


def version() -> str:
    return load().toast_version().decode()


def last_fused_path() -> str:
    """How the last pointing_to_map call on this thread staged its inputs ("tma" / "cp.async (...)")."""
    return load().toast_last_fused_path().decode()


def release() -> None:
    load().toast_release()


def _check(rc: int, name: str):
    if rc != 0:
        msg = load().toast_last_error().decode()
        raise ToastError(f"{name} failed ({rc}): {msg}")


def _dev(t: Optional[torch.Tensor], dtype, name: str):
    """Device pointer of a contiguous CUDA tensor of `dtype` (None -> NULL)."""
    if t is None:
        return None
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise ToastError(f"{name} must be a CUDA tensor (no CPU fallback)")
    if t.dtype != dtype:
        raise ToastError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ToastError(f"{name} must be contiguous")
    return t.data_ptr()


def _stream(stream) -> Optional[int]:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


def intervals_host(intervals) -> np.ndarray:
    """[(first, last), ...] inclusive or an [n, 2] int64 array -> packed [n, 2] int64 host array."""
    if isinstance(intervals, np.ndarray) and intervals.dtype.names:
        a = np.stack([intervals["first"], intervals["last"]], axis=1).astype(np.int64)
    else:
        a = np.asarray(intervals, dtype=np.int64).reshape(-1, 2)
    return np.ascontiguousarray(a)


def _iv(intervals):
    a = intervals_host(intervals)
    return a, (a.ctypes.data if len(a) else None), len(a)


# ----------------------------------------------------------------------------- entries

def pointing_detector(fp_quats, boresight, intervals, quats, shared_flags=None, shared_flag_mask=0,
                      quat_index=None, stream=None):
    n_det, n_samp = fp_quats.shape[0], boresight.shape[0]
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_pointing_detector(_dev(fp_quats, torch.float64, "fp_quats"),
                                        _dev(boresight, torch.float64, "boresight"),
                                        _dev(quat_index, torch.int32, "quat_index"),
                                        _dev(quats, torch.float64, "quats"), ivp, niv,
                                        _dev(shared_flags, torch.uint8, "shared_flags"), shared_flag_mask, n_det,
                                        n_samp, _stream(stream))
    _check(rc, "toast_pointing_detector")
    return quats


def pixels_healpix(quats, intervals, nside, nest, n_pix_submap, pixels, hit_submaps=None, shared_flags=None,
                   shared_flag_mask=0, quat_index=None, pixel_index=None, n_det=None, stream=None):
    n_samp = quats.shape[1]
    n_det = quats.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_pixels_healpix(_dev(quat_index, torch.int32, "quat_index"), _dev(quats, torch.float64, "quats"),
                                     _dev(shared_flags, torch.uint8, "shared_flags"), shared_flag_mask,
                                     _dev(pixel_index, torch.int32, "pixel_index"),
                                     _dev(pixels, torch.int64, "pixels"), ivp, niv,
                                     _dev(hit_submaps, torch.uint8, "hit_submaps"), n_pix_submap, nside, int(nest),
                                     n_det, n_samp, _stream(stream))
    _check(rc, "toast_pixels_healpix")
    return pixels


def stokes_weights_iqu(quats, intervals, epsilon, cal, weights, hwp=None, quat_index=None, weight_index=None,
                       n_det=None, stream=None):
    n_samp = quats.shape[1]
    n_det = quats.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_stokes_weights_iqu(_dev(quat_index, torch.int32, "quat_index"),
                                         _dev(quats, torch.float64, "quats"),
                                         _dev(weight_index, torch.int32, "weight_index"),
                                         _dev(weights, torch.float64, "weights"), _dev(hwp, torch.float64, "hwp"),
                                         _dev(epsilon, torch.float64, "epsilon"), float(cal), ivp, niv, n_det, n_samp,
                                         _stream(stream))
    _check(rc, "toast_stokes_weights_iqu")
    return weights


def build_noise_weighted(zmap, global2local, n_pix_submap, pixels, weights, det_data, det_scale, intervals,
                         det_flags=None, det_flag_mask=0, shared_flags=None, shared_flag_mask=0, pixel_index=None,
                         weight_index=None, data_index=None, flag_index=None, n_det=None, stream=None):
    nnz = weights.shape[-1]
    n_samp = pixels.shape[1]
    n_det = pixels.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_build_noise_weighted(
        _dev(global2local, torch.int64, "global2local"), _dev(zmap, torch.float64, "zmap"), n_pix_submap, nnz,
        _dev(pixel_index, torch.int32, "pixel_index"), _dev(pixels, torch.int64, "pixels"),
        _dev(weight_index, torch.int32, "weight_index"), _dev(weights, torch.float64, "weights"),
        _dev(data_index, torch.int32, "data_index"), _dev(det_data, torch.float64, "det_data"),
        _dev(flag_index, torch.int32, "flag_index"), _dev(det_flags, torch.uint8, "det_flags"), det_flag_mask,
        _dev(det_scale, torch.float64, "det_scale"), _dev(shared_flags, torch.uint8, "shared_flags"),
        shared_flag_mask, ivp, niv, n_det, n_samp, _stream(stream))
    _check(rc, "toast_build_noise_weighted")
    return zmap


def scan_map(mapdata, global2local, n_pix_submap, pixels, weights, det_data, intervals, data_scale=1.0,
             should_zero=False, should_subtract=False, pixel_index=None, weight_index=None, data_index=None,
             n_det=None, stream=None):
    nnz = weights.shape[-1]
    n_samp = pixels.shape[1]
    n_det = pixels.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_scan_map(_dev(global2local, torch.int64, "global2local"), n_pix_submap,
                               _dev(mapdata, torch.float64, "mapdata"), nnz, _dev(data_index, torch.int32, "data_index"),
                               _dev(det_data, torch.float64, "det_data"), _dev(pixel_index, torch.int32, "pixel_index"),
                               _dev(pixels, torch.int64, "pixels"), _dev(weight_index, torch.int32, "weight_index"),
                               _dev(weights, torch.float64, "weights"), ivp, niv, float(data_scale), int(should_zero),
                               int(should_subtract), n_det, n_samp, _stream(stream))
    _check(rc, "toast_scan_map")
    return det_data


def pointing_to_map(fp_quats, boresight, epsilon, cal, det_scale, det_data, intervals, nside, nest, nnz,
                    global2local, n_pix_submap, zmap, hwp=None, det_flags=None, det_flag_mask=0, shared_flags=None,
                    shared_flag_mask=0, hit_submaps=None, pixels_out=None, weights_out=None, stream=None):
    n_det, n_samp = fp_quats.shape[0], boresight.shape[0]
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_pointing_to_map(
        _dev(fp_quats, torch.float64, "fp_quats"), _dev(boresight, torch.float64, "boresight"),
        _dev(hwp, torch.float64, "hwp"), _dev(epsilon, torch.float64, "epsilon"), float(cal),
        _dev(det_scale, torch.float64, "det_scale"), _dev(det_data, torch.float64, "det_data"),
        _dev(det_flags, torch.uint8, "det_flags"), det_flag_mask, _dev(shared_flags, torch.uint8, "shared_flags"),
        shared_flag_mask, ivp, niv, nside, int(nest), nnz, _dev(global2local, torch.int64, "global2local"),
        n_pix_submap, _dev(zmap, torch.float64, "zmap"), _dev(hit_submaps, torch.uint8, "hit_submaps"),
        _dev(pixels_out, torch.int64, "pixels_out"), _dev(weights_out, torch.float64, "weights_out"), n_det, n_samp,
        _stream(stream))
    _check(rc, "toast_pointing_to_map")
    return zmap


def pointing_to_tod(fp_quats, boresight, epsilon, cal, intervals, nside, nest, nnz, global2local, n_pix_submap,
                    mapdata, det_data, data_scale=1.0, should_zero=False, should_subtract=False, hwp=None,
                    shared_flags=None, shared_flag_mask=0, stream=None):
    """f1: fused A1 -> A2 -> A3 -> A5, scanning `mapdata` into `det_data` in place."""
    n_det, n_samp = fp_quats.shape[0], boresight.shape[0]
    keep, ivp, niv = _iv(intervals)
    rc = load().toast_pointing_to_tod(
        _dev(fp_quats, torch.float64, "fp_quats"), _dev(boresight, torch.float64, "boresight"),
        _dev(hwp, torch.float64, "hwp"), _dev(epsilon, torch.float64, "epsilon"), float(cal),
        _dev(shared_flags, torch.uint8, "shared_flags"), shared_flag_mask, ivp, niv, nside, int(nest), nnz,
        _dev(global2local, torch.int64, "global2local"), n_pix_submap, _dev(mapdata, torch.float64, "mapdata"),
        float(data_scale), int(should_zero), int(should_subtract), _dev(det_data, torch.float64, "det_data"), n_det,
        n_samp, _stream(stream))
    _check(rc, "toast_pointing_to_tod")
    return det_data


def stokes_weights_i(weights, cal, intervals, n_det=None, weight_index=None, stream=None):
    n_det = weights.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    _check(load().toast_stokes_weights_i(_dev(weight_index, torch.int32, "weight_index"),
                                         _dev(weights, torch.float64, "weights"), float(cal), ivp, niv, n_det,
                                         weights.shape[1], _stream(stream)), "toast_stokes_weights_i")
    return weights


def noise_weight(det_data, det_weights, intervals, data_index=None, n_det=None, stream=None):
    n_det = det_weights.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    _check(load().toast_noise_weight(_dev(data_index, torch.int32, "data_index"),
                                     _dev(det_data, torch.float64, "det_data"),
                                     _dev(det_weights, torch.float64, "det_weights"), ivp, niv, n_det,
                                     det_data.shape[1], _stream(stream)), "toast_noise_weight")
    return det_data


def template_offset_add_to_signal(step_length, amp_offset, amplitudes, det_data, intervals, data_index=None,
                                  n_det=None, stream=None):
    n_det = amp_offset.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    _check(load().toast_template_offset_add_to_signal(
        int(step_length), _dev(amp_offset, torch.int64, "amp_offset"), _dev(amplitudes, torch.float64, "amplitudes"),
        _dev(data_index, torch.int32, "data_index"), _dev(det_data, torch.float64, "det_data"), ivp, niv, n_det,
        det_data.shape[1], _stream(stream)), "toast_template_offset_add_to_signal")
    return det_data


def template_offset_project_signal(step_length, amp_offset, amplitudes, det_data, intervals, det_flags=None,
                                   det_flag_mask=0, data_index=None, flag_index=None, n_det=None, stream=None):
    n_det = amp_offset.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    _check(load().toast_template_offset_project_signal(
        int(step_length), _dev(amp_offset, torch.int64, "amp_offset"), _dev(amplitudes, torch.float64, "amplitudes"),
        _dev(data_index, torch.int32, "data_index"), _dev(det_data, torch.float64, "det_data"),
        _dev(flag_index, torch.int32, "flag_index"), _dev(det_flags, torch.uint8, "det_flags"), det_flag_mask, ivp,
        niv, n_det, det_data.shape[1], _stream(stream)), "toast_template_offset_project_signal")
    return amplitudes


def template_offset_apply_diag_precond(offset_var, amp_in, amp_out, stream=None):
    _check(load().toast_template_offset_apply_diag_precond(
        _dev(offset_var, torch.float64, "offset_var"), _dev(amp_in, torch.float64, "amp_in"),
        _dev(amp_out, torch.float64, "amp_out"), amp_in.numel(), _stream(stream)),
        "toast_template_offset_apply_diag_precond")
    return amp_out


def pointing_to_map_raw(args: tuple):
    """Call toast_pointing_to_map with a pre-marshalled argument tuple (bench inner loop)."""
    _check(load().toast_pointing_to_map(*args), "toast_pointing_to_map")
