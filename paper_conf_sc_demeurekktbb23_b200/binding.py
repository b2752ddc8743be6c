"""Thin ctypes binding of libtoastb200.so (include/toast_b200.h), same entry-point names.

Argument marshalling only: torch CUDA tensors -> device pointers, the tensors' device's current
torch stream -> cudaStream_t, host intervals -> a packed int64 array.  Every step of the path
runs in the library's kernels; there is NO CPU fallback — if the library is missing or a tensor
is not on the GPU this raises.  Shapes are checked here (the C ABI cannot see sizes), so a
mismatch raises instead of becoming an out-of-bounds device access, and every call runs on the
device its tensors live on (they must share one).
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


class MapOptions(ctypes.Structure):
    """toast_map_options_t (include/toast_b200.h)."""
    _fields_ = [("gamma", P), ("iau", I32), ("map_f32", I32), ("dropped", P)]


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
    L.toast_stokes_weights_iqu_ex.argtypes = [P, P, P, P, P, P, P, I32, D, P, I64, I64, I64, P]
    L.toast_build_noise_weighted.argtypes = [P, P, I64, I64, P, P, P, P, P, P, P, P, U8, P, P, U8, P, I64, I64, I64,
                                             P]
    L.toast_scan_map.argtypes = [P, I64, P, I64, P, P, P, P, P, P, P, I64, D, I32, I32, I64, I64, P]
    L.toast_pointing_to_map.argtypes = [P, P, P, P, D, P, P, P, U8, P, U8, P, I64, I64, I32, I64, P, I64, P, P, P, P,
                                        I64, I64, P]
    L.toast_pointing_to_map_ex.argtypes = [P, P, P, P, D, P, P, P, U8, P, U8, P, I64, I64, I32, I64, P, I64, P, P, P,
                                           P, I64, I64, ctypes.POINTER(MapOptions), P]
    L.toast_pointing_to_tod.argtypes = [P, P, P, P, D, P, U8, P, I64, I64, I32, I64, P, I64, P, D, I32, I32, P, I64,
                                        I64, P]
    L.toast_pointing_to_tod_ex.argtypes = [P, P, P, P, D, P, U8, P, I64, I64, I32, I64, P, I64, P, D, I32, I32, P,
                                           I64, I64, ctypes.POINTER(MapOptions), P]
    L.toast_stokes_weights_i.argtypes = [P, P, D, P, I64, I64, I64, P]
    L.toast_noise_weight.argtypes = [P, P, P, P, I64, I64, I64, P]
    L.toast_template_offset_add_to_signal.argtypes = [I64, P, P, P, P, P, I64, I64, I64, P]
    L.toast_template_offset_project_signal.argtypes = [I64, P, P, P, P, P, P, U8, P, I64, I64, I64, P]
    L.toast_template_offset_apply_diag_precond.argtypes = [P, P, P, I64, P]
    L.toast_synth_tod.argtypes = [P, P, P, I64, I64, ctypes.c_uint64, ctypes.c_uint64, P]
    L.toast_map_allreduce_nvls.argtypes = [P, I64, P, I32, I32, P]
    for name in EXPORTED[4:]:
        getattr(L, name).restype = I32
    _lib = L
    return L


EXPORTED = ("toast_last_error", "toast_version", "toast_last_fused_path", "toast_release", "toast_pointing_detector",
            "toast_pixels_healpix", "toast_stokes_weights_iqu", "toast_stokes_weights_iqu_ex",
            "toast_build_noise_weighted", "toast_scan_map", "toast_pointing_to_map", "toast_pointing_to_map_ex",
            "toast_pointing_to_tod", "toast_pointing_to_tod_ex", "toast_stokes_weights_i", "toast_noise_weight",
            "toast_template_offset_add_to_signal", "toast_template_offset_project_signal",
            "toast_template_offset_apply_diag_precond", "toast_synth_tod")


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


class _Call:
    """Collects the tensors of one call: dtype / contiguity / shape checks, one common device,
    and that device's current stream."""

    def __init__(self, name: str):
        self.name = name
        self.device = None

    def __call__(self, t: Optional[torch.Tensor], dtype, what: str, shape=None, min_numel=None):
        """Device pointer of a contiguous CUDA tensor of `dtype` (None -> NULL).  `shape`: the
        exact shape required (entries None = any); `min_numel`: a lower bound on the size."""
        if t is None:
            return None
        if not isinstance(t, torch.Tensor) or not t.is_cuda:
            raise ToastError(f"{self.name}: {what} must be a CUDA tensor (no CPU fallback)")
        if t.dtype != dtype:
            raise ToastError(f"{self.name}: {what} must be {dtype}, got {t.dtype}")
        if not t.is_contiguous():
            raise ToastError(f"{self.name}: {what} must be contiguous")
        if shape is not None:
            if t.dim() != len(shape) or any(s is not None and int(a) != int(s) for a, s in zip(t.shape, shape)):
                raise ToastError(f"{self.name}: {what} has shape {tuple(t.shape)}, expected "
                                 f"{tuple('*' if s is None else s for s in shape)}")
        if min_numel is not None and t.numel() < min_numel:
            raise ToastError(f"{self.name}: {what} has {t.numel()} elements, needs at least {min_numel}")
        if self.device is None:
            self.device = t.device
        elif t.device != self.device:
            raise ToastError(f"{self.name}: tensors on {self.device} and {t.device}; all must share one device")
        return t.data_ptr()

    def run(self, fn, *args, stream=None):
        """Call fn(*args, cudaStream_t) on the tensors' device with its current stream (or `stream`)."""
        dev = self.device if self.device is not None else torch.device("cuda", torch.cuda.current_device())
        with torch.cuda.device(dev):
            st = stream if stream is not None else torch.cuda.current_stream(dev)
            rc = fn(*args, st.cuda_stream)
        _check(rc, self.name)


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


def _rows(index, n_det, c, what):
    """Rows an index array can address (None: n_det)."""
    if index is None:
        return n_det
    c(index, torch.int32, what, shape=(n_det,))
    return int(index.max()) + 1 if n_det > 0 else 0


def _n_submap(nside, n_pix_submap):
    """Submaps of a valid geometry; None (shape unchecked here) when nside / n_pix_submap are
    invalid, so that the library's own validation reports them (TOAST_EINVAL)."""
    if nside < 1 or nside & (nside - 1) or n_pix_submap < 1 or (12 * nside * nside) % n_pix_submap:
        return None
    return 12 * nside * nside // n_pix_submap


def _map_shape(zmap, n_pix_submap, nnz):
    """[n_local][n_pix_submap][nnz]; a [1][1][nnz] placeholder is accepted for a map domain with
    no storage at all (global2local = -1 everywhere, e.g. a full sky at nside 2^29)."""
    if isinstance(zmap, torch.Tensor) and tuple(zmap.shape) == (1, 1, nnz):
        return (1, 1, nnz)
    return (None, n_pix_submap, nnz)


def _options(c, gamma, iau, map_f32, dropped, n_det):
    if gamma is None and not iau and not map_f32 and dropped is None:
        return None
    return MapOptions(c(gamma, torch.float64, "gamma", shape=(n_det,)), int(bool(iau)), int(bool(map_f32)),
                      c(dropped, torch.int64, "dropped", shape=(1,)))


# ----------------------------------------------------------------------------- entries

def pointing_detector(fp_quats, boresight, intervals, quats, shared_flags=None, shared_flag_mask=0,
                      quat_index=None, stream=None):
    c = _Call("toast_pointing_detector")
    n_det, n_samp = fp_quats.shape[0], boresight.shape[0]
    keep, ivp, niv = _iv(intervals)
    rows = _rows(quat_index, n_det, c, "quat_index")
    c.run(load().toast_pointing_detector, c(fp_quats, torch.float64, "fp_quats", shape=(n_det, 4)),
          c(boresight, torch.float64, "boresight", shape=(n_samp, 4)), c(quat_index, torch.int32, "quat_index"),
          c(quats, torch.float64, "quats", shape=(None, n_samp, 4), min_numel=rows * n_samp * 4), ivp, niv,
          c(shared_flags, torch.uint8, "shared_flags", shape=(n_samp,)), shared_flag_mask, n_det, n_samp,
          stream=stream)
    return quats


def pixels_healpix(quats, intervals, nside, nest, n_pix_submap, pixels, hit_submaps=None, shared_flags=None,
                   shared_flag_mask=0, quat_index=None, pixel_index=None, n_det=None, stream=None):
    c = _Call("toast_pixels_healpix")
    n_samp = quats.shape[1]
    n_det = quats.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    qrows = _rows(quat_index, n_det, c, "quat_index")
    prows = _rows(pixel_index, n_det, c, "pixel_index")
    c.run(load().toast_pixels_healpix, c(quat_index, torch.int32, "quat_index"),
          c(quats, torch.float64, "quats", shape=(None, n_samp, 4), min_numel=qrows * n_samp * 4),
          c(shared_flags, torch.uint8, "shared_flags", shape=(n_samp,)), shared_flag_mask,
          c(pixel_index, torch.int32, "pixel_index"),
          c(pixels, torch.int64, "pixels", shape=(None, n_samp), min_numel=prows * n_samp), ivp, niv,
          c(hit_submaps, torch.uint8, "hit_submaps", shape=(_n_submap(nside, n_pix_submap),)), n_pix_submap, nside,
          int(nest), n_det, n_samp, stream=stream)
    return pixels


def stokes_weights_iqu(quats, intervals, epsilon, cal, weights, hwp=None, quat_index=None, weight_index=None,
                       n_det=None, stream=None, gamma=None, iau=False):
    c = _Call("toast_stokes_weights_iqu")
    n_samp = quats.shape[1]
    n_det = quats.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    qrows = _rows(quat_index, n_det, c, "quat_index")
    wrows = _rows(weight_index, n_det, c, "weight_index")
    c.run(load().toast_stokes_weights_iqu_ex, c(quat_index, torch.int32, "quat_index"),
          c(quats, torch.float64, "quats", shape=(None, n_samp, 4), min_numel=qrows * n_samp * 4),
          c(weight_index, torch.int32, "weight_index"),
          c(weights, torch.float64, "weights", shape=(None, n_samp, 3), min_numel=wrows * n_samp * 3),
          c(hwp, torch.float64, "hwp", shape=(n_samp,)), c(epsilon, torch.float64, "epsilon", shape=(n_det,)),
          c(gamma, torch.float64, "gamma", shape=(n_det,)), int(bool(iau)), float(cal), ivp, niv, n_det, n_samp,
          stream=stream)
    return weights


def build_noise_weighted(zmap, global2local, n_pix_submap, pixels, weights, det_data, det_scale, intervals,
                         det_flags=None, det_flag_mask=0, shared_flags=None, shared_flag_mask=0, pixel_index=None,
                         weight_index=None, data_index=None, flag_index=None, n_det=None, stream=None):
    c = _Call("toast_build_noise_weighted")
    nnz = weights.shape[-1]
    n_samp = pixels.shape[1]
    n_det = pixels.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    prows = _rows(pixel_index, n_det, c, "pixel_index")
    wrows = _rows(weight_index, n_det, c, "weight_index")
    drows = _rows(data_index, n_det, c, "data_index")
    frows = _rows(flag_index, n_det, c, "flag_index")
    c.run(load().toast_build_noise_weighted,
          c(global2local, torch.int64, "global2local", shape=(None,)),
          c(zmap, torch.float64, "zmap", shape=(None, n_pix_submap, nnz)), n_pix_submap, nnz,
          c(pixel_index, torch.int32, "pixel_index"),
          c(pixels, torch.int64, "pixels", shape=(None, n_samp), min_numel=prows * n_samp),
          c(weight_index, torch.int32, "weight_index"),
          c(weights, torch.float64, "weights", shape=(None, n_samp, nnz), min_numel=wrows * n_samp * nnz),
          c(data_index, torch.int32, "data_index"),
          c(det_data, torch.float64, "det_data", shape=(None, n_samp), min_numel=drows * n_samp),
          c(flag_index, torch.int32, "flag_index"),
          c(det_flags, torch.uint8, "det_flags", shape=(None, n_samp), min_numel=frows * n_samp), det_flag_mask,
          c(det_scale, torch.float64, "det_scale", shape=(n_det,)),
          c(shared_flags, torch.uint8, "shared_flags", shape=(n_samp,)), shared_flag_mask, ivp, niv, n_det, n_samp,
          stream=stream)
    return zmap


def scan_map(mapdata, global2local, n_pix_submap, pixels, weights, det_data, intervals, data_scale=1.0,
             should_zero=False, should_subtract=False, pixel_index=None, weight_index=None, data_index=None,
             n_det=None, stream=None):
    c = _Call("toast_scan_map")
    nnz = weights.shape[-1]
    n_samp = pixels.shape[1]
    n_det = pixels.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    prows = _rows(pixel_index, n_det, c, "pixel_index")
    wrows = _rows(weight_index, n_det, c, "weight_index")
    drows = _rows(data_index, n_det, c, "data_index")
    c.run(load().toast_scan_map, c(global2local, torch.int64, "global2local", shape=(None,)), n_pix_submap,
          c(mapdata, torch.float64, "mapdata", shape=(None, n_pix_submap, nnz)), nnz,
          c(data_index, torch.int32, "data_index"),
          c(det_data, torch.float64, "det_data", shape=(None, n_samp), min_numel=drows * n_samp),
          c(pixel_index, torch.int32, "pixel_index"),
          c(pixels, torch.int64, "pixels", shape=(None, n_samp), min_numel=prows * n_samp),
          c(weight_index, torch.int32, "weight_index"),
          c(weights, torch.float64, "weights", shape=(None, n_samp, nnz), min_numel=wrows * n_samp * nnz), ivp, niv,
          float(data_scale), int(should_zero), int(should_subtract), n_det, n_samp, stream=stream)
    return det_data


def pointing_to_map(fp_quats, boresight, epsilon, cal, det_scale, det_data, intervals, nside, nest, nnz,
                    global2local, n_pix_submap, zmap, hwp=None, det_flags=None, det_flag_mask=0, shared_flags=None,
                    shared_flag_mask=0, hit_submaps=None, pixels_out=None, weights_out=None, stream=None, gamma=None,
                    iau=False, dropped=None):
    """A6: the fused entry.  `zmap` fp64, or float32 (the map_f32 option); `gamma` [n_det] / `iau`
    (reading R3); `dropped`: an int64 [1] device counter of skipped det-samples (debug)."""
    c = _Call("toast_pointing_to_map")
    n_det, n_samp = fp_quats.shape[0], boresight.shape[0]
    keep, ivp, niv = _iv(intervals)
    map_f32 = isinstance(zmap, torch.Tensor) and zmap.dtype == torch.float32
    opts = _options(c, gamma, iau, map_f32, dropped, n_det)
    c.run(load().toast_pointing_to_map_ex,
          c(fp_quats, torch.float64, "fp_quats", shape=(n_det, 4)),
          c(boresight, torch.float64, "boresight", shape=(n_samp, 4)), c(hwp, torch.float64, "hwp", shape=(n_samp,)),
          c(epsilon, torch.float64, "epsilon", shape=(n_det,)), float(cal),
          c(det_scale, torch.float64, "det_scale", shape=(n_det,)),
          c(det_data, torch.float64, "det_data", shape=(n_det, n_samp)),
          c(det_flags, torch.uint8, "det_flags", shape=(n_det, n_samp)), det_flag_mask,
          c(shared_flags, torch.uint8, "shared_flags", shape=(n_samp,)), shared_flag_mask, ivp, niv, nside,
          int(nest), nnz, c(global2local, torch.int64, "global2local", shape=(_n_submap(nside, n_pix_submap),)),
          n_pix_submap,
          c(zmap, torch.float32 if map_f32 else torch.float64, "zmap", shape=_map_shape(zmap, n_pix_submap, nnz)),
          c(hit_submaps, torch.uint8, "hit_submaps", shape=(_n_submap(nside, n_pix_submap),)),
          c(pixels_out, torch.int64, "pixels_out", shape=(n_det, n_samp)),
          c(weights_out, torch.float64, "weights_out", shape=(n_det, n_samp, nnz)), n_det, n_samp,
          None if opts is None else ctypes.byref(opts), stream=stream)
    return zmap


def pointing_to_tod(fp_quats, boresight, epsilon, cal, intervals, nside, nest, nnz, global2local, n_pix_submap,
                    mapdata, det_data, data_scale=1.0, should_zero=False, should_subtract=False, hwp=None,
                    shared_flags=None, shared_flag_mask=0, stream=None, gamma=None, iau=False):
    """f1: fused A1 -> A2 -> A3 -> A5, scanning `mapdata` (fp64 or float32) into `det_data` in place."""
    c = _Call("toast_pointing_to_tod")
    n_det, n_samp = fp_quats.shape[0], boresight.shape[0]
    keep, ivp, niv = _iv(intervals)
    map_f32 = isinstance(mapdata, torch.Tensor) and mapdata.dtype == torch.float32
    opts = _options(c, gamma, iau, map_f32, None, n_det)
    c.run(load().toast_pointing_to_tod_ex,
          c(fp_quats, torch.float64, "fp_quats", shape=(n_det, 4)),
          c(boresight, torch.float64, "boresight", shape=(n_samp, 4)), c(hwp, torch.float64, "hwp", shape=(n_samp,)),
          c(epsilon, torch.float64, "epsilon", shape=(n_det,)), float(cal),
          c(shared_flags, torch.uint8, "shared_flags", shape=(n_samp,)), shared_flag_mask, ivp, niv, nside,
          int(nest), nnz, c(global2local, torch.int64, "global2local", shape=(_n_submap(nside, n_pix_submap),)),
          n_pix_submap,
          c(mapdata, torch.float32 if map_f32 else torch.float64, "mapdata", shape=(None, n_pix_submap, nnz)),
          float(data_scale), int(should_zero), int(should_subtract),
          c(det_data, torch.float64, "det_data", shape=(n_det, n_samp)), n_det, n_samp,
          None if opts is None else ctypes.byref(opts), stream=stream)
    return det_data


def stokes_weights_i(weights, cal, intervals, n_det=None, weight_index=None, stream=None):
    c = _Call("toast_stokes_weights_i")
    n_det = weights.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rows = _rows(weight_index, n_det, c, "weight_index")
    c.run(load().toast_stokes_weights_i, c(weight_index, torch.int32, "weight_index"),
          c(weights, torch.float64, "weights", shape=(None, weights.shape[1]), min_numel=rows * weights.shape[1]),
          float(cal), ivp, niv, n_det, weights.shape[1], stream=stream)
    return weights


def noise_weight(det_data, det_weights, intervals, data_index=None, n_det=None, stream=None):
    c = _Call("toast_noise_weight")
    n_det = det_weights.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rows = _rows(data_index, n_det, c, "data_index")
    c.run(load().toast_noise_weight, c(data_index, torch.int32, "data_index"),
          c(det_data, torch.float64, "det_data", shape=(None, det_data.shape[1]), min_numel=rows * det_data.shape[1]),
          c(det_weights, torch.float64, "det_weights", shape=(n_det,)), ivp, niv, n_det, det_data.shape[1],
          stream=stream)
    return det_data


def template_offset_add_to_signal(step_length, amp_offset, amplitudes, det_data, intervals, data_index=None,
                                  n_det=None, stream=None):
    c = _Call("toast_template_offset_add_to_signal")
    n_det = amp_offset.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    rows = _rows(data_index, n_det, c, "data_index")
    c.run(load().toast_template_offset_add_to_signal, int(step_length),
          c(amp_offset, torch.int64, "amp_offset", shape=(n_det,)), c(amplitudes, torch.float64, "amplitudes"),
          c(data_index, torch.int32, "data_index"),
          c(det_data, torch.float64, "det_data", shape=(None, det_data.shape[1]), min_numel=rows * det_data.shape[1]),
          ivp, niv, n_det, det_data.shape[1], stream=stream)
    return det_data


def template_offset_project_signal(step_length, amp_offset, amplitudes, det_data, intervals, det_flags=None,
                                   det_flag_mask=0, data_index=None, flag_index=None, n_det=None, stream=None):
    c = _Call("toast_template_offset_project_signal")
    n_det = amp_offset.shape[0] if n_det is None else n_det
    keep, ivp, niv = _iv(intervals)
    drows = _rows(data_index, n_det, c, "data_index")
    frows = _rows(flag_index, n_det, c, "flag_index")
    ns = det_data.shape[1]
    c.run(load().toast_template_offset_project_signal, int(step_length),
          c(amp_offset, torch.int64, "amp_offset", shape=(n_det,)), c(amplitudes, torch.float64, "amplitudes"),
          c(data_index, torch.int32, "data_index"),
          c(det_data, torch.float64, "det_data", shape=(None, ns), min_numel=drows * ns),
          c(flag_index, torch.int32, "flag_index"),
          c(det_flags, torch.uint8, "det_flags", shape=(None, ns), min_numel=frows * ns), det_flag_mask, ivp, niv,
          n_det, ns, stream=stream)
    return amplitudes


def template_offset_apply_diag_precond(offset_var, amp_in, amp_out, stream=None):
    c = _Call("toast_template_offset_apply_diag_precond")
    n = amp_in.numel()
    c.run(load().toast_template_offset_apply_diag_precond, c(offset_var, torch.float64, "offset_var", shape=(n,)),
          c(amp_in, torch.float64, "amp_in", shape=(n,)), c(amp_out, torch.float64, "amp_out", shape=(n,)), n,
          stream=stream)
    return amp_out


def synth_tod(out, sigma, det_ids, seed: int, stream_id: int = 1, stream=None):
    """The seeded synthetic timestream on the device (include/toast_b200_synth.h): a bench / test
    INPUT generator, bit-identical to synth.tod_rows; none of the method's arithmetic."""
    c = _Call("toast_synth_tod")
    n_det, n_samp = out.shape
    c.run(load().toast_synth_tod, c(out, torch.float64, "out", shape=(n_det, n_samp)),
          c(sigma, torch.float64, "sigma", shape=(n_det,)), c(det_ids, torch.int64, "det_ids", shape=(n_det,)),
          n_det, n_samp, int(seed) & ((1 << 64) - 1), int(stream_id), stream=stream)
    return out


def map_allreduce_nvls(buf: torch.Tensor, mc_ptr: int, pads_dev_ptr: int, rank: int, world: int, stream=None):
    """toast_map_allreduce_nvls on `buf` (an f64 tensor in symmetric memory whose multicast mapping
    starts at device address `mc_ptr`; `pads_dev_ptr` the device array of the ranks' signal pads).
    Every rank's `buf` holds the sum over ranks afterwards (stream order)."""
    c = _Call("toast_map_allreduce_nvls")
    c(buf, torch.float64, "buf")
    c.run(load().toast_map_allreduce_nvls, ctypes.c_void_p(int(mc_ptr)), buf.numel(),
          ctypes.c_void_p(int(pads_dev_ptr)) if pads_dev_ptr else None, int(rank), int(world), stream=stream)
    return buf


def pointing_to_map_raw(args: tuple):
    """Call toast_pointing_to_map with a pre-marshalled argument tuple (bench inner loop)."""
    _check(load().toast_pointing_to_map(*args), "toast_pointing_to_map")
