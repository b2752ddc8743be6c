"""The C-ABI library loads and exports every symbol include/toast_b200.h declares; host-side
argument validation rejects bad arguments before touching the GPU (CPU only: no compute)."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "toast_b200.h")
HEADERS = sorted(os.path.join(ROOT, "include", f) for f in os.listdir(os.path.join(ROOT, "include")) if f.endswith(".h"))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_demeurekktbb23_b200 import _build, binding
    _build.build()
    return binding.load()


def declared_functions():
    src = "".join(open(h).read() for h in HEADERS)
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(toast_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_six_entries():
    names = declared_functions()
    for n in ("toast_pointing_detector", "toast_pixels_healpix", "toast_stokes_weights_iqu",
              "toast_build_noise_weighted", "toast_scan_map", "toast_pointing_to_map", "toast_last_error",
              "toast_release", "toast_version"):
        assert n in names


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_sc_demeurekktbb23_b200 import _build
    out = subprocess.run(["nm", "-D", "--defined-only", _build.LIB], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (toast_[a-z0-9_]+)", out))
    missing = [n for n in declared_functions() if n not in exported]
    assert not missing, f"declared but not exported: {missing}"
    for n in declared_functions():
        getattr(lib, n)  # resolvable through ctypes


def test_library_is_sm100a(lib):
    from paper_conf_sc_demeurekktbb23_b200 import _build
    out = subprocess.run(["cuobjdump", "--list-elf", _build.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version(lib):
    assert b"toastb200" in lib.toast_version()


def _einval(rc, lib, pattern):
    assert rc == -1
    assert re.search(pattern, lib.toast_last_error().decode()), lib.toast_last_error()


def test_validation_rejects_before_any_launch(lib):
    iv_bad = np.array([[0, 10], [5, 20]], np.int64)
    iv_out = np.array([[0, 100]], np.int64)
    iv_ok = np.array([[0, 9]], np.int64)
    # pixels_healpix: nside not a power of two / submap not dividing npix / nest flag
    _einval(lib.toast_pixels_healpix(None, None, None, 0, None, None, iv_ok.ctypes.data, 1, None, 16, 3, 0, 1, 10,
                                     None), lib, "power of two")
    _einval(lib.toast_pixels_healpix(None, None, None, 0, None, None, iv_ok.ctypes.data, 1, None, 7, 4, 0, 1, 10,
                                     None), lib, "does not divide")
    _einval(lib.toast_pixels_healpix(None, None, None, 0, None, None, iv_ok.ctypes.data, 1, None, 16, 4, 2, 1, 10,
                                     None), lib, "nest")
    _einval(lib.toast_pixels_healpix(None, None, None, 0, None, None, iv_ok.ctypes.data, 1, None, 16, 1 << 30, 0, 1,
                                     10, None), lib, "power of two")
    # required pointers
    _einval(lib.toast_pixels_healpix(None, None, None, 0, None, None, iv_ok.ctypes.data, 1, None, 16, 4, 0, 1, 10,
                                     None), lib, "NULL")
    # intervals overlapping / outside
    dummy = ctypes.c_void_p(16)
    _einval(lib.toast_pointing_detector(dummy, dummy, None, dummy, iv_bad.ctypes.data, 2, None, 0, 1, 100, None), lib,
            "overlap")
    _einval(lib.toast_pointing_detector(dummy, dummy, None, dummy, iv_out.ctypes.data, 1, None, 0, 1, 50, None), lib,
            "outside")
    # nnz
    _einval(lib.toast_build_noise_weighted(dummy, dummy, 16, 2, None, dummy, None, dummy, None, dummy, None, None, 0,
                                           dummy, None, 0, iv_ok.ctypes.data, 1, 1, 10, None), lib, "nnz")
    _einval(lib.toast_scan_map(dummy, 0, dummy, 3, None, dummy, None, dummy, None, dummy, iv_ok.ctypes.data, 1, 1.0,
                               0, 0, 1, 10, None), lib, "n_pix_submap")
    _einval(lib.toast_pointing_to_map(dummy, dummy, None, dummy, 1.0, dummy, dummy, None, 0, None, 0,
                                      iv_ok.ctypes.data, 1, 64, 0, 2, dummy, 16, dummy, None, None, None, 1, 10, None),
            lib, "nnz")
    _einval(lib.toast_stokes_weights_iqu(None, dummy, None, dummy, None, None, 1.0, iv_ok.ctypes.data, 1, 1, 10, None),
            lib, "epsilon")
    _einval(lib.toast_pointing_detector(dummy, dummy, None, dummy, iv_ok.ctypes.data, 1, None, 0, -1, 10, None), lib,
            "n_det")
    # the NVLS map exchange (f3): sizes, ranks, pads
    _einval(lib.toast_map_allreduce_nvls(dummy, -1, None, 0, 1, None), lib, "< 0")
    _einval(lib.toast_map_allreduce_nvls(dummy, 10, dummy, 2, 2, None), lib, "out of range")
    _einval(lib.toast_map_allreduce_nvls(dummy, 10, dummy, 0, 0, None), lib, "out of range")
    _einval(lib.toast_map_allreduce_nvls(None, 10, dummy, 0, 1, None), lib, "mc is NULL")
    _einval(lib.toast_map_allreduce_nvls(dummy, 10, None, 0, 2, None), lib, "pads is NULL")


def test_binding_refuses_cpu_tensors():
    torch = pytest.importorskip("torch")
    from paper_conf_sc_demeurekktbb23_b200 import binding
    binding.load()
    with pytest.raises(binding.ToastError, match="CUDA tensor"):
        binding.pointing_detector(torch.zeros(1, 4, dtype=torch.float64), torch.zeros(10, 4, dtype=torch.float64),
                                  [(0, 9)], torch.zeros(1, 10, 4, dtype=torch.float64))
