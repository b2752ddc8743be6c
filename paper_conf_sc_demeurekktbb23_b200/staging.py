"""Host <-> device staging of a synthetic workload (PyTorch = device memory only).

``DeviceWorkload`` holds the HBM-resident inputs of one observation exactly in the layouts
include/toast_b200.h documents, plus the map buffers, and builds the argument tuple of
``toast_pointing_to_map`` once so the timed loop is a single C call per step.
"""
from __future__ import annotations

import dataclasses
from typing import Optional

import numpy as np
import torch

from . import binding
from .synth import Workload


def _t(a, dtype, device, pin=False):
    if a is None:
        return None
    t = torch.from_numpy(np.ascontiguousarray(a)).to(dtype)
    if device == "cpu":
        return t.pin_memory() if pin else t
    return t.to(device, non_blocking=False)


@dataclasses.dataclass
class DeviceWorkload:
    w: Workload
    fp_quats: torch.Tensor
    boresight: torch.Tensor
    hwp: Optional[torch.Tensor]
    epsilon: torch.Tensor
    det_scale: torch.Tensor
    det_data: torch.Tensor
    det_flags: Optional[torch.Tensor]
    shared_flags: Optional[torch.Tensor]
    global2local: torch.Tensor
    zmap: torch.Tensor
    hit_submaps: torch.Tensor
    intervals: np.ndarray

    @classmethod
    def upload(cls, w: Workload, device="cuda", det_data: Optional[torch.Tensor] = None, alloc_map: bool = True):
        n_local = w.n_submap
        dd = det_data if det_data is not None else _t(w.det_data, torch.float64, device)
        return cls(
            w=w,
            fp_quats=_t(w.fp_quats, torch.float64, device),
            boresight=_t(w.boresight, torch.float64, device),
            hwp=_t(w.hwp, torch.float64, device),
            epsilon=_t(w.epsilon, torch.float64, device),
            det_scale=_t(w.det_scale, torch.float64, device),
            det_data=dd,
            det_flags=_t(w.det_flags, torch.uint8, device),
            shared_flags=_t(w.shared_flags, torch.uint8, device),
            global2local=_t(w.global2local, torch.int64, device),
            zmap=torch.zeros((n_local if alloc_map else 1, w.n_pix_submap if alloc_map else 1, w.nnz),
                             dtype=torch.float64, device=device),
            hit_submaps=torch.zeros(w.n_submap, dtype=torch.uint8, device=device),
            intervals=binding.intervals_host(w.intervals),
        )

    def pointing_to_map(self, zmap=None, hit_submaps=None, pixels_out=None, weights_out=None, stream=None,
                        gamma=None, iau=False, dropped=None):
        w = self.w
        return binding.pointing_to_map(
            self.fp_quats, self.boresight, self.epsilon, w.cal, self.det_scale, self.det_data, self.intervals,
            w.nside, w.nest, w.nnz, self.global2local, w.n_pix_submap, self.zmap if zmap is None else zmap,
            hwp=self.hwp, det_flags=self.det_flags, det_flag_mask=w.det_flag_mask, shared_flags=self.shared_flags,
            shared_flag_mask=w.shared_flag_mask, hit_submaps=self.hit_submaps if hit_submaps is None else hit_submaps,
            pixels_out=pixels_out, weights_out=weights_out, stream=stream, gamma=gamma, iau=iau, dropped=dropped)

    def raw_args(self, stream=None, zmap=None, det_data=None, global2local=None):
        """Pre-marshalled argument tuple of toast_pointing_to_map (no per-call Python checks)."""
        w = self.w
        st = (stream or torch.cuda.current_stream()).cuda_stream
        p = lambda t: None if t is None else t.data_ptr()  # noqa: E731
        iv = self.intervals
        return (p(self.fp_quats), p(self.boresight), p(self.hwp), p(self.epsilon), float(w.cal), p(self.det_scale),
                p(self.det_data if det_data is None else det_data), p(self.det_flags), w.det_flag_mask,
                p(self.shared_flags), w.shared_flag_mask, iv.ctypes.data if len(iv) else None, len(iv), w.nside,
                int(w.nest), w.nnz, p(self.global2local if global2local is None else global2local), w.n_pix_submap, p(self.zmap if zmap is None else zmap),
                p(self.hit_submaps), None, None, w.n_det, w.n_samp, st)
