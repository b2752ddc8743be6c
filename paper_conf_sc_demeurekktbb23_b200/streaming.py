"""Host-resident timestreams through the fused entry: the end-to-end path of a user whose data
lives in (pinned) host memory (bench.py `e2e`).

A C4 day is 52 GB of TOD; it crosses PCIe / C2C once per call, in detector blocks through two
device staging buffers: the copy of block b+1 (a side stream) overlaps the fused kernel on block
b (the caller's stream), and every block accumulates into the same device map.  The kernels are
toast_pointing_to_map calls on detector subsets (pointer offsets into the staged rows); this
module is plumbing (pinned buffers, streams, events) only.
"""
from __future__ import annotations

import dataclasses
from typing import Optional

import torch

from . import binding


@dataclasses.dataclass
class HostInputs:
    """Pinned host copies of one observation's inputs (layouts as include/toast_b200.h)."""
    fp_quats: torch.Tensor            # [n_det][4] f64
    boresight: torch.Tensor           # [n_samp][4] f64
    epsilon: torch.Tensor             # [n_det] f64
    det_scale: torch.Tensor           # [n_det] f64
    det_data: torch.Tensor            # [n_det][n_samp] f64
    hwp: Optional[torch.Tensor] = None
    det_flags: Optional[torch.Tensor] = None
    shared_flags: Optional[torch.Tensor] = None

    def nbytes(self) -> int:
        return sum(t.numel() * t.element_size() for t in (self.fp_quats, self.boresight, self.epsilon,
                                                         self.det_scale, self.det_data, self.hwp, self.det_flags,
                                                         self.shared_flags) if t is not None)


class Streamer:
    """Reusable device buffers for streaming HostInputs of one shape through the fused entry."""

    def __init__(self, n_det: int, n_samp: int, block_dets: int, device, with_hwp: bool, with_det_flags: bool,
                 with_shared_flags: bool):
        self.n_det, self.n_samp, self.block = n_det, n_samp, min(block_dets, max(n_det, 1))
        f64 = dict(dtype=torch.float64, device=device)
        self.fp_quats = torch.empty((n_det, 4), **f64)
        self.boresight = torch.empty((n_samp, 4), **f64)
        self.epsilon = torch.empty(n_det, **f64)
        self.det_scale = torch.empty(n_det, **f64)
        self.hwp = torch.empty(n_samp, **f64) if with_hwp else None
        self.shared_flags = torch.empty(n_samp, dtype=torch.uint8, device=device) if with_shared_flags else None
        self.tod = [torch.empty((self.block, n_samp), **f64) for _ in range(2)]
        self.flags = ([torch.empty((self.block, n_samp), dtype=torch.uint8, device=device) for _ in range(2)]
                      if with_det_flags else None)
        self.copy_stream = torch.cuda.Stream(device=device)
        self.copied = [torch.cuda.Event() for _ in range(2)]
        self.consumed = [torch.cuda.Event() for _ in range(2)]

    def pointing_to_map(self, host: HostInputs, intervals, nside, nest, nnz, global2local, n_pix_submap, zmap, cal,
                        det_flag_mask=0, shared_flag_mask=0, hit_submaps=None, stream=None):
        """zmap += the fused pointing->map of `host` (all detectors), streamed in detector blocks."""
        st = stream or torch.cuda.current_stream()
        cs = self.copy_stream
        cs.wait_stream(st)  # the previous call's kernels are done with the staging buffers
        with torch.cuda.stream(cs):
            for dev, h in ((self.fp_quats, host.fp_quats), (self.boresight, host.boresight),
                           (self.epsilon, host.epsilon), (self.det_scale, host.det_scale), (self.hwp, host.hwp),
                           (self.shared_flags, host.shared_flags)):
                if dev is not None:
                    dev.copy_(h, non_blocking=True)
        small = torch.cuda.Event()
        small.record(cs)
        st.wait_event(small)
        launches = 0
        for i, d0 in enumerate(range(0, self.n_det, self.block)):
            d1 = min(self.n_det, d0 + self.block)
            b = i & 1
            with torch.cuda.stream(cs):
                if i >= 2:
                    cs.wait_event(self.consumed[b])  # the kernel two blocks ago has read buffer b
                self.tod[b][:d1 - d0].copy_(host.det_data[d0:d1], non_blocking=True)
                if self.flags is not None:
                    self.flags[b][:d1 - d0].copy_(host.det_flags[d0:d1], non_blocking=True)
                self.copied[b].record(cs)
            st.wait_event(self.copied[b])
            binding.pointing_to_map(self.fp_quats[d0:d1], self.boresight, self.epsilon[d0:d1], cal,
                                    self.det_scale[d0:d1], self.tod[b][:d1 - d0], intervals, nside, nest, nnz,
                                    global2local, n_pix_submap, zmap, hwp=self.hwp,
                                    det_flags=None if self.flags is None else self.flags[b][:d1 - d0],
                                    det_flag_mask=det_flag_mask, shared_flags=self.shared_flags,
                                    shared_flag_mask=shared_flag_mask, hit_submaps=hit_submaps, stream=st)
            self.consumed[b].record(st)
            launches += 1
        return launches
