"""Multi-GPU plumbing for the pointing->map path: sharding plan and the map
reduction.  One process per GPU; torch.distributed (NCCL on B200, gloo on CPU for tests)
carries the ONE real exchange step of the method — the sum of the per-rank partial maps
("build_noise_weighted accumulate noise-weighted timestreams onto a sky map", PAPER.md:120,
with detectors and observations spread over processes).

    plan = plan_shards(units, world)          # LPT over (observation, detector-block) units
    hits = union_hit_submaps(hit_submaps)     # all_reduce(MAX) of the hit flags (tiny)
    reduce_map(zmap, hit_submaps=hits)        # pack hit submaps -> all_reduce(SUM) -> unpack

Sparse, distributed map domain:

    g2l, n_hit = compact_global2local(hits)   # storage for hit submaps only (-1 elsewhere)
    own = MapOwnership.make(n_hit, world)     # contiguous blocks of hit submaps per rank
    zc = alloc_compact_map(own, nps, nnz, dev)  # toast_pointing_to_map(..., g2l, zmap=zc)
    block, _ = reduce_scatter_map(zc, own)    # this rank's owned, fully summed submaps

Packing to the union of hit submaps shrinks the all-reduce to the sky actually observed
(the dense map is 4.8 GB at nside 4096); the pack/unpack are index_select / index_copy on the
device (memory plumbing, not method arithmetic).
"""
from __future__ import annotations

import dataclasses
import heapq
from typing import List, Optional, Sequence, Tuple

import torch
import torch.distributed as dist


@dataclasses.dataclass(frozen=True)
class Unit:
    """A shardable piece of work: detectors [d0, d1) of observation `obs`."""
    obs: int
    d0: int
    d1: int
    det_samples: int


def make_units(n_obs: int, n_det: int, det_samples_per_det: Sequence[int], det_block: int) -> List[Unit]:
    """Cut every observation into detector blocks of `det_block` detectors."""
    units = []
    for o in range(n_obs):
        for d0 in range(0, n_det, det_block):
            d1 = min(n_det, d0 + det_block)
            units.append(Unit(o, d0, d1, (d1 - d0) * int(det_samples_per_det[o])))
    return units


def plan_shards(units: Sequence[Unit], world: int) -> List[List[Unit]]:
    """Longest-processing-time-first assignment of units to `world` ranks (balances
    det-samples; deterministic: ties broken by unit order and rank id)."""
    heap = [(0, r) for r in range(world)]
    out: List[List[Unit]] = [[] for _ in range(world)]
    order = sorted(range(len(units)), key=lambda i: (-units[i].det_samples, i))
    for i in order:
        load, r = heapq.heappop(heap)
        out[r].append(units[i])
        heapq.heappush(heap, (load + units[i].det_samples, r))
    for r in range(world):
        out[r].sort(key=lambda u: (u.obs, u.d0))
    return out


def work_plan(n_obs: int, n_det: int, world: int, rank: int, shard: str, det_block: int = 256,
              first_obs: int = 0) -> List[Tuple[int, Optional[Tuple[int, int]]]]:
    """This rank's work as (observation, detector range or None = all) pairs — the plan bench.py
    runs:
      shard="det": one observation (n_obs = 1) cut into `world` contiguous detector blocks
                   (C4: 2048 / 8 = 256 detectors per GPU), or several observations cut into
                   `det_block` blocks and LPT-balanced (C5m); strong scaling;
      shard="obs": observation first_obs + rank on every rank (weak scaling)."""
    if shard == "obs":
        return [(first_obs + rank, None)]
    if world == 1:
        return [(first_obs + o, None) for o in range(n_obs)]
    if n_obs == 1:
        per = -(-n_det // world)
        lo, hi = min(n_det, rank * per), min(n_det, (rank + 1) * per)
        return [(first_obs, (lo, hi))] if hi > lo else []
    units = make_units(n_obs, n_det, [1] * n_obs, det_block)
    return [(first_obs + u.obs, (u.d0, u.d1)) for u in plan_shards(units, world)[rank]]


def union_hit_submaps(hit_submaps: torch.Tensor, group=None) -> torch.Tensor:
    """In-place all_reduce(MAX) of the per-rank hit-submap flags (uint8, n_submap)."""
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        if hit_submaps.dtype == torch.uint8 and hit_submaps.device.type == "cpu":
            tmp = hit_submaps.to(torch.int32)  # gloo has no uint8 MAX
            dist.all_reduce(tmp, op=dist.ReduceOp.MAX, group=group)
            hit_submaps.copy_(tmp.to(torch.uint8))
        else:
            dist.all_reduce(hit_submaps, op=dist.ReduceOp.MAX, group=group)
    return hit_submaps


def hit_local_submaps(hit_submaps: torch.Tensor, global2local: torch.Tensor) -> torch.Tensor:
    """Local storage indices of the hit submaps (those with storage), sorted."""
    g = torch.nonzero(hit_submaps, as_tuple=False).flatten()
    loc = global2local.index_select(0, g)
    return torch.sort(loc[loc >= 0]).values


def reduce_map(zmap: torch.Tensor, group=None, hit_submaps: Optional[torch.Tensor] = None,
               global2local: Optional[torch.Tensor] = None, nvls: Optional["NvlsReducer"] = None
               ) -> Tuple[torch.Tensor, int]:
    """Sum the per-rank partial maps (zmap [n_local_submap][n_pix_submap][nnz]) in place.

    With `hit_submaps` (already the union over ranks) only those submaps travel: packed into
    a contiguous buffer, all-reduced, unpacked.  With `nvls` the sum runs in the switch through
    toast_map_allreduce_nvls instead of NCCL.  Returns (zmap, bytes all-reduced)."""
    if not (dist.is_initialized() and dist.get_world_size(group) > 1):
        return zmap, 0

    def allreduce(t):
        if nvls is not None:
            nvls.allreduce_(t)
        else:
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)

    if hit_submaps is None:
        allreduce(zmap)
        return zmap, zmap.numel() * zmap.element_size()
    if global2local is None:
        global2local = torch.arange(hit_submaps.numel(), device=zmap.device)
    idx = hit_local_submaps(hit_submaps.to(zmap.device), global2local.to(zmap.device))
    packed = zmap.index_select(0, idx)
    allreduce(packed)
    zmap.index_copy_(0, idx, packed)
    return zmap, packed.numel() * packed.element_size()


# ----------------------------------------------------------------------------- NVLS map exchange
# SURVEY 8(f) f3 / 8(e) step 3 done in the switch by our own kernel (toast_map_allreduce_nvls:
# multimem.ld_reduce / multimem.st over a multicast mapping) instead of NCCL's all_reduce.  The
# buffer lives in torch symmetric memory, which creates the per-rank mappings, the multicast
# object and the signal pads (plumbing only); the reduction itself is the library's kernel.

class NvlsReducer:
    """A symmetric-memory f64 buffer of `numel` elements with a multicast mapping over the
    group's ranks.  `allreduce_(t)` sums `t` (numel <= capacity) over the ranks in place, through
    the buffer (or directly, when `t` is a view of `self.buf` starting at its first element).
    Raises RuntimeError when the GPUs / driver have no multicast (NVLS) support."""

    def __init__(self, numel: int, device, group=None):
        import torch.distributed._symmetric_memory as symm_mem
        group = group or dist.group.WORLD
        self.buf = symm_mem.empty(int(numel), dtype=torch.float64, device=device)
        self.hdl = symm_mem.rendezvous(self.buf, group.group_name)
        if not self.hdl.has_multicast_support or not int(self.hdl.multicast_ptr):
            raise RuntimeError("no multicast (NVLS) mapping on this device / driver / group")
        self.rank, self.world = int(self.hdl.rank), int(self.hdl.world_size)
        self.mc_ptr = int(self.hdl.multicast_ptr)
        self.pads = int(self.hdl.signal_pad_ptrs_dev)

    def allreduce_(self, t: torch.Tensor) -> torch.Tensor:
        from . import binding
        n = t.numel()
        if n > self.buf.numel():
            raise ValueError(f"{n} elements > the NVLS buffer's {self.buf.numel()}")
        inplace = t.data_ptr() == self.buf.data_ptr() and t.is_contiguous()
        view = self.buf[:n]
        if not inplace:
            view.copy_(t.reshape(-1))
        binding.map_allreduce_nvls(view, self.mc_ptr, self.pads, self.rank, self.world)
        if not inplace:
            t.copy_(view.view_as(t))
        return t


# ----------------------------------------------------------------------------- sparse map domain
# the map is stored for hit submaps only (TOAST's pixel distribution: a
# global2local table with -1 for submaps without local storage, "accumulate ...
# onto a sky map"), and after accumulation each rank OWNS a contiguous block of the hit
# submaps: reduce_scatter instead of all_reduce halves the bytes each rank sends and leaves the
# map distributed, as TOAST's distributed map domain does.  On NCCL over NVSwitch the
# collective runs in the switch (NVLS) when NCCL enables it; there is no second implementation.

def compact_global2local(hit_submaps: torch.Tensor) -> Tuple[torch.Tensor, int]:
    """global2local of a hit-submap-only map: hit submaps get storage 0..n_hit-1 in global
    order, the others -1 (the fused kernel skips their samples' map update — only samples in
    unhit submaps, i.e. none, when hit_submaps is the union over ranks).  Returns (g2l int64,
    n_hit)."""
    hit = hit_submaps.to(torch.bool)
    g2l = torch.full(hit.shape, -1, dtype=torch.int64, device=hit_submaps.device)
    idx = torch.nonzero(hit, as_tuple=False).flatten()
    g2l[idx] = torch.arange(idx.numel(), dtype=torch.int64, device=hit_submaps.device)
    return g2l, int(idx.numel())


@dataclasses.dataclass(frozen=True)
class MapOwnership:
    """Which rank owns which compact submaps after reduce_scatter_map: rank r owns compact
    indices [r * per_rank, min(n_hit, (r + 1) * per_rank)); the compact map is padded to
    world * per_rank submaps so every rank's block has the same size (NCCL reduce_scatter)."""
    n_hit: int
    world: int
    per_rank: int

    @classmethod
    def make(cls, n_hit: int, world: int) -> "MapOwnership":
        return cls(n_hit, world, max(1, -(-n_hit // world)))

    @property
    def padded(self) -> int:
        return self.per_rank * self.world

    def owned(self, rank: int) -> Tuple[int, int]:
        lo = min(self.n_hit, rank * self.per_rank)
        return lo, min(self.n_hit, lo + self.per_rank)

    def owner(self, compact_index: int) -> int:
        return compact_index // self.per_rank


def alloc_compact_map(own: MapOwnership, n_pix_submap: int, nnz: int, device, dtype=torch.float64) -> torch.Tensor:
    """A compact map [padded][n_pix_submap][nnz]: compact_global2local indexes its first n_hit
    submaps; the padding submaps are never written (no global submap maps to them)."""
    return torch.zeros((own.padded, n_pix_submap, nnz), dtype=dtype, device=device)


def _reduce_scatter(out: torch.Tensor, inp: torch.Tensor, group=None):
    if dist.get_backend(group) == "nccl":
        dist.reduce_scatter_tensor(out, inp, op=dist.ReduceOp.SUM, group=group)
    else:  # gloo has no reduce_scatter: the same result through all_reduce + this rank's slice
        tmp = inp.clone()
        dist.all_reduce(tmp, op=dist.ReduceOp.SUM, group=group)
        r = dist.get_rank(group)
        out.copy_(tmp.narrow(0, r * out.shape[0], out.shape[0]))


def reduce_scatter_map(zmap_compact: torch.Tensor, own: MapOwnership, group=None) -> Tuple[torch.Tensor, int]:
    """Sum the per-rank compact partial maps; return THIS rank's owned block
    [per_rank][n_pix_submap][nnz] (rows past n_hit are padding) and the bytes each rank
    contributes to the collective."""
    assert zmap_compact.shape[0] == own.padded, (zmap_compact.shape, own)
    out = torch.empty((own.per_rank,) + tuple(zmap_compact.shape[1:]), dtype=zmap_compact.dtype,
                      device=zmap_compact.device)
    if not (dist.is_initialized() and dist.get_world_size(group) > 1):
        out.copy_(zmap_compact[:own.per_rank])
        return out, 0
    _reduce_scatter(out, zmap_compact.contiguous(), group)
    return out, zmap_compact.numel() * zmap_compact.element_size()


def gather_map(owned: torch.Tensor, own: MapOwnership, global2local: torch.Tensor, n_submap: int,
               group=None) -> torch.Tensor:
    """Reassemble the full dense map [n_submap][n_pix_submap][nnz] from the owned blocks (for
    output; the distributed map itself never needs it).  Unhit submaps are 0."""
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        blocks = torch.empty((own.padded,) + tuple(owned.shape[1:]), dtype=owned.dtype, device=owned.device)
        if dist.get_backend(group) == "nccl":
            dist.all_gather_into_tensor(blocks, owned.contiguous(), group=group)
        else:
            parts = [torch.empty_like(owned) for _ in range(own.world)]
            dist.all_gather(parts, owned.contiguous(), group=group)
            blocks = torch.cat(parts)
    else:
        blocks = owned
    full = torch.zeros((n_submap,) + tuple(owned.shape[1:]), dtype=owned.dtype, device=owned.device)
    g2l = global2local.to(owned.device)
    hit = torch.nonzero(g2l >= 0, as_tuple=False).flatten()
    full[hit] = blocks[g2l[hit]]
    return full
