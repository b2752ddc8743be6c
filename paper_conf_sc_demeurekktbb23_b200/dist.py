"""Multi-GPU plumbing for the pointing->map path: sharding plan and the map
reduction.  One process per GPU; torch.distributed (NCCL on B200, gloo on CPU for tests)
carries the ONE real exchange step of the method — the sum of the per-rank partial maps
("build_noise_weighted accumulate noise-weighted timestreams onto a sky map", PAPER.md:120,
with detectors and observations spread over processes).

    plan = plan_shards(units, world)          # LPT over (observation, detector-block) units
    hits = union_hit_submaps(hit_submaps)     # all_reduce(MAX) of the hit flags (tiny)
    reduce_map(zmap, hit_submaps=hits)        # pack hit submaps -> all_reduce(SUM) -> unpack

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
               global2local: Optional[torch.Tensor] = None) -> Tuple[torch.Tensor, int]:
    """Sum the per-rank partial maps (zmap [n_local_submap][n_pix_submap][nnz]) in place.

    With `hit_submaps` (already the union over ranks) only those submaps travel: packed into
    a contiguous buffer, all-reduced, unpacked.  Returns (zmap, bytes all-reduced)."""
    if not (dist.is_initialized() and dist.get_world_size(group) > 1):
        return zmap, 0
    if hit_submaps is None:
        dist.all_reduce(zmap, op=dist.ReduceOp.SUM, group=group)
        return zmap, zmap.numel() * zmap.element_size()
    if global2local is None:
        global2local = torch.arange(hit_submaps.numel(), device=zmap.device)
    idx = hit_local_submaps(hit_submaps.to(zmap.device), global2local.to(zmap.device))
    packed = zmap.index_select(0, idx)
    dist.all_reduce(packed, op=dist.ReduceOp.SUM, group=group)
    zmap.index_copy_(0, idx, packed)
    return zmap, packed.numel() * packed.element_size()
