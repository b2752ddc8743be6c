"""Multi-rank map reduction on CPU (gloo, world_size 2): the sum over shards of the oracle's
partial maps equals the oracle full map (SURVEY 8(c) 'A7 sharded'), with and without
hit-submap packing; plus the LPT sharding plan."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_demeurekktbb23_b200 import dist as tdist


def test_plan_balances_and_covers():
    units = tdist.make_units(n_obs=3, n_det=100, det_samples_per_det=[1000, 3000, 500], det_block=32)
    for world in (1, 2, 3, 8):
        plan = tdist.plan_shards(units, world)
        got = sorted((u.obs, u.d0) for r in plan for u in r)
        assert got == sorted((u.obs, u.d0) for u in units)
        loads = [sum(u.det_samples for u in r) for r in plan]
        assert max(loads) - min(loads) <= max(u.det_samples for u in units)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, packed, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_sc_demeurekktbb23_b200 import synth
    n_det = 6
    units = tdist.make_units(1, n_det, [1], det_block=2)
    mine = tdist.plan_shards(units, world)[rank]
    full = synth.make_workload("c2", n_det=n_det, n_samp=20_000, nside=32)
    z = np.zeros((full.n_submap, full.n_pix_submap, 3))
    hits = np.zeros(full.n_submap, np.uint8)
    for u in mine:
        w = synth.make_workload("c2", n_det=n_det, n_samp=20_000, nside=32, det_range=(u.d0, u.d1))
        oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals,
                               w.nside, w.nest, 3, w.global2local, w.n_pix_submap, zmap=z, hwp=w.hwp,
                               det_flags=w.det_flags, det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                               shared_flag_mask=w.shared_flag_mask, hit_submaps=hits)
    zt = torch.from_numpy(z)
    ht = torch.from_numpy(hits)
    if packed:
        tdist.union_hit_submaps(ht)
        _, nbytes = tdist.reduce_map(zt, hit_submaps=ht)
    else:
        _, nbytes = tdist.reduce_map(zt)
    if rank == 0:
        q.put((zt.numpy().copy(), ht.numpy().copy(), nbytes))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("packed", [False, True])
def test_two_rank_map_reduction_equals_full_map(packed):
    import oracle
    from paper_conf_sc_demeurekktbb23_b200 import synth
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, packed, q)) for r in range(2)]
    for p in procs:
        p.start()
    zsum, hits, nbytes = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    w = synth.make_workload("c2", n_det=6, n_samp=20_000, nside=32)
    zref = np.zeros((w.n_submap, w.n_pix_submap, 3)); absmap = np.zeros_like(zref)
    href = np.zeros(w.n_submap, np.uint8)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, zmap=zref, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, hit_submaps=href, absmap=absmap)
    from parity import check_map
    check_map(zsum, zref, absmap)
    if packed:
        np.testing.assert_array_equal(hits, href)
        assert nbytes == int(href.sum()) * w.n_pix_submap * 3 * 8
        assert nbytes < zref.nbytes


def _worker_sparse(rank, world, port, q):
    """f3: every rank accumulates its shard into the COMPACT (hit-submap-only) map, then
    reduce_scatter leaves each rank its owned block; gathered, it is the oracle full map."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_sc_demeurekktbb23_b200 import synth
    n_det = 6
    mine = tdist.plan_shards(tdist.make_units(1, n_det, [1], det_block=2), world)[rank]
    full = synth.make_workload("c2", n_det=n_det, n_samp=20_000, nside=32)
    kw = lambda w: dict(hwp=w.hwp, det_flags=w.det_flags, det_flag_mask=w.det_flag_mask,  # noqa: E731
                        shared_flags=w.shared_flags, shared_flag_mask=w.shared_flag_mask)
    # pass 1 (pixel distribution): hit submaps of this rank's shard from A1 -> A2 (no map)
    hits = np.zeros(full.n_submap, np.uint8)
    for u in mine:
        w = synth.make_workload("c2", n_det=n_det, n_samp=20_000, nside=32, det_range=(u.d0, u.d1))
        quats = oracle.pointing_detector(w.fp_quats, w.boresight, w.intervals, w.shared_flags, w.shared_flag_mask)
        oracle.pixels_healpix(quats, w.intervals, w.nside, w.nest, w.n_pix_submap, w.shared_flags, w.shared_flag_mask,
                              hit_submaps=hits)
    ht = tdist.union_hit_submaps(torch.from_numpy(hits))
    g2l, n_hit = tdist.compact_global2local(ht)
    own = tdist.MapOwnership.make(n_hit, world)
    zc = tdist.alloc_compact_map(own, full.n_pix_submap, 3, "cpu")
    z_np = zc.numpy()
    for u in mine:
        w = synth.make_workload("c2", n_det=n_det, n_samp=20_000, nside=32, det_range=(u.d0, u.d1))
        oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals,
                               w.nside, w.nest, 3, g2l.numpy(), w.n_pix_submap, zmap=z_np, **kw(w))
    block, nbytes = tdist.reduce_scatter_map(zc, own)
    lo, hi = own.owned(rank)
    assert block.shape[0] == own.per_rank and hi - lo <= own.per_rank
    full_map = tdist.gather_map(block, own, g2l, full.n_submap)
    q.put((rank, full_map.numpy().copy(), ht.numpy().copy(), n_hit, lo, hi, block.numpy().copy()))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_sparse_map_domain_reduce_scatter():
    import oracle
    from paper_conf_sc_demeurekktbb23_b200 import synth
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_sparse, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted((q.get(timeout=120) for _ in range(2)), key=lambda r: r[0])
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    w = synth.make_workload("c2", n_det=6, n_samp=20_000, nside=32)
    zref = np.zeros((w.n_submap, w.n_pix_submap, 3)); absmap = np.zeros_like(zref)
    href = np.zeros(w.n_submap, np.uint8)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, zmap=zref, hwp=w.hwp, det_flags=w.det_flags,
                           det_flag_mask=w.det_flag_mask, shared_flags=w.shared_flags,
                           shared_flag_mask=w.shared_flag_mask, hit_submaps=href, absmap=absmap)
    from parity import check_map
    n_hit = int(href.sum())
    assert 0 < n_hit < w.n_submap  # the sparse domain is actually smaller than the sky
    hit_idx = np.nonzero(href)[0]
    for rank, full_map, hits, nh, lo, hi, block in res:
        np.testing.assert_array_equal(hits, href)
        assert nh == n_hit
        check_map(full_map, zref, absmap)
        # the owned block holds exactly this rank's slice of the hit submaps, fully summed
        check_map(block[:hi - lo], zref[hit_idx[lo:hi]], absmap[hit_idx[lo:hi]])
    assert res[0][5] == res[1][4]  # the two blocks tile the hit submaps


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_work_plan_covers_every_detector_once(world):
    """bench.py's sharding (dist.work_plan): the ranks' detector ranges partition the focal plane
    (one observation, C4 style) / the (observation, block) units (several, C5m style)."""
    for n_obs in (1, 18):
        seen = []
        for r in range(world):
            for o, dr in tdist.work_plan(n_obs, 2048, world, r, "det"):
                lo, hi = dr if dr is not None else (0, 2048)
                seen += [(o, d) for d in range(lo, hi)]
        assert sorted(seen) == [(o, d) for o in range(n_obs) for d in range(2048)]
    assert [tdist.work_plan(1, 64, world, r, "obs") for r in range(world)] == [[(r, None)] for r in range(world)]


def _bench_plan_worker(rank, world, port, q):
    """Each rank runs THE bench's plan (dist.work_plan) on a C4-shaped detector split, accumulates
    its units with the oracle, and the packed reduction sums them."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_sc_demeurekktbb23_b200 import synth
    n_det, n_samp = 12, 6000
    base = synth.make_workload("c4", n_det=n_det, n_samp=n_samp, nside=64)
    z = np.zeros((base.n_submap, base.n_pix_submap, 3))
    hits = np.zeros(base.n_submap, np.uint8)
    for o, dr in tdist.work_plan(1, n_det, world, rank, "det"):
        w = synth.make_workload("c4", n_det=n_det, n_samp=n_samp, nside=64, obs=o, det_range=dr)
        oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals,
                               w.nside, w.nest, 3, w.global2local, w.n_pix_submap, zmap=z, hit_submaps=hits)
    zt, ht = torch.from_numpy(z), torch.from_numpy(hits)
    tdist.union_hit_submaps(ht)
    tdist.reduce_map(zt, hit_submaps=ht)
    if rank == 0:
        q.put(zt.numpy().copy())
    dist.barrier()


def test_bench_work_plan_reduced_equals_full_oracle_map():
    import oracle
    from paper_conf_sc_demeurekktbb23_b200 import synth
    from parity import check_map
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_plan_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    zsum = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    w = synth.make_workload("c4", n_det=12, n_samp=6000, nside=64)
    zref = np.zeros_like(zsum); absmap = np.zeros_like(zsum)
    oracle.pointing_to_map(w.fp_quats, w.boresight, w.epsilon, w.cal, w.det_scale, w.det_data, w.intervals, w.nside,
                           w.nest, 3, w.global2local, w.n_pix_submap, zmap=zref, absmap=absmap)
    check_map(zsum, zref, absmap)
