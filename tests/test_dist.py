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
