"""World-size-2 CPU (gloo) tests of the multi-rank host logic.

* the NCCL unique id made on rank 0 reaches every rank intact;
* band sharding is exact: each rank's oracle energy over its own rows, summed
  with an all-reduce, then the temperature solve, equals the unsharded step
  (this is the decomposition the library performs with ncclAllReduce);
* the row partition covers every row once, contiguously.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_heislersdms24_b200 import dist as bdist
from paper_conf_ipps_heislersdms24_b200 import inputs as gen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_heislersdms24_b200 import bte
        import oracle
        nid = bdist.share_nccl_id(dist, rank, make_id=bte.nccl_unique_id)
        ids = [None] * world
        dist.all_gather_object(ids, nid)
        cfg = gen.small_3d_config((5, 4, 3), n_spectral=4)
        p = oracle.problem_from_config(cfg)
        I, T = p.initial_state(cfg.t_init, ic_eps=0.2)
        b_lo, b_hi = bdist.band_range(rank, world, p.nb)
        # one sharded step: local rows only, then the energy all-reduce, then Newton
        In = p.update_intensity(T, I, cfg.dt, b_lo, b_hi)
        E_loc = p.energy(In, b_lo, b_hi)
        E = torch.from_numpy(E_loc.copy())
        dist.all_reduce(E)
        T1, _ = p.newton(E.numpy(), T)
        Tg = [None] * world
        dist.all_gather_object(Tg, T1)
        rows = [None] * world
        dist.all_gather_object(rows, (b_lo, b_hi, In[b_lo:b_hi]))
        q.put((rank, ids[0] == ids[-1] and len(ids[0]) == 128, Tg, rows))
    finally:
        dist.destroy_process_group()


def test_two_rank_band_sharded_step_matches_unsharded(oracle_mod):
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    res.sort()
    assert all(r[1] for r in res), "NCCL id did not reach every rank intact"
    cfg = gen.small_3d_config((5, 4, 3), n_spectral=4)
    p = oracle_mod.problem_from_config(cfg)
    I, T = p.initial_state(cfg.t_init, ic_eps=0.2)
    I1, T1 = p.run(I, T, cfg.dt, 1)
    Tg = res[0][2]
    assert np.array_equal(Tg[0], Tg[1])  # replicated temperature is bitwise identical
    assert np.max(np.abs(Tg[0] / T1 - 1)) < 1e-13
    rows = res[0][3]
    Ish = np.concatenate([r[2] for r in rows], axis=0)
    assert [(r[0], r[1]) for r in rows] == [bdist.band_range(g, 2, p.nb) for g in range(2)]
    assert np.array_equal(Ish, I1)


@pytest.mark.parametrize("nb,world", [(55, 8), (55, 4), (55, 2), (13, 2), (3, 3), (8, 8)])
def test_band_partition_covers_rows(nb, world):
    rs = [bdist.band_range(g, world, nb) for g in range(world)]
    assert rs[0][0] == 0 and rs[-1][1] == nb
    assert all(rs[g][1] == rs[g + 1][0] for g in range(world - 1))
    sizes = [hi - lo for lo, hi in rs]
    assert max(sizes) - min(sizes) <= 1 and min(sizes) >= 1
