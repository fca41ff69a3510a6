"""Cell partitioning host logic, on CPU.

* partition_cells (recursive coordinate bisection) covers every cell once,
  balances the parts and splits a box on its longest axis;
* the rank grid (part = rank % P, band group = rank // P);
* world-size-2 gloo: the halo rule the library implements -- a rank needs,
  for every cut face of its cells, the neighbour part's old-level value in the
  directions with s_d . n_f < 0 at that face (upwind inflow, Eq. 3,
  L264-267) -- is sufficient: each rank receives exactly those values over
  gloo, every other non-owned value is poisoned with NaN, and the oracle's
  step of the owned cells (intensity, energy, temperature) is bitwise the
  unpartitioned step.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_heislersdms24_b200 import dist as bdist
from paper_conf_ipps_heislersdms24_b200 import inputs as gen


@pytest.mark.parametrize("n_parts", [1, 2, 3, 5, 8])
def test_partition_cells_cover_and_balance(n_parts):
    cfg = gen.small_3d_config((13, 7, 5))
    parts = bdist.partition_cells(cfg.mesh["cell_centre"], n_parts)
    nc = cfg.mesh["n_cells"]
    assert parts.shape == (nc,) and parts.min() == 0 and parts.max() == n_parts - 1
    sizes = np.bincount(parts, minlength=n_parts)
    assert sizes.sum() == nc and sizes.max() - sizes.min() <= 2
    assert np.array_equal(parts, bdist.partition_cells(cfg.mesh["cell_centre"], n_parts))  # deterministic


def test_partition_cells_bisects_longest_axis():
    cfg = gen.small_3d_config((16, 4, 4))
    parts = bdist.partition_cells(cfg.mesh["cell_centre"], 2)
    x = cfg.mesh["cell_centre"][:, 0]
    assert x[parts == 0].max() < x[parts == 1].min()


@pytest.mark.parametrize("n_parts", [1, 2, 3, 5, 8])
def test_slab_partition_whole_layers(n_parts):
    cfg = gen.small_3d_config((6, 5, 8))
    parts = bdist.slab_partition(cfg.mesh["cell_centre"], n_parts)
    z = cfg.mesh["cell_centre"][:, 2]
    for p in range(n_parts):  # every part a contiguous range of whole z layers
        zs = np.unique(z[parts == p])
        assert zs.size >= 1
        assert not np.isin(zs, z[parts != p]).any()
    assert np.all(np.diff([z[parts == p].min() for p in range(n_parts)]) > 0)


@pytest.mark.parametrize("world,P", [(8, 8), (8, 4), (8, 2), (6, 3), (4, 1)])
def test_rank_grid(world, P):
    seen = {bdist.rank_grid(r, world, P) for r in range(world)}
    assert seen == {(p, g) for p in range(P) for g in range(world // P)}


def halo_plan(mesh, dirs, parts, reader, writer):
    """Cells of `writer` that cut faces of `reader` point to, and the directions
    with s . n < 0 at any such face (the reading side's normal)."""
    off, nbr, nrm = mesh["face_offsets"], mesh["face_nbr"], mesh["face_normal"]
    cells, normals = set(), []
    for g in np.flatnonzero(parts == reader):
        for f in range(off[g], off[g + 1]):
            h = nbr[f]
            if h >= 0 and parts[h] == writer:
                cells.add(int(h))
                normals.append(nrm[f])
    if not cells:
        return np.zeros(0, np.int64), np.zeros(0, np.int64)
    mu = dirs["s"] @ np.asarray(normals).T  # [nd][faces]
    return np.array(sorted(cells), np.int64), np.flatnonzero((mu < 0).any(axis=1))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cfgs():
    return [gen.make_config("C1"), gen.small_3d_config((8, 5, 4), n_spectral=2), gen.make_config("C6t")]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        out = []
        for cfg in _cfgs():
            parts = bdist.partition_cells(cfg.mesh["cell_centre"], world)
            me, other = bdist.rank_grid(rank, world, world)[0], 1 - rank
            p = oracle.problem_from_config(cfg)
            I, T = p.initial_state(cfg.t_init, ic_eps=0.2)
            own = np.flatnonzero(parts == me)
            # halo exchange over gloo: send what the other part reads, receive what I read
            s_cells, s_dirs = halo_plan(cfg.mesh, cfg.dirs, parts, other, me)
            r_cells, r_dirs = halo_plan(cfg.mesh, cfg.dirs, parts, me, other)
            send = torch.from_numpy(np.ascontiguousarray(I[:, s_dirs][:, :, s_cells]))
            recv = torch.empty((p.nb, r_dirs.size, r_cells.size), dtype=torch.float64)
            reqs = [dist.isend(send, other), dist.irecv(recv, other)]
            for r in reqs:
                r.wait()
            Iloc = np.full_like(I, np.nan)  # only owned values and the received halo
            Iloc[:, :, own] = I[:, :, own]
            Iloc[np.ix_(np.arange(p.nb), r_dirs, r_cells)] = recv.numpy()
            Tloc = np.full_like(T, np.nan)
            Tloc[own] = T[own]
            upd = p.update_intensity(Tloc, Iloc, cfg.dt)
            Inew, E = upd[:, :, own], p.energy(upd)[own]  # (per-cell: NaN elsewhere does not enter)
            out.append((cfg.name, own, Inew, E, int(s_dirs.size), int(r_dirs.size)))
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_two_rank_halo_rule_is_sufficient(oracle_mod):
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    for k, cfg in enumerate(_cfgs()):
        p = oracle_mod.problem_from_config(cfg)
        I, T = p.initial_state(cfg.t_init, ic_eps=0.2)
        Ifull = p.update_intensity(T, I, cfg.dt)
        Efull = p.energy(Ifull)
        nd = cfg.dirs["n_dirs"]
        covered = np.zeros(cfg.mesh["n_cells"], bool)
        for r in range(world):
            name, own, Inew, E, nsd, nrd = res[r][k]
            assert name == cfg.name
            assert not covered[own].any()
            covered[own] = True
            assert np.array_equal(Inew, Ifull[:, :, own]), name  # bitwise: same code, same inputs
            assert np.array_equal(E, Efull[own]), name
            assert 0 < nrd <= nd and 0 < nsd <= nd
            if name != "C6t":  # axis-aligned cuts: only the inflow half of the set crosses
                assert nrd == nsd == nd // 2
        assert covered.all()
