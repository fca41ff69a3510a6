"""The multi-rank step through bte_step, on one GPU.

The pool reaches one GPU at a time, so NCCL can never run with world > 1
here.  The in-process communicator (bte_group_create, csrc/bte_group.cu) runs
the library's multi-rank code path unchanged -- bte_create with world > 1, the
band split (L773-775), the per-step reduce-scatter of the energy over a padded
n_cells (P does not divide it), the temperature solve of each rank's chunk of
cells at c_lo > 0, the all-gather of T with the -T failure marker, the
all-reduce variant, the cell-partition halo send / receive group and the
band-group split -- with the collectives done as device copies between the
ranks' buffers.  Every rank is a host thread with its own context; results are
compared with the unpartitioned CPU oracle (relative 1e-10 on I, 1e-9 on T)
and T must be bitwise identical on every rank.
"""
import dataclasses
import threading

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import dist as bdist
from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import RTOL_I, RTOL_T, assert_parity, oracle_run, rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bte():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


def run_ranks(bte, cfg, world, nsteps, n_cell_parts=1, parts=None, expect=None, **kw):
    """world ranks as threads on one in-process group; each creates its
    context, applies the seeded IC, steps and reads back its state.  Returns
    per rank (b_lo, b_hi, owned ids, I, T, stats, error)."""
    out = [None] * world
    part_kw = {}
    if n_cell_parts > 1:
        if parts is None:
            cen = cfg.mesh["cell_centre"]
            parts = (bdist.slab_partition(cen, n_cell_parts) if cfg.mesh["dim"] == 3
                     else bdist.partition_cells(cen, n_cell_parts))
        part_kw = dict(cell_part=parts, n_cell_parts=n_cell_parts)
    with bte.Group(world) as g:
        def rank(r):
            try:
                with bte.solver_from_config(cfg, rank=r, world=world, group=g, **part_kw, **kw) as s:
                    bte.apply_ic(s, cfg)
                    err = None
                    try:
                        s.step(cfg.dt, nsteps)
                    except bte.BTEError as e:
                        err = e.status
                    out[r] = (s.b_lo, s.b_hi, s.local_cells(), s.intensity(), s.temperature(), s.stats(), err)
            except Exception as e:  # pragma: no cover - reported below
                out[r] = e
        ts = [threading.Thread(target=rank, args=(r,)) for r in range(world)]
        for t in ts:
            t.start()
        for t in ts:
            t.join(timeout=600)
        assert not any(t.is_alive() for t in ts), "a rank hung"
    for o in out:
        if isinstance(o, Exception):
            raise o
    return out


def assemble(cfg, out):
    nb, nd, nc = cfg.bands["n_bands"], cfg.dirs["n_dirs"], cfg.mesh["n_cells"]
    I = np.full((nb, nd, nc), np.nan)
    T = np.full(nc, np.nan)
    for b_lo, b_hi, ids, Il, Tl, _, _ in out:
        if np.isnan(T[ids]).all():
            T[ids] = Tl
        else:  # every band group of a cell part holds the same T: identical bits
            assert np.array_equal(T[ids], Tl)
        I[b_lo:b_hi][:, :, ids] = Il
    assert not np.isnan(I).any() and not np.isnan(T).any()
    return I, T


# ------------------------------------------------------------------ band sharding (8(e))
@pytest.mark.parametrize("mode", ["shard", "replicated"])
@pytest.mark.parametrize("world", [2, 3, 4])
def test_band_sharding_through_bte_step(bte, oracle_mod, monkeypatch, mode, world):
    """C2 (13 rows, 4096 cells: 4096 % 3 != 0, so the reduce-scatter is padded)
    band-sharded over 2-4 ranks, 12 steps through bte_step, both exchange
    modes; the row split is L773-775's."""
    monkeypatch.setenv("BTE_SHARD_NEWTON", mode)
    cfg = dataclasses.replace(gen.make_config("C2"), nsteps=12)
    Io, To = oracle_run(oracle_mod, cfg, 12)
    out = run_ranks(bte, cfg, world, 12)
    assert [(o[0], o[1]) for o in out] == [bdist.band_range(r, world, 13) for r in range(world)]
    Ig, Tg = assemble(cfg, out)
    assert_parity(Ig, Tg, Io, To)
    for o in out:
        assert o[5]["steps"] == 12 and o[6] is None


@pytest.mark.parametrize("kernel", ["warp", "thread"])
def test_band_sharding_box3d_rate_law(bte, oracle_mod, monkeypatch, kernel):
    """The benched box kernel, band-sharded over 3 ranks (chunk solves at
    c_lo > 0 in both Newton kernels), with temperature-dependent rates."""
    monkeypatch.setenv("BTE_NEWTON", kernel)
    cfg = gen.small_3d_config((34, 9, 7), n_spectral=5)
    law = gen.with_rate_law(cfg.bands)
    cfg = dataclasses.replace(cfg, bands=law, dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, law, cfg.dirs, t_max=350.0))
    Io, To = oracle_run(oracle_mod, cfg, 10)
    out = run_ranks(bte, cfg, 3, 10)
    assert all(o[5]["flux_variant"] == 6 for o in out)
    Ig, Tg = assemble(cfg, out)
    assert_parity(Ig, Tg, Io, To)


def test_band_sharding_more_than_128_rows(bte, oracle_mod):
    """200 band-rows in all (the warp solve's lanes carry 8 rows each), 2
    ranks of 100: every row enters every cell's temperature."""
    mesh = gen.gen_mesh((9, 7), (1e-6, 1e-6))
    bands = gen.gen_bands_si(146)
    assert bands["n_bands"] > 128
    dirs = gen.gen_dirs_product(2, 4)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    cfg = gen.Config("nb200", mesh, bands, dirs, bcs, 300.0, 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs), 6,
                     ic_eps=0.1)
    Io, To = oracle_run(oracle_mod, cfg, 6)
    out = run_ranks(bte, cfg, 2, 6)
    Ig, Tg = assemble(cfg, out)
    assert_parity(Ig, Tg, Io, To)


def test_band_sharding_enoconv_on_every_rank(bte, oracle_mod):
    """The failing strip (16 x 2, pulse at x = 9, 10) band-sharded over 2 ranks
    (one row each): the cells that fail (x = 12, internal box ids 24, 25) lie
    in rank 1's chunk of the solve (c_lo = 16), the -T marker reaches rank 0
    through the all-gather, and every rank returns ENOCONV after step 4 with
    the oracle's state of that step."""
    cfg = gen.failing_strip_config(nx=16, x0=9)
    p = oracle_mod.problem_from_config(cfg)
    I0, T0 = p.initial_state(cfg.t_init, mult_fn=cfg.ic_mult)
    Io, To, _, k, rc = p.run_until_failure(I0, T0, cfg.dt, cfg.nsteps)
    assert k == 4
    out = run_ranks(bte, cfg, 2, cfg.nsteps)
    for o in out:
        assert o[6] == bte.BTE_ENOCONV and o[5]["steps"] == 4
    Ig, Tg = assemble(cfg, out)
    assert rel_err(Ig, Io) <= RTOL_I and rel_err(Tg, To) <= RTOL_T


# ------------------------------------------------------------------ cell partitioning (N3)
@pytest.mark.parametrize("parts,groups", [(3, 1), (2, 2)])
def test_cell_partitions_through_bte_step(bte, oracle_mod, parts, groups):
    """C2 cut into coordinate-bisection parts, alone (3 x 1) and hybrid with
    band sharding (2 parts x 2 band groups: the halo send / receive group within
    a band group, the energy over the split communicator of a part)."""
    cfg = dataclasses.replace(gen.make_config("C2"), nsteps=10)
    Io, To = oracle_run(oracle_mod, cfg, 10)
    out = run_ranks(bte, cfg, parts * groups, 10, n_cell_parts=parts)
    Ig, Tg = assemble(cfg, out)
    assert_parity(Ig, Tg, Io, To)
    assert all(o[5]["halo_bytes"] > 0 for o in out)


def test_zslab_box_partitions_rate_law(bte, oracle_mod):
    """A 3-D box grid cut into 2 z slabs x 2 band groups (the box kernel reads
    the neighbour slab's halo layer), temperature-dependent rates: the ranks
    agree on the dt bound of the hottest cell (all-reduce max) every step."""
    cfg = gen.small_3d_config((34, 9, 12), n_spectral=3)
    law = gen.with_rate_law(cfg.bands)
    cfg = dataclasses.replace(cfg, bands=law, dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, law, cfg.dirs, t_max=350.0))
    Io, To = oracle_run(oracle_mod, cfg, 8)
    out = run_ranks(bte, cfg, 4, 8, n_cell_parts=2)
    assert all(o[5]["flux_variant"] == 6 for o in out)
    Ig, Tg = assemble(cfg, out)
    assert_parity(Ig, Tg, Io, To)


def test_group_size_mismatch_is_einval(bte):
    cfg = gen.make_config("C1")
    with bte.Group(3) as g:
        with pytest.raises(bte.BTEError) as e:
            bte.solver_from_config(cfg, rank=0, world=2, group=g)
        assert e.value.status == bte.BTE_EINVAL


def test_band_sharding_rates_now(bte, oracle_mod):
    """Band sharding over 3 ranks with the literal rate bookkeeping (reading
    26): the chunk solves and the finish kernel keep the rate temperature at T."""
    cfg = gen.small_3d_config((34, 9, 7), n_spectral=5)
    law = gen.with_rate_law(cfg.bands)
    cfg = dataclasses.replace(cfg, bands=law, dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, law, cfg.dirs, t_max=350.0))
    Io, To = oracle_run(oracle_mod, cfg, 10, rates_now=True)
    out = run_ranks(bte, cfg, 3, 10, rates_now=True)
    Ig, Tg = assemble(cfg, out)
    assert_parity(Ig, Tg, Io, To)
