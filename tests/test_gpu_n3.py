"""GPU parity of cell partitioning, through the C ABI.

The paper's cell-parallel split (L728-735, L768-772, Fig. 3-4): every rank
owns a part of the cells and, before each step, receives the old-level
intensities its cut faces read from the neighbour parts (halo), optionally
combined with band sharding (world = parts x band groups; the energy is
reduced over the ranks of the same part).  The pool reaches one GPU at a time,
so the ranks are emulated on one device as independent contexts without a
communicator: the test moves the halo with bte_halo_export / bte_halo_import
(what the library's NCCL group of sends / receives does) and sums the energy of
the band groups (the all-reduce).  Results must match the unpartitioned CPU
oracle to the north-star tolerance (relative 1e-10 on I, 1e-9 on T).
"""
import dataclasses

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import dist as bdist
from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import assert_parity, oracle_run

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bte():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


def run_partitioned(bte, cfg, n_parts, groups, nsteps, parts=None, T0=None, **kw):
    """world = n_parts x groups emulated ranks (rank r: part r % P, band group
    r // P).  IC: the config's seeded IC (groups == 1) or equilibrium at T0.
    Returns the assembled global I, T and every rank's stats."""
    if parts is None:
        parts = bdist.partition_cells(cfg.mesh["cell_centre"], n_parts)
    world = n_parts * groups
    ss = [bte.solver_from_config(cfg, rank=r, world=world, cell_part=parts, n_cell_parts=n_parts, **kw)
          for r in range(world)]
    try:
        for s in ss:
            if T0 is None:
                assert groups == 1
                bte.apply_ic(s, cfg)
            else:
                s.set_equilibrium(T0[s.local_cells()])
        for _ in range(nsteps):
            for g in range(groups):
                grp = ss[g * n_parts:(g + 1) * n_parts]  # index in the group = part
                bufs = {(a, b): grp[a].halo_export(b) for a in range(n_parts) for b in range(n_parts) if a != b}
                for (a, b), buf in bufs.items():
                    grp[b].halo_import(a, buf)
            for s in ss:
                s.step_begin(cfg.dt)
            if groups > 1:
                for p in range(n_parts):
                    rk = [ss[g * n_parts + p] for g in range(groups)]
                    E = sum(r.energy() for r in rk)
                    for r in rk:
                        r.set_energy(E)
            for s in ss:
                s.step_finish()
        nc = cfg.mesh["n_cells"]
        nb, nd = cfg.bands["n_bands"], cfg.dirs["n_dirs"]
        I = np.full((nb, nd, nc), np.nan)
        T = np.full(nc, np.nan)
        for s in ss:
            ids = s.local_cells()
            assert np.array_equal(ids, np.flatnonzero(parts == parts[ids[0]]))
            Tl = s.temperature()
            if s.b_lo == 0:
                T[ids] = Tl
            else:  # every band group solves the same cells: identical bits
                assert np.array_equal(T[ids], Tl)
            I[s.b_lo:s.b_hi][:, :, ids] = s.intensity()
        stats = [s.stats() for s in ss]
    finally:
        for s in ss:
            s.close()
    assert np.all(np.isfinite(I)) and np.all(np.isfinite(T))
    return I, T, stats


@pytest.mark.parametrize("n_parts", [2, 3, 5])
def test_c1_cell_parts(bte, oracle_mod, n_parts):
    cfg = gen.make_config("C1")
    Io, To = oracle_run(oracle_mod, cfg, cfg.nsteps)
    Ig, Tg, st = run_partitioned(bte, cfg, n_parts, 1, cfg.nsteps)
    assert_parity(Ig, Tg, Io, To)
    assert all(s["halo_bytes"] > 0 for s in st)


def test_c2_four_parts(bte, oracle_mod):
    cfg = gen.make_config("C2")
    Io, To = oracle_run(oracle_mod, cfg, 30)
    Ig, Tg, _ = run_partitioned(bte, cfg, 4, 1, 30)
    assert_parity(Ig, Tg, Io, To)


def test_triangles_three_parts(bte, oracle_mod):
    """Unstructured triangles (C6t, N2): cut faces with many distinct normals."""
    cfg = gen.make_config("C6t")
    Io, To = oracle_run(oracle_mod, cfg, 30)
    Ig, Tg, _ = run_partitioned(bte, cfg, 3, 1, 30)
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("shape,n_parts", [((13, 7, 5), 4), ((34, 9, 5), 2), ((6, 5, 4), 7)])
def test_3d_cell_parts(bte, oracle_mod, shape, n_parts):
    cfg = gen.small_3d_config(shape, n_spectral=3)
    Io, To = oracle_run(oracle_mod, cfg, 10)
    Ig, Tg, _ = run_partitioned(bte, cfg, n_parts, 1, 10)
    assert_parity(Ig, Tg, Io, To)


def test_slab_rotation_cell_parts(bte, oracle_mod):
    cfg = gen.small_3d_config((13, 7, 5), n_spectral=3)
    Io, To = oracle_run(oracle_mod, cfg, 8)
    Ig, Tg, st = run_partitioned(bte, cfg, 3, 1, 8, max_spare_slabs=2)
    assert st[0]["spare_slabs"] == 2
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("n_parts,groups", [(2, 2), (3, 2), (2, 3)])
def test_hybrid_band_x_cell(bte, oracle_mod, n_parts, groups):
    """Parts x band groups: halo within a band group, energy over a part."""
    cfg = gen.make_config("C2")
    rng = np.random.default_rng(11)
    T0 = 300.0 + 20 * rng.random(cfg.mesh["n_cells"])
    p = oracle_mod.problem_from_config(cfg)
    Io, To = p.run(p.equilibrium(T0), T0, cfg.dt, 10)
    Ig, Tg, _ = run_partitioned(bte, cfg, n_parts, groups, 10, T0=T0)
    assert_parity(Ig, Tg, Io, To)


def test_rate_law_cell_parts(bte, oracle_mod):
    cfg = gen.small_3d_config((13, 7, 5), n_spectral=3)
    law = gen.with_rate_law(cfg.bands)
    cfg = dataclasses.replace(cfg, bands=law,
                              dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, law, cfg.dirs, t_max=350.0))
    Io, To = oracle_run(oracle_mod, cfg, 8)
    Ig, Tg, _ = run_partitioned(bte, cfg, 3, 1, 8)
    assert_parity(Ig, Tg, Io, To)


def test_halo_segments_z_slabs(bte):
    """Two z-slabs of a 3-D box: one segment each way, the face layer's cells,
    and only the directions that cross the cut (half of a product set with no
    s_z = 0): nb_loc x nd/2 x n_x n_y doubles each way."""
    cfg = gen.small_3d_config((8, 6, 4), n_spectral=2)
    nz = 4
    parts = np.zeros(cfg.mesh["n_cells"], np.int32)
    z = cfg.mesh["cell_centre"][:, 2]
    parts[z > np.median(z)] = 1
    ss = [bte.solver_from_config(cfg, rank=r, world=2, cell_part=parts, n_cell_parts=2) for r in range(2)]
    try:
        nb, nd = cfg.bands["n_bands"], cfg.dirs["n_dirs"]
        s01, r01 = ss[0].halo_size(1)
        s10, r10 = ss[1].halo_size(0)
        assert s01 == r10 and s10 == r01
        assert s01 == nb * (nd // 2) * 8 * 6 and s10 == s01
        assert ss[0].halo_size(0) == (0, 0)
        with pytest.raises(bte.BTEError):
            ss[0].halo_size(2)
        assert ss[0].n_cells + ss[1].n_cells == cfg.mesh["n_cells"] and ss[0].n_cells == 8 * 6 * nz // 2
        with pytest.raises(bte.BTEError):  # no communicator: the caller moves the halo
            ss[0].step(cfg.dt, 1)
    finally:
        for s in ss:
            s.close()


def test_partition_errors(bte):
    cfg = gen.make_config("C1")
    nc = cfg.mesh["n_cells"]
    parts = bdist.partition_cells(cfg.mesh["cell_centre"], 2)
    with pytest.raises(bte.BTEError) as e:  # world not a multiple of the parts
        bte.solver_from_config(cfg, rank=0, world=3, cell_part=parts, n_cell_parts=2)
    assert e.value.status == bte.BTE_EINVAL
    with pytest.raises(bte.BTEError):  # part 2 has no cells
        bte.solver_from_config(cfg, rank=2, world=3, cell_part=parts, n_cell_parts=3)
    bad = parts.copy()
    bad[7] = 5
    with pytest.raises(bte.BTEError):  # part id out of range
        bte.solver_from_config(cfg, rank=0, world=2, cell_part=bad, n_cell_parts=2)
    one = np.zeros(nc, np.int32)  # one part: no halo, the whole mesh
    with bte.solver_from_config(cfg, cell_part=one, n_cell_parts=1) as s:
        assert s.n_cells == nc and s.stats()["halo_bytes"] == 0
        assert np.array_equal(s.local_cells(), np.arange(nc))


def _zslab_parts(cfg, bounds):
    """Part id per cell from the z layer: part k owns layers [bounds[k], bounds[k+1])."""
    nx, ny, nz = cfg.mesh["shape"]
    z = np.arange(cfg.mesh["n_cells"]) // (nx * ny)
    return (np.searchsorted(np.asarray(bounds[1:-1]), z, side="right")).astype(np.int32)


@pytest.mark.parametrize("shape,bounds", [((34, 9, 8), (0, 4, 8)), ((34, 9, 8), (0, 2, 5, 8)),
                                          ((16, 9, 6), (0, 1, 2, 4, 6)), ((32, 16, 9), (0, 5, 9))])
def test_zslab_partition_box_kernel(bte, oracle_mod, shape, bounds):
    """Cell parts made of whole z layers of a structured 3-D grid keep the box
    kernel (halo layers around the owned ones; 1-layer parts included)."""
    cfg = gen.small_3d_config(shape, n_spectral=3)
    parts = _zslab_parts(cfg, bounds)
    Io, To = oracle_run(oracle_mod, cfg, 8)
    Ig, Tg, st = run_partitioned(bte, cfg, len(bounds) - 1, 1, 8, parts=parts)
    assert all(s["flux_variant"] == 6 for s in st)
    assert_parity(Ig, Tg, Io, To)


def test_zslab_partition_walls_law_hybrid(bte, oracle_mod):
    """z-slab parts with specular z walls (the z-mirrored ghost at the global
    walls), the rate law, and a 2 x 2 hybrid with band groups."""
    cfg = gen.small_3d_config((34, 9, 8), n_spectral=3)
    bcs = gen.gen_bcs_walls(cfg.mesh, {w: (gen.SYMMETRY, 0) for w in range(6)})
    law = gen.with_rate_law(cfg.bands)
    c_spec = dataclasses.replace(cfg, bcs=bcs)
    c_law = dataclasses.replace(cfg, bands=law,
                                dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, law, cfg.dirs, t_max=350.0))
    parts = _zslab_parts(cfg, (0, 3, 8))
    for c in (c_spec, c_law):
        Io, To = oracle_run(oracle_mod, c, 6)
        Ig, Tg, st = run_partitioned(bte, c, 2, 1, 6, parts=parts)
        assert all(s["flux_variant"] == 6 for s in st)
        assert_parity(Ig, Tg, Io, To)
    rng = np.random.default_rng(4)
    T0 = 300.0 + 20 * rng.random(cfg.mesh["n_cells"])
    p = oracle_mod.problem_from_config(cfg)
    Io, To = p.run(p.equilibrium(T0), T0, cfg.dt, 6)
    Ig, Tg, st = run_partitioned(bte, cfg, 2, 2, 6, parts=parts, T0=T0)
    assert all(s["flux_variant"] == 6 for s in st)
    assert_parity(Ig, Tg, Io, To)
