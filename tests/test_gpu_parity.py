"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Element by element on the same seeded inputs: relative 1e-10 on I and 1e-9 on
T (north star), at sizes that span several thread blocks with ragged tails, in
every launch configuration the library can pick (band groups, block sizes,
direction chunking, slab rotation), plus sampled outputs at the full bench
size.
"""
import dataclasses

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import RTOL_I, RTOL_T, assert_parity, gpu_run, oracle_run, rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bte():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


def _cfg(name, steps=None, **kw):
    cfg = gen.make_config(name)
    if steps is not None:
        cfg = dataclasses.replace(cfg, nsteps=steps)
    return dataclasses.replace(cfg, **kw) if kw else cfg


# ------------------------------------------------------------------ configs
def test_c1_full_50_steps(bte, oracle_mod):
    cfg = _cfg("C1")
    Io, To = oracle_run(oracle_mod, cfg, cfg.nsteps)
    Ig, Tg, st = gpu_run(cfg, cfg.nsteps)
    assert_parity(Ig, Tg, Io, To)
    assert st["flux_variant"] == 6  # a 2-D quad grid with Fig.-1 walls: the box kernel
    assert st["steps"] == cfg.nsteps
    assert To.max() > 300.5  # the hot spot moved heat in


@pytest.mark.parametrize("bg", [1, 2, 4, 8])
@pytest.mark.parametrize("threads", [64, 256])
def test_c1_launch_configs(bte, oracle_mod, bg, threads):
    cfg = _cfg("C1", steps=20)
    Io, To = oracle_run(oracle_mod, cfg, 20)
    Ig, Tg, st = gpu_run(cfg, 20, band_group=bg, block_threads=threads)
    assert_parity(Ig, Tg, Io, To)


def test_c2_100_steps(bte, oracle_mod):
    cfg = _cfg("C2", steps=100)
    Io, To = oracle_run(oracle_mod, cfg, 100)
    Ig, Tg, st = gpu_run(cfg, 100)
    assert_parity(Ig, Tg, Io, To)
    assert st["newton_iter_max"] >= 2


@pytest.mark.parametrize("spare", [1, 3, 5])
def test_slab_rotation_matches(bte, oracle_mod, spare):
    """Slab rotation (nb + k slabs, band batches per launch) == oracle."""
    cfg = _cfg("C2", steps=30)
    Io, To = oracle_run(oracle_mod, cfg, 30)
    Ig, Tg, st = gpu_run(cfg, 30, max_spare_slabs=spare, band_group=4)
    assert st["spare_slabs"] == spare
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("shape", [(6, 5, 4), (13, 7, 5), (33, 9, 3)])
def test_3d_ragged(bte, oracle_mod, shape):
    cfg = gen.small_3d_config(shape, n_spectral=3, ntheta=4, nphi=8)
    Io, To = oracle_run(oracle_mod, cfg, 25)
    Ig, Tg, _ = gpu_run(cfg, 25)
    assert_parity(Ig, Tg, Io, To)


def test_3d_400_dirs_55_rows_small_mesh(bte, oracle_mod):
    """The bench's band table and direction set on a small 3-D mesh."""
    h = 8.2e-6
    mesh = gen.gen_mesh((7, 6, 5), (h, h, h))
    bands, dirs = gen.gen_bands_si(40), gen.gen_dirs_product(20, 20)
    bcs = gen.gen_bcs_fig1(mesh, radius=2 * h)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    cfg = gen.Config("3d55", mesh, bands, dirs, bcs, 300.0, dt, 10, ic_eps=0.1)
    Io, To = oracle_run(oracle_mod, cfg, 10)
    Ig, Tg, _ = gpu_run(cfg, 10)
    assert_parity(Ig, Tg, Io, To)


def test_c3_mesh_scaled_short(bte, oracle_mod):
    """C3 (paper's 120 x 120, 55 rows) with 24 of the 400 directions, 5 steps."""
    cfg = _cfg("C3")
    dirs = gen.gen_dirs_product(4, 6)
    dt = 0.5 * gen.cartesian_dt_bound(cfg.mesh, cfg.bands, dirs)
    cfg = dataclasses.replace(cfg, dirs=dirs, dt=dt)
    Io, To = oracle_run(oracle_mod, cfg, 5)
    Ig, Tg, _ = gpu_run(cfg, 5)
    assert_parity(Ig, Tg, Io, To)


def test_c3_paper_faithful_dt(bte, oracle_mod):
    """Paper regime: IC 300 K, dt = 1 ps (L1328), reduced direction set."""
    cfg = gen.make_config("C3", variant="paper")
    dirs = gen.gen_dirs_inplane(20)  # the paper's 2-D set of 20 (L594-595)
    cfg = dataclasses.replace(cfg, dirs=dirs, bands=gen.select_bands(cfg.bands, np.arange(0, 55, 6)))
    Io, To = oracle_run(oracle_mod, cfg, 20)
    Ig, Tg, _ = gpu_run(cfg, 20)
    assert_parity(Ig, Tg, Io, To)


# ------------------------------------------------------------------ edge cases
def test_single_cell_all_walls(bte, oracle_mod):
    mesh = gen.gen_mesh((1, 1), (1e-6, 1e-6))
    bands = gen.gen_bands_si(4)
    dirs = gen.gen_dirs_product(2, 8)
    bcs = gen.gen_bcs_walls(mesh, {gen.WALL_XM: (gen.ISOTHERMAL, 320.0), gen.WALL_XP: (gen.SYMMETRY, 0),
                                   gen.WALL_YM: (gen.ISOTHERMAL, 290.0), gen.WALL_YP: (gen.SYMMETRY, 0)})
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    cfg = gen.Config("1cell", mesh, bands, dirs, bcs, 300.0, dt, 10, ic_eps=0.2)
    Io, To = oracle_run(oracle_mod, cfg, 10)
    Ig, Tg, st = gpu_run(cfg, 10)
    assert st["n_interior_cells"] == 0  # the one cell has four wall faces
    assert_parity(Ig, Tg, Io, To)


def test_no_boundary_cells_periodic_like(bte, oracle_mod):
    """A mesh with no boundary faces at all (a periodic 4 x 3 torus)."""
    mesh = gen.gen_mesh((4, 3), (1e-6, 1e-6))
    nbr = mesh["face_nbr"].reshape(-1, 4).copy()
    c = np.arange(12)
    i, j = c % 4, c // 4
    nbr[:, 0] = (i - 1) % 4 + 4 * j
    nbr[:, 1] = (i + 1) % 4 + 4 * j
    nbr[:, 2] = i + 4 * ((j - 1) % 3)
    nbr[:, 3] = i + 4 * ((j + 1) % 3)
    mesh = dict(mesh, face_nbr=nbr.ravel(), n_bfaces=0)
    bcs = {"n_bfaces": 0, "kind": np.zeros(0, np.int32), "t_wall": np.zeros(0)}
    bands, dirs = gen.gen_bands_si(3), gen.gen_dirs_inplane(12)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    cfg = gen.Config("torus", mesh, bands, dirs, bcs, 300.0, dt, 10, ic_eps=0.3)
    Io, To = oracle_run(oracle_mod, cfg, 15)
    Ig, Tg, st = gpu_run(cfg, 15)
    assert st["n_interior_cells"] == 12
    assert_parity(Ig, Tg, Io, To)


def test_ballistic_row_with_R1(bte, oracle_mod):
    """A tau = inf band-row (no scattering) under temp_rule 1 (c_b = 1/v_b)."""
    mesh = gen.gen_mesh((9, 7), (1e-6, 1e-6))
    bands = gen.gen_bands_si(3)
    bands["tau"][1] = np.inf
    dirs = gen.gen_dirs_inplane(16)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    cfg = gen.Config("ballistic", mesh, bands, dirs, bcs, 300.0, dt, 10, ic_eps=0.1, temp_rule=1)
    Io, To = oracle_run(oracle_mod, cfg, 30)
    Ig, Tg, _ = gpu_run(cfg, 30)
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("bg", [1, 2, 4])
def test_generic_face_path_2d_3d(bte, oracle_mod, bg):
    """The generic (unpaired) face-slot kernel: forced on a 3-D Fig.-1 problem,
    and chosen by the library for a 2-D mesh with split (hanging) faces."""
    cfg = gen.small_3d_config((9, 5, 4), n_spectral=2)
    Io, To = oracle_run(oracle_mod, cfg, 12)
    Ig, Tg, _ = gpu_run(cfg, 12, generic_faces=True, band_group=bg)
    assert_parity(Ig, Tg, Io, To)
    c2 = _cfg("C1", steps=12)
    bands = gen.gen_bands_si(3)
    c2 = dataclasses.replace(c2, mesh=gen.split_faces(c2.mesh), bands=bands,
                             dt=0.5 * gen.cartesian_dt_bound(c2.mesh, bands, c2.dirs))
    Io, To = oracle_run(oracle_mod, c2, 12)
    Ig, Tg, _ = gpu_run(c2, 12, band_group=bg)
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("bg", [1, 3, 4, 8])
def test_register_pipelined_kernel(bte, oracle_mod, bg):
    """The register-pipelined generic-face kernel (BTE_FLAG_NO_TMA): paired meshes
    then take the generic layout, uniform and per-cell geometry."""
    cfg = gen.small_3d_config((13, 7, 5), n_spectral=3, ntheta=4, nphi=8)
    Io, To = oracle_run(oracle_mod, cfg, 10)
    Ig, Tg, _ = gpu_run(cfg, 10, tma=False, band_group=bg)
    assert_parity(Ig, Tg, Io, To)
    c2 = _cfg("C2", steps=10)
    Io, To = oracle_run(oracle_mod, c2, 10)
    Ig, Tg, _ = gpu_run(c2, 10, tma=False, band_group=bg)
    assert_parity(Ig, Tg, Io, To)


def test_graded_mesh_per_cell_geometry(bte, oracle_mod):
    """Non-uniform (graded) cell sizes: paired but not uniform geometry, on the
    TMA kernel and the register kernel."""
    cfg = gen.small_3d_config((9, 8, 5), n_spectral=2)
    m = dict(cfg.mesh)
    scale = np.repeat(1.0 + 0.5 * (np.arange(m["n_cells"]) % 3), 6)
    m["face_area"] = m["face_area"] * scale
    m["cell_volume"] = m["cell_volume"] * (1.0 + 0.5 * (np.arange(m["n_cells"]) % 3)) * 1.7
    cfg = dataclasses.replace(cfg, mesh=m, dt=0.25 * cfg.dt)
    Io, To = oracle_run(oracle_mod, cfg, 10)
    for tma in (True, False):
        Ig, Tg, _ = gpu_run(cfg, 10, tma=tma)
        assert_parity(Ig, Tg, Io, To)


def test_locality_order_is_invisible(bte):
    """The Morton-order hint changes only the internal layout: bitwise equal."""
    cfg = gen.small_3d_config((11, 6, 5), n_spectral=3)
    a = gpu_run(cfg, 8, locality=True)
    b = gpu_run(cfg, 8, locality=False)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


def test_permuted_unstructured_order(bte, oracle_mod):
    """Random cell labels and face order: the generic connectivity path."""
    cfg = gen.small_3d_config((7, 5, 4), n_spectral=2)
    mesh, _ = gen.permute_mesh(cfg.mesh, seed=11)
    cfg = dataclasses.replace(cfg, mesh=mesh)
    Io, To = oracle_run(oracle_mod, cfg, 15)
    Ig, Tg, _ = gpu_run(cfg, 15)
    assert_parity(Ig, Tg, Io, To)


def test_zero_steps_is_identity_and_dt_bound(bte, oracle_mod):
    cfg = _cfg("C1")
    with bte.solver_from_config(cfg) as s:
        bte.apply_ic(s, cfg)
        I0 = s.intensity()
        s.step(cfg.dt, 0)
        assert np.array_equal(s.intensity(), I0)
        assert abs(s.dt_bound() / cfg.extra["dt_bound"] - 1) < 1e-12
        with pytest.raises(bte.BTEError) as e:
            s.step(s.dt_bound() * 1.01, 1)
        assert e.value.status == bte.BTE_EINVAL
        with pytest.raises(bte.BTEError):
            s.step(-1.0, 1)


def test_equilibrium_invariance_full_bench_size(bte):
    """P1 at the bench size: all walls at T0, uniform IC -> I and T stay put."""
    cfg = _cfg("C4")
    bcs = gen.gen_bcs_fig1(cfg.mesh, t_hot=300.0)
    with bte.Solver(cfg.mesh, cfg.bands, cfg.dirs, bcs, t_init=300.0) as s:
        I0 = s.intensity(0, 1)
        s.step(cfg.dt, 3)
        T = s.temperature()
        assert np.max(np.abs(T / 300.0 - 1)) < 1e-13
        assert rel_err(s.intensity(0, 1), I0) < 1e-13
        last = s.b_hi - 1
        I_last = s.intensity(last, last + 1)
    with bte.Solver(cfg.mesh, cfg.bands, cfg.dirs, bcs, t_init=300.0) as s2:
        assert rel_err(I_last, s2.intensity(last, last + 1)) < 1e-13


def test_split_step_band_sharding_emulated(bte, oracle_mod):
    """Band sharding over 2 'ranks' on one device: each context owns half the
    rows; the caller sums the energy partials (the all-reduce) and both finish.
    Must equal the single-context result and the oracle."""
    cfg = _cfg("C2", steps=10)
    rng = np.random.default_rng(9)
    T0 = 300.0 + 20 * rng.random(cfg.mesh["n_cells"])
    p = oracle_mod.problem_from_config(cfg)
    Io, To = p.run(p.equilibrium(T0), T0, cfg.dt, 10)
    ranks = [bte.solver_from_config(cfg, rank=r, world=2) for r in range(2)]
    try:
        for s in ranks:
            s.set_equilibrium(T0)
        with pytest.raises(bte.BTEError):
            ranks[0].step(cfg.dt, 1)  # no communicator: split calls only
        for _ in range(10):
            for s in ranks:
                s.step_begin(cfg.dt)
            E = ranks[0].energy() + ranks[1].energy()
            for s in ranks:
                s.set_energy(E)
                s.step_finish()
        Ts = [s.temperature() for s in ranks]
        assert np.array_equal(Ts[0], Ts[1])
        Ig = np.concatenate([s.intensity() for s in ranks], axis=0)
        assert [(s.b_lo, s.b_hi) for s in ranks] == [(0, 6), (6, 13)]
    finally:
        for s in ranks:
            s.close()
    assert_parity(Ig, Ts[0], Io, To)


@pytest.mark.parametrize("newton", ["auto", "thread", "lanes8", "warp"])
def test_nccl_allreduce_path_one_rank(bte, monkeypatch, newton):
    """The NCCL code path (dlopen, ncclCommInitRank, per-step ncclAllReduce of E
    summed by sum_slots_kernel) on a one-rank communicator: bitwise equal to the
    fused single-GPU path, whose solve kernel sums the energy slots itself (in
    sum_slots_kernel's order) -- for the thread-per-cell and the 8 / 32-lane solves."""
    if newton != "auto":
        monkeypatch.setenv("BTE_NEWTON", newton)
    cfg = _cfg("C2", steps=5)
    a = gpu_run(cfg, 5)
    b = gpu_run(cfg, 5, nccl_id=bte.nccl_unique_id(), profile=True)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert b[2]["ms_allreduce"] > 0.0


def test_profile_stats(bte):
    cfg = _cfg("C2")
    with bte.solver_from_config(cfg, profile=True) as s:
        s.step(cfg.dt, 3)
        st = s.stats()
    assert st["steps"] == 3 and st["kernel_launches"] >= 6 and st["kernel_launches"] % 3 == 0
    assert st["ms_flux_interior"] > 0 and st["ms_newton"] > 0 and st["ms_total"] > 0
    assert st["updates"] == 3 * cfg.n_updates_per_step


def test_nan_energy_reports_enoconv(bte):
    cfg = _cfg("C1")
    with bte.solver_from_config(cfg) as s:
        I = s.intensity()
        I[:, :, 5] = -1.0  # negative energy in one cell: no temperature exists
        s.set_intensity(I)
        with pytest.raises(bte.BTEError) as e:
            s.solve_temperature()
        assert e.value.status == bte.BTE_ENOCONV


def test_nccl_sharded_solve_modes_one_rank(bte, monkeypatch):
    """The band-sharded step exchange on a one-rank communicator, both modes:
    reduce-scatter + chunk solve + all-gather (default) and all-reduce +
    replicated solve (BTE_SHARD_NEWTON=replicated); both bitwise equal to the
    single-GPU path, with and without the rate law, on the box kernel."""
    cfg = gen.small_3d_config((34, 9, 5), n_spectral=3)
    law = dataclasses.replace(cfg, bands=gen.with_rate_law(cfg.bands),
                              dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, gen.with_rate_law(cfg.bands), cfg.dirs,
                                                               t_max=350.0))
    for c in (cfg, law):
        a = gpu_run(c, 6)
        for mode in ("shard", "replicated"):
            monkeypatch.setenv("BTE_SHARD_NEWTON", mode)
            b = gpu_run(c, 6, nccl_id=bte.nccl_unique_id())
            assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]), mode
        monkeypatch.delenv("BTE_SHARD_NEWTON")


def test_nccl_sharded_step_reports_enoconv(bte):
    """A failed cell in the chunk solve is flagged on every rank (negative
    marker through the all-gather) and keeps T^n."""
    cfg = _cfg("C1")
    with bte.solver_from_config(cfg, nccl_id=bte.nccl_unique_id()) as s:
        T_before = s.temperature()
        I = s.intensity()
        I[:, :, 5] = -1e13  # the step's energy of cell 5 stays negative
        s.set_intensity(I)
        with pytest.raises(bte.BTEError) as e:
            s.step(cfg.dt, 1)
        assert e.value.status == bte.BTE_ENOCONV
        assert s.temperature()[5] == T_before[5]


def test_c3_full_size_elementwise(bte, oracle_mod):
    """C3 exactly as benched (2-D 120 x 120, all 55 rows, all 400 directions,
    seeded IC, dt = 0.5 x bound), 3 steps, every element against the oracle."""
    cfg = _cfg("C3")
    Io, To = oracle_run(oracle_mod, cfg, 3)
    Ig, Tg, st = gpu_run(cfg, 3)
    assert st["flux_variant"] == 6
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("name", ["C1", "C2", "box3d", "law2d"])
def test_cuda_graph_replay_is_bitwise_equal(bte, oracle_mod, name):
    """bte_step(n >= 4) on one GPU replays a captured 2-step CUDA graph; the
    per-phase profiling mode launches every kernel instead.  Same bits, for odd
    n, a dt change (re-capture) and the rate law (rate halves flip per step)."""
    if name == "box3d":
        cfg = gen.small_3d_config((34, 9, 5), n_spectral=3)
    elif name == "law2d":
        c0 = _cfg("C2")
        law = gen.with_rate_law(c0.bands)
        cfg = dataclasses.replace(c0, bands=law, dt=0.5 * gen.cartesian_dt_bound(c0.mesh, law, c0.dirs, t_max=350.0))
    else:
        cfg = _cfg(name)
    out = []
    for profile in (False, True):
        with bte.solver_from_config(cfg, profile=profile) as s:
            bte.apply_ic(s, cfg)
            s.step(cfg.dt, 7)
            s.step(0.5 * cfg.dt, 6)
            s.step(cfg.dt, 5)
            st = s.stats()
            out.append((s.intensity(), s.temperature(), st["steps"], st["updates"], st["graph_replays"]))
    assert np.array_equal(out[0][0], out[1][0]) and np.array_equal(out[0][1], out[1][1])
    assert out[0][2:4] == out[1][2:4] == (18, 18 * cfg.n_updates_per_step)
    assert out[0][4] >= 6 and out[1][4] == 0  # graph replays (7 + 6 + 5 steps) / none when profiling
    if name == "C1":  # and the graph path against the oracle
        p = oracle_mod.problem_from_config(cfg)
        I, T, Tr = p.initial_state(cfg.t_init, ic_eps=cfg.ic_eps, with_tr=True)
        I, T, Tr = p.run(I, T, cfg.dt, 7, Tr=Tr)
        I, T, Tr = p.run(I, T, 0.5 * cfg.dt, 6, Tr=Tr)
        I, T, Tr = p.run(I, T, cfg.dt, 5, Tr=Tr)
        assert_parity(out[0][0], out[0][1], I, T)


def test_cuda_graph_with_nccl_one_rank(bte, monkeypatch):
    """The graph path with the NCCL exchange captured (one-rank communicator,
    both exchange modes): bitwise equal to launching every kernel."""
    cfg = _cfg("C2")
    ref = gpu_run(cfg, 9, profile=True)  # no graph, no communicator
    for mode in ("shard", "replicated"):
        monkeypatch.setenv("BTE_SHARD_NEWTON", mode)
        g = gpu_run(cfg, 9, nccl_id=bte.nccl_unique_id())
        assert np.array_equal(ref[0], g[0]) and np.array_equal(ref[1], g[1]), mode
        assert g[2]["graph_replays"] >= 3 and ref[2]["graph_replays"] == 0, mode
