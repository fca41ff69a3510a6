"""GPU parity, round 2: the temperature solve's bisection branch in both
Newton kernels, the ENOCONV stop at the failing step, the built-in I0
prefactors, and the benched 3-D box path at the north star's 100-step horizon.

Everything through the C ABI (bte.py), element by element against the CPU
oracle on the same seeded inputs (RTOL_I = 1e-10 on I, RTOL_T = 1e-9 on T).
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


# ------------------------------------------------------------------ bisection
@pytest.mark.parametrize("kernel", ["warp", "thread"])
@pytest.mark.parametrize("name", ["C2", "box3d55"])
def test_bisection_branch_both_newton_kernels(bte, oracle_mod, monkeypatch, kernel, name):
    """newton_max_iter = 1: every cell's solve leaves Newton unconverged and
    takes the bisection safeguard (iters > maxit reported), in the warp-per-cell
    kernel and the thread-per-cell kernel (BTE_NEWTON forces either; the IC's
    re-solve always runs the thread kernel).  Against the oracle with the same
    maxit, 10 steps."""
    monkeypatch.setenv("BTE_NEWTON", kernel)
    if name == "C2":
        cfg = dataclasses.replace(gen.make_config("C2"), nsteps=10)
    else:  # the bench's 55 rows on a 3-D box grid with two tiles per axis, 24 directions
        h = 8.2e-6
        mesh = gen.gen_mesh((34, 9, 5), (h, h, h))
        bands, dirs = gen.gen_bands_si(40), gen.gen_dirs_product(4, 6)
        bcs = gen.gen_bcs_fig1(mesh, radius=4 * h)
        cfg = gen.Config("box3d55", mesh, bands, dirs, bcs, 300.0, 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs),
                         10, ic_eps=0.1)
    Io, To = oracle_run(oracle_mod, cfg, 10, maxit=1)
    Ig, Tg, st = gpu_run(cfg, 10, newton_max_iter=1)
    assert st["newton_iter_max"] == 2  # (maxit + 1: the bisection branch ran)
    assert_parity(Ig, Tg, Io, To)


def test_bisection_c3_full_size(bte, oracle_mod, monkeypatch):
    """C3 exactly as benched (120 x 120, 55 rows, 400 directions) with the
    bisection branch in the warp kernel (the one C3 runs), 2 steps, every element."""
    cfg = gen.make_config("C3")
    Io, To = oracle_run(oracle_mod, cfg, 2, maxit=1)
    Ig, Tg, st = gpu_run(cfg, 2, newton_max_iter=1)
    assert st["newton_iter_max"] == 2
    assert_parity(Ig, Tg, Io, To)


# ------------------------------------------------------------------ ENOCONV at the failing step
@pytest.mark.parametrize("kw", [{}, {"profile": True}, {"box": False}, {"tma": False},
                                {"newton": "thread"}, {"newton": "warp", "profile": True}])
def test_enoconv_stops_at_failing_step(bte, oracle_mod, monkeypatch, kw):
    """inputs.failing_strip_config fails in step 4 of 10.  bte_step returns
    ENOCONV with the state at the end of step 4 (the oracle's, failed cells at
    their step-3 T), 4 steps counted; with and without the 2-step CUDA graph,
    on the box kernel, the paired TMA kernel and the register kernel, both
    Newton kernels.  A further bte_step fails in its first step."""
    kw = dict(kw)
    if "newton" in kw:
        monkeypatch.setenv("BTE_NEWTON", kw.pop("newton"))
    cfg = gen.failing_strip_config()
    p = oracle_mod.problem_from_config(cfg)
    I0, T0 = p.initial_state(cfg.t_init, mult_fn=cfg.ic_mult)
    Io, To, _, k, rc = p.run_until_failure(I0, T0, cfg.dt, cfg.nsteps)
    assert rc == oracle_mod.ENOCONV and k == 4
    with bte.solver_from_config(cfg, **kw) as s:
        bte.apply_ic(s, cfg)
        with pytest.raises(bte.BTEError) as e:
            s.step(cfg.dt, cfg.nsteps)
        assert e.value.status == bte.BTE_ENOCONV
        st = s.stats()
        assert st["steps"] == 4
        Ig, Tg = s.intensity(), s.temperature()
        with pytest.raises(bte.BTEError) as e:
            s.step(cfg.dt, 3)
        assert e.value.status == bte.BTE_ENOCONV and s.stats()["steps"] == 5
    assert rel_err(Ig, Io) <= RTOL_I
    assert rel_err(Tg, To) <= RTOL_T


# ------------------------------------------------------------------ built-in prefactors
def test_i0_prefactor_null_uses_builtin_dispersion(bte):
    """bte_bands.i0_prefactor = NULL: C_b from the library's built-in Si
    dispersion gives the same state as the generator's C_b."""
    cfg = dataclasses.replace(gen.make_config("C2"), nsteps=5)
    a = gpu_run(cfg, 5)
    b = gpu_run(cfg, 5, i0_prefactor=False)
    assert rel_err(b[0], a[0]) < 1e-13 and rel_err(b[1], a[1]) < 1e-13
    bad = dict(cfg.bands, omega=cfg.bands["omega"] * 1.5)  # above the LA branch maximum
    with pytest.raises(bte.BTEError) as e:
        bte.Solver(cfg.mesh, bad, cfg.dirs, cfg.bcs, i0_prefactor=False)
    assert e.value.status == bte.BTE_EINVAL


# ------------------------------------------------------------------ benched 3-D path, 100 steps
def test_box3d_bench_tables_100_steps(bte, oracle_mod):
    """The benched 3-D path at the north star's horizon: the bench's 55-row x
    400-direction tables on a 34 x 10 x 10 box grid (two 32 x 8 tiles per
    axis with ragged tails, two z ranges of L = 8), seeded IC, 100 steps, in
    the bench's launch plan (5 band-rows x 20 orbits per CTA), every element."""
    h = 8.2e-6
    mesh = gen.gen_mesh((34, 10, 10), (h, h, h))
    bands, dirs = gen.gen_bands_si(40), gen.gen_dirs_product(20, 20)
    bcs = gen.gen_bcs_fig1(mesh, radius=4 * h)
    cfg = gen.Config("box100", mesh, bands, dirs, bcs, 300.0, 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs), 100,
                     ic_eps=0.1)
    Io, To = oracle_run(oracle_mod, cfg, 100)
    Ig, Tg, st = gpu_run(cfg, 100, band_group=5, dir_chunk=80)
    assert st["flux_variant"] == 6 and st["band_group"] == 5 and st["dir_chunks"] == 5
    assert_parity(Ig, Tg, Io, To)


# ------------------------------------------------------------------ full-size C4, direction-dependent state
def _neighbourhood(mesh, cells):
    off, nbr = mesh["face_offsets"], mesh["face_nbr"]
    sub = set(int(c) for c in cells)
    for c in cells:
        sub.update(int(v) for v in nbr[off[c]:off[c + 1]] if v >= 0)
    return np.array(sorted(sub))


def _sample_cells(cfg, seed):
    nc = cfg.mesh["n_cells"]
    nx, ny, nz = cfg.mesh["shape"]
    rng = np.random.default_rng(seed)
    corners = [0, nx - 1, nx * ny - 1, nc - 1, nx * (ny - 1), nc - nx, nx * ny * (nz - 1)]
    return np.unique(np.concatenate([corners, rng.integers(0, nc, 24),
                                     [nx // 2 + nx * (ny // 2) + nx * ny * (nz - 1), nx // 2 + nx * (ny // 2)]]))


def _gpu_sampled_step(s, cfg, cells):
    nc = cfg.mesh["n_cells"]
    T_ic = s.temperature()
    s.step(cfg.dt, 1)
    Tg = s.temperature()
    Ig_sel = np.empty((cells.size, s.n_bands, s.n_dirs))
    buf = np.empty((1, s.n_dirs, nc))
    for b in range(s.n_bands):
        s.intensity(b, b + 1, out=buf)
        Ig_sel[:, b, :] = buf[0][:, cells].T
    return T_ic, Ig_sel, Tg


def test_sampled_full_size_c4_bench_ic(bte, oracle_mod):
    """C4 at full size in the bench's launch configuration from the bench's
    seeded, direction-dependent IC (equilibrium at t_init x the generator's
    per-(band, direction, cell) multiplier, T from its energy): one step, the
    sampled cells (corners, wall centres, random) against the oracle's subset
    step, whose face-neighbour state is rebuilt from the same generator."""
    cfg = gen.make_config("C4")
    nc, nb, nd = cfg.mesh["n_cells"], cfg.bands["n_bands"], cfg.dirs["n_dirs"]
    cells = _sample_cells(cfg, 12)
    sub = _neighbourhood(cfg.mesh, cells)
    p = oracle_mod.problem_from_config(cfg)
    I_sub = np.empty((nb, nd, sub.size))
    for b in range(nb):
        I_sub[b] = p.I0(b, cfg.t_init) * gen.ic_multiplier(nd, nc, b, cfg.ic_eps)[:, sub]
    T_sub = p.subset_initial(sub, I_sub, cfg.t_init)
    Io_sel, To_sel = p.step_subset(sub, I_sub, T_sub, np.searchsorted(sub, cells), cfg.dt)
    with bte.solver_from_config(cfg) as s:
        bte.apply_ic(s, cfg)
        T_ic, Ig_sel, Tg = _gpu_sampled_step(s, cfg, cells)
    assert rel_err(T_ic[sub], T_sub) <= RTOL_T
    assert rel_err(Ig_sel, Io_sel) <= RTOL_I
    assert rel_err(Tg[cells], To_sel) <= RTOL_T


def test_sampled_full_size_c5_direction_dependent(bte, oracle_mod):
    """C5 (96^3, 156 GB of state, slab rotation) at full size: a non-uniform
    and direction-dependent state I = I0_b(T0_c) x m_b(d) (seeded random T0,
    a per-(band, direction) multiplier), T from its energy, one step; sampled
    cells against the oracle's subset step."""
    cfg = gen.make_config("C5")
    nc, nb, nd = cfg.mesh["n_cells"], cfg.bands["n_bands"], cfg.dirs["n_dirs"]
    rng = np.random.default_rng(6)
    T0 = 300.0 + 40.0 * rng.random(nc)
    mult = 1.0 + 0.1 * np.sin(0.37 * np.arange(nd)[None, :] + 1.3 * np.arange(nb)[:, None])  # [nb][nd]
    cells = _sample_cells(cfg, 13)
    sub = _neighbourhood(cfg.mesh, cells)
    p = oracle_mod.problem_from_config(cfg)
    I_sub = np.empty((nb, nd, sub.size))
    for b in range(nb):
        I_sub[b] = np.array([p.I0(b, t) for t in T0[sub]])[None, :] * mult[b][:, None]
    T_sub = p.subset_initial(sub, I_sub, T0[sub])
    Io_sel, To_sel = p.step_subset(sub, I_sub, T_sub, np.searchsorted(sub, cells), cfg.dt)
    with bte.solver_from_config(cfg) as s:
        st = s.stats()
        assert st["spare_slabs"] < s.n_bands and st["flux_variant"] == 6  # slab rotation, box kernel
        s.set_equilibrium(T0)
        buf = np.empty((1, nd, nc))
        for b in range(nb):
            s.intensity(b, b + 1, out=buf)
            buf[0] *= mult[b][:, None]
            s.set_intensity(buf, b, b + 1)
        s.solve_temperature()
        T_ic, Ig_sel, Tg = _gpu_sampled_step(s, cfg, cells)
    assert rel_err(T_ic[sub], T_sub) <= RTOL_T
    assert rel_err(Ig_sel, Io_sel) <= RTOL_I
    assert rel_err(Tg[cells], To_sel) <= RTOL_T
