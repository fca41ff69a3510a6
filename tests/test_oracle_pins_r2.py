"""More pins of the CPU oracle (round 2).

* The bisection safeguard of the temperature solve (the
  solve itself L407-418, L555-561): forced with newton_maxit = 1, and reached
  on its own when Newton from a far guess does not converge in 50 steps; both
  against the closed form of the gray inverse (P3) and the 55-row round trip
  (P13).  A flipped bracket, a wrong midpoint test or a wrong growth direction
  fails these.
* The subset step (sampled checks of full-size fields with a direction-
  dependent state) against the full-field step, which P1-P13 pin.
* The ENOCONV semantics of a failing step ("the state at the
  failing step"): oracle.run_until_failure against the step-by-step pieces.
"""
import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen

HBAR, KB = 1.054571817e-34, 1.380649e-23


def _gray(oracle_mod, maxit, rtol):
    mesh = gen.gen_mesh((5, 4), (1e-6, 1e-6))
    bands = gen.gen_bands_si(1)
    dirs = gen.gen_dirs_inplane(8)
    p = oracle_mod.Problem(mesh, bands, dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY), maxit=maxit, rtol=rtol)
    W = dirs["w"].sum()
    theta = HBAR * bands["omega"][0] / KB
    return p, W * p.weight(0) * bands["C"][0], theta, mesh["n_cells"]


@pytest.mark.parametrize("guess", [0.4, 1.0, 3.0])
def test_p3_bisection_gray_closed_form(oracle_mod, guess):
    """maxit = 1: Newton cannot meet |dT| <= rtol T in one step from a 3x /
    0.4x guess, so every cell takes the bisection branch (iters = -1) on a
    bracket grown downwards (guess above the root) or upwards (below); the
    result is the closed form T = theta / log1p(W c C / E) to 1e-13."""
    p, wcc, theta, nc = _gray(oracle_mod, maxit=1, rtol=1e-14)
    T_true = np.linspace(60.0, 900.0, nc)
    E = wcc / np.expm1(theta / T_true)
    T, iters = p.newton(E, T_true * guess if guess != 1.0 else T_true * 1.05)
    assert (iters == -1).all()
    T_closed = theta / np.log1p(wcc / E)
    assert np.max(np.abs(T / T_closed - 1)) < 1e-13


def test_p3_bisection_after_maxit(oracle_mod):
    """Default maxit = 50 from a far guess (2000 K) to 3-30 K: the coldest
    cells do not converge by Newton and fall back to bisection on their own;
    every cell agrees with the closed form."""
    p, wcc, theta, nc = _gray(oracle_mod, maxit=50, rtol=1e-14)
    T_true = np.linspace(3.0, 30.0, nc)
    E = wcc / np.expm1(theta / T_true)
    T, iters = p.newton(E, np.full(nc, 2000.0))
    assert (iters == -1).sum() >= 2 and (iters > 0).sum() >= 2
    assert np.max(np.abs(T / (theta / np.log1p(wcc / E)) - 1)) < 1e-13


def test_p13_bisection_round_trip_55_rows(oracle_mod):
    """P13 through the bisection branch: T -> E(T) -> (maxit 1) -> T, 55 rows,
    both temperature rules."""
    mesh = gen.gen_mesh((7, 3), (1e-6, 1e-6))
    bands = gen.gen_bands_si(40)
    dirs = gen.gen_dirs_product(4, 8)
    for rule in (0, 1):
        p = oracle_mod.Problem(mesh, bands, dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY), temp_rule=rule,
                               maxit=1, rtol=1e-14)
        T = np.linspace(20.0, 1500.0, mesh["n_cells"])
        E = p.energy(p.equilibrium(T))
        Tn, iters = p.newton(E, T * 1.15)
        assert (iters == -1).all()
        assert np.max(np.abs(Tn / T - 1)) < 1e-13


def test_bisection_matches_newton_in_a_run(oracle_mod):
    """A whole 20-step run with the bisection solve (maxit 1, rtol 1e-14)
    equals the Newton run to the temperature tolerance."""
    cfg = gen.small_3d_config((6, 5, 4), n_spectral=2)
    out = []
    for maxit, rtol in ((50, 1e-12), (1, 1e-14)):
        p = oracle_mod.problem_from_config(cfg, maxit=maxit, rtol=rtol)
        I, T = p.initial_state(cfg.t_init, ic_eps=cfg.ic_eps)
        out.append(p.run(I, T, cfg.dt, 20))
    assert np.max(np.abs(out[1][1] / out[0][1] - 1)) < 1e-12
    assert np.max(np.abs(out[1][0] / out[0][0] - 1)) < 1e-11


# ----------------------------------------------------------------- subsets
@pytest.mark.parametrize("law", [False, True])
def test_subset_step_equals_full_step(oracle_mod, law):
    """oracle.step_subset on sampled cells + their face neighbours, with a
    direction-dependent seeded state, is bitwise the full-field step there;
    subset_initial is bitwise the full-field temperature."""
    cfg = gen.small_3d_config((7, 6, 5), n_spectral=3)
    bands = gen.with_rate_law(cfg.bands) if law else cfg.bands
    p = oracle_mod.Problem(cfg.mesh, bands, cfg.dirs, cfg.bcs)
    I, T, Tr = p.initial_state(cfg.t_init, ic_eps=0.1, with_tr=True)
    I1, T1, _ = p.run(I, T, cfg.dt, 1, Tr=Tr)
    rng = np.random.default_rng(3)
    nc = cfg.mesh["n_cells"]
    sel_cells = np.unique(np.concatenate([[0, nc - 1], rng.integers(0, nc, 8)]))
    off, nbr = cfg.mesh["face_offsets"], cfg.mesh["face_nbr"]
    sub = set(sel_cells.tolist())
    for c in sel_cells:
        sub.update(int(v) for v in nbr[off[c]:off[c + 1]] if v >= 0)
    sub = np.array(sorted(sub))
    sel = np.searchsorted(sub, sel_cells)
    T_sub = p.subset_initial(sub, I[:, :, sub], cfg.t_init, Tr_sub=Tr[sub])
    assert np.array_equal(T_sub, T[sub])
    out, T1s = p.step_subset(sub, I[:, :, sub], T[sub], sel, cfg.dt, Tr_sub=Tr[sub])
    assert np.array_equal(out, np.transpose(I1[:, :, sel_cells], (2, 0, 1)))
    assert np.array_equal(T1s, T1[sel_cells])
    with pytest.raises(RuntimeError):  # a neighbour missing from the subset
        p.step_subset(sel_cells, I[:, :, sel_cells], T[sel_cells], np.arange(sel_cells.size), cfg.dt,
                      Tr_sub=Tr[sel_cells])


# ----------------------------------------------------------------- ENOCONV
def test_failing_step_state(oracle_mod):
    """The strip of inputs.failing_strip_config fails in step 4: steps 1-3
    succeed, the returned state is step 4's update of step 3's state, the
    failed cells keep their step-3 temperature and every other cell has its
    converged step-4 temperature."""
    cfg = gen.failing_strip_config()
    p = oracle_mod.problem_from_config(cfg)
    I0, T0 = p.initial_state(cfg.t_init, mult_fn=cfg.ic_mult)
    If, Tf, _, k, rc = p.run_until_failure(I0, T0, cfg.dt, cfg.nsteps)
    assert rc == oracle_mod.ENOCONV and k == 4
    I3, T3 = p.run(I0, T0, cfg.dt, 3)
    I4 = p.update_intensity(T3, I3, cfg.dt)
    assert np.array_equal(If, I4)
    E4 = p.energy(I4)
    bad = E4 <= 0
    assert bad.any() and (~bad).any()
    assert np.array_equal(Tf[bad], T3[bad])
    with pytest.raises(RuntimeError):
        p.newton(E4, T3)
    pg = oracle_mod.problem_from_config(cfg)
    Tg, _ = pg.newton(np.where(bad, 1.0, E4), T3)  # the good cells alone converge
    assert np.array_equal(Tf[~bad], Tg[~bad])
