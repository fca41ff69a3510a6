"""Pins of the CPU oracle against what the paper and the mathematics fix.

SURVEY.md 8(c) pins P1-P13.  None of these re-types the oracle's update
formula: each checks an invariant, a closed form, a textbook special case,
an independent (dense-matrix / bisection) formulation, or paper values.
"""
import json
import math
import os

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen

HBAR, KB = 1.054571817e-34, 1.380649e-23
GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_counts.json")


def _prob(oracle_mod, mesh, bands, dirs, bcs, rule=0):
    return oracle_mod.Problem(mesh, bands, dirs, bcs, temp_rule=rule)


def _fig1_small(nx=8, ny=6, nspec=4, dirs=None, t_hot=350.0, h=1e-6):
    mesh = gen.gen_mesh((nx, ny), (h, h))
    bands = gen.gen_bands_si(nspec)
    dirs = dirs or gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, t_hot=t_hot, radius=2 * h)
    return mesh, bands, dirs, bcs


# ----------------------------------------------------------------- P12 (paper values)
def test_p12_band_rows_match_paper():
    g = json.load(open(GOLDEN))
    b = gen.gen_bands_si(g["n_spectral_bands"])
    assert b["n_bands"] == g["band_rows"]
    assert int((b["polarization"] == gen.TA).sum()) == g["ta_rows"]
    assert g["dirs_2d"] * b["n_bands"] == g["dof_per_cell_2d"]
    assert gen.gen_dirs_product(20, 20)["n_dirs"] * b["n_bands"] == g["pdes_3d"]
    nc = g["mesh_2d"][0] * g["mesh_2d"][1]
    assert abs(nc * g["dof_per_cell_2d"] / g["total_dof_2d_approx"] - 1) < 0.02
    # the same rule on the C2 config: 10 spectral -> 13 rows
    assert gen.gen_bands_si(10)["n_bands"] == 13


def test_direction_sets_are_quadratures():
    for d in (gen.gen_dirs_product(20, 20), gen.gen_dirs_product(4, 8), gen.gen_dirs_inplane(20)):
        assert abs(d["w"].sum() - 4 * np.pi) < 1e-12
        assert np.allclose(np.linalg.norm(d["s"], axis=1), 1.0, atol=1e-15)
        # first moment vanishes (symmetric set)
        assert np.abs((d["w"][:, None] * d["s"]).sum(0)).max() < 1e-12


# ----------------------------------------------------------------- P1 (invariant)
@pytest.mark.parametrize("dim", [2, 3])
def test_p1_equilibrium_invariance(oracle_mod, dim):
    if dim == 2:
        mesh, bands, dirs, _ = _fig1_small()
    else:
        mesh = gen.gen_mesh((5, 4, 3), (1e-6,) * 3)
        bands, dirs = gen.gen_bands_si(4), gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, t_hot=300.0, radius=2e-6)  # every ISO wall at T0
    p = _prob(oracle_mod, mesh, bands, dirs, bcs)
    T0 = np.full(mesh["n_cells"], 300.0)
    I0 = p.equilibrium(T0)
    dt = 0.9 * gen.cartesian_dt_bound(mesh, bands, dirs)
    # first step: flux terms cancel and I0(T) - I = 0 exactly -> bit-identical
    I1, T1 = p.run(I0, T0, dt, 1)
    assert np.array_equal(I1, I0)
    assert np.max(np.abs(T1 / 300.0 - 1.0)) < 1e-15
    # later steps only see the rounding of T (sum_d w_d I0 != W I0 in floating point)
    I, T = p.run(I0, T0, dt, 20)
    assert np.max(np.abs(I / I0 - 1.0)) < 2e-14
    assert np.max(np.abs(T / 300.0 - 1.0)) < 1e-14


# ----------------------------------------------------------------- P2 (invariant)
def _total_energy(p, I, vols, vg):
    # sum_c V_c sum_b (1/v_b) sum_d w_d I  (energy density of the intensity field)
    w = p.keep["w"]
    e = np.einsum("d,bdc->bc", w, I) / vg[:, None]
    return float((e * vols[None, :]).sum())


@pytest.mark.parametrize("shape", [(6, 5), (4, 3, 3)])
def test_p2_energy_conserved_under_reflective_walls_R2(oracle_mod, shape):
    mesh = gen.gen_mesh(shape, (1e-6,) * len(shape))
    bands = gen.gen_bands_si(4)
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_uniform(mesh, gen.SYMMETRY)
    p = _prob(oracle_mod, mesh, bands, dirs, bcs, rule=0)
    I0, T0 = p.initial_state(300.0, ic_eps=0.3)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    e0 = _total_energy(p, I0, mesh["cell_volume"], bands["vg"])
    I, T = p.run(I0, T0, dt, 30)
    e1 = _total_energy(p, I, mesh["cell_volume"], bands["vg"])
    assert abs(e1 / e0 - 1.0) < 1e-13
    # R1 (c_b = 1/v_b) does not conserve it for non-gray bands: the rule matters
    p1 = _prob(oracle_mod, mesh, bands, dirs, bcs, rule=1)
    T0r1, _ = p1.newton(p1.energy(I0), T0)
    Ir1, _ = p1.run(I0, T0r1, dt, 30)
    assert abs(_total_energy(p1, Ir1, mesh["cell_volume"], bands["vg"]) / e0 - 1.0) > 1e-6


# ----------------------------------------------------------------- P3 (closed form)
def test_p3_gray_newton_closed_form(oracle_mod):
    mesh = gen.gen_mesh((5, 4), (1e-6, 1e-6))
    bands = gen.gen_bands_si(1)
    dirs = gen.gen_dirs_inplane(8)
    p = _prob(oracle_mod, mesh, bands, dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY))
    rng = np.random.default_rng(7)
    c = p.weight(0)
    W = dirs["w"].sum()
    theta = HBAR * bands["omega"][0] / KB
    T_true = rng.uniform(50.0, 900.0, mesh["n_cells"])
    # E that corresponds to T_true, written from the closed form of I0's inverse
    Cb = bands["C"][0]
    E = W * c * Cb / np.expm1(theta / T_true)
    T, _ = p.newton(E, np.full(mesh["n_cells"], 300.0))
    T_closed = theta / np.log1p(W * c * Cb / E)
    assert np.max(np.abs(T / T_closed - 1)) < 1e-13
    assert np.max(np.abs(T / T_true - 1)) < 1e-12


# ----------------------------------------------------------------- P13 (round trip)
def test_p13_temperature_round_trip_55_rows(oracle_mod):
    mesh = gen.gen_mesh((7, 3), (1e-6, 1e-6))
    bands = gen.gen_bands_si(40)
    dirs = gen.gen_dirs_product(4, 8)
    for rule in (0, 1):
        p = _prob(oracle_mod, mesh, bands, dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY), rule)
        T = np.linspace(20.0, 1500.0, mesh["n_cells"])
        E = p.energy(p.equilibrium(T))
        Tn, iters = p.newton(E, T * 1.15)
        assert np.max(np.abs(Tn / T - 1)) < 1e-13
        assert (iters >= 1).all()


# ----------------------------------------------------------------- P4 (mirror)
def _mirror_index(dirs, axis):
    s = dirs["s"].copy()
    s[:, axis] *= -1
    return np.array([int(np.argmin(np.abs(dirs["s"] - v).sum(1))) for v in s])


def test_p4_mirror_symmetry_fig1(oracle_mod):
    nx, ny = 10, 6
    mesh, bands, dirs, bcs = _fig1_small(nx, ny)
    p = _prob(oracle_mod, mesh, bands, dirs, bcs)
    T0 = np.full(mesh["n_cells"], 300.0)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    I, T = p.run(p.equilibrium(T0), T0, dt, 25)
    Tg = T.reshape(ny, nx)
    assert Tg.max() > 300.5  # the hot spot has heated the domain
    assert np.max(np.abs(Tg / Tg[:, ::-1] - 1)) < 1e-13
    m = _mirror_index(dirs, 0)
    Ig = I.reshape(bands["n_bands"], dirs["n_dirs"], ny, nx)
    assert np.max(np.abs(Ig / Ig[:, m][:, :, :, ::-1] - 1)) < 1e-13


# ----------------------------------------------------------------- P5 (brute force)
def _dense_step_operator(mesh, bands, dirs, bcs, T, dt, rule_weights):
    """Independent formulation: assemble I^{n+1} = M I^n + q face by face."""
    nc, nb, nd = mesh["n_cells"], bands["n_bands"], dirs["n_dirs"]
    n = nb * nd * nc
    idx = lambda b, d, c: (b * nd + d) * nc + c
    M = np.zeros((n, n))
    q = np.zeros(n)
    theta = HBAR * bands["omega"] / KB
    I0 = lambda b, t: bands["C"][b] / np.expm1(theta[b] / t)
    refl = {}
    off = mesh["face_offsets"]
    for b in range(nb):
        inv_tau = 0.0 if np.isinf(bands["tau"][b]) else 1.0 / bands["tau"][b]
        for d in range(nd):
            s = dirs["s"][d]
            for c in range(nc):
                row = idx(b, d, c)
                k = dt * bands["vg"][b] / mesh["cell_volume"][c]
                M[row, row] += 1.0 - dt * inv_tau
                q[row] += dt * inv_tau * I0(b, T[c])
                for f in range(off[c], off[c + 1]):
                    nrm = mesh["face_normal"][f]
                    a = mesh["face_area"][f]
                    mu = float(s @ nrm)
                    nbr = mesh["face_nbr"][f]
                    if mu > 0:
                        M[row, row] -= k * a * mu
                    elif nbr >= 0:
                        M[row, idx(b, d, nbr)] -= k * a * mu
                    else:
                        bf = -1 - nbr
                        if bcs["kind"][bf] == gen.ISOTHERMAL:
                            q[row] -= k * a * mu * I0(b, bcs["t_wall"][bf])
                        else:
                            key = (tuple(nrm), d)
                            if key not in refl:
                                rs = s - 2 * mu * nrm
                                refl[key] = int(np.argmin(np.abs(dirs["s"] - rs).sum(1)))
                            M[row, idx(b, refl[key], c)] -= k * a * mu
    return M, q


def _bisect_T(bands, W, wts, E, lo=1.0, hi=5000.0):
    theta = HBAR * bands["omega"] / KB
    g = lambda t: W * np.sum(wts * bands["C"] / np.expm1(theta / t)) - E
    for _ in range(200):
        mid = 0.5 * (lo + hi)
        lo, hi = (mid, hi) if g(mid) < 0 else (lo, mid)
    return 0.5 * (lo + hi)


@pytest.mark.parametrize("nb", [1, 3])
def test_p5_brute_force_dense_operator(oracle_mod, nb):
    mesh = gen.gen_mesh((4, 4), (1e-6, 1e-6))
    # 1 row (gray) / 3 rows (2 LA + 1 TA of the 3-band Si table)
    bands = gen.gen_bands_si(1) if nb == 1 else gen.select_bands(gen.gen_bands_si(3), [0, 1, 3])
    assert bands["n_bands"] == nb and (nb == 1 or bands["polarization"][2] == gen.TA)
    dirs = gen.gen_dirs_inplane(8)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    p = _prob(oracle_mod, mesh, bands, dirs, bcs)
    I, T = p.initial_state(300.0, ic_eps=0.2)
    dt = 0.7 * gen.cartesian_dt_bound(mesh, bands, dirs)
    wts = 1.0 / (bands["vg"] * bands["tau"])  # R2 weights, written independently
    W = dirs["w"].sum()
    for _ in range(3):
        M, q = _dense_step_operator(mesh, bands, dirs, bcs, T, dt, wts)
        I_ref = (M @ I.ravel() + q).reshape(I.shape)
        I_or, T_or = p.run(I, T, dt, 1)
        assert np.max(np.abs(I_or / I_ref - 1)) < 1e-13
        E = np.einsum("b,d,bdc->c", wts, dirs["w"], I_ref)
        T_ref = np.array([_bisect_T(bands, W, wts, e) for e in E])
        assert np.max(np.abs(T_or / T_ref - 1)) < 1e-13
        I, T = I_or, T_or


# ----------------------------------------------------------------- P6 (1D upwind)
def test_p6_courant_one_exact_shift(oracle_mod):
    nx = 8
    mesh = gen.gen_mesh((nx, 1), (1.0, 1.0))
    bands = gen.gen_bands_custom(omega=1e13, vg=1.0, tau=np.inf, C=1.0)
    dirs = gen.gen_dirs_axes2d()  # +x, -x, +y, -y
    t_w, t_e = 250.0, 400.0
    bcs = gen.gen_bcs_walls(mesh, {gen.WALL_XM: (gen.ISOTHERMAL, t_w), gen.WALL_XP: (gen.ISOTHERMAL, t_e),
                                   gen.WALL_YM: (gen.SYMMETRY, 0), gen.WALL_YP: (gen.SYMMETRY, 0)})
    p = _prob(oracle_mod, mesh, bands, dirs, bcs, rule=1)
    I = np.arange(1, 1 + 4 * nx, dtype=np.float64).reshape(1, 4, nx)
    T = np.full(nx, 300.0)
    gw, ge = p.I0(0, t_w), p.I0(0, t_e)
    for step in range(1, 4):
        In, T = p.run(I, T, 1.0, 1)
        # +x: shift right by one cell, west-wall ghost enters at cell 0
        assert np.array_equal(In[0, 0, 1:], I[0, 0, :-1])
        assert abs(In[0, 0, 0] / gw - 1) < 1e-15
        # -x: shift left, east-wall ghost enters at the last cell
        assert np.array_equal(In[0, 1, :-1], I[0, 1, 1:])
        assert abs(In[0, 1, -1] / ge - 1) < 1e-15
        # +-y: only reflective walls in y -> the pair exchanges exactly
        assert np.array_equal(In[0, 2], I[0, 3]) and np.array_equal(In[0, 3], I[0, 2])
        I = In


# ----------------------------------------------------------------- P7 (images)
def test_p7_method_of_images(oracle_mod):
    nx, ny, h = 12, 5, 1e-6
    bands = gen.gen_bands_si(3)
    dirs = gen.gen_dirs_product(4, 8)
    full = gen.gen_mesh((nx, ny), (h, h))
    half = gen.gen_mesh((nx // 2, ny), (h, h))
    hot = lambda fc: 300 + 50 * np.exp(-2 * (fc[:, 0] - 0.5 * nx * h) ** 2 / (2 * h) ** 2)
    walls = lambda: {gen.WALL_XM: (gen.SYMMETRY, 0), gen.WALL_XP: (gen.SYMMETRY, 0),
                     gen.WALL_YM: (gen.ISOTHERMAL, 300.0), gen.WALL_YP: (gen.ISOTHERMAL, hot)}
    pf = _prob(oracle_mod, full, bands, dirs, gen.gen_bcs_walls(full, walls()))
    ph = _prob(oracle_mod, half, bands, dirs, gen.gen_bcs_walls(half, walls()))
    dt = 0.5 * gen.cartesian_dt_bound(full, bands, dirs)
    If, Tf = pf.run(pf.equilibrium(300.0), np.full(nx * ny, 300.0), dt, 20)
    Ih, Th = ph.run(ph.equilibrium(300.0), np.full(nx // 2 * ny, 300.0), dt, 20)
    assert Tf.max() > 300.2
    assert np.max(np.abs(Tf.reshape(ny, nx)[:, : nx // 2] / Th.reshape(ny, nx // 2) - 1)) < 1e-13
    Ifg = If.reshape(bands["n_bands"], dirs["n_dirs"], ny, nx)[..., : nx // 2]
    assert np.max(np.abs(Ifg / Ih.reshape(Ifg.shape) - 1)) < 1e-13


# ----------------------------------------------------------------- P8 (relaxation)
def test_p8_relaxation_closed_form(oracle_mod):
    mesh = gen.gen_mesh((1, 1), (1e-6, 1e-6))
    bands = gen.gen_bands_custom(omega=2e13, vg=5e3, tau=2e-12, C=1e6)
    dirs = gen.gen_dirs_inplane(8)
    p = _prob(oracle_mod, mesh, bands, dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY))
    # g constant on reflection orbits with zero weighted mean: cos(2 phi) on the
    # orbit representative (phi -> pi - phi, phi -> -phi keep cos 2 phi).
    phi = (np.arange(8) + 0.5) * np.pi / 4
    g = np.where(np.isclose(np.abs(np.cos(phi)), np.cos(np.pi / 8)), 1.0, -1.0)  # sign cos 2phi
    assert abs((dirs["w"] * g).sum()) == 0.0
    Ts, eps = 310.0, 0.05
    I0s = p.I0(0, Ts)
    I = (I0s * (1 + eps * g)).reshape(1, 8, 1)
    T, _ = p.newton(p.energy(I), np.array([300.0]))
    dt = 0.3e-12
    n = 25
    In, Tn = p.run(I, T, dt, n)
    expect = I0s + (1 - dt / 2e-12) ** n * (I - I0s)
    assert np.max(np.abs(In / expect - 1)) < 1e-13
    assert abs(Tn[0] / Ts - 1) < 1e-13


# ----------------------------------------------------------------- P9 (ballistic)
def test_p9_ballistic_slab_steady_state(oracle_mod):
    nx = 6
    mesh = gen.gen_mesh((nx, 1), (1.0, 1.0))
    bands = gen.gen_bands_custom(omega=[1e13, 3e13], vg=[1.0, 0.7], tau=np.inf, C=[1.0, 2.0])
    dirs = gen.gen_dirs_inplane(8)
    t1, t2 = 280.0, 330.0
    bcs = gen.gen_bcs_walls(mesh, {gen.WALL_XM: (gen.ISOTHERMAL, t1), gen.WALL_XP: (gen.ISOTHERMAL, t2),
                                   gen.WALL_YM: (gen.SYMMETRY, 0), gen.WALL_YP: (gen.SYMMETRY, 0)})
    p = _prob(oracle_mod, mesh, bands, dirs, bcs, rule=1)
    T0 = np.full(nx, 300.0)
    I, T = p.run(p.equilibrium(T0), T0, 0.5, 3000)
    sx = dirs["s"][:, 0]
    for b in range(2):
        exp_b = np.where(sx > 0, p.I0(b, t1), p.I0(b, t2))[:, None]
        assert np.max(np.abs(I[b] / exp_b - 1)) < 1e-13
    W = dirs["w"].sum()
    E_expect = sum(p.weight(b) * 0.5 * W * (p.I0(b, t1) + p.I0(b, t2)) for b in range(2))
    assert np.max(np.abs(p.energy(I) / E_expect - 1)) < 1e-13


# ----------------------------------------------------------------- P10 (max principle)
def test_p10_max_principle_at_bound(oracle_mod):
    mesh, bands, dirs, bcs = _fig1_small(8, 8, nspec=4, t_hot=350.0)
    p = _prob(oracle_mod, mesh, bands, dirs, bcs)
    T0 = np.full(mesh["n_cells"], 300.0)
    dt = gen.cartesian_dt_bound(mesh, bands, dirs)  # CFL-extreme: exactly the bound
    I, T = p.run(p.equilibrium(T0), T0, dt, 40)
    lo = p.equilibrium(np.full(mesh["n_cells"], 300.0))
    hi = p.equilibrium(np.full(mesh["n_cells"], 350.0))
    assert (I >= lo * (1 - 1e-14)).all() and (I <= hi * (1 + 1e-14)).all()
    assert T.min() >= 300.0 * (1 - 1e-14) and T.max() <= 350.0
    assert T.max() > 301.0


# ----------------------------------------------------------------- P11 (relabelling)
def test_p11_permutation_invariance(oracle_mod):
    mesh, bands, dirs, bcs = _fig1_small(7, 5, nspec=2)
    pm, perm = gen.permute_mesh(mesh)
    p = _prob(oracle_mod, mesh, bands, dirs, bcs)
    q = _prob(oracle_mod, pm, bands, dirs, bcs)
    I, T = p.initial_state(300.0, ic_eps=0.2)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    I1, T1 = p.run(I, T, dt, 10)
    I2, T2 = q.run(I[:, :, perm], T[perm], dt, 10)
    assert np.max(np.abs(I2 / I1[:, :, perm] - 1)) < 1e-14
    assert np.max(np.abs(T2 / T1[perm] - 1)) < 1e-14


# ----------------------------------------------------------------- helpers of the oracle
def test_sampled_step_matches_full_step(oracle_mod):
    cfg = gen.small_3d_config((5, 4, 3))
    p = oracle_mod.problem_from_config(cfg)
    rng = np.random.default_rng(3)
    T0 = 300.0 + 20.0 * rng.random(cfg.mesh["n_cells"])
    full = p.update_intensity(T0, p.equilibrium(T0), cfg.dt)
    T1, _ = p.newton(p.energy(full), T0)
    cells = np.array([0, 7, 33, cfg.mesh["n_cells"] - 1])
    out, T1s = p.step_cells_equilibrium(T0, cells, cfg.dt)
    assert np.array_equal(out, np.transpose(full[:, :, cells], (2, 0, 1)))
    assert np.array_equal(T1s, T1[cells])


def test_unclosed_reflection_is_rejected(oracle_mod):
    mesh = gen.gen_mesh((3, 3), (1e-6, 1e-6))
    dirs = gen.gen_dirs_inplane(7)  # odd in-plane set: x-mirror not in the set
    p = _prob(oracle_mod, mesh, gen.gen_bands_si(1), dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY))
    with pytest.raises(ValueError):
        p.reflection_map()
