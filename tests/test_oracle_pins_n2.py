"""Pins of the oracle on unstructured meshes.

The face-based method (Eq. 3: any polyhedral cell, "A_i is the area
of face i") on triangle meshes: each pin checks what the mathematics fixes,
independently of the oracle's loop -- equilibrium invariance (a closed cell's
sum_f A_f n_f = 0), exact energy conservation with specular walls (R2), cell
relabelling, and the dense affine step map assembled face by face.
"""
import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests.test_oracle_pins import _bisect_T, _dense_step_operator, _total_energy


def _tri(nx=5, ny=4, h=1e-6):
    return gen.gen_mesh_tri((nx, ny), (h, 1.5 * h))


def test_triangle_mesh_is_closed_and_consistent():
    m = _tri(6, 5)
    off = m["face_offsets"]
    for c in range(m["n_cells"]):
        f = slice(off[c], off[c + 1])
        assert np.abs((m["face_area"][f][:, None] * m["face_normal"][f]).sum(0)).max() < 1e-21
        assert abs(np.linalg.norm(m["face_normal"][f], axis=1) - 1).max() < 1e-15
    assert abs(m["cell_volume"].sum() - 6 * 5 * 1e-6 * 1.5e-6) < 1e-24


def test_n2_equilibrium_invariance_triangles(oracle_mod):
    m = _tri()
    bands, dirs = gen.gen_bands_si(3), gen.gen_dirs_inplane(12)
    bcs = gen.gen_bcs_fig1(m, t_hot=300.0, radius=2e-6)
    p = oracle_mod.Problem(m, bands, dirs, bcs)
    T0 = np.full(m["n_cells"], 300.0)
    I0 = p.equilibrium(T0)
    dt = 0.9 * gen.general_dt_bound(m, bands, dirs)
    I, T = p.run(I0, T0, dt, 20)
    assert np.max(np.abs(I / I0 - 1)) < 2e-14 and np.max(np.abs(T / 300.0 - 1)) < 1e-14


def test_n2_energy_conserved_specular_triangles(oracle_mod):
    m = _tri(6, 5)
    bands, dirs = gen.gen_bands_si(4), gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_uniform(m, gen.SYMMETRY)
    p = oracle_mod.Problem(m, bands, dirs, bcs)
    I0, T0 = p.initial_state(300.0, ic_eps=0.3)
    dt = 0.5 * gen.general_dt_bound(m, bands, dirs)
    e0 = _total_energy(p, I0, m["cell_volume"], bands["vg"])
    I, T = p.run(I0, T0, dt, 30)
    assert abs(_total_energy(p, I, m["cell_volume"], bands["vg"]) / e0 - 1) < 1e-13


def test_n2_permutation_invariance_triangles(oracle_mod):
    m = _tri(5, 4)
    pm, perm = gen.permute_mesh(m, seed=3)
    bands, dirs = gen.gen_bands_si(2), gen.gen_dirs_inplane(8)
    bcs = gen.gen_bcs_fig1(m, radius=2e-6)
    p = oracle_mod.Problem(m, bands, dirs, bcs)
    q = oracle_mod.Problem(pm, bands, dirs, bcs)
    I, T = p.initial_state(300.0, ic_eps=0.2)
    dt = 0.5 * gen.general_dt_bound(m, bands, dirs)
    I1, T1 = p.run(I, T, dt, 10)
    I2, T2 = q.run(I[:, :, perm], T[perm], dt, 10)
    assert np.max(np.abs(I2 / I1[:, :, perm] - 1)) < 1e-14
    assert np.max(np.abs(T2 / T1[perm] - 1)) < 1e-14


def test_n2_brute_force_dense_operator_triangles(oracle_mod):
    m = _tri(3, 2)
    bands = gen.select_bands(gen.gen_bands_si(3), [0, 3])
    dirs = gen.gen_dirs_inplane(8)
    bcs = gen.gen_bcs_fig1(m, radius=2e-6)
    p = oracle_mod.Problem(m, bands, dirs, bcs)
    I, T = p.initial_state(300.0, ic_eps=0.2)
    dt = 0.7 * gen.general_dt_bound(m, bands, dirs)
    wts = 1.0 / (bands["vg"] * bands["tau"])
    W = dirs["w"].sum()
    for _ in range(3):
        M, q = _dense_step_operator(m, bands, dirs, bcs, T, dt, wts)
        I_ref = (M @ I.ravel() + q).reshape(I.shape)
        I, T = p.run(I, T, dt, 1)
        assert np.max(np.abs(I / I_ref - 1)) < 1e-13
        E = np.einsum("b,d,bdc->c", wts, dirs["w"], I_ref)
        T_ref = np.array([_bisect_T(bands, W, wts, e) for e in E])
        assert np.max(np.abs(T / T_ref - 1)) < 1e-12


@pytest.mark.parametrize("name", ["C6", "C6t"])
def test_n2_fig10_corner_source_stays_bounded(oracle_mod, name):
    """Fig.-10 workload: the corner source heats the material within the wall
    range (max principle, P10) and the hottest cell is next to the corner."""
    cfg = gen.make_config(name)
    p = oracle_mod.problem_from_config(cfg)
    I, T = p.initial_state(cfg.t_init, ic_eps=0.0)
    I, T = p.run(I, T, cfg.dt, 100)
    assert 100.0 * (1 - 1e-14) <= T.min() and T.max() <= 150.0 and T.max() > 105.0
    cen = cfg.mesh["cell_centre"]
    hot = cen[np.argmax(T)]
    assert hot[0] < 0.25 * cen[:, 0].max() and hot[1] > 0.75 * cen[:, 1].max()


# ----------------------------------------------------------------- N4 (R3 first-law step)
def _rule_run(oracle_mod, rule, eps, steps=1, t_hot=350.0):
    mesh = gen.gen_mesh((6, 5), (1e-6, 1e-6))
    bands, dirs = gen.gen_bands_si(4), gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, t_hot=t_hot, radius=2e-6)
    p = oracle_mod.Problem(mesh, bands, dirs, bcs, temp_rule=rule)
    T0 = np.full(mesh["n_cells"], 300.0)
    I0 = p.equilibrium(T0)
    from paper_conf_ipps_heislersdms24_b200.inputs import ic_multiplier
    for b in range(bands["n_bands"]):
        I0[b] *= ic_multiplier(dirs["n_dirs"], mesh["n_cells"], b, eps)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    return p.run(I0, T0, dt, steps)


def test_n4_r3_is_second_order_close_to_r1(oracle_mod):
    """R3 is one Newton step of the R1 equation from T^n: its error against the
    converged R1 temperature is quadratic in the temperature change, so halving
    the perturbation divides the gap by ~4 (and equilibrium gives no change)."""
    gaps, moves = [], []
    for eps in (0.08, 0.04, 0.02):
        _, T1 = _rule_run(oracle_mod, 1, eps)
        _, T3 = _rule_run(oracle_mod, 2, eps)
        gaps.append(np.max(np.abs(T3 - T1)))
        moves.append(np.max(np.abs(T1 - 300.0)))
    assert gaps[0] > 0 and all(g < 1e-2 * m for g, m in zip(gaps, moves))
    r1, r2 = gaps[0] / gaps[1], gaps[1] / gaps[2]
    assert 3.0 < r1 < 5.0 and 3.0 < r2 < 5.0, (gaps, moves)
    _, Te = _rule_run(oracle_mod, 2, 0.0, steps=5, t_hot=300.0)  # equilibrium: nothing moves
    assert np.max(np.abs(Te / 300.0 - 1)) < 1e-14
