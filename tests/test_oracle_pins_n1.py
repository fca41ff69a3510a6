"""Pins of the oracle's temperature-dependent relaxation times.

The paper keeps I0 and tau as per-cell variables that depend on the
temperature (L666-669; `beta` per cell, L1352-1353).  Reading 22:
1/tau_b(T) = a_b + b_b T exp(-theta_b/T), evaluated at the rate temperature
Tr, and the rates of step n are those of the temperature of step n-1 (Tr <- T
after the intensity update, before the temperature solve), so the R2 weights
of the solve and the relaxation of the next step use the same rates.

Each pin checks something the mathematics fixes, not the oracle's own loop:
a T-independent law is the constant-tau method bit for bit; equilibrium is
invariant; energy is conserved exactly under specular walls (only with the
lag of reading 22); the relaxation closed form at the rate of T*; and an
independent dense-matrix formulation with its own rate bookkeeping.
"""
import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests.test_oracle_pins import HBAR, KB, _bisect_T, _total_energy

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")


def _law(a, b, theta, T):
    return a + b * T * np.exp(-theta / T)


def test_n1_t_independent_law_is_constant_tau_bitwise(oracle_mod):
    """b = 0: 1/tau = a exactly; with a = 2^40 /s, tau = 2^-40 s is exact too."""
    mesh = gen.gen_mesh((6, 5), (1e-6, 1e-6))
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    omega, vg, C = [1e13, 3e13, 6e13], [8e3, 6e3, 3e3], [1e5, 3e6, 2e7]
    const = gen.gen_bands_custom(omega=omega, vg=vg, tau=[2.0 ** -40, 2.0 ** -38, 2.0 ** -41], C=C)
    law = dict(const, rate_a=np.array([2.0 ** 40, 2.0 ** 38, 2.0 ** 41]), rate_b=np.zeros(3),
               rate_theta=np.full(3, 140.0))
    for rule in (0, 1):
        p = oracle_mod.Problem(mesh, const, dirs, bcs, temp_rule=rule)
        q = oracle_mod.Problem(mesh, law, dirs, bcs, temp_rule=rule)
        I, T = p.initial_state(300.0, ic_eps=0.2)
        Iq, Tq, Trq = q.initial_state(300.0, ic_eps=0.2, with_tr=True)
        assert np.array_equal(I, Iq) and np.array_equal(T, Tq)
        dt = 0.5 * gen.cartesian_dt_bound(mesh, const, dirs)
        I1, T1 = p.run(I, T, dt, 15)
        I2, T2, _ = q.run(Iq, Tq, dt, 15, Tr=Trq)
        assert np.array_equal(I1, I2) and np.array_equal(T1, T2)


@pytest.mark.parametrize("dim", [2, 3])
def test_n1_equilibrium_invariance(oracle_mod, dim):
    shape = (6, 5) if dim == 2 else (4, 4, 3)
    mesh = gen.gen_mesh(shape, (1e-6,) * dim)
    bands = gen.with_rate_law(gen.gen_bands_si(4))
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, t_hot=320.0, t_cold=320.0, radius=2e-6)
    p = oracle_mod.Problem(mesh, bands, dirs, bcs)
    T0 = np.full(mesh["n_cells"], 320.0)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs, t_max=320.0)
    I, T, Tr = p.run(p.equilibrium(T0), T0, dt, 20, Tr=T0)
    assert np.max(np.abs(I / p.equilibrium(T0) - 1)) < 2e-14
    assert np.max(np.abs(T / 320.0 - 1)) < 1e-14 and np.max(np.abs(Tr / 320.0 - 1)) < 1e-14


@pytest.mark.parametrize("shape", [(6, 5), (4, 3, 3)])
def test_n1_energy_conserved_with_lagged_rates(oracle_mod, shape):
    """All walls specular, non-gray, strongly perturbed IC: the R2 balance with
    the lagged rates makes sum_c V sum_b (1/v_b) sum_d w_d I an exact invariant."""
    mesh = gen.gen_mesh(shape, (1e-6,) * len(shape))
    bands = gen.with_rate_law(gen.gen_bands_si(4))
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_uniform(mesh, gen.SYMMETRY)
    p = oracle_mod.Problem(mesh, bands, dirs, bcs)
    I0, T0, Tr0 = p.initial_state(300.0, ic_eps=0.4, with_tr=True)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs, t_max=T0.max() * 1.2)
    e0 = _total_energy(p, I0, mesh["cell_volume"], bands["vg"])
    I, T, Tr = p.run(I0, T0, dt, 30, Tr=Tr0)
    assert abs(_total_energy(p, I, mesh["cell_volume"], bands["vg"]) / e0 - 1) < 1e-13
    # the rates did change with the cell temperatures
    r0 = np.array([p.rate(0, t) for t in Tr0])
    r1 = np.array([p.rate(0, t) for t in Tr])
    assert np.max(np.abs(r1 / r0 - 1)) > 1e-4


def test_n1_relaxation_closed_form_at_rate_of_T_star(oracle_mod):
    """Single cell, specular walls, gray, a reflection-symmetric zero-mean
    perturbation: T stays T*, so every step relaxes at 1/tau(T*)."""
    mesh = gen.gen_mesh((1, 1), (1e-6, 1e-6))
    a, b, th = 1.0e11, 1.5e9, 140.0
    bands = dict(gen.gen_bands_custom(omega=2e13, vg=5e3, tau=1.0, C=1e6),
                 rate_a=np.array([a]), rate_b=np.array([b]), rate_theta=np.array([th]))
    dirs = gen.gen_dirs_inplane(8)
    p = oracle_mod.Problem(mesh, bands, dirs, gen.gen_bcs_uniform(mesh, gen.SYMMETRY))
    phi = (np.arange(8) + 0.5) * np.pi / 4
    g = np.where(np.isclose(np.abs(np.cos(phi)), np.cos(np.pi / 8)), 1.0, -1.0)
    Ts, eps = 310.0, 0.05
    I0s = p.I0(0, Ts)
    I = (I0s * (1 + eps * g)).reshape(1, 8, 1)
    T, _ = p.newton(p.energy(I, Tr=[Ts]), np.array([300.0]), Tr=[Ts])
    dt, n = 0.2e-12, 25
    In, Tn, Trn = p.run(I, T, dt, n, Tr=[Ts])
    rate = _law(a, b, th, Ts)
    expect = I0s + (1 - dt * rate) ** n * (I - I0s)
    assert np.max(np.abs(In / expect - 1)) < 1e-13
    assert abs(Tn[0] / Ts - 1) < 1e-13 and abs(Trn[0] / Ts - 1) < 1e-13


def _dense_step(mesh, bands, dirs, bcs, T, inv_tau, dt):
    """I^{n+1} = M I^n + q assembled face by face, per-(band, cell) rates."""
    nc, nb, nd = mesh["n_cells"], bands["n_bands"], dirs["n_dirs"]
    n = nb * nd * nc
    idx = lambda b, d, c: (b * nd + d) * nc + c
    M, q = np.zeros((n, n)), np.zeros(n)
    theta = HBAR * bands["omega"] / KB
    I0 = lambda b, t: bands["C"][b] / np.expm1(theta[b] / t)
    off = mesh["face_offsets"]
    for b in range(nb):
        for d in range(nd):
            s = dirs["s"][d]
            for c in range(nc):
                row = idx(b, d, c)
                k = dt * bands["vg"][b] / mesh["cell_volume"][c]
                M[row, row] += 1.0 - dt * inv_tau[b, c]
                q[row] += dt * inv_tau[b, c] * I0(b, T[c])
                for f in range(off[c], off[c + 1]):
                    nrm, a, nbr = mesh["face_normal"][f], mesh["face_area"][f], mesh["face_nbr"][f]
                    mu = float(s @ nrm)
                    if mu > 0:
                        M[row, row] -= k * a * mu
                    elif nbr >= 0:
                        M[row, idx(b, d, nbr)] -= k * a * mu
                    elif bcs["kind"][-1 - nbr] == gen.ISOTHERMAL:
                        q[row] -= k * a * mu * I0(b, bcs["t_wall"][-1 - nbr])
                    else:
                        rs = s - 2 * mu * nrm
                        e = int(np.argmin(np.abs(dirs["s"] - rs).sum(1)))
                        M[row, idx(b, e, c)] -= k * a * mu
    return M, q


def test_n1_brute_force_dense_operator_with_rate_bookkeeping(oracle_mod):
    """4 x 4 Fig.-1 mesh, 3 non-gray rows, 3 steps: the dense affine map with
    rates at Tr, then Tr <- T, E and a bisection T with R2 weights at the new Tr,
    kept here independently of the oracle."""
    mesh = gen.gen_mesh((4, 4), (1e-6, 1e-6))
    bands = gen.with_rate_law(gen.select_bands(gen.gen_bands_si(3), [0, 1, 3]))
    dirs = gen.gen_dirs_inplane(8)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    p = oracle_mod.Problem(mesh, bands, dirs, bcs)
    I, T, Tr = p.initial_state(300.0, ic_eps=0.2, with_tr=True)
    dt = 0.6 * gen.cartesian_dt_bound(mesh, bands, dirs, t_max=360.0)
    W = dirs["w"].sum()
    ra, rb, rt = bands["rate_a"], bands["rate_b"], bands["rate_theta"]
    for _ in range(3):
        inv_tau = _law(ra[:, None], rb[:, None], rt[:, None], Tr[None, :])
        M, q = _dense_step(mesh, bands, dirs, bcs, T, inv_tau, dt)
        I_ref = (M @ I.ravel() + q).reshape(I.shape)
        Tr_ref = T.copy()
        wts = _law(ra[:, None], rb[:, None], rt[:, None], Tr_ref[None, :]) / bands["vg"][:, None]
        E = np.einsum("bc,d,bdc->c", wts, dirs["w"], I_ref)
        T_ref = np.array([_bisect_T(bands, W, wts[:, c], E[c]) for c in range(mesh["n_cells"])])
        I, T, Tr = p.run(I, T, dt, 1, Tr=Tr)
        assert np.max(np.abs(I / I_ref - 1)) < 1e-13
        assert np.max(np.abs(T / T_ref - 1)) < 1e-12
        assert np.array_equal(Tr, Tr_ref)


# ----------------------------------------------------------------- rates_now (reading 26)
def test_n1_rates_now_t_independent_law_equals_lagged(oracle_mod):
    """A T-independent law (b = 0): the two rate bookkeepings are the same
    method, bit for bit (nothing in the rates can lag)."""
    mesh = gen.gen_mesh((6, 5), (1e-6, 1e-6))
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    bands = dict(gen.gen_bands_custom(omega=[1e13, 3e13, 6e13], vg=[8e3, 6e3, 3e3], tau=1.0, C=[1e5, 3e6, 2e7]),
                 rate_a=np.array([2.0 ** 40, 2.0 ** 38, 2.0 ** 41]), rate_b=np.zeros(3), rate_theta=np.full(3, 140.0))
    out = []
    for now in (False, True):
        p = oracle_mod.Problem(mesh, bands, dirs, bcs, rates_now=now)
        I, T, Tr = p.initial_state(300.0, ic_eps=0.2, with_tr=True)
        dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
        out.append(p.run(I, T, dt, 12, Tr=Tr))
    assert np.array_equal(out[0][0], out[1][0]) and np.array_equal(out[0][1], out[1][1])


def test_n1_rates_now_equilibrium_invariance(oracle_mod):
    mesh = gen.gen_mesh((4, 4, 3), (1e-6,) * 3)
    bands = gen.with_rate_law(gen.gen_bands_si(4))
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_fig1(mesh, t_hot=320.0, t_cold=320.0, radius=2e-6)
    p = oracle_mod.Problem(mesh, bands, dirs, bcs, rates_now=True)
    T0 = np.full(mesh["n_cells"], 320.0)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs, t_max=320.0)
    I, T, _ = p.run(p.equilibrium(T0), T0, dt, 20, Tr=T0)
    assert np.max(np.abs(I / p.equilibrium(T0) - 1)) < 2e-14 and np.max(np.abs(T / 320.0 - 1)) < 1e-14


def test_n1_rates_now_breaks_exact_energy_balance(oracle_mod):
    """Why the lag is the default: with the rates of the step's own
    temperature the R2 weights of the solve that produced T^n (rates at
    T^{n-1}) and the relaxation of step n differ, and the specular-wall energy
    invariant drifts (while the lagged bookkeeping keeps it to 1e-13)."""
    mesh = gen.gen_mesh((6, 5), (1e-6, 1e-6))
    bands = gen.with_rate_law(gen.gen_bands_si(4))
    dirs = gen.gen_dirs_product(4, 8)
    bcs = gen.gen_bcs_uniform(mesh, gen.SYMMETRY)
    drift = []
    for now in (False, True):
        p = oracle_mod.Problem(mesh, bands, dirs, bcs, rates_now=now)
        I0, T0, Tr0 = p.initial_state(300.0, ic_eps=0.4, with_tr=True)
        dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs, t_max=T0.max() * 1.2)
        e0 = _total_energy(p, I0, mesh["cell_volume"], bands["vg"])
        I, _, _ = p.run(I0, T0, dt, 30, Tr=Tr0)
        drift.append(abs(_total_energy(p, I, mesh["cell_volume"], bands["vg"]) / e0 - 1))
    assert drift[0] < 1e-13 and drift[1] > 1e-9


def test_n1_rates_now_brute_force_dense_operator(oracle_mod):
    """The dense affine map with the rates of the step's own T, then E and a
    bisection T with R2 weights at that T, kept independently of the oracle."""
    mesh = gen.gen_mesh((4, 4), (1e-6, 1e-6))
    bands = gen.with_rate_law(gen.select_bands(gen.gen_bands_si(3), [0, 1, 3]))
    dirs = gen.gen_dirs_inplane(8)
    bcs = gen.gen_bcs_fig1(mesh, radius=2e-6)
    p = oracle_mod.Problem(mesh, bands, dirs, bcs, rates_now=True)
    I, T, Tr = p.initial_state(300.0, ic_eps=0.2, with_tr=True)
    dt = 0.6 * gen.cartesian_dt_bound(mesh, bands, dirs, t_max=360.0)
    W = dirs["w"].sum()
    ra, rb, rt = bands["rate_a"], bands["rate_b"], bands["rate_theta"]
    for _ in range(3):
        inv_tau = _law(ra[:, None], rb[:, None], rt[:, None], T[None, :])
        M, q = _dense_step(mesh, bands, dirs, bcs, T, inv_tau, dt)
        I_ref = (M @ I.ravel() + q).reshape(I.shape)
        wts = inv_tau / bands["vg"][:, None]
        E = np.einsum("bc,d,bdc->c", wts, dirs["w"], I_ref)
        T_ref = np.array([_bisect_T(bands, W, wts[:, c], E[c]) for c in range(mesh["n_cells"])])
        I, T, Tr = p.run(I, T, dt, 1, Tr=Tr)
        assert np.max(np.abs(I / I_ref - 1)) < 1e-13
        assert np.max(np.abs(T / T_ref - 1)) < 1e-12
