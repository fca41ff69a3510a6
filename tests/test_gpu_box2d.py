"""GPU parity of the box kernel on 2-D structured grids (flux_variant 6).

The paper's own meshes are 2-D quad grids (Fig. 1: 120 x 120 with
an isothermal hot top wall, an isothermal bottom and specular sides; Fig. 10).
On them the box kernel runs one layer: 32 x 8 cell tiles, one stage per
(band-row, orbit of 4 mirrored directions), the specular ghosts of the
contiguous axis from the partner slot, and the isothermal wall ghosts of grid
axis 1 (Eq. 6, I0_b(T_wall)) as staged rows of the side table.  Element by
element against the oracle (relative 1e-10 on I, 1e-9 on T), on shapes with
ragged tiles in both axes and every wall combination the kernel accepts.
"""
import dataclasses

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import assert_parity, gpu_run, oracle_run

pytestmark = pytest.mark.gpu

BOX = 6
I, S = gen.ISOTHERMAL, gen.SYMMETRY


@pytest.fixture(scope="module")
def bte_lib():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


def _cfg2(shape, walls=None, n_spectral=3, dirs=None, eps=0.1, steps=15, law=False):
    h = 1e-6
    mesh = gen.gen_mesh(shape, (h, h))
    bands = gen.gen_bands_si(n_spectral)
    if law:
        bands = gen.with_rate_law(bands)
    dirs = gen.gen_dirs_product(4, 8) if dirs is None else dirs
    bcs = gen.gen_bcs_fig1(mesh, radius=2 * h) if walls is None else gen.gen_bcs_walls(mesh, walls)
    bound = gen.cartesian_dt_bound(mesh, bands, dirs, t_max=350.0 if law else None)
    return gen.Config(name=f"box2d{shape}", mesh=mesh, bands=bands, dirs=dirs, bcs=bcs, t_init=300.0,
                      dt=0.5 * bound, nsteps=steps, ic_eps=eps, extra={"dt_bound": bound})


def _check(oracle_mod, cfg, variant=BOX, steps=None, **kw):
    steps = cfg.nsteps if steps is None else steps
    Io, To = oracle_run(oracle_mod, cfg, steps)
    Ig, Tg, st = gpu_run(cfg, steps, **kw)
    assert st["flux_variant"] == variant
    assert_parity(Ig, Tg, Io, To)
    return st


@pytest.mark.parametrize("shape", [(16, 16), (40, 24), (34, 9), (66, 13), (32, 8), (2, 30), (96, 1)])
def test_fig1_walls_ragged_tiles(bte_lib, oracle_mod, shape):
    _check(oracle_mod, _cfg2(shape))


def test_c1_and_c2(bte_lib, oracle_mod):
    _check(oracle_mod, gen.make_config("C1"))
    c2 = gen.make_config("C2")
    _check(oracle_mod, c2, steps=60)


def test_box_and_tma_agree_2d(bte_lib, oracle_mod):
    cfg = gen.make_config("C2")
    a = _check(oracle_mod, cfg, steps=20)
    b = _check(oracle_mod, cfg, steps=20, variant=4, box=False)
    assert a["steps"] == b["steps"] == 20


@pytest.mark.parametrize("walls", [
    {gen.WALL_XM: (S, 0), gen.WALL_XP: (S, 0), gen.WALL_YM: (S, 0), gen.WALL_YP: (S, 0)},      # closed box
    {gen.WALL_XM: (S, 0), gen.WALL_XP: (S, 0), gen.WALL_YM: (I, 330.0), gen.WALL_YP: (S, 0)},  # one hot wall
    {gen.WALL_XM: (S, 0), gen.WALL_XP: (S, 0), gen.WALL_YM: (S, 0), gen.WALL_YP: (I, 280.0)},
    {gen.WALL_XM: (I, 320.0), gen.WALL_XP: (I, 290.0), gen.WALL_YM: (S, 0), gen.WALL_YP: (S, 0)},  # iso on x
])
def test_wall_combinations(bte_lib, oracle_mod, walls):
    _check(oracle_mod, _cfg2((36, 22), walls=walls))


def test_direction_on_a_mirror_plane_falls_back(bte_lib, oracle_mod):
    """A direction with s_x = 0 (n_phi = 6 puts one at phi = 90 deg) has no
    4-member orbit: the TMA kernel runs instead."""
    _check(oracle_mod, _cfg2((40, 24), dirs=gen.gen_dirs_product(4, 6)), variant=4)


def test_mixed_wall_kinds_fall_back(bte_lib, oracle_mod):
    """Isothermal sides on both axes: not a box grid (TMA kernel)."""
    walls = {gen.WALL_XM: (I, 320.0), gen.WALL_XP: (S, 0), gen.WALL_YM: (I, 290.0), gen.WALL_YP: (S, 0)}
    _check(oracle_mod, _cfg2((36, 22), walls=walls), variant=4)


def test_inplane_directions_and_paper_set(bte_lib, oracle_mod):
    _check(oracle_mod, _cfg2((40, 24), dirs=gen.gen_dirs_inplane(20)))
    _check(oracle_mod, _cfg2((40, 24), dirs=gen.gen_dirs_product(20, 20), n_spectral=1, steps=6))


@pytest.mark.parametrize("spare,nbb,dc", [(2, 0, 0), (3, 2, 8), (0, 1, 4), (0, 4, 16)])
def test_rotation_and_work_split(bte_lib, oracle_mod, spare, nbb, dc):
    cfg = _cfg2((40, 24), n_spectral=5)
    _check(oracle_mod, cfg, max_spare_slabs=spare, band_group=nbb, dir_chunk=dc)


@pytest.mark.parametrize("rule", [0, 1])
def test_rate_law(bte_lib, oracle_mod, rule):
    cfg = dataclasses.replace(_cfg2((40, 24), law=True), temp_rule=rule)
    _check(oracle_mod, cfg)


def test_fig10_elongated(bte_lib, oracle_mod):
    _check(oracle_mod, gen.make_config("C6"), steps=60)


def test_c3_mesh_full_rows(bte_lib, oracle_mod):
    """The paper's 120 x 120 mesh, all 55 rows, 32 directions, 4 steps."""
    cfg = gen.make_config("C3")
    dirs = gen.gen_dirs_product(4, 8)
    cfg = dataclasses.replace(cfg, dirs=dirs, dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, cfg.bands, dirs))
    _check(oracle_mod, cfg, steps=4)


def test_equilibrium_invariance(bte_lib):
    """P1 on the 2-D box path: equilibrium IC with every wall at T0 stays put."""
    walls = {w: (I, 300.0) if w in (gen.WALL_YM, gen.WALL_YP) else (S, 0)
             for w in (gen.WALL_XM, gen.WALL_XP, gen.WALL_YM, gen.WALL_YP)}
    cfg = _cfg2((40, 24), walls=walls, eps=0.0)
    with bte_lib.solver_from_config(cfg) as s:
        I0 = s.intensity()
        s.step(cfg.dt, 10)
        assert s.stats()["flux_variant"] == BOX
        assert np.max(np.abs(s.intensity() / I0 - 1)) <= 2e-14
        assert np.max(np.abs(s.temperature() / 300.0 - 1)) <= 2e-14
