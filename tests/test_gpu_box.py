"""GPU parity of the box kernel (structured 3-D grids, flux_variant 6).

The box kernel marches 32 x 8 cell tiles through the layers of grid axis 2
with tensor copies, takes the specular ghosts of the axis-0/1 walls from the
mirrored direction staged in the same orbit (Eq. 6) and the axis-2
ghost layer from the isothermal side table or the z-mirrored direction.  Each
case is compared element by element with the oracle (relative 1e-10 on I,
1e-9 on T), on shapes with ragged tiles and ragged layer ranges.
"""
import dataclasses

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import assert_parity, gpu_run, oracle_run

pytestmark = pytest.mark.gpu

BOX = 6


def _cfg3(shape, walls=None, spacing=(1e-6, 1e-6, 1e-6), n_spectral=3, ntheta=4, nphi=8, eps=0.1, steps=12):
    mesh = gen.gen_mesh(shape, spacing)
    bands = gen.gen_bands_si(n_spectral)
    dirs = gen.gen_dirs_product(ntheta, nphi)
    bcs = gen.gen_bcs_fig1(mesh, radius=2 * spacing[0]) if walls is None else gen.gen_bcs_walls(mesh, walls)
    bound = gen.cartesian_dt_bound(mesh, bands, dirs)
    return gen.Config(name=f"box{shape}", mesh=mesh, bands=bands, dirs=dirs, bcs=bcs, t_init=300.0,
                      dt=0.5 * bound, nsteps=steps, ic_eps=eps, extra={"dt_bound": bound})


@pytest.fixture(scope="module")
def bte_lib():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


def _check(oracle_mod, cfg, steps=None, variant=BOX, **kw):
    steps = cfg.nsteps if steps is None else steps
    Io, To = oracle_run(oracle_mod, cfg, steps)
    Ig, Tg, st = gpu_run(cfg, steps, **kw)
    assert st["flux_variant"] == variant
    assert_parity(Ig, Tg, Io, To)
    return Ig, Tg, st


@pytest.mark.parametrize("shape", [(6, 5, 4), (34, 9, 7), (64, 17, 19), (2, 3, 1), (40, 8, 9)])
def test_box_fig1_ragged(bte_lib, oracle_mod, shape):
    """Fig.-1 walls (axis-2 isothermal Gaussian top / 300 K bottom, specular
    sides): ragged 32 x 8 tiles, layer ranges shorter than L, one layer."""
    _check(oracle_mod, _cfg3(shape))


def test_box_all_specular(bte_lib, oracle_mod):
    """Specular on all six sides: the axis-2 ghost layer is the z-mirrored
    direction's wall layer (tensor copy at another direction coordinate)."""
    walls = {w: (gen.SYMMETRY, 0) for w in range(6)}
    _check(oracle_mod, _cfg3((34, 10, 9), walls=walls, eps=0.3))


def test_box_isothermal_on_x_axis(bte_lib, oracle_mod):
    """Isothermal walls on mesh x: x becomes the marching axis (axis
    permutation), y contiguous; anisotropic cells give a different A/V per axis."""
    walls = {gen.WALL_XM: (gen.ISOTHERMAL, 320.0), gen.WALL_XP: (gen.ISOTHERMAL, 290.0),
             gen.WALL_YM: (gen.SYMMETRY, 0), gen.WALL_YP: (gen.SYMMETRY, 0),
             gen.WALL_ZM: (gen.SYMMETRY, 0), gen.WALL_ZP: (gen.SYMMETRY, 0)}
    _check(oracle_mod, _cfg3((11, 12, 7), walls=walls, spacing=(1e-6, 2e-6, 1.5e-6)))


def test_box_mixed_axis2_sides(bte_lib, oracle_mod):
    """One axis-2 side isothermal, the other specular."""
    walls = {gen.WALL_XM: (gen.SYMMETRY, 0), gen.WALL_XP: (gen.SYMMETRY, 0),
             gen.WALL_YM: (gen.SYMMETRY, 0), gen.WALL_YP: (gen.SYMMETRY, 0),
             gen.WALL_ZM: (gen.ISOTHERMAL, 330.0), gen.WALL_ZP: (gen.SYMMETRY, 0)}
    _check(oracle_mod, _cfg3((8, 9, 10), walls=walls))


@pytest.mark.parametrize("nbb,dchunk", [(1, 4), (2, 8), (7, 0), (0, 12)])
def test_box_work_split(bte_lib, oracle_mod, nbb, dchunk):
    """Band-rows per CTA (band_group) and orbits per CTA (dir_chunk) only
    change the work split and the energy slots."""
    cfg = _cfg3((34, 9, 5), n_spectral=4, ntheta=4, nphi=8)
    _check(oracle_mod, cfg, band_group=nbb, dir_chunk=dchunk)


@pytest.mark.parametrize("spare", [1, 2, 5])
def test_box_slab_rotation(bte_lib, oracle_mod, spare):
    cfg = _cfg3((16, 9, 6), n_spectral=4)
    Ig, Tg, st = _check(oracle_mod, cfg, max_spare_slabs=spare)
    assert st["spare_slabs"] == spare


def test_box_bench_tables(bte_lib, oracle_mod):
    """The bench's 55 band-rows and 400 directions (100 orbits) on a small grid."""
    h = 8.2e-6
    mesh = gen.gen_mesh((34, 9, 6), (h, h, h))
    bands, dirs = gen.gen_bands_si(40), gen.gen_dirs_product(20, 20)
    bcs = gen.gen_bcs_fig1(mesh, radius=2 * h)
    dt = 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs)
    _check(oracle_mod, gen.Config("box55", mesh, bands, dirs, bcs, 300.0, dt, 6, ic_eps=0.1))


def test_box_and_tma_agree(bte_lib, oracle_mod):
    """box=False falls back to the TMA kernel; both match the oracle."""
    cfg = _cfg3((34, 9, 7))
    _check(oracle_mod, cfg)
    _check(oracle_mod, cfg, variant=4, box=False)


def test_box_odd_extents_fall_back(bte_lib):
    """All extents odd: no 16-byte-aligned contiguous axis -> not the box kernel."""
    _, _, st = gpu_run(_cfg3((7, 5, 3)), 1)
    assert st["flux_variant"] != BOX
