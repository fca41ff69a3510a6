"""GPU parity on the Fig.-10 workload and unstructured meshes.

C6: the paper's second example (L1169-1178) on a Cartesian grid (paired-face
TMA kernel); C6t: the same domain as a triangle mesh (generic-face kernel with
the locality order from the centroids).  Element by element against the
oracle: relative 1e-10 on I, 1e-9 on T.
"""
import dataclasses

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import assert_parity, gpu_run, oracle_run

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bte_lib():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


@pytest.mark.parametrize("name,variant", [("C6", 6), ("C6t", 7)])
def test_fig10_workload(bte_lib, oracle_mod, name, variant):
    cfg = gen.make_config(name)
    Io, To = oracle_run(oracle_mod, cfg, 100)
    Ig, Tg, st = gpu_run(cfg, 100)
    assert st["flux_variant"] == variant
    assert_parity(Ig, Tg, Io, To)
    assert To.max() > 100.5


def test_triangles_relabelled(bte_lib, oracle_mod):
    cfg = gen.make_config("C6t")
    mesh, _ = gen.permute_mesh(cfg.mesh, seed=21)
    cfg = dataclasses.replace(cfg, mesh=mesh)
    Io, To = oracle_run(oracle_mod, cfg, 30)
    Ig, Tg, _ = gpu_run(cfg, 30)
    assert_parity(Ig, Tg, Io, To)


def test_triangles_with_rate_law(bte_lib, oracle_mod):
    cfg = gen.make_config("C6t")
    bands = gen.with_rate_law(cfg.bands)
    cfg = dataclasses.replace(cfg, bands=bands, dt=0.5 * gen.general_dt_bound(cfg.mesh, bands, cfg.dirs, t_max=150.0))
    Io, To = oracle_run(oracle_mod, cfg, 40)
    Ig, Tg, st = gpu_run(cfg, 40)
    assert st["flux_variant"] == 7
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("bg", [1, 2, 4])
def test_triangles_band_groups(bte_lib, oracle_mod, bg):
    cfg = gen.make_config("C6t")
    Io, To = oracle_run(oracle_mod, cfg, 20)
    Ig, Tg, _ = gpu_run(cfg, 20, band_group=bg)
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("bg", [1, 2, 4])
@pytest.mark.parametrize("tma", [True, False])
def test_triangles_kernels_and_groups(bte_lib, oracle_mod, bg, tma):
    """Both generic-face kernels (TMA-staged 7, register 0) in every band group."""
    cfg = gen.make_config("C6t")
    Io, To = oracle_run(oracle_mod, cfg, 20)
    Ig, Tg, st = gpu_run(cfg, 20, band_group=bg, tma=tma)
    assert st["flux_variant"] == (7 if tma else 0)
    assert_parity(Ig, Tg, Io, To)


def test_split_faces_3d_generic(bte_lib, oracle_mod):
    """A 3-D mesh with split (hanging) faces: more than 6 faces per cell (MF 8)."""
    cfg = gen.small_3d_config((7, 6, 5), n_spectral=3)
    cfg = dataclasses.replace(cfg, mesh=gen.split_faces(cfg.mesh))
    Io, To = oracle_run(oracle_mod, cfg, 10)
    for tma, v in ((True, 7), (False, 0)):
        Ig, Tg, st = gpu_run(cfg, 10, tma=tma)
        assert st["flux_variant"] == v
        assert_parity(Ig, Tg, Io, To)


def test_c3t_full_size_bench_launch(bte_lib, oracle_mod):
    """C3t exactly as the bench runs it (28,800 triangles, 55 rows x 400
    directions: the TMA-staged generic kernel with its bank-conflict-aware
    staging positions and face-slot order, 13 groups of 4 rows + a ragged
    group of 3 in one launch), seeded IC, 3 steps, every element."""
    cfg = gen.make_config("C3t")
    Io, To = oracle_run(oracle_mod, cfg, 3)
    Ig, Tg, st = gpu_run(cfg, 3)
    assert st["flux_variant"] == 7 and st["band_group"] == 4
    assert st["flux_launches"] == 3  # (one launch per step)
    assert_parity(Ig, Tg, Io, To)
