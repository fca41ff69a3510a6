"""GPU parity of the alternative temperature outputs.

temp_rule 2 (R3): one linearised first-law step per step (L413-415).
bte_get_temperature_rule: the temperature of the current state under R2, R1
(energy-equivalent) or R3, without changing the state.  Against the oracle:
relative 1e-10 on I, 1e-9 on T.
"""
import dataclasses

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import inputs as gen
from tests._parity import RTOL_T, assert_parity, gpu_run, oracle_run, rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bte_lib():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


@pytest.mark.parametrize("cfg_fn", [
    lambda: dataclasses.replace(gen.make_config("C2"), nsteps=40),
    lambda: gen.small_3d_config((34, 9, 6), n_spectral=3),
])
def test_r3_stepping(bte_lib, oracle_mod, cfg_fn):
    cfg = dataclasses.replace(cfg_fn(), temp_rule=2)
    Io, To = oracle_run(oracle_mod, cfg, cfg.nsteps)
    Ig, Tg, _ = gpu_run(cfg, cfg.nsteps)
    assert_parity(Ig, Tg, Io, To)


@pytest.mark.parametrize("law", [False, True])
def test_temperature_of_state_under_each_rule(bte_lib, oracle_mod, law):
    cfg = gen.small_3d_config((34, 9, 6), n_spectral=3)
    if law:
        bands = gen.with_rate_law(cfg.bands)
        cfg = dataclasses.replace(cfg, bands=bands,
                                  dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, bands, cfg.dirs, t_max=350.0))
    p = oracle_mod.problem_from_config(cfg)
    I, T, Tr = p.initial_state(cfg.t_init, ic_eps=cfg.ic_eps, with_tr=True)
    I, T, Tr = p.run(I, T, cfg.dt, 6, Tr=Tr)
    expect = {}
    for rule in (0, 1, 2):
        q = oracle_mod.Problem(cfg.mesh, cfg.bands, cfg.dirs, cfg.bcs, temp_rule=rule)
        expect[rule], _ = q.newton(q.energy(I, Tr=Tr), T, Tr=Tr)
    assert rel_err(expect[0], T) < 1e-12  # R2 of an R2 state is its own T
    with bte_lib.solver_from_config(cfg) as s:
        bte_lib.apply_ic(s, cfg)
        s.step(cfg.dt, 6)
        for rule in (0, 1, 2):
            assert rel_err(s.temperature_rule(rule), expect[rule]) <= RTOL_T, rule
        # the state is untouched: keep stepping and stay on the oracle's path
        s.step(cfg.dt, 3)
        Io, To, _ = p.run(I, T, cfg.dt, 3, Tr=Tr)
        assert_parity(s.intensity(), s.temperature(), Io, To)
