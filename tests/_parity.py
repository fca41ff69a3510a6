"""Shared helpers of the parity tests: run one config on both sides.

The oracle side only ever sees generator arrays; the CUDA side only ever sees
generator arrays.  Neither feeds the other.
"""
import numpy as np

RTOL_I = 1e-10  # north star: relative 1e-10 on I after 100 FP64 steps
RTOL_T = 1e-9   # north star: relative 1e-9 on T


def oracle_run(oracle_mod, cfg, nsteps, ic_eps=None, **pkw):
    p = oracle_mod.problem_from_config(cfg, **pkw)
    I, T, Tr = p.initial_state(cfg.t_init, ic_eps=cfg.ic_eps if ic_eps is None else ic_eps, with_tr=True,
                               mult_fn=getattr(cfg, "ic_mult", None))
    if nsteps:
        I, T, Tr = p.run(I, T, cfg.dt, nsteps, Tr=Tr)
    return I, T


def gpu_run(cfg, nsteps, ic_eps=None, **kw):
    from paper_conf_ipps_heislersdms24_b200 import bte
    import dataclasses
    c2 = dataclasses.replace(cfg, ic_eps=cfg.ic_eps if ic_eps is None else ic_eps)
    with bte.solver_from_config(c2, **kw) as s:
        bte.apply_ic(s, c2)
        if nsteps:
            s.step(c2.dt, nsteps)
        return s.intensity(), s.temperature(), s.stats()


def rel_err(a, b):
    return float(np.max(np.abs(a / b - 1.0)))


def assert_parity(Ig, Tg, Io, To, rtol_i=RTOL_I, rtol_t=RTOL_T):
    assert Ig.shape == Io.shape and Tg.shape == To.shape
    assert np.all(np.isfinite(Ig)) and np.all(np.isfinite(Tg))
    ei, et = rel_err(Ig, Io), rel_err(Tg, To)
    assert ei <= rtol_i, f"I relative error {ei:.3e} > {rtol_i}"
    assert et <= rtol_t, f"T relative error {et:.3e} > {rtol_t}"
    return ei, et
