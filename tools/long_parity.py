#!/usr/bin/env python
"""Parity at the paper's horizon: a workload run N steps on the GPU (bte_step)
and in the CPU oracle side by side, compared element by element every CHECK
steps (max relative error on I and T).  Test infrastructure (loads oracle/).

    python tools/long_parity.py C3 1000 100      (BASELINE.json configs[2]: 1000 steps)
    python tools/long_parity.py C4 100 25        (the bench's workload at the north star's 100 steps)
    python tools/long_parity.py C4+law 40 20     (with temperature-dependent relaxation times)
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen  # noqa: E402


def main():
    name, n, check = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
    law = name.endswith("+law")  # N1: tau(T), dt as in bench.py --rate-law
    cfg = gen.make_config(name[:-4] if law else name)
    if law:
        import dataclasses
        lb = gen.with_rate_law(cfg.bands)
        cfg = dataclasses.replace(cfg, bands=lb, dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, lb, cfg.dirs, t_max=350.0))
    p = oracle.problem_from_config(cfg)
    I, T, Tr = p.initial_state(cfg.t_init, ic_eps=cfg.ic_eps, with_tr=True, mult_fn=getattr(cfg, "ic_mult", None))
    print(f"{name}: {cfg.mesh['n_cells']} cells x {cfg.dirs['n_dirs']} dirs x {cfg.bands['n_bands']} rows, "
          f"dt {cfg.dt:.4g} s, {n} steps, compared every {check}", flush=True)
    worst_i = worst_t = 0.0
    with bte.solver_from_config(cfg) as s:
        bte.apply_ic(s, cfg)
        done = 0
        while done < n:
            k = min(check, n - done)
            t0 = time.time()
            I, T, Tr = p.run(I, T, cfg.dt, k, Tr=Tr)
            t1 = time.time()
            s.step(cfg.dt, k)
            Ig, Tg = s.intensity(), s.temperature()
            done += k
            ei = max(float(np.max(np.abs(Ig[b] / I[b] - 1.0))) for b in range(I.shape[0]))  # (row by row: C4's
            et = float(np.max(np.abs(Tg / T - 1.0)))                                         #  state is 23 GB)
            del Ig
            worst_i, worst_t = max(worst_i, ei), max(worst_t, et)
            print(f"step {done:5d}: max rel err I {ei:.3e}  T {et:.3e}   T in [{T.min():.4f}, {T.max():.4f}] K"
                  f"   (oracle {t1 - t0:.1f} s)", flush=True)
    ok = worst_i <= 1e-10 and worst_t <= 1e-9
    print(f"worst over the run: I {worst_i:.3e}, T {worst_t:.3e} -> {'within' if ok else 'OUTSIDE'} "
          f"the north star's 1e-10 / 1e-9", flush=True)
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
