#!/usr/bin/env python
"""Box-kernel work-split sweep (one process, the config built once).

    python tools/sweep_box.py C4 "5:80 5:60:6:8 1:80 ..."   (band_group:dir_chunk[:stages:L], 0 = auto)
    python tools/sweep_box.py C3:128x120 "..."               (C3's tables on another grid)
    python tools/sweep_box.py C4+law "..."                   (the rate law, dt as in bench.py --rate-law)

Equilibrium IC (the flux kernel's time does not depend on the values); prints
the flux-kernel time per step from the library's CUDA events and the fraction
of MEASURED_PEAKS hbm_gbs at 16 B per update.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen  # noqa: E402


def main():
    name = sys.argv[1]
    law = name.endswith("+law")
    name = name[:-4] if law else name
    combos = [tuple(int(x) for x in c.split(":")) for c in sys.argv[2].split()]
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 10
    if ":" in name:  # e.g. "C3:128x120": the config's bands / directions / walls on another grid
        base, shape = name.split(":")
        cfg = gen.make_config(base)
        shape = tuple(int(v) for v in shape.split("x"))
        h = cfg.mesh["spacing"][0]
        mesh = gen.gen_mesh(shape, (h,) * len(shape))
        import dataclasses
        cfg = dataclasses.replace(cfg, mesh=mesh, bcs=gen.gen_bcs_fig1(mesh, radius=4 * h))
    else:
        cfg = gen.make_config(name)
    if law:  # N1: temperature-dependent tau, dt = 0.5 x the bound at the hot wall (bench.py --rate-law)
        import dataclasses
        lb = gen.with_rate_law(cfg.bands)
        cfg = dataclasses.replace(cfg, bands=lb, dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, lb, cfg.dirs, t_max=350.0))
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    nc, nd, nb = cfg.mesh["n_cells"], cfg.dirs["n_dirs"], cfg.bands["n_bands"]
    for combo in combos:
        nbb, dc = combo[:2]
        for key, v in zip(("BTE_BOX_STAGES", "BTE_BOX_L"), combo[2:]):
            os.environ[key] = str(v)
        with bte.solver_from_config(cfg, profile=True, band_group=nbb, dir_chunk=dc,
                                    stream=torch.cuda.current_stream()) as s:
            s.step(cfg.dt, 3)
            torch.cuda.synchronize()
            s.reset_stats()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            s.step(cfg.dt, steps)
            e1.record()
            torch.cuda.synchronize()
            st = s.stats()
            ms = e0.elapsed_time(e1) / steps
            fl = st["ms_flux_interior"] / steps
            gbs = 16.0 * nc * nd * nb / (fl / 1e3) / 1e9
            print(f"{name} {combo} -> nbb {st['band_group']} chunks {st['dir_chunks']}: "
                  f"step {ms:.3f} ms ({nc * nd * nb / ms / 1e9:.4g}e12 upd/s)  flux {fl:.3f} ms "
                  f"{gbs:.0f} GB/s frac {gbs / peak:.3f}", flush=True)


if __name__ == "__main__":
    main()
