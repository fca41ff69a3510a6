#!/usr/bin/env python
"""Per-rank flux time of cell partitioning (z slabs of a box grid), emulated on
one GPU.

    python tools/cells_flux.py [C4] [1 2 4 8]

For each P, ranks of P z-slab parts (the first, a middle and the last part)
are created with world = P and no communicator; one halo import (the exchange
itself is NCCL's job) then bte_step_begin runs the rank's flux launches, timed
with the library's CUDA events.  Prints the kernel in use, the halo bytes per
step and the compute strong-scaling estimate t(1) / (P max_rank t(P)).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_heislersdms24_b200 import bte, dist, inputs as gen  # noqa: E402


def flux_ms(cfg, parts, P, rank, reps=5):
    kw = dict(rank=rank, world=P, cell_part=parts, n_cell_parts=P) if P > 1 else {}
    with bte.solver_from_config(cfg, profile=True, stream=torch.cuda.current_stream(), **kw) as s:
        for q in range(P):
            n_send, n_recv = s.halo_size(q) if P > 1 else (0, 0)
            if n_recv:
                s.halo_import(q, np.full(n_recv, 1e6))
        s.step_begin(cfg.dt)
        s.set_energy(s.energy())
        s.step_finish()
        s.reset_stats()
        for _ in range(reps):
            s.step_begin(cfg.dt)
            s.set_energy(s.energy())
            s.step_finish()
        st = s.stats()
        return st["ms_flux_interior"] / reps, bte.FLUX_VARIANTS[st["flux_variant"]], st["halo_bytes"], s.n_cells


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C4"
    Ps = [int(x) for x in sys.argv[2:]] or [1, 2, 4, 8]
    cfg = gen.make_config(name)
    t1 = None
    for P in Ps:
        parts = dist.slab_partition(cfg.mesh["cell_centre"], P)
        res = [flux_ms(cfg, parts, P, r) for r in sorted({0, P // 2, P - 1})]
        tmax = max(r[0] for r in res)
        t1 = tmax if P == 1 else t1
        print(f"{name} P={P}: " + "  ".join(f"[{r[1]} cells {r[3]} flux {r[0]:.3f} ms halo {r[2] / 1e6:.0f} MB]"
                                            for r in res)
              + f"  -> compute strong-scaling eff {t1 / (P * tmax):.3f}", flush=True)


if __name__ == "__main__":
    main()
