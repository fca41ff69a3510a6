#!/usr/bin/env python
"""Per-rank flux time of the band-sharded path, emulated on one GPU.

    python tools/shard_flux.py [C4] [1 2 4 8]

For each N, rank 0 and rank N-1 of N (the smallest / largest row counts) are
created with world = N and no communicator; bte_step_begin runs the rank's
flux launches (+ the slot reduction), timed with the library's CUDA events.
Strong-scaling estimate of the compute part: t(N=1) / (N * max_rank t(N)).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen  # noqa: E402


def flux_ms(cfg, rank, world, reps=5):
    with bte.solver_from_config(cfg, rank=rank, world=world, profile=True,
                                stream=torch.cuda.current_stream()) as s:
        s.step_begin(cfg.dt)
        s.set_energy(s.energy())
        s.step_finish()
        s.reset_stats()
        for _ in range(reps):
            s.step_begin(cfg.dt)
            s.set_energy(s.energy())
            s.step_finish()
        st = s.stats()
        return st["ms_flux_interior"] / reps, s.b_hi - s.b_lo, st["band_group"], st["dir_chunks"]


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C4"
    Ns = [int(x) for x in sys.argv[2:]] or [1, 2, 4, 8]
    cfg = gen.make_config(name)
    t1 = None
    for N in Ns:
        res = [flux_ms(cfg, r, N) for r in sorted({0, N - 1})]
        tmax = max(r[0] for r in res)
        t1 = tmax if N == 1 else t1
        eff = t1 / (N * tmax) if t1 else float("nan")
        print(f"{name} N={N}: " + "  ".join(f"rows {r[1]} nbb {r[2]} chunks {r[3]} flux {r[0]:.3f} ms" for r in res)
              + f"  -> compute strong-scaling eff {eff:.3f}", flush=True)


if __name__ == "__main__":
    main()
