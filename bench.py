#!/usr/bin/env python
"""Benchmark: cell.dir.band updates/s of the explicit phonon-BTE step on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--impl ours|reference]

N > 1 is launched by torch.distributed.run (one rank per GPU); band-rows are
sharded across ranks with one NCCL all-reduce of the per-cell energy per step
(strong scaling: the problem is fixed, each rank owns ~nb/N rows).

A step is one pass of the whole hot path (upwind flux + relaxation + boundary
faces + energy reduction + all-reduce + Newton temperature solve) over the
workload.  Default workload: BASELINE.json configs[3], 3-D 64 x 64 x 32 hex
mesh, 40 spectral bands (55 band-rows), 400 directions, Fig.-1 walls, seeded
+-10 % IC; FP64.  Each state copy is 23 GB, far larger than the 126 MB L2, so
no L2 flush is needed between steps.

Prints ONE JSON line on rank 0 (see DESIGN.md 6 for every key).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "cell*dir*band updates/s"
WORKLOADS = {
    "C3": "2-D 120x120 quad mesh (525 um), 55 band-rows (40 spectral), 400 dirs, Fig.1 walls",
    "C3t": "2-D 120x120 quads split into 28800 triangles (525 um), 55 band-rows, 400 dirs, Fig.1 walls",
    "C4": "3-D 64x64x32 hex mesh (8.2 um cells), 55 band-rows (40 spectral), 400 dirs, Fig.1 walls",
    "C5": "3-D 96x96x96 hex mesh (8.2 um cells), 55 band-rows (40 spectral), 400 dirs, Fig.1 walls",
}
E2E_MAX_GB = 64  # largest per-rank state the end-to-end leg pins on the host
BYTES_PER_UPDATE = 16  # algorithmic: read I^n once, write I^{n+1} once


def _peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            pk = json.load(f)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def _traffic_from_profiles(config, alg_bytes_per_step):
    """DRAM bytes (read + write) of the dominant flux kernel per step, like
    `achieved`: the committed `ncu --set full` capture of one launch of this
    workload (profiles/ncu_flux_summary.json, one entry per config) gives its
    DRAM bytes over the algorithmic bytes of the rows it covered; times the
    step's algorithmic bytes.  None if no capture exists for the workload."""
    path = os.path.join(ROOT, "profiles", "ncu_flux_summary.json")
    try:
        with open(path) as f:
            d = json.load(f)
        e = d.get(config)
        if e and e.get("traffic_over_alg"):
            return float(e["traffic_over_alg"]) * alg_bytes_per_step, e.get("source")
    except Exception:
        pass
    return None, None


class ClockSampler:
    """nvidia-smi sampling of SM clocks and throttle reasons during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None
        self.path = None

    def __enter__(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        # Wait until the sampler is live (its first row written), so that a
        # short timed region is still bracketed by samples.
        t0 = time.time()
        self.n0 = 0
        while self.proc is not None and time.time() - t0 < 10.0:
            self.n0 = len(self._rows())
            if self.n0:
                break
            time.sleep(0.05)
        return self

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def _rows(self):
        rows = []
        try:
            for line in open(self.path):
                f = [x.strip() for x in line.split(",")]
                if len(f) >= 9:
                    rows.append(f)
        except Exception:
            pass
        return rows

    def summary(self):
        rows = self._rows()
        during = rows[self.n0:] if self.proc is not None else []
        if during:
            rows = during
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        smax = max(float(r[2]) for r in rows if r[2].replace(".", "").isdigit())
        loaded = [x for x in sm if x > 0.5 * smax] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower().startswith("active")})
        out = {"sm_mhz": statistics.median(loaded), "sm_max_mhz": smax, "reasons": reasons,
               "samples": len(rows)}
        if not during:
            out["note"] = "timed region shorter than the sampling interval: samples bracketing it"
        return out


def _dist():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    import platform
    return platform.processor() or "unknown"


def _oracle_sample(cfg, rows):
    """The oracle's problem on a bounded sample of the workload -- the full
    mesh and direction set, the first `rows` band-rows -- in the state the GPU
    arm starts from: the seeded IC (equilibrium at t_init x the generator's
    multiplier), T from the sample's energy (oracle Newton).  Untimed."""
    import numpy as np
    import oracle
    from paper_conf_ipps_heislersdms24_b200 import inputs as gen
    bands = gen.select_bands(cfg.bands, np.arange(rows))
    p = oracle.Problem(cfg.mesh, bands, cfg.dirs, cfg.bcs, temp_rule=cfg.temp_rule)
    I, T, Tr = p.initial_state(cfg.t_init, ic_eps=cfg.ic_eps, with_tr=True)
    p.reflection_map()
    return p, I, T, Tr


def _time_oracle_steps(p, I, T, Tr, dt, steps):
    """Per-step wall times of the oracle's explicit step (oracle_run, one step each)."""
    out = []
    for _ in range(steps):
        t0 = time.perf_counter()
        I, T, Tr = p.run(I, T, dt, 1, Tr=Tr)
        out.append(time.perf_counter() - t0)
    return out, (I, T, Tr)


def cpu_baseline(cfg, budget_s=12.0):
    """The oracle as it stands, on this host's cores (OpenMP over cells, all
    cores), on a bounded sample of the workload (about budget_s of CPU work):
    the full mesh and direction set, the first k band-rows, from the seeded IC
    the GPU arm runs, 3 timed steps (Newton takes its steady-state iteration
    count after the first).  Plus the same oracle on ONE core (a subprocess with
    OMP_NUM_THREADS=1, one row, one step)."""
    cores = os.cpu_count() or 1
    os.environ.setdefault("OMP_NUM_THREADS", str(cores))
    nc, nd, nb = cfg.mesh["n_cells"], cfg.dirs["n_dirs"], cfg.bands["n_bands"]
    p, I, T, Tr = _oracle_sample(cfg, 1)
    t1 = _time_oracle_steps(p, I, T, Tr, cfg.dt, 1)[0][0]
    k = int(max(1, min(nb, budget_s / 3.0 / max(t1, 1e-3))))
    p, I, T, Tr = _oracle_sample(cfg, k)
    ts, _ = _time_oracle_steps(p, I, T, Tr, cfg.dt, 3)
    t = sum(ts)
    upd = nc * nd * k * len(ts)
    out = {"value": upd / t, "unit": "updates/s", "cores": int(os.environ["OMP_NUM_THREADS"]), "kind": "oracle",
           "cpu_model": _cpu_model(), "host_cores": cores,
           "sample": f"{cfg.name}: full mesh ({nc} cells) x {nd} dirs x first {k} of {nb} band-rows, seeded IC, "
                     f"3 steps, {t:.2f} s, OMP_NUM_THREADS={os.environ['OMP_NUM_THREADS']}"}
    try:  # one core
        env = dict(os.environ, OMP_NUM_THREADS="1")
        r = subprocess.run([sys.executable, os.path.abspath(__file__), "--_oracle-1core", "--config", cfg.name],
                           env=env, capture_output=True, text=True, timeout=600)
        one = json.loads(r.stdout.strip().splitlines()[-1])
        out["one_core"] = one
    except Exception as e:  # noqa: BLE001 - reported, never fatal
        out["one_core"] = {"error": str(e)[:200]}
    return out


def _oracle_one_core(args):
    cfg = _bench_config(args)
    nc, nd = cfg.mesh["n_cells"], cfg.dirs["n_dirs"]
    p, I, T, Tr = _oracle_sample(cfg, 1)
    ts, _ = _time_oracle_steps(p, I, T, Tr, cfg.dt, 2)
    t = ts[-1]  # (the second step: Newton at its steady-state iteration count)
    print(json.dumps({"value": nc * nd / t, "unit": "updates/s", "cores": 1,
                      "sample": f"{cfg.name}: full mesh x {nd} dirs x band-row 0, 1 step after 1 untimed, {t:.2f} s"}))


def _bench_config(args):
    import dataclasses
    from paper_conf_ipps_heislersdms24_b200 import inputs as gen
    cfg = gen.make_config(args.config)
    if args.ic_eps is not None:
        cfg = dataclasses.replace(cfg, ic_eps=args.ic_eps)
    if args.rate_law:  # N1: temperature-dependent tau, dt = 0.5 x the bound at the hot wall
        bands = gen.with_rate_law(cfg.bands)
        cfg = dataclasses.replace(cfg, bands=bands,
                                  dt=0.5 * gen.cartesian_dt_bound(cfg.mesh, bands, cfg.dirs, t_max=350.0))
    return cfg


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, on this host's cores, on
    the same workload / metric (rank 0 only; other ranks exit 0).  One bounded
    sample of the workload (full mesh and directions, the first k band-rows,
    the seeded IC; built untimed), then W untimed and K timed oracle steps;
    value = sample updates / median step time."""
    rank, world, _ = _dist()
    if rank != 0:
        return
    cfg = _bench_config(args)
    cores = os.cpu_count() or 1
    os.environ.setdefault("OMP_NUM_THREADS", str(cores))
    nc, nd, nb = cfg.mesh["n_cells"], cfg.dirs["n_dirs"], cfg.bands["n_bands"]
    p, I, T, Tr = _oracle_sample(cfg, 1)
    t1 = _time_oracle_steps(p, I, T, Tr, cfg.dt, 1)[0][0]
    k = int(max(1, min(nb, 4.0 / max(t1, 1e-3))))  # ~4 s per step
    p, I, T, Tr = _oracle_sample(cfg, k)
    _, (I, T, Tr) = _time_oracle_steps(p, I, T, Tr, cfg.dt, args.warmup)
    ts, _ = _time_oracle_steps(p, I, T, Tr, cfg.dt, args.steps)
    v = nc * nd * k / statistics.median(ts)
    cb = {"value": v, "unit": "updates/s", "cores": int(os.environ["OMP_NUM_THREADS"]), "kind": "oracle",
          "cpu_model": _cpu_model(),
          "sample": f"{cfg.name}: full mesh ({nc} cells) x {nd} dirs x first {k} of {nb} band-rows, seeded IC, "
                    f"{args.warmup} untimed + {args.steps} timed steps (median {statistics.median(ts):.2f} s)"}
    line = {"metric": METRIC, "value": v, "unit": "updates/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "higher_is_better": True, "impl": "reference", "dtype": "f64",
            "data": "synthetic", "scaling": "strong",
            "config": {"workload": WORKLOADS[args.config], "name": args.config,
                       "relaxation": "tau(T) law" if args.rate_law else "constant tau"},
            "vs_baseline": None, "cpu_baseline": cb,
            "e2e": {"value": v, "unit": "updates/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_ours(args):
    import numpy as np
    import torch

    rank, world, local = _dist()
    assert world == args.gpus or (world == 1 and args.gpus == 1), "launch N>1 with torch.distributed.run"
    torch.cuda.set_device(local)
    pg = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        pg = dist
    from paper_conf_ipps_heislersdms24_b200 import bte
    from paper_conf_ipps_heislersdms24_b200 import inputs as gen

    cfg = _bench_config(args)
    nccl_id = None
    if world > 1:
        from paper_conf_ipps_heislersdms24_b200.dist import share_nccl_id
        nccl_id = share_nccl_id(pg, rank)
    stream = torch.cuda.current_stream()
    part_kw = {}
    if args.cell_parts > 1:  # cell partitioning, x band groups = world / cell_parts
        from paper_conf_ipps_heislersdms24_b200.dist import partition_cells, slab_partition
        assert world % args.cell_parts == 0, "--cell-parts must divide the number of GPUs"
        cen = cfg.mesh["cell_centre"]  # 3-D grids: z slabs (the box kernel keeps running); else bisection
        parts = slab_partition(cen, args.cell_parts) if cfg.mesh["dim"] == 3 else partition_cells(cen, args.cell_parts)
        part_kw = dict(cell_part=parts, n_cell_parts=args.cell_parts)
    s = bte.solver_from_config(cfg, rank=rank, world=world, device=local, nccl_id=nccl_id, stream=stream, **part_kw,
                               profile=True, band_group=args.band_group, block_threads=args.block_threads,
                               max_spare_slabs=args.max_spare, dir_chunk=args.dir_chunk,
                               locality=not args.no_locality, tma=not args.no_tma,
                               box=not args.no_box)
    bte.apply_ic(s, cfg)
    nb_loc = s.b_hi - s.b_lo
    nc, nd, nb = cfg.mesh["n_cells"], cfg.dirs["n_dirs"], cfg.bands["n_bands"]
    nc_loc = s.n_cells  # owned cells (all of them without --cell-parts)
    dt = cfg.dt

    def barrier():
        if pg is not None:
            pg.barrier()

    # ---- warm-up
    s.step(dt, args.warmup)
    torch.cuda.synchronize()
    s.reset_stats()

    # ---- timed region: K steps, device-resident state
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        torch.cuda.synchronize()
        e0.record(stream)
        s.step(dt, args.steps)
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
    ms = e0.elapsed_time(e1)
    st = s.stats()
    clocks = clk.summary()
    if pg is not None:
        t = torch.tensor([ms], device="cuda", dtype=torch.float64)
        pg.all_reduce(t, op=pg.ReduceOp.MAX)
        ms = float(t.item())
    total_updates = nc * nd * nb * args.steps  # whole job, all ranks
    value = total_updates / (ms / 1e3)

    # ---- roofline of the dominant kernel (the flux kernel: a1-a3 over every
    # cell), from the library's CUDA events on the launching stream over the
    # timed region.  A step launches it once per band-group segment; achieved =
    # algorithmic bytes of all flux launches of a step / their summed time.
    flux_launches_per_step = st["flux_launches"] / args.steps
    t_flux = st["ms_flux_interior"] / args.steps / 1e3
    alg_bytes = BYTES_PER_UPDATE * nc_loc * nd * nb_loc  # per step, this rank
    peak, peak_src = _peaks()
    achieved = alg_bytes / t_flux / 1e9 if t_flux > 0 else None
    traffic, traffic_src = (_traffic_from_profiles(args.config + ("+law" if args.rate_law else ""), alg_bytes)
                            if world == 1 else (None, None))
    roof = {"bound": "hbm", "kernel": "bte::flux_*_kernel (all cells; a1+a2+a3)", "achieved": achieved, "peak": peak,
            "unit": "GB/s", "frac": (achieved / peak) if achieved else None, "traffic": traffic,
            "peak_source": peak_src, "traffic_source": traffic_src,
            "alg_bytes_per_step": alg_bytes, "flux_launches_per_step": flux_launches_per_step,
            "kernel_ms_per_step": t_flux * 1e3,
            "share_of_step": st["ms_flux_interior"] / ms if ms > 0 else None,
            "step_alg_GBs": BYTES_PER_UPDATE * nc_loc * nd * nb_loc * args.steps / (ms / 1e3) / 1e9}
    phases = {k: st[k] / args.steps for k in ("ms_flux_interior", "ms_flux_boundary", "ms_allreduce", "ms_newton",
                                              "ms_halo")}

    # ---- end-to-end through the public API with host buffers: upload the state
    # (pinned host -> device) once, then every step bte_step + read T back.
    e2e = None
    state_gb = nb_loc * nd * nc_loc * 8 / 1e9
    if not args.no_e2e and state_gb > E2E_MAX_GB:  # C5: the host copy would need ~156 GB of pinned RAM
        e2e = {"skipped": f"state {state_gb:.0f} GB per rank > {E2E_MAX_GB} GB of pinned host memory"}
    elif not args.no_e2e:
        e2e = _e2e(s, pg, world, nb_loc, nd, nc_loc, dt, total_updates, args)

    cb = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cb = cpu_baseline(cfg)
    _emit(locals())


def _e2e(s, pg, world, nb_loc, nd, nc, dt, total_updates, args):
    import torch
    def barrier():
        if pg is not None:
            pg.barrier()
    pin_I = torch.empty((nb_loc, nd, nc), dtype=torch.float64).pin_memory()
    pin_T = torch.empty((nc,), dtype=torch.float64).pin_memory()
    s.intensity(out=pin_I.numpy())
    barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    s.set_intensity(pin_I)
    for _ in range(args.steps):
        s.step(dt, 1)
        s.temperature(out=pin_T.numpy())
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    if pg is not None:
        t = torch.tensor([e2e_s], device="cuda", dtype=torch.float64)
        pg.all_reduce(t, op=pg.ReduceOp.MAX)
        e2e_s = float(t.item())
    e2e = {"value": total_updates / e2e_s, "unit": "updates/s",
           "h2d_bytes_per_step": int(nb_loc * nd * nc * 8 / args.steps),  # (this rank's state, once per K steps)
           "d2h_bytes_per_step": int(nc * 8),
           "how": "timed: bte_set_intensity(state from pinned host) once + K x (bte_step(dt,1) + "
                  "bte_get_temperature(pinned host)); wall clock, max over ranks"}
    return e2e


def bte_variant(st):
    from paper_conf_ipps_heislersdms24_b200.bte import FLUX_VARIANTS
    return FLUX_VARIANTS.get(st.get("flux_variant"), "?")


def _emit(v):
    rank, world, args, s, pg = v["rank"], v["world"], v["args"], v["s"], v["pg"]
    value, ms, nc, nd, nb, dt, roof, cb, e2e, clocks, st, phases = (
        v[k] for k in ("value", "ms", "nc", "nd", "nb", "dt", "roof", "cb", "e2e", "clocks", "st", "phases"))
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "updates/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOADS[args.config], "name": args.config, "n_cells": nc, "n_dirs": nd,
                       "n_band_rows": nb, "dt": dt,
                       "parallelism": (f"band-shard x{world}" if args.cell_parts == 1 else
                                       f"band-shard x{world // args.cell_parts} x cell-part x{args.cell_parts}"),
                       "halo_bytes_per_step_rank0": st["halo_bytes"],
                       "relaxation": "tau(T) law" if args.rate_law else "constant tau",
                       "l2": f"state {nc * nd * nb * 8 / 1e9:.1f} GB per copy >> 126 MB L2 (no flush needed)"},
            "roofline": roof, "cpu_baseline": cb, "e2e": e2e, "clocks": clocks,
            "gpu_launches": st["kernel_launches"], "phases_ms_per_step": phases,
            "newton_iter_max": st["newton_iter_max"], "band_group": st["band_group"],
            "block_threads": st["block_threads"], "dir_chunks": st["dir_chunks"],
            "spare_slabs": st["spare_slabs"], "flux_kernel": bte_variant(st),
        }
        print(json.dumps(line), flush=True)
    s.close()
    if pg is not None:
        pg.destroy_process_group()


def _spawn_ranks(args):
    """`python bench.py --gpus N` without a launcher: re-run this command under
    torch.distributed.run, one rank per GPU on this node (127.0.0.1 rendezvous);
    rank 0 prints the JSON line."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    sys.stdout.flush()
    os.execv(sys.executable, cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C4", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--band-group", type=int, default=0)
    ap.add_argument("--block-threads", type=int, default=0)
    ap.add_argument("--max-spare", type=int, default=0)
    ap.add_argument("--dir-chunk", type=int, default=0)
    ap.add_argument("--no-locality", action="store_true", help="keep row-major cell order (no Morton hint)")
    ap.add_argument("--no-tma", action="store_true", help="register-pipelined flux kernel instead of TMA-staged")
    ap.add_argument("--no-box", action="store_true", help="structured grids: TMA-staged kernel instead of the box kernel")
    ap.add_argument("--rate-law", action="store_true",
                    help="temperature-dependent relaxation times (SURVEY 8(f) N1) instead of constant tau")
    ap.add_argument("--ic-eps", type=float, default=None, help="override the IC perturbation (0: equilibrium IC)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the end-to-end leg (profiling runs)")
    ap.add_argument("--cell-parts", type=int, default=1,
                    help="cell partitioning (SURVEY 8(f) N3) into K parts x world/K band groups (default 1)")
    ap.add_argument("--_oracle-1core", dest="oracle_1core", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    if args.oracle_1core:
        return _oracle_one_core(args)
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return _spawn_ranks(args)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
