#!/usr/bin/env python
"""Summarise ncu captures into profiles/ (run here, on the CPU box).

    python tools/ncu_summary.py full  <rep.ncu-rep> <out.json> [--config C4] [--bands-in-launch 48 --bands 55]
    python tools/ncu_summary.py launches <launches.csv> <out.json>

`full`: per captured kernel the duration, DRAM bytes read/written, achieved
DRAM throughput, occupancy, registers and the top stall reasons.
`launches`: per kernel name the launch count, total/mean device time and its
share of all captured time (cold-cache, serialised: compare shares only).
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

KEYS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct_peak",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "l1tex__t_sector_hit_rate.pct": "l1_hit_pct",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct_peak",
    "smsp__inst_executed.sum": "instructions",
}
UNIT = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1.0, "Tbyte": 1e12,
        "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9, "second": 1.0,
        "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0}


def _num(v, unit):
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return v
    return x * UNIT.get(unit, 1.0)


def full(rep, out, config=None, bands_in_launch=None, bands=None):
    if rep.endswith(".csv"):  # a raw-page export (ncu -i REP --page raw --csv) made on the GPU box
        raw = open(rep).read()
    else:
        raw = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    kernels = []
    for r in rows[2:]:
        k = {"name": r[hdr.index("Kernel Name")]}
        for key, short in KEYS.items():
            if key in hdr:
                i = hdr.index(key)
                k[short] = _num(r[i], units[i])
        stalls = {}
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    stalls[h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]] = float(r[i])
                except ValueError:
                    pass
        k["top_stalls"] = dict(sorted(stalls.items(), key=lambda kv: -kv[1])[:5])
        if "dram_read" in k and "duration" in k:
            k["dram_bytes"] = k["dram_read"] + k["dram_write"]
            k["dram_GBs"] = k["dram_bytes"] / k["duration"] / 1e9
        kernels.append(k)
    res = {"source": rep, "config": config, "kernels": kernels}
    flux = [k for k in kernels if "flux" in k["name"]]
    if flux:
        res["dram_bytes_per_launch"] = flux[0]["dram_bytes"]
        res["flux_kernel"] = flux[0]["name"]
        if bands_in_launch and bands:  # the captured launch covers bands_in_launch of the step's rows
            res["dram_bytes_per_step"] = flux[0]["dram_bytes"] * bands / bands_in_launch
            res["bands_in_launch"], res["bands_per_step"] = bands_in_launch, bands
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    for k in kernels:
        print(f"{k['name'][:60]:60s} {k.get('duration', 0)*1e3:8.3f} ms  DRAM {k.get('dram_bytes', 0)/1e9:7.2f} GB "
              f"({k.get('dram_GBs', 0):7.1f} GB/s)  occ {k.get('achieved_occupancy_pct', 0):5.1f}%  regs {k.get('registers')}")


def launches(path, out):
    text = open(path).read()
    lines = [l for l in text.splitlines() if l.startswith('"')]
    rows = list(csv.reader(io.StringIO("\n".join(lines))))
    hdr = rows[0]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    ui = hdr.index("Metric Unit") if "Metric Unit" in hdr else None
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        if r[mi] != "gpu__time_duration.sum":
            continue
        t = _num(r[vi], r[ui] if ui is not None else "nsecond")
        if isinstance(t, str):
            continue
        if ui is None:
            t *= 1e-9
        a = agg[r[ki].split("(")[0]]
        a[0] += 1
        a[1] += t
    tot = sum(v[1] for v in agg.values())
    step = {k: v for k, v in agg.items() if any(t in k for t in ("flux", "newton", "sum_slots"))}
    tot_step = sum(v[1] for v in step.values()) or 1.0
    res = {k: {"launches": v[0], "total_ms": v[1] * 1e3, "mean_ms": v[1] * 1e3 / v[0], "share": v[1] / tot,
               "share_of_step_kernels": (v[1] / tot_step) if k in step else None}
           for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])}
    with open(out, "w") as f:
        json.dump({"source": path, "kernels": res,
                   "note": "cold-cache serialised ncu times; share_of_step_kernels = share among the step's kernels"},
                  f, indent=1)
    for k, v in res.items():
        ss = v["share_of_step_kernels"]
        print(f"{k[:60]:60s} n={v['launches']:4d} mean {v['mean_ms']:9.3f} ms share {v['share']*100:5.1f}%"
              + (f"  step-share {ss*100:5.1f}%" if ss is not None else ""))


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "full":
        arg = lambda k, d=None: sys.argv[sys.argv.index(k) + 1] if k in sys.argv else d
        bil, nb = arg("--bands-in-launch"), arg("--bands")
        full(sys.argv[2], sys.argv[3], arg("--config", "C4"), int(bil) if bil else None, int(nb) if nb else None)
    else:
        launches(sys.argv[2], sys.argv[3])
