#!/usr/bin/env python
"""Build profiles/ncu_flux_summary.json (bench.py's roofline.traffic source):
one entry per workload from the `ncu --set full` captures of its flux kernel.

    python tools/flux_summary.py TAG C4=profiles/r02_ncu_box_C4.json C5=...:10 C3=... C3t=...

(":ROWS": the band-rows the captured launch covers, if not all of the step's --
C5 at one GPU rotates slabs: 11 rows per launch in the bench, 10 under ncu,
whose own allocations leave one spare slab less.)

Each input is a tools/ncu_summary.py `full` JSON of ONE flux launch; the entry
keeps its DRAM bytes (read + write, cold cache), its duration and the
algorithmic bytes of that launch (16 B per update of the rows it covers).
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# rows of the step one captured launch covers (C5 at one GPU: slab rotation, 11 of 55 rows)
ROWS_IN_LAUNCH = {"C5": 11}


def main():
    from paper_conf_ipps_heislersdms24_b200 import inputs as gen
    tag = sys.argv[1]
    out = {"note": "ncu --set full --clock-control none of one flux launch per workload (cold cache); "
                   "bench.py: roofline.traffic = dram_bytes_per_launch x flux launches per step",
           "round": tag,
           "use": "bench.py: roofline.traffic = traffic_over_alg x the step's algorithmic bytes"}
    for spec in sys.argv[2:]:
        cfg_name, path = spec.split("=", 1)
        rows = None
        if ":" in path:
            path, r = path.rsplit(":", 1)
            rows = int(r)
        d = json.load(open(path))
        cfg = gen.make_config(cfg_name[:-4] if cfg_name.endswith("+law") else cfg_name)  # (C4+law: the rate law)
        rows = rows or ROWS_IN_LAUNCH.get(cfg_name, cfg.bands["n_bands"])
        alg = 16.0 * cfg.mesh["n_cells"] * cfg.dirs["n_dirs"] * rows
        k = [k for k in d["kernels"] if "flux" in k["name"]][0]
        out[cfg_name] = {"source": os.path.relpath(path, ROOT), "flux_kernel": k["name"],
                         "dram_bytes_per_launch": k["dram_bytes"], "dram_read": k["dram_read"],
                         "dram_write": k["dram_write"], "duration_s": k["duration"],
                         "alg_bytes_per_launch": alg, "traffic_over_alg": k["dram_bytes"] / alg,
                         "rows_in_launch": rows}
    with open(os.path.join(ROOT, "profiles", "ncu_flux_summary.json"), "w") as f:
        json.dump(out, f, indent=1)
    for c, e in out.items():
        if isinstance(e, dict):
            print(f"{c:4s} {e['duration_s']*1e3:8.3f} ms  DRAM {e['dram_bytes_per_launch']/1e9:7.2f} GB  "
                  f"alg {e['alg_bytes_per_launch']/1e9:7.2f} GB  x{e['traffic_over_alg']:.3f}")


if __name__ == "__main__":
    main()
