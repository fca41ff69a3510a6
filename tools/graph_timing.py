#!/usr/bin/env python
"""Per-step time with and without the 2-step CUDA graph (small, launch-bound
configs).  python tools/graph_timing.py C1 C2 C3"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen  # noqa: E402

for name in sys.argv[1:] or ["C1", "C2"]:
    cfg = gen.make_config(name)
    res = {}
    for label in ("graph", "no-graph"):
        if label == "no-graph":
            os.environ["BTE_NO_GRAPH"] = "1"
        else:
            os.environ.pop("BTE_NO_GRAPH", None)
        with bte.solver_from_config(cfg) as s:
            s.step(cfg.dt, 20)
            torch.cuda.synchronize()
            n = 400
            t0 = time.perf_counter()
            s.step(cfg.dt, n)
            torch.cuda.synchronize()
            res[label] = (time.perf_counter() - t0) / n * 1e6
            launches = s.stats()["kernel_launches"]
    print(f"{name}: {res['graph']:.1f} us/step with the graph, {res['no-graph']:.1f} us/step launching "
          f"(x{res['no-graph'] / res['graph']:.2f})", flush=True)
