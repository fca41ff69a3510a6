#!/usr/bin/env python
"""Per-step flux time of a long run with the GPU's SM / memory clocks, power
and temperatures read (NVML) after every step: is a sustained slowdown a clock
or a memory effect?   python tools/step_trend.py [C4] [steps] [pause_s] [eq]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import pynvml  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 60
pause = float(sys.argv[3]) if len(sys.argv) > 3 else 0.0  # idle seconds between steps
eq = len(sys.argv) > 4 and sys.argv[4] == "eq"             # equilibrium IC, walls at T0: constant values
cfg = gen.make_config(name)
if eq:
    import dataclasses
    cfg = dataclasses.replace(cfg, ic_eps=0.0, bcs=gen.gen_bcs_fig1(cfg.mesh, t_hot=300.0))
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
with bte.solver_from_config(cfg, profile=True, stream=torch.cuda.current_stream()) as s:
    bte.apply_ic(s, cfg)
    for i in range(n):
        s.reset_stats()
        s.step(cfg.dt, 1)
        st = s.stats()
        sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
        mem = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_MEM)
        pw = pynvml.nvmlDeviceGetPowerUsage(h) / 1000
        t = pynvml.nvmlDeviceGetTemperature(h, pynvml.NVML_TEMPERATURE_GPU)
        reasons = pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(h)
        if pause:
            import time
            time.sleep(pause)
        print(f"{i:3d} flux {st['ms_flux_interior']:.3f} ms  sm {sm} MHz mem {mem} MHz  {pw:.0f} W  {t} C  "
              f"reasons 0x{reasons:x}", flush=True)
