#!/usr/bin/env python
"""Average board power over 100 C4 steps (NVML energy counter) against the
enforced power limit: is the sustained step power-capped?"""
import os, sys, time
sys.path.insert(0, os.getcwd())
import pynvml, torch
from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen
pynvml.nvmlInit(); h = pynvml.nvmlDeviceGetHandleByIndex(0)
print("enforced limit W", pynvml.nvmlDeviceGetEnforcedPowerLimit(h) / 1000, "default", pynvml.nvmlDeviceGetPowerManagementDefaultLimit(h) / 1000)
cfg = gen.make_config("C4")
with bte.solver_from_config(cfg) as s:
    bte.apply_ic(s, cfg)
    s.step(cfg.dt, 3); torch.cuda.synchronize()
    e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h); t0 = time.time()
    s.step(cfg.dt, 100); torch.cuda.synchronize()
    e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h); t1 = time.time()
    print("100 steps %.3f s, avg power %.0f W" % (t1 - t0, (e1 - e0) / 1000 / (t1 - t0)))
    print("reasons 0x%x" % pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(h), "sm", pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
