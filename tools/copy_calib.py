"""Calibration: DRAM bytes and time of a plain device copy (torch), 8 GB each way."""
import torch
n = 1 << 30  # 8 GB of fp64
a = torch.empty(n, dtype=torch.float64, device="cuda").fill_(1.0)
b = torch.empty_like(a)
for _ in range(3):
    b.copy_(a)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    b.copy_(a)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 5
print(f"copy 8 GB: {ms:.3f} ms  {2 * 8 * n / ms / 1e6:.1f} GB/s")
