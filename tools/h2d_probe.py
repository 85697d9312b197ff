"""Diagnostic: raw pinned host -> device copy bandwidth (the PCIe ceiling of bench.py's e2e)."""
import torch, time
n = 1 << 30
h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for _ in range(3): d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): d.copy_(h, non_blocking=True)
e1.record(); torch.cuda.synchronize()
print("H2D pinned 1 GiB x10:", 10 * n / (e0.elapsed_time(e1) / 1e3) / 1e9, "GB/s")
s2 = torch.cuda.Stream()
d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True)
torch.cuda.synchronize()
e0.record()
for _ in range(5):
    d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): d2.copy_(h2, non_blocking=True)
torch.cuda.synchronize(); e1.record(); torch.cuda.synchronize()
print("H2D two streams:", 10 * n / (e0.elapsed_time(e1) / 1e3) / 1e9, "GB/s")
