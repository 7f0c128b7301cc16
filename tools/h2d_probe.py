"""Host->device copy rate of the e2e inputs (measurement helper)."""
import time
import torch

n = 144_000_000 // 4
h = torch.empty(n, dtype=torch.float32).pin_memory()
d = torch.empty(n, dtype=torch.float32, device="cuda")
for _ in range(3):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(10):
    d.copy_(h, non_blocking=True)
b.record()
torch.cuda.synchronize()
ms = a.elapsed_time(b) / 10
print(f"H2D 144 MB pinned: {ms:.3f} ms = {144e6 / ms / 1e6:.1f} GB/s")
s = torch.cuda.Stream()
x = torch.randn(4096, 4096, device="cuda")
torch.cuda.synchronize()
a.record()
with torch.cuda.stream(s):
    for _ in range(10):
        d.copy_(h, non_blocking=True)
for _ in range(200):
    x = x * 1.0001
b.record()
torch.cuda.synchronize()
print(f"H2D on a side stream beside kernels: {a.elapsed_time(b):.3f} ms for 10 copies + 200 kernels")
