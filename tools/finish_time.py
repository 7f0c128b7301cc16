"""Host-side cost of dt_fit's readback at C2 (measurement helper): wall time of dt_fit
(graph replay) against the device time of the same calls (CUDA events)."""
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_metzgd23_b200 as dt  # noqa: E402

X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
for _ in range(3):
    t = dt.dt_fit(X, y, 12, 1)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
n = 20
a.record()
t0 = time.perf_counter()
for _ in range(n):
    t = dt.dt_fit(X, y, 12, 1)
t1 = time.perf_counter()
b.record()
torch.cuda.synchronize()
print(sys.argv[1] if len(sys.argv) > 1 else "", f"wall {1e3 * (t1 - t0) / n:.3f} ms/fit, events {a.elapsed_time(b) / n:.3f} ms/fit, nodes {t.size}")
