"""Forest fit timing for A/B (measurement helper): 16 trees of the C2 table, depth 12."""
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_metzgd23_b200 as dt  # noqa: E402

X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
dt.dt_forest_fit(X, y, 2, 12, 1, seed=1)
torch.cuda.synchronize()
ts = []
for _ in range(3):
    t0 = time.perf_counter()
    fo = dt.dt_forest_fit(X, y, 16, 12, 1, seed=1)
    torch.cuda.synchronize()
    ts.append((time.perf_counter() - t0) * 1e3)
print(sys.argv[1] if len(sys.argv) > 1 else "", "forest 16 trees ms:", [round(t, 1) for t in ts])
