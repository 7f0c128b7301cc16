"""Runs a few C2 fits (1M x 16, depth 12) for ncu captures (development aid)."""
import sys
import torch
sys.path.insert(0, '.')
import paper_conf_ipps_metzgd23_b200 as dt
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
X, y = dt.dt_gen_table(1, 1_000_000, d=16)
for _ in range(reps):
    t = dt.dt_fit(X, y, 12, 1)
torch.cuda.synchronize()
print("nodes", t.size, "evals", t.split_evals)
