"""One BASELINE configs[2] fit (100M x 32, depth 16) -- for ncu launch lists (measurement helper)."""
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_metzgd23_b200 as dt  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000_000
X, y = dt.dt_gen_table(3, n, d=32, cnn_pool_bits=22, gpu_pool_bits=12, device="cuda")
torch.cuda.synchronize()
t = dt.dt_fit(X, y, 16, 1)
print("nodes", t.size, "depth", t.depth)
