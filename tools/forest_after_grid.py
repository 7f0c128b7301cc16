"""Forest fit timing right after bench.py's DSE and C5 grid sections (its fit plans still cached).
usage: python tools/forest_after_grid.py"""
import sys
import time
import torch
sys.path.insert(0, '.')
import bench
import paper_conf_ipps_metzgd23_b200 as dt

sys.argv = [sys.argv[0]]
args = bench.parse()
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()
X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
dt.dt_fit(X, y, 12, 1)
Xdse = dt.dt_gen_dse(3, 0, 1 << 28, 10, device=dev)
tdse = dt.dt_fit(X, y, 20, 128)
out = torch.empty(1 << 28, dtype=torch.float64, device=dev)
dt.dt_predict(tdse, Xdse, out=out)
del Xdse, out
torch.cuda.synchronize()
t0 = time.perf_counter()
bench.extra_configs(args, dev, stream)
torch.cuda.synchronize()
print("extra_configs s", time.perf_counter() - t0, flush=True)
for tag, T in (("warm", 2), ("timed", 16), ("again", 16)):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    fo = dt.dt_forest_fit(X, y, T, 12, 1, seed=1)
    torch.cuda.synchronize()
    print(tag, (time.perf_counter() - t0) * 1e3, "ms", flush=True)
    del fo
