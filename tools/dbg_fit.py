"""Quick GPU parity probe (development aid): small fits vs the oracle, first mismatch."""
import sys, time
import numpy as np
import torch
sys.path.insert(0, '.')
import datagen, oracle
import paper_conf_ipps_metzgd23_b200 as dt

def cmp(g, o):
    if len(g) != len(o):
        return f"len {len(g)} vs {len(o)}"
    for f in ("feature", "left", "right", "depth", "n_samples", "threshold", "value"):
        if not np.array_equal(g[f], o[f]):
            i = int(np.nonzero(g[f] != o[f])[0][0])
            return f"{f} @ {i}: {g[i]} vs {o[i]}"
    if not np.allclose(g["impurity"], o["impurity"], rtol=1e-9, atol=1e-12):
        return "impurity"
    return None

cases = [(1, 3, "ties", 2, 1), (10, 2, "ties", -1, 1), (100, 3, "ties", 3, 1), (1000, 4, "ties", -1, 1),
         (1000, 4, "continuous", 12, 1), (5000, 16, "mixed", 12, 1), (20000, 8, "ties", -1, 2),
         (3000, 8, "collinear", -1, 1), (4097, 3, "ties", 10, 1), (39, 1, "continuous", -1, 1),
         (20000, 32, "continuous", 12, 64), (2, 1, "ties", -1, 1)]
bad = 0
for n, d, kind, D, m in cases:
    X, y = datagen.random_table(d * 1000 + n, n, d, kind=kind, int_y=True, y_range=50)
    o = oracle.fit(X, y, D, m)
    try:
        t = dt.dt_fit(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), D, m)
        torch.cuda.synchronize()
        r = cmp(t.nodes, o)
    except Exception as e:
        r = f"EXC {e}"
    print(n, d, kind, D, m, "OK" if r is None else r, flush=True)
    bad += r is not None
X, y = datagen.cnn_gpu_table(1, 200_000)
o = oracle.fit(X, y, 12, 1)
t = dt.dt_fit(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), 12, 1)
r = cmp(t.nodes, o)
print("c2-200k", "OK" if r is None else r)
Xd, yd = torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda()
for _ in range(3):
    t = dt.dt_fit(Xd, yd, 12, 1)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(10):
    t = dt.dt_fit(Xd, yd, 12, 1)
torch.cuda.synchronize()
print("c2-200k ms/fit", (time.perf_counter() - t0) / 10 * 1e3)
print("BAD", bad)
