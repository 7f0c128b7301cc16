import sys, numpy as np, torch
sys.path.insert(0, '.')
import datagen, oracle
import paper_conf_ipps_metzgd23_b200 as dt
n = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
d = int(sys.argv[2]) if len(sys.argv) > 2 else 16
D = int(sys.argv[3]) if len(sys.argv) > 3 else 6
X, y = datagen.random_table(1, n, d, kind="ties", int_y=True)
t = dt.dt_fit(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), D, 1)
o = oracle.fit(X, y, D, 1)
g = t.nodes
print("nodes", len(g), len(o), all(np.array_equal(g[f], o[f]) for f in ("feature", "threshold", "left", "n_samples", "value")))
