import sys, numpy as np, torch
sys.path.insert(0, '.')
import datagen, oracle
import paper_conf_ipps_metzgd23_b200 as dt
lib = dt.load_library(sys.argv[1]); dt._lib = lib
for (n, d, D) in ((300, 2, 3), (5000, 4, 3), (20000, 16, 6)):
    X, y = datagen.random_table(1, n, d, kind="ties", int_y=True)
    try:
        t = dt.dt_fit(torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda(), D, 1)
        o = oracle.fit(X, y, D, 1); g = t.nodes
        print(n, d, D, "nodes", len(g), len(o), all(np.array_equal(g[f], o[f]) for f in ("feature", "threshold", "left", "n_samples", "value")), flush=True)
    except Exception as e:
        print(n, d, D, "ERR", e, flush=True); break
