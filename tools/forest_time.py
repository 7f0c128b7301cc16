"""Forest fit timing after other cached fit plans exist (diagnoses the plan cache's
effect on dt_forest_fit).  usage: python tools/forest_time.py"""
import sys
import time
import torch
sys.path.insert(0, '.')
import paper_conf_ipps_metzgd23_b200 as dt


def tf(X, y, T):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    fo = dt.dt_forest_fit(X, y, T, 12, 1, seed=1)
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) * 1e3, fo


X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
print("fresh: warm", tf(X, y, 2)[0], "timed", tf(X, y, 16)[0], "again", tf(X, y, 16)[0], flush=True)
dt.dt_fit(X, y, 12, 1)
X2, y2 = dt.dt_gen_table(5, 7_000_000, d=16, device="cuda")
for m in (1, 2):
    dt.dt_fit(X2, y2, 16, m)
torch.cuda.synchronize()
print("after c5-shaped plans: warm", tf(X, y, 2)[0], "timed", tf(X, y, 16)[0], "again", tf(X, y, 16)[0], flush=True)
dt.dt_fit(X2, y2, 16, 4)
dt.dt_release_workspace()
print("after release: warm", tf(X, y, 2)[0], "timed", tf(X, y, 16)[0], flush=True)
