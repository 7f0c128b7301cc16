"""Small workloads of every library entry point, for compute-sanitizer (memcheck, racecheck,
synccheck): fits in integer and real mode (direct enqueue and graph replay),
the row-sharded fit on thread ranks, predict / eval / LOO / forest / KNN / factored DSE.
Usage: compute-sanitizer --tool <t> python tools/sanitize_fits.py"""
import sys
import threading

import numpy as np
import torch

sys.path.insert(0, ".")
import datagen  # noqa: E402
import paper_conf_ipps_metzgd23_b200 as dt  # noqa: E402


def cuda(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


for n, d, kind, D, m, real in [(3000, 5, "ties", -1, 1, False), (4097, 3, "continuous", 8, 2, True),
                               (9000, 16, "mixed", 10, 1, False)]:
    X, y = datagen.random_table(n, n, d, kind=kind, int_y=not real)
    Xd, yd = cuda(X), cuda(y)
    for _ in range(2):
        t = dt.dt_fit(Xd, yd, D, m)
    yh = dt.dt_predict(t, Xd)
    dt.dt_eval(yd, yh, d)
    dt.dt_predict_eval(t, Xd, yd, d)
    print("fit", n, d, kind, D, m, t.size, flush=True)
# row-sharded fit, 2 thread ranks
X, y = datagen.random_table(5, 6000, 6, kind="ties", int_y=True)
Xd, yd = cuda(X), cuda(y)
comms = dt.dt_comm_init_local(2)
res = [None, None]


def run(r):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        a, b = (0, 2500) if r == 0 else (2500, 6000)
        res[r] = dt.dt_fit_sharded(comms[r], Xd[a:b], yd[a:b], a, 6000, 8, 1, stream=s)


th = [threading.Thread(target=run, args=(r,)) for r in range(2)]
for t_ in th:
    t_.start()
for t_ in th:
    t_.join()
print("sharded", res[0].size, flush=True)
Xp, yp = datagen.paper_table(0)
dt.dt_loo(cuda(Xp), cuda(yp), -1, 1)
fo = dt.dt_forest_fit(Xd, yd, 3, 6, 1, seed=1)
dt.dt_forest_predict(fo, Xd)
dt.dt_knn_predict(Xd[:500].contiguous(), yd[:500].contiguous(), Xd[:300].contiguous(), 5)
Xc, yc = datagen.cnn_gpu_table(3, 20000)
tc = dt.dt_fit(cuda(Xc), cuda(yc), 8, 4)
cnn, gpu, src = datagen.dse_tables(3, 0, 64, 32)
dt.dt_predict_dse(tc, cuda(cnn), cuda(gpu), src)
cnn, gpu, src = datagen.dse_tables(3, 5, 50, 37)  # ragged last GPU group
dt.dt_predict_dse(tc, cuda(cnn), cuda(gpu), src)
big = dt.dt_fit(cuda(Xc), cuda(yc), -1, 1)       # large specialised trees: full-tree fallback groups
dt.dt_predict_dse(big, cuda(cnn), cuda(gpu), src)
dt.dt_profile_enable(True, graph=True)           # the fit graph with event-record nodes
for _ in range(2):
    dt.dt_fit(cuda(Xc), cuda(yc), 6, 2)
dt.dt_profile_enable(False)
torch.cuda.synchronize()
print("SANITIZE_DONE", flush=True)
