"""Feature-sharded CART decomposition across REAL process boundaries (gloo, world 2, CPU).

Each rank searches only its features (global feature j*world + rank) with exact
rationals (oracle/exact.py), the ranks all_gather their per-node bests, and every rank
reduces them in the fixed order of the library's decide step (highest gain, then lowest
global feature; positions within a feature are already lowest-first).  The resulting
tree must equal the exact greedy tree on every rank -- the host-side logic of
dt_fit_sharded (Multi-GPU), without a GPU.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sharded_tree(X, y, rank, world, max_depth, min_leaf):
    from fractions import Fraction

    from oracle import exact
    yy = [Fraction(int(v)) for v in y]
    n, d = X.shape
    mine = [f for f in range(d) if f % world == rank]
    nodes, queue, head = [None], [(list(range(n)), 0, 0)], 0
    while head < len(queue):
        rows, depth, idx = queue[head]
        head += 1
        ys = [yy[r] for r in rows]
        nd = dict(feature=-1, left=-1, threshold=0.0, n=len(rows), depth=depth)
        nodes[idx] = nd
        searchable = (max_depth < 0 or depth < max_depth) and len(rows) >= 2 * min_leaf and min(ys) != max(ys)
        best = None
        if searchable:
            for f, i, gain, thr, L, R in exact.candidates(X[:, mine], yy, rows, min_leaf):
                if best is None or gain > best[0]:
                    best = (gain, mine[f], thr, L, R)
        recs = [None] * world
        dist.all_gather_object(recs, None if best is None else (str(best[0]), best[1], best[2]))
        win = None
        for r in recs:  # fixed order: highest gain, then lowest global feature
            if r is None:
                continue
            g = Fraction(r[0])
            if win is None or g > win[0] or (g == win[0] and r[1] < win[1]):
                win = (g, r[1], r[2])
        if not searchable or win is None:
            continue
        f, thr = win[1], win[2]
        L = [r for r in rows if float(X[r, f]) <= thr]
        R = [r for r in rows if float(X[r, f]) > thr]
        li = len(nodes)
        nodes.extend([None, None])
        nd.update(feature=f, left=li, threshold=thr)
        queue.append((L, depth + 1, li))
        queue.append((R, depth + 1, li + 1))
    return [(nd["feature"], nd["left"], nd["threshold"], nd["n"]) for nd in nodes]


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import datagen
    from oracle import exact
    ok = True
    for seed in range(6):
        X, y = datagen.random_table(seed, 24, 5, kind=("ties", "collinear", "mixed")[seed % 3],
                                    int_y=True, y_range=6)
        for D, m in ((-1, 1), (2, 2)):
            got = _sharded_tree(X, y, rank, world, D, m)
            ref = exact.greedy_tree(X, list(map(int, y)), D, m)
            want = [(nd["feature"], nd["left"], nd["threshold"], nd["n"]) for nd in ref]
            ok &= got == want
    q.put((rank, ok))
    dist.destroy_process_group()


def test_feature_sharded_decomposition_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert sorted(r for r, _ in res) == [0, 1]
    assert all(ok for _, ok in res)


def _eval_worker(rank, world, port, q):
    """Row-sharded evaluation (dt_eval_sharded's decomposition): each rank reduces its rows
    to (sum |e|/max(|y|, eps), SSE, n, mean, M2), the ranks all_gather the partials and
    merge them in rank order (Chan); every rank must get the full-array metrics."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    rng = np.random.default_rng(0)
    y = rng.uniform(1, 1e4, 1001)
    yh = y + rng.standard_normal(1001) * 50
    lo, hi = (0, 400) if rank == 0 else (400, 1001)
    ys, hs = y[lo:hi], yh[lo:hi]
    e = ys - hs
    mean = ys.mean()
    part = torch.tensor([np.sum(np.abs(e) / np.maximum(np.abs(ys), np.finfo(float).eps)), np.sum(e * e),
                         float(len(ys)), mean, np.sum((ys - mean) ** 2)], dtype=torch.float64)
    parts = [torch.zeros(5, dtype=torch.float64) for _ in range(world)]
    dist.all_gather(parts, part)
    ape = sse = n = m = M2 = 0.0
    for p in parts:  # rank order
        pa, ps, pn, pm, pM = p.tolist()
        ape, sse = ape + pa, sse + ps
        if n == 0:
            n, m, M2 = pn, pm, pM
        else:
            tot = n + pn
            delta = pm - m
            m = m + delta * (pn / tot)
            M2 = M2 + pM + delta * delta * (n * pn / tot)
            n = tot
    r2 = 1 - sse / M2
    mape, r2o, _ = oracle.evaluate(y, yh, 3)
    q.put((rank, abs(ape / n - mape) <= 1e-12 * mape and abs(r2 - r2o) <= 1e-12 * abs(r2o) and n == 1001))
    dist.destroy_process_group()


def test_row_sharded_eval_decomposition_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_eval_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert sorted(r for r, _ in res) == [0, 1]
    assert all(ok for _, ok in res)


def _grid_worker(rank, world, port, q):
    """grid_search's rank split + gather (SURVEY 8e "LOO / grid") across real processes, with
    the library's fit / all-depth eval replaced by deterministic stand-ins (no GPU): every
    rank must return exactly the single-process grid."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import types
    src = open(os.path.join(os.path.dirname(__file__), "..", "paper_conf_ipps_metzgd23_b200", "__init__.py")).read()
    body = src[src.index("def grid_search("):src.index("\nclass Comm")]
    ns = {}

    class FakeTree:
        def __init__(self, m):
            self.split_evals, self.depth = 1000 + m, 5

    ns["dt_fit"] = lambda X, y, D, m, stream=None: FakeTree(m)
    ns["dt_predict_eval_depths"] = lambda t, Xv, yv, p, stream=None: [
        (t.split_evals * 1e-3 + d, float(d), -float(d)) for d in range(t.depth + 1)]
    exec(body, ns)
    X = types.SimpleNamespace(shape=(10, 4))

    def gather(obj):
        lst = [None] * world
        dist.all_gather_object(lst, obj)
        return lst
    depths, ms = list(range(1, 9)), [1, 2, 4, 8, 16, 32, 64]
    got = ns["grid_search"](X, None, None, None, depths, ms, rank=rank, world=world, gather=gather)
    want = ns["grid_search"](X, None, None, None, depths, ms)
    q.put((rank, got == want and len(got[0]) == len(depths) * len(ms)))
    dist.destroy_process_group()


def test_grid_search_rank_split_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_grid_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert sorted(r for r, _ in res) == [0, 1]
    assert all(ok for _, ok in res)
