"""Value-range row-sharded CART across REAL process boundaries (gloo, world 2, CPU): the
host-side logic of dt_fit_sharded without a GPU.

Each rank holds a contiguous block of rows.  The presort: a local sort by the 64-bit key
(flip(x) << 32 | row id), exact splitters by 64 bisection rounds on the ranks' summed
counts, an all-to-all of the entries; rank p must then hold exactly the global sorted
positions [p n / P, (p + 1) n / P) of every feature list.  The levels: per (node, feature)
each rank all_gathers its boundary record (count, sum of y, last x) and forms its rank
carries (entries, S' and neighbour x of the lower ranks), scores its own positions with
exact rationals (oracle/exact.py definitions), the ranks all_gather their per-node bests
and reduce them in the library's fixed order (highest gain, then lowest feature, then
lowest position), OR together the go-left rows of their split-feature parts and partition
their lists stably.  The resulting tree must equal the exact greedy tree on every rank.
"""
import os
import socket
from fractions import Fraction

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


def _flip(x):
    u = int(np.float32(x).view(np.uint32))
    if (u << 1) & 0xFFFFFFFF == 0:
        u = 0  # -0.0 == +0.0
    return (~u) & 0xFFFFFFFF if u & 0x80000000 else u | 0x80000000


def _gather(obj, world):
    lst = [None] * world
    dist.all_gather_object(lst, obj)
    return lst


def _value_range_presort(X, rank, world):
    """Per feature: this rank's sorted (key, row) entries after the exchange."""
    n, d = X.shape
    lo, hi = rank * n // world, (rank + 1) * n // world
    local = [sorted((_flip(X[r, f]) << 32 | r) for r in range(lo, hi)) for f in range(d)]
    # splitters: max composite K with global count(< K) <= t_b, t_b = b n / world
    bounds = [[0, (1 << 64) - 1] for _ in range(d * (world - 1))]
    for _ in range(64):
        mids = [(a + (b - a) // 2) for a, b in bounds]
        cnt = [sum(1 for v in local[i // (world - 1)] if v < mids[i]) for i in range(len(mids))]
        tot = [sum(c) for c in zip(*_gather(cnt, world))]
        for i, (a, b) in enumerate(bounds):
            if b - a > 1:
                t = (i % (world - 1) + 1) * n // world
                bounds[i] = [mids[i], b] if tot[i] <= t else [a, mids[i]]
    cuts = [[0] + [bounds[f * (world - 1) + q][0] for q in range(world - 1)] + [1 << 64] for f in range(d)]
    send = [[[v for v in local[f] if cuts[f][q] <= v < cuts[f][q + 1]] for f in range(d)] for q in range(world)]
    got = _gather(send, world)  # got[src][dst][f]
    mine = [sorted(v for src in range(world) for v in got[src][rank][f]) for f in range(d)]
    return [[(v >> 32, v & 0xFFFFFFFF) for v in lst] for lst in mine]


def _sharded_tree(X, y, rank, world, max_depth, min_leaf):
    n, d = X.shape
    yy = [Fraction(int(v)) for v in y]
    lists = _value_range_presort(X, rank, world)
    # the exchange must leave rank p with global sorted positions [p n / P, (p+1) n / P)
    for f in range(d):
        glob = sorted(range(n), key=lambda r: (_flip(X[r, f]), r))
        assert [r for _, r in lists[f]] == glob[rank * n // world:(rank + 1) * n // world]
    segs = {0: [[r for _, r in lists[f]] for f in range(d)]}  # node -> per-feature local rows (sorted)
    nodes, queue, head = [None], [(0, 0, n)], 0
    while head < len(queue):
        idx, depth, N = queue[head]
        head += 1
        nd = dict(feature=-1, left=-1, threshold=0.0, n=N)
        nodes[idx] = nd
        seg = segs.pop(idx)
        ys0 = [yy[r] for r in seg[0]]
        mm = _gather((min(ys0) if ys0 else None, max(ys0) if ys0 else None), world)
        lo_y = min(a for a, _ in mm if a is not None)
        hi_y = max(b for _, b in mm if b is not None)
        searchable = (max_depth < 0 or depth < max_depth) and N >= 2 * min_leaf and lo_y != hi_y
        best = None
        if searchable:
            recs = _gather([(len(seg[f]), sum((yy[r] for r in seg[f]), Fraction(0)),
                             float(X[seg[f][-1], f]) if seg[f] else None) for f in range(d)], world)
            tot = [sum((recs[q][f][1] for q in range(world)), Fraction(0)) for f in range(d)]
            for f in range(d):
                ioff = sum(recs[q][f][0] for q in range(rank))
                soff = sum((recs[q][f][1] for q in range(rank)), Fraction(0))
                xprev = None
                for q in range(rank):
                    if recs[q][f][0]:
                        xprev = recs[q][f][2]
                S = soff
                for t, r in enumerate(seg[f]):
                    i, x = ioff + t, float(X[r, f])
                    if i >= max(min_leaf, 1) and N - i >= min_leaf and xprev is not None and np.float32(xprev) < np.float32(x):
                        nl, nr = i, N - i
                        gain = (S * nr - (tot[f] - S) * nl) ** 2 / (N * nl * nr)  # = SSE_P - SSE_L - SSE_R
                        if best is None or gain > best[0]:  # strict >: lowest position per feature
                            best = (gain, f, i, float(xprev) / 2.0 + x / 2.0)
                    S += yy[r]
                    xprev = x
        bests = _gather(None if best is None else (str(best[0]), best[1], best[2], best[3]), world)
        win = None
        for b in bests:  # rank order: highest gain, then lowest feature, then lowest position
            if b is None:
                continue
            g = Fraction(b[0])
            if win is None or g > win[0] or (g == win[0] and (b[1] < win[1] or (b[1] == win[1] and b[2] < win[2]))):
                win = (g, b[1], b[2], b[3])
        if not searchable or win is None:
            continue
        f, i, thr = win[1], win[2], win[3]
        ioff = sum(c for c in _gather(len(seg[f]), world)[:rank])
        left_mine = {r for t, r in enumerate(seg[f]) if ioff + t < i}
        left = set().union(*_gather(left_mine, world))  # the OR-allreduce of the go-left bitmap
        li = len(nodes)
        nodes.extend([None, None])
        nd.update(feature=f, left=li, threshold=thr)
        segs[li] = [[r for r in seg[g] if r in left] for g in range(d)]
        segs[li + 1] = [[r for r in seg[g] if r not in left] for g in range(d)]
        queue.append((li, depth + 1, i))
        queue.append((li + 1, depth + 1, N - i))
    return [(nd["feature"], nd["left"], nd["threshold"], nd["n"]) for nd in nodes]


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import datagen
    from oracle import exact
    ok = True
    for seed in range(6):
        X, y = datagen.random_table(seed, 24, 3, kind=("ties", "collinear", "mixed")[seed % 3],
                                    int_y=True, y_range=6)
        for D, m in ((-1, 1), (2, 2)):
            got = _sharded_tree(X, y, rank, world, D, m)
            ref = exact.greedy_tree(X, list(map(int, y)), D, m)
            want = [(nd["feature"], nd["left"], nd["threshold"], nd["n"]) for nd in ref]
            ok &= got == want
    q.put((rank, ok))
    dist.destroy_process_group()


def test_value_range_sharded_decomposition_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
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
    ns["dt_fit_grid"] = lambda X, y, D, ms, stream=None: [FakeTree(m) for m in ms]
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
