"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

The oracle cannot fit 100M x 32 (hours single-threaded), so at full size the GPU result
is checked ("sampled outputs ... else via properties that hold at any size"):

* properties of the whole node array that hold at any size: BFS links, child counts sum
  to the parent's, the parent's value is the count-weighted mean of its children's, leaf
  counts sum to n, depth <= max_depth, the root value equals the fp64 mean of y;
* sampled nodes, one by one: the rows that reach a node are gathered (kept in row order)
  and the oracle fits a depth-1 tree on exactly those rows; in integer mode (the
  generator's integer-microsecond targets) its split feature, threshold, child counts
  and value must equal the node's bit for bit (greedy CART decides every node from its
  own rows only, Readings R4/R8);
* DSE prediction (configs[3] shape on one GPU, 2^28 candidates, depth-20 tree): sampled
  candidates predicted by the oracle must match bit for bit;
* the bench's KNN (2^16 x 2^20) and Random Forest (16 trees of 1M rows) lines: sampled
  queries / rows against the oracle, one full-size bootstrap tree exactly.
"""
import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dt():
    import paper_conf_ipps_metzgd23_b200 as m
    return m


def _check_array(nodes, n, max_depth):
    feat, left, right = nodes["feature"], nodes["left"], nodes["right"]
    cnt, val, dep = nodes["n_samples"], nodes["value"], nodes["depth"]
    assert cnt[0] == n
    internal = feat >= 0
    assert np.all(right[internal] == left[internal] + 1)
    assert np.all(left[~internal] == -1)
    li, ri = left[internal], right[internal]
    assert np.all(li > np.nonzero(internal)[0])  # BFS: children after the parent
    assert np.array_equal(cnt[li] + cnt[ri], cnt[internal])
    assert np.all(dep[li] == dep[internal] + 1)
    wmean = (val[li] * cnt[li] + val[ri] * cnt[ri]) / cnt[internal]
    np.testing.assert_allclose(wmean, val[internal], rtol=1e-9, atol=1e-12)
    assert cnt[~internal].sum() == n
    assert dep.max() <= max_depth


def _route(nodes, X, depth):
    """Node index of every row after `depth` steps down the tree (torch on the GPU: test
    infrastructure; leaves keep their rows)."""
    feat = torch.from_numpy(nodes["feature"].astype(np.int64)).cuda()
    thr = torch.from_numpy(nodes["threshold"]).cuda()
    left = torch.from_numpy(nodes["left"].astype(np.int64)).cuda()
    node = torch.zeros(X.shape[0], dtype=torch.int64, device=X.device)
    for _ in range(depth):
        f = feat[node]
        internal = f >= 0
        x = torch.gather(X, 1, f.clamp(min=0).unsqueeze(1)).squeeze(1).double()
        child = left[node] + (x > thr[node]).long()
        node = torch.where(internal, child, node)
    return node


def _sampled_nodes(nodes, lo, hi, k, rng):
    internal = np.nonzero((nodes["feature"] >= 0) & (nodes["n_samples"] >= lo) & (nodes["n_samples"] <= hi))[0]
    assert len(internal) > 0
    deep = sorted(internal, key=lambda i: -int(nodes["depth"][i]))[: max(1, k // 2)]
    rest = rng.choice(internal, size=min(k - len(deep), len(internal)), replace=False)
    return sorted(set(int(i) for i in list(deep) + list(rest)))


def test_fit_c3_full_size(dt):
    """BASELINE configs[2] at full size on one B200: 100M x 32 (S32, seed 3, pools 2^22 CNNs x
    2^12 GPUs), depth 16."""
    n, d, D = 100_000_000, 32, 16
    dt.dt_release_workspace()
    torch.cuda.empty_cache()
    X, y = dt.dt_gen_table(3, n, d=d, cnn_pool_bits=22, gpu_pool_bits=12, device="cuda")
    # the device generator is the shared input recipe: spot-check rows against datagen
    for r0 in (0, n // 2 + 17, n - 1000):
        Xh, yh = datagen.cnn_gpu_table(3, 1000, d=d, row0=r0, cnn_pool_bits=22, gpu_pool_bits=12)
        assert np.array_equal(X[r0:r0 + 1000].cpu().numpy(), Xh)
        assert np.array_equal(y[r0:r0 + 1000].cpu().numpy(), yh)
    tree = dt.dt_fit(X, y, D, 1)
    torch.cuda.synchronize()
    dt.dt_release_workspace()
    nodes = tree.nodes
    _check_array(nodes, n, D)
    mean = float(y.sum().item()) / n
    assert abs(nodes["value"][0] - mean) <= 1e-9 * abs(mean)
    # integer mode (Reading R17): integral targets, max|y| * n < 2^52
    assert bool((torch.floor(y) == y).all()) and float(y.abs().max()) * n < 2.0 ** 52
    rng = np.random.default_rng(0)
    picks = _sampled_nodes(nodes, 2000, 400_000, 6, rng)
    for k in picks:
        at = _route(nodes, X, int(nodes["depth"][k]))
        idx = torch.nonzero(at == k).squeeze(1)  # ascending row order
        assert idx.numel() == nodes["n_samples"][k]
        Xs, ys = X[idx].cpu().numpy(), y[idx].cpu().numpy()
        o = oracle.fit(Xs, ys, 1, 1)
        L = nodes["left"][k]
        assert o["feature"][0] == nodes["feature"][k], k
        assert o["threshold"][0] == nodes["threshold"][k], k
        assert o["value"][0] == nodes["value"][k], k
        assert o["n_samples"][1] == nodes["n_samples"][L], k
        assert o["n_samples"][2] == nodes["n_samples"][L + 1], k
    del X, y
    torch.cuda.empty_cache()


def test_dse_predict_bench_size_sampled(dt):
    """bench.py's DSE line: 2^28 candidates (configs[3] shape on one GPU) on the depth-20,
    min_samples_leaf-128 tree fitted on the configs[1] table; sampled predictions must
    equal the oracle's bit for bit."""
    dt.dt_release_workspace()
    torch.cuda.empty_cache()
    X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
    tree = dt.dt_fit(X, y, 20, 128)
    nd = 1 << 28
    Xd = dt.dt_gen_dse(3, 0, nd, 10, device="cuda")
    out = dt.dt_predict(tree, Xd)
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    idx = np.unique(np.concatenate([rng.integers(0, nd, 200_000), np.arange(1000), np.arange(nd - 1000, nd)]))
    ti = torch.from_numpy(idx).cuda()
    Xs = Xd[ti].cpu().numpy()
    # the candidates are the shared recipe's rows
    Xr = datagen.dse_candidates(3, 0, 1000)
    assert np.array_equal(Xs[:1000], Xr)
    assert np.array_equal(out[ti].cpu().numpy(), oracle.predict(tree.nodes, Xs))
    del Xd, out
    torch.cuda.empty_cache()


def test_knn_bench_size_sampled(dt):
    """bench.py's KNN line: 2^16 training rows of the configs[1] table x 2^20 held-out
    queries, k = 5; sampled queries equal the oracle's bit for bit."""
    X, y = dt.dt_gen_table(1, 1 << 16, d=16, device="cuda")
    Xq, _ = dt.dt_gen_table(2, 1 << 20, d=16, device="cuda")
    out = dt.dt_knn_predict(X, y, Xq, 5)
    torch.cuda.synchronize()
    idx = np.unique(np.concatenate([[0, (1 << 20) - 1], np.random.default_rng(5).integers(0, 1 << 20, 300)]))
    ti = torch.from_numpy(idx).cuda()
    want = oracle.knn_predict(X.cpu().numpy(), y.cpu().numpy(), Xq[ti].cpu().numpy(), 5)
    assert np.array_equal(out[ti].cpu().numpy(), want)


def test_forest_bench_size(dt):
    """bench.py's forest line (16 bagged trees of the configs[1] table, depth 12): tree 0
    equals the oracle's tree of the same bootstrap sample at full size (integer mode), and
    sampled forest predictions equal the oracle's tree-order mean of the GPU's trees."""
    X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
    fo = dt.dt_forest_fit(X, y, 16, 12, 1, seed=1)
    Xh, yh = X.cpu().numpy(), y.cpu().numpy()
    idx = oracle.bootstrap(1, 0, len(yh))
    o = oracle.fit(Xh[idx], yh[idx], 12, 1)
    g = fo.tree(0).nodes
    for f in ("feature", "threshold", "left", "n_samples", "value"):
        assert np.array_equal(g[f], o[f]), f
    Xv, _ = dt.dt_gen_table(2, 1_000_000, d=16, device="cuda")
    out = dt.dt_forest_predict(fo, Xv)
    rows = np.random.default_rng(6).integers(0, 1_000_000, 5000)
    trees = [fo.tree(t).nodes for t in range(16)]
    Xs = Xv[torch.from_numpy(rows).cuda()].cpu().numpy()
    assert np.array_equal(out[torch.from_numpy(rows).cuda()].cpu().numpy(), oracle.forest_predict(trees, Xs))


def test_fit_predict_beyond_2_24_nodes(dt):
    """A fully grown tree with more than 2^24 nodes (distinct x and y, max_depth -1, Reading
    R2): the packed 8-byte predict node has a 24-bit child field, so such trees take the
    16-byte wide form (dt_internal.cuh).  Checks: node array properties, every training row
    predicts its own target (interpolation), sampled rows bit-exact against the oracle's
    predict on the GPU's node array, and dt_predict_eval through the wide form."""
    n = (1 << 23) + 4099
    rng = np.random.default_rng(24)
    X = rng.permutation(n).astype(np.float32)[:, None]
    y = rng.permutation(n).astype(np.float64)
    Xd, yd = torch.from_numpy(X).cuda(), torch.from_numpy(y).cuda()
    t = dt.dt_fit(Xd, yd, -1, 1)
    nodes = t.nodes
    assert len(nodes) == 2 * n - 1 and len(nodes) >= (1 << 24)
    _check_array(nodes, n, 10_000)
    yh = dt.dt_predict(t, Xd)
    assert torch.equal(yh, yd)
    m = dt.dt_predict_eval(t, Xd, yd, 1)
    assert m["mape"] == 0.0 and m["r2"] == 1.0
    # unseen rows (between the training values) against the oracle, sampled
    q = (rng.integers(0, n, 4096) + rng.uniform(-0.6, 0.6, 4096)).astype(np.float32)[:, None]
    got = dt.dt_predict(t, torch.from_numpy(q).cuda()).cpu().numpy()
    assert np.array_equal(got, oracle.predict(nodes, q))
    # the same node array through dt_tree_from_nodes (host-built wide form)
    t2 = dt.dt_tree_from_nodes(nodes, 1)
    assert np.array_equal(dt.dt_predict(t2, torch.from_numpy(q).cuda()).cpu().numpy(), got)
    with pytest.raises(dt.DTError):
        dt.dt_predict_eval_depths(t, Xd, yd, 1)
    del t, t2
    dt.dt_release_workspace()
