"""Factored DSE predict (T_est = t_dca + n * t_pm):
candidate (i, j) = CNN row i composed with GPU row j, never materialised.

The oracle side is the plain definition: compose every candidate row explicitly and
predict it with oracle.predict (the CPU tree walk).  Predictions from the same tree must
be bit-exact (BASELINE.json contract).
"""
import numpy as np
import pytest

import datagen
import oracle


def test_dse_tables_compose_to_candidates():
    """The factor tables are the shared recipe's cross product (no GPU)."""
    cnn, gpu, src = datagen.dse_tables(3, 5, 7, 16)
    X = datagen.dse_candidates(3, 5 << 4, 7 << 4, gpu_bits=4)
    comp = np.concatenate([np.repeat(cnn, 16, axis=0), np.tile(gpu, (7, 1))], axis=1)
    assert np.array_equal(comp, X)
    assert src == list(range(10)) + [-1, -2, -3, -4, -5, -6]


def _compose(cnn, gpu, src):
    n_cnn, n_gpu = len(cnn), len(gpu)
    X = np.empty((n_cnn * n_gpu, len(src)), dtype=np.float32)
    for f, c in enumerate(src):
        X[:, f] = np.repeat(cnn[:, c], n_gpu) if c >= 0 else np.tile(gpu[:, -1 - c], n_cnn)
    return X


torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def dt():
    import paper_conf_ipps_metzgd23_b200 as m
    return m


@pytest.mark.gpu
@pytest.mark.parametrize("n_cnn,n_gpu,D,m", [(1, 1, 3, 1), (7, 1024, 20, 128), (33, 37, 12, 1),
                                           (256, 1000, 8, 4)])
def test_predict_dse_matches_oracle(dt, n_cnn, n_gpu, D, m):
    X, y = datagen.cnn_gpu_table(1, 50_000)
    nodes = oracle.fit(X, y, D, m)
    tree = dt.dt_tree_from_nodes(nodes, 16)
    cnn, gpu, src = datagen.dse_tables(3, 11, n_cnn, n_gpu)
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    want = oracle.predict(nodes, _compose(cnn, gpu, src))
    assert np.array_equal(out.cpu().numpy(), want)


@pytest.mark.gpu
def test_predict_dse_interleaved_columns_and_global_tree(dt):
    """Arbitrary feature_src (CNN and GPU columns interleaved, one column used twice) and
    a tree too large for shared memory beside the GPU table (read through L1/L2)."""
    rng = np.random.default_rng(4)
    n = 120_000
    X = rng.integers(0, 1000, size=(n, 6)).astype(np.float32)
    y = np.floor(rng.random(n) * 1e6)
    nodes = oracle.fit(X, y, -1, 1)
    assert len(nodes) * 8 > 227 * 1024  # forces the global-tree path
    tree = dt.dt_tree_from_nodes(nodes, 6)
    cnn = rng.integers(0, 1000, size=(5, 3)).astype(np.float32)
    gpu = rng.integers(0, 1000, size=(4000, 4)).astype(np.float32)
    src = [-3, 0, -1, 2, 0, -4]
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    assert np.array_equal(out.cpu().numpy(), oracle.predict(nodes, _compose(cnn, gpu, src)))
    # the same candidates through dt_predict (materialised rows)
    Xc = torch.from_numpy(_compose(cnn, gpu, src)).cuda()
    assert torch.equal(dt.dt_predict(tree, Xc), out)


@pytest.mark.gpu
def test_predict_dse_bench_size_sampled(dt):
    """bench.py's factored line: 2^20 CNNs x 2^10 GPUs (BASELINE configs[3]) on the
    depth-20 / min_samples_leaf-128 tree; sampled CNN rows checked bit for bit."""
    X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
    tree = dt.dt_fit(X, y, 20, 128)
    n_cnn, n_gpu = 1 << 20, 1 << 10
    cnn, gpu, src = datagen.dse_tables(3, 0, n_cnn, n_gpu)
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    torch.cuda.synchronize()
    rows = np.unique(np.concatenate([[0, 1, n_cnn - 1], np.random.default_rng(2).integers(0, n_cnn, 40)]))
    for i in rows:
        want = oracle.predict(tree.nodes, _compose(cnn[i:i + 1], gpu, src))
        assert np.array_equal(out[i * n_gpu:(i + 1) * n_gpu].cpu().numpy(), want), i
    del out
    torch.cuda.empty_cache()


@pytest.mark.gpu
def test_predict_dse_rejects_bad_args(dt):
    X, y = datagen.cnn_gpu_table(1, 1000)
    tree = dt.dt_tree_from_nodes(oracle.fit(X, y, 3, 1), 16)
    cnn, gpu, src = datagen.dse_tables(3, 0, 2, 4)
    bad = list(src)
    bad[0] = 10  # CNN column out of range
    with pytest.raises(dt.DTError):
        dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), bad)


@pytest.mark.gpu
def test_predict_dse_large_gpu_table(dt):
    """2^16 GPU rows (2048 groups of GPU-specialised trees, no shared-memory table limit)
    and a ragged last group: bit-exact against the composed rows."""
    X, y = datagen.cnn_gpu_table(1, 50_000)
    nodes = oracle.fit(X, y, 14, 8)
    tree = dt.dt_tree_from_nodes(nodes, 16)
    cnn, gpu, src = datagen.dse_tables(3, 0, 3, (1 << 16) - 5)
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    assert np.array_equal(out.cpu().numpy(), oracle.predict(nodes, _compose(cnn, gpu, src)))


def _chain_tree(depth, src, rng):
    """A caterpillar tree: internal node 2k (depth k) splits feature f_k, its left child
    2k+1 is a leaf, its right child 2k+2 the next internal node; deeper than the
    specialiser's stack for depth > 62 (the full-tree path)."""
    import oracle as o
    n = 2 * depth + 1
    nodes = np.zeros(n, dtype=o.NODE_DTYPE)
    nodes["feature"] = -1
    nodes["left"] = -1
    nodes["right"] = -1
    for k in range(depth):
        i = 2 * k
        nodes[i]["feature"] = k % len(src)
        nodes[i]["left"], nodes[i]["right"] = i + 1, i + 2
        nodes[i]["threshold"] = float(rng.integers(0, 60))
        nodes[i + 1]["depth"] = k + 1
        nodes[i + 2]["depth"] = k + 1
    nodes["value"] = np.arange(n, dtype=np.float64) * 1.5
    nodes["n_samples"] = 1
    return nodes


@pytest.mark.gpu
@pytest.mark.parametrize("depth", [5, 61, 100])
def test_predict_dse_deep_chain(dt, depth):
    """Trees whose specialised walk needs every step (and, at depth 100, the full-tree
    fallback): bit-exact."""
    rng = np.random.default_rng(depth)
    src = [0, -1, 1, -2, 2, -3]
    nodes = _chain_tree(depth, src, rng)
    tree = dt.dt_tree_from_nodes(nodes, len(src))
    cnn = rng.integers(0, 64, size=(40, 3)).astype(np.float32)
    gpu = rng.integers(0, 64, size=(70, 3)).astype(np.float32)
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    assert np.array_equal(out.cpu().numpy(), oracle.predict(nodes, _compose(cnn, gpu, src)))


@pytest.mark.gpu
def test_predict_dse_edge_cases(dt):
    """A single-leaf tree; NaN / inf CNN and GPU features (x > t is false: left, as in
    dt_predict); more than 32 CNN columns (the rank form's limit: full-tree walks); one
    GPU row; every case against dt_predict on the composed rows and the oracle."""
    rng = np.random.default_rng(11)
    # single leaf
    X, y = datagen.cnn_gpu_table(1, 1000)
    nodes = oracle.fit(X, y, 0, 1)
    tree = dt.dt_tree_from_nodes(nodes, 16)
    cnn, gpu, src = datagen.dse_tables(3, 0, 5, 7)
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    assert np.array_equal(out.cpu().numpy(), np.full(35, nodes["value"][0]))
    # non-finite features
    X, y = datagen.cnn_gpu_table(1, 20_000)
    nodes = oracle.fit(X, y, 10, 4)
    tree = dt.dt_tree_from_nodes(nodes, 16)
    cnn, gpu, src = datagen.dse_tables(3, 0, 40, 33)
    cnn[::3, 0] = np.nan
    cnn[1::5, 4] = np.inf
    gpu[::4, 1] = -np.inf
    gpu[2::7, 0] = np.nan
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    Xc = _compose(cnn, gpu, src)
    ref = dt.dt_predict(tree, torch.from_numpy(Xc).cuda())
    assert torch.equal(out, ref)
    # > 32 CNN columns (tree features reach column 40), one GPU row
    n = 30_000
    Xw = rng.integers(0, 50, size=(n, 42)).astype(np.float32)
    yw = np.floor(rng.random(n) * 1e4)
    nodes = oracle.fit(Xw, yw, 8, 2)
    tree = dt.dt_tree_from_nodes(nodes, 42)
    src = list(range(41)) + [-1]
    cnn = rng.integers(0, 50, size=(64, 41)).astype(np.float32)
    gpu = rng.integers(0, 50, size=(1, 1)).astype(np.float32)
    out = dt.dt_predict_dse(tree, torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda(), src)
    assert np.array_equal(out.cpu().numpy(), oracle.predict(nodes, _compose(cnn, gpu, src)))
