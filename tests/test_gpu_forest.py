"""Random Forest (bagged CART) through the C ABI vs the oracle.

Integer mode (the generator's integer-microsecond targets): every tree identical to the
oracle's tree of the same bootstrap sample, predictions bit-exact.  Real mode: trees by
root path with exact-tie adjudication (treecmp); forest predictions from the GPU's own
trees bit-exact against the oracle's forest mean of those trees.
"""
import numpy as np
import pytest

import datagen
import oracle
import treecmp

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dt():
    import paper_conf_ipps_metzgd23_b200 as m
    return m


def _cuda(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("seed,t,n", [(0, 0, 1), (1, 0, 10), (7, 3, 100_003), (2**63 + 5, 99, 777)])
def test_bootstrap_bitexact(dt, seed, t, n):
    got = dt.dt_bootstrap(seed, t, n).cpu().numpy().view(np.uint32)
    assert np.array_equal(got, oracle.bootstrap(seed, t, n))


@pytest.mark.parametrize("n,d,kind,T,D,m", [(3000, 4, "ties", 5, -1, 1), (20000, 16, "mixed", 4, 8, 3),
                                            (1, 2, "ties", 2, 3, 1), (50000, 8, "collinear", 3, 12, 1)])
def test_forest_integer_mode_exact(dt, n, d, kind, T, D, m):
    X, y = datagen.random_table(n + d, n, d, kind=kind, int_y=True)
    fo = dt.dt_forest_fit(_cuda(X), _cuda(y), T, D, m, seed=n)
    want = oracle.forest_fit(X, y, T, D, m, seed=n)
    assert fo.num_trees == T
    for t in range(T):
        g, o = fo.tree(t).nodes, want[t]
        assert len(g) == len(o)
        for f in ("feature", "left", "threshold", "n_samples", "value", "depth"):
            assert np.array_equal(g[f], o[f]), (t, f)
    Xq, _ = datagen.random_table(n + 1, 5000, d, kind=kind, int_y=True)
    yh = dt.dt_forest_predict(fo, _cuda(Xq)).cpu().numpy()
    assert np.array_equal(yh, oracle.forest_predict(want, Xq))


def test_forest_real_mode_contract(dt):
    X, y = datagen.random_table(3, 20000, 6, kind="continuous", int_y=False)
    T = 3
    fo = dt.dt_forest_fit(_cuda(X), _cuda(y), T, 10, 2, seed=9)
    want = oracle.forest_fit(X, y, T, 10, 2, seed=9)
    for t in range(T):
        idx = oracle.bootstrap(9, t, len(X))
        treecmp.compare(fo.tree(t).nodes, want[t], X[idx], y[idx])
    Xq, _ = datagen.random_table(4, 7000, 6, kind="continuous", int_y=False)
    yh = dt.dt_forest_predict(fo, _cuda(Xq)).cpu().numpy()
    assert np.array_equal(yh, oracle.forest_predict([fo.tree(t).nodes for t in range(T)], Xq))


def test_forest_c2_schema(dt):
    """The bench's forest workload shape (configs[1] schema, depth 12) at 200k rows."""
    X, y = datagen.cnn_gpu_table(1, 200_000)
    T = 2
    fo = dt.dt_forest_fit(_cuda(X), _cuda(y), T, 12, 1, seed=1)
    want = oracle.forest_fit(X, y, T, 12, 1, seed=1)
    ev = 0
    for t in range(T):
        assert fo.tree(t).nodes.tobytes() == want[t].tobytes() or all(
            np.array_equal(fo.tree(t).nodes[f], want[t][f]) for f in ("feature", "threshold", "left", "value"))
        ev += fo.tree(t).split_evals
    assert fo.split_evals == ev
    Xv, _ = datagen.cnn_gpu_table(2, 50_000)
    assert np.array_equal(dt.dt_forest_predict(fo, _cuda(Xv)).cpu().numpy(), oracle.forest_predict(want, Xv))


def test_forest_rejects_bad_args(dt):
    X, y = datagen.random_table(1, 100, 3, kind="ties", int_y=True)
    with pytest.raises(dt.DTError):
        dt.dt_forest_fit(_cuda(X), _cuda(y), 0)
    fo = dt.dt_forest_fit(_cuda(X), _cuda(y), 1)
    with pytest.raises(dt.DTError):
        dt.dt_forest_predict(fo, _cuda(np.zeros((4, 2), np.float32)))


def test_forest_scratch_reuse_across_shapes(dt):
    """The bootstrap scratch is cached across dt_forest_fit calls (csrc/forest.cu): the
    same forest again, a different shape in between, and after dt_release_workspace all
    give the oracle's trees (integer mode, bit-exact)."""
    tabs = {n: datagen.random_table(n, n, 6, kind="mixed", int_y=True) for n in (4000, 2500)}
    want = {n: oracle.forest_fit(X, y, 2, 6, 2, seed=3) for n, (X, y) in tabs.items()}
    for step, n in enumerate((4000, 4000, 2500, 4000, "release", 2500)):
        if n == "release":
            dt.dt_release_workspace()
            continue
        X, y = tabs[n]
        fo = dt.dt_forest_fit(_cuda(X), _cuda(y), 2, 6, 2, seed=3)
        for t in range(2):
            g, o = fo.tree(t).nodes, want[n][t]
            assert len(g) == len(o), (step, t)
            for f in ("feature", "left", "threshold", "n_samples", "value"):
                assert np.array_equal(g[f], o[f]), (step, t, f)
