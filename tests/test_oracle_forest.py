"""Pins of the oracle's Random Forest (bagged CART; P:203, P:231;
Readings R20, R21) -- all CPU, "-m 'not gpu'".

* the bootstrap generator against its written definition (numpy, independent of the C
  code) and against the sampling distribution it must have (Poisson(1) counts, 1 - 1/e
  distinct rows);
* depth-0 forests against the closed form (mean over trees of the bootstrap means);
* the forest against scikit-learn: DecisionTreeRegressor grown on the same bootstrap
  samples (tie-free data) and averaged in tree order, like RandomForestRegressor does.
"""
import math

import numpy as np
import pytest

import datagen
import oracle
import treecmp
from test_oracle_props import _sklearn_nodes

M64 = (1 << 64) - 1


def _bootstrap_def(seed, t, n):
    """Reading R21, written out with Python integers."""
    out = np.empty(n, dtype=np.uint32)
    for i in range(n):
        z = (seed + 0x9E3779B97F4A7C15 * ((t << 32) + i + 1)) & M64
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
        z ^= z >> 31
        out[i] = z % n
    return out


@pytest.mark.parametrize("seed,t,n", [(0, 0, 1), (1, 0, 10), (7, 3, 1000), (2**63 + 5, 99, 777)])
def test_bootstrap_matches_definition(seed, t, n):
    assert np.array_equal(oracle.bootstrap(seed, t, n), _bootstrap_def(seed, t, n))


def test_bootstrap_distribution():
    n = 200_000
    idx = oracle.bootstrap(3, 1, n)
    counts = np.bincount(idx, minlength=n)
    # fraction of rows drawn at least once -> 1 - (1 - 1/n)^n ~ 1 - 1/e (sd ~ 0.001)
    assert abs((counts > 0).mean() - (1 - math.exp(-1))) < 0.005
    # counts ~ Poisson(1): P(k) = e^-1 / k!
    for k in range(5):
        want = math.exp(-1) / math.factorial(k)
        assert abs((counts == k).mean() - want) < 0.005, k
    # different trees draw different samples
    assert not np.array_equal(idx, oracle.bootstrap(3, 2, n))


def test_depth0_forest_is_mean_of_bootstrap_means():
    X, y = datagen.random_table(4, 500, 3, kind="ties", int_y=True)
    trees = oracle.forest_fit(X, y, 7, max_depth=0, seed=11)
    acc = 0.0
    for t in range(7):
        yb = y[_bootstrap_def(11, t, 500)]
        m = float(np.sum(yb)) / 500  # integral sums < 2^53: exact, then one rounding
        assert len(trees[t]) == 1 and trees[t]["value"][0] == m
        acc = acc + m
    yh = oracle.forest_predict(trees, X[:10])
    assert np.all(yh == acc / 7)


@pytest.mark.parametrize("seed", range(3))
def test_forest_matches_sklearn_trees_on_bootstrap_samples(seed):
    """Each tree vs sklearn's DecisionTreeRegressor on the same bootstrap sample (root
    path; exact gain ties adjudicated, treecmp) and on its in-bag rows' predictions (an
    exact tie between features induces the same in-bag partition, so those agree even
    where the two libraries picked different features); the forest = the tree-order mean
    of its trees' predictions (sklearn's RandomForestRegressor averaging)."""
    sk = pytest.importorskip("sklearn.tree")
    X, y = datagen.random_table(seed, 400, 4, kind="continuous", int_y=False)
    T, D, m = 5, 6, 2
    trees = oracle.forest_fit(X, y, T, D, m, seed=seed)
    Xq, _ = datagen.random_table(seed + 100, 300, 4, kind="continuous", int_y=False)
    acc = np.zeros(len(Xq))
    for t in range(T):
        idx = oracle.bootstrap(seed, t, len(X))
        est = sk.DecisionTreeRegressor(max_depth=D, min_samples_leaf=m, random_state=0).fit(X[idx], y[idx])
        st = treecmp.compare(trees[t], _sklearn_nodes(est), X[idx], y[idx], same_thresholds=False,
                             value_rel=1e-12, impurity=False)
        assert st["compared"] > 5
        np.testing.assert_allclose(oracle.predict(trees[t], X[idx]), est.predict(X[idx]), rtol=1e-12)
        acc = acc + oracle.predict(trees[t], Xq)
    assert np.array_equal(oracle.forest_predict(trees, Xq), acc / T)


def test_forest_single_tree_sample_is_the_tree():
    """T = 1: the forest predicts exactly what its one tree predicts."""
    X, y = datagen.random_table(9, 300, 3, kind="mixed", int_y=True)
    trees = oracle.forest_fit(X, y, 1, -1, 1, seed=5)
    assert np.array_equal(oracle.forest_predict(trees, X), oracle.predict(trees[0], X))
