"""Pins of the oracle's KNN regression (Table II P:214;
Reading R22) -- all CPU, "-m 'not gpu'".

* tie-heavy small-integer data, where every distance is exact in fp64: brute force by
  sorting (exact squared distance, row index) -- pins the neighbour set, the tie-break to
  the lower index and the order of the final sum;
* scikit-learn KNeighborsRegressor (brute force, Euclidean, uniform weights) on tie-free
  continuous data;
* special cases: k = 1 on the training rows returns their targets; k = n_train returns
  the mean of all targets.
"""
import numpy as np
import pytest

import datagen
import oracle


@pytest.mark.parametrize("seed,k", [(0, 1), (1, 3), (2, 5), (3, 17)])
def test_knn_brute_force_exact_ties(seed, k):
    rng = np.random.default_rng(seed)
    Xtr = rng.integers(0, 4, size=(60, 3)).astype(np.float32)   # many equal distances
    ytr = rng.integers(0, 1000, size=60).astype(np.float64)
    Xq = rng.integers(0, 4, size=(40, 3)).astype(np.float32)
    got = oracle.knn_predict(Xtr, ytr, Xq, k)
    for q in range(len(Xq)):
        d2 = ((Xq[q].astype(np.int64) - Xtr.astype(np.int64)) ** 2).sum(axis=1)  # exact
        order = np.lexsort((np.arange(len(Xtr)), d2))[:k]                         # (dist, index)
        s = 0.0
        for i in order:
            s = s + ytr[i]
        assert got[q] == s / k, q


@pytest.mark.parametrize("seed", range(3))
def test_knn_matches_sklearn_tie_free(seed):
    nb = pytest.importorskip("sklearn.neighbors")
    Xtr, ytr = datagen.random_table(seed, 800, 5, kind="continuous", int_y=False)
    Xq, _ = datagen.random_table(seed + 50, 300, 5, kind="continuous", int_y=False)
    for k in (1, 5, 12):
        est = nb.KNeighborsRegressor(n_neighbors=k, algorithm="brute").fit(Xtr.astype(np.float64), ytr)
        np.testing.assert_allclose(oracle.knn_predict(Xtr, ytr, Xq, k), est.predict(Xq.astype(np.float64)),
                                   rtol=1e-12)


def test_knn_special_cases():
    Xtr, ytr = datagen.random_table(7, 200, 4, kind="continuous", int_y=False)
    assert np.array_equal(oracle.knn_predict(Xtr, ytr, Xtr, 1), ytr)
    allk = oracle.knn_predict(Xtr, ytr, Xtr[:5], 200)
    np.testing.assert_allclose(allk, np.full(5, ytr.mean()), rtol=1e-12)
    with pytest.raises(ValueError):
        oracle.knn_predict(Xtr, ytr, Xtr[:2], 201)
