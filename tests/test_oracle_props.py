"""Oracle invariants, metamorphic relations, library cross-check and metric closed forms
(all CPU, "-m 'not gpu'").  SURVEY 4, T2-T5."""
import math

import numpy as np
import pytest

import datagen
import oracle
import treecmp


def _route(nodes, X):
    """Leaf index each row lands in (plain traversal, test-local)."""
    out = np.empty(len(X), dtype=np.int64)
    for r in range(len(X)):
        k = 0
        while nodes[k]["feature"] >= 0:
            k = nodes[k]["left"] if float(X[r, nodes[k]["feature"]]) <= nodes[k]["threshold"] else nodes[k]["right"]
        out[r] = k
    return out


CASES = [(s, n, d, kind, iy) for s, (n, d, kind, iy) in enumerate([
    (200, 3, "ties", True), (300, 4, "mixed", True), (257, 5, "continuous", False),
    (150, 4, "collinear", True), (400, 2, "ties", False), (123, 6, "continuous", True)])]


@pytest.mark.parametrize("seed,n,d,kind,iy", CASES)
@pytest.mark.parametrize("D,m", [(-1, 1), (4, 3), (2, 1), (0, 1), (6, 7)])
def test_invariants(seed, n, d, kind, iy, D, m):
    X, y = datagen.random_table(seed, n, d, kind=kind, int_y=iy)
    nodes = oracle.fit(X, y, D, m)
    leaf = _route(nodes, X)
    for k, nd in enumerate(nodes):
        if nd["feature"] >= 0:
            L, R = nodes[nd["left"]], nodes[nd["right"]]
            assert nd["right"] == nd["left"] + 1                       # BFS links
            assert nd["left"] > k
            assert L["depth"] == R["depth"] == nd["depth"] + 1
            assert L["n_samples"] + R["n_samples"] == nd["n_samples"]  # n = n_L + n_R
            sse_p = nd["impurity"] * nd["n_samples"]
            sse_c = L["impurity"] * L["n_samples"] + R["impurity"] * R["n_samples"]
            assert sse_c <= sse_p * (1 + 1e-12) + 1e-12                 # child SSE <= parent
        else:
            assert nd["left"] == nd["right"] == -1
            assert nd["n_samples"] >= m or k == 0                      # min_samples_leaf
            rows = np.nonzero(leaf == k)[0]
            assert len(rows) == nd["n_samples"]                         # rows route to leaf
            mu = math.fsum(y[rows]) / len(rows)
            assert nd["value"] == pytest.approx(mu, rel=1e-14, abs=1e-14)  # value = mean
            var = math.fsum((y[rows] - mu) ** 2) / len(rows)
            assert nd["impurity"] == pytest.approx(var, rel=1e-10, abs=1e-12)
        if D >= 0:
            assert nd["depth"] <= D
    # row multiset preserved: leaves partition the rows
    assert sum(int(nd["n_samples"]) for nd in nodes if nd["feature"] < 0) == n


def test_scale_y_by_power_of_two():
    for seed in range(6):
        X, y = datagen.random_table(seed, 300, 4, kind=("ties", "continuous")[seed % 2], int_y=seed % 3 != 0)
        a = oracle.fit(X, y, 8, 2)
        for k in (-3, 5):
            b = oracle.fit(X, y * 2.0 ** k, 8, 2)
            for f in ("feature", "left", "right", "threshold", "n_samples"):
                assert np.array_equal(a[f], b[f])
            assert np.array_equal(a["value"] * 2.0 ** k, b["value"])


def test_row_permutation_integer_mode():
    """Integer mode: every sum exact, so the tree does not depend on row order."""
    for seed in range(6):
        X, y = datagen.random_table(seed, 250, 3, kind="ties", int_y=True)
        perm = np.random.default_rng(seed).permutation(len(y))
        a = oracle.fit(X, y, -1, 1)
        b = oracle.fit(X[perm], y[perm], -1, 1)
        # structure identical up to the order of tied rows, which does not enter splits
        for f in ("feature", "left", "right", "threshold", "n_samples", "value"):
            assert np.array_equal(a[f], b[f])


def test_truncation_equivalence():
    """fit(D, m) == truncate(fit(inf, m), D)."""
    X, y = datagen.random_table(3, 500, 5, kind="mixed", int_y=True)
    for m in (1, 4):
        full = oracle.fit(X, y, -1, m)
        for D in (0, 1, 3, 5):
            t = oracle.fit(X, y, D, m)
            keep = [k for k in range(len(full)) if full[k]["depth"] <= D]
            assert len(keep) == len(t)
            sub = full[keep]
            cut = sub["depth"] == D
            for f in ("n_samples", "value", "depth", "impurity"):
                assert np.array_equal(sub[f], t[f])
            assert np.array_equal(np.where(cut, 0.0, sub["threshold"]), t["threshold"])
            assert np.array_equal(np.where(cut, -1, sub["feature"]), t["feature"])
            assert np.array_equal(np.where(cut, -1, sub["left"]), t["left"])


def test_duplicate_column_lower_index():
    X, y = datagen.random_table(11, 300, 3, kind="ties", int_y=True)
    X2 = np.concatenate([X, X[:, :1]], axis=1)  # col 3 duplicates col 0
    a = oracle.fit(X2, y, -1, 1)
    assert not np.any(a["feature"] == 3)
    X3 = np.concatenate([X[:, :1], X], axis=1)  # col 0 duplicates col 1
    b = oracle.fit(X3, y, -1, 1)
    assert not np.any(b["feature"] == 1)


def test_interpolation_fully_grown():
    """D = inf, m = 1, distinct feature vectors: the tree interpolates (MAPE 0, R^2 1)."""
    X, y = datagen.random_table(5, 400, 3, kind="continuous", int_y=False)
    nodes = oracle.fit(X, y, -1, 1)
    yhat = oracle.predict(nodes, X)
    mape, r2, adj = oracle.evaluate(y, yhat, 3)
    assert mape == 0.0 and r2 == 1.0 and adj == 1.0


def _sklearn_nodes(est):
    """sklearn's pre-order tree -> our BFS node array (right = left + 1)."""
    t = est.tree_
    order, q, head = [], [0], 0
    while head < len(q):
        k = q[head]; head += 1
        order.append(k)
        if t.children_left[k] != -1:
            q += [t.children_left[k], t.children_right[k]]
    pos = {k: i for i, k in enumerate(order)}
    out = np.zeros(len(order), dtype=oracle.NODE_DTYPE)
    for i, k in enumerate(order):
        leaf = t.children_left[k] == -1
        out[i]["feature"] = -1 if leaf else t.feature[k]
        out[i]["left"] = -1 if leaf else pos[t.children_left[k]]
        out[i]["right"] = -1 if leaf else pos[t.children_right[k]]
        out[i]["threshold"] = 0.0 if leaf else t.threshold[k]
        out[i]["value"] = t.value[k].ravel()[0]
        out[i]["impurity"] = t.impurity[k]
        out[i]["n_samples"] = t.n_node_samples[k]
    for i in range(len(out)):
        if out[i]["feature"] >= 0:
            out[out[i]["left"]]["depth"] = out[i]["depth"] + 1
            out[out[i]["right"]]["depth"] = out[i]["depth"] + 1
    return out


@pytest.mark.parametrize("seed", range(4))
def test_matches_sklearn_on_tie_free_data(seed):
    """Library cross-check (T4): sklearn DecisionTreeRegressor(squared_error, best) on
    continuous tie-free data, compared by root path; where the two pick different splits
    the exact gains must tie within 1e-12 (sklearn breaks ties by a random feature order,
    skl _splitter.pyx, so an exact tie may go either way)."""
    sk = pytest.importorskip("sklearn.tree")
    X, y = datagen.random_table(seed, 600, 4, kind="continuous", int_y=False)
    for D, m in ((4, 1), (7, 5), (-1, 20), (-1, 1)):
        est = sk.DecisionTreeRegressor(criterion="squared_error", splitter="best",
                                       max_depth=None if D < 0 else D, min_samples_leaf=m,
                                       random_state=seed).fit(X, y)
        st = treecmp.compare(oracle.fit(X, y, D, m), _sklearn_nodes(est), X, y,
                             same_thresholds=False, value_rel=1e-12, impurity=False)
        assert st["compared"] > 10


# ------------------------------------------------------------------ metrics ----

def test_metric_closed_forms():
    rng = np.random.default_rng(0)
    y = rng.uniform(1, 100, 1000)
    yhat = y + rng.standard_normal(1000)
    mape, r2, adj = oracle.evaluate(y, yhat, 5)
    ybar = math.fsum(y) / len(y)
    sse = math.fsum((y - yhat) ** 2)
    sst = math.fsum((y - ybar) ** 2)
    assert r2 == pytest.approx(1 - sse / sst, rel=1e-13)
    assert adj == pytest.approx(1 - (1 - r2) * (len(y) - 1) / (len(y) - 5 - 1), rel=1e-13)
    assert mape == pytest.approx(math.fsum(np.abs(y - yhat) / np.abs(y)) / len(y), rel=1e-13)
    # perfect prediction
    assert oracle.evaluate(y, y, 5) == (0.0, 1.0, 1.0)
    # mean prediction -> R^2 = 0 exactly (SST == SSE computed the same way)
    m, r, a = oracle.evaluate(y, np.full_like(y, ybar), 5)
    assert abs(r) < 1e-15
    # SST = 0 rule (sklearn force_finite): R^2 = 1 if SSE = 0 else 0
    c = np.full(10, 3.0)
    assert oracle.evaluate(c, c, 1)[1] == 1.0
    assert oracle.evaluate(c, c + 1, 1)[1] == 0.0
    # adj undefined when n - p - 1 <= 0
    assert math.isnan(oracle.evaluate(y[:3], yhat[:3], 2)[2])
    # MAPE denominator max(|y|, eps): y = 0 rows
    z = np.zeros(4)
    assert oracle.evaluate(z, z + 1e-16, 1)[0] == pytest.approx(1e-16 / np.finfo(float).eps)


def test_metrics_match_sklearn():
    skm = pytest.importorskip("sklearn.metrics")
    rng = np.random.default_rng(1)
    y = rng.uniform(-5, 50, 777)
    yhat = y * 1.1 + rng.standard_normal(777)
    mape, r2, _ = oracle.evaluate(y, yhat, 3)
    assert mape == pytest.approx(skm.mean_absolute_percentage_error(y, yhat), rel=1e-12)
    assert r2 == pytest.approx(skm.r2_score(y, yhat), rel=1e-12)


def test_loo_matches_explicit_refits():
    X, y = datagen.paper_table(0)
    oof = oracle.loo(X, y, -1, 1)
    for i in (0, 7, 39):
        keep = np.arange(40) != i
        t = oracle.fit(X[keep], y[keep], -1, 1)
        assert oracle.predict(t, X[i:i + 1])[0] == oof[i]


def test_importances_sum_to_one_and_match_sklearn():
    sk = pytest.importorskip("sklearn.tree")
    X, y = datagen.random_table(2, 500, 4, kind="continuous", int_y=False)
    nodes = oracle.fit(X, y, 6, 10)
    imp = oracle.importances(nodes, 4)
    assert imp.sum() == pytest.approx(1.0, rel=1e-14)
    est = sk.DecisionTreeRegressor(max_depth=6, min_samples_leaf=10, random_state=0).fit(X, y)
    # only meaningful where the trees are identical (no tie decided differently)
    st = treecmp.compare(nodes, _sklearn_nodes(est), X, y, same_thresholds=False, impurity=False)
    assert st["exempt"] == 0
    assert np.allclose(imp, est.feature_importances_, rtol=1e-9, atol=1e-12)
