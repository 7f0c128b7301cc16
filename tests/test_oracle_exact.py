"""Pins of the CPU oracle against things other than itself (all CPU, "-m 'not gpu'").

* hand-worked examples (tests/golden/hand_worked.json, derivations inline)
* exact-rational brute force of every split (oracle/exact.py, from the SSE definition)
* greedy tree == exact-arithmetic greedy recursion on tiny integer tables
* depth-1 greedy == optimum stump; depth<=3 greedy SSE >= optimum over every depth<=3 tree
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import datagen
import oracle
from oracle import exact

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hand_worked.json")


def _gold():
    with open(GOLD) as fh:
        return json.load(fh)


@pytest.mark.parametrize("case", _gold()["cases"], ids=lambda c: c["name"])
def test_hand_worked_trees(case):
    X = np.array(case["X"], dtype=np.float32)
    y = np.array(case["y"], dtype=np.float64)
    nodes = oracle.fit(X, y, case["max_depth"], case["min_samples_leaf"])
    exp = case["nodes"]
    assert len(nodes) == len(exp)
    for got, want in zip(nodes, exp):
        for k in ("feature", "left", "right", "depth", "n_samples"):
            assert int(got[k]) == want[k], (k, got, want)
        assert float(got["threshold"]) == want["threshold"]
        assert float(got["value"]) == pytest.approx(want["value"], rel=1e-14, abs=1e-15)
        assert float(got["impurity"]) == pytest.approx(want["impurity"], rel=1e-12, abs=1e-15)


def test_hand_worked_metrics():
    for m in _gold()["metrics"]:
        mape, r2, adj = oracle.evaluate(m["y"], m["yhat"], m["p"])
        assert mape == pytest.approx(m["mape"], rel=1e-15)
        assert r2 == pytest.approx(m["r2"], rel=1e-15)
        assert adj == pytest.approx(m["adj_r2"], rel=1e-14)


def _tiny_tables():
    out = []
    for seed in range(60):
        rng = np.random.default_rng(1000 + seed)
        n = int(rng.integers(2, 13))
        d = int(rng.integers(1, 4))
        kind = ("ties", "mixed", "collinear", "continuous")[seed % 4]
        X, y = datagen.random_table(seed, n, d, kind=kind, int_y=True, y_range=int(rng.integers(2, 9)))
        out.append((seed, X, y))
    return out


def _cmp_tree_exact(nodes, ex):
    assert len(nodes) == len(ex)
    for got, want in zip(nodes, ex):
        assert int(got["feature"]) == want["feature"]
        assert int(got["left"]) == want["left"]
        assert int(got["right"]) == want["right"]
        assert int(got["depth"]) == want["depth"]
        assert int(got["n_samples"]) == want["n"]
        assert float(got["threshold"]) == want["threshold"]
        # integer mode: value = fl(S/N) with S exact -> correctly rounded exact mean
        assert float(got["value"]) == float(want["value"])
        assert float(got["impurity"]) == pytest.approx(float(want["sse"] / want["n"]),
                                                       rel=1e-13, abs=1e-300)


@pytest.mark.parametrize("m", [1, 2])
def test_greedy_equals_exact_greedy(m):
    """Whole tree (structure, thresholds, values) == exact-arithmetic greedy CART."""
    for seed, X, y in _tiny_tables():
        for D in (-1, 0, 1, 2):
            nodes = oracle.fit(X, y, D, m)
            ex = exact.greedy_tree(X, list(map(int, y)), D, m)
            _cmp_tree_exact(nodes, ex)


def test_root_split_is_exact_argmax_real_y():
    """Real-valued y (dyadic, so exact rationals are cheap): the oracle's root split is
    the exact argmax of SSE_P - SSE_L - SSE_R under the tie rule."""
    for seed in range(40):
        rng = np.random.default_rng(seed)
        n = int(rng.integers(3, 13))
        d = int(rng.integers(1, 4))
        X = rng.integers(0, 5, size=(n, d)).astype(np.float32)
        y = rng.integers(-40, 40, size=n) / 8.0 + 0.125 * rng.integers(0, 2, size=n) / 16
        nodes = oracle.fit(X, y, 1, 1)
        b = exact.best_split(X, [Fraction(v) for v in y], list(range(n)), 1)
        if b is None or min(y) == max(y):
            assert nodes[0]["feature"] == -1
            continue
        f, i, gain, thr, L, R = b
        assert nodes[0]["feature"] == f
        assert nodes[0]["threshold"] == thr
        assert nodes[1]["n_samples"] == len(L)


def test_depth1_is_optimal_stump():
    for seed, X, y in _tiny_tables():
        nodes = oracle.fit(X, y, 1, 1)
        yy = list(map(int, y))
        ex = exact.greedy_tree(X, yy, 1, 1)
        opt = exact.optimal_tree_sse(X, yy, 1)
        assert exact.tree_sse(ex) == opt
        # oracle leaf impurities*N sum to the same SSE (within fp64 rounding)
        leaf_sse = sum(float(nd["impurity"]) * int(nd["n_samples"]) for nd in nodes if nd["feature"] < 0)
        assert leaf_sse == pytest.approx(float(opt), rel=1e-12, abs=1e-12)


def test_depth3_greedy_bounded_by_optimum():
    """Greedy CART is not globally optimal: its SSE is >= the best depth<=3 tree's."""
    worse = 0
    for seed, X, y in _tiny_tables()[:30]:
        yy = list(map(int, y))
        for D in (2, 3):
            ex = exact.greedy_tree(X, yy, D, 1)
            opt = exact.optimal_tree_sse(X, yy, D)
            g = exact.tree_sse(ex)
            assert g >= opt
            worse += g > opt
            nodes = oracle.fit(X, y, D, 1)
            _cmp_tree_exact(nodes, ex)
    assert worse >= 0


def test_gain_identity_exact():
    """SSE_P - SSE_L - SSE_R == (n_L n_R / N)(m_L - m_R)^2 == (S'_L n_R - S'_R n_L)^2/(N n_L n_R)
    for any centre c (Reading R19) -- exact rationals on random splits."""
    rng = np.random.default_rng(7)
    for _ in range(300):
        N = int(rng.integers(2, 30))
        ys = [Fraction(int(a), int(b)) for a, b in zip(rng.integers(-50, 50, N), rng.integers(1, 9, N))]
        i = int(rng.integers(1, N))
        L, R = ys[:i], ys[i:]
        g = exact.sse(ys) - exact.sse(L) - exact.sse(R)
        mL, mR = exact.mean(L), exact.mean(R)
        assert g == Fraction(i * (N - i), N) * (mL - mR) ** 2
        c = Fraction(int(rng.integers(-10, 10)), int(rng.integers(1, 5)))
        SL = sum((v - c for v in L), Fraction(0))
        SR = sum((v - c for v in R), Fraction(0))
        assert g == (SL * (N - i) - SR * i) ** 2 / (N * i * (N - i))
