"""Exact-rational brute force for CART -- TEST INFRASTRUCTURE ONLY (pins the oracle).

Everything here uses ``fractions.Fraction`` so no rounding happens anywhere except where
a value is deliberately converted to float for comparison.  It is written straight from
the *definition* of a regression tree's split criterion (CART):

    gain(S -> L, R) = SSE(S) - SSE(L) - SSE(R),   SSE(T) = sum_{r in T} (y_r - mean_T)^2

not from the closed form the oracle evaluates, so it is an independent check of the
oracle's algebra (sign, operand order, centering) and of its tie rule (Reading R4:
lowest feature, then lowest threshold).

Used only on tiny inputs (n <= ~14, d <= 3).
"""
from __future__ import annotations

from fractions import Fraction
from functools import lru_cache

import numpy as np


def sse(ys) -> Fraction:
    """Sum of squared deviations from the mean, by definition."""
    ys = [Fraction(v) for v in ys]
    if not ys:
        return Fraction(0)
    mean = sum(ys, Fraction(0)) / len(ys)
    return sum(((v - mean) ** 2 for v in ys), Fraction(0))


def mean(ys) -> Fraction:
    ys = [Fraction(v) for v in ys]
    return sum(ys, Fraction(0)) / len(ys)


def candidates(X, y, rows, min_leaf):
    """Every valid (feature, position) split of the node ``rows`` with its exact gain.

    Rows are ordered by (x_f, row id); position i puts the first i rows left.  A
    position is valid iff x[i-1] < x[i] (exact f32 compare) and both sides keep
    >= min_leaf rows.  Yields (f, i, gain, threshold, left_rows, right_rows).
    """
    X = np.asarray(X, dtype=np.float32)
    n_rows = len(rows)
    parent = sse([y[r] for r in rows])
    for f in range(X.shape[1]):
        order = sorted(rows, key=lambda r: (float(X[r, f]), r))
        for i in range(1, n_rows):
            lo, hi = X[order[i - 1], f], X[order[i], f]
            if not (lo < hi) or i < min_leaf or n_rows - i < min_leaf:
                continue
            L, R = order[:i], order[i:]
            gain = parent - sse([y[r] for r in L]) - sse([y[r] for r in R])
            thr = float(lo) / 2.0 + float(hi) / 2.0  # midpoint, Reading R5 (fp64)
            yield f, i, gain, thr, sorted(L), sorted(R)


def best_split(X, y, rows, min_leaf):
    """Exact argmax of the gain; ties -> lowest feature, then lowest position (R4)."""
    best = None
    for cand in candidates(X, y, rows, min_leaf):
        if best is None or cand[2] > best[2]:
            best = cand
    return best


def greedy_tree(X, y, max_depth=-1, min_leaf=1):
    """Exact-arithmetic greedy CART in BFS order (Readings R8, R9).

    Returns a list of dicts with feature, left, right, depth, threshold, value (Fraction),
    sse (Fraction), n, rows.
    """
    n = len(y)
    nodes = [None]
    queue = [(list(range(n)), 0, 0)]
    head = 0
    while head < len(queue):
        rows, depth, idx = queue[head]
        head += 1
        ys = [y[r] for r in rows]
        nd = dict(feature=-1, left=-1, right=-1, depth=depth, threshold=0.0,
                  value=mean(ys), sse=sse(ys), n=len(rows), rows=rows)
        nodes[idx] = nd
        if max_depth >= 0 and depth >= max_depth:
            continue
        if len(rows) < 2 * min_leaf:
            continue
        if min(ys) == max(ys):
            continue
        b = best_split(X, y, rows, min_leaf)
        if b is None:
            continue
        f, i, gain, thr, L, R = b
        li = len(nodes)
        nodes.extend([None, None])
        nd.update(feature=f, left=li, right=li + 1, threshold=thr)
        queue.append((L, depth + 1, li))
        queue.append((R, depth + 1, li + 1))
    return nodes


def tree_sse(nodes) -> Fraction:
    return sum((nd["sse"] for nd in nodes if nd["feature"] < 0), Fraction(0))


def optimal_tree_sse(X, y, max_depth, min_leaf=1):
    """min over EVERY tree of depth <= max_depth (same split validity) of the total SSE.

    opt(S, 0) = SSE(S);  opt(S, k) = min(SSE(S), min_{valid (f,i)} opt(L,k-1)+opt(R,k-1)).
    Exhaustive over all trees by recursion with memoisation on the row set.
    """
    X = np.asarray(X, dtype=np.float32)

    @lru_cache(maxsize=None)
    def opt(rows, k):
        base = sse([y[r] for r in rows])
        if k == 0:
            return base
        best = base
        for f, i, gain, thr, L, R in candidates(X, y, list(rows), min_leaf):
            v = opt(tuple(L), k - 1) + opt(tuple(R), k - 1)
            if v < best:
                best = v
        return best

    return opt(tuple(range(len(y))), max_depth)
