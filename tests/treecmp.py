"""Tree comparison under the parity contract (BASELINE.json north_star).

* Trees are compared by ROOT PATH, not by raw BFS index.
* Where both trees split a node the same way, the children are compared recursively.
* Where they split differently, the two choices are re-scored EXACTLY (Fractions,
  definition SSE_P - SSE_L - SSE_R on the node's training rows).  The node is exempt iff
  the exact relative gap between the two gains is <= ``gap_rel`` (1e-12); otherwise the
  comparison fails.  An exempt node's subtree is not compared further.
* With ``exact_ties=True`` (integer mode) no exemption is allowed at all: the trees must
  be identical everywhere including exact ties.
* Leaf / node values must agree within ``value_rel`` relative (abs floor ``value_abs``).
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np


class TreeMismatch(AssertionError):
    pass


def _exact_gain(X, y_frac, rows, f, t):
    L = [r for r in rows if float(X[r, f]) <= t]
    R = [r for r in rows if float(X[r, f]) > t]
    if not L or not R:
        return Fraction(-1)

    def sse(rs):
        vs = [y_frac[r] for r in rs]
        mu = sum(vs, Fraction(0)) / len(vs)
        return sum(((v - mu) ** 2 for v in vs), Fraction(0))

    return sse(rows) - sse(L) - sse(R)


def compare(a, b, X, y, *, same_thresholds=True, exact_ties=False, gap_rel=1e-12,
            value_rel=1e-9, value_abs=1e-12, impurity=True):
    """Returns dict(compared=#nodes compared, exempt=#exempt nodes)."""
    X = np.asarray(X, dtype=np.float32)
    y = np.asarray(y, dtype=np.float64)
    y_frac = None
    stats = dict(compared=0, exempt=0)
    stack = [(0, 0, np.arange(len(y)))]
    while stack:
        ka, kb, rows = stack.pop()
        na, nb = a[ka], b[kb]
        stats["compared"] += 1
        where = f"node a#{ka} / b#{kb} (n={len(rows)})"
        if int(na["n_samples"]) != len(rows) or int(nb["n_samples"]) != len(rows):
            raise TreeMismatch(f"{where}: n_samples {na['n_samples']} vs {nb['n_samples']} vs rows {len(rows)}")
        if int(na["depth"]) != int(nb["depth"]):
            raise TreeMismatch(f"{where}: depth")
        for key in ("value", "impurity") if impurity else ("value",):
            va, vb = float(na[key]), float(nb[key])
            if abs(va - vb) > max(value_rel * max(abs(va), abs(vb)), value_abs):
                raise TreeMismatch(f"{where}: {key} {va!r} vs {vb!r}")
        fa, fb = int(na["feature"]), int(nb["feature"])
        if fa < 0 and fb < 0:
            continue
        if (fa < 0) != (fb < 0):
            raise TreeMismatch(f"{where}: leaf vs split (features {fa}, {fb})")
        ta, tb = float(na["threshold"]), float(nb["threshold"])
        go_a = X[rows, fa].astype(np.float64) <= ta
        go_b = X[rows, fb].astype(np.float64) <= tb
        same = fa == fb and (ta == tb if same_thresholds else bool(np.array_equal(go_a, go_b)))
        if not same:
            if exact_ties:
                raise TreeMismatch(f"{where}: split (f={fa}, t={ta!r}) vs (f={fb}, t={tb!r}) in exact mode")
            if y_frac is None:
                y_frac = [Fraction(float(v)) for v in y]
            rl = [int(r) for r in rows]
            ga = _exact_gain(X, y_frac, rl, fa, ta)
            gb = _exact_gain(X, y_frac, rl, fb, tb)
            top = max(ga, gb)
            gap = abs(ga - gb)
            if top > 0 and gap > Fraction(gap_rel) * top:
                raise TreeMismatch(f"{where}: split (f={fa}, t={ta!r}, gain={float(ga)!r}) vs "
                                   f"(f={fb}, t={tb!r}, gain={float(gb)!r}); exact rel gap "
                                   f"{float(gap / top):.3e} > {gap_rel}")
            stats["exempt"] += 1
            continue
        for ca, cb, mask in ((int(na["left"]), int(nb["left"]), go_a),
                             (int(na["right"]), int(nb["right"]), ~go_a)):
            stack.append((ca, cb, rows[mask]))
    return stats
