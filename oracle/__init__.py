"""CPU oracle for the CART hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product library
(``paper_conf_ipps_metzgd23_b200``) never imports it and shares no code with it.

``cart_oracle.c`` is the slow, obviously-correct single-threaded C implementation
(fit / predict / eval / LOO / importances); ``exact.py`` is the exact-rational brute
force that pins it.  See the header of ``cart_oracle.c`` for citations.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cart_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

NODE_DTYPE = np.dtype([
    ("feature", "<i4"), ("left", "<i4"), ("right", "<i4"), ("depth", "<i4"),
    ("threshold", "<f8"), ("value", "<f8"), ("impurity", "<f8"), ("n_samples", "<i8"),
])
assert NODE_DTYPE.itemsize == 48


def build() -> str:
    """Compile the oracle (gcc, -O2 -ffp-contract=off, no fast-math) if stale."""
    if (not os.path.exists(_LIB)) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                               "-shared", "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        lib.oracle_fit.argtypes = [P, P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                   ctypes.c_int64, ctypes.POINTER(P),
                                   ctypes.POINTER(ctypes.c_int64),
                                   ctypes.POINTER(ctypes.c_int32),
                                   ctypes.POINTER(ctypes.c_int64)]
        lib.oracle_fit.restype = ctypes.c_int
        lib.oracle_free.argtypes = [P]
        lib.oracle_predict.argtypes = [P, ctypes.c_int64, P, ctypes.c_int64, ctypes.c_int32, P]
        lib.oracle_eval.argtypes = [P, P, ctypes.c_int64, ctypes.c_int32, P]
        lib.oracle_loo.argtypes = [P, P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                   ctypes.c_int64, P]
        lib.oracle_loo.restype = ctypes.c_int
        lib.oracle_importances.argtypes = [P, ctypes.c_int64, ctypes.c_int32, P]
        lib.oracle_knn.argtypes = [P, P, ctypes.c_int64, ctypes.c_int32, P, ctypes.c_int64,
                                   ctypes.c_int32, P]
        lib.oracle_bootstrap.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int64, P]
        lib.oracle_forest_predict.argtypes = [P, P, ctypes.c_int32, P, ctypes.c_int64,
                                              ctypes.c_int32, P]
        _lib = lib
    return _lib


class OracleError(RuntimeError):
    pass


def _f32(X):
    X = np.ascontiguousarray(X, dtype=np.float32)
    if X.ndim != 2:
        raise ValueError("X must be 2-D (n x d)")
    return X


def _f64(y):
    return np.ascontiguousarray(y, dtype=np.float64)


def fit(X, y, max_depth: int = -1, min_samples_leaf: int = 1, return_mode: bool = False,
        return_evals: bool = False):
    """Greedy CART regression fit; returns a structured node array (BFS, 48 B/node).

    With ``return_mode`` / ``return_evals`` also returns the integer-mode flag and the
    split-eval count (sum over searched nodes of N*d, the headline numerator).
    """
    lib = _load()
    X = _f32(X)
    y = _f64(y)
    n, d = X.shape
    if y.shape != (n,):
        raise ValueError("y must have shape (n,)")
    out = ctypes.c_void_p()
    cnt = ctypes.c_int64()
    mode = ctypes.c_int32()
    evals = ctypes.c_int64()
    st = lib.oracle_fit(X.ctypes.data, y.ctypes.data, n, d, max_depth, min_samples_leaf,
                        ctypes.byref(out), ctypes.byref(cnt), ctypes.byref(mode),
                        ctypes.byref(evals))
    if st != 0:
        raise OracleError(f"oracle_fit status {st}")
    buf = (ctypes.c_char * (cnt.value * 48)).from_address(out.value)
    nodes = np.frombuffer(bytes(buf), dtype=NODE_DTYPE).copy()
    lib.oracle_free(out)
    res = (nodes,)
    if return_mode:
        res += (bool(mode.value),)
    if return_evals:
        res += (int(evals.value),)
    return res if len(res) > 1 else nodes


def predict(nodes, X):
    lib = _load()
    X = _f32(X)
    nodes = np.ascontiguousarray(nodes, dtype=NODE_DTYPE)
    yhat = np.empty(X.shape[0], dtype=np.float64)
    lib.oracle_predict(nodes.ctypes.data, len(nodes), X.ctypes.data, X.shape[0], X.shape[1],
                       yhat.ctypes.data)
    return yhat


def evaluate(y, yhat, p: int):
    """Returns (mape_fraction, r2, adj_r2)."""
    lib = _load()
    y = _f64(y)
    yhat = _f64(yhat)
    out = np.empty(3, dtype=np.float64)
    lib.oracle_eval(y.ctypes.data, yhat.ctypes.data, len(y), p, out.ctypes.data)
    return float(out[0]), float(out[1]), float(out[2])


def loo(X, y, max_depth: int = -1, min_samples_leaf: int = 1):
    """Leave-one-out out-of-fold predictions."""
    lib = _load()
    X = _f32(X)
    y = _f64(y)
    yhat = np.empty(X.shape[0], dtype=np.float64)
    st = lib.oracle_loo(X.ctypes.data, y.ctypes.data, X.shape[0], X.shape[1], max_depth,
                        min_samples_leaf, yhat.ctypes.data)
    if st != 0:
        raise OracleError(f"oracle_loo status {st}")
    return yhat


def importances(nodes, d: int):
    lib = _load()
    nodes = np.ascontiguousarray(nodes, dtype=NODE_DTYPE)
    imp = np.empty(d, dtype=np.float64)
    lib.oracle_importances(nodes.ctypes.data, len(nodes), d, imp.ctypes.data)
    return imp


# ------------------------------------------------------------ random forest (NEXT-2) ----

def bootstrap(seed: int, t: int, n: int):
    """Row indices of tree t's bootstrap sample (n draws with replacement, Reading R21)."""
    lib = _load()
    idx = np.empty(n, dtype=np.uint32)
    lib.oracle_bootstrap(ctypes.c_uint64(seed), t, n, idx.ctypes.data)
    return idx


def forest_fit(X, y, n_trees: int, max_depth: int = -1, min_samples_leaf: int = 1, seed: int = 0):
    """Bagged CART (Reading R20): tree t = fit on (X[idx_t], y[idx_t])."""
    X = _f32(X)
    y = _f64(y)
    trees = []
    for t in range(n_trees):
        idx = bootstrap(seed, t, X.shape[0])
        trees.append(fit(X[idx], y[idx], max_depth, min_samples_leaf))
    return trees


def forest_predict(trees, X):
    """Mean of the trees' predictions, summed in tree order, divided by T."""
    lib = _load()
    X = _f32(X)
    arrs = [np.ascontiguousarray(t, dtype=NODE_DTYPE) for t in trees]
    ptrs = (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])
    counts = np.array([len(a) for a in arrs], dtype=np.int64)
    yhat = np.empty(X.shape[0], dtype=np.float64)
    lib.oracle_forest_predict(ptrs, counts.ctypes.data, len(arrs), X.ctypes.data, X.shape[0],
                              X.shape[1], yhat.ctypes.data)
    return yhat


# ------------------------------------------------------------- KNN regression (NEXT-4) ----

def knn_predict(Xtr, ytr, Xq, k: int = 5):
    """KNN regression (Table II; Reading R22): mean y of the k nearest training rows
    by fp64 squared Euclidean distance (fma-accumulated in feature order), ties to the
    lower training row index."""
    lib = _load()
    Xtr = _f32(Xtr)
    ytr = _f64(ytr)
    Xq = _f32(Xq)
    if not (1 <= k <= Xtr.shape[0]):
        raise ValueError("need 1 <= k <= n_train")
    yhat = np.empty(Xq.shape[0], dtype=np.float64)
    lib.oracle_knn(Xtr.ctypes.data, ytr.ctypes.data, Xtr.shape[0], Xtr.shape[1], Xq.ctypes.data,
                   Xq.shape[0], k, yhat.ctypes.data)
    return yhat

