"""B200-native exact CART (Metz, Goli & Drechsler, IPDPS'23 -- the Decision-Tree
performance model): thin Python binding over the C ABI of ``libdt.so``
(``include/dt.h``).

Argument marshalling only: every step runs in the CUDA kernels of ``libdt.so``.  Tensors
are torch CUDA tensors (X float32 n x d row-major contiguous, y float64); the work is
enqueued on torch's current stream.  There is no CPU fallback: importing this package
without a built ``libdt.so`` raises, and every call raises ``DTError`` on failure.

Names follow the C ABI: ``dt_fit``, ``dt_predict``, ``dt_eval``, ``dt_predict_eval``,
``dt_loo``, ``dt_gen_table``, ``dt_gen_dse``; ``Tree`` wraps ``dt_tree*``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DT_LIB_PATH") or os.path.join(_HERE, "libdt.so")

NODE_DTYPE = np.dtype([
    ("feature", "<i4"), ("left", "<i4"), ("right", "<i4"), ("depth", "<i4"),
    ("threshold", "<f8"), ("value", "<f8"), ("impurity", "<f8"), ("n_samples", "<i8"),
])

STATUS = {0: "DT_OK", 1: "DT_ERR_INVALID_ARG", 2: "DT_ERR_NONFINITE", 3: "DT_ERR_OOM",
          4: "DT_ERR_CUDA", 5: "DT_ERR_NCCL", 6: "DT_ERR_TOO_LARGE"}

SYMBOLS = ("dt_fit", "dt_fit_grid", "dt_tree_size", "dt_tree_nodes", "dt_tree_depth", "dt_tree_num_features",
           "dt_tree_split_evals", "dt_tree_from_nodes", "dt_tree_free", "dt_predict", "dt_eval",
           "dt_predict_eval", "dt_loo", "dt_gen_table", "dt_gen_dse", "dt_last_error",
           "dt_version", "dt_profile_enable", "dt_profile_reset", "dt_launch_count",
           "dt_profile_kinds", "dt_profile_get", "dt_comm_unique_id_bytes", "dt_comm_unique_id",
           "dt_comm_init", "dt_comm_init_local", "dt_comm_free", "dt_comm_rank", "dt_comm_world",
           "dt_fit_sharded", "dt_eval_sharded", "dt_tree_truncate", "dt_predict_eval_depths",
           "dt_importances", "dt_release_workspace", "dt_predict_dse", "dt_forest_fit",
           "dt_forest_num_trees", "dt_forest_tree", "dt_forest_split_evals", "dt_forest_predict",
           "dt_forest_free", "dt_bootstrap", "dt_knn_predict")


class DTError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class dt_metrics(ctypes.Structure):
    _fields_ = [("mape", ctypes.c_double), ("r2", ctypes.c_double), ("adj_r2", ctypes.c_double),
                ("n", ctypes.c_int64), ("p", ctypes.c_int32)]


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libdt.so and declare the C signatures.  Raises if the library is missing."""
    if not os.path.exists(path):
        raise ImportError(f"{path} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(path)
    P, I64, I32, U64, D = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double
    sig = {
        "dt_fit": ([P, P, I64, I32, I32, I64, P, ctypes.POINTER(P)], ctypes.c_int),
        "dt_fit_grid": ([P, P, I64, I32, I32, P, I32, P, P], ctypes.c_int),
        "dt_tree_size": ([P], I64),
        "dt_tree_nodes": ([P], P),
        "dt_tree_depth": ([P], I32),
        "dt_tree_num_features": ([P], I32),
        "dt_tree_split_evals": ([P], I64),
        "dt_tree_from_nodes": ([P, I64, I32, ctypes.POINTER(P)], ctypes.c_int),
        "dt_tree_free": ([P], None),
        "dt_predict": ([P, P, I64, I32, P, P], ctypes.c_int),
        "dt_eval": ([P, P, I64, I32, P, ctypes.POINTER(dt_metrics)], ctypes.c_int),
        "dt_predict_eval": ([P, P, P, I64, I32, I32, P, ctypes.POINTER(dt_metrics)], ctypes.c_int),
        "dt_loo": ([P, P, I64, I32, I32, I64, P, P], ctypes.c_int),
        "dt_gen_table": ([U64, I64, I64, I32, I32, I32, I32, D, P, P, P], ctypes.c_int),
        "dt_gen_dse": ([U64, I64, I64, I32, P, P], ctypes.c_int),
        "dt_last_error": ([], ctypes.c_char_p),
        "dt_version": ([], ctypes.c_char_p),
        "dt_profile_enable": ([ctypes.c_int], None),
        "dt_profile_reset": ([], None),
        "dt_launch_count": ([], I64),
        "dt_profile_kinds": ([], I32),
        "dt_profile_get": ([I32, ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(I64),
                            ctypes.POINTER(D), ctypes.POINTER(D)], ctypes.c_int),
        "dt_comm_unique_id_bytes": ([], I32),
        "dt_comm_unique_id": ([P], ctypes.c_int),
        "dt_comm_init": ([P, I32, I32, I32, ctypes.POINTER(P)], ctypes.c_int),
        "dt_comm_init_local": ([I32, P], ctypes.c_int),
        "dt_comm_free": ([P], None),
        "dt_comm_rank": ([P], I32),
        "dt_comm_world": ([P], I32),
        "dt_fit_sharded": ([P, P, P, I64, I64, I64, I32, I32, I64, P, ctypes.POINTER(P)], ctypes.c_int),
        "dt_tree_truncate": ([P, I32, ctypes.POINTER(P)], ctypes.c_int),
        "dt_predict_eval_depths": ([P, P, P, I64, I32, I32, P, P], ctypes.c_int),
        "dt_importances": ([P, P, P], ctypes.c_int),
        "dt_release_workspace": ([], ctypes.c_int),
        "dt_predict_dse": ([P, P, I64, I32, P, I64, I32, P, P, P], ctypes.c_int),
        "dt_forest_fit": ([P, P, I64, I32, I32, I32, I64, U64, P, ctypes.POINTER(P)], ctypes.c_int),
        "dt_forest_num_trees": ([P], I32),
        "dt_forest_tree": ([P, I32], P),
        "dt_forest_split_evals": ([P], I64),
        "dt_forest_predict": ([P, P, I64, I32, P, P], ctypes.c_int),
        "dt_forest_free": ([P], None),
        "dt_bootstrap": ([U64, I32, I64, P, P], ctypes.c_int),
        "dt_knn_predict": ([P, P, I64, I32, P, I64, I32, P, P], ctypes.c_int),
        "dt_eval_sharded": ([P, P, P, I64, I32, P, ctypes.POINTER(dt_metrics)], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = res
    return lib


_lib = load_library()


def _check(st: int):
    if st != 0:
        raise DTError(st, _lib.dt_last_error().decode())


def _stream(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dev(t, dtype, ndim, name):
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA torch.Tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if t.dim() != ndim or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous {ndim}-D tensor")
    return ctypes.c_void_p(t.data_ptr())


def _same(*pairs):
    """Argument checks before any device work: every tensor on one device, and every
    (name, actual, expected) length equal.  A short output or label vector would make
    the kernels read or write past its allocation."""
    devs = {t.device for t in pairs[0] if t is not None}
    if len(devs) > 1:
        raise ValueError(f"tensors on different devices: {sorted(map(str, devs))}")
    for name, got, want in pairs[1:]:
        if got != want:
            raise ValueError(f"{name} has {got} elements, expected {want}")


class Tree:
    """Owns a ``dt_tree*`` (or borrows one from its ``owner``, e.g. a Forest).  ``nodes``
    is a numpy structured copy (BFS, 48 B/node)."""

    def __init__(self, handle: ctypes.c_void_p, owner=None):
        self._h = handle
        self._owner = owner

    @property
    def handle(self):
        return self._h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and getattr(self, "_owner", None) is None and _lib is not None:
            _lib.dt_tree_free(h)
        self._h = None

    @property
    def size(self) -> int:
        return int(_lib.dt_tree_size(self._h))

    @property
    def depth(self) -> int:
        return int(_lib.dt_tree_depth(self._h))

    @property
    def num_features(self) -> int:
        return int(_lib.dt_tree_num_features(self._h))

    @property
    def split_evals(self) -> int:
        return int(_lib.dt_tree_split_evals(self._h))

    @property
    def nodes(self) -> np.ndarray:
        n = self.size
        ptr = _lib.dt_tree_nodes(self._h)
        buf = (ctypes.c_char * (n * NODE_DTYPE.itemsize)).from_address(ptr)
        return np.frombuffer(bytes(buf), dtype=NODE_DTYPE).copy()


def dt_fit(X, y, max_depth: int = -1, min_samples_leaf: int = 1, stream=None) -> Tree:
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    yp = _dev(y, torch.float64, 1, "y")
    n, d = X.shape
    _same((X, y), ("y", y.shape[0], n))
    h = ctypes.c_void_p()
    _check(_lib.dt_fit(xp, yp, n, d, max_depth, min_samples_leaf, _stream(stream), ctypes.byref(h)))
    return Tree(h)


def dt_fit_grid(X, y, max_depth: int, min_samples_leafs, stream=None):
    """[dt_fit(X, y, max_depth, m) for m in min_samples_leafs] from ONE presort (include/dt.h)."""
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    yp = _dev(y, torch.float64, 1, "y")
    n, d = X.shape
    _same((X, y), ("y", y.shape[0], n))
    ms = (ctypes.c_int64 * len(min_samples_leafs))(*[int(m) for m in min_samples_leafs])
    hs = (ctypes.c_void_p * len(min_samples_leafs))()
    _check(_lib.dt_fit_grid(xp, yp, n, d, max_depth, ms, len(min_samples_leafs), _stream(stream), hs))
    return [Tree(ctypes.c_void_p(h)) for h in hs]


def dt_tree_from_nodes(nodes: np.ndarray, d: int) -> Tree:
    nodes = np.ascontiguousarray(nodes).astype(NODE_DTYPE, copy=False)
    h = ctypes.c_void_p()
    _check(_lib.dt_tree_from_nodes(nodes.ctypes.data, len(nodes), d, ctypes.byref(h)))
    return Tree(h)


def dt_predict(tree: Tree, X, out=None, stream=None):
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    n, d = X.shape
    if out is None:
        out = torch.empty(n, dtype=torch.float64, device=X.device)
    op = _dev(out, torch.float64, 1, "out")
    _same((X, out), ("out", out.shape[0], n))
    _check(_lib.dt_predict(tree.handle, xp, n, d, op, _stream(stream)))
    return out


def dt_predict_dse(tree: Tree, cnn, gpu, feature_src, out=None, stream=None):
    """Factored DSE predict (include/dt.h): yhat[i * n_gpu + j] = prediction of CNN row i
    composed with GPU row j; feature_src[f] = CNN column c >= 0 or -1 - GPU column."""
    import torch
    n_cnn, dc = cnn.shape
    n_gpu, dg = gpu.shape
    src = (ctypes.c_int32 * len(feature_src))(*[int(v) for v in feature_src])
    if len(feature_src) != tree.num_features:
        raise ValueError("feature_src needs one entry per tree feature")
    if out is None:
        out = torch.empty(n_cnn * n_gpu, dtype=torch.float64, device=cnn.device)
    _same((cnn, gpu, out), ("out", out.numel(), n_cnn * n_gpu))
    _check(_lib.dt_predict_dse(tree.handle, _dev(cnn, torch.float32, 2, "cnn"), n_cnn, dc,
                               _dev(gpu, torch.float32, 2, "gpu"), n_gpu, dg, src,
                               _dev(out, torch.float64, 1, "out"), _stream(stream)))
    return out


def _metrics(m: dt_metrics):
    return dict(mape=m.mape, r2=m.r2, adj_r2=m.adj_r2, n=m.n, p=m.p)


def dt_eval(y, yhat, p: int, stream=None) -> dict:
    import torch
    yp = _dev(y, torch.float64, 1, "y")
    hp = _dev(yhat, torch.float64, 1, "yhat")
    _same((y, yhat), ("yhat", yhat.shape[0], y.shape[0]))
    m = dt_metrics()
    _check(_lib.dt_eval(yp, hp, y.shape[0], p, _stream(stream), ctypes.byref(m)))
    return _metrics(m)


def dt_predict_eval(tree: Tree, X, y, p: int, stream=None) -> dict:
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    yp = _dev(y, torch.float64, 1, "y")
    _same((X, y), ("y", y.shape[0], X.shape[0]))
    m = dt_metrics()
    _check(_lib.dt_predict_eval(tree.handle, xp, yp, X.shape[0], X.shape[1], p, _stream(stream),
                                ctypes.byref(m)))
    return _metrics(m)


def dt_loo(X, y, max_depth: int = -1, min_samples_leaf: int = 1, out=None, stream=None):
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    yp = _dev(y, torch.float64, 1, "y")
    n, d = X.shape
    if out is None:
        out = torch.empty(n, dtype=torch.float64, device=X.device)
    op = _dev(out, torch.float64, 1, "out")
    _same((X, y, out), ("y", y.shape[0], n), ("out", out.shape[0], n))
    _check(_lib.dt_loo(xp, yp, n, d, max_depth, min_samples_leaf, op, _stream(stream)))
    return out


def dt_gen_table(seed: int, n: int, d: int = 16, real: bool = False, row0: int = 0,
                 cnn_pool_bits: int = 16, gpu_pool_bits: int = 8, unit_us: float = 1.0,
                 with_y: bool = True, device="cuda", stream=None):
    import torch
    X = torch.empty((n, d), dtype=torch.float32, device=device)
    y = torch.empty(n, dtype=torch.float64, device=device) if with_y else None
    _check(_lib.dt_gen_table(seed, row0, n, d, int(real), cnn_pool_bits, gpu_pool_bits, unit_us,
                             ctypes.c_void_p(X.data_ptr()),
                             ctypes.c_void_p(y.data_ptr() if y is not None else 0), _stream(stream)))
    return X, y


def dt_gen_dse(seed: int, row0: int, n: int, gpu_bits: int = 10, out=None, device="cuda",
               stream=None):
    import torch
    if out is None:
        out = torch.empty((n, 16), dtype=torch.float32, device=device)
    if not out.is_cuda or out.dtype != torch.float32 or not out.is_contiguous():
        raise TypeError("out must be a contiguous float32 CUDA tensor")
    _same((out,), ("out", out.numel(), n * 16))
    _check(_lib.dt_gen_dse(seed, row0, n, gpu_bits, ctypes.c_void_p(out.data_ptr()), _stream(stream)))
    return out


def dt_profile_enable(on: bool = True, graph: bool = False):
    """Measurement hooks (include/dt.h): graph=True keeps dt_fit's CUDA-graph replay and
    times its kernel groups with event-record nodes inside the graph."""
    _lib.dt_profile_enable((2 if graph else 1) if on else 0)


def dt_profile_reset():
    _lib.dt_profile_reset()


def dt_launch_count() -> int:
    return int(_lib.dt_launch_count())


def dt_profile() -> dict:
    """{kind: dict(launches, ms, alg_bytes)} for every kind with >= 1 recorded launch."""
    out = {}
    for k in range(int(_lib.dt_profile_kinds())):
        name = ctypes.c_char_p()
        cnt = ctypes.c_int64()
        ms = ctypes.c_double()
        by = ctypes.c_double()
        _check(_lib.dt_profile_get(k, ctypes.byref(name), ctypes.byref(cnt), ctypes.byref(ms),
                                   ctypes.byref(by)))
        if cnt.value:
            out[name.value.decode()] = dict(launches=int(cnt.value), ms=float(ms.value),
                                            alg_bytes=float(by.value))
    return out


def dt_tree_truncate(tree: Tree, depth: int) -> Tree:
    h = ctypes.c_void_p()
    _check(_lib.dt_tree_truncate(tree.handle, depth, ctypes.byref(h)))
    return Tree(h)


def dt_predict_eval_depths(tree: Tree, X, y, p: int, stream=None):
    """[(mape, r2, adj_r2)] for every truncation depth 0..tree.depth, one pass."""
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    yp = _dev(y, torch.float64, 1, "y")
    _same((X, y), ("y", y.shape[0], X.shape[0]))
    out = np.empty(3 * (tree.depth + 1), dtype=np.float64)
    _check(_lib.dt_predict_eval_depths(tree.handle, xp, yp, X.shape[0], X.shape[1], p,
                                       _stream(stream), out.ctypes.data))
    return [tuple(out[3 * i:3 * i + 3]) for i in range(tree.depth + 1)]


def dt_importances(tree: Tree, stream=None) -> np.ndarray:
    out = np.empty(tree.num_features, dtype=np.float64)
    _check(_lib.dt_importances(tree.handle, out.ctypes.data, _stream(stream)))
    return out


def grid_search(X, y, Xv, yv, depths, min_leafs, p=None, stream=None, rank=0, world=1, gather=None):
    """(max_depth x min_samples_leaf) grid with held-out evaluation (BASELINE configs[4]):
    dt_fit_grid (one presort, one deep fit at max(depths) per m), then
    dt_predict_eval_depths -- every (D, m) tree is a truncation of the deep one.  Returns {(D, m): (mape, r2, adj_r2)} and the split evals
    actually performed.

    Multi-GPU ("LOO / grid"): with ``world`` ranks each fits the m values
    ``min_leafs[rank::world]`` on its own GPU (data replicated) and ``gather(obj)`` --
    e.g. a torch.distributed all_gather_object wrapper returning the list of every rank's
    object -- merges the per-fit results, so every rank returns the whole grid."""
    p = X.shape[1] if p is None else p
    dmax = max(depths)
    out, evals = {}, 0
    mine = list(min_leafs)[rank::world]
    trees = dt_fit_grid(X, y, dmax, mine, stream=stream) if mine else []
    for m, t in zip(mine, trees):
        evals += t.split_evals
        per = dt_predict_eval_depths(t, Xv, yv, p, stream=stream)
        for D in depths:
            out[(D, m)] = per[min(D, t.depth)]
    if world > 1:
        parts = gather((out, evals))
        out, evals = {}, 0
        for o, e in parts:
            out.update(o)
            evals += e
    return out, evals


class Comm:
    """Owns a ``dt_comm*`` (one rank of a row-sharded fit)."""

    def __init__(self, handle: ctypes.c_void_p):
        self._h = handle

    @property
    def handle(self):
        return self._h

    @property
    def rank(self) -> int:
        return int(_lib.dt_comm_rank(self._h))

    @property
    def world(self) -> int:
        return int(_lib.dt_comm_world(self._h))

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.dt_comm_free(h)
            self._h = None


def dt_comm_init_nccl(rank: int, world: int, broadcast, device: int = None) -> Comm:
    """NCCL communicator on CUDA device ``device`` (default: the current one);
    ``broadcast(obj)`` must return rank 0's object on every rank (e.g. a
    torch.distributed broadcast_object_list wrapper)."""
    if device is None:
        import torch
        device = torch.cuda.current_device()
    nb = int(_lib.dt_comm_unique_id_bytes())
    uid = (ctypes.c_char * nb)()
    if rank == 0:
        _check(_lib.dt_comm_unique_id(uid))
    raw = broadcast(bytes(uid) if rank == 0 else None)
    uid = (ctypes.c_char * nb).from_buffer_copy(raw)
    h = ctypes.c_void_p()
    _check(_lib.dt_comm_init(uid, rank, world, int(device), ctypes.byref(h)))
    return Comm(h)


def dt_comm_init_local(world: int):
    """``world`` communicators for host threads of this process (single-GPU sharding)."""
    arr = (ctypes.c_void_p * world)()
    _check(_lib.dt_comm_init_local(world, arr))
    return [Comm(ctypes.c_void_p(arr[i])) for i in range(world)]


def dt_fit_sharded(comm: Comm, X_local, y_local, row_offset: int, n_global: int, max_depth: int = -1,
                   min_samples_leaf: int = 1, stream=None) -> Tree:
    """Value-range row-sharded fit (include/dt.h): this rank's rows row_offset ..
    row_offset + n_local - 1 of the n_global-row table; every rank returns the same tree."""
    import torch
    n, d = X_local.shape
    _same((X_local, y_local), ("y_local", y_local.shape[0], n))
    xp = _dev(X_local, torch.float32, 2, "X_local") if n else ctypes.c_void_p(0)
    yp = _dev(y_local, torch.float64, 1, "y_local") if n else ctypes.c_void_p(0)
    h = ctypes.c_void_p()
    _check(_lib.dt_fit_sharded(comm.handle, xp, yp, n, row_offset, n_global, d, max_depth, min_samples_leaf,
                               _stream(stream), ctypes.byref(h)))
    return Tree(h)


class Forest:
    """Owns a ``dt_forest*`` (bagged CART, include/dt.h)."""

    def __init__(self, handle: ctypes.c_void_p):
        self._h = handle

    @property
    def handle(self):
        return self._h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:
            _lib.dt_forest_free(h)
        self._h = None

    @property
    def num_trees(self) -> int:
        return int(_lib.dt_forest_num_trees(self._h))

    @property
    def split_evals(self) -> int:
        return int(_lib.dt_forest_split_evals(self._h))

    def tree(self, t: int) -> Tree:
        p = _lib.dt_forest_tree(self._h, t)
        if not p:
            raise IndexError(t)
        return Tree(ctypes.c_void_p(p), owner=self)


def dt_forest_fit(X, y, n_trees: int, max_depth: int = -1, min_samples_leaf: int = 1,
                  seed: int = 0, stream=None) -> Forest:
    import torch
    xp = _dev(X, torch.float32, 2, "X")
    yp = _dev(y, torch.float64, 1, "y")
    n, d = X.shape
    _same((X, y), ("y", y.shape[0], n))
    h = ctypes.c_void_p()
    _check(_lib.dt_forest_fit(xp, yp, n, d, n_trees, max_depth, min_samples_leaf,
                              ctypes.c_uint64(seed), _stream(stream), ctypes.byref(h)))
    return Forest(h)


def dt_forest_predict(forest: Forest, X, out=None, stream=None):
    import torch
    n, d = X.shape
    if out is None:
        out = torch.empty(n, dtype=torch.float64, device=X.device)
    _same((X, out), ("out", out.shape[0], n))
    _check(_lib.dt_forest_predict(forest.handle, _dev(X, torch.float32, 2, "X"), n, d,
                                  _dev(out, torch.float64, 1, "out"), _stream(stream)))
    return out


def dt_bootstrap(seed: int, tree: int, n: int, device="cuda", stream=None):
    import torch
    out = torch.empty(n, dtype=torch.int32, device=device)  # u32 bits
    _check(_lib.dt_bootstrap(ctypes.c_uint64(seed), tree, n, ctypes.c_void_p(out.data_ptr()),
                             _stream(stream)))
    return out


def dt_knn_predict(Xtr, ytr, Xq, k: int = 5, out=None, stream=None):
    """KNN regression (include/dt.h dt_knn_predict)."""
    import torch
    ntr, d = Xtr.shape
    nq = Xq.shape[0]
    if Xq.shape[1] != d:
        raise ValueError("Xq must have the training rows' d columns")
    if out is None:
        out = torch.empty(nq, dtype=torch.float64, device=Xq.device)
    _same((Xtr, ytr, Xq, out), ("ytr", ytr.shape[0], ntr), ("out", out.shape[0], nq))
    _check(_lib.dt_knn_predict(_dev(Xtr, torch.float32, 2, "Xtr"), _dev(ytr, torch.float64, 1, "ytr"), ntr, d,
                               _dev(Xq, torch.float32, 2, "Xq"), nq, k, _dev(out, torch.float64, 1, "out"),
                               _stream(stream)))
    return out


def dt_release_workspace():
    """Free the cached fit plan and trim the device memory pool (include/dt.h)."""
    _check(_lib.dt_release_workspace())


def dt_eval_sharded(comm: "Comm", y, yhat, p: int, stream=None) -> dict:
    """Metrics of rows split over the ranks (include/dt.h); same result on every rank."""
    import torch
    m = dt_metrics()
    n = y.shape[0]
    _same((y, yhat), ("yhat", yhat.shape[0], n))
    yp = _dev(y, torch.float64, 1, "y") if n else ctypes.c_void_p(0)
    hp = _dev(yhat, torch.float64, 1, "yhat") if n else ctypes.c_void_p(0)
    _check(_lib.dt_eval_sharded(comm.handle, yp, hp, n, p, _stream(stream), ctypes.byref(m)))
    return _metrics(m)


def version() -> str:
    return _lib.dt_version().decode()
