"""C-ABI boundary checks that need no GPU: the library loads, exports every symbol that
include/dt.h declares, the node layout matches, and host-side validation rejects bad
arguments before any launch (SURVEY 8(b) conventions)."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "dt.h")


def _declared():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dt_[a-z_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def dt():
    import paper_conf_ipps_metzgd23_b200 as m
    return m


def test_every_declared_symbol_is_exported(dt):
    names = _declared()
    assert len(names) >= 16
    lib = ctypes.CDLL(dt.LIB_PATH)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    assert set(dt.SYMBOLS) == set(names)  # the binding declares every entry point


def test_node_layout_matches_oracle(dt):
    import oracle
    assert dt.NODE_DTYPE.itemsize == 48
    assert dt.NODE_DTYPE == oracle.NODE_DTYPE
    src = open(HDR).read()
    assert "int32_t feature;" in src and "int64_t n_samples;" in src


def test_built_for_sm100a(dt):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", dt.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version(dt):
    assert "sm_100a" in dt.version()


def test_host_validation_without_gpu(dt):
    lib = dt._lib
    h = ctypes.c_void_p()
    P = ctypes.c_void_p
    # NULL pointers / bad sizes are rejected before any CUDA call
    assert lib.dt_fit(None, None, 10, 4, 3, 1, None, ctypes.byref(h)) == 1
    assert lib.dt_fit(P(16), P(16), 0, 4, 3, 1, None, ctypes.byref(h)) == 1
    assert lib.dt_fit(P(16), P(16), 10, 0, 3, 1, None, ctypes.byref(h)) == 1
    assert lib.dt_fit(P(16), P(16), 10, 256, 3, 1, None, ctypes.byref(h)) == 1
    assert lib.dt_fit(P(16), P(16), 10, 4, -2, 1, None, ctypes.byref(h)) == 1
    assert lib.dt_fit(P(16), P(16), 10, 4, 3, 0, None, ctypes.byref(h)) == 1
    assert lib.dt_fit(P(16), P(16), 1 << 32, 4, 3, 1, None, ctypes.byref(h)) == 6
    assert b"min_samples_leaf" in lib.dt_last_error() or lib.dt_last_error()
    assert lib.dt_predict(None, P(16), 10, 4, P(16), None) == 1
    m = dt.dt_metrics()
    assert lib.dt_eval(P(16), P(16), 0, 1, None, ctypes.byref(m)) == 1
    assert lib.dt_eval(P(16), P(16), 10, -1, None, ctypes.byref(m)) == 1
    assert lib.dt_loo(P(16), P(16), 65, 4, -1, 1, P(16), None) == 6
    assert lib.dt_loo(P(16), P(16), 1, 4, -1, 1, P(16), None) == 1
    assert lib.dt_gen_table(0, 0, 10, 8, 0, 16, 8, 1.0, P(16), None, None) == 1
    # next rows: forest, KNN, factored DSE, sharded eval
    assert lib.dt_forest_fit(P(16), P(16), 10, 4, 0, 3, 1, 0, None, ctypes.byref(h)) == 1
    assert lib.dt_forest_fit(None, P(16), 10, 4, 2, 3, 1, 0, None, ctypes.byref(h)) == 1
    assert lib.dt_forest_predict(None, P(16), 10, 4, P(16), None) == 1
    assert lib.dt_bootstrap(0, -1, 10, P(16), None) == 1
    assert lib.dt_bootstrap(0, 0, 1 << 32, P(16), None) == 6
    assert lib.dt_knn_predict(P(16), P(16), 10, 4, P(16), 5, 11, P(16), None) == 1
    assert lib.dt_knn_predict(P(16), P(16), 10, 4, P(16), 5, 0, P(16), None) == 1
    assert lib.dt_knn_predict(P(16), P(16), 1 << 32, 4, P(16), 5, 3, P(16), None) == 6
    src = (ctypes.c_int32 * 4)(0, 1, -1, -2)
    assert lib.dt_predict_dse(None, P(16), 2, 2, P(16), 2, 2, src, P(16), None) == 1
    assert lib.dt_eval_sharded(None, P(16), P(16), 10, 1, None, ctypes.byref(m)) == 1


def test_tree_from_nodes_rejects_bad_links(dt):
    nodes = np.zeros(3, dtype=dt.NODE_DTYPE)
    nodes["feature"] = [0, -1, -1]
    nodes["left"] = [1, -1, -1]
    nodes["right"] = [2, -1, -1]
    nodes["depth"] = [0, 1, 1]
    bad = nodes.copy()
    bad["right"][0] = 1  # right != left + 1
    h = ctypes.c_void_p()
    assert dt._lib.dt_tree_from_nodes(bad.ctypes.data, 3, 4, ctypes.byref(h)) == 1
    bad = nodes.copy()
    bad["feature"][0] = 4  # feature >= d
    assert dt._lib.dt_tree_from_nodes(bad.ctypes.data, 3, 4, ctypes.byref(h)) == 1
    bad = nodes.copy()
    bad["depth"][2] = 2
    assert dt._lib.dt_tree_from_nodes(bad.ctypes.data, 3, 4, ctypes.byref(h)) == 1
    bad = nodes.copy()
    bad["threshold"][0] = np.nan
    assert dt._lib.dt_tree_from_nodes(bad.ctypes.data, 3, 4, ctypes.byref(h)) == 2


def test_oracle_not_imported_by_product():
    """The product package must not import or link the oracle (boundary)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_metzgd23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in txt.replace("no CPU fallback", ""), f


def test_product_fails_loudly_without_library(tmp_path):
    """No CPU fallback: loading the binding from a path without libdt.so raises."""
    import importlib.util
    import shutil
    import subprocess
    import sys
    pkg = tmp_path / "paper_conf_ipps_metzgd23_b200"
    pkg.mkdir()
    src = os.path.join(ROOT, "paper_conf_ipps_metzgd23_b200", "__init__.py")
    shutil.copy(src, pkg / "__init__.py")
    r = subprocess.run([sys.executable, "-c", "import paper_conf_ipps_metzgd23_b200"], cwd=tmp_path,
                       capture_output=True, text=True)
    assert r.returncode != 0 and "not built" in r.stderr
    assert importlib.util.find_spec("oracle") is not None  # the oracle stays test infrastructure

