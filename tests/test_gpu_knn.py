"""KNN regression through the C ABI vs the oracle: predictions
bit-exact (same fp64 distance definition, same (distance, row) order, same sum order)."""
import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dt():
    import paper_conf_ipps_metzgd23_b200 as m
    return m


def _cuda(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("ntr,nq,d,k,kind", [(1, 3, 2, 1, "ties"), (60, 40, 3, 5, "ties"), (1000, 777, 4, 16, "ties"),
                                             (5000, 3000, 16, 5, "continuous"), (2049, 513, 7, 3, "mixed"),
                                             (300, 100, 32, 1, "continuous"), (4096, 257, 16, 16, "collinear")])
def test_knn_bitexact(dt, ntr, nq, d, k, kind):
    Xtr, ytr = datagen.random_table(ntr, ntr, d, kind=kind, int_y=(kind != "continuous"))
    Xq, _ = datagen.random_table(ntr + 1, nq, d, kind=kind, int_y=True)
    got = dt.dt_knn_predict(_cuda(Xtr), _cuda(ytr), _cuda(Xq), k).cpu().numpy()
    assert np.array_equal(got, oracle.knn_predict(Xtr, ytr, Xq, k))


def test_knn_paper_schema(dt):
    """The bench's KNN workload shape: configs[1] schema rows, k = 5 (sklearn default)."""
    Xtr, ytr = datagen.cnn_gpu_table(1, 20000)
    Xq, _ = datagen.cnn_gpu_table(2, 2000)
    got = dt.dt_knn_predict(_cuda(Xtr), _cuda(ytr), _cuda(Xq), 5).cpu().numpy()
    assert np.array_equal(got, oracle.knn_predict(Xtr, ytr, Xq, 5))


def test_knn_rejects_bad_args(dt):
    X, y = datagen.random_table(1, 10, 3, kind="ties", int_y=True)
    with pytest.raises(dt.DTError):
        dt.dt_knn_predict(_cuda(X), _cuda(y), _cuda(X), 11)       # k > n_train
    with pytest.raises(dt.DTError):
        dt.dt_knn_predict(_cuda(X), _cuda(y), _cuda(X), 0)
    X9, y9 = datagen.random_table(1, 40, 9, kind="ties", int_y=True)
    with pytest.raises(dt.DTError):
        dt.dt_knn_predict(_cuda(X9), _cuda(y9), _cuda(X9), 3)     # d = 9 not compiled
