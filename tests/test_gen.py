"""Generator properties (shared input module; no method arithmetic)."""
import numpy as np
import pytest

import gen


@pytest.mark.parametrize("n,nnz,seed", [(1000, 10000, 1), (20000, 100000, 2), (64, 64, 3),
                                        (50, 1001, 4)])
def test_graph_shape_exact_symmetric_selflooped(n, nnz, seed):
    g = gen.powerlaw_graph(n, nnz, gamma=2.5, n_comm=4, seed=seed)
    assert g.nnz == n + 2 * ((nnz - n) // 2)
    assert g.row_ptr[0] == 0 and g.row_ptr[-1] == g.nnz
    assert (np.diff(g.row_ind) >= 0).all()
    assert np.array_equal(np.repeat(np.arange(n), np.diff(g.row_ptr)), g.row_ind)
    key = g.row_ind.astype(np.int64) * n + g.col_ind
    assert (np.diff(key) > 0).all()                       # sorted, deduplicated
    rkey = np.sort(g.col_ind.astype(np.int64) * n + g.row_ind)
    assert np.array_equal(np.sort(key), rkey)             # symmetric
    assert (key[np.isin(key, np.arange(n) * (n + 1))].size == n)  # self-loops


def test_graph_deterministic_and_seed_sensitive():
    a = gen.powerlaw_graph(3000, 40000, seed=7)
    b = gen.powerlaw_graph(3000, 40000, seed=7)
    c = gen.powerlaw_graph(3000, 40000, seed=8)
    assert np.array_equal(a.col_ind, b.col_ind) and np.array_equal(a.val, b.val)
    assert not np.array_equal(a.col_ind, c.col_ind)


def test_gcn_values():
    g = gen.powerlaw_graph(500, 5000, seed=5, val_mode="gcn")
    d = np.diff(g.row_ptr).astype(np.float64)
    ref = (1.0 / np.sqrt(d[g.row_ind] * d[g.col_ind])).astype(np.float32)
    assert np.array_equal(g.val, ref)


def test_features_blockwise_regeneration():
    X = gen.features(3, 100, 24)
    Y = gen.features(3, 40, 24, row0=30)
    assert np.array_equal(X[30:70], Y)
    Z = gen.features(3, 100, 24, ld=32)
    assert np.array_equal(Z[:, :24], X) and not Z[:, 24:].any()
    assert np.abs(X).max() < 1 and np.abs(X).min() > 0
