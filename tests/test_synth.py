"""Seeded input generators: determinism, numpy/C++ agreement, counting."""
import numpy as np
import pytest

from synth import configs as C
from synth import graphs as G


@pytest.mark.parametrize("w", [C.CORA, C.PUBMED, C.scaled(C.REDDIT, 0.01)])
def test_numpy_and_cpp_generators_agree(w):
    if G._load_lib() is None:
        pytest.skip("synth/_synth_gen.so not built")
    a = G.sbm(w.spec, impl="np")
    b = G.sbm(w.spec, impl="c")
    assert np.array_equal(a.rowptr, b.rowptr) and np.array_equal(a.col, b.col)
    assert a.nnz == 2 * w.spec.m_target


def test_symmetric_no_selfloops_no_dups():
    g = G.sbm(C.CORA.spec)
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    assert not np.any(rows == g.col)
    fwd = set(zip(rows.tolist(), g.col.tolist()))
    assert len(fwd) == g.nnz
    assert all((b, a) in fwd for a, b in fwd)


def test_train_mask_fraction_and_determinism():
    m = C.train_mask(100_000, 7)
    assert abs(m.mean() - 0.8) < 0.01
    assert np.array_equal(m, C.train_mask(100_000, 7))


@pytest.mark.parametrize("d", [0.1, 1.0])
def test_rmat_series_counts_and_determinism(d):
    """RMAT-d (Table I): 10,240 vertices, exactly round(d% * n^2)
    undirected edges (so nnz(A+I) = 2m + n = Table I's count within 2%),
    symmetric, no self-loops / duplicates, 32 labels, deterministic."""
    w = C.RMAT[d]
    g = C.graph(w)
    m = int(round(d / 100 * 10_240 ** 2))
    assert g.n == 10_240 and g.nnz == 2 * m
    table1 = {0.1: 216_700, 1.0: 2_100_000}[d]
    assert abs((g.nnz + g.n) - table1) / table1 < 0.02
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    assert not np.any(rows == g.col)
    keys = rows * g.n + g.col
    assert np.all(np.diff(keys) > 0)                       # sorted, no duplicates
    rev = np.sort(g.col.astype(np.int64) * g.n + rows)
    np.testing.assert_array_equal(rev, keys)               # symmetric
    assert set(np.unique(C.labels(w, g))) == set(range(32))
    g2 = C.graph(w)
    np.testing.assert_array_equal(g2.col, g.col)
