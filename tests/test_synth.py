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
