"""Host planner (libpcgcn.so, C++) vs the plan oracle (oracle/plan.py):
bit-exact on every exported array.  CPU only (plans built with
build_device=0), plus ABI symbol / error-path checks."""
import functools
import os
import re

import numpy as np
import pytest

from oracle import plan as PL
from synth import configs as C
from synth import graphs as G

L = pytest.importorskip("paper_conf_ipps_tianmyd20_b200._lib")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@functools.lru_cache(maxsize=None)
def _reddit_small():
    """C3's recipe at 1% (2,328 vertices, 573K edges: dense, so the numpy
    generator would loop over duplicate draws for a minute; the C++ twin is
    bit-identical, tests/test_synth.py)."""
    return C.graph(C.scaled(C.REDDIT, 0.01), impl="c")


def test_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "pcgcn.h")).read()
    names = set(re.findall(r"\b(pcgcn_[a-z0-9_]+)\s*\(", hdr))
    assert len(names) >= 20
    for nm in sorted(names):
        assert hasattr(L.lib, nm), nm


def _compare(g, P, theta, part=None, norm="sym", order="id", grain="block"):
    pl = L.Plan(g.n, g.rowptr, g.col, P, theta, part=part, build_device=False,
                norm=L.NORM_NONE if norm == "none" else L.NORM_SYM,
                order=L.ORDER_DEGREE if order == "degree" else L.ORDER_ID,
                grain=L.GRAIN_TILE if grain == "tile" else L.GRAIN_BLOCK)
    ref = PL.build(g.n, g.rowptr, g.col, P, theta, part=part, norm=norm, order=order, grain=grain)
    for name in L.X_NAMES:
        got = pl.export(name)
        exp = np.asarray(ref[name]).reshape(-1)
        if name == "sweeps":
            exp = np.array([ref["sweeps"]])
        assert got.dtype == L.X_DTYPES[L.X_NAMES.index(name)]
        if name == "r":
            assert np.array_equal(got.view(np.uint32), exp.astype(np.float32).view(np.uint32)), name
        else:
            assert np.array_equal(got, exp.astype(got.dtype)), name
    st = pl.stats()
    assert st["nnz"] == g.n + len(np.unique(np.stack([np.repeat(np.arange(g.n), np.diff(g.rowptr)), g.col], 1)
                                             [np.repeat(np.arange(g.n), np.diff(g.rowptr)) != g.col], axis=0))
    assert st["nnz_sparse"] + st["nnz_dense"] == st["nnz"]
    return pl, ref


@pytest.mark.parametrize("theta", [0.0, 0.02, 0.1, 2.0])
def test_bitexact_cora(theta):
    _compare(G.sbm(C.CORA.spec), 8, theta)


@pytest.mark.parametrize("order,grain", [("degree", "block"), ("id", "tile"), ("degree", "tile")])
@pytest.mark.parametrize("theta", [0.0, 0.03, 0.1, 0.3, 2.0])
def test_bitexact_order_and_tile_grain(theta, order, grain):
    """Vertex order DEGREE and the per-chunk (TILE) mode decision (DESIGN.md
    readings #24, #25): bit-exact vs the oracle's independent derivation."""
    _compare(G.sbm(C.CORA.spec), 8, theta, order=order, grain=grain)
    _compare(_reddit_small(), 12, theta, order=order, grain=grain)
    _compare(G.messy_random(700, 4000, 3), 5, theta, order=order, grain=grain)


@pytest.mark.parametrize("theta", [0.0, 0.05, 2.0])
def test_bitexact_pubmed_scaled(theta):
    w = C.scaled(C.PUBMED, 0.25)
    _compare(C.graph(w), 11, theta)


def test_bitexact_reddit_scaled():
    _compare(_reddit_small(), 13, 0.03)


def test_bitexact_messy_input_and_override():
    g = G.messy_random(300, 1500, 5)
    rng = np.random.default_rng(1)
    part = rng.integers(0, 7, g.n).astype(np.int32)
    _compare(g, 7, 0.05, part=part)
    _compare(g, 5, 0.3)
    _compare(g, 1, 0.0, norm="none")


def test_bitexact_cliques_dense_tiles():
    g = G.cliques([200, 130, 64, 3, 1], seed=9)
    _compare(g, 5, 0.5)
    _compare(g, 3, 0.0)


def test_deterministic_across_runs():
    g = C.graph(C.scaled(C.PUBMED, 0.2))
    a = L.Plan(g.n, g.rowptr, g.col, 9, 0.04, build_device=False)
    b = L.Plan(g.n, g.rowptr, g.col, 9, 0.04, build_device=False)
    for name in L.X_NAMES:
        assert np.array_equal(a.export(name), b.export(name))


def test_rejects_asymmetric_and_bad_args():
    g = G.from_edges(4, [(0, 1), (1, 2)], symmetrize=False)
    with pytest.raises(L.PcgcnError) as e:
        L.Plan(g.n, g.rowptr, g.col, 2, 0.1, build_device=False)
    assert e.value.code == L.ENOTSYM
    g = G.path(5)
    for P, th in ((0, 0.1), (6, 0.1), (2, -1.0)):
        with pytest.raises(L.PcgcnError) as e:
            L.Plan(g.n, g.rowptr, g.col, P, th, build_device=False)
        assert e.value.code == L.EINVAL


def test_device_plan_needs_gpu():
    """No CPU fallback: asking for device structures without a GPU fails loudly."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    g = G.path(5)
    with pytest.raises(L.PcgcnError) as e:
        L.Plan(g.n, g.rowptr, g.col, 1, 0.1, build_device=True)
    assert e.value.code == L.ECUDA


def test_shard_ranges_partition_rows():
    g = C.graph(C.scaled(C.PUBMED, 0.2))
    for world in (2, 3, 4):
        prev = 0
        for rank in range(world):
            pl = L.Plan(g.n, g.rowptr, g.col, 12, 0.05, build_device=False, rank=rank, world=world)
            st = pl.stats()
            assert st["row_lo"] == prev
            prev = st["row_hi"]
        assert prev == g.n
