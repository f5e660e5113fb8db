"""Seeded synthetic graphs shaped like the paper's workloads.

Input infrastructure only — no part of the PCGCN method lives here.  Every
generator returns an undirected graph as a symmetric CSR over vertex ids
``0..n-1`` with int64 ``rowptr`` and int32 ``col`` (sources ascending per row),
no duplicate edges and no self-loops.  (The planner and the oracle both still
accept duplicates / self-loops / asymmetric input and handle them themselves.)

Model: a nested degree-corrected SBM.  Vertices (in *generation order*) are
grouped into classes, each class split into sub-communities.  Edge number ``e``
draws, from the counter-based stream of ``synth.rng``:
  * ``u`` with probability proportional to an integer propensity ``w[u]``;
  * a level: sub-community of ``u`` (prob ``p_sub``), class of ``u``
    (``p_class``) or the whole graph (rest);
  * ``v`` proportional to ``w`` inside that level's range.
Self-pairs are dropped, duplicates collapse.  Generation-order vertices are
then relabelled by a seeded random permutation, so locality is hidden from the
partitioner.  The edge count is made exact: counters are added until at least
``m_target`` distinct edges exist, then a seeded hash-ranked subset of the
surplus is dropped (never the sorted tail — SURVEY.md §8(d) pitfall).

The O(m) part has a bit-identical multithreaded C++ twin (``csrc/synth_gen.cpp``)
used for the large configurations; the tests check the two agree.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

from . import rng as R

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "_synth_gen.so")


@dataclass
class Graph:
    n: int
    rowptr: np.ndarray  # int64 [n+1]
    col: np.ndarray  # int32 [nnz]
    labels: np.ndarray | None = None  # int32 [n] class of each vertex
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])


@dataclass
class SBMSpec:
    """Nested DC-SBM recipe.  ``class_sizes`` sum to n."""

    class_sizes: list
    sub_size: int  # target sub-community size (0 => one sub per class)
    p_sub: float
    p_class: float
    m_target: int  # undirected edges (without self-loops)
    alpha: float = 2.5  # Pareto tail exponent of the propensities
    cap: float = 200.0  # propensity cap, as a multiple of the minimum
    seed: int = 0
    class_weight: list | None = None  # per-class propensity (tiered SBM); replaces the Pareto draw

    @property
    def n(self) -> int:
        return int(sum(self.class_sizes))


def _split_sizes(total: int, parts: int) -> np.ndarray:
    q, r = divmod(total, parts)
    return np.array([q + 1] * r + [q] * (parts - r), dtype=np.int64)


def _structure(spec: SBMSpec):
    """Per-vertex arrays in generation order (O(n), numpy only)."""
    n = spec.n
    class_sizes = np.asarray(spec.class_sizes, dtype=np.int64)
    class_start = np.concatenate([[0], np.cumsum(class_sizes)]).astype(np.int64)
    sub_sizes = []
    for cs in class_sizes:
        ns = 1 if spec.sub_size <= 0 else max(1, int(round(cs / spec.sub_size)))
        sub_sizes.append(_split_sizes(int(cs), ns))
    sub_sizes = np.concatenate(sub_sizes)
    sub_start = np.concatenate([[0], np.cumsum(sub_sizes)]).astype(np.int64)
    class_of = np.repeat(np.arange(len(class_sizes), dtype=np.int32), class_sizes)
    sub_of = np.repeat(np.arange(len(sub_sizes), dtype=np.int32), sub_sizes)
    if spec.class_weight is not None:
        x = np.asarray(spec.class_weight, dtype=np.float64)[class_of]
    else:
        g = np.random.default_rng([spec.seed, 1])
        u = g.random(n)
        x = np.minimum((1.0 - u) ** (-1.0 / (spec.alpha - 1.0)), spec.cap)
    w = np.maximum(1, np.rint(x * 64.0)).astype(np.int64)
    cdf = np.concatenate([[0], np.cumsum(w)]).astype(np.int64)
    id_of = np.random.default_rng([spec.seed, 2]).permutation(n).astype(np.int64)
    return dict(n=n, cdf=cdf, class_of=class_of, class_start=class_start,
                sub_of=sub_of, sub_start=sub_start, id_of=id_of)


def _edge_keys_np(st, spec: SBMSpec, c0: int, c1: int) -> np.ndarray:
    """Canonical keys min(a,b)*n+max(a,b) of edges for counters [c0, c1)."""
    n = st["n"]
    cdf = st["cdf"]
    key = R.stream_key(spec.seed, 7)
    ctr = np.arange(c0, c1, dtype=np.uint64)
    d0 = R.draws(key, ctr * np.uint64(3))
    d1 = R.draws(key, ctr * np.uint64(3) + np.uint64(1))
    d2 = R.draws(key, ctr * np.uint64(3) + np.uint64(2))
    lvl = R.to_unit(d0)
    W = np.uint64(cdf[-1])
    gu = np.searchsorted(cdf, (d1 % W).astype(np.int64), side="right") - 1
    sub = st["sub_of"][gu]
    cls = st["class_of"][gu]
    lo = np.zeros_like(gu)
    hi = np.full_like(gu, n)
    m_sub = lvl < spec.p_sub
    m_cls = (~m_sub) & (lvl < spec.p_sub + spec.p_class)
    lo[m_sub] = st["sub_start"][sub[m_sub]]
    hi[m_sub] = st["sub_start"][sub[m_sub] + 1]
    lo[m_cls] = st["class_start"][cls[m_cls]]
    hi[m_cls] = st["class_start"][cls[m_cls] + 1]
    base = cdf[lo]
    span = (cdf[hi] - base).astype(np.uint64)
    gv = np.searchsorted(cdf, base + (d2 % span).astype(np.int64), side="right") - 1
    ok = gu != gv
    a = st["id_of"][gu[ok]]
    b = st["id_of"][gv[ok]]
    lo_id = np.minimum(a, b).astype(np.uint64)
    hi_id = np.maximum(a, b).astype(np.uint64)
    return lo_id * np.uint64(n) + hi_id


def _drop_surplus(keys: np.ndarray, target: int, seed: int) -> np.ndarray:
    if len(keys) <= target:
        return keys
    dk = R.stream_key(seed, 11)
    with np.errstate(over="ignore"):
        h = R.mix64(keys ^ dk)
    order = np.lexsort((keys, h))
    return np.sort(keys[order[:target]])


def _keys_to_csr(n: int, keys: np.ndarray):
    a = (keys // np.uint64(n)).astype(np.int64)
    b = (keys % np.uint64(n)).astype(np.int64)
    src = np.concatenate([a, b])
    dst = np.concatenate([b, a])
    order = np.lexsort((dst, src))
    src = src[order]
    dst = dst[order]
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(src, minlength=n), out=rowptr[1:])
    return rowptr, dst.astype(np.int32)


def _load_lib():
    if not os.path.exists(_LIB_PATH):
        return None
    lib = ctypes.CDLL(_LIB_PATH)
    lib.synth_sbm_csr.restype = ctypes.c_int64
    return lib


def sbm(spec: SBMSpec, impl: str = "auto") -> Graph:
    """Generate the nested DC-SBM graph of ``spec`` (exactly m_target edges)."""
    st = _structure(spec)
    n = st["n"]
    if impl == "auto":
        impl = "c" if (spec.m_target > 2_000_000 and _load_lib() is not None) else "np"
    if impl == "c":
        rowptr, col = _sbm_c(st, spec)
    else:
        m_gen = spec.m_target
        while True:
            keys = np.unique(_edge_keys_np(st, spec, 0, m_gen))
            if len(keys) >= spec.m_target:
                break
            m_gen = m_gen + ((spec.m_target - len(keys)) * 5) // 4 + 64
        keys = _drop_surplus(keys, spec.m_target, spec.seed)
        rowptr, col = _keys_to_csr(n, keys)
    labels = np.empty(n, dtype=np.int32)
    labels[st["id_of"]] = st["class_of"]
    return Graph(n=n, rowptr=rowptr, col=col, labels=labels,
                 meta=dict(kind="nested-dcsbm", m_undirected=spec.m_target, seed=spec.seed))


def _sbm_c(st, spec: SBMSpec):
    lib = _load_lib()
    if lib is None:
        raise RuntimeError("synth/_synth_gen.so not built (run __graft_entry__.build())")
    n = st["n"]
    P = ctypes.c_void_p
    arrs = {k: np.ascontiguousarray(st[k]) for k in
            ("cdf", "class_of", "class_start", "sub_of", "sub_start", "id_of")}
    rowptr = np.empty(n + 1, dtype=np.int64)
    col = np.empty(2 * spec.m_target, dtype=np.int32)
    rc = lib.synth_sbm_csr(
        ctypes.c_int64(n), P(arrs["cdf"].ctypes.data), P(arrs["class_of"].ctypes.data),
        P(arrs["class_start"].ctypes.data), P(arrs["sub_of"].ctypes.data),
        P(arrs["sub_start"].ctypes.data), P(arrs["id_of"].ctypes.data),
        ctypes.c_double(spec.p_sub), ctypes.c_double(spec.p_class),
        ctypes.c_uint64(int(R.stream_key(spec.seed, 7))),
        ctypes.c_uint64(int(R.stream_key(spec.seed, 11))),
        ctypes.c_int64(spec.m_target), P(rowptr.ctypes.data), P(col.ctypes.data))
    if rc != spec.m_target:
        raise RuntimeError(f"synth_sbm_csr returned {rc}, expected {spec.m_target}")
    return rowptr, col


@dataclass
class RMATSpec:
    """R-MAT graph (Chakrabarti et al. 2004; the paper's synthetic family,
    PAPER.md L251, Table I): n vertices, ``m_target`` distinct
    undirected edges (density = m_target / n^2), quadrant probabilities
    (a, b, c, d = 1-a-b-c) over ceil(log2 n) levels; pairs with an endpoint
    >= n and self-pairs are redrawn, duplicates collapse; ids shuffled."""

    n: int
    m_target: int
    a: float = 0.45
    b: float = 0.22
    c: float = 0.22
    seed: int = 0


def _rmat_keys(spec: RMATSpec, c0: int, c1: int) -> np.ndarray:
    n = spec.n
    levels = max(1, int(np.ceil(np.log2(n))))
    key = R.stream_key(spec.seed, 17)
    ctr = np.arange(c0, c1, dtype=np.uint64)
    u = np.zeros(len(ctr), dtype=np.int64)
    v = np.zeros(len(ctr), dtype=np.int64)
    ab, abc = spec.a + spec.b, spec.a + spec.b + spec.c
    for lvl in range(levels):
        x = R.to_unit(R.draws(key, ctr * np.uint64(levels) + np.uint64(lvl)))
        ubit = (x >= ab).astype(np.int64)                       # quadrants c, d: lower half
        vbit = (((x >= spec.a) & (x < ab)) | (x >= abc)).astype(np.int64)  # quadrants b, d: right half
        u = (u << 1) | ubit
        v = (v << 1) | vbit
    ok = (u < n) & (v < n) & (u != v)
    perm = np.random.default_rng([spec.seed, 2]).permutation(n).astype(np.int64)
    a_, b_ = perm[u[ok]], perm[v[ok]]
    return (np.minimum(a_, b_).astype(np.uint64) * np.uint64(n) + np.maximum(a_, b_).astype(np.uint64))


def rmat(spec: RMATSpec) -> Graph:
    """R-MAT graph with exactly m_target undirected edges (seeded subset of
    the surplus dropped, as in sbm()).  Labels: 32 classes by the vertex's
    position in generation order (its leading quadrant path, R-MAT's
    recursive communities)."""
    n = spec.n
    if spec.m_target > n * (n - 1) // 2:
        raise ValueError("m_target exceeds the number of vertex pairs")
    # counters are consumed in order, batch after batch: the edge set after c
    # counters does not depend on the batch sizes
    seen = np.zeros(n * n, dtype=bool)  # pair bitmap (n = 10,240: 105 MB)
    have, c = 0, 0
    while have < spec.m_target:
        step = max(1 << 20, min(1 << 24, 2 * (spec.m_target - have)))
        seen[_rmat_keys(spec, c, c + step)] = True
        have = int(np.count_nonzero(seen))
        c += step
    keys = _drop_surplus(np.flatnonzero(seen).astype(np.uint64), spec.m_target, spec.seed)
    rowptr, col = _keys_to_csr(n, keys)
    perm = np.random.default_rng([spec.seed, 2]).permutation(n).astype(np.int64)
    levels = max(1, int(np.ceil(np.log2(n))))
    labels = np.empty(n, dtype=np.int32)
    labels[perm] = (np.arange(n, dtype=np.int64) * 32 // n).astype(np.int32)
    return Graph(n=n, rowptr=rowptr, col=col, labels=labels,
                 meta=dict(kind="rmat", m_undirected=spec.m_target, seed=spec.seed))


# ---------------------------------------------------------------------------
# Tiny hand-made graphs (test fixtures; closed forms live in the tests)
# ---------------------------------------------------------------------------

def from_edges(n: int, edges, symmetrize: bool = True, keep_dups: bool = False) -> Graph:
    """CSR from an explicit edge list.  With keep_dups, duplicates and
    self-loops are kept verbatim (to exercise the planner's cleaning)."""
    e = np.asarray(list(edges), dtype=np.int64).reshape(-1, 2)
    if symmetrize:
        e = np.concatenate([e, e[:, ::-1]])
    if not keep_dups:
        e = e[e[:, 0] != e[:, 1]]
        if len(e):
            e = np.unique(e, axis=0)
    order = np.lexsort((e[:, 1], e[:, 0])) if len(e) else np.zeros(0, dtype=np.int64)
    e = e[order]
    rowptr = np.zeros(n + 1, dtype=np.int64)
    if len(e):
        np.cumsum(np.bincount(e[:, 0], minlength=n), out=rowptr[1:])
    return Graph(n=n, rowptr=rowptr, col=e[:, 1].astype(np.int32) if len(e) else np.zeros(0, np.int32))


def path(n: int) -> Graph:
    return from_edges(n, [(i, i + 1) for i in range(n - 1)])


def cycle(n: int) -> Graph:
    return from_edges(n, [(i, (i + 1) % n) for i in range(n)])


def star(leaves: int) -> Graph:
    return from_edges(leaves + 1, [(0, i) for i in range(1, leaves + 1)])


def complete(n: int) -> Graph:
    return from_edges(n, [(i, j) for i in range(n) for j in range(i + 1, n)])


def empty(n: int) -> Graph:
    return from_edges(n, [])


def cliques(sizes, seed: int | None = None) -> Graph:
    """Disjoint cliques; ids shuffled by ``seed`` if given."""
    n = int(sum(sizes))
    ids = np.arange(n) if seed is None else np.random.default_rng(seed).permutation(n)
    edges = []
    s = 0
    for k in sizes:
        for i in range(s, s + k):
            for j in range(i + 1, s + k):
                edges.append((ids[i], ids[j]))
        s += k
    g = from_edges(n, edges)
    lab = np.empty(n, dtype=np.int32)
    s = 0
    for c, k in enumerate(sizes):
        lab[ids[s:s + k]] = c
        s += k
    g.labels = lab
    return g


def random_graph(n: int, p: float, seed: int) -> Graph:
    """Erdos-Renyi G(n, p) (may contain isolated vertices)."""
    g = np.random.default_rng(seed)
    iu = np.triu_indices(n, 1)
    m = g.random(len(iu[0])) < p
    return from_edges(n, list(zip(iu[0][m], iu[1][m])))


def messy_random(n: int, m: int, seed: int) -> Graph:
    """Symmetric graph with duplicate edges and input self-loops kept."""
    g = np.random.default_rng(seed)
    e = g.integers(0, n, size=(m, 2))
    return from_edges(n, [tuple(x) for x in e], symmetrize=True, keep_dups=True)
