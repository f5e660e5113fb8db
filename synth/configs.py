"""The BASELINE.json workloads as seeded synthetic recipes.

Input infrastructure only.  Sizes follow the paper's counting convention
(Table I): nnz(A+I) = 2*m + n.
  C1 Cora-shaped   n=2,708   m=5,278       1433 -> 16 -> 7    P=8
  C2 Pubmed-shaped n=19,717  m=44,324      500  -> 16 -> 3    P=32  (nnz 108,365 = Table I)
  C3 Reddit-shaped n=232,965 m=57,307,946  602  -> 128 -> 41  P=128
  C4 SBM-4M        n=4,194,304 m=~398M     128  -> 128 -> 32  P=2048
  C5 PL-32M        n=33,554,432 m=500M     128  -> 128 -> 32  P=16384
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from . import rng as R
from .graphs import Graph, RMATSpec, SBMSpec, rmat, sbm


@dataclass
class Workload:
    name: str
    spec: SBMSpec
    f_in: int
    hidden: int
    classes: int
    P: int
    feat_kind: str  # "binary" | "tfidf" | "normal"
    feat_seed: int
    theta_seed: int


def _zipf_sizes(n: int, k: int, s: float) -> list:
    w = (np.arange(1, k + 1, dtype=np.float64)) ** (-s)
    raw = w / w.sum() * n
    base = np.floor(raw).astype(np.int64)
    rem = n - int(base.sum())
    order = np.argsort(-(raw - base), kind="stable")
    base[order[:rem]] += 1
    return [int(x) for x in base]


CORA = Workload(
    "cora", SBMSpec([351, 217, 418, 818, 426, 298, 180], sub_size=64, p_sub=0.60, p_class=0.20,
                    m_target=5_278, alpha=2.5, cap=125.0, seed=1001),
    f_in=1433, hidden=16, classes=7, P=8, feat_kind="binary", feat_seed=1002, theta_seed=1003)

PUBMED = Workload(
    "pubmed", SBMSpec([4_103, 7_739, 7_875], sub_size=128, p_sub=0.60, p_class=0.20,
                      m_target=44_324, alpha=2.5, cap=110.0, seed=2001),
    f_in=500, hidden=16, classes=3, P=32, feat_kind="tfidf", feat_seed=2002, theta_seed=2003)

REDDIT = Workload(
    "reddit", SBMSpec(_zipf_sizes(232_965, 41, 0.8), sub_size=0, p_sub=0.0, p_class=0.75,
                      m_target=57_307_946, alpha=2.5, cap=200.0, seed=3001),
    f_in=602, hidden=128, classes=41, P=128, feat_kind="normal", feat_seed=3002, theta_seed=3003)

# C4: 256 communities of 16,384 in 4 tiers x 64 with intra degree d_in in
# {8, 32, 128, 512} (intra block density 0.05%..3.1%) + 10% inter-community
# edges: the dual-mode threshold sweep graph.
_C4_TIERS = [8.0] * 64 + [32.0] * 64 + [128.0] * 64 + [512.0] * 64
SBM4M = Workload(
    "sbm4m", SBMSpec([16_384] * 256, sub_size=0, p_sub=0.0, p_class=0.9,
                     m_target=int(round(64 * 16_384 * (8 + 32 + 128 + 512) / 2 / 0.9)), seed=4001,
                     class_weight=[t / 8.0 for t in _C4_TIERS]),
    f_in=128, hidden=128, classes=32, P=2048, feat_kind="normal", feat_seed=4002, theta_seed=4003)

# C5: clustered power-law graph (BASELINE configs[4]): a degree-corrected SBM
# with 4,096 communities of 8,192 vertices, 90% of edge draws inside the
# community, Pareto(2.2) propensities (degree tail exponent ~2.2) capped at
# 16,000x the minimum, 500M undirected edges -> nnz(A+I) = 1.034 B, average
# degree ~30.  Hubs saturate their community (duplicate
# draws collapse), so the largest degrees are ~10^4, not the 10^5 cap.
PL32M = Workload(
    "pl32m", SBMSpec([8_192] * 4_096, sub_size=0, p_sub=0.0, p_class=0.9, m_target=500_000_000,
                     alpha=2.2, cap=16_000.0, seed=5001),
    f_in=128, hidden=128, classes=32, P=16384, feat_kind="normal", feat_seed=5002, theta_seed=5003)

# C5's recipe at test size (sharded-path tests): 256 communities of 128 vertices,
# 90% of draws inside the community, Pareto(2.2) propensities, 250K edges.
PL_SMALL = Workload(
    "pl-small", SBMSpec([128] * 256, sub_size=0, p_sub=0.0, p_class=0.9, m_target=250_000,
                        alpha=2.2, cap=1_000.0, seed=5101),
    f_in=128, hidden=128, classes=32, P=64, feat_kind="normal", feat_seed=5102, theta_seed=5103)

# RMAT-{0.1,0.5,1,5,10}: the paper's synthetic density series (L251, Table I
# L223-L227: 10,240 vertices, density = m / n^2, 128 features, 32 labels),
# regenerated for the Table III (L263-L281) sel / full / hybrid replica.  The
# model is this repo's 2-layer GCN with the paper's hid = 64 (L255).
RMAT = {d: Workload(f"rmat-{d:g}", RMATSpec(10_240, int(round(d / 100 * 10_240 ** 2)), seed=6001 + i),
                    f_in=128, hidden=64, classes=32, P=16, feat_kind="normal", feat_seed=6101 + i,
                    theta_seed=6201 + i)
        for i, d in enumerate((0.1, 0.5, 1.0, 5.0, 10.0))}

WORKLOADS = {w.name: w for w in (CORA, PUBMED, REDDIT, SBM4M, PL32M, PL_SMALL, *RMAT.values())}


def labels(w: Workload, g: Graph) -> np.ndarray:
    """Vertex labels in [0, classes): the planted community modulo the class
    count (C4 / C5 have more communities than classes)."""
    return (g.labels % w.classes).astype(np.int32)


def scaled(w: Workload, frac: float, name: str | None = None) -> Workload:
    """Same recipe at a fraction of the vertices and edges (test sizes)."""
    sizes = [max(2, int(round(c * frac))) for c in w.spec.class_sizes]
    spec = SBMSpec(sizes, w.spec.sub_size, w.spec.p_sub, w.spec.p_class,
                   max(1, int(round(w.spec.m_target * frac))), w.spec.alpha, w.spec.cap, w.spec.seed,
                   w.spec.class_weight)
    return Workload(name or f"{w.name}@{frac}", spec, w.f_in, w.hidden, w.classes,
                    max(1, int(round(w.P * frac ** 0.5))), w.feat_kind, w.feat_seed, w.theta_seed)


def _cache_key(w: Workload) -> str:
    """Workload recipe + generator source digest: a cache entry written by
    another generator version is never read back."""
    import hashlib
    import os
    h = hashlib.sha1(repr(w.spec).encode())
    d = os.path.dirname(os.path.abspath(__file__))
    for f in ("graphs.py", "rng.py", os.path.join("csrc", "synth_gen.cpp")):
        p = os.path.join(d, f)
        if os.path.exists(p):
            h.update(open(p, "rb").read())
    return f"{w.name}-{h.hexdigest()[:16]}"


def graph(w: Workload, impl: str = "auto") -> Graph:
    """The workload's graph.  PCGCN_GRAPH_CACHE=<dir> (benchmark scripts only)
    keeps generated graphs as .npy files so one GPU job can reuse a C5-sized
    graph across several processes instead of regenerating it (minutes)."""
    import os
    cdir = os.environ.get("PCGCN_GRAPH_CACHE")
    if cdir:
        base = os.path.join(cdir, _cache_key(w))
        if os.path.exists(base + ".done"):
            lab = np.load(base + ".labels.npy") if os.path.exists(base + ".labels.npy") else None
            return Graph(int(np.load(base + ".rowptr.npy", mmap_mode="r").shape[0] - 1),
                         np.load(base + ".rowptr.npy"), np.load(base + ".col.npy"), lab, {"cached": base})
    g = rmat(w.spec) if isinstance(w.spec, RMATSpec) else sbm(w.spec, impl=impl)
    if cdir:
        os.makedirs(cdir, exist_ok=True)
        np.save(base + ".rowptr.npy", g.rowptr)
        np.save(base + ".col.npy", g.col)
        if g.labels is not None:
            np.save(base + ".labels.npy", g.labels)
        open(base + ".done", "w").close()
    return g


def features(w: Workload, n: int) -> np.ndarray:
    """X [n x f_in] float32, row i belongs to vertex id i."""
    g = np.random.default_rng([w.feat_seed, 0])
    if w.feat_kind == "binary":
        return (g.random((n, w.f_in), dtype=np.float32) < 0.0127).astype(np.float32)
    if w.feat_kind == "tfidf":
        idf = g.uniform(0.5, 3.0, size=w.f_in).astype(np.float32)
        mask = g.random((n, w.f_in), dtype=np.float32) < 0.10
        return (mask * g.random((n, w.f_in), dtype=np.float32) * idf).astype(np.float32)
    return g.standard_normal((n, w.f_in), dtype=np.float32)


def train_mask(n: int, seed: int) -> np.ndarray:
    """80% of vertices, chosen by hash(id, seed)."""
    h = R.draws(R.stream_key(seed, 13), np.arange(n, dtype=np.uint64))
    return (h % np.uint64(10)) < np.uint64(8)


def glorot(fan_in: int, fan_out: int, seed: int, idx: int) -> np.ndarray:
    a = np.sqrt(6.0 / (fan_in + fan_out))
    g = np.random.default_rng([seed, idx])
    return g.uniform(-a, a, size=(fan_in, fan_out)).astype(np.float32)


def thetas(w: Workload):
    return glorot(w.f_in, w.hidden, w.theta_seed, 0), glorot(w.hidden, w.classes, w.theta_seed, 1)
