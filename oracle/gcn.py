"""fp64 CPU oracle of PCGCN's hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this module.  It shares no code with the
CUDA path (``paper_conf_ipps_tianmyd20_b200``) and never imports it.

What it computes is the *plain definition* with no partitioning: PCGCN only
reorders a commutative/associative sum (§III-A.c, "PCGCN is equal
to the original GCN and can produce the same numerical results"), so the oracle
for the partition-centric propagation is the un-partitioned GCN layer.

  Eq. (1):   Z = D̃^-1/2 A D̃^-1/2 X Θ
  with Kipf's renormalisation Ã = A + I, d̃ = Ã·1 (reading #1 in DESIGN.md:
  the paper writes A but uses D̃ and cites [1]).
  Alg. 1, PAPER.md L101-L125 (transform, then propagate, per layer), with
  ℓ = 2 and ReLU between the layers (Kipf's model, L203; reading #14).
  Backward: not described by the paper (reading A4); derived by the chain rule,
  using Âᵀ = Â (symmetric input, reading #2).

Pins (tests/test_oracle.py): dense brute force, K_n, cycles, the P3/P4 path
worked example (tests/golden/path_graph.txt), stars, the universal eigenvector
s = sqrt(d̃), disjoint cliques, the empty graph, adjoint identity, finite
differences and torch-fp64 autograd of the same model, the uniform-logit
closed form of softmax-CE.
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp


# ---------------------------------------------------------------------------
# Graph and normalisation  (Eq. 1; readings #1-#4)
# ---------------------------------------------------------------------------

def binary_adjacency(n: int, rowptr, col) -> sp.csr_matrix:
    """A: binary, symmetric, no self-loops, duplicates collapsed (reading #3).

    Row v holds the in-neighbours of v (CSR convention of Fig. 5(a)).
    Raises ValueError if the input is not symmetric (reading #2)."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(rowptr))
    keep = rows != col
    A = sp.csr_matrix((np.ones(int(keep.sum())), (rows[keep], col[keep])), shape=(n, n))
    A.sum_duplicates()
    A.data[:] = 1.0
    if (A != A.T).nnz != 0:
        raise ValueError("input graph is not symmetric")
    A.sort_indices()
    return A


def normalized_adjacency(n: int, rowptr, col, norm: str = "sym"):
    """Return (Â, d̃, r) with Â = D̃^-1/2 (A+I) D̃^-1/2 (norm='sym') or
    Â = A + I (norm='none', used by the integer-exact pin), d̃ = 1 + deg and
    r = d̃^-1/2, all fp64."""
    A = binary_adjacency(n, rowptr, col)
    At = (A + sp.identity(n, format="csr")).tocsr()
    At.sort_indices()
    dt = np.asarray(At.sum(axis=1)).ravel()
    r = 1.0 / np.sqrt(dt)
    if norm == "none":
        return At, dt, r
    D = sp.diags(r)
    Ahat = (D @ At @ D).tocsr()
    Ahat.sort_indices()
    return Ahat, dt, r


def aggregate(Ahat: sp.csr_matrix, Y: np.ndarray) -> np.ndarray:
    """Z = Â·Y in fp64 — the propagation h_k = Σ_i f(E_{k,i}, a_i) of Alg. 1
    (L118-L121) summed over all k at once."""
    return np.asarray(Ahat @ np.asarray(Y, dtype=np.float64))


def clean_degrees(n: int, rowptr, col) -> np.ndarray:
    """deg_i = |N(i)| after dropping self-loops and duplicates (reading #3).

    Rows whose sources are strictly ascending and exclude i are already
    clean, so their degree is the row length; other rows are deduplicated
    explicitly.  (Row-chunked so a 10^9-edge graph fits in host memory.)"""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    col = np.asarray(col)
    deg = np.diff(rowptr).astype(np.int64)
    step = max(1, int(n * 32_000_000 // max(1, len(col))))
    for a in range(0, n, step):
        b = min(n, a + step)
        e0, e1 = int(rowptr[a]), int(rowptr[b])
        if e1 == e0:
            continue
        c = col[e0:e1].astype(np.int64)
        r = np.repeat(np.arange(a, b, dtype=np.int64), np.diff(rowptr[a:b + 1]))
        first = np.zeros(e1 - e0, dtype=bool)
        st = rowptr[a:b] - e0
        first[st[st < e1 - e0]] = True          # first entry of each (non-empty) row
        bad = (c == r)
        bad[1:] |= (~first[1:]) & (c[1:] <= c[:-1])
        dirty = np.unique(r[bad])
        for i in dirty:
            s = col[rowptr[i]:rowptr[i + 1]]
            deg[i] = len(np.unique(s[s != i]))
    return deg


def aggregate_rows(n: int, rowptr, col, Y: np.ndarray, rows, norm: str = "sym", deg=None) -> np.ndarray:
    """Z_i for selected rows only, straight from the edge definition
    (pin P15 at full scale): Z_i = r_i Σ_{j∈N(i)∪{i}} r_j Y_j, r = (1+deg)^-½.
    ``deg`` (optional) is clean_degrees() of the same graph, to reuse it."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    col = np.asarray(col)
    if deg is None and norm != "none":
        deg = clean_degrees(n, rowptr, col)
    out = np.zeros((len(rows), Y.shape[1]), dtype=np.float64)
    for t, i in enumerate(rows):
        s = col[rowptr[i]:rowptr[i + 1]]
        nb = np.concatenate([np.unique(s[s != i]), [i]])
        if norm == "none":
            out[t] = np.asarray(Y[nb], dtype=np.float64).sum(axis=0)
            continue
        wj = 1.0 / np.sqrt(deg[nb] + 1.0)
        ri = 1.0 / np.sqrt(deg[i] + 1.0)
        out[t] = ri * (wj[:, None] * np.asarray(Y[nb], dtype=np.float64)).sum(axis=0)
    return out


# ---------------------------------------------------------------------------
# 2-layer GCN (Alg. 1 with L = 2; Kipf's model)  — forward, loss, backward
# ---------------------------------------------------------------------------

def forward(Ahat, X, Th0, Th1):
    """a¹ = X Θ0, P1 = Â a¹, H1 = ReLU(P1), a² = H1 Θ1, L = Â a²  (Alg. 1)."""
    X = np.asarray(X, dtype=np.float64)
    P1 = aggregate(Ahat, X @ np.asarray(Th0, dtype=np.float64))
    H1 = np.maximum(P1, 0.0)
    L = aggregate(Ahat, H1 @ np.asarray(Th1, dtype=np.float64))
    return P1, H1, L


def softmax_ce(L, labels, train):
    """loss = (1/|T|) Σ_{i∈T} [logsumexp(L_i) − L_{i,y_i}],
    dL = (softmax(L) − onehot(y)) ⊙ [i∈T] / |T|   (reading #14)."""
    L = np.asarray(L, dtype=np.float64)
    train = np.asarray(train, dtype=bool)
    m = L.max(axis=1, keepdims=True)
    e = np.exp(L - m)
    s = e.sum(axis=1, keepdims=True)
    lse = (m + np.log(s)).ravel()
    nT = int(train.sum())
    idx = np.arange(L.shape[0])
    loss = float(((lse - L[idx, labels]) * train).sum() / nT)
    dL = e / s
    dL[idx, labels] -= 1.0
    dL *= (train[:, None] / nT)
    return loss, dL


def backward(Ahat, X, Th0, Th1, P1, H1, dL):
    """Chain rule through Alg. 1 (the paper is silent on the backward, reading A4):
    G1 = Âᵀ dL = Â dL, ∇Θ1 = H1ᵀ G1, dP1 = (G1 Θ1ᵀ) ⊙ [P1 > 0],
    G0 = Â dP1, ∇Θ0 = Xᵀ G0."""
    X = np.asarray(X, dtype=np.float64)
    G1 = aggregate(Ahat.T.tocsr(), dL)
    gTh1 = H1.T @ G1
    dP1 = (G1 @ np.asarray(Th1, dtype=np.float64).T) * (P1 > 0)
    G0 = aggregate(Ahat.T.tocsr(), dP1)
    gTh0 = X.T @ G0
    return dict(G1=G1, dP1=dP1, G0=G0, gTh0=gTh0, gTh1=gTh1)


def epoch(Ahat, X, Th0, Th1, labels, train):
    """One full-batch epoch (fwd + loss + bwd), returning every intermediate."""
    P1, H1, L = forward(Ahat, X, Th0, Th1)
    loss, dL = softmax_ce(L, labels, train)
    g = backward(Ahat, X, Th0, Th1, P1, H1, dL)
    return dict(P1=P1, H1=H1, L=L, loss=loss, dL=dL, **g)


# ---------------------------------------------------------------------------
# ℓ-layer GCN (Alg. 1 with general ℓ; the paper's Table II model has ℓ = 4,
# hid = 64, L255) — SURVEY.md §8(f) F2
# ---------------------------------------------------------------------------

def forward_l(Ahat, X, Ths):
    """Alg. 1 (L101-L125) for ℓ = len(Ths) layers: a^l = h^{l-1} Θ_l (L114),
    P_l = Â a^l (L118-L121), h^l = ReLU(P_l) between layers (reading #14),
    logits = P_ℓ.  Returns (Ps, Hs) with Hs[l] the INPUT of layer l (Hs[0] = X)."""
    H = np.asarray(X, dtype=np.float64)
    Ps, Hs = [], [H]
    for l, Th in enumerate(Ths):
        P = aggregate(Ahat, H @ np.asarray(Th, dtype=np.float64))
        Ps.append(P)
        if l < len(Ths) - 1:
            H = np.maximum(P, 0.0)
            Hs.append(H)
    return Ps, Hs


def backward_l(Ahat, Ths, Ps, Hs, dL):
    """Chain rule through forward_l: G_ℓ = Â dL; for l = ℓ..1:
    ∇Θ_l = h^{l-1}ᵀ G_l, and (l > 1) dP_{l-1} = (G_l Θ_lᵀ) ⊙ [P_{l-1} > 0],
    G_{l-1} = Â dP_{l-1}  (Âᵀ = Â, reading #2)."""
    AT = Ahat.T.tocsr()
    G = aggregate(AT, dL)
    grads = [None] * len(Ths)
    Gs = [None] * len(Ths)
    for l in range(len(Ths) - 1, -1, -1):
        Gs[l] = G
        grads[l] = Hs[l].T @ G
        if l > 0:
            dP = (G @ np.asarray(Ths[l], dtype=np.float64).T) * (Ps[l - 1] > 0)
            G = aggregate(AT, dP)
    return grads, Gs


def epoch_l(Ahat, X, Ths, labels, train):
    """One full-batch epoch of the ℓ-layer model."""
    Ps, Hs = forward_l(Ahat, X, Ths)
    loss, dL = softmax_ce(Ps[-1], labels, train)
    grads, Gs = backward_l(Ahat, Ths, Ps, Hs, dL)
    return dict(Ps=Ps, Hs=Hs, loss=loss, dL=dL, grads=grads, Gs=Gs)


def adam(Th, g, m, v, t, lr=0.01, b1=0.9, b2=0.999, eps=1e-8):
    """Adam (Kingma & Ba, Alg. 1) with bias correction; t starts at 1.
    (Reading #14: the paper's model is Kipf's, trained with Adam; SGD needs
    no oracle — the parity tests read the SGD step back as (Θ - Θ')/lr.)"""
    m = b1 * m + (1 - b1) * g
    v = b2 * v + (1 - b2) * g * g
    mh = m / (1 - b1 ** t)
    vh = v / (1 - b2 ** t)
    return Th - lr * mh / (np.sqrt(vh) + eps), m, v
