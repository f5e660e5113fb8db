"""Pins of the fp64 oracle against what the paper and mathematics fix
(SURVEY.md §8(c) pins P1-P16).  CPU only."""
import math
import os

import numpy as np
import pytest

from oracle import gcn as O
from synth import configs as C
from synth import graphs as G

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _ahat(g, norm="sym"):
    return O.normalized_adjacency(g.n, g.rowptr, g.col, norm)[0]


# P1: dense brute force from the raw edge list (handles duplicates, input
# self-loops and isolated vertices by explicit loops)
@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_p1_dense_bruteforce(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 64))
    g = G.messy_random(n, int(rng.integers(0, 3 * n)), seed)
    A = np.zeros((n, n))
    for v in range(n):
        for j in g.col[g.rowptr[v]:g.rowptr[v + 1]]:
            if j != v:
                A[v, j] = 1.0
    At = A + np.eye(n)
    d = At.sum(axis=1)
    Ad = np.empty((n, n))
    for i in range(n):
        for j in range(n):
            Ad[i, j] = At[i, j] / math.sqrt(d[i] * d[j])
    Ahat = _ahat(g).toarray()
    np.testing.assert_allclose(Ahat, Ad, rtol=0, atol=1e-15)
    Y = rng.standard_normal((n, 5))
    np.testing.assert_allclose(O.aggregate(_ahat(g), Y), Ad @ Y, rtol=1e-13, atol=1e-13)


def test_p2_complete_graph_mean():
    n = 17
    Y = np.random.default_rng(5).standard_normal((n, 6))
    Z = O.aggregate(_ahat(G.complete(n)), Y)
    np.testing.assert_allclose(Z, np.repeat(Y.mean(axis=0, keepdims=True), n, 0), rtol=1e-13, atol=1e-14)


def test_p3_cycle_closed_form_and_row_sums():
    n = 11
    Y = np.random.default_rng(6).standard_normal((n, 3))
    Z = O.aggregate(_ahat(G.cycle(n)), Y)
    exp = (np.roll(Y, 1, 0) + Y + np.roll(Y, -1, 0)) / 3.0
    np.testing.assert_allclose(Z, exp, rtol=1e-13, atol=1e-14)
    # d-regular => rows of Â sum to 1
    np.testing.assert_allclose(np.asarray(_ahat(G.cycle(n)).sum(axis=1)).ravel(), 1.0, atol=1e-15)


def test_p4_path_worked_example():
    lines = [l for l in open(os.path.join(GOLD, "path_graph.txt")) if not l.startswith("#")]
    for l in lines:
        vals = l.split()
        n = int(vals[0])
        exp = np.array([float(v) for v in vals[1:]])
        Y = np.arange(1, n + 1, dtype=np.float64)[:, None]
        Z = O.aggregate(_ahat(G.path(n)), Y).ravel()
        np.testing.assert_allclose(Z, exp, rtol=1e-14)


def test_p5_star_entries():
    A = _ahat(G.star(3)).toarray()
    assert A[0, 0] == pytest.approx(0.25, abs=1e-15)
    assert A[0, 1] == pytest.approx(0.35355339059327, abs=1e-13)
    assert A[1, 1] == pytest.approx(0.5, abs=1e-15)
    assert A[1, 2] == 0.0


@pytest.mark.parametrize("which", ["cora", "random"])
def test_p6_universal_eigenvector(which):
    g = G.sbm(C.CORA.spec) if which == "cora" else G.random_graph(80, 0.1, 3)
    Ahat, dt, _ = O.normalized_adjacency(g.n, g.rowptr, g.col)
    s = np.sqrt(dt)[:, None]
    np.testing.assert_allclose(O.aggregate(Ahat, s), s, rtol=1e-13)


def test_p7_disjoint_cliques_mean():
    sizes = [5, 9, 1, 13]
    g = G.cliques(sizes, seed=4)
    Y = np.random.default_rng(7).standard_normal((g.n, 4))
    Z = O.aggregate(_ahat(g), Y)
    for c in range(len(sizes)):
        m = g.labels == c
        np.testing.assert_allclose(Z[m], np.repeat(Y[m].mean(0, keepdims=True), m.sum(), 0),
                                   rtol=1e-13, atol=1e-14)


def test_p8_empty_graph_identity():
    Y = np.random.default_rng(8).standard_normal((9, 3))
    np.testing.assert_array_equal(O.aggregate(_ahat(G.empty(9)), Y), Y)


def test_p9_integer_exact_none_norm():
    g = G.random_graph(40, 0.2, 9)
    Y = np.random.default_rng(9).integers(-50, 50, size=(40, 3)).astype(np.float64)
    At = _ahat(g, "none")
    Z = O.aggregate(At, Y)
    # brute force integer sums
    for v in range(g.n):
        nb = list(g.col[g.rowptr[v]:g.rowptr[v + 1]]) + [v]
        assert np.array_equal(Z[v], Y[nb].sum(0))


def test_p11_adjoint():
    g = G.sbm(C.CORA.spec)
    Ahat = _ahat(g)
    rng = np.random.default_rng(11)
    U = rng.standard_normal((g.n, 4))
    V = rng.standard_normal((g.n, 4))
    lhs = np.sum(U * O.aggregate(Ahat, V))
    rhs = np.sum(O.aggregate(Ahat, U) * V)
    assert abs(lhs - rhs) <= 1e-12 * max(1.0, abs(lhs))


def test_rejects_asymmetric():
    g = G.from_edges(3, [(0, 1)], symmetrize=False)
    with pytest.raises(ValueError):
        O.normalized_adjacency(g.n, g.rowptr, g.col)


def test_aggregate_rows_matches_full():
    g = G.messy_random(50, 120, 12)
    Y = np.random.default_rng(12).standard_normal((50, 3))
    rows = [0, 7, 49, 23]
    np.testing.assert_allclose(O.aggregate_rows(g.n, g.rowptr, g.col, Y, rows),
                               O.aggregate(_ahat(g), Y)[rows], rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(O.aggregate_rows(g.n, g.rowptr, g.col, Y, rows, "none"),
                               O.aggregate(_ahat(g, "none"), Y)[rows], rtol=1e-13)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_clean_degrees_matches_binary_adjacency(seed):
    """clean_degrees (row-chunked, with the clean-row shortcut) equals the row
    sums of the binary A built by scipy's duplicate collapsing, on messy input
    (duplicates, self-loops, unsorted rows) with trailing empty rows, and on a
    clean sorted CSR."""
    g = G.messy_random(60, 200, seed)
    n = g.n + 5                                       # 5 isolated trailing vertices
    rowptr = np.concatenate([g.rowptr, np.full(5, g.rowptr[-1])])
    rng = np.random.default_rng(seed)
    col = g.col.copy()
    for i in range(g.n):                              # shuffle inside rows
        rng.shuffle(col[rowptr[i]:rowptr[i + 1]])
    A = O.binary_adjacency(n, rowptr, col)
    np.testing.assert_array_equal(O.clean_degrees(n, rowptr, col), np.asarray(A.sum(axis=1)).ravel())
    c = G.cycle(40)
    np.testing.assert_array_equal(O.clean_degrees(c.n, c.rowptr, c.col), np.full(40, 2))


def _tiny_problem(seed=13, n=30, f=7, h=5, c=4):
    g = G.random_graph(n, 0.15, seed)
    rng = np.random.default_rng(seed)
    X = rng.standard_normal((n, f))
    Th0 = rng.standard_normal((f, h)) * 0.5
    Th1 = rng.standard_normal((h, c)) * 0.5
    y = rng.integers(0, c, n)
    T = rng.random(n) < 0.7
    return g, X, Th0, Th1, y, T


# P12: finite differences of the loss
def test_p12_finite_differences():
    g, X, Th0, Th1, y, T = _tiny_problem()
    Ahat = _ahat(g)
    out = O.epoch(Ahat, X, Th0, Th1, y, T)

    def loss(a, b):
        return O.softmax_ce(O.forward(Ahat, X, a, b)[2], y, T)[0]

    h = 1e-6
    rng = np.random.default_rng(0)
    for Th, gname, which in ((Th0, "gTh0", 0), (Th1, "gTh1", 1)):
        for _ in range(6):
            i, j = rng.integers(0, Th.shape[0]), rng.integers(0, Th.shape[1])
            P, M = Th.copy(), Th.copy()
            P[i, j] += h
            M[i, j] -= h
            fd = (loss(P, Th1) - loss(M, Th1)) / (2 * h) if which == 0 else \
                 (loss(Th0, P) - loss(Th0, M)) / (2 * h)
            an = out[gname][i, j]
            assert abs(fd - an) <= 1e-7 * max(1.0, abs(an)) + 1e-9


# P13: torch fp64 autograd of the same 2-layer GCN
def test_p13_torch_autograd():
    torch = pytest.importorskip("torch")
    g, X, Th0, Th1, y, T = _tiny_problem(seed=14)
    Ahat = _ahat(g)
    out = O.epoch(Ahat, X, Th0, Th1, y, T)
    A = torch.tensor(Ahat.toarray(), dtype=torch.float64)
    Xt = torch.tensor(X)
    a = torch.tensor(Th0, requires_grad=True)
    b = torch.tensor(Th1, requires_grad=True)
    L = A @ torch.relu(A @ Xt @ a) @ b
    Tm = torch.tensor(T)
    ce = torch.nn.functional.cross_entropy(L[Tm], torch.tensor(y)[Tm])
    ce.backward()
    assert abs(ce.item() - out["loss"]) < 1e-13
    np.testing.assert_allclose(a.grad.numpy(), out["gTh0"], rtol=1e-11, atol=1e-14)
    np.testing.assert_allclose(b.grad.numpy(), out["gTh1"], rtol=1e-11, atol=1e-14)
    np.testing.assert_allclose(L.detach().numpy(), out["L"], rtol=1e-12, atol=1e-14)


# P12/P13 for the ℓ-layer model: finite differences and torch
# fp64 autograd of the same ℓ = 4 network
def _deep_problem(seed=15, n=28, dims=(6, 5, 4, 5, 3)):
    g = G.random_graph(n, 0.2, seed)
    rng = np.random.default_rng(seed)
    X = rng.standard_normal((n, dims[0]))
    Ths = [rng.standard_normal((dims[i], dims[i + 1])) * 0.6 for i in range(len(dims) - 1)]
    y = rng.integers(0, dims[-1], n)
    T = rng.random(n) < 0.7
    return g, X, Ths, y, T


def test_deep_finite_differences():
    g, X, Ths, y, T = _deep_problem()
    Ahat = _ahat(g)
    out = O.epoch_l(Ahat, X, Ths, y, T)

    def loss(ths):
        return O.softmax_ce(O.forward_l(Ahat, X, ths)[0][-1], y, T)[0]

    h = 1e-6
    rng = np.random.default_rng(1)
    for l in range(len(Ths)):
        for _ in range(4):
            i, j = rng.integers(0, Ths[l].shape[0]), rng.integers(0, Ths[l].shape[1])
            P = [t.copy() for t in Ths]
            M = [t.copy() for t in Ths]
            P[l][i, j] += h
            M[l][i, j] -= h
            fd = (loss(P) - loss(M)) / (2 * h)
            an = out["grads"][l][i, j]
            assert abs(fd - an) <= 1e-7 * max(1.0, abs(an)) + 1e-9, (l, fd, an)


def test_deep_torch_autograd_and_two_layer_special_case():
    torch = pytest.importorskip("torch")
    g, X, Ths, y, T = _deep_problem(seed=16)
    Ahat = _ahat(g)
    out = O.epoch_l(Ahat, X, Ths, y, T)
    A = torch.tensor(Ahat.toarray(), dtype=torch.float64)
    ts = [torch.tensor(t, requires_grad=True) for t in Ths]
    H = torch.tensor(X)
    for l, t in enumerate(ts):
        H = A @ H @ t
        if l < len(ts) - 1:
            H = torch.relu(H)
    Tm = torch.tensor(T)
    ce = torch.nn.functional.cross_entropy(H[Tm], torch.tensor(y)[Tm])
    ce.backward()
    assert abs(ce.item() - out["loss"]) < 1e-13
    for t, gr in zip(ts, out["grads"]):
        np.testing.assert_allclose(t.grad.numpy(), gr, rtol=1e-11, atol=1e-14)
    # ℓ = 2 is the 2-layer model of forward()/backward()
    g2, X2, Th0, Th1, y2, T2 = _tiny_problem(seed=17)
    A2 = _ahat(g2)
    o2 = O.epoch(A2, X2, Th0, Th1, y2, T2)
    ol = O.epoch_l(A2, X2, [Th0, Th1], y2, T2)
    np.testing.assert_allclose(ol["grads"][0], o2["gTh0"], rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(ol["grads"][1], o2["gTh1"], rtol=1e-12, atol=1e-15)


# P14: uniform logits
def test_p14_softmax_ce_uniform():
    n, c = 12, 5
    L = np.full((n, c), 0.37)
    y = np.arange(n) % c
    T = np.arange(n) % 3 != 0
    loss, dL = O.softmax_ce(L, y, T)
    assert loss == pytest.approx(math.log(c), abs=1e-14)
    exp = (1.0 / c - np.eye(c)[y]) * (T[:, None] / T.sum())
    np.testing.assert_allclose(dL, exp, atol=1e-15)


def test_adam_first_step_closed_form():
    g = np.array([[0.3, -2.0], [1e-3, 0.0]])
    Th = np.zeros_like(g)
    new, m, v = O.adam(Th, g, np.zeros_like(g), np.zeros_like(g), 1, lr=0.01)
    # m̂ = g, v̂ = g² after bias correction => step = lr * g / (|g| + eps)
    np.testing.assert_allclose(new, -0.01 * g / (np.abs(g) + 1e-8), rtol=1e-12)


def test_adam_constant_gradient_any_step():
    """For a constant gradient the bias corrections are exact at every t:
    m_t = (1-b1^t) g and v_t = (1-b2^t) g^2, so m̂ = g, v̂ = g^2 and every step
    moves by lr·g/(|g|+eps) (Kingma & Ba, §2-3).  Checks t = 1..6, including
    the t = 2 state the GPU Adam is compared against."""
    g = np.array([0.3, -2.0, 1e-3, 0.0, 7.5])
    Th, m, v = np.zeros_like(g), np.zeros_like(g), np.zeros_like(g)
    for t in range(1, 7):
        Th, m, v = O.adam(Th, g, m, v, t, lr=0.01)
        np.testing.assert_allclose(m, (1 - 0.9 ** t) * g, rtol=1e-12)
        np.testing.assert_allclose(v, (1 - 0.999 ** t) * g * g, rtol=1e-12)
        np.testing.assert_allclose(Th, -0.01 * t * g / (np.abs(g) + 1e-8), rtol=1e-12, atol=1e-300)


def test_adam_two_steps_sign_flip_and_scale_invariance():
    """t = 2 with g2 = -g1: m_2 = b1(1-b1) g - (1-b1) g = -(1-b1)^2 g, so
    m̂_2 = -(1-b1)^2/(1-b1^2) g = -(0.01/0.19) g, while v̂_2 = g^2 (both terms
    carry g^2).  And Adam is invariant to a positive rescaling of all
    gradients up to eps (a wrong power of v or a missing sqrt breaks it)."""
    g = np.array([0.5, -3.0, 2e-2])
    Th1, m, v = O.adam(np.zeros_like(g), g, np.zeros_like(g), np.zeros_like(g), 1)
    Th2, m, v = O.adam(Th1, -g, m, v, 2)
    step2 = Th2 - Th1
    np.testing.assert_allclose(step2, 0.01 * (0.01 / 0.19) * g / np.abs(g), rtol=1e-6)
    for c in (1e-2, 10.0, 1e3):
        a, ma, va = O.adam(np.ones(3), c * g, np.zeros(3), np.zeros(3), 1, eps=0.0)
        a, _, _ = O.adam(a, c * 0.5 * g, ma, va, 2, eps=0.0)
        b, mb, vb = O.adam(np.ones(3), g, np.zeros(3), np.zeros(3), 1, eps=0.0)
        b, _, _ = O.adam(b, 0.5 * g, mb, vb, 2, eps=0.0)
        np.testing.assert_allclose(a, b, rtol=1e-12)


# P16: Table I counting convention (nnz(A+I) = 2m + n)
def test_p16_counting_convention():
    g = G.sbm(C.PUBMED.spec)
    assert g.n == 19_717
    assert g.nnz + g.n == 108_365  # Table I pubmed "#edge 108.3K"
    gc = G.sbm(C.CORA.spec)
    assert gc.nnz + gc.n == 13_264
    At = _ahat(g, "none")
    assert At.nnz == 108_365
