"""GPU parity: the CUDA path through the C ABI vs the fp64 oracle on the same
seeded inputs (run on a B200: pytest -m gpu).

Error metric (reading #18): condition-scaled
    err = max_{i,f} |z - z*| / (|Â|·|Y|)_{i,f}
which equals the plain relative error for nonnegative inputs and is immune to
cancellation in mixed-sign sums.  Gates (BASELINE.json north_star):
sparse fp32 <= 1e-5, dense tcgen05 2xTF32 <= 1e-5, integer-exact regime
bitwise; plan arrays bit-exact (tests/test_plan_abi.py).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import gcn as O  # noqa: E402
from synth import configs as C  # noqa: E402
from synth import graphs as G  # noqa: E402

L = pytest.importorskip("paper_conf_ipps_tianmyd20_b200._lib")

TOL = 1e-5


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.init()


def _ld(F):
    return (F + 3) // 4 * 4


def aggregate_gpu(g, Y, P, theta, *, dense=L.DENSE_TF32X2, norm=L.NORM_SYM, part=None, backward=False,
                  flags=0, f_max=None, **plan_kw):
    F = Y.shape[1]
    f_max = f_max or max(128, F)
    pl = L.Plan(g.n, g.rowptr, g.col, P, theta, norm=norm, dense_prec=dense, part=part, f_max=f_max, **plan_kw)
    perm = pl.perm()
    Yp = np.zeros((g.n, _ld(F)), dtype=np.float32)
    Yp[:, :F] = Y[perm]
    Yd = torch.from_numpy(Yp).cuda()
    Zd = torch.full((g.n, _ld(F)), float("nan"), device="cuda")
    if backward:
        pl.backward(Yd, Zd, F=F, flags=flags)
    else:
        pl.forward(Yd, Zd, F=F, flags=flags)
    torch.cuda.synchronize()
    Z = np.empty((g.n, F), dtype=np.float64)
    Z[perm] = Zd.cpu().numpy()[:, :F]
    return Z, pl, Zd


def cond_err(g, Y, Z, norm="sym"):
    Ahat = O.normalized_adjacency(g.n, g.rowptr, g.col, norm)[0]
    Zs = O.aggregate(Ahat, Y.astype(np.float64))
    scale = O.aggregate(abs(Ahat), np.abs(Y.astype(np.float64)))
    scale = np.maximum(scale, 1e-30)
    return float(np.max(np.abs(Z - Zs) / scale)), Zs


def _feat(n, F, seed, nonneg=False):
    rng = np.random.default_rng(seed)
    Y = rng.standard_normal((n, F)).astype(np.float32)
    return np.abs(Y) if nonneg else Y


SMALL = {
    "path": lambda: G.path(37),
    "cycle": lambda: G.cycle(300),
    "star": lambda: G.star(260),
    "complete": lambda: G.complete(150),
    "cliques": lambda: G.cliques([130, 70, 200, 5, 1], seed=2),
    "empty": lambda: G.empty(77),
    "messy": lambda: G.messy_random(700, 4000, 3),
    "cora": lambda: G.sbm(C.CORA.spec),
}


@pytest.mark.parametrize("name", list(SMALL))
@pytest.mark.parametrize("mode", ["sparse", "dense_tc", "dense_simt", "hybrid", "dense_bf16", "hybrid_tile",
                                  "dense_bf3", "hybrid_tile_bf3"])
@pytest.mark.parametrize("F", [1, 7, 16, 24, 32, 33, 40, 41, 48, 64, 128])
def test_aggregation_parity(name, mode, F):
    g = SMALL[name]()
    P = max(1, min(8, g.n // 40))
    theta = {"sparse": 2.0, "dense_tc": 0.0, "dense_simt": 0.0, "hybrid": 0.05, "dense_bf16": 0.0,
             "hybrid_tile": 0.05, "dense_bf3": 0.0, "hybrid_tile_bf3": 0.05}[mode]
    dense = {"dense_simt": L.DENSE_FP32_SIMT, "dense_bf16": L.DENSE_BF16X1, "dense_bf3": L.DENSE_BF16X3,
             "hybrid_tile_bf3": L.DENSE_BF16X3}.get(mode, L.DENSE_TF32X2)
    kw = dict(order=L.ORDER_DEGREE, grain=L.GRAIN_TILE) if mode.startswith("hybrid_tile") else {}
    Y = _feat(g.n, F, 11)
    Z, pl, _ = aggregate_gpu(g, Y, P, theta, dense=dense, **kw)
    err, _ = cond_err(g, Y, Z)
    # bf16 inputs (PCGCN_DENSE_BF16X1): |rounding| <= 2^-9 per term; gate 2e-2 (north star)
    tol = 2e-2 if mode == "dense_bf16" else TOL
    assert err <= tol, (name, mode, F, err, pl.stats())
    if mode == "dense_bf16":
        assert err <= 2.0 ** -8, err   # what the rounding bound predicts


def test_closed_forms_complete_and_cycle_dense():
    g = G.complete(200)
    Y = _feat(g.n, 64, 3)
    Z, pl, _ = aggregate_gpu(g, Y, 1, 0.0)
    assert pl.stats()["nnz_dense"] == 200 * 200
    np.testing.assert_allclose(Z, np.repeat(Y.astype(np.float64).mean(0, keepdims=True), 200, 0),
                               rtol=2e-6, atol=2e-6)
    g = G.cycle(500)
    Y = _feat(g.n, 16, 4)
    Z, _, _ = aggregate_gpu(g, Y, 5, 2.0)
    exp = (np.roll(Y, 1, 0) + Y + np.roll(Y, -1, 0)).astype(np.float64) / 3.0
    np.testing.assert_allclose(Z, exp, rtol=1e-5, atol=1e-6)


@pytest.mark.parametrize("mode", ["sparse", "dense_tc", "dense_simt", "hybrid", "hybrid_tile", "dense_bf3"])
def test_integer_exact_bitwise(mode):
    """Pin P9: Ã unnormalised, small integers -> every order gives the exact
    sum, so GPU (either mode, any partition, any grain) == oracle bitwise."""
    g = G.cliques([300, 129, 64, 33, 2], seed=5)
    rng = np.random.default_rng(9)
    Y = rng.integers(-1000, 1000, size=(g.n, 40)).astype(np.float32)
    theta = {"sparse": 2.0, "dense_tc": 0.0, "dense_simt": 0.0, "hybrid": 0.3, "hybrid_tile": 0.3,
             "dense_bf3": 0.0}[mode]
    dense = {"dense_simt": L.DENSE_FP32_SIMT, "dense_bf3": L.DENSE_BF16X3}.get(mode, L.DENSE_TF32X2)
    kw = dict(order=L.ORDER_DEGREE, grain=L.GRAIN_TILE) if mode == "hybrid_tile" else {}
    Z, _, _ = aggregate_gpu(g, Y, 5, theta, dense=dense, norm=L.NORM_NONE, **kw)
    exp = O.aggregate(O.normalized_adjacency(g.n, g.rowptr, g.col, "none")[0], Y.astype(np.float64))
    assert np.array_equal(Z, exp)


@pytest.mark.parametrize("dense", ["tf32x2", "bf16x3"])
@pytest.mark.parametrize("F", [16, 41, 128, 200])
def test_dense_long_accumulation_accuracy(F, dense):
    """Full mode on rows with thousands of dense terms, all-positive values
    whose tf32 lo part matters (1 - 2^-24): the tensor core's biased TMEM
    accumulation must not build up (groups of <= 8 chunks are folded into
    fp32 registers).  Expected: every row = d̃·x exactly up to fp32 rounding."""
    g = G.cliques([2000, 1500])
    x = np.float32(1.0 - 2.0 ** -24)
    Y = np.full((g.n, F), x, dtype=np.float32)
    Z, pl, _ = aggregate_gpu(g, Y, 2, 0.0, norm=L.NORM_NONE, f_max=256,
                             dense=L.DENSE_BF16X3 if dense == "bf16x3" else L.DENSE_TF32X2)
    assert pl.stats()["nnz_dense"] == pl.stats()["nnz"]
    size = np.where(g.labels == 0, 2000, 1500)[:, None]
    rel = np.abs(Z - size * float(x)) / (size * float(x))
    # gate 1e-5 (north star); with group folding this is ~2.5e-6, without it
    # (63 chunks x 8 MMAs in one TMEM chain) it exceeds 1e-5
    assert rel.max() < 1e-5, rel.max()


def test_partition_invariance_integer_regime():
    """L131 §III-A.c: only the summation order changes — bitwise under P9."""
    g = G.sbm(C.CORA.spec)
    Y = np.random.default_rng(1).integers(-50, 50, size=(g.n, 16)).astype(np.float32)
    outs = []
    for P, theta, part in ((8, 0.05, None), (3, 2.0, None), (8, 0.0, None),
                           (6, 0.01, np.random.default_rng(2).integers(0, 6, g.n))):
        Z, _, _ = aggregate_gpu(g, Y, P, theta, norm=L.NORM_NONE, part=part)
        outs.append(Z)
    for Z in outs[1:]:
        assert np.array_equal(Z, outs[0])


def test_relabel_invariance_tolerance():
    g = G.sbm(C.CORA.spec)
    Y = _feat(g.n, 16, 3)
    Z1, _, _ = aggregate_gpu(g, Y, 8, 0.05)
    perm = np.random.default_rng(3).permutation(g.n)
    inv = np.argsort(perm)
    # relabel vertex v -> inv[v]
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    g2 = G.from_edges(g.n, list(zip(inv[rows], inv[g.col])), symmetrize=False)
    Z2, _, _ = aggregate_gpu(g2, Y[perm], 8, 0.05)
    np.testing.assert_allclose(Z2, Z1[perm], rtol=1e-5, atol=1e-6)


def test_backward_equals_forward_and_deterministic():
    g = G.sbm(C.PUBMED.spec)
    Y = _feat(g.n, 16, 8)
    Zf, _, Zf_d = aggregate_gpu(g, Y, 32, 0.02)
    Zb, _, Zb_d = aggregate_gpu(g, Y, 32, 0.02, backward=True)
    assert torch.equal(Zf_d, Zb_d)
    Z2, _, Z2_d = aggregate_gpu(g, Y, 32, 0.02)
    assert torch.equal(Zf_d, Z2_d)


def test_epilogue_flags_relu_mask_prescaled():
    g = G.sbm(C.CORA.spec)
    F = 41
    Y = _feat(g.n, F, 12)
    pl = L.Plan(g.n, g.rowptr, g.col, 8, 0.03)
    perm = pl.perm()
    Ahat, dt, r = O.normalized_adjacency(g.n, g.rowptr, g.col)
    Zs = O.aggregate(Ahat, Y.astype(np.float64))[perm]
    rp = r[perm][:, None]
    Yp = np.zeros((g.n, 44), np.float32)
    Yp[:, :F] = (Y[perm] * rp).astype(np.float32)  # prescaled input
    Yd = torch.from_numpy(Yp).cuda()
    Z = torch.zeros(g.n, 44, device="cuda")
    mask = torch.zeros(g.n, 2, dtype=torch.int32, device="cuda")
    pl.forward(Yd, Z, F=F, flags=L.IN_PRESCALED | L.RELU | L.MASK_OUT | L.OUT_PRESCALED, mask=mask)
    torch.cuda.synchronize()
    Zc = Z.cpu().numpy()[:, :F].astype(np.float64)
    np.testing.assert_allclose(Zc, np.maximum(Zs, 0) * rp, rtol=1e-5, atol=1e-6)
    m = mask.cpu().numpy().view(np.uint32)
    bits = ((m[:, :, None] >> np.arange(32, dtype=np.uint32)) & 1).reshape(g.n, 64)[:, :F]
    agree = bits.astype(bool) == (Zs > 0)
    near0 = np.abs(Zs) < 1e-6
    assert np.all(agree | near0)
    assert np.all(bits.reshape(g.n, 64)[:, F:] == 0) if bits.shape[1] > F else True


def _np(t):
    return t.detach().cpu().numpy().astype(np.float64)


@pytest.mark.parametrize("path", ["tcgen05", "simt"])
@pytest.mark.parametrize("M,K,N", [(1000, 602, 128), (2708, 1433, 16), (777, 128, 41), (5, 3, 7),
                                   (20000, 602, 128)])
def test_gemms(M, K, N, path):
    """xw / xtg / dwt vs numpy fp64.  'tcgen05' passes 16-byte aligned rows
    and a workspace (3xTF32 engine); 'simt' passes unaligned X (fp32 cores)."""
    rng = np.random.default_rng(M + K + N)
    ldk = _ld(K) if path == "tcgen05" else K
    Xfull = torch.zeros(M, ldk, device="cuda")
    Xfull[:, :K] = torch.from_numpy(rng.standard_normal((M, K)).astype(np.float32)).cuda()
    X = Xfull[:, :K] if path == "tcgen05" else Xfull
    W = torch.from_numpy(rng.standard_normal((K, N)).astype(np.float32)).cuda()
    s = torch.from_numpy(rng.random(M).astype(np.float32) + 0.5).cuda()
    ldn = _ld(N)
    Y = torch.full((M, ldn), float("nan"), device="cuda")
    import ctypes
    work = torch.zeros(L.gemm_xw_work_floats(K, N), device="cuda") if path == "tcgen05" else None
    L.gemm_xw(X, W, ctypes.c_void_p(s.data_ptr()), Y, N=N, work=work)
    torch.cuda.synchronize()
    exp = _np(s)[:, None] * (_np(X) @ _np(W))
    scale = _np(s)[:, None] * (np.abs(_np(X)) @ np.abs(_np(W)))
    assert np.max(np.abs(_np(Y)[:, :N] - exp) / scale) < TOL
    assert np.all(_np(Y)[:, N:] == 0)
    # Xᵀ D
    D = torch.from_numpy(rng.standard_normal((M, N)).astype(np.float32)).cuda()
    Gm = torch.zeros(K, N, device="cuda")
    work = torch.zeros(L.gemm_xtg_work_floats(M, K, N), device="cuda")
    L.gemm_xtg(X, D, Gm, work)
    torch.cuda.synchronize()
    exp = _np(X).T @ _np(D)
    scale = np.abs(_np(X)).T @ np.abs(_np(D))
    assert np.max(np.abs(_np(Gm) - exp) / scale) < TOL
    # diag(s)((D Wᵀ) ⊙ mask)  with W [K2 x N]
    K2 = K
    W2 = torch.from_numpy(rng.standard_normal((K2, N)).astype(np.float32)).cuda()
    mw = (K2 + 31) // 32
    mbits = rng.integers(0, 2**32, size=(M, mw), dtype=np.uint64).astype(np.uint32)
    mask = torch.from_numpy(mbits.view(np.int32)).cuda()
    O_ = torch.full((M, _ld(K2)), float("nan"), device="cuda")
    if path == "tcgen05":   # 16-byte rows + workspace: the engine path (K2 <= 256), else fp32 cores
        Dp = torch.zeros(M, _ld(N), device="cuda")
        Dp[:, :N] = D
        L.gemm_dwt(Dp, W2, mask, ctypes.c_void_p(s.data_ptr()), O_, M=M, N=N, K=K2,
                   work=torch.zeros(L.gemm_dwt_work_floats(K2, N), device="cuda"))
    else:
        L.gemm_dwt(D, W2, mask, ctypes.c_void_p(s.data_ptr()), O_)
    torch.cuda.synchronize()
    mk = ((mbits[:, :, None] >> np.arange(32, dtype=np.uint32)) & 1).reshape(M, mw * 32)[:, :K2]
    exp = _np(s)[:, None] * ((_np(D) @ _np(W2).T) * mk)
    scale = _np(s)[:, None] * (np.abs(_np(D)) @ np.abs(_np(W2)).T) + 1e-30
    assert np.max(np.abs(_np(O_)[:, :K2] - exp) / scale) < TOL
    assert np.all(_np(O_)[:, K2:] == 0)


def test_softmax_ce_and_adam():
    rng = np.random.default_rng(4)
    M, Cc = 5000, 41
    Lg = rng.standard_normal((M, Cc)).astype(np.float32) * 3
    y = rng.integers(0, Cc, M).astype(np.int32)
    T = rng.random(M) < 0.8
    Ld = torch.zeros(M, 44, device="cuda")
    Ld[:, :Cc] = torch.from_numpy(Lg).cuda()
    dL = torch.zeros_like(Ld)
    loss = torch.zeros(1, device="cuda")
    work = torch.zeros(L.CE_WORK_FLOATS, device="cuda")
    L.softmax_ce(Ld, torch.from_numpy(y).cuda(), torch.from_numpy(T.astype(np.uint8)).cuda(), 1.0 / T.sum(),
                 None, dL, loss, work, C=Cc)
    torch.cuda.synchronize()
    l_ref, dL_ref = O.softmax_ce(Lg, y, T)
    assert abs(loss.item() - l_ref) <= 1e-5 * abs(l_ref)
    np.testing.assert_allclose(_np(dL)[:, :Cc], dL_ref, rtol=0, atol=1e-7 / T.sum() * 50)
    # Adam: two steps vs oracle
    th = rng.standard_normal(1000).astype(np.float32)
    gs = [rng.standard_normal(1000).astype(np.float32) for _ in range(2)]
    td = torch.from_numpy(th.copy()).cuda()
    m = torch.zeros_like(td)
    v = torch.zeros_like(td)
    step = torch.zeros(1, dtype=torch.int32, device="cuda")
    ref, mr, vr = th.astype(np.float64), np.zeros(1000), np.zeros(1000)
    for t, g_ in enumerate(gs, 1):
        L.adam(td, torch.from_numpy(g_).cuda(), m, v, 0.01, step)
        ref, mr, vr = O.adam(ref, g_.astype(np.float64), mr, vr, t)
    torch.cuda.synchronize()
    assert step.item() == 2
    np.testing.assert_allclose(_np(td), ref, rtol=1e-5, atol=1e-6)


@pytest.mark.parametrize("wname,theta,theta_c", [("cora", 0.05, None), ("pubmed", 0.02, None), ("cora", 2.0, None),
                                                  ("pubmed", 0.0, None), ("cora", 0.01, 0.005),
                                                  ("pubmed", 0.02, 2.0)])
def test_epoch_parity(wname, theta, theta_c):
    """Rows a4-a13 of one 2-layer GCN epoch + an SGD step vs the fp64 oracle,
    every output gated at a condition-scaled 1e-5 (tests/epoch_check.py);
    theta_c: a second plan for the width-C aggregations (per-width modes, as
    bench.py runs them)."""
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from epoch_check import OracleEpoch, check_gcn2_epoch
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    y = g.labels
    T = C.train_mask(g.n, w.theta_seed)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta_c) if theta_c is not None else None
    perm = pl.perm()
    model = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1, plan_c=pl_c)
    model.epoch()
    torch.cuda.synchronize()
    ref = OracleEpoch(g, X, Th0, Th1, y, T)
    check_gcn2_epoch(model, ref, perm, lr=0.1, Th0=Th0, Th1=Th1)


@pytest.mark.parametrize("d,theta,theta_c,grain", [(1.0, 0.02, 0.02, "block"), (5.0, 0.1, 2.0, "block"),
                                                   (10.0, 0.2, 0.1, "block"), (10.0, 0.0, 2.0, "block"),
                                                   (1.0, 0.1, 0.05, "tile"), (5.0, 0.2, 0.3, "tile"),
                                                   (10.0, 0.3, 0.2, "tile"), (10.0, 0.1, 0.1, "tile_bf3"),
                                                   (1.0, 0.05, 0.08, "tile_bf3")])
def test_rmat_hybrid_epoch_parity(d, theta, theta_c, grain):
    """SURVEY F1 / Table III workloads (RMAT-1, -5, -10: n = 10,240, 128 -> 64 -> 32,
    P = 16): mixed selective/full plans, one per
    width, as bench.py --table3 runs them — a full epoch vs the oracle."""
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from epoch_check import OracleEpoch, check_gcn2_epoch
    w = C.RMAT[d]
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    y = C.labels(w, g)
    T = C.train_mask(g.n, w.theta_seed)
    kw = dict(f_max=128, order=L.ORDER_DEGREE, grain=L.GRAIN_TILE) if grain.startswith("tile") else dict(f_max=128)
    if grain.endswith("bf3"):
        kw["dense_prec"] = L.DENSE_BF16X3
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, **kw)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta_c, **kw)
    st, st_c = pl.stats(), pl_c.stats()
    if 0 < theta < 1:
        assert 0 < st["nnz_dense"] < st["nnz"], st            # a mixed plan
    perm = pl.perm()
    model = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1, plan_c=pl_c)
    model.capture(warmup=0)
    model.replay()                                              # the CUDA-graph path bench.py times
    torch.cuda.synchronize()
    ref = OracleEpoch(g, X, Th0, Th1, y, T)
    check_gcn2_epoch(model, ref, perm, lr=0.1, Th0=Th0, Th1=Th1)


def test_cuda_graph_replay_matches_eager():
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    w = C.CORA
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, 1)
    pl = L.Plan(g.n, g.rowptr, g.col, 8, 0.05)
    perm = pl.perm()
    a = GCN2(pl, X[perm], g.labels[perm], T[perm], Th0, Th1)
    b = GCN2(pl, X[perm], g.labels[perm], T[perm], Th0, Th1)
    for _ in range(3):
        a.epoch()
    b.capture(warmup=1)
    b.replay()
    b.replay()
    torch.cuda.synchronize()
    assert torch.equal(a.theta, b.theta)
    assert a.step_ctr.item() == b.step_ctr.item() == 3


@pytest.mark.parametrize("F", [41, 128])
def test_calibrate_theta(F):
    """L161: θ = T_f·p/T_s from the two measured times, and a plan built with
    that θ puts exactly the blocks of density > θ in the full mode."""
    p = 0.05
    th, tf, ts = L.calibrate(F, 1024, p)
    assert tf > 0 and ts > 0
    assert th == pytest.approx(tf * p / ts, rel=1e-5)
    if not 0 < th < 1:
        return
    g = G.sbm(C.PUBMED.spec)
    pl = L.Plan(g.n, g.rowptr, g.col, 32, th, build_device=0)
    k, i = pl.export("blk_k"), pl.export("blk_i")
    nnz, dense = pl.export("blk_nnz"), pl.export("blk_dense")
    ps = np.diff(pl.export("pstart")).astype(np.float64)
    rho = nnz / (ps[k] * ps[i])
    assert np.array_equal(dense.astype(bool), rho > np.float64(np.float32(th)))


def test_dense_pair_kernel_subprocess():
    """The opt-in CTA-pair (tcgen05 cta_group::2) full-mode kernel, enabled
    with PCGCN_DENSE_PAIR=1 in a fresh process: integer-exact regime bitwise
    vs the oracle, and condition-scaled 1e-5 on a hybrid Cora plan, F=128."""
    import os
    import subprocess
    import sys
    code = r'''
import sys, numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_ipps_tianmyd20_b200 import _lib as L
from oracle import gcn as O
from synth import configs as C, graphs as G
for g, P, theta, norm in ((G.cliques([300, 129, 64, 33, 2], seed=5), 5, 0.0, "none"),
                          (C.graph(C.CORA), 8, 0.02, "sym"), (G.cliques([200] * 9), 3, 0.0, "none")):
    rng = np.random.default_rng(3)
    Y = (rng.integers(-1000, 1000, size=(g.n, 128)) if norm == "none" else rng.standard_normal((g.n, 128))).astype(np.float32)
    pl = L.Plan(g.n, g.rowptr, g.col, P, theta, norm=L.NORM_NONE if norm == "none" else L.NORM_SYM)
    perm = pl.perm()
    Yd = torch.from_numpy(np.ascontiguousarray(Y[perm])).cuda(); Z = torch.zeros_like(Yd)
    pl.forward(Yd, Z, F=128); torch.cuda.synchronize()
    Zo = np.empty((g.n, 128)); Zo[perm] = Z.cpu().numpy()
    A = O.normalized_adjacency(g.n, g.rowptr, g.col, norm)[0]
    ref = O.aggregate(A, Y.astype(np.float64))
    if norm == "none":
        assert np.array_equal(Zo, ref), "pair kernel: integer regime not exact"
    else:
        sc = O.aggregate(abs(A), np.abs(Y.astype(np.float64)))
        err = np.max(np.abs(Zo - ref) / np.maximum(sc, 1e-30))
        assert err <= 1e-5, err
print("ok")
'''
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, PCGCN_DENSE_PAIR="1")
    out = subprocess.run([sys.executable, "-c", code], check=True, env=env, cwd=root, capture_output=True,
                         text=True, timeout=300)
    assert out.stdout.strip().endswith("ok")


def _hubs(n_leaf=5000, extra=3):
    """Stars joined at their leaves: hub rows with 1-5 long-row segments
    (> SEG_EDGES = 1024 selective edges) next to short rows."""
    edges = []
    base = 0
    for k, leaves in enumerate([n_leaf, 1100, 2047, 1025]):
        hub = base
        edges += [(hub, hub + i) for i in range(1, leaves + 1)]
        base += leaves + 1
    rng = np.random.default_rng(7)
    e = rng.integers(0, base, size=(extra * base, 2))
    edges += [tuple(x) for x in e if x[0] != x[1]]
    return G.from_edges(base, edges)


@pytest.mark.parametrize("F", [1, 7, 41, 128, 200])
@pytest.mark.parametrize("ldpad", [0, 16])
def test_long_rows_segments(F, ldpad):
    """Rows longer than SEG_EDGES go through the segment pass and are summed
    from their segment partials (reading #22); values, ReLU and the
    mask vs the oracle, with row strides padded past roundup(F, 4)."""
    g = _hubs()
    pl = L.Plan(g.n, g.rowptr, g.col, 4, 2.0, f_max=256)
    assert pl.stats()["shard_segments"] >= 5 + 2 + 2 + 2
    perm = pl.perm()
    ld = _ld(F) + ldpad
    Y = _feat(g.n, F, 21)
    Yp = np.zeros((g.n, ld), np.float32)
    Yp[:, :F] = Y[perm]
    Yd = torch.from_numpy(Yp).cuda()
    Zd = torch.full((g.n, ld), float("nan"), device="cuda")
    mw = (F + 31) // 32
    mask = torch.zeros(g.n, mw, dtype=torch.int32, device="cuda")
    pl.forward(Yd, Zd, F=F, flags=L.RELU | L.MASK_OUT, mask=mask)
    torch.cuda.synchronize()
    Ahat = O.normalized_adjacency(g.n, g.rowptr, g.col)[0]
    Zs = O.aggregate(Ahat, Y.astype(np.float64))[perm]
    scale = np.maximum(O.aggregate(abs(Ahat), np.abs(Y.astype(np.float64)))[perm], 1e-30)
    Zc = Zd.cpu().numpy()[:, :F].astype(np.float64)
    err = np.max(np.abs(Zc - np.maximum(Zs, 0)) / scale)
    assert err <= TOL, err
    m = mask.cpu().numpy().view(np.uint32)
    bits = ((m[:, :, None] >> np.arange(32, dtype=np.uint32)) & 1).reshape(g.n, 32 * mw)
    assert np.all((bits[:, :F].astype(bool) == (Zs > 0)) | (np.abs(Zs) < 1e-6 * scale))
    assert np.all(bits[:, F:] == 0)
    # run to run bitwise (dynamic row scheduling does not change any row's order)
    Z2 = torch.full_like(Zd, float("nan"))
    pl.forward(Yd, Z2, F=F, flags=L.RELU | L.MASK_OUT, mask=mask)
    torch.cuda.synchronize()
    assert torch.equal(Z2[:, :F], Zd[:, :F])


@pytest.mark.parametrize("F,ld", [(41, 48), (42, 48), (47, 48), (48, 48), (41, 56), (48, 64)])
@pytest.mark.parametrize("gname", ["hubs", "cora", "cliques"])
def test_partial_warp_layout(gname, F, ld):
    """41..48 features in 32-byte aligned rows take the G = 6 lane layout (five
    rows per load instruction, two idle lanes, slots combined by a fixed
    shuffle sequence): values, ReLU, mask (incl. its zero tail) vs the oracle,
    long-row segments included, and run-to-run bitwise."""
    g = {"hubs": _hubs, "cora": lambda: G.sbm(C.CORA.spec),
         "cliques": lambda: G.cliques([130, 70, 200, 5, 1], seed=2)}[gname]()
    pl = L.Plan(g.n, g.rowptr, g.col, 4, 0.05 if gname != "hubs" else 2.0, f_max=128)
    perm = pl.perm()
    Y = _feat(g.n, F, 23)
    Yp = np.zeros((g.n, ld), np.float32)
    Yp[:, :F] = Y[perm]
    Yd = torch.from_numpy(Yp).cuda()
    assert Yd.data_ptr() % 32 == 0
    Zd = torch.full((g.n, ld), float("nan"), device="cuda")
    mw = (F + 31) // 32
    mask = torch.full((g.n, mw), -1, dtype=torch.int32, device="cuda")
    pl.forward(Yd, Zd, F=F, flags=L.RELU | L.MASK_OUT, mask=mask)
    torch.cuda.synchronize()
    Ahat = O.normalized_adjacency(g.n, g.rowptr, g.col)[0]
    Zs = O.aggregate(Ahat, Y.astype(np.float64))[perm]
    scale = np.maximum(O.aggregate(abs(Ahat), np.abs(Y.astype(np.float64)))[perm], 1e-30)
    Zc = Zd.cpu().numpy()[:, :F].astype(np.float64)
    assert np.max(np.abs(Zc - np.maximum(Zs, 0)) / scale) <= TOL
    m = mask.cpu().numpy().view(np.uint32)
    bits = ((m[:, :, None] >> np.arange(32, dtype=np.uint32)) & 1).reshape(g.n, 32 * mw)
    assert np.all((bits[:, :F].astype(bool) == (Zs > 0)) | (np.abs(Zs) < 1e-6 * scale))
    assert np.all(bits[:, F:] == 0)
    Z2 = torch.full_like(Zd, float("nan"))
    pl.forward(Yd, Z2, F=F, flags=L.RELU | L.MASK_OUT, mask=mask)
    torch.cuda.synchronize()
    assert torch.equal(Z2[:, :F], Zd[:, :F])


@pytest.mark.parametrize("wname,theta,nl", [("cora", 0.05, 4), ("pubmed", 0.0, 4), ("cora", 2.0, 3),
                                            ("pubmed", 0.02, 2)])
def test_epoch_parity_deep(wname, theta, nl):
    """The ℓ-layer model (the paper's Table II shape ℓ = 4, L255)
    vs the oracle's forward_l/backward_l + one SGD step, every activation,
    gradient and the loss gated at a condition-scaled 1e-5 whose scales are
    compounded layer by layer (tests/epoch_check.py)."""
    from paper_conf_ipps_tianmyd20_b200.gcn import GCNL
    from epoch_check import OracleEpochL, check_gcnl_epoch
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    X = C.features(w, g.n)
    dims = [w.f_in] + [w.hidden] * (nl - 1) + [w.classes]
    Ths = [C.glorot(dims[i], dims[i + 1], w.theta_seed, 10 + i) for i in range(nl)]
    y = C.labels(w, g)
    T = C.train_mask(g.n, w.theta_seed)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta)
    perm = pl.perm()
    model = GCNL(pl, X[perm], y[perm], T[perm], Ths, optimizer="sgd", lr=0.1)
    model.epoch()
    torch.cuda.synchronize()
    ref = OracleEpochL(g, X, Ths, y, T)
    check_gcnl_epoch(model, ref, perm, lr=0.1)


_KNOB_CODE = r'''
import sys, numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_ipps_tianmyd20_b200 import _lib as L
from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
from synth import configs as C, graphs as G
out = {}
# selective rows of every length class (hub rows with long-row segments, short
# rows) next to dense tiles (cliques)
edges, base = [], 0
for leaves in (5000, 1100, 2047, 1025):
    edges += [(base, base + i) for i in range(1, leaves + 1)]
    base += leaves + 1
for sz in (300, 200, 129, 64):
    ii, jj = np.triu_indices(sz, 1)
    edges += list(zip((base + ii).tolist(), (base + jj).tolist()))
    base += sz
e = np.random.default_rng(7).integers(0, base, size=(3 * base, 2))
edges += [tuple(x) for x in e.tolist() if x[0] != x[1]]
g = G.from_edges(base, edges)
rng = np.random.default_rng(11)
import os
dp = getattr(L, os.environ.get("PCGCN_TEST_DENSE", "DENSE_TF32X2"))
for F, theta, ld in ((128, 0.02, 128), (41, 0.04, 44), (40, 0.04, 48), (32, 2.0, 32), (41, 0.03, 48)):
    pl = L.Plan(g.n, g.rowptr, g.col, 8, theta, dense_prec=dp)
    Y = torch.from_numpy(rng.standard_normal((g.n, ld)).astype(np.float32)).cuda()
    Y[:, F:] = 0
    Z = torch.zeros_like(Y)
    M = torch.zeros(g.n, (F + 31) // 32, dtype=torch.int32, device="cuda")
    pl.forward(Y, Z, F=F, flags=L.RELU | L.MASK_OUT, mask=M)
    torch.cuda.synchronize()
    out[f"agg{F}_{ld}"] = Z.cpu().numpy()
    out[f"mask{F}_{ld}"] = M.cpu().numpy()
# one epoch (the xtg / dwt GEMMs included)
w = C.PUBMED
gp = C.graph(w)
X = C.features(w, gp.n)
Th0, Th1 = C.thetas(w)
T = C.train_mask(gp.n, w.theta_seed)
pl = L.Plan(gp.n, gp.rowptr, gp.col, w.P, 0.02)
perm = pl.perm()
m = GCN2(pl, X[perm], gp.labels[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1)
m.epoch()
torch.cuda.synchronize()
out["gTh0"] = m.gTh0.cpu().numpy()
out["gTh1"] = m.gTh1.cpu().numpy()
out["loss"] = np.array([m.loss.item()])
np.savez(sys.argv[1], **out)
'''


@pytest.mark.parametrize("knob,bitwise", [({"PCGCN_ROWS_PER_TICKET": "1"}, True),
                                          ({"PCGCN_ROWS_PER_TICKET": "16"}, True),
                                          ({"PCGCN_OVERLAP": "1"}, True),
                                          ({"PCGCN_XTG_PRESPLIT": "1"}, True),
                                          ({"PCGCN_DENSE_BLOCKED": "0"}, True),
                                          ({"PCGCN_SPARSE_V8": "0"}, False),
                                          ({"PCGCN_SPARSE_FSPLIT": "32"}, False),
                                          ({"PCGCN_SPARSE_G6": "0"}, False),
                                          ({"PCGCN_TC_DYN": "0"}, True),
                                          ({"PCGCN_TC_DYN_ORDER": "plan"}, True),
                                          ({"PCGCN_SPARSE_MROW": "0"}, False),
                                          ({"PCGCN_SPARSE_MROW": "1"}, False),
                                          ({"PCGCN_SPARSE_MROW": "1", "PCGCN_MROW_SORT": "1"}, False),
                                          ({"PCGCN_SEG_INLINE": "1"}, True),
                                          ({"PCGCN_SEG_INLINE": "1", "PCGCN_SEG_AHEAD": "64"}, True),
                                          ({"PCGCN_SEG_INLINE": "1", "PCGCN_SEG_AHEAD": "1"}, True)])
def test_scheduling_knobs_do_not_change_results(tmp_path, knob, bitwise, base=None):
    """Row-block tickets, inline vs separate long-row segments (the same
    partials added in the same order), the full-mode/segment overlap, the in-kernel xtg B
    conversion and the window-blocked full-mode B layout change only scheduling (every output row is still reduced by
    one warp in the same order; the MMA sequence and the hi/lo split are the
    same), so aggregation outputs, masks, gradients and the loss must be
    bitwise identical to the default configuration.  The lane-layout knobs
    (16- vs 32-byte vectors, column slices, G = 6, multi-row warps) sum a row in
    another fixed order: within 2e-6 of the largest output, masks self-consistent."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = {}
    for tag, extra in (("default", base or {}), ("knob", {**(base or {}), **knob})):
        env = {k: v for k, v in os.environ.items() if not k.startswith("PCGCN_")}
        env.update(extra)
        f = str(tmp_path / f"{tag}.npz")
        subprocess.run([sys.executable, "-c", _KNOB_CODE, f], check=True, env=env, cwd=root, capture_output=True,
                       text=True, timeout=600)
        res[tag] = np.load(f)
    for k in res["default"].files:
        a, b = res["default"][k], res["knob"][k]
        if bitwise:
            assert np.array_equal(a, b), (knob, k, float(np.max(np.abs(a.astype(np.float64) - b))))
        elif k.startswith("mask"):
            # 16- vs 32-byte lane vectors sum a row's edges in another (fixed)
            # order: each run's mask must be exactly its own [Z > 0]
            F, ld = (int(x) for x in k[4:].split("_"))
            for tag in ("default", "knob"):
                Z = res[tag][f"agg{F}_{ld}"][:, :F]
                want = np.zeros_like(res[tag][k])
                for c in range(F):
                    want[:, c // 32] |= ((Z[:, c] > 0).astype(np.int64) << (c % 32)).astype(np.uint32).view(np.int32)
                assert np.array_equal(res[tag][k], want), (knob, tag, k)
        else:
            scale = max(float(np.max(np.abs(a))), 1e-30)
            assert float(np.max(np.abs(a.astype(np.float64) - b))) <= 2e-6 * scale, (knob, k)


def test_multirow_degree_grouping_is_bitwise(tmp_path):
    """Multi-row warps group a 32-row ticket's rows by degree (PCGCN_MROW_SORT):
    which slot gathers a row changes, the row's own sequential sum does not —
    outputs, masks, gradients and the loss are bitwise identical with and
    without the grouping."""
    test_scheduling_knobs_do_not_change_results(tmp_path, {"PCGCN_MROW_SORT": "1"}, True,
                                                base={"PCGCN_SPARSE_MROW": "1"})


def test_stacked_bf16x3_parts_match_three_mmas(tmp_path):
    """bf16x3 full mode for F <= 64 stacks the three bf16 parts along N (one
    MMA per K-step, the epilogue adds the three column blocks); PCGCN_TC_STACK=0
    issues one MMA per part.  Same products, another fp32 association: within
    2e-6 of the largest output, masks self-consistent."""
    test_scheduling_knobs_do_not_change_results(tmp_path, {"PCGCN_TC_STACK": "0"}, False,
                                                base={"PCGCN_TEST_DENSE": "DENSE_BF16X3"})


@pytest.mark.parametrize("wname,theta,dense", [("cora", 0.01, "tf32x2"), ("pubmed", 0.0, "bf16x3"),
                                               ("cora", 0.005, "bf16x3"), ("pubmed", 2.0, "tf32x2"),
                                               ("cora", 0.005, "bf16x1"), ("pubmed", 0.01, "bf16x1")])
def test_fused_split_is_bitwise(wname, theta, dense):
    """pcgcn_gemm_xw_split / pcgcn_gemm_dwt_split write the full mode's window
    blocks in the GEMM epilogue and the aggregations then skip their split pass
    (IN_SPLIT): every output of the epoch is bitwise identical to the unfused
    epoch (same window-block bits, same MMAs)."""
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    kw = dict(order=L.ORDER_DEGREE, grain=L.GRAIN_TILE,
              dense_prec={"bf16x3": L.DENSE_BF16X3, "bf16x1": L.DENSE_BF16X1}.get(dense, L.DENSE_TF32X2))
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, **kw)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta * 2 if theta < 1 else theta, **kw)
    perm = pl.perm()
    outs = []
    for fuse in (True, False):
        m = GCN2(pl, X[perm], g.labels[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1, plan_c=pl_c,
                 fuse_split=fuse)
        assert m.fuse == fuse
        m.epoch()
        torch.cuda.synchronize()
        outs.append([t.clone() for t in (m.Y0, m.H1, m.mask1, m.Y1, m.Lg, m.G1, m.dP1, m.G0, m.grad, m.theta)])
    for a, b in zip(*outs):
        assert torch.equal(a, b)


def test_plan_with_negative_theta_calibrates_first():
    """θ < 0 in pcgcn_plan: the L161 calibration runs on the device first and
    the plan uses the θ it returns (reported in the stats); the plan then
    aggregates within the usual gate."""
    g = G.sbm(C.PUBMED.spec)
    pl = L.Plan(g.n, g.rowptr, g.col, 32, -1.0, f_max=64)
    th = pl.stats()["theta"]
    assert 0.0 < th < 1.0 and pl.theta == th
    Y = _feat(g.n, 48, 3)
    Z, _, _ = aggregate_gpu(g, Y, 32, th, f_max=64)
    err, _ = cond_err(g, Y, Z)
    assert err <= TOL
    with pytest.raises(L.PcgcnError):
        L.Plan(g.n, g.rowptr, g.col, 32, -1.0, build_device=False)
