"""At-scale parity on the bench workloads — C3 (Reddit-shaped: 233K vertices,
114.8M nnz(A+I), P=128) in the launch configuration bench.py times (hybrid
plans at the widths H=128 and C=41), C4 at 1/16 scale, and C5 (clustered
power-law, 33.5M vertices, 1.03B nnz(A+I), P=16384) at full size.  The full fp64 oracle does not
finish in seconds here, so:
  * P15  sampled rows: Z_i = r_i Σ_j r_j Y_j computed one by one in fp64
         (oracle.gcn.aggregate_rows) for seeded random rows + the
         highest-degree rows, condition-scaled error <= 1e-5;
  * P6   the universal eigenvector s = sqrt(d̃): Â·s = s for every row.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import gcn as O  # noqa: E402
from synth import configs as C  # noqa: E402

L = pytest.importorskip("paper_conf_ipps_tianmyd20_b200._lib")


@pytest.fixture(scope="module")
def c3():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    w = C.REDDIT
    g = C.graph(w)
    return w, g, O.clean_degrees(g.n, g.rowptr, g.col)


@pytest.fixture(scope="module")
def c3_epoch(c3):
    """The bench workload (C3 inputs exactly as bench.py builds them) and its
    full fp64 oracle epoch with condition scales (tests/epoch_check.py):
    ~8 sparse fp64 products of 115M entries on the host, a few minutes."""
    from epoch_check import OracleEpoch
    w, g, _ = c3
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    y = C.labels(w, g)
    T = C.train_mask(g.n, w.theta_seed)
    return w, g, X, Th0, Th1, y, T, OracleEpoch(g, X, Th0, Th1, y, T)


# θ pairs (F = H plan, F = C plan): the pair BENCH_r01 selected with its measured
# grid (0.0418, 0.056), the grid's neighbours, and all-selective
@pytest.mark.parametrize("theta,theta_c,cfg", [(0.0418, 0.056, "block"), (0.028, 0.04, "block"), (2.0, 2.0, "block"),
                                               (0.066, 0.066, "tile"), (0.045, 0.08, "tile"),
                                               (0.066, 0.066, "tile_bf3"), (0.04, 0.05, "tile_bf3")])
def test_c3_bench_epoch_all_rows(c3_epoch, theta, theta_c, cfg):
    """The exact launch configuration bench.py times on C3 (two plans, one per
    width; activation strides 128 / 48; one CUDA-graph replay of the epoch),
    with SGD so the update can be read back: H1, logits, loss, G1, G0, ∇Θ1,
    ∇Θ0 on ALL rows vs the full fp64 oracle epoch, condition-scaled 1e-5."""
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from epoch_check import check_gcn2_epoch
    w, g, X, Th0, Th1, y, T, ref = c3_epoch
    fmax = max(w.hidden, w.classes)
    kw = dict(f_max=fmax)
    if cfg.startswith("tile"):     # bench.py's default: degree order, per-chunk modes
        kw.update(order=L.ORDER_DEGREE, grain=L.GRAIN_TILE)
    if cfg.endswith("bf3"):
        kw.update(dense_prec=L.DENSE_BF16X3)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, **kw)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta_c, **kw)
    if theta < 1:
        assert pl.stats()["nnz_dense"] > 0 and pl_c.stats()["nnz_dense"] > 0
    perm = pl.perm()
    model = GCN2(pl, np.ascontiguousarray(X[perm]), y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1,
                 plan_c=pl_c)
    assert (model.ldH, model.ldC) == (128, 48)
    model.capture(warmup=0)
    model.replay()
    torch.cuda.synchronize()
    rep = {}
    check_gcn2_epoch(model, ref, perm, lr=0.1, Th0=Th0, Th1=Th1, report=rep)
    print("c3 bench epoch", theta, theta_c, cfg, rep)


@pytest.mark.parametrize("theta,theta_c", [(0.02, 0.03), (0.01, 0.015)])
def test_c3_bench_epoch_bf16x1(c3_epoch, theta, theta_c):
    """bench.py --dense bf16x1 (the paper's 16-bit full mode, L191-L193): the
    same launch configuration with bf16-rounded full-mode inputs, all rows of
    every epoch output vs the fp64 oracle at the north star's stated bf16 gate
    (2e-2, condition-scaled; tests/epoch_check.py TOL_BF16) — and the fp32
    selective part keeps the error well inside it."""
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from epoch_check import check_gcn2_epoch, TOL_BF16, BAND_BF16, BAND_FRAC_BF16
    w, g, X, Th0, Th1, y, T, ref = c3_epoch
    kw = dict(f_max=max(w.hidden, w.classes), order=L.ORDER_DEGREE, grain=L.GRAIN_TILE,
              dense_prec=L.DENSE_BF16X1)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, **kw)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta_c, **kw)
    assert pl.stats()["nnz_dense"] > 0 and pl_c.stats()["nnz_dense"] > 0
    perm = pl.perm()
    model = GCN2(pl, np.ascontiguousarray(X[perm]), y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1,
                 plan_c=pl_c)
    model.capture(warmup=0)
    model.replay()
    torch.cuda.synchronize()
    rep = {}
    check_gcn2_epoch(model, ref, perm, lr=0.1, Th0=Th0, Th1=Th1, report=rep, tol=TOL_BF16, band_rel=BAND_BF16,
                     band_frac=BAND_FRAC_BF16)
    print("c3 bench epoch bf16x1", theta, theta_c, rep)
    # the bf16 rounding is the only error above fp32 level: it must show, and stay bounded
    assert max(rep[k] for k in ("H1", "L", "G1", "G0")) <= 2.0 ** -6


@pytest.fixture(scope="module")
def c4s():
    """C4 (tiered SBM, BASELINE configs[3]) at 1/16 scale: 262K vertices,
    communities of 1,024 in four density tiers."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    w = C.scaled(C.SBM4M, 1 / 16)
    g = C.graph(w)
    return w, g, O.clean_degrees(g.n, g.rowptr, g.col)


@pytest.fixture(scope="module")
def c5():
    """C5 (BASELINE configs[4]) at full size: ~3 min to generate + plan."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    w = C.PL32M
    g = C.graph(w)
    return w, g, O.clean_degrees(g.n, g.rowptr, g.col)


@pytest.mark.parametrize("F,theta", [(128, 0.01), (32, 0.002)])
def test_c4_scaled_sampled_rows_and_eigenvector(c4s, F, theta):
    _check(c4s, F, theta)


@pytest.mark.parametrize("F,theta", [(128, 0.02), (41, 0.04), (128, 2.0)])
def test_c3_sampled_rows_and_eigenvector(c3, F, theta):
    _check(c3, F, theta)


@pytest.mark.parametrize("F,theta", [(128, 0.05)])
def test_c5_full_size_sampled_rows_and_eigenvector(c5, F, theta):
    """The bench's C5 launch configuration (calibrated θ ~ 0.04-0.05 leaves
    every block in the selective mode; hub rows run through the segment
    pass).  Y is passed un-prescaled (the plan's prescale pass runs first)."""
    _check(c5, F, theta, both_modes=False, n_sample=1500)


def _check(wgd, F, theta, both_modes=True, n_sample=1500):
    w, g, deg = wgd
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, f_max=128)
    st = pl.stats()
    if theta < 1 and both_modes:
        assert st["nnz_dense"] > 0 and st["nnz_sparse"] > 0   # both modes exercised
    perm = pl.perm()
    inv = np.argsort(perm)
    ld = (F + 3) // 4 * 4
    rng = np.random.default_rng(31)
    Y = rng.standard_normal((g.n, F)).astype(np.float32)
    s = np.sqrt(deg + 1.0)                       # universal eigenvector s = sqrt(d̃)
    Y[:, 0] = s.astype(np.float32)
    Yp = np.zeros((g.n, ld), np.float32)
    Yp[:, :F] = Y[perm]
    Yd = torch.from_numpy(Yp).cuda()
    Zd = torch.zeros_like(Yd)
    pl.forward(Yd, Zd, F=F)                      # un-prescaled input: Z = Â·Y
    torch.cuda.synchronize()
    Z = Zd.cpu().numpy()[:, :F][inv]             # back to vertex ids
    # P6 on every row (column 0 carries fp32(s): compare with the fp32-rounded input's image)
    s32 = Y[:, 0].astype(np.float64)
    rel = np.abs(Z[:, 0] - s32) / s32
    assert rel.max() < 2e-5, rel.max()
    # P15 sampled rows (seeded random + the 64 highest-degree vertices)
    rows = np.unique(np.concatenate([rng.choice(g.n, n_sample, replace=False), np.argsort(-deg)[:64]]))
    ref = O.aggregate_rows(g.n, g.rowptr, g.col, Y, rows, deg=deg)
    scale = O.aggregate_rows(g.n, g.rowptr, g.col, np.abs(Y), rows, deg=deg)
    err = np.max(np.abs(Z[rows] - ref) / np.maximum(scale, 1e-30))
    assert err <= 1e-5, err
