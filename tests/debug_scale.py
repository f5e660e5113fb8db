"""Diagnostic (not collected by pytest): universal-eigenvector check on C3 per
mode; prints the worst rows as 'edges missing' = (s_i - Z_i) * s_i (= count of
absent unit terms, since r_j s_j = 1)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from oracle import gcn as O  # noqa: E402
from paper_conf_ipps_tianmyd20_b200 import _lib as L  # noqa: E402
from synth import configs as C  # noqa: E402

w = C.REDDIT
g = C.graph(w)
deg = O.clean_degrees(g.n, g.rowptr, g.col)
print("max degree", deg.max(), "rows with d>20000:", np.sum(deg > 20000), flush=True)
s = np.sqrt(deg + 1.0)
for theta, dense, F in ((2.0, L.DENSE_TF32X2, 128), (0.02, L.DENSE_TF32X2, 128), (0.02, L.DENSE_FP32_SIMT, 128),
                        (0.0, L.DENSE_TF32X2, 16), (0.02, L.DENSE_TF32X2, 41)):
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, dense_prec=dense, f_max=128)
    st = pl.stats()
    perm = pl.perm()
    inv = np.argsort(perm)
    ld = (F + 3) // 4 * 4
    Yp = np.zeros((g.n, ld), np.float32)
    Yp[:, :F] = s[perm].astype(np.float32)[:, None]
    Yd = torch.from_numpy(Yp).cuda()
    Zd = torch.zeros_like(Yd)
    pl.forward(Yd, Zd, F=F)
    torch.cuda.synchronize()
    Z = Zd.cpu().numpy()[:, :F][inv].astype(np.float64)
    s32 = s.astype(np.float32).astype(np.float64)
    rel = np.abs(Z - s32[:, None]) / s32[:, None]
    worst = np.argsort(-rel.max(1))[:5]
    print(f"theta={theta} dense={dense} F={F} dense_edges={st['nnz_dense']} max rel {rel.max():.3e}", flush=True)
    for v in worst:
        c = int(np.argmax(rel[v]))
        miss = (s32[v] - Z[v, c]) * s32[v]
        print(f"   v={v} deg={deg[v]} plan_row={inv[v]} col={c} rel={rel[v, c]:.3e} missing_terms={miss:.3f} "
              f"cols_bad={np.sum(rel[v] > 1e-5)}", flush=True)
