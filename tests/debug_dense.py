"""Diagnostic (not collected by pytest): full-mode kernels on tiny integer
cases, printing where the tcgen05 result departs from the exact answer."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_tianmyd20_b200 import _lib as L  # noqa: E402
from synth import graphs as G  # noqa: E402


def run(g, F, dense, P=1, theta=0.0, Y=None):
    pl = L.Plan(g.n, g.rowptr, g.col, P, theta, norm=L.NORM_NONE, dense_prec=dense)
    perm = pl.perm()
    ld = (F + 3) // 4 * 4
    if Y is None:
        Y = (np.arange(g.n)[:, None] * 16 + np.arange(F)[None, :]).astype(np.float32)
    Yp = np.zeros((g.n, ld), np.float32)
    Yp[:, :F] = Y[perm]
    Yd = torch.from_numpy(Yp).cuda()
    Z = torch.full((g.n, ld), -7.0, device="cuda")
    pl.forward(Yd, Z, F=F)
    torch.cuda.synchronize()
    Zp = Z.cpu().numpy()[:, :F]
    out = np.empty_like(Zp)
    out[perm] = Zp
    rows = np.repeat(np.arange(g.n), np.diff(g.rowptr))
    exp = Y.astype(np.float64).copy()
    np.add.at(exp, rows, Y[g.col])
    return out, exp, pl


for name, g in (("path37", G.path(37)), ("K128", G.complete(128)), ("K200", G.complete(200))):
    for F in (16, 1, 32, 48, 128):
        for dense, dn in ((L.DENSE_FP32_SIMT, "simt"), (L.DENSE_TF32X2, "tc")):
            out, exp, pl = run(g, F, dense)
            bad = np.argwhere(out != exp)
            print(f"{name} F={F} {dn}: mismatches {len(bad)}/{out.size} chunks={pl.stats()['chunks']}", flush=True)
            if len(bad) and dn == "tc" and F in (16, 32):
                np.set_printoptions(linewidth=200, threshold=2000)
                print(" got[:6,:8]\n", out[:6, :8], "\n exp[:6,:8]\n", exp[:6, :8])
                print(" got[-3:,:8]\n", out[-3:, :8], "\n exp[-3:,:8]\n", exp[-3:, :8])
