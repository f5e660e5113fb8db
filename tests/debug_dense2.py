"""Diagnostic (not collected by pytest): full mode with values whose tf32 lo
part matters (1 - 2^-24), integer-free; vary the number of row tiles per
persistent CTA.  Prints relative deficit per row (2^-12 ~ 'lo missing')."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_tianmyd20_b200 import _lib as L  # noqa: E402
from synth import graphs as G  # noqa: E402

x = np.float32(1.0 - 2.0 ** -24)
for ncl, size in ((4, 100), (100, 100), (300, 100), (600, 100), (300, 300)):
    g = G.cliques([size] * ncl)
    for F in (16, 128):
        pl = L.Plan(g.n, g.rowptr, g.col, max(1, g.n // 1000), 0.0, norm=L.NORM_NONE, f_max=128)
        st = pl.stats()
        ld = (F + 3) // 4 * 4
        Yd = torch.full((g.n, ld), float(x), device="cuda")
        Zd = torch.zeros_like(Yd)
        pl.forward(Yd, Zd, F=F)
        torch.cuda.synchronize()
        Z = Zd.cpu().numpy()[:, :F].astype(np.float64)
        exp = size * float(x)
        rel = (exp - Z) / exp
        bad = np.argwhere(np.abs(rel) > 1e-6)
        print(f"cliques {ncl}x{size} F={F} tiles={st['row_tiles']} chunks={st['chunks']} max rel {np.abs(rel).max():.3e} "
              f"bad rows {len(np.unique(bad[:, 0])) if len(bad) else 0}", flush=True)
        if len(bad):
            perm = pl.perm()
            inv = np.argsort(perm)
            rows = np.unique(bad[:, 0])
            print("   first bad plan rows:", sorted(inv[rows])[:10], " tile of first:", sorted(inv[rows])[0] // 128,
                  flush=True)
