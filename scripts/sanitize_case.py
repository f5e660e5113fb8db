"""Tiny end-to-end cases for compute-sanitizer (memcheck / racecheck /
synccheck): every kernel family of libpcgcn on small graphs — selective rows
(short rows, long-row segments, partial-warp layout), tf32x2 / bf16x3 /
bf16x1 / SIMT full mode, both grains, the transform and gradient GEMMs,
softmax-CE, Adam, halo pack/unpack — one eager GCN2 epoch each."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_tianmyd20_b200 import _lib as L  # noqa: E402
from paper_conf_ipps_tianmyd20_b200.gcn import GCN2  # noqa: E402
from synth import configs as C  # noqa: E402
from synth import graphs as G  # noqa: E402


def hubs():
    edges, base = [], 0
    for leaves in (1500, 1025):
        edges += [(base, base + i) for i in range(1, leaves + 1)]
        base += leaves + 1
    for sz in (200, 130):
        ii, jj = np.triu_indices(sz, 1)
        edges += list(zip((base + ii).tolist(), (base + jj).tolist()))
        base += sz
    e = np.random.default_rng(7).integers(0, base, size=(2 * base, 2))
    edges += [tuple(x) for x in e.tolist() if x[0] != x[1]]
    return G.from_edges(base, edges)


def main():
    torch.cuda.set_device(0)
    w = C.CORA
    for g, H, Cc in ((C.graph(w), 16, 7), (hubs(), 128, 41)):
        X = np.random.default_rng(1).standard_normal((g.n, 40)).astype(np.float32)
        y = (np.arange(g.n) % Cc).astype(np.int32)
        T = np.arange(g.n) % 5 != 0
        Th0 = C.glorot(40, H, 3, 0)
        Th1 = C.glorot(H, Cc, 3, 1)
        for dense, theta, kw in ((L.DENSE_TF32X2, 0.05, {}), (L.DENSE_BF16X3, 0.02, dict(order=1, grain=1)),
                                 (L.DENSE_BF16X1, 0.0, {}), (L.DENSE_FP32_SIMT, 0.1, {}), (L.DENSE_TF32X2, 2.0, {})):
            pl = L.Plan(g.n, g.rowptr, g.col, 4, theta, dense_prec=dense, f_max=128, **kw)
            perm = pl.perm()
            m = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="adam", lr=0.01)
            m.epoch()
            torch.cuda.synchronize()
            assert np.isfinite(m.loss.item())
            pl.destroy()
        # halo pack / unpack on a 2-shard plan (shard 0's lists), device side only
        pl = L.Plan(g.n, g.rowptr, g.col, 4, 0.05, rank=0, world=2)
        Y = torch.randn(g.n, 16, device="cuda")
        ns = sum(len(pl.halo(q, True)) for q in range(2))
        nr = sum(len(pl.halo(q, False)) for q in range(2))
        sb = torch.empty(max(ns, 1), 16, device="cuda")
        pl.halo_pack(Y, sb, 16)
        rb = torch.randn(max(nr, 1), 16, device="cuda")
        pl.halo_unpack(rb[:nr], Y, 16)
        torch.cuda.synchronize()
    print("sanitize cases done")


if __name__ == "__main__":
    main()
