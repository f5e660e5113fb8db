"""One eager 2-layer GCN epoch of a bench configuration, for ncu (run with
`ncu --profile-from-start off ...`: only the epoch between
cudaProfilerStart/Stop is captured).  Prints the plan statistics and, per
aggregation, the algorithmic byte counts the profile is compared against.

    python scripts/profile_epoch.py --workload reddit --theta 0.0389 --theta-c 0.08 \
        [--order degree] [--grain tile] [--dense bf16x3]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_tianmyd20_b200 import _lib as L  # noqa: E402
from paper_conf_ipps_tianmyd20_b200.gcn import GCN2  # noqa: E402
from synth import configs as C  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="reddit")
    ap.add_argument("--theta", type=float, required=True)
    ap.add_argument("--theta-c", type=float, default=None)
    ap.add_argument("--order", default="degree")
    ap.add_argument("--grain", default="tile")
    ap.add_argument("--dense", default="bf16x3")
    ap.add_argument("--epochs", type=int, default=1)
    a = ap.parse_args()
    kw = dict(order=L.ORDER_DEGREE if a.order == "degree" else L.ORDER_ID,
              grain=L.GRAIN_TILE if a.grain == "tile" else L.GRAIN_BLOCK,
              dense_prec=L.DENSE_BF16X3 if a.dense == "bf16x3" else L.DENSE_TF32X2)
    w = C.WORKLOADS[a.workload]
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    y = C.labels(w, g)
    fmax = max(w.hidden, w.classes)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, a.theta, f_max=fmax, **kw)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, a.theta_c, f_max=fmax, **kw) if a.theta_c is not None else None
    perm = pl.perm()
    m = GCN2(pl, np.ascontiguousarray(X[perm]), y[perm], T[perm], Th0, Th1, optimizer="adam", lr=0.01, plan_c=pl_c)
    for _ in range(2):
        m.epoch()
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for _ in range(a.epochs):
        m.epoch()
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(json.dumps({"plan": pl.stats(), "plan_c": (pl_c or pl).stats(), "launches_per_epoch": m.launches_per_epoch(),
                      "args": vars(a)}))


if __name__ == "__main__":
    main()
