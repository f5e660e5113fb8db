"""Test infrastructure (imports oracle/, so it lives under tests/).  Full (not extrapolated) fp64 oracle epoch on the host cores, once with BLAS
limited to 1 thread and once with all cores (SURVEY.md
§8(d) "Oracle timing beside the GPU").  Prints one JSON line per workload.

    python tests/oracle_epoch_time.py [cora pubmed reddit]
"""
import json
import os
import platform
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from threadpoolctl import threadpool_limits, threadpool_info  # noqa: E402

from oracle import gcn as O  # noqa: E402
from synth import configs as C  # noqa: E402


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
        for l in out.splitlines():
            if l.startswith("Model name"):
                return l.split(":", 1)[1].strip()
    except Exception:
        pass
    return platform.processor()


def main():
    names = sys.argv[1:] or ["cora", "pubmed", "reddit"]
    cores = len(os.sched_getaffinity(0))
    for name in names:
        w = C.WORKLOADS[name]
        g = C.graph(w)
        X = C.features(w, g.n)
        Th0, Th1 = C.thetas(w)
        y = C.labels(w, g)
        T = C.train_mask(g.n, w.theta_seed)
        t0 = time.perf_counter()
        Ahat = O.normalized_adjacency(g.n, g.rowptr, g.col)[0]
        t_norm = time.perf_counter() - t0
        res = {"workload": name, "n": g.n, "nnz": int(Ahat.nnz), "normalize_s": t_norm, "cpu": cpu_model(),
               "affinity_cores": cores}
        for label, lim in (("1_thread", 1), ("all_cores", cores)):
            with threadpool_limits(limits=lim):
                blas = max([i.get("num_threads", 1) for i in threadpool_info()] or [1])
                t0 = time.perf_counter()
                out = O.epoch(Ahat, X, Th0, Th1, y, T)
                res[label] = {"epoch_s": time.perf_counter() - t0, "blas_threads": blas}
                del out
        res["note"] = ("one full fp64 epoch (oracle.gcn.epoch: 4 scipy SpMMs single-threaded + numpy GEMMs on "
                       "`blas_threads`), after the Â build (normalize_s); no sampling, no extrapolation")
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
