#!/usr/bin/env python
"""PCGCN hot-path benchmark: 2-layer GCN epoch ms + aggregation GB/s on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload reddit|pubmed|cora] [--theta auto|<float>] [--P <int>]

A step is one full-batch training epoch of the 2-layer GCN (SURVEY.md §8(a)
rows a4-a14: both transforms, four partition-centric aggregations, loss,
backward, Adam) over the Reddit-shaped synthetic graph (BASELINE.json
configs[2]; the north-star target config), replayed as one CUDA graph.
Timing: CUDA events on the launching stream around every step, L2 flushed
(256 MiB write) between steps outside the events, barrier + synchronize
around the K timed steps, max over ranks.  Prints ONE JSON line on rank 0.

--impl reference times the fp64 CPU oracle (oracle/, the only other place
bench.py runs it) on a bounded row sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

MEASURED_PEAKS = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM_GBS = 6650.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="reddit")
    ap.add_argument("--theta", default="auto")
    ap.add_argument("--theta-c", type=float, default=None, help="fixed θ of the width-C plan (with a fixed --theta)")
    ap.add_argument("--P", type=int, default=0)
    ap.add_argument("--order", default="auto", choices=["auto", "id", "degree"],
                    help="vertex order inside a partition (pcgcn_opts.vertex_order)")
    ap.add_argument("--grain", default="auto", choices=["auto", "block", "tile"],
                    help="unit of the selective/full decision (pcgcn_opts.mode_grain)")
    ap.add_argument("--fuse-split", default="on", choices=["on", "off"],
                    help="transform GEMMs write the full mode's window blocks (pcgcn_gemm_*_split)")
    ap.add_argument("--dense", default="bf16x3", choices=["tf32x2", "bf16x3", "bf16x1"],
                    help="full-mode arithmetic (pcgcn_opts.dense_prec)")
    ap.add_argument("--oracle-frac", type=float, default=0.02)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--eager", action="store_true", help="no CUDA graph")
    ap.add_argument("--sweep", default="", help="comma list of θ: per-θ aggregation times (Table III replica)")
    ap.add_argument("--f2", default="",
                    help="F2 sensitivity: 'L1,L2,..:H1,H2,..' epoch ms of the l-layer GCN over layers x hidden")
    ap.add_argument("--f3", type=int, default=0,
                    help="F3 convergence study (§V-E): epochs of Adam training, fp32 vs bf16 full mode")
    ap.add_argument("--f3-signal", type=float, default=0.015, help="F3: class-signal strength of the features")
    ap.add_argument("--f3-seeds", type=int, default=3, help="F3: initialisations")
    ap.add_argument("--table3", action="store_true",
                    help="Table III replica on RMAT-{0.1..10}: epoch ms of PCGCN-sel / -full / hybrid")
    ap.add_argument("--calib-curve", default="",
                    help="calibration curve (SURVEY §8(d)): 'F1,F2,..' widths; T_s(ρ), T_f per full-mode precision")
    return ap.parse_args()


def run_calib_curve(args):
    """The L161 calibration generalised to a curve: synthetic
    2048-row partition blocks joined by random bipartite blocks of density ρ,
    timed once all-selective (T_s) and once with the ρ-blocks in the full mode
    (T_f), per width F and full-mode precision; the break-even density is where
    T_s(ρ) = T_f (the θ L161 predicts from one point is T_f·p/T_s)."""
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    Fs = [int(x) for x in args.calib_curve.split(",")]
    dens = (0.0025, 0.005, 0.01, 0.02, 0.03, 0.05, 0.1, 0.2, 0.5)
    precs = {"bf16x3": L.DENSE_BF16X3, "bf16x1": L.DENSE_BF16X1, "tf32x2": L.DENSE_TF32X2}
    rows = []
    for pname in ("bf16x3", "bf16x1"):
        for F in Fs:
            pts = []
            for rho in dens:
                th, tf, ts = L.calibrate(F, 2048, rho, dense_prec=precs[pname])
                pts.append({"rho": rho, "T_full_ms": tf, "T_sel_ms": ts, "theta_L161": th})
                log(f"[calib] {pname} F={F} rho={rho} T_f={tf:.4f} T_s={ts:.4f} theta={th:.4f}")
            # break-even: first density where the full mode is not slower (linear interpolation)
            be = None
            for a, b in zip(pts, pts[1:]):
                da, db = a["T_sel_ms"] - a["T_full_ms"], b["T_sel_ms"] - b["T_full_ms"]
                if da < 0 <= db:
                    be = a["rho"] + (b["rho"] - a["rho"]) * (-da) / (db - da)
                    break
            if be is None and pts and pts[0]["T_sel_ms"] >= pts[0]["T_full_ms"]:
                be = dens[0]
            rows.append({"dense": pname, "F": F, "points": pts, "break_even_rho": be})
    print(json.dumps({"calib_curve": rows, "block_rows": 2048,
                      "note": "pcgcn_calibrate_prec: T_s = all-selective forward, T_f = the rho-blocks in the full "
                              "mode (diagonal self-loop blocks selective in both); L161 theta = T_f*rho/T_s"}),
          flush=True)


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ---------------------------------------------------------------------------
# clocks during the timed region
# ---------------------------------------------------------------------------
class ClockSampler:
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.lines = []
        if self.proc is not None:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                out = ""
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in getattr(self, "lines", []):
            f = [x.strip() for x in l.split(",")]
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except (ValueError, IndexError):
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------
# workload
# ---------------------------------------------------------------------------
def load_workload(name):
    from synth import configs as C
    w = C.WORKLOADS[name]
    t0 = time.time()
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    log(f"[bench] {name}: n={g.n} nnz(A)={g.nnz} generated in {time.time() - t0:.1f}s")
    return w, g, X, Th0, Th1, C.labels(w, g), T


def workload_str(w, g):
    """config.workload of both arms (the generator emits no duplicates or
    self-loops, so nnz(A+I) = nnz(A) + n)."""
    idx = {'cora': 0, 'pubmed': 1, 'reddit': 2, 'sbm4m': 3, 'pl32m': 4}.get(w.name)
    return (f"{w.name}-shaped DC-SBM (BASELINE configs[{idx}]) n={g.n} nnz(A+I)={g.nnz + g.n} "
            f"F={w.f_in}->{w.hidden}->{w.classes}")


HUGE_NNZ = 500_000_000  # C5-sized graphs: single calibrated plan, row-wise oracle sample, serial e2e


def _ld_bytes(F):
    """Row stride in bytes of an activation of width F (gcn._ld)."""
    return 4 * ((F + 3) // 4 * 4 if F <= 16 else (F + 15) // 16 * 16)


def hbm_peak():
    try:
        j = json.load(open(MEASURED_PEAKS))
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def agg_bytes(st, n, rows, F, dense_rows, nchunks):
    """Algorithmic HBM bytes of one aggregation call (SURVEY.md §8(d) B_min):
    index stream + row pointers + r + read Y once + write Z (+ Zd round trip
    for rows with full-mode blocks) + full-mode bit tiles."""
    nnz_s = st["shard_nnz_sparse"]
    b = nnz_s * 4 + (rows + 1) * 8 + rows * 4 + n * F * 4 + rows * F * 4
    b += 2 * dense_rows * F * 4 + nchunks * (512 + 4)
    return int(b)


def agg_bpc(st, rows, F, dense_rows, nchunks, bf3=False, bf1=False):
    """Partition-centric bytes model of one aggregation (SURVEY.md §8(d) B_pc;
    PAPER.md L129 §III-A.b): structure (indices, row pointers, r) + every
    destination partition's distinct selective source rows read once
    (stats shard_src_rows_pc) + the output + the full mode's bit tiles and
    B windows (one per chunk) + the Zd round trip of rows with chunks."""
    npad = (F + 15) // 16 * 16
    b = st["shard_nnz_sparse"] * 4 + (rows + 1) * 8 + rows * 4
    b += 4 * F * (st["shard_src_rows_pc"] + rows)
    b += nchunks * (516 + (6 if bf3 else 2 if bf1 else 8) * 32 * npad) + 2 * dense_rows * F * 4
    return int(b)


# ---------------------------------------------------------------------------
# oracle (CPU baseline / reference arm): bounded row sample of one epoch
# ---------------------------------------------------------------------------
class OracleSample:
    """Times the fp64 oracle's epoch operations restricted to a seeded random
    sample of output rows (fraction ``frac``) and extrapolates to the full
    epoch (x 1/frac).  Full-height inputs of each aggregation are prepared
    untimed (their values do not change the cost)."""

    def __init__(self, w, g, X, Th0, Th1, labels, T, frac, seed=7):
        from oracle import gcn as O
        self.O = O
        t0 = time.time()
        rng = np.random.default_rng(seed)
        H, C = Th0.shape[1], Th1.shape[1]
        self.rowwise = g.nnz > HUGE_NNZ
        if self.rowwise:
            # C5: scipy's Â (1e9 fp64 entries) and fp64 copies of X do not fit the
            # budget; the oracle's per-row definition (aggregate_rows, P15) on a
            # fixed 2,000-row sample, fp32 inputs (X itself: cost does not depend
            # on the values) converted to fp64 row by row
            self.g = g
            self.rows = np.sort(rng.choice(g.n, size=2000, replace=False))
            self.deg = O.clean_degrees(g.n, g.rowptr, g.col)
            self.YH, self.YC = X[:, :H], X[:, :C]
            self.XS = X[self.rows].astype(np.float64)
        else:
            self.Ahat = O.normalized_adjacency(g.n, g.rowptr, g.col)[0]
            self.rows = np.sort(rng.choice(g.n, size=max(1, int(g.n * frac)), replace=False))
            self.AS = self.Ahat[self.rows]
            self.XS = X[self.rows].astype(np.float64)
            self.YH = rng.standard_normal((g.n, H))
            self.YC = rng.standard_normal((g.n, C))
        self.frac = len(self.rows) / g.n
        self.Th0 = Th0.astype(np.float64)
        self.Th1 = Th1.astype(np.float64)
        self.labels = labels[self.rows]
        self.T = T[self.rows]
        self.nT = int(T.sum())
        log(f"[bench] oracle sample prepared in {time.time() - t0:.1f}s (frac={self.frac:.4f})")

    def _agg(self, Y):
        if self.rowwise:
            g = self.g
            return self.O.aggregate_rows(g.n, g.rowptr, g.col, Y, self.rows, deg=self.deg)
        return self.O.aggregate(self.AS, Y)

    def epoch_ms(self):
        O = self.O
        t0 = time.perf_counter()
        a1 = self.XS @ self.Th0                     # a4 (sampled rows)
        P1 = self._agg(self.YH)                     # a5/a6
        H1 = np.maximum(P1, 0.0)
        a2 = H1 @ self.Th1                          # a7
        Lg = self._agg(self.YC)                     # a8
        loss, dL = O.softmax_ce(Lg, self.labels, self.T)   # a9
        G1 = self._agg(self.YC)                     # a10
        g1 = H1.T @ G1                              # a11
        dP1 = (G1 @ self.Th1.T) * (P1 > 0)
        G0 = self._agg(self.YH)                     # a12
        g0 = self.XS.T @ G0                         # a13
        th0 = self.Th0 - 0.01 * g0                  # a14
        th1 = self.Th1 - 0.01 * g1
        del a1, a2, loss, dL, dP1, th0, th1
        return (time.perf_counter() - t0) * 1e3 / self.frac

    def cores(self):
        try:
            from threadpoolctl import threadpool_info
            blas = max([i.get("num_threads", 1) for i in threadpool_info()] or [1])
        except Exception:
            blas = 1
        return int(blas), len(os.sched_getaffinity(0))


def run_reference(args, rank, world):
    if rank != 0:
        return
    w, g, X, Th0, Th1, labels, T = load_workload(args.workload)
    osamp = OracleSample(w, g, X, Th0, Th1, labels, T, args.oracle_frac)
    for _ in range(args.warmup):
        osamp.epoch_ms()
    ts = [osamp.epoch_ms() for _ in range(args.steps)]
    v = float(np.mean(ts))
    blas, cores = osamp.cores()
    sample = (f"{len(osamp.rows)} seeded random output rows ({osamp.frac:.2%} of n) of every epoch op "
              f"(4 aggregations scipy fp64 single-threaded, GEMMs numpy BLAS {blas} threads), x1/frac: each "
              f"step times the sample and reports the epoch it extrapolates to (the full, unextrapolated "
              f"oracle epoch is profiles/r2_oracle_epoch.json)")
    line = {
        "impl": "reference", "metric": "2-layer GCN epoch ms",
        "value": v, "unit": "ms", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": v, "higher_is_better": False, "scaling": "strong", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_str(w, g),
                   "parallelism": "cpu", "extrapolated": True,
                   "sample_seconds_per_step": float(np.mean(ts)) * osamp.frac / 1e3},
        "cpu_baseline": {"value": v, "unit": "ms", "cores": blas, "host_cores": cores, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": v, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
# Table III replica
# ---------------------------------------------------------------------------
def run_table3(args):
    """Epoch ms of the 2-layer GCN on the regenerated RMAT series under three
    executors: PCGCN-sel (θ = 2: every block selective), PCGCN-full (θ = 0:
    every non-empty block in the tcgen05 full mode) and the hybrid PCGCN with
    θ from the paper's procedure (L161, pcgcn_calibrate) — plus the best
    hybrid over a θ grid.  The paper's claim (Table III): hybrid <= min(sel,
    full), full wins on the dense graphs.  CUDA-graph replays, median of
    ``--steps`` after ``--warmup``."""
    import torch
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    rows = []
    for d, w in C.RMAT.items():
        g = C.graph(w)
        resolve_plan_defaults(args, g)
        X = C.features(w, g.n)
        Th0, Th1 = C.thetas(w)
        T = C.train_mask(g.n, w.theta_seed)
        lab = C.labels(w, g)
        th0, _, _ = L.calibrate(w.hidden, max(64, g.n // w.P), 0.05)
        ent = {"workload": w.name, "n": g.n, "nnz": int(g.nnz + g.n), "P": w.P, "F": f"{w.f_in}->{w.hidden}->{w.classes}",
               "theta_L161": th0}

        def epoch_ms(theta):
            pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, f_max=max(w.hidden, w.classes), **plan_kw(args))
            perm = pl.perm()
            m = GCN2(pl, np.ascontiguousarray(X[perm]), lab[perm], T[perm], Th0, Th1, optimizer="adam", lr=0.01,
                     device=dev)
            m.capture(warmup=1)
            for _ in range(max(3, args.warmup)):
                m.replay()
            ts = []
            for _ in range(args.steps):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                m.replay()
                b.record()
                torch.cuda.synchronize(dev)
                ts.append(a.elapsed_time(b))
            st = pl.stats()
            del m
            pl.destroy()
            return float(np.median(ts)), st["nnz_dense"] / st["nnz"]
        ent["sel_ms"], _ = epoch_ms(2.0)
        ent["full_ms"], _ = epoch_ms(0.0)
        ent["hybrid_ms"], ent["hybrid_dense_frac"] = epoch_ms(th0)
        grid = {}
        for th in (0.01, 0.02, 0.05, 0.1, 0.2, 0.4):
            grid[th] = epoch_ms(th)
        ent["grid"] = {str(k): {"ms": v[0], "dense_frac": v[1]} for k, v in grid.items()}
        grid = {k: v[0] for k, v in grid.items()}
        bt = min(grid, key=grid.get)
        ent["hybrid_grid_best"] = {"theta": bt, "ms": grid[bt]}
        ent["ordering_holds"] = ent["hybrid_ms"] <= 1.05 * min(ent["sel_ms"], ent["full_ms"])
        ent["ordering_holds_grid"] = grid[bt] <= min(ent["sel_ms"], ent["full_ms"])
        ent["plan"] = {"order": args.order, "grain": args.grain, "dense": args.dense}
        log(f"[table3] {ent}")
        rows.append(ent)
    print(json.dumps({"table3": rows, "metric": "2-layer GCN epoch ms", "unit": "ms", "steps": args.steps,
                      "model": "2-layer GCN (hid 64, Adam), synthetic RMAT (a,b,c,d)=(0.45,0.22,0.22,0.11)",
                      "paper": "Table III L263-L281 (l=4, hid=64, 1080Ti/2080Ti) — context"}), flush=True)


def run_f3(args):
    """SURVEY F3 / PAPER.md §V-E (L330-L334, Fig. 9): test accuracy of the
    same 2-layer GCN trained with the exact fp32 selective mode (θ = 2), the
    fp32-accurate hybrid (tf32 hi/lo full mode), the bf16 hybrid and the bf16
    all-full executor (PCGCN_DENSE_BF16X1: the paper's 16-bit tensor-core
    policy), 80/20 split, over ``--f3-seeds`` initialisations.  The features
    carry a WEAK class signal (class mean vectors x ``--f3-signal`` added to
    the synthetic features; 0.015 puts the fp32 test accuracy of C2 in the
    70-90% band, tuned with the fp64 oracle) so the task does not saturate and
    a precision effect could show.  Reports each variant's accuracy delta to
    fp32 per seed and its mean / max."""
    import torch
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    w, g, X, Th0, Th1, labels, T = load_workload(args.workload)
    resolve_plan_defaults(args, g)
    mu = np.random.default_rng([w.feat_seed, 99]).standard_normal((w.classes, w.f_in)).astype(np.float32)
    X = (X + args.f3_signal * mu[labels]).astype(np.float32)
    theta_h = float(args.theta) if args.theta != "auto" else 0.05
    variants = [("fp32_selective", 2.0, L.DENSE_TF32X2), ("tf32x2_hybrid", theta_h, L.DENSE_TF32X2),
                ("bf16_hybrid", theta_h, L.DENSE_BF16X1), ("bf16_full", 0.0, L.DENSE_BF16X1)]
    seeds = list(range(args.f3_seeds))
    curves = {name: {"per_seed": []} for name, _, _ in variants}
    for sd in seeds:
        th0 = C.glorot(w.f_in, w.hidden, w.theta_seed + 100 * sd, 0)
        th1 = C.glorot(w.hidden, w.classes, w.theta_seed + 100 * sd, 1)
        for name, th, prec in variants:
            kw = plan_kw(args)
            kw["dense_prec"] = prec
            pl = L.Plan(g.n, g.rowptr, g.col, args.P or w.P, th, f_max=max(w.hidden, w.classes), **kw)
            perm = pl.perm()
            lab = labels[perm]
            test = torch.from_numpy(~T[perm]).to(dev)
            labd = torch.from_numpy(lab.astype(np.int64)).to(dev)
            m = GCN2(pl, np.ascontiguousarray(X[perm]), lab, T[perm], th0, th1, optimizer="adam", lr=0.01,
                     device=dev)
            acc = []
            for ep in range(args.f3):
                m.epoch()
                if ep % 10 == 9 or ep == args.f3 - 1:
                    pred = m.Lg[:, :w.classes].argmax(dim=1)   # logits of the forward just run
                    acc.append(float((pred[test] == labd[test]).float().mean().item()))
            st = pl.stats()
            curves[name]["per_seed"].append({"seed": sd, "final_test_acc": acc[-1], "test_acc_every10": acc,
                                             "dense_edge_frac": st["nnz_dense"] / st["nnz"], "theta": th})
            log(f"[f3] seed {sd} {name}: {acc[-1]:.4f} dense={st['nnz_dense'] / st['nnz']:.3f}")
            del m
            pl.destroy()
    for name in curves:
        d = [curves[name]["per_seed"][i]["final_test_acc"] - curves["fp32_selective"]["per_seed"][i]["final_test_acc"]
             for i in range(len(seeds))]
        curves[name]["acc_delta_vs_fp32"] = d
        curves[name]["acc_delta_mean"] = float(np.mean(d))
        curves[name]["acc_delta_max_abs"] = float(np.max(np.abs(d)))
        curves[name]["final_test_acc_mean"] = float(np.mean([e["final_test_acc"] for e in curves[name]["per_seed"]]))
    print(json.dumps({"f3": curves, "workload": w.name, "epochs": args.f3, "optimizer": "adam lr 0.01",
                      "signal": args.f3_signal, "seeds": len(seeds),
                      "paper": "§V-E: PCGCN-TC accuracy drop 0.08% (pubmed), 0.19% (reddit-s) — context"}), flush=True)


def run_f2(args):
    """the paper-shaped l-layer model (Table II: l = 4, hid = 64,
    L255) and its sensitivity to the hidden size and depth (L314, L326: the
    runtime grows ~linearly in both) on one workload; one plan (θ fixed or
    the L161 calibration at the first hidden size), CUDA-graph replays."""
    import torch
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCNL
    from synth import configs as C
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    w, g, X, Th0, Th1, labels, T = load_workload(args.workload)
    layers_s, hid_s = args.f2.split(":")
    layers = [int(x) for x in layers_s.split(",")]
    hids = [int(x) for x in hid_s.split(",")]
    P = args.P or w.P
    if args.theta == "auto":
        theta, _, _ = L.calibrate(hids[0], max(64, min(8192, g.n // P)), 0.05)
    else:
        theta = float(args.theta)
    pl = L.Plan(g.n, g.rowptr, g.col, P, theta, f_max=max(max(hids), w.classes))
    perm = pl.perm()
    Xp = np.ascontiguousarray(X[perm])
    out = []
    for nl in layers:
        for h in hids:
            dims = [w.f_in] + [h] * (nl - 1) + [w.classes]
            ths = [C.glorot(dims[i], dims[i + 1], w.theta_seed, 20 + i) for i in range(nl)]
            m = GCNL(pl, Xp, labels[perm], T[perm], ths, optimizer="adam", lr=0.01, device=dev)
            m.capture(warmup=1)
            for _ in range(max(3, args.warmup)):
                m.replay()
            ts = []
            for _ in range(args.steps):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                m.replay()
                b.record()
                torch.cuda.synchronize(dev)
                ts.append(a.elapsed_time(b))
            ent = {"layers": nl, "hidden": h, "epoch_ms": float(np.median(ts))}
            log(f"[f2] {ent}")
            out.append(ent)
            del m
            torch.cuda.empty_cache()
    print(json.dumps({"f2": out, "workload": w.name, "n": g.n, "nnz": int(g.nnz + g.n), "P": P, "theta": theta,
                      "metric": "l-layer GCN epoch ms", "unit": "ms", "steps": args.steps,
                      "paper": "Table II model l=4 hid=64 (L255); sensitivity L314/L326 — context"}), flush=True)


# ---------------------------------------------------------------------------
# our arm
# ---------------------------------------------------------------------------
def resolve_plan_defaults(args, g):
    """--order/--grain auto: degree order + per-chunk modes where the full mode
    pays (C3: 9.6 -> 8.3 ms), the paper's id order + per-block modes on
    C5-sized graphs, where chunks of hub rows cost a full-height window split
    (15 ms per F=128 call) for no selective-pass saving (measured: 212 vs 160 ms
    epoch, profiles/r2_c5_*.json)."""
    huge = g.nnz > HUGE_NNZ
    if args.order == "auto":
        args.order = "id" if huge else "degree"
    if args.grain == "auto":
        args.grain = "block" if huge else "tile"


def plan_kw(args):
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    return dict(order=L.ORDER_DEGREE if args.order == "degree" else L.ORDER_ID,
                grain=L.GRAIN_TILE if args.grain == "tile" else L.GRAIN_BLOCK,
                dense_prec={"bf16x3": L.DENSE_BF16X3, "bf16x1": L.DENSE_BF16X1}.get(args.dense, L.DENSE_TF32X2))


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    import torch
    import torch.distributed as dist
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    if args.impl == "reference":
        run_reference(args, rank, world)
        if world > 1:
            dist.destroy_process_group()
        return
    if args.table3:
        run_table3(args)
        return
    if args.calib_curve:
        run_calib_curve(args)
        return
    if args.f2:
        run_f2(args)
        return
    if args.f3:
        run_f3(args)
        return

    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from paper_conf_ipps_tianmyd20_b200.dist import RowExchange

    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    w, g, X, Th0, Th1, labels, T = load_workload(args.workload)
    resolve_plan_defaults(args, g)
    P = args.P or w.P
    fmax = max(w.hidden, w.classes)
    theta_c = None
    if args.theta == "auto":
        # 1) the paper's procedure (L161) on synthetic p-blocks -> initial θ0
        avg_part = max(64, min(8192, g.n // P))
        theta0, t_f, t_s = L.calibrate(w.hidden, avg_part, 0.05)
        theta_src = (f"L161 synthetic: T_f={t_f:.4f}ms T_s={t_s:.4f}ms at p=0.05 ({avg_part}-row blocks, F={w.hidden})"
                     f" -> theta0={theta0:.4g}; ")
    if args.theta == "auto" and g.nnz > HUGE_NNZ:
        # C5: every plan costs ~a minute of host time and Y' buffers of 17 GB:
        # the paper's procedure alone (L161), one plan for both widths
        theta = theta0
        theta_src += "single plan (C5-sized graph: no in-situ refinement / grid)"
    elif args.theta == "auto":
        # 2) in-situ refinement per width on this workload (pcgcn_refine_theta)
        pl0 = L.Plan(g.n, g.rowptr, g.col, P, theta0, f_max=fmax, rank=rank, world=world, **plan_kw(args))
        perm = pl0.perm()
        Xp = np.ascontiguousarray(X[perm])
        m0 = GCN2(pl0, Xp, labels[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.0, device=dev,
                  exchange=RowExchange(pl0.row_lo, pl0.row_hi) if world > 1 else None)
        m0.epoch()
        torch.cuda.synchronize(dev)
        thH, ccH, ceH = L.refine_theta(pl0, m0.Y0, m0.H1, w.hidden)
        thC, ccC, ceC = L.refine_theta(pl0, m0.Y1, m0.Lg, w.classes)
        theta_src += (f"in-situ linear: F={w.hidden} {ccH:.2f} ns/chunk {ceH:.4f} ns/edge -> {thH:.4g}, "
                      f"F={w.classes} {ccC:.2f} ns/chunk {ceC:.4f} ns/edge -> {thC:.4g}; ")
        Y0, Y1 = m0.Y0.clone(), m0.Y1.clone()
        del m0, pl0
        # 3) measured choice: time both widths on plans over a θ grid, keep the fastest per width
        #    (large graphs: the in-situ estimates plus the L161 value only — each plan costs seconds)
        if g.nnz < 200_000_000:
            base = ((0.02, 0.03, 0.045, 0.06, 0.08, 0.11, 0.15) if args.grain == "tile"
                    else (0.01, 0.014, 0.02, 0.028, 0.04, 0.056, 0.08))
            grid = sorted({round(x, 4) for x in (*base, thH, thC) if x > 0})
        else:
            grid = sorted({round(x, 5) for x in (thH, thC, theta0) if x > 0})
        ZH = torch.empty(g.n, Y0.shape[1], device=dev)
        ZC = torch.empty(g.n, Y1.shape[1], device=dev)
        widths = ((w.hidden, Y0, ZH), (w.classes, Y1, ZC))

        def time_fwd(pt, F, Yin, Zout, reps):
            ts = []
            for it in range(reps + 1):
                a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a_.record()
                pt.forward(Yin, Zout, F=F, flags=L.IN_PRESCALED)
                b_.record()
                torch.cuda.synchronize(dev)
                if it:
                    ts.append(a_.elapsed_time(b_))
            t = float(np.median(ts))
            if world > 1:
                tt = torch.tensor([t], device=dev)
                dist.all_reduce(tt, op=dist.ReduceOp.MAX)
                t = float(tt.item())
            return t

        # stage 1: every grid θ, 6 timed calls per width; stage 2: the 3 best per
        # width again, interleaved, 3 x 8 calls (run-to-run noise of single
        # forward timings is ~2%, about the gap between neighbouring θ)
        plans, t1 = {}, {F: {} for F, _, _ in widths}
        for th in grid:
            plans[th] = L.Plan(g.n, g.rowptr, g.col, P, th, f_max=fmax, rank=rank, world=world, **plan_kw(args))
            for F, Yin, Zout in widths:
                t1[F][th] = time_fwd(plans[th], F, Yin, Zout, 6)
        best = {}
        for F, Yin, Zout in widths:
            top = sorted(t1[F], key=t1[F].get)[:3]
            acc = {th: [] for th in top}
            for _ in range(3):
                for th in top:
                    acc[th].append(time_fwd(plans[th], F, Yin, Zout, 8))
            tb = {th: float(np.median(v)) for th, v in acc.items()}
            bt = min(tb, key=tb.get)
            best[F] = (bt, tb[bt])
        for pt in plans.values():
            pt.destroy()
        del plans
        theta, theta_c = best[w.hidden][0], best[w.classes][0]
        theta_src += (f"measured grid {grid} (3 best re-timed): F={w.hidden} -> {theta} ({best[w.hidden][1]:.3f} ms), "
                      f"F={w.classes} -> {theta_c} ({best[w.classes][1]:.3f} ms)")
        del Y0, Y1, ZH, ZC
    else:
        theta, theta_src = float(args.theta), "fixed"
        theta_c = args.theta_c
    t0 = time.time()
    pl = L.Plan(g.n, g.rowptr, g.col, P, theta, f_max=fmax, rank=rank, world=world, **plan_kw(args))
    pl_c = L.Plan(g.n, g.rowptr, g.col, P, theta_c, f_max=fmax, rank=rank, world=world, **plan_kw(args)) if theta_c else None
    st = pl.stats()
    st_c = pl_c.stats() if pl_c else st
    log(f"[bench] plans in {time.time() - t0:.1f}s theta={theta:.4g} theta_c={theta_c} ({theta_src}) stats={st}")
    perm = pl.perm()
    Xp = np.ascontiguousarray(X[perm])
    exch = RowExchange(pl.row_lo, pl.row_hi) if world > 1 else None
    model = GCN2(pl, Xp, labels[perm], T[perm], Th0, Th1, optimizer="adam", lr=0.01, device=dev, exchange=exch,
                 plan_c=pl_c, fuse_split=args.fuse_split == "on")
    use_graph = world == 1 and not args.eager
    stream = torch.cuda.current_stream(dev)
    if use_graph:
        model.capture(warmup=1)

    def step():
        if use_graph:
            model.replay()
        else:
            model.epoch()

    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize(dev)

    # ---- timed region ----
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with ClockSampler(local) as clk:
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        for i in range(args.steps):
            flush.zero_()
            evs[i][0].record()
            step()
            evs[i][1].record()
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
    times = [a.elapsed_time(b) for a, b in evs]
    ms = float(np.mean(times))
    if world > 1:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    clocks = clk.summary()

    # ---- instrumented eager pass: per-step durations on the launching stream ----
    names, marks = [], []

    def hook(name):
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        names.append(name)
        marks.append(e)

    per = {}
    kern = {}  # per-kernel event times inside each aggregation call (PCGCN_PROFILE)
    reps = 3
    for _ in range(reps):
        names.clear(); marks.clear()
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e0.record()
        model.epoch(hook=hook, agg_flags=L.PROFILE)
        torch.cuda.synchronize(dev)
        prev = e0
        for nm, e in zip(names, marks):
            per[nm] = per.get(nm, 0.0) + prev.elapsed_time(e) / reps
            prev = e
    # the PROFILE events of the last call of each aggregation are re-read per call:
    # run each aggregation once more in isolation to attribute kernel times
    for nm, plan_k, fn in (("a5a6_agg_fwd_H", pl,
                            lambda: pl.forward(model.Y0, model.H1, F=w.hidden,
                                               flags=L.IN_PRESCALED | L.RELU | L.MASK_OUT | L.PROFILE,
                                               mask=model.mask1)),
                           ("a8_agg_fwd_C", model.plan_c,
                            lambda: model.plan_c.forward(model.Y1, model.Lg, F=w.classes,
                                                         flags=L.IN_PRESCALED | L.PROFILE))):
        acc = {}
        for _ in range(reps):
            flush.zero_()
            fn()
            for k, v in plan_k.last_timings().items():
                acc[k] = acc.get(k, 0.0) + v / reps
        kern[nm] = acc
    peak, peak_src = hbm_peak()
    # L2-resident stream: the gather kernels' on-chip roofline.  Single probes
    # vary run to run (11.6 vs 17.2 TB/s seen at 64 MiB), so take the best of
    # 3 repetitions at each of several L2-resident sizes.
    l2_gbs = max(L.probe_read_gbs(mb << 20, 50) for mb in (16, 32, 48, 64) for _ in range(3))
    hbm_probe = L.probe_read_gbs(4 << 30, 3)
    # random-row gather ceilings at the kernel's row size (pcgcn_probe_gather_gbs):
    # rows served by L1 (64 KB buffer), by L2 (64 MB) and by HBM (4 GB)
    rb = _ld_bytes(w.hidden)
    gprobe = {lvl: max(L.probe_gather_gbs(nb, rb, 256) for _ in range(3))
              for lvl, nb in (("l1", 64 << 10), ("l2", 64 << 20), ("hbm", 4 << 30))}
    rows = pl.row_hi - pl.row_lo
    dense_rows = int(st["row_tiles"]) * 128 if world == 1 else int(st["shard_chunks"] > 0) * rows
    bH = agg_bytes(st, g.n, rows, w.hidden, dense_rows, st["shard_chunks"])
    bC = agg_bytes(st_c, g.n, rows, w.classes, int(st_c["row_tiles"]) * 128 if world == 1 else rows, st_c["shard_chunks"])
    t_agg = per["a5a6_agg_fwd_H"]
    agg_total = sum(per[k] for k in per if "agg" in k)
    # dominant kernel: the selective gather of the F=H aggregations (largest share of the epoch)
    t_sp = kern["a5a6_agg_fwd_H"]["sparse"]
    fp4 = (w.hidden + 3) // 4 * 4
    b_sp = (st["shard_nnz_sparse"] * 4 + (rows + 1) * 8 + rows * 4 + g.n * w.hidden * 4 + rows * w.hidden * 4
            + dense_rows * w.hidden * 4 + rows * ((w.hidden + 31) // 32) * 4)
    achieved = b_sp / (t_sp * 1e-3) / 1e9
    gather = st["shard_nnz_sparse"] * fp4 * 4 / (t_sp * 1e-3) / 1e9
    t_tc = kern["a5a6_agg_fwd_H"]["dense_tc"]
    npad = (w.hidden + 15) // 16 * 16
    bf3 = args.dense == "bf16x3"
    bf16 = args.dense in ("bf16x3", "bf16x1")
    # executed MMA flops per chunk: 2 (hi, lo) tf32 products, 3 bf16 parts, or 1 bf16 product
    tc_flops = st["shard_chunks"] * 2 * 128 * 32 * npad * {"bf16x3": 3, "bf16x1": 1}.get(args.dense, 2)
    tc_tf = tc_flops / (t_tc * 1e-3) / 1e12 if t_tc > 0 else None
    try:
        tc_peak = float(json.load(open(MEASURED_PEAKS))["bf16_tflops"]) / (1 if bf16 else 2)
    except Exception:
        tc_peak = 1590.0 / (1 if bf16 else 2)
    traffic = l2_read = lts_pct = dram_pct = None
    traffic_cfg = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        try:
            tj = json.load(open(tpath)).get(w.name, {})
            traffic = tj.get("sparse_agg_F%d" % w.hidden)
            l2_read = tj.get("sparse_agg_F%d_l2_read_bytes" % w.hidden)
            lts_pct = tj.get("sparse_agg_F%d_lts_pct" % w.hidden)
            dram_pct = tj.get("sparse_agg_F%d_dram_pct" % w.hidden)
            traffic_cfg = tj.get("config")
        except Exception:
            traffic = None
    # the binding unit of the selective gather per its ncu capture: the L2 (LTS)
    # or HBM, whichever runs closer to its sustained peak
    l2_bound = lts_pct is not None and l2_read and (dram_pct is None or lts_pct >= dram_pct)

    # ---- e2e: host buffers, H2D of the step's inputs and D2H of the loss inside the region ----
    e2e = None
    if not args.no_e2e:
        Xh = torch.zeros(model.X.shape, dtype=torch.float32).pin_memory()  # same padded layout as model.X
        Xh[:, :w.f_in] = torch.from_numpy(np.ascontiguousarray(Xp[pl.row_lo:pl.row_hi]))
        lab_h = model.labels.cpu().pin_memory()
        tr_h = model.train.cpu().pin_memory()
        loss_h = torch.empty(1, dtype=torch.float32).pin_memory()
        h2d = Xh.numel() * 4 + lab_h.numel() * 4 + tr_h.numel()
        # (a) serial: copy the step's inputs, run it, read the loss back — per-step events
        e2e_ev = []
        for i in range(args.steps):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            model.X.copy_(Xh, non_blocking=True)
            model.labels.copy_(lab_h, non_blocking=True)
            model.train.copy_(tr_h, non_blocking=True)
            step()
            loss_h.copy_(model.loss, non_blocking=True)
            b.record()
            e2e_ev.append((a, b))
        torch.cuda.synchronize(dev)
        serial_ms = float(np.mean([a.elapsed_time(b) for a, b in e2e_ev]))
    if not args.no_e2e and g.nnz > HUGE_NNZ:
        # C5: a second set of device inputs (17 GB of X) does not fit next to the
        # epoch's buffers: the serial path (copy, step, read back) is the e2e value
        if world > 1:
            t = torch.tensor([serial_ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            serial_ms = float(t[0])
        e2e = {"value": serial_ms, "unit": "ms", "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": 4,
               "pipeline": "serial: H2D of the step's inputs, the epoch, D2H of the loss"}
    elif not args.no_e2e:
        # (b) pipelined input path (double-buffered inputs, copy stream): step k+1's
        #     H2D overlaps step k's epoch; every step still copies its inputs from
        #     pinned host memory and reads its loss back inside the timed region
        bufs = [(model.X, model.labels, model.train),
                (model.X.clone(), model.labels.clone(), model.train.clone())]
        graphs = []
        if use_graph:
            for bx in bufs:
                model.X, model.labels, model.train = bx
                graphs.append(model.capture(warmup=1))
        model.X, model.labels, model.train = bufs[0]
        cs = torch.cuda.Stream(device=dev)
        cur = torch.cuda.current_stream(dev)
        ev_copy = [torch.cuda.Event() for _ in range(2)]
        ev_done = [torch.cuda.Event() for _ in range(2)]
        loss_hs = [torch.empty(1, dtype=torch.float32).pin_memory() for _ in range(args.steps)]

        def copy_into(bi):
            with torch.cuda.stream(cs):
                for dst, src in zip(bufs[bi], (Xh, lab_h, tr_h)):
                    dst.copy_(src, non_blocking=True)
                ev_copy[bi].record(cs)

        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        e_a, e_b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e_a.record(cur)
        cs.wait_event(e_a)
        copy_into(0)
        for k in range(args.steps):
            bi = k % 2
            cur.wait_event(ev_copy[bi])
            if use_graph:
                graphs[bi].replay()
            else:
                model.X, model.labels, model.train = bufs[bi]
                model.epoch()
            loss_hs[k].copy_(model.loss, non_blocking=True)
            ev_done[bi].record(cur)
            if k + 1 < args.steps:
                nb = (k + 1) % 2
                if k >= 1:
                    cs.wait_event(ev_done[nb])  # buffer nb was read by step k-1
                copy_into(nb)
        e_b.record(cur)
        torch.cuda.synchronize(dev)
        e2e_ms = e_a.elapsed_time(e_b) / args.steps
        model.X, model.labels, model.train = bufs[0]
        if use_graph:
            model._graph = graphs[0]
        if world > 1:
            t = torch.tensor([e2e_ms, serial_ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_ms, serial_ms = float(t[0]), float(t[1])
        e2e = {"value": e2e_ms, "unit": "ms", "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": 4,
               "pipeline": "double-buffered inputs on a copy stream: step k+1's H2D overlaps step k",
               "serial_value": serial_ms}

    sweep = None
    if args.sweep:
        # Table III replica (L263-L281): forward aggregation at both widths per θ
        # (θ >= 1: PCGCN-sel; small θ: full mode for every block above it; the
        # hybrid = the calibrated plans above).  Times: median of 3 warm calls.
        sweep = []
        ZH = torch.empty(model.H1.shape, device=dev)
        ZC = torch.empty(model.Lg.shape, device=dev)
        for th in [float(x) for x in args.sweep.split(",")]:
            try:
                pt = L.Plan(g.n, g.rowptr, g.col, P, th, f_max=fmax, rank=rank, world=world, **plan_kw(args))
            except Exception as e:  # e.g. a full-mode plan that does not fit (the paper's "oom", L276)
                sweep.append({"theta": th, "error": str(e)[:120]})
                continue
            ent = {"theta": th, "nnz_dense": pt.stats()["nnz_dense"], "chunks": pt.stats()["chunks"]}
            for key, F, Yin, Zout in (("agg_ms_H", w.hidden, model.Y0, ZH), ("agg_ms_C", w.classes, model.Y1, ZC)):
                ts = []
                for it in range(4):
                    a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a_.record()
                    pt.forward(Yin, Zout, F=F, flags=L.IN_PRESCALED)
                    b_.record()
                    torch.cuda.synchronize(dev)
                    if it:
                        ts.append(a_.elapsed_time(b_))
                ent[key] = float(np.median(ts))
            pt.destroy()
            sweep.append(ent)
            log(f"[bench] sweep {ent}")

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            osamp = OracleSample(w, g, X, Th0, Th1, labels, T, args.oracle_frac)
            v = float(np.mean([osamp.epoch_ms() for _ in range(2)]))
            blas, cores = osamp.cores()
            cpu = {"value": v, "unit": "ms", "cores": blas, "host_cores": cores, "kind": "oracle",
                   "sample": f"{len(osamp.rows)} seeded random output rows ({osamp.frac:.2%}) of every epoch op, "
                             f"extrapolated x1/frac; scipy SpMM single-threaded, numpy GEMMs {blas} BLAS threads"}
        except Exception as e:  # the baseline must never break the GPU line
            cpu = {"value": None, "unit": "ms", "cores": None, "kind": "oracle", "sample": f"failed: {e}"}

    if rank == 0:
        line = {
            "metric": "2-layer GCN epoch ms", "value": ms, "unit": "ms", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None,
            "dtype": "f32" if args.dense != "bf16x1" else "f32 (selective) + bf16 (full mode, fp32 accumulate)",
            "data": "synthetic",
            "config": {
                "workload": workload_str(w, g),
                "P": P, "theta": theta, "theta_c": theta_c if theta_c else theta, "theta_source": theta_src, "optimizer": "adam",
                "plan_options": {"vertex_order": args.order, "mode_grain": args.grain, "dense_prec": args.dense,
                                 "fused_split": bool(model.fuse)},
                "parallelism": f"dp-rows{world}" if world > 1 else "single",
                "l2": "flushed (256 MiB write) between timed steps",
                "cuda_graph": use_graph,
                "plan": {k: st[k] for k in ("blocks_nonempty", "blocks_dense", "nnz_sparse", "nnz_dense",
                                            "row_tiles", "chunks", "intra_edges", "lp_sweeps", "clusters",
                                            "partition_ms", "plan_ms")},
            },
            "roofline": {"kernel": "sparse_agg (selective-mode gather), layer-1 forward, F=%d" % w.hidden,
                         "bound": "l2" if l2_bound else "hbm",
                         "achieved": (l2_read / (t_sp * 1e-3) / 1e9) if l2_bound else achieved,
                         "peak": (l2_read / (t_sp * 1e-3) / 1e9 / (lts_pct / 100.0)) if l2_bound else peak,
                         "unit": "GB/s",
                         "frac": (lts_pct / 100.0) if l2_bound else achieved / peak,
                         "traffic": traffic,
                         "peak_source": ("L2: achieved L2->L1 bytes per launch (ncu) / live event time, against the "
                                         "LTS sustained peak ncu reports for this kernel (lts__throughput % of peak, "
                                         "the most-utilised unit); HBM view below") if l2_bound else peak_src,
                         "hbm_view": {"algorithmic_bytes": b_sp, "achieved": achieved, "peak": peak, "frac": achieved / peak,
                                      "peak_source": peak_src, "ncu_dram_pct": dram_pct,
                                      "dram_bytes_per_launch": traffic},
                         "algorithmic_bytes": b_sp, "ms": t_sp,
                         "traffic_source": "profiles/traffic.json (ncu --set full, dram read+write per launch)",
                         "traffic_config": traffic_cfg,
                         "l2_view": {"l2_read_bytes": l2_read,
                                     "achieved": (l2_read / (t_sp * 1e-3) / 1e9) if l2_read else None,
                                     "unit": "GB/s",
                                     "ncu_lts_throughput_pct": lts_pct,
                                     "bytes_source": "ncu lts__t_sectors_srcunit_tex_op_read x 32 per launch "
                                                     "(profiles/traffic.json); ncu_lts_throughput_pct = the L2's "
                                                     "own %-of-peak (lts__throughput), time-weighted over the pass",
                                     "probe_peak": l2_gbs,
                                     "probe_note": "streaming-read probe; the gather's L2->L1 rate exceeds it "
                                                   "(partition-ordered rows), so the ncu % is the L2 roofline",
                                     "gather_bytes": st["shard_nnz_sparse"] * fp4 * 4,
                                     "gather_GBs": gather,
                                     "peak_source": "measured: max of pcgcn_probe_read_gbs over 16-64 MiB L2-resident buffers, 3 reps each"},
                         "hbm_probe_GBs": hbm_probe,
                         "gather_view": {"row_bytes": rb, "rows": st["shard_nnz_sparse"],
                                         "achieved": st["shard_nnz_sparse"] * rb / (t_sp * 1e-3) / 1e9,
                                         "unit": "GB/s",
                                         "ceilings": gprobe,
                                         "frac_of_l2_ceiling": st["shard_nnz_sparse"] * rb / (t_sp * 1e-3) / 1e9 / gprobe["l2"],
                                         "frac_of_hbm_ceiling": st["shard_nnz_sparse"] * rb / (t_sp * 1e-3) / 1e9 / gprobe["hbm"],
                                         "source": "pcgcn_probe_gather_gbs: the kernel's access pattern (random "
                                                   "rows of row_bytes, 8 in flight per lane, 32 warps/SM) from "
                                                   "64 KB / 64 MB / 4 GB buffers, best of 3"}},
            "bytes_views": {
                "aggregation": f"layer-1 forward, F={w.hidden} (selective + full mode)",
                "B_min": bH, "B_pc": agg_bpc(st, rows, w.hidden, dense_rows, st["shard_chunks"], args.dense == "bf16x3",
                                 args.dense == "bf16x1"),
                "ncu_dram_selective": traffic,
                "dram_over_B_min_selective": (traffic / b_sp) if traffic else None,
                "src_rows_pc": st["shard_src_rows_pc"],
                "note": "B_min = compulsory bytes; B_pc = each destination partition reads its distinct selective "
                        "sources once; ncu DRAM bytes of the selective kernels per launch (cold cache)"},
            "tensor_view": {"kernel": "tc_engine<A_BITS> full-mode tiles, layer-1 forward",
                            "ms": t_tc, "achieved": tc_tf, "unit": "TFLOP/s (bf16)" if bf16 else "TFLOP/s (tf32)",
                            "peak": tc_peak, "frac": (tc_tf / tc_peak) if tc_tf else None,
                            "peak_source": ("measured bf16 dense (MEASURED_PEAKS.json)" if bf16 else
                                            "measured bf16 dense (MEASURED_PEAKS.json) x 0.5 (tf32:bf16 nominal ratio)")},
            "agg_kernels_ms": kern,
            "agg_GBs": {"fwd_H": bH / (per["a5a6_agg_fwd_H"] * 1e-3) / 1e9,
                        "fwd_C": bC / (per["a8_agg_fwd_C"] * 1e-3) / 1e9,
                        "bwd_C": bC / (per["a10_agg_bwd_C"] * 1e-3) / 1e9,
                        "bwd_H": bH / (per["a12_agg_bwd_H"] * 1e-3) / 1e9},
            "step_breakdown_ms": {k: round(v, 4) for k, v in per.items()},
            "agg_share": agg_total / max(sum(per.values()), 1e-9),
            "theta_sweep": sweep,
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": model.launches_per_epoch() * args.steps,
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
