"""2-layer GCN training step on the PCGCN C ABI.

Alg. 1 with L = 2 — per layer: transform a^l = h^{l-1} w^l
(L114, pcgcn_gemm_xw) then partition-centric propagation (L118-L121,
pcgcn_forward) — followed by the softmax-CE loss, the backward through both
layers (pcgcn_backward reuses the forward plan since Âᵀ = Â) and the update.
PyTorch only owns device memory, the stream and (optionally) the CUDA graph;
every arithmetic step runs in libpcgcn's kernels.

Prescaling: Â = D̃^-½ Ã D̃^-½, so every producer of an aggregation input writes
diag(r)·Y (r = d̃^-½) and the aggregation applies r_i once in its epilogue:
    a4  Y0' = diag(r)·X·Θ0                 gemm_xw(rowscale=r)
    a5/6 H1 = ReLU(Â X Θ0), mask1          forward(IN_PRESCALED|RELU|MASK_OUT)
    a7  Y1' = diag(r)·H1·Θ1                gemm_xw(rowscale=r)
    a8  Lg  = Â H1 Θ1                      forward(IN_PRESCALED)
    a9  loss, dL' = diag(r)·dL             softmax_ce(rowscale=r)
    a10 G1  = Â dL                          backward(IN_PRESCALED)
    a11 ∇Θ1 = H1ᵀ G1 ; dP1' = diag(r)((G1Θ1ᵀ)⊙mask1)   gemm_xtg, gemm_dwt
    a12 G0  = Â dP1                         backward(IN_PRESCALED)
    a13 ∇Θ0 = Xᵀ G0                         gemm_xtg
    a14 Θ ← Adam/SGD(Θ, ∇Θ)  (all-reduce of ∇Θ first when sharded)
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _lib as L


def _ld(F: int) -> int:
    """Row stride (floats) of an activation of width F: 16-byte rows, and
    64-byte rows above 16 features so a gathered row touches the fewest
    128-byte lines (F=41: 48, two lines per row at any row index)."""
    return (F + 3) // 4 * 4 if F <= 16 else (F + 15) // 16 * 16


class GCN2:
    def __init__(self, plan: L.Plan, X_plan: np.ndarray, labels_plan: np.ndarray, train_plan: np.ndarray,
                 Th0: np.ndarray, Th1: np.ndarray, *, optimizer: str = "adam", lr: float = 0.01,
                 device: str | torch.device = "cuda", exchange=None, plan_c: L.Plan | None = None,
                 narrow: bool = False, fuse_split: bool = True):
        """All row-indexed host arrays are already in plan order (X_plan = X[perm]).
        ``exchange`` (sharded runs): object with ``gather(full, lo, hi, plan=)``
        and ``allreduce(t)``; rows owned here are plan.row_lo:plan.row_hi.
        ``plan_c`` (optional): plan of the same graph and partition with its own
        θ, used for the width-C aggregations (per-width mode choice).
        ``narrow`` (sharded runs, SURVEY.md §8(e) "narrowest-width exchange"):
        every rank keeps X for all n rows and computes Y0' for all of them (no
        width-H exchange before layer 1); the backward exchanges G1 (width C)
        and the ReLU bit mask instead of dP1' (width H), and recomputes
        dP1' = diag(r)((G1Θ1ᵀ)⊙mask1) for all rows."""
        self.plan = plan
        self.plan_c = plan_c if plan_c is not None else plan
        assert (self.plan_c.row_lo, self.plan_c.row_hi) == (plan.row_lo, plan.row_hi)
        self.dev = torch.device(device)
        self.n = plan.n
        self.lo, self.hi = plan.row_lo, plan.row_hi
        self.rows = self.hi - self.lo
        self.f_in = X_plan.shape[1]
        self.H = Th0.shape[1]
        self.C = Th1.shape[1]
        self.optimizer = optimizer
        self.lr = lr
        self.exchange = exchange
        self.narrow = bool(narrow and exchange is not None)
        # single GPU: the transform GEMMs also write the full mode's window blocks
        # (pcgcn_gemm_*_split) and the aggregations skip their split pass (IN_SPLIT)
        self.fuse = bool(fuse_split and exchange is None and max(Th0.shape[1], Th1.shape[1]) <= 128)
        assert max(self.H, self.C) <= plan.f_max
        d, f32 = self.dev, torch.float32
        n, rows, H, C = self.n, self.rows, self.H, self.C
        self.ldH, self.ldC = _ld(H), _ld(C)
        # X rows padded to a multiple of 4 floats (16-byte rows: TMA-loadable)
        self.ldX = _ld(self.f_in)
        xr = slice(0, n) if self.narrow else slice(self.lo, self.hi)
        self.X_all = torch.zeros(xr.stop - xr.start, self.ldX, dtype=f32, device=d)
        self.X_all[:, :self.f_in] = torch.from_numpy(np.ascontiguousarray(X_plan[xr], dtype=np.float32)).to(d)
        self.X = self.X_all[self.lo:self.hi] if self.narrow else self.X_all
        self.labels = torch.from_numpy(np.ascontiguousarray(labels_plan[self.lo:self.hi], dtype=np.int32)).to(d)
        self.train = torch.from_numpy(np.ascontiguousarray(train_plan[self.lo:self.hi], dtype=np.uint8)).to(d)
        self.inv_nT = 1.0 / float(np.count_nonzero(train_plan))
        # parameters (flat, Θ0 then Θ1) and optimiser state
        self.theta = torch.from_numpy(np.concatenate([Th0.ravel(), Th1.ravel()]).astype(np.float32)).to(d)
        self.Th0 = self.theta[: self.f_in * H].view(self.f_in, H)
        self.Th1 = self.theta[self.f_in * H:].view(H, C)
        self.grad = torch.zeros_like(self.theta)
        self.gTh0 = self.grad[: self.f_in * H].view(self.f_in, H)
        self.gTh1 = self.grad[self.f_in * H:].view(H, C)
        self.m = torch.zeros_like(self.theta)
        self.v = torch.zeros_like(self.theta)
        self.step_ctr = torch.zeros(1, dtype=torch.int32, device=d)
        # activations: inputs of aggregations span all n rows (sources), outputs the shard
        # peer mode (dist.PeerExchange): the aggregation inputs hold only
        # this shard's rows, in IPC/peer-mapped buffers the other shards read directly
        self.peer = exchange is not None and getattr(exchange, "peer", False)
        if self.peer:
            self.narrow = False
            self.fuse = False
        ain = (lambda key, w: exchange.local_buffer(key, rows, w)) if self.peer else \
            (lambda key, w: torch.zeros(n, w, dtype=f32, device=d))
        self.Y0 = ain("Y0", self.ldH)
        self.H1 = torch.zeros(rows, self.ldH, dtype=f32, device=d)
        mw = (H + 31) // 32
        # narrow: full-height mask / G1 (exchanged), the local rows are views
        self.mask1_all = torch.zeros(n if self.narrow else rows, mw, dtype=torch.int32, device=d)
        self.mask1 = self.mask1_all[self.lo:self.hi] if self.narrow else self.mask1_all
        self.Y1 = ain("Y1", self.ldC)
        self.Lg = torch.zeros(rows, self.ldC, dtype=f32, device=d)
        self.dL = ain("dL", self.ldC)
        self.G1_all = torch.zeros(n if self.narrow else rows, self.ldC, dtype=f32, device=d)
        self.G1 = self.G1_all[self.lo:self.hi] if self.narrow else self.G1_all
        self.dP1 = ain("dP1", self.ldH)
        self.G0 = torch.zeros(rows, self.ldH, dtype=f32, device=d)
        self.loss = torch.zeros(1, dtype=f32, device=d)
        self.ce_work = torch.zeros(L.CE_WORK_FLOATS, dtype=f32, device=d)
        wk = max(L.gemm_xtg_work_floats(rows, self.f_in, H), L.gemm_xtg_work_floats(rows, H, C))
        self.xtg_work = torch.zeros(max(wk, 1), dtype=f32, device=d)
        wk = max(L.gemm_xw_work_floats(self.f_in, H), L.gemm_xw_work_floats(H, C), L.gemm_dwt_work_floats(H, C))
        self.xw_work = torch.zeros(wk, dtype=f32, device=d)
        if self.narrow:
            wk = max(wk, L.gemm_xw_work_floats(self.f_in, H))
            self.xw_work = torch.zeros(wk, dtype=f32, device=d)
        self.r = plan.rowscale_ptr()  # device [n]
        self.r_local = None if self.lo == 0 else self.r + 4 * self.lo
        self._graph = None

    # -- one epoch -------------------------------------------------------
    def _r_rows(self):
        import ctypes
        return ctypes.c_void_p(self.r + 4 * self.lo) if self.lo else ctypes.c_void_p(self.r)

    def _local(self, full):
        return full if self.peer else full[self.lo:self.hi]

    def _gather(self, full, plan):
        if self.exchange is not None:
            self.exchange.gather(full, self.lo, self.hi, plan=plan)

    def _agg(self, plan, key, Y, Z, F, flags, mask=None, backward=False, stream=None):
        """One aggregation: from the full-height input, or (peer mode) from every
        shard's own buffer through the peer table."""
        if self.peer:
            peers, ld = self.exchange.peers(key), Y.shape[1]
            if backward:
                plan.backward_peer(peers, ld, Z, F, flags=flags, stream=stream)
            else:
                plan.forward_peer(peers, ld, Z, F, flags=flags, mask=mask, stream=stream)
        elif backward:
            plan.backward(Y, Z, F=F, flags=flags, stream=stream)
        else:
            plan.forward(Y, Z, F=F, flags=flags, mask=mask, stream=stream)

    def epoch(self, stream=None, hook=None, agg_flags=0):
        """One epoch; ``hook(name)`` (optional) is called after every step so a
        caller can record CUDA events between them."""
        mark = hook or (lambda name: None)
        rr = self._r_rows()
        H, C, p = self.H, self.C, self.plan
        # layer 1
        if self.narrow:   # Y0' for all n rows from the replicated X: no width-H exchange
            L.gemm_xw(self.X_all, self.Th0, ctypes.c_void_p(self.r), self.Y0, M=self.n, K=self.f_in, N=H,
                      work=self.xw_work, stream=stream)
        elif self.fuse:
            L.gemm_xw_split(p, self.X, self.Th0, rr, self.Y0, M=self.rows, K=self.f_in, N=H, work=self.xw_work,
                            stream=stream)
        else:
            L.gemm_xw(self.X, self.Th0, rr, self._local(self.Y0), M=self.rows, K=self.f_in, N=H, work=self.xw_work,
                      stream=stream)
        mark("a4_gemm_xw0")
        if not self.narrow:
            self._gather(self.Y0, p)
        mark("x_gather_y0")
        sf = L.IN_SPLIT if self.fuse else 0
        self._agg(p, "Y0", self.Y0, self.H1, H, L.IN_PRESCALED | L.RELU | L.MASK_OUT | sf | agg_flags, mask=self.mask1,
                  stream=stream)
        mark("a5a6_agg_fwd_H")
        # layer 2
        if self.fuse:
            L.gemm_xw_split(self.plan_c, self.H1, self.Th1, rr, self.Y1, M=self.rows, K=H, N=C, work=self.xw_work,
                            stream=stream)
        else:
            L.gemm_xw(self.H1, self.Th1, rr, self._local(self.Y1), M=self.rows, K=H, N=C, work=self.xw_work,
                      stream=stream)
        mark("a7_gemm_xw1")
        self._gather(self.Y1, self.plan_c)
        mark("x_gather_y1")
        self._agg(self.plan_c, "Y1", self.Y1, self.Lg, C, L.IN_PRESCALED | sf | agg_flags, stream=stream)
        mark("a8_agg_fwd_C")
        # loss
        L.softmax_ce(self.Lg, self.labels, self.train, self.inv_nT, rr, self._local(self.dL), self.loss,
                     self.ce_work, M=self.rows, C=C, stream=stream)
        mark("a9_softmax_ce")
        self._gather(self.dL, self.plan_c)
        mark("x_gather_dl")
        # backward
        self._agg(self.plan_c, "dL", self.dL, self.G1, C, L.IN_PRESCALED | agg_flags, backward=True, stream=stream)
        mark("a10_agg_bwd_C")
        L.gemm_xtg(self.H1, self.G1, self.gTh1, self.xtg_work, M=self.rows, K=H, N=C, stream=stream)
        if self.narrow:   # exchange G1 (width C) and the mask, recompute dP1' for all rows
            self.exchange.gather(self.G1_all, self.lo, self.hi, plan=None)
            self.exchange.gather(self.mask1_all.view(torch.float32), self.lo, self.hi, plan=None)
            L.gemm_dwt(self.G1_all, self.Th1, self.mask1_all, ctypes.c_void_p(self.r), self.dP1, M=self.n, N=C, K=H,
                       work=self.xw_work, stream=stream)
        elif self.fuse:
            L.gemm_dwt_split(p, self.G1, self.Th1, self.mask1, rr, self.dP1, M=self.rows, N=C, K=H,
                             work=self.xw_work, stream=stream)
        else:
            L.gemm_dwt(self.G1, self.Th1, self.mask1, rr, self._local(self.dP1), M=self.rows, N=C, K=H,
                       work=self.xw_work, stream=stream)
        mark("a11_gemm_xtg1_dwt")
        if not self.narrow:
            self._gather(self.dP1, p)
        mark("x_gather_dp1")
        self._agg(p, "dP1", self.dP1, self.G0, H, L.IN_PRESCALED | sf | agg_flags, backward=True, stream=stream)
        mark("a12_agg_bwd_H")
        L.gemm_xtg(self.X, self.G0, self.gTh0, self.xtg_work, M=self.rows, K=self.f_in, N=H, stream=stream)
        mark("a13_gemm_xtg0")
        if self.exchange is not None:
            self.exchange.allreduce(self.grad)
            self.exchange.allreduce(self.loss)
        mark("x_allreduce")
        # update
        if self.optimizer == "adam":
            L.adam(self.theta, self.grad, self.m, self.v, self.lr, self.step_ctr, stream=stream)
        elif self.optimizer == "sgd":
            L.sgd(self.theta, self.grad, self.lr, stream=stream)
        mark("a14_update")

    def launches_per_epoch(self) -> int:
        """Kernel launches of libpcgcn per epoch (for the bench's gpu_launches)."""
        def agg(plan):
            st = plan.stats()
            # split + full-mode tiles, segment pass (long rows), selective rows
            return 1 + (2 if st["shard_chunks"] > 0 else 0) + (1 if st["shard_segments"] > 0 else 0)

        np16 = lambda f: (f + 15) // 16 * 16  # noqa: E731
        xw = lambda ld, f: 2 + (1 if ld > np16(f) else 0)  # noqa: E731  W split + engine (+ pad zeroing)
        n = xw(self.ldH, self.H) + xw(self.ldC, self.C)      # a4, a7
        n += 2 * agg(self.plan) + 2 * agg(self.plan_c)       # a5/a6, a8, a10, a12
        if self.fuse:                                        # split passes fused into xw0, xw1, dwt
            n -= sum(1 for pl in (self.plan, self.plan_c, self.plan) if pl.stats()["shard_chunks"] > 0)
        n += 2                                               # a9 softmax-CE + loss reduction
        xtg = lambda f: 2 if np16(f) <= 128 else 3  # noqa: E731  engine (in-kernel B split) + slice sum
        n += xtg(self.C) + xtg(self.H)                       # a11, a13
        n += 2 + (1 if self.ldH > np16(self.H) else 0)       # a11 dwt: W split + engine (+ pad zeroing)
        n += 2 if self.optimizer == "adam" else 1            # a14
        ex = self.exchange
        if ex is not None and hasattr(ex, "mode"):            # halo pack + unpack per halo-mode gather
            gathered = [self.plan_c, self.plan_c] + ([] if self.narrow else [self.plan, self.plan])
            n += sum(2 for pl in gathered if ex.mode(pl) == "halo")
        return n

    # -- CUDA graph ------------------------------------------------------
    def capture(self, warmup: int = 2):
        s = torch.cuda.Stream(device=self.dev)
        s.wait_stream(torch.cuda.current_stream(self.dev))
        with torch.cuda.stream(s):
            for _ in range(warmup):
                self.epoch(stream=s)
        torch.cuda.current_stream(self.dev).wait_stream(s)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            self.epoch(stream=s)
        self._graph = g
        return g

    def replay(self):
        self._graph.replay()


class GCNL:
    """ℓ-layer GCN (Alg. 1 with general ℓ, L101-L125; the paper's Table II
    model is ℓ = 4, hid = 64, L255 — SURVEY.md §8(f) F2) as a sequence of ABI
    calls, single GPU.  dims = [F_in, hid, ..., hid, C]; layer l: Y_l' =
    diag(r)·H_{l-1}·Θ_l (gemm_xw), H_l = ReLU(Â Y_l) with its bit mask (hidden
    layers) or the logits (last layer); backward: G_l = Â dY_l, ∇Θ_l =
    H_{l-1}ᵀ G_l (gemm_xtg), dY_{l-1}' = diag(r)((G_l Θ_lᵀ) ⊙ mask_{l-1})
    (gemm_dwt).  ``plan`` serves the hidden widths, ``plan_c`` the class
    width (per-width modes)."""

    def __init__(self, plan: L.Plan, X_plan: np.ndarray, labels_plan: np.ndarray, train_plan: np.ndarray,
                 thetas, *, optimizer: str = "adam", lr: float = 0.01, device="cuda", plan_c: L.Plan | None = None):
        self.plan = plan
        self.plan_c = plan_c if plan_c is not None else plan
        assert plan.row_lo == 0 and plan.row_hi == plan.n, "GCNL is single-GPU"
        self.dev = torch.device(device)
        d, f32 = self.dev, torch.float32
        self.n = n = plan.n
        self.dims = [X_plan.shape[1]] + [t.shape[1] for t in thetas]
        for l, t in enumerate(thetas):
            assert t.shape[0] == self.dims[l]
        self.nl = len(thetas)
        self.optimizer, self.lr = optimizer, lr
        assert max(self.dims[1:]) <= plan.f_max
        ld = [_ld(f) for f in self.dims]
        self.ld = ld
        self.X = torch.zeros(n, ld[0], dtype=f32, device=d)
        self.X[:, :self.dims[0]] = torch.from_numpy(np.ascontiguousarray(X_plan, dtype=np.float32)).to(d)
        self.labels = torch.from_numpy(np.ascontiguousarray(labels_plan, dtype=np.int32)).to(d)
        self.train = torch.from_numpy(np.ascontiguousarray(train_plan, dtype=np.uint8)).to(d)
        self.inv_nT = 1.0 / float(np.count_nonzero(train_plan))
        flat = np.concatenate([np.asarray(t, np.float32).ravel() for t in thetas])
        self.theta = torch.from_numpy(flat).to(d)
        self.grad = torch.zeros_like(self.theta)
        self.Th, self.gTh, o = [], [], 0
        for l in range(self.nl):
            k = self.dims[l] * self.dims[l + 1]
            self.Th.append(self.theta[o:o + k].view(self.dims[l], self.dims[l + 1]))
            self.gTh.append(self.grad[o:o + k].view(self.dims[l], self.dims[l + 1]))
            o += k
        self.m = torch.zeros_like(self.theta)
        self.v = torch.zeros_like(self.theta)
        self.step_ctr = torch.zeros(1, dtype=torch.int32, device=d)
        z = lambda w: torch.zeros(n, w, dtype=f32, device=d)  # noqa: E731
        self.Y = [z(ld[l + 1]) for l in range(self.nl)]          # prescaled transform outputs
        self.H = [z(ld[l + 1]) for l in range(self.nl - 1)]      # hidden activations
        self.mask = [torch.zeros(n, (self.dims[l + 1] + 31) // 32, dtype=torch.int32, device=d)
                     for l in range(self.nl - 1)]
        self.Lg = z(ld[-1])
        self.dY = [z(ld[l + 1]) for l in range(self.nl)]         # backward aggregation inputs (prescaled)
        self.G = [z(ld[l + 1]) for l in range(self.nl)]
        self.loss = torch.zeros(1, dtype=f32, device=d)
        self.ce_work = torch.zeros(L.CE_WORK_FLOATS, dtype=f32, device=d)
        wk = max(max(L.gemm_xtg_work_floats(n, self.dims[l], self.dims[l + 1]) for l in range(self.nl)), 1)
        self.xtg_work = torch.zeros(wk, dtype=f32, device=d)
        wk = max(max(L.gemm_xw_work_floats(self.dims[l], self.dims[l + 1]) for l in range(self.nl)),
                 max(L.gemm_dwt_work_floats(self.dims[l], self.dims[l + 1]) for l in range(self.nl)))
        self.xw_work = torch.zeros(wk, dtype=f32, device=d)
        import ctypes
        self.rr = ctypes.c_void_p(plan.rowscale_ptr())
        self._graph = None

    def _plan(self, l):
        return self.plan_c if l == self.nl - 1 else self.plan

    def epoch(self, stream=None, hook=None, agg_flags=0):
        mark = hook or (lambda name: None)
        n, dims, rr = self.n, self.dims, self.rr
        Hin = self.X
        for l in range(self.nl):
            L.gemm_xw(Hin, self.Th[l], rr, self.Y[l], M=n, K=dims[l], N=dims[l + 1], work=self.xw_work, stream=stream)
            mark(f"xw{l}")
            if l < self.nl - 1:
                self._plan(l).forward(self.Y[l], self.H[l], F=dims[l + 1],
                                      flags=L.IN_PRESCALED | L.RELU | L.MASK_OUT | agg_flags, mask=self.mask[l],
                                      stream=stream)
                Hin = self.H[l]
            else:
                self._plan(l).forward(self.Y[l], self.Lg, F=dims[l + 1], flags=L.IN_PRESCALED | agg_flags,
                                      stream=stream)
            mark(f"agg_fwd{l}")
        L.softmax_ce(self.Lg, self.labels, self.train, self.inv_nT, rr, self.dY[-1], self.loss, self.ce_work,
                     M=n, C=dims[-1], stream=stream)
        mark("softmax_ce")
        for l in range(self.nl - 1, -1, -1):
            self._plan(l).backward(self.dY[l], self.G[l], F=dims[l + 1], flags=L.IN_PRESCALED | agg_flags,
                                   stream=stream)
            mark(f"agg_bwd{l}")
            Hl = self.X if l == 0 else self.H[l - 1]
            L.gemm_xtg(Hl, self.G[l], self.gTh[l], self.xtg_work, M=n, K=dims[l], N=dims[l + 1], stream=stream)
            if l > 0:
                L.gemm_dwt(self.G[l], self.Th[l], self.mask[l - 1], rr, self.dY[l - 1], M=n, N=dims[l + 1],
                           K=dims[l], work=self.xw_work, stream=stream)
            mark(f"grad{l}")
        if self.optimizer == "adam":
            L.adam(self.theta, self.grad, self.m, self.v, self.lr, self.step_ctr, stream=stream)
        elif self.optimizer == "sgd":
            L.sgd(self.theta, self.grad, self.lr, stream=stream)
        mark("update")

    def capture(self, warmup: int = 2):
        s = torch.cuda.Stream(device=self.dev)
        s.wait_stream(torch.cuda.current_stream(self.dev))
        with torch.cuda.stream(s):
            for _ in range(warmup):
                self.epoch(stream=s)
        torch.cuda.current_stream(self.dev).wait_stream(s)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            self.epoch(stream=s)
        self._graph = g
        return g

    def replay(self):
        self._graph.replay()
