"""Thin ctypes binding of libpcgcn.so (include/pcgcn.h) — argument marshalling only.

Every compute step runs in the library's sm_100a kernels; there is no CPU
fallback.  Importing this module fails loudly if the shared library is missing.
Device buffers are torch CUDA tensors (PyTorch is used for device memory,
streams and process groups only).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libpcgcn.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_ipps_tianmyd20_b200.build`"
                      " (no CPU fallback exists)")
lib = ctypes.CDLL(LIB_PATH)

c_i32, c_i64, c_f32, c_u32, c_vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_float, ctypes.c_uint32, ctypes.c_void_p

# status codes
OK, EINVAL, ENOTSYM, ECUDA, ENOMEM, ENCCL, EUNSUP = range(7)
NORM_SYM, NORM_NONE = 0, 1
DENSE_TF32X2, DENSE_FP32_SIMT, DENSE_BF16X1, DENSE_BF16X3 = 0, 1, 2, 3
ORDER_ID, ORDER_DEGREE = 0, 1
GRAIN_BLOCK, GRAIN_TILE = 0, 1
IN_PRESCALED, RELU, MASK_OUT, OUT_PRESCALED, PROFILE, IN_SPLIT = 1, 2, 4, 8, 16, 32
TIMING_NAMES = ("prescale", "split", "dense_tc", "sparse")
X_NAMES = ["part", "perm", "pstart", "r", "blk_k", "blk_i", "blk_nnz", "blk_dense", "sp_rowptr", "sp_col",
           "rt_row0", "rt_nrows", "rt_cptr", "ch_col0", "bits", "zd_index", "sweeps"]
X_DTYPES = [np.int32, np.int32, np.int64, np.float32, np.int32, np.int32, np.int64, np.uint8, np.int64,
            np.int32, np.int32, np.int32, np.int64, np.int32, np.uint32, np.int32, np.int32]
CE_WORK_FLOATS = 1024


class Csr(ctypes.Structure):
    _fields_ = [("n", c_i64), ("nnz", c_i64), ("rowptr", c_vp), ("col", c_vp)]


class Opts(ctypes.Structure):
    _fields_ = [("norm", c_i32), ("dense_prec", c_i32), ("f_max", c_i32), ("lp_sweeps", c_i32),
                ("part", c_vp), ("build_device", c_i32), ("rank", c_i32), ("world", c_i32),
                ("vertex_order", c_i32), ("mode_grain", c_i32)]


class Stats(ctypes.Structure):
    _fields_ = [("n", c_i64), ("nnz", c_i64), ("P", c_i32), ("lp_sweeps", c_i32), ("clusters", c_i64),
                ("blocks_nonempty", c_i64), ("blocks_dense", c_i64), ("nnz_sparse", c_i64),
                ("nnz_dense", c_i64), ("intra_edges", c_i64), ("row_tiles", c_i64), ("chunks", c_i64),
                ("row_lo", c_i64), ("row_hi", c_i64), ("shard_nnz_sparse", c_i64), ("shard_chunks", c_i64),
                ("theta", ctypes.c_double), ("partition_ms", ctypes.c_double), ("plan_ms", ctypes.c_double),
                ("device_bytes", c_i64), ("shard_segments", c_i64), ("src_rows_pc", c_i64),
                ("shard_src_rows_pc", c_i64), ("halo_recv_rows", c_i64), ("halo_send_rows", c_i64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


def _sig(name, res, *args):
    f = getattr(lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


_sig("pcgcn_opts_default", None, ctypes.POINTER(Opts))
_sig("pcgcn_plan", c_i32, ctypes.POINTER(Csr), c_i32, c_f32, ctypes.POINTER(Opts), ctypes.POINTER(c_vp))
_sig("pcgcn_destroy", None, c_vp)
_sig("pcgcn_forward", c_i32, c_vp, c_vp, c_i64, c_vp, c_i64, c_i32, c_u32, c_vp, c_vp)
_sig("pcgcn_backward", c_i32, c_vp, c_vp, c_i64, c_vp, c_i64, c_i32, c_u32, c_vp)
_sig("pcgcn_gemm_xw_work_floats", c_i64, c_i32, c_i32)
_sig("pcgcn_gemm_xw", c_i32, c_vp, c_i64, c_vp, c_i64, c_vp, c_vp, c_i64, c_i64, c_i32, c_i32, c_vp, c_vp)
_sig("pcgcn_gemm_xtg_work_floats", c_i64, c_i64, c_i32, c_i32)
_sig("pcgcn_gemm_xtg", c_i32, c_vp, c_i64, c_vp, c_i64, c_vp, c_i64, c_i32, c_i32, c_vp, c_vp)
_sig("pcgcn_gemm_dwt", c_i32, c_vp, c_i64, c_vp, c_vp, c_vp, c_vp, c_i64, c_i64, c_i32, c_i32, c_vp, c_vp)
_sig("pcgcn_gemm_dwt_work_floats", c_i64, c_i32, c_i32)
_sig("pcgcn_gemm_xw_split", c_i32, c_vp, c_vp, c_i64, c_vp, c_i64, c_vp, c_vp, c_i64, c_i64, c_i32, c_i32, c_vp, c_vp)
_sig("pcgcn_gemm_dwt_split", c_i32, c_vp, c_vp, c_i64, c_vp, c_vp, c_vp, c_vp, c_i64, c_i64, c_i32, c_i32, c_vp, c_vp)
_sig("pcgcn_softmax_ce", c_i32, c_vp, c_i64, c_vp, c_vp, c_i64, c_i32, c_f32, c_vp, c_vp, c_vp, c_vp, c_vp)
_sig("pcgcn_adam", c_i32, c_vp, c_vp, c_vp, c_vp, c_i64, c_f32, c_f32, c_f32, c_f32, c_vp, c_vp)
_sig("pcgcn_sgd", c_i32, c_vp, c_vp, c_i64, c_f32, c_vp)
_sig("pcgcn_plan_perm", c_i32, c_vp, c_vp)
_sig("pcgcn_plan_stats", c_i32, c_vp, ctypes.POINTER(Stats))
_sig("pcgcn_plan_rowscale", c_vp, c_vp)
_sig("pcgcn_plan_export_bytes", c_i64, c_vp, c_i32)
_sig("pcgcn_plan_export", c_i32, c_vp, c_i32, c_vp, c_i64)
_sig("pcgcn_calibrate", c_i32, c_i32, c_i32, c_f32, ctypes.POINTER(c_f32), ctypes.POINTER(c_f32),
     ctypes.POINTER(c_f32))
_sig("pcgcn_calibrate_prec", c_i32, c_i32, c_i32, c_f32, c_i32, ctypes.POINTER(c_f32), ctypes.POINTER(c_f32),
     ctypes.POINTER(c_f32))
_sig("pcgcn_plan_last_timings", c_i32, c_vp, ctypes.POINTER(c_f32))
_sig("pcgcn_refine_theta", c_i32, c_vp, c_vp, c_i64, c_vp, c_i64, c_i32, ctypes.POINTER(c_f32),
     ctypes.POINTER(c_f32), ctypes.POINTER(c_f32))
_sig("pcgcn_probe_read_gbs", c_i32, c_i64, c_i32, ctypes.POINTER(c_f32))
_sig("pcgcn_probe_gather_gbs", c_i32, c_i64, c_i32, c_i32, ctypes.POINTER(c_f32))
_sig("pcgcn_plan_shard_rows", c_i32, c_vp, c_vp)
_sig("pcgcn_plan_halo_rows", c_i64, c_vp, c_i32, c_i32)
_sig("pcgcn_plan_halo_export", c_i32, c_vp, c_i32, c_i32, c_vp, c_i64)
_sig("pcgcn_halo_pack", c_i32, c_vp, c_vp, c_i64, c_i32, c_vp, c_vp)
_sig("pcgcn_halo_unpack", c_i32, c_vp, c_vp, c_vp, c_i64, c_i32, c_vp)
_sig("pcgcn_nccl_unique_id", c_i32, c_vp)
_sig("pcgcn_nccl_comm_init", c_i32, c_vp, c_i32, c_i32, ctypes.POINTER(c_vp))
_sig("pcgcn_nccl_comm_destroy", None, c_vp)
_sig("pcgcn_halo_exchange", c_i32, c_vp, c_vp, c_i64, c_i32, c_vp, c_vp, c_vp, c_vp)
_sig("pcgcn_forward_peer", c_i32, c_vp, c_vp, c_i64, c_vp, c_i64, c_i32, c_u32, c_vp, c_vp)
_sig("pcgcn_backward_peer", c_i32, c_vp, c_vp, c_i64, c_vp, c_i64, c_i32, c_u32, c_vp)
_sig("pcgcn_ipc_alloc", c_i32, c_i64, ctypes.POINTER(c_vp))
_sig("pcgcn_ipc_free", None, c_vp)
_sig("pcgcn_ipc_handle", c_i32, c_vp, c_vp)
_sig("pcgcn_ipc_open", c_i32, c_vp, ctypes.POINTER(c_vp))
_sig("pcgcn_ipc_close", None, c_vp)
_sig("pcgcn_last_error", ctypes.c_char_p)
_sig("pcgcn_abi_version", c_i32)


class PcgcnError(RuntimeError):
    def __init__(self, code, where):
        msg = lib.pcgcn_last_error().decode(errors="replace")
        super().__init__(f"{where} failed with status {code}: {msg}")
        self.code = code


def check(code, where):
    if code != OK:
        raise PcgcnError(code, where)


def _ptr(t):
    """device pointer of a torch tensor (or None)."""
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


class Plan:
    """pcgcn_plan / pcgcn_forward / pcgcn_backward / pcgcn_destroy."""

    def __init__(self, n, rowptr, col, P, theta, *, norm=NORM_SYM, dense_prec=DENSE_TF32X2, f_max=128,
                 lp_sweeps=10, part=None, build_device=True, rank=0, world=1, order=ORDER_ID,
                 grain=GRAIN_BLOCK):
        self._h = None
        self.n = int(n)
        rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int32)
        A = Csr(self.n, int(rowptr[-1]), rowptr.ctypes.data, col.ctypes.data)
        o = Opts()
        lib.pcgcn_opts_default(ctypes.byref(o))
        o.norm, o.dense_prec, o.f_max, o.lp_sweeps = norm, dense_prec, f_max, lp_sweeps
        if part is not None:
            part = np.ascontiguousarray(part, dtype=np.int32)
            o.part = part.ctypes.data
        o.build_device = 1 if build_device else 0
        o.rank, o.world = rank, world
        o.vertex_order, o.mode_grain = order, grain
        h = c_vp()
        check(lib.pcgcn_plan(ctypes.byref(A), int(P), float(theta), ctypes.byref(o), ctypes.byref(h)), "pcgcn_plan")
        self._h = h
        self.P = int(P)
        self.f_max = f_max
        st = self.stats()
        self.theta = st["theta"]
        self.row_lo, self.row_hi = st["row_lo"], st["row_hi"]

    def __del__(self):
        self.destroy()

    def destroy(self):
        h = getattr(self, "_h", None)
        if h and lib is not None:  # lib may already be torn down at interpreter exit
            lib.pcgcn_destroy(h)
        self._h = None

    def stats(self):
        s = Stats()
        check(lib.pcgcn_plan_stats(self._h, ctypes.byref(s)), "pcgcn_plan_stats")
        return s.as_dict()

    def perm(self):
        out = np.empty(self.n, dtype=np.int32)
        check(lib.pcgcn_plan_perm(self._h, out.ctypes.data), "pcgcn_plan_perm")
        return out

    def export(self, name):
        w = X_NAMES.index(name)
        nbytes = lib.pcgcn_plan_export_bytes(self._h, w)
        out = np.empty(nbytes // np.dtype(X_DTYPES[w]).itemsize, dtype=X_DTYPES[w])
        if nbytes:
            check(lib.pcgcn_plan_export(self._h, w, out.ctypes.data, nbytes), "pcgcn_plan_export")
        return out

    def shard_rows(self, world):
        out = np.zeros(world + 1, dtype=np.int64)
        check(lib.pcgcn_plan_shard_rows(self._h, out.ctypes.data), "pcgcn_plan_shard_rows")
        return out

    def halo(self, q, send):
        """Plan rows of the halo list for peer q (send: rows of this shard q reads;
        else rows of shard q this shard reads)."""
        k = lib.pcgcn_plan_halo_rows(self._h, int(q), int(bool(send)))
        if k < 0:
            raise ValueError(f"bad peer {q}")
        out = np.empty(k, dtype=np.int32)
        if k:
            check(lib.pcgcn_plan_halo_export(self._h, int(q), int(bool(send)), out.ctypes.data, k),
                  "pcgcn_plan_halo_export")
        return out

    def halo_pack(self, Y, buf, w=None, stream=None):
        w = Y.shape[1] if w is None else w
        check(lib.pcgcn_halo_pack(self._h, _ptr(Y), Y.stride(0), w, _ptr(buf), _stream(stream)), "pcgcn_halo_pack")

    def halo_unpack(self, buf, Y, w=None, stream=None):
        w = Y.shape[1] if w is None else w
        check(lib.pcgcn_halo_unpack(self._h, _ptr(buf), _ptr(Y), Y.stride(0), w, _stream(stream)),
              "pcgcn_halo_unpack")

    def halo_exchange(self, Y, sendbuf, recvbuf, comm, w=None, stream=None):
        """pack -> NCCL grouped send/recv (in libpcgcn) -> unpack."""
        w = Y.shape[1] if w is None else w
        check(lib.pcgcn_halo_exchange(self._h, _ptr(Y), Y.stride(0), w, _ptr(sendbuf), _ptr(recvbuf), comm,
                                      _stream(stream)), "pcgcn_halo_exchange")

    def forward_peer(self, peers, ldy, Z, F, flags=0, mask=None, stream=None):
        """Selective pass reading sources from the shards' own buffers (device
        pointers, one per shard)."""
        tab = (c_vp * len(peers))(*[int(x) for x in peers])
        check(lib.pcgcn_forward_peer(self._h, tab, ldy, _ptr(Z), Z.stride(0), F, flags, _ptr(mask), _stream(stream)),
              "pcgcn_forward_peer")

    def backward_peer(self, peers, ldz, dY, F, flags=0, stream=None):
        tab = (c_vp * len(peers))(*[int(x) for x in peers])
        check(lib.pcgcn_backward_peer(self._h, tab, ldz, _ptr(dY), dY.stride(0), F, flags, _stream(stream)),
              "pcgcn_backward_peer")

    def rowscale_ptr(self):
        return lib.pcgcn_plan_rowscale(self._h)

    def last_timings(self):
        """{kernel: ms} of the last PROFILE-flagged forward/backward (syncs)."""
        ms = (c_f32 * 4)()
        check(lib.pcgcn_plan_last_timings(self._h, ms), "pcgcn_plan_last_timings")
        return dict(zip(TIMING_NAMES, [float(x) for x in ms]))

    def forward(self, Y, Z, F=None, flags=0, mask=None, stream=None):
        F = Y.shape[1] if F is None else F
        check(lib.pcgcn_forward(self._h, _ptr(Y), Y.stride(0), _ptr(Z), Z.stride(0), F, flags, _ptr(mask),
                                _stream(stream)), "pcgcn_forward")

    def backward(self, dZ, dY, F=None, flags=0, stream=None):
        F = dZ.shape[1] if F is None else F
        check(lib.pcgcn_backward(self._h, _ptr(dZ), dZ.stride(0), _ptr(dY), dY.stride(0), F, flags,
                                 _stream(stream)), "pcgcn_backward")


def gemm_xw_work_floats(K, N):
    return int(lib.pcgcn_gemm_xw_work_floats(K, N))


def gemm_xw(X, W, s, Y, M=None, K=None, N=None, work=None, stream=None):
    M = X.shape[0] if M is None else M
    K = X.shape[1] if K is None else K
    N = W.shape[1] if N is None else N
    check(lib.pcgcn_gemm_xw(_ptr(X), X.stride(0), _ptr(W), W.stride(0), s, _ptr(Y), Y.stride(0), M, K, N,
                            _ptr(work), _stream(stream)), "pcgcn_gemm_xw")


def gemm_xw_split(plan, X, W, s, Y, M=None, K=None, N=None, work=None, stream=None):
    """gemm_xw + the plan's full-mode window blocks of Y (consume with IN_SPLIT)."""
    M = X.shape[0] if M is None else M
    K = X.shape[1] if K is None else K
    N = W.shape[1] if N is None else N
    check(lib.pcgcn_gemm_xw_split(plan._h, _ptr(X), X.stride(0), _ptr(W), W.stride(0), s, _ptr(Y), Y.stride(0), M, K,
                                  N, _ptr(work), _stream(stream)), "pcgcn_gemm_xw_split")


def gemm_dwt_split(plan, D, W, mask, s, O, M=None, N=None, K=None, work=None, stream=None):
    M = D.shape[0] if M is None else M
    K = W.shape[0] if K is None else K
    N = W.shape[1] if N is None else N
    check(lib.pcgcn_gemm_dwt_split(plan._h, _ptr(D), D.stride(0), _ptr(W), _ptr(mask), s, _ptr(O), O.stride(0), M, N,
                                   K, _ptr(work), _stream(stream)), "pcgcn_gemm_dwt_split")


def gemm_xtg_work_floats(M, K, N):
    return int(lib.pcgcn_gemm_xtg_work_floats(M, K, N))


def gemm_xtg(X, D, G, work, M=None, K=None, N=None, stream=None):
    M = X.shape[0] if M is None else M
    K = X.shape[1] if K is None else K
    N = G.shape[1] if N is None else N
    check(lib.pcgcn_gemm_xtg(_ptr(X), X.stride(0), _ptr(D), D.stride(0), _ptr(G), M, K, N, _ptr(work),
                             _stream(stream)), "pcgcn_gemm_xtg")


def gemm_dwt_work_floats(K, N):
    return int(lib.pcgcn_gemm_dwt_work_floats(K, N))


def gemm_dwt(D, W, mask, s, O, M=None, N=None, K=None, work=None, stream=None):
    M = D.shape[0] if M is None else M
    K = W.shape[0] if K is None else K
    N = W.shape[1] if N is None else N
    check(lib.pcgcn_gemm_dwt(_ptr(D), D.stride(0), _ptr(W), _ptr(mask), s, _ptr(O), O.stride(0), M, N, K,
                             _ptr(work), _stream(stream)), "pcgcn_gemm_dwt")


def softmax_ce(L, labels, train, inv_nT, s, dL, loss, work, M=None, C=None, stream=None):
    M = L.shape[0] if M is None else M
    C = L.shape[1] if C is None else C
    assert dL.stride(0) == L.stride(0)
    check(lib.pcgcn_softmax_ce(_ptr(L), L.stride(0), _ptr(labels), _ptr(train), M, C, float(inv_nT), s,
                               _ptr(dL), _ptr(loss), _ptr(work), _stream(stream)), "pcgcn_softmax_ce")


def adam(theta, grad, m, v, lr, step, b1=0.9, b2=0.999, eps=1e-8, stream=None):
    check(lib.pcgcn_adam(_ptr(theta), _ptr(grad), _ptr(m), _ptr(v), theta.numel(), lr, b1, b2, eps, _ptr(step),
                         _stream(stream)), "pcgcn_adam")


def sgd(theta, grad, lr, stream=None):
    check(lib.pcgcn_sgd(_ptr(theta), _ptr(grad), theta.numel(), lr, _stream(stream)), "pcgcn_sgd")


def refine_theta(plan, Y, Z, F, stream=None):
    """In-situ θ for width F on the plan's own workload: (θ_F, ns/chunk, ns/edge)."""
    th, cc, ce = c_f32(), c_f32(), c_f32()
    check(lib.pcgcn_refine_theta(plan._h, _ptr(Y), Y.stride(0), _ptr(Z), Z.stride(0), F, ctypes.byref(th),
                                 ctypes.byref(cc), ctypes.byref(ce)), "pcgcn_refine_theta")
    return th.value, cc.value, ce.value


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    check(lib.pcgcn_nccl_unique_id(buf), "pcgcn_nccl_unique_id")
    return buf.raw


def nccl_comm_init(uid: bytes, rank: int, world: int):
    comm = c_vp()
    check(lib.pcgcn_nccl_comm_init(ctypes.create_string_buffer(uid, 128), rank, world, ctypes.byref(comm)),
          "pcgcn_nccl_comm_init")
    return comm


def nccl_comm_destroy(comm):
    lib.pcgcn_nccl_comm_destroy(comm)


class IpcBuffer:
    """A device buffer in its own allocation, shareable with other processes by
    CUDA IPC; ``tensor`` views it as a float32 [rows x cols] torch tensor."""

    def __init__(self, rows, cols):
        import torch
        p = c_vp()
        check(lib.pcgcn_ipc_alloc(int(rows) * int(cols) * 4 or 16, ctypes.byref(p)), "pcgcn_ipc_alloc")
        self.ptr = p.value
        self.rows, self.cols = int(rows), int(cols)

        class _Cai:
            __cuda_array_interface__ = {"shape": (self.rows, self.cols), "typestr": "<f4", "data": (self.ptr, False),
                                        "version": 3, "strides": None}
        self.tensor = torch.as_tensor(_Cai(), device="cuda")

    def handle(self) -> bytes:
        buf = ctypes.create_string_buffer(64)
        check(lib.pcgcn_ipc_handle(c_vp(self.ptr), buf), "pcgcn_ipc_handle")
        return buf.raw

    def free(self):
        if self.ptr:
            lib.pcgcn_ipc_free(c_vp(self.ptr))
            self.ptr = None


def ipc_open(handle: bytes) -> int:
    p = c_vp()
    check(lib.pcgcn_ipc_open(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)), "pcgcn_ipc_open")
    return p.value


def ipc_close(ptr: int):
    lib.pcgcn_ipc_close(c_vp(ptr))


def probe_read_gbs(nbytes, iters=20):
    v = c_f32()
    check(lib.pcgcn_probe_read_gbs(int(nbytes), int(iters), ctypes.byref(v)), "pcgcn_probe_read_gbs")
    return v.value


def calibrate(F, block_rows=2048, p_ref=0.05, dense_prec=None):
    th, tf, ts = c_f32(), c_f32(), c_f32()
    if dense_prec is None:
        check(lib.pcgcn_calibrate(F, block_rows, p_ref, ctypes.byref(th), ctypes.byref(tf), ctypes.byref(ts)),
              "pcgcn_calibrate")
    else:
        check(lib.pcgcn_calibrate_prec(F, block_rows, p_ref, dense_prec, ctypes.byref(th), ctypes.byref(tf),
                                       ctypes.byref(ts)), "pcgcn_calibrate_prec")
    return th.value, tf.value, ts.value


def probe_gather_gbs(nbytes, row_bytes=512, steps=256):
    """Random-row gather bandwidth (GB/s) from a buffer of nbytes (pcgcn_probe_gather_gbs)."""
    v = c_f32()
    check(lib.pcgcn_probe_gather_gbs(int(nbytes), int(row_bytes), int(steps), ctypes.byref(v)),
          "pcgcn_probe_gather_gbs")
    return float(v.value)
