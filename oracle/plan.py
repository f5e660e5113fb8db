"""Plan oracle — TEST INFRASTRUCTURE ONLY (same import rule as oracle/gcn.py).

An independent numpy re-derivation, from the written spec (SURVEY.md §8(c)
item 4 and DESIGN.md §3a "Plan spec"), of everything the host planner exports.
The tests compare it bit-exactly with ``pcgcn_plan_export``.

Paper passages it follows:
  * 2-D partition into K vertex blocks V_k and K×K edge blocks E_{k,i}
    (§III-A.a, Fig. 4).  E_{k,i} = edges whose destination is in
    V_k and source in V_i (reading #5: destination-major, row-block k).
  * locality-aware partitioner (L97: METIS) -> deterministic synchronous label
    propagation + packing (reading #8).
  * mode choice θ = T_f·p/T_s, full iff p' > θ (L161 §III-B.c; strict, #10);
    p' is the block density nnz/(|V_k|·|V_i|) (reading #9).
  * selective blocks merged into one CSR (L179 §IV-B), Dst/Src convention of
    Fig. 5(a) (L171-L173): row v lists the in-neighbours of v.
  * full blocks stored dense with missing edges = 0 (L151-L153, L175); here
    as 128-row × 32-column bit tiles (reading #6, layout in DESIGN.md).
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp

from .gcn import binary_adjacency

TILE_M = 128  # destination rows per dense row tile
TILE_K = 32   # source columns per dense chunk


def label_propagation(A, T: int = 10):
    """Synchronous LP on Ã = A + I.  label_i ← argmax_l |{j ∈ N(i)∪{i}: label_j = l}|,
    ties -> smallest label; start label_i = i; at most T sweeps, stop when
    nothing changes.  Returns (labels, sweeps_run)."""
    n = A.shape[0]
    lab = np.arange(n, dtype=np.int64)
    indptr = A.indptr.astype(np.int64)
    rows = np.concatenate([np.repeat(np.arange(n, dtype=np.int64), np.diff(indptr)),
                           np.arange(n, dtype=np.int64)])
    nbr = np.concatenate([A.indices.astype(np.int64), np.arange(n, dtype=np.int64)])
    it = 0
    for it in range(1, T + 1):
        l = lab[nbr]
        order = np.lexsort((l, rows))
        r_s, l_s = rows[order], l[order]
        brk = np.ones(len(r_s), dtype=bool)
        brk[1:] = (r_s[1:] != r_s[:-1]) | (l_s[1:] != l_s[:-1])
        start = np.flatnonzero(brk)
        cnt = np.diff(np.append(start, len(r_s)))
        ur, ul = r_s[start], l_s[start]
        # per row: max count, then smallest label
        o2 = np.lexsort((ul, -cnt, ur))
        first = np.ones(len(o2), dtype=bool)
        first[1:] = ur[o2][1:] != ur[o2][:-1]
        new = np.empty(n, dtype=np.int64)
        new[ur[o2][first]] = ul[o2][first]
        if np.array_equal(new, lab):
            return lab, it
        lab = new
    return lab, it


def pack(labels: np.ndarray, P: int) -> np.ndarray:
    """Clusters ordered by (size desc, smallest member asc); members by id;
    the sequence cut into P consecutive chunks with numpy array_split sizes."""
    n = len(labels)
    uniq, inv = np.unique(labels, return_inverse=True)
    size = np.bincount(inv, minlength=len(uniq))
    minid = np.full(len(uniq), n, dtype=np.int64)
    np.minimum.at(minid, inv, np.arange(n))
    corder = np.lexsort((minid, -size))
    rank = np.empty(len(uniq), dtype=np.int64)
    rank[corder] = np.arange(len(uniq))
    seq = np.lexsort((np.arange(n), rank[inv]))
    part = np.empty(n, dtype=np.int32)
    pos = 0
    for k, chunk in enumerate(np.array_split(np.arange(n), P)):
        part[seq[chunk]] = k
        pos += len(chunk)
    return part


def build(n: int, rowptr, col, P: int, theta: float, part=None, norm: str = "sym", order: str = "id",
          grain: str = "block"):
    """Every plan array, in export order.  ``part`` overrides the partitioner.

    order: "id" — vertices of a block by ascending id; "degree" — by descending
           degree, ties by id (reading #24).
    grain: "block" — the paper's rule per partition pair E_{k,i} (L161):
           full iff nnz/(|V_k||V_i|) > θ; "tile" — the same rule per chunk
           (128-row tile of V_k x 32-aligned source window), density =
           nnz/(tile rows · min(32, n - window start)) (reading #25)."""
    A = binary_adjacency(n, rowptr, col)
    deg = np.diff(A.indptr).astype(np.int64)
    dt = deg + 1
    r = (1.0 / np.sqrt(dt.astype(np.float64))).astype(np.float32)
    if norm == "none":
        r = np.ones(n, dtype=np.float32)
    sweeps = 0
    if part is None:
        lab, sweeps = label_propagation(A)
        part = pack(lab, P)
    part = np.asarray(part, dtype=np.int32)
    if order == "degree":
        perm = np.lexsort((np.arange(n), -deg, part)).astype(np.int32)  # new -> old
    else:
        perm = np.lexsort((np.arange(n), part)).astype(np.int32)
    inv = np.empty(n, dtype=np.int64)
    inv[perm] = np.arange(n)
    psize = np.bincount(part, minlength=P).astype(np.int64)
    pstart = np.concatenate([[0], np.cumsum(psize)]).astype(np.int64)

    # Ã in plan order (rows = destinations, cols = sources), sorted
    At = (A + sp.identity(n, format="csr")).tocsr()
    rows_old = np.repeat(np.arange(n, dtype=np.int64), np.diff(At.indptr))
    dst = inv[rows_old]
    src = inv[At.indices.astype(np.int64)]
    o = np.lexsort((src, dst))
    dst, src = dst[o], src[o]
    pd = np.searchsorted(pstart, dst, side="right") - 1
    ps = np.searchsorted(pstart, src, side="right") - 1

    # block table (non-empty blocks, sorted by (k, i))
    bkey = pd * P + ps
    ub, bcnt = np.unique(bkey, return_counts=True)
    blk_k = (ub // P).astype(np.int32)
    blk_i = (ub % P).astype(np.int32)
    blk_nnz = bcnt.astype(np.int64)
    dens = blk_nnz.astype(np.float64) / (psize[blk_k].astype(np.float64) * psize[blk_i].astype(np.float64))
    blk_dense = (dens > np.float64(np.float32(theta))).astype(np.uint8)

    # split edges by mode
    if grain == "tile":
        # chunk of an edge: (destination row tile inside its partition, 32-aligned source window)
        tkey = pd * (n // TILE_M + 2) + (dst - pstart[pd]) // TILE_M
        ckey = tkey * ((n + TILE_K - 1) // TILE_K) + src // TILE_K
        uc, cinv, ccnt = np.unique(ckey, return_inverse=True, return_counts=True)
        c_pd = np.zeros(len(uc), dtype=np.int64)
        c_pd[cinv] = pd
        c_dst = np.zeros(len(uc), dtype=np.int64)
        c_dst[cinv] = dst
        c_src = np.zeros(len(uc), dtype=np.int64)
        c_src[cinv] = src
        t0 = pstart[c_pd] + (c_dst - pstart[c_pd]) // TILE_M * TILE_M
        rows_t = np.minimum(t0 + TILE_M, pstart[c_pd + 1]) - t0
        w0 = c_src // TILE_K * TILE_K
        cols_w = np.minimum(TILE_K, n - w0)
        cdense = ccnt.astype(np.float64) / (rows_t.astype(np.float64) * cols_w.astype(np.float64)) \
            > np.float64(np.float32(theta))
        emode = cdense[cinv].astype(np.uint8)
        # a block is marked full-mode iff it holds full-mode edges
        blk_dense = np.zeros(len(ub), dtype=np.uint8)
        blk_dense[np.searchsorted(ub, bkey[emode == 1])] = 1
    else:
        dense_of = dict(zip(ub.tolist(), blk_dense.tolist()))
        emode = (np.array([dense_of[b] for b in bkey.tolist()], dtype=np.uint8) if len(bkey)
                 else np.zeros(0, np.uint8))
    sm = emode == 0
    sp_rowptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(dst[sm], minlength=n), out=sp_rowptr[1:])
    sp_col = src[sm].astype(np.int32)

    # dense tiles
    dd, ds = dst[~sm], src[~sm]
    rt_row0, rt_nrows, rt_cptr, ch_col0, bits = [], [], [0], [], []
    zd_index = np.full(n, -1, dtype=np.int32)
    if len(dd):
        kd = np.searchsorted(pstart, dd, side="right") - 1
        t_of = (dd - pstart[kd]) // TILE_M
        # chunk = 32-aligned global source window (shared by the full-mode
        # blocks of one row tile that overlap it); group key: (k, t, window)
        c_of = ds // TILE_K
        order = np.lexsort((ds, dd, c_of, t_of, kd))
        kd, t_of, c_of, dd, ds = kd[order], t_of[order], c_of[order], dd[order], ds[order]
        tile_key = np.stack([kd, t_of], 1)
        chunk_key = np.stack([kd, t_of, c_of], 1)
        brk_c = np.ones(len(dd), dtype=bool)
        brk_c[1:] = np.any(chunk_key[1:] != chunk_key[:-1], axis=1)
        brk_t = np.ones(len(dd), dtype=bool)
        brk_t[1:] = np.any(tile_key[1:] != tile_key[:-1], axis=1)
        cstarts = np.flatnonzero(brk_c)
        cends = np.append(cstarts[1:], len(dd))
        for a, b in zip(cstarts, cends):
            if brk_t[a]:
                if len(rt_row0):
                    rt_cptr.append(len(ch_col0))
                k, t = int(kd[a]), int(t_of[a])
                r0 = int(pstart[k] + t * TILE_M)
                rt_row0.append(r0)
                rt_nrows.append(int(min(TILE_M, pstart[k + 1] - r0)))
            c0 = int(c_of[a] * TILE_K)
            ch_col0.append(c0)
            w = np.zeros(TILE_M, dtype=np.uint32)
            rr = (dd[a:b] - rt_row0[-1]).astype(np.int64)
            cc = (ds[a:b] - c0).astype(np.int64)
            np.bitwise_or.at(w, rr, (np.uint32(1) << cc.astype(np.uint32)))
            bits.append(w)
        rt_cptr.append(len(ch_col0))
        for t, (r0, nr) in enumerate(zip(rt_row0, rt_nrows)):
            zd_index[r0:r0 + nr] = t * TILE_M + np.arange(nr, dtype=np.int32)
    return dict(
        part=part, perm=perm, pstart=pstart, r=r[perm].copy(), sweeps=sweeps,
        blk_k=blk_k, blk_i=blk_i, blk_nnz=blk_nnz, blk_dense=blk_dense,
        sp_rowptr=sp_rowptr, sp_col=sp_col,
        rt_row0=np.asarray(rt_row0, dtype=np.int32), rt_nrows=np.asarray(rt_nrows, dtype=np.int32),
        rt_cptr=np.asarray(rt_cptr if rt_row0 else [0], dtype=np.int64),
        ch_col0=np.asarray(ch_col0, dtype=np.int32),
        bits=(np.concatenate(bits) if bits else np.zeros(0, np.uint32)).astype(np.uint32),
        zd_index=zd_index,
    )
