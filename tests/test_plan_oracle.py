"""Pins of the plan oracle (oracle/plan.py) against the written plan spec and
hand-worked cases (pins P17/P18).  CPU only."""
import numpy as np
import pytest

from oracle import gcn as O
from oracle import plan as PL
from synth import configs as C
from synth import graphs as G


def test_lp_path_hand_worked():
    # P3 0-1-2.  sweep 1: v0 sees {0,1}->0 (tie, smallest), v1 {0,1,2}->0, v2 {1,2}->1
    # sweep 2: v2 sees {0 (from v1), 1 (self)} -> tie -> 0.  sweep 3: no change.
    g = G.path(3)
    lab, sweeps = PL.label_propagation(O.binary_adjacency(g.n, g.rowptr, g.col))
    assert lab.tolist() == [0, 0, 0]
    assert sweeps == 3


def test_lp_cliques_take_smallest_member():
    sizes = [4, 6, 3, 7]
    g = G.cliques(sizes, seed=21)
    lab, sweeps = PL.label_propagation(O.binary_adjacency(g.n, g.rowptr, g.col))
    for c in range(len(sizes)):
        members = np.flatnonzero(g.labels == c)
        assert set(lab[members].tolist()) == {int(members.min())}
    assert sweeps == 2


def test_lp_isolated_vertex_keeps_own_label():
    g = G.from_edges(4, [(1, 2)])
    lab, _ = PL.label_propagation(O.binary_adjacency(g.n, g.rowptr, g.col))
    assert lab.tolist() == [0, 1, 1, 3]


def test_pack_order_and_sizes():
    labels = np.array([5, 5, 2, 2, 2, 9, 5, 5, 1])   # clusters: 5:{0,1,6,7} 2:{2,3,4} 9:{5} 1:{8}
    part = PL.pack(labels, 3)
    # sequence = [0,1,6,7 | 2,3,4 | 5 | 8] (size desc, then smallest member)
    # array_split(9, 3) = [0,1,6] [7,2,3] [4,5,8]
    assert part.tolist() == [0, 0, 1, 1, 2, 2, 0, 1, 2]
    part = PL.pack(labels, 4)   # sizes 3,2,2,2
    assert np.bincount(part).tolist() == [3, 2, 2, 2]


def test_p18_paper_csr_fragment():
    # Fig. 5(a) / L173: vertex 0 with in-neighbours {1, 2}, Val = 1.
    # Plan with P=1 (identity permutation) and Ã = A + I: row 0 = [0, 1, 2].
    g = G.from_edges(4, [(0, 1), (0, 2), (2, 3)])
    pl = PL.build(g.n, g.rowptr, g.col, P=1, theta=2.0, norm="none")
    assert pl["perm"].tolist() == [0, 1, 2, 3]
    assert pl["sp_rowptr"][1] == 3
    assert pl["sp_col"][:3].tolist() == [0, 1, 2]


@pytest.mark.parametrize("theta", [0.0, 0.05, 0.2, 2.0])
def test_p17_invariants(theta):
    w = C.scaled(C.PUBMED, 0.1)
    g = C.graph(w)
    P = 6
    pl = PL.build(g.n, g.rowptr, g.col, P=P, theta=theta)
    n = g.n
    nnz_t = g.nnz + n  # generator emits no duplicates / self-loops
    assert sorted(pl["perm"].tolist()) == list(range(n))
    sizes = np.diff(pl["pstart"])
    assert set(sizes.tolist()) <= {n // P, -(-n // P)}
    assert pl["blk_nnz"].sum() == nnz_t
    pop = int(np.unpackbits(pl["bits"].view(np.uint8)).sum())
    assert pl["sp_rowptr"][-1] + pop == nnz_t
    dens = pl["blk_nnz"] / (sizes[pl["blk_k"]] * sizes[pl["blk_i"]])
    assert np.array_equal(pl["blk_dense"].astype(bool), dens > np.float32(theta))
    if theta == 0.0:
        assert pl["blk_dense"].all() and pl["sp_rowptr"][-1] == 0
    if theta >= 1.0:
        assert not pl["blk_dense"].any() and len(pl["rt_row0"]) == 0
    # dense rows map to zd rows, others -1
    has = pl["zd_index"] >= 0
    for r0, nr in zip(pl["rt_row0"], pl["rt_nrows"]):
        assert has[r0:r0 + nr].all()


def test_tie_at_theta_is_sparse():
    # one block: K_4 plus self loops = 16 of 16 -> density 1; theta = 1 -> sparse
    g = G.complete(4)
    pl = PL.build(g.n, g.rowptr, g.col, P=1, theta=1.0)
    assert pl["blk_dense"].tolist() == [0]
    # P=2 on a 4-path 0-1-2-3 with part [0,0,1,1]: block (0,1) has 1 edge of 4 -> 0.25
    g = G.path(4)
    pl = PL.build(g.n, g.rowptr, g.col, P=2, theta=0.25, part=np.array([0, 0, 1, 1]))
    d = dict(zip(zip(pl["blk_k"].tolist(), pl["blk_i"].tolist()), pl["blk_dense"].tolist()))
    assert d[(0, 1)] == 0 and d[(0, 0)] == 1   # (0,0) = 4/4 = 1 > 0.25


def test_dense_tiles_reconstruct_matrix():
    """Bits + sparse CSR reassemble Ã exactly (in plan order)."""
    g = G.cliques([40, 150, 7, 90], seed=3)
    pl = PL.build(g.n, g.rowptr, g.col, P=4, theta=0.5)
    n = g.n
    M = np.zeros((n, n), dtype=np.int64)
    for v in range(n):
        for j in pl["sp_col"][pl["sp_rowptr"][v]:pl["sp_rowptr"][v + 1]]:
            M[v, j] += 1
    for t, (r0, nr) in enumerate(zip(pl["rt_row0"], pl["rt_nrows"])):
        for c in range(pl["rt_cptr"][t], pl["rt_cptr"][t + 1]):
            w = pl["bits"][c * 128:(c + 1) * 128]
            for rr in range(128):
                for b in range(32):
                    if (int(w[rr]) >> b) & 1:
                        assert rr < nr
                        M[r0 + rr, pl["ch_col0"][c] + b] += 1
    At = O.normalized_adjacency(n, g.rowptr, g.col, "none")[0].toarray()
    inv = np.argsort(pl["perm"])
    Ap = np.zeros_like(M)
    Ap[np.ix_(inv, inv)] = At
    assert np.array_equal(M, Ap)


def test_r_bits():
    g = G.star(5)
    pl = PL.build(g.n, g.rowptr, g.col, P=1, theta=2.0)
    assert pl["r"][0] == np.float32(1 / np.sqrt(6.0))
    assert pl["r"][1] == np.float32(1 / np.sqrt(2.0))


def _dense_matrix_from_plan(pl, n):
    """Ã in plan order rebuilt from the selective CSR and the bit chunks, with
    the mode of every entry (1 = full mode)."""
    M = np.zeros((n, n), dtype=np.int64)
    mode = np.zeros((n, n), dtype=np.int64)
    for v in range(n):
        for j in pl["sp_col"][pl["sp_rowptr"][v]:pl["sp_rowptr"][v + 1]]:
            M[v, j] += 1
    for t, (r0, nr) in enumerate(zip(pl["rt_row0"], pl["rt_nrows"])):
        for c in range(pl["rt_cptr"][t], pl["rt_cptr"][t + 1]):
            w = pl["bits"][c * 128:(c + 1) * 128]
            for rr in range(nr):
                for b in range(32):
                    if (int(w[rr]) >> b) & 1:
                        M[r0 + rr, pl["ch_col0"][c] + b] += 1
                        mode[r0 + rr, pl["ch_col0"][c] + b] = 1
    return M, mode


@pytest.mark.parametrize("theta", [0.0, 0.05, 0.2, 0.6, 2.0])
def test_degree_order_and_tile_grain_invariants(theta):
    """Readings #24/#25 by brute force on the reassembled matrix: (a) inside
    every partition the vertices run by descending degree (ties by id); (b)
    every 128-row tile x 32-aligned window sub-block of Ã (in plan order) is
    wholly full-mode iff its density nnz/(rows·min(32, n-c0)) > θ, else wholly
    selective; (c) bits + CSR reassemble Ã exactly."""
    g = G.cliques([40, 150, 7, 90, 300], seed=3)
    rng = np.random.default_rng(5)
    # sprinkle random edges so sub-block densities vary
    e = rng.integers(0, g.n, size=(2000, 2))
    g = G.from_edges(g.n, list(zip(*np.nonzero(
        O.normalized_adjacency(g.n, g.rowptr, g.col, "none")[0].toarray() - np.eye(g.n)))) +
        [tuple(x) for x in e.tolist() if x[0] != x[1]])
    n = g.n
    pl = PL.build(g.n, g.rowptr, g.col, P=3, theta=theta, order="degree", grain="tile")
    deg = np.diff(O.binary_adjacency(n, g.rowptr, g.col).indptr)
    perm = pl["perm"]
    for k in range(3):
        seg = perm[pl["pstart"][k]:pl["pstart"][k + 1]]
        key = list(zip((-deg[seg]).tolist(), seg.tolist()))
        assert key == sorted(key)
    M, mode = _dense_matrix_from_plan(pl, n)
    At = O.normalized_adjacency(n, g.rowptr, g.col, "none")[0].toarray()
    inv = np.argsort(perm)
    Ap = np.zeros_like(M)
    Ap[np.ix_(inv, inv)] = At
    assert np.array_equal(M, Ap)
    for k in range(3):
        for r0 in range(pl["pstart"][k], pl["pstart"][k + 1], 128):
            r1 = min(r0 + 128, pl["pstart"][k + 1])
            for c0 in range(0, n, 32):
                sub = M[r0:r1, c0:c0 + 32]
                if sub.sum() == 0:
                    continue
                dense = sub.sum() / (sub.shape[0] * sub.shape[1]) > np.float32(theta)
                md = mode[r0:r1, c0:c0 + 32][sub > 0]
                assert md.all() if dense else not md.any(), (k, r0, c0, theta)
