"""Multi-process plumbing of the sharded path, world_size 2.

CPU (gloo): the row exchange and the gradient all-reduce.  GPU (one device,
two processes, gloo carrying CUDA tensors): a full sharded epoch through the
C ABI against the unsharded one — rows bitwise identical (each output row is
still reduced by one warp in the same order, halo rows are copies), loss and
gradients within the all-reduce reassociation tolerance."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _exchange_worker(rank, world, port, ranges, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200.dist import RowExchange
    _init(rank, world, port)
    lo, hi = ranges[rank]
    n = ranges[-1][1]
    full = torch.full((n, 3), -1.0)
    full[lo:hi] = torch.arange(lo, hi, dtype=torch.float32)[:, None] * 10 + rank
    ex = RowExchange(lo, hi, n=n)
    ex.gather(full)
    g = torch.full((4,), float(rank + 1))
    ex.allreduce(g)
    q.put((rank, full.numpy().copy(), g.numpy().copy()))
    dist.destroy_process_group()


def test_row_exchange_gloo_world2():
    ranges = [(0, 7), (7, 19)]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_exchange_worker, args=(r, 2, port, ranges, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    owner = np.array([0] * 7 + [1] * 12)
    exp = np.arange(19)[:, None] * 10.0 + owner[:, None]
    for rank, full, g in out:
        assert np.array_equal(full, np.repeat(exp, 3, 1))
        assert np.array_equal(g, np.full(4, 3.0))


def test_row_exchange_rejects_gaps():
    """Shard ranges must tile [0, n) in rank order (checked without a process group)."""
    from paper_conf_ipps_tianmyd20_b200.dist import check_ranges
    check_ranges([(0, 7), (7, 19)], 19)
    check_ranges([(0, 0), (0, 5)], 5)                 # an empty shard is allowed
    for bad, n in (([(0, 7), (8, 19)], 19),          # gap
                   ([(0, 8), (7, 19)], 19),          # overlap
                   ([(1, 7), (7, 19)], 19),          # does not start at 0
                   ([(0, 7), (7, 18)], 19),          # does not reach n
                   ([(0, 7), (9, 7)], None)):        # negative range
        with pytest.raises(ValueError):
            check_ranges(bad, n)


# ---------------------------------------------------------------------------
# GPU: sharded epoch vs unsharded, two processes on one device
# ---------------------------------------------------------------------------

def _epoch_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.dist import RowExchange
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    _init(rank, world, port)
    torch.cuda.set_device(0)
    w = C.PUBMED
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, 0.02, rank=rank, world=world)
    perm = pl.perm()
    model = GCN2(pl, X[perm], g.labels[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1,
                 exchange=RowExchange(pl.row_lo, pl.row_hi))
    model.epoch()
    torch.cuda.synchronize()
    q.put((rank, pl.row_lo, pl.row_hi, model.H1.cpu().numpy(), model.G0.cpu().numpy(),
           model.loss.item(), model.grad.cpu().numpy(), model.theta.cpu().numpy()))
    dist.destroy_process_group()


@pytest.mark.gpu
def test_sharded_epoch_matches_unsharded():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_epoch_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=600) for _ in ps])
    for p in ps:
        p.join(timeout=60)
    w = C.PUBMED
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, 0.02)
    perm = pl.perm()
    ref = GCN2(pl, X[perm], g.labels[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1)
    ref.epoch()
    torch.cuda.synchronize()
    H1 = ref.H1.cpu().numpy()
    G0 = ref.G0.cpu().numpy()
    assert res[0][1] == 0 and res[-1][2] == g.n and res[0][2] == res[1][1]
    for rank, lo, hi, h1, g0, loss, grad, theta in res:
        assert np.array_equal(h1, H1[lo:hi])          # forward rows: bitwise
        assert np.array_equal(g0, G0[lo:hi])          # backward rows: bitwise
        assert abs(loss - ref.loss.item()) <= 1e-6 * abs(ref.loss.item())
        gr = ref.grad.cpu().numpy()
        # different row slicing of the fp32 split-K reductions: same 1e-4
        # relative gate as the single-GPU gradient parity (test_gpu_parity)
        assert np.max(np.abs(grad - gr)) <= 1e-4 * np.max(np.abs(gr))
    assert np.array_equal(res[0][7], res[1][7])       # replicas agree after the update


# ---------------------------------------------------------------------------
# halo lists and the halo exchange
# ---------------------------------------------------------------------------

def _halo_brute(pl_r, n, ranges, r):
    """Rows of other shards that shard r reads: selective sources of its rows
    and every row of its chunks' 32-source windows (from the exported plan)."""
    lo, hi = ranges[r]
    rp, col = pl_r.export("sp_rowptr"), pl_r.export("sp_col")
    need = set(col[rp[lo]:rp[hi]].tolist())
    r0, nr, cp, c0 = pl_r.export("rt_row0"), pl_r.export("rt_nrows"), pl_r.export("rt_cptr"), pl_r.export("ch_col0")
    for t in range(len(r0)):
        if lo <= r0[t] < hi:
            for c in range(cp[t], cp[t + 1]):
                need.update(range(c0[c], min(c0[c] + 32, n)))
    return {q: sorted(j for j in need if ranges[q][0] <= j < ranges[q][1]) for q in range(len(ranges)) if q != r}


@pytest.mark.parametrize("world,theta", [(2, 0.05), (3, 0.0), (4, 2.0)])
def test_halo_lists_match_brute_force(world, theta):
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from synth import configs as C
    w = C.PUBMED
    g = C.graph(w)
    pls = [L.Plan(g.n, g.rowptr, g.col, w.P, theta, build_device=False, rank=r, world=world) for r in range(world)]
    row0 = pls[0].shard_rows(world)
    ranges = list(zip(row0[:-1].tolist(), row0[1:].tolist()))
    for r, pl in enumerate(pls):
        assert (pl.row_lo, pl.row_hi) == ranges[r]
        assert np.array_equal(pl.shard_rows(world), row0)
        exp = _halo_brute(pl, g.n, ranges, r)
        for q in range(world):
            if q == r:
                assert len(pl.halo(q, False)) == 0 and len(pl.halo(q, True)) == 0
                continue
            assert pl.halo(q, False).tolist() == exp[q], (r, q)
            # what r sends to q is exactly what q receives from r
            assert np.array_equal(pl.halo(q, True), pls[q].halo(r, False))
        st = pl.stats()
        assert st["halo_recv_rows"] == sum(len(v) for v in exp.values())


def _halo_worker(rank, world, port, q):
    """HaloExchange over gloo with host-only plans: the plan's pack/unpack
    (device kernels in the product) are replaced by their definition on host
    tensors, so this checks the split sizes, peer order and transport."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.dist import HaloExchange
    from synth import configs as C
    _init(rank, world, port)
    w = C.PUBMED
    g = C.graph(w)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, 0.05, build_device=False, rank=rank, world=world)
    send_rows = np.concatenate([pl.halo(p, True) for p in range(world)]).astype(np.int64)
    recv_rows = np.concatenate([pl.halo(p, False) for p in range(world)]).astype(np.int64)
    pl.halo_pack = lambda Y, buf, w_: buf.copy_(Y[torch.from_numpy(send_rows)])
    pl.halo_unpack = lambda buf, Y, w_: Y.index_copy_(0, torch.from_numpy(recv_rows), buf)
    ex = HaloExchange([pl], threshold=1.1)
    full = torch.full((g.n, 4), -1.0)
    full[pl.row_lo:pl.row_hi] = torch.arange(pl.row_lo, pl.row_hi, dtype=torch.float32)[:, None]
    ex.gather(full, pl.row_lo, pl.row_hi, plan=pl)
    q.put((rank, ex.mode(pl), recv_rows, full.numpy().copy(), pl.row_lo, pl.row_hi))
    dist.destroy_process_group()


def test_halo_exchange_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_halo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=180) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, mode, recv_rows, full, lo, hi in out:
        assert mode == "halo"
        got = full[:, 0]
        assert np.array_equal(got[lo:hi], np.arange(lo, hi))               # own rows untouched
        assert np.array_equal(got[recv_rows], recv_rows.astype(np.float32))  # halo rows arrived
        rest = np.setdiff1d(np.setdiff1d(np.arange(len(got)), np.arange(lo, hi)), recv_rows)
        assert np.all(got[rest] == -1.0)                                   # nothing else moved


def _halo_epoch_worker(rank, world, port, q, wname, theta, narrow, threshold):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.dist import HaloExchange
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    _init(rank, world, port)
    torch.cuda.set_device(0)
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    y = C.labels(w, g)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, rank=rank, world=world)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta * 2 if theta < 1 else theta, rank=rank, world=world)
    perm = pl.perm()
    ex = HaloExchange([pl, pl_c], threshold=threshold)
    model = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1, exchange=ex, plan_c=pl_c,
                 narrow=narrow)
    model.epoch()
    torch.cuda.synchronize()
    # bytes a halo-mode epoch must move into this rank: Y0', dP1' (width ldH, plan's
    # halo) and Y1', dL' (width ldC, plan_c's halo)
    expect = 4 * (2 * model.ldH * pl.stats()["halo_recv_rows"] + 2 * model.ldC * pl_c.stats()["halo_recv_rows"])
    q.put((rank, pl.row_lo, pl.row_hi, model.H1.cpu().numpy(), model.Lg.cpu().numpy(), model.G0.cpu().numpy(),
           model.loss.item(), model.grad.cpu().numpy(), model.theta.cpu().numpy(), ex.mode(pl), ex.mode(pl_c),
           (ex.bytes_moved, expect)))
    dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("wname,theta,narrow,threshold", [("pl-small", 0.05, False, 1.1),
                                                          ("pubmed", 0.02, False, 1.1),
                                                          ("pubmed", 0.02, True, 0.5),
                                                          ("pl-small", 0.05, True, 1.1)])
def test_sharded_halo_epoch_matches_unsharded(wname, theta, narrow, threshold):
    """Halo exchange (only the rows each shard reads move) and the narrow
    variant (Y0' recomputed from replicated X, G1 + mask exchanged instead of
    dP1'): output rows bitwise equal to the unsharded epoch, gradients within
    the all-reduce reassociation tolerance; on the clustered power-law graph
    (C5's recipe at test size, synth.configs.PL_SMALL) the halo moves a fraction of the remote rows."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_halo_epoch_worker, args=(r, 2, port, q, wname, theta, narrow, threshold))
          for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=900) for _ in ps], key=lambda t: t[0])
    for p in ps:
        p.join(timeout=60)
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    y = C.labels(w, g)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta)
    pl_c = L.Plan(g.n, g.rowptr, g.col, w.P, theta * 2 if theta < 1 else theta)
    perm = pl.perm()
    ref = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1, plan_c=pl_c)
    ref.epoch()
    torch.cuda.synchronize()
    H1, Lg, G0 = ref.H1.cpu().numpy(), ref.Lg.cpu().numpy(), ref.G0.cpu().numpy()
    gr = ref.grad.cpu().numpy()
    for rank, lo, hi, h1, lg, g0, loss, grad, theta_new, m_h, m_c, moved in res:
        if threshold > 1:
            assert m_h == "halo" and m_c == "halo"
        assert np.array_equal(h1, H1[lo:hi])
        assert np.array_equal(lg, Lg[lo:hi])
        assert np.array_equal(g0, G0[lo:hi])
        assert abs(loss - ref.loss.item()) <= 1e-6 * abs(ref.loss.item())
        assert np.max(np.abs(grad - gr)) <= 1e-5 * np.max(np.abs(gr))
        if threshold > 1 and not narrow:
            full_ag = 4 * (g.n - (hi - lo)) * (ref.ldH * 2 + ref.ldC * 2)
            assert moved[0] == moved[1], moved           # exactly the planner's halo rows moved
            if wname.startswith("pl"):
                assert moved[0] < 0.75 * full_ag, (moved, full_ag)   # clustered graph: well below an all-gather
    assert np.array_equal(res[0][8], res[1][8])


def _nccl_lib_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.dist import HaloExchange
    from synth import configs as C
    _init(rank, world, port)
    torch.cuda.set_device(0)
    w = C.PL_SMALL
    g = C.graph(w)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, 0.05, rank=rank, world=world)
    try:
        ex = HaloExchange([pl], threshold=1.1, transport="lib")
    except L.PcgcnError as e:        # NCCL refuses two ranks on one device
        q.put((rank, "skip", str(e)))
        dist.destroy_process_group()
        return
    full = torch.full((g.n, 8), -1.0, device="cuda")
    full[pl.row_lo:pl.row_hi] = torch.arange(pl.row_lo, pl.row_hi, dtype=torch.float32, device="cuda")[:, None]
    ex.gather(full, pl.row_lo, pl.row_hi, plan=pl)
    torch.cuda.synchronize()
    recv_rows = np.concatenate([pl.halo(p_, False) for p_ in range(world)]).astype(np.int64)
    q.put((rank, "ok", (recv_rows, full.cpu().numpy(), pl.row_lo, pl.row_hi)))
    ex.close()
    dist.destroy_process_group()


@pytest.mark.gpu
def test_halo_exchange_in_library_nccl():
    """pcgcn_halo_exchange (pack -> libpcgcn's NCCL group of send/recv ->
    unpack), two ranks; skipped when NCCL refuses two ranks on one device
    (the 1-GPU test box)."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_nccl_lib_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    if any(o[1] == "skip" for o in out):
        pytest.skip("NCCL: " + [o[2] for o in out if o[1] == "skip"][0][:200])
    for rank, _, (recv_rows, full, lo, hi) in out:
        got = full[:, 0]
        assert np.array_equal(got[lo:hi], np.arange(lo, hi))
        assert np.array_equal(got[recv_rows], recv_rows.astype(np.float32))


def test_nccl_unique_id_host():
    """The in-library NCCL bootstrap creates a 128-byte id without a GPU."""
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    a, b = L.nccl_unique_id(), L.nccl_unique_id()
    assert len(a) == 128 and a != b


# ---------------------------------------------------------------------------
# device-initiated peer gather: sources read from the owners' buffers
# ---------------------------------------------------------------------------

def _peer_worker(rank, world, port, q, wname, F, ld, theta):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from synth import configs as C
    _init(rank, world, port)
    torch.cuda.set_device(0)
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta, rank=rank, world=world)
    row0 = pl.shard_rows(world)
    Y = np.random.default_rng(5).standard_normal((g.n, ld)).astype(np.float32)
    Y[:, F:] = 0
    buf = L.IpcBuffer(pl.row_hi - pl.row_lo, ld)        # this shard's rows only
    buf.tensor.copy_(torch.from_numpy(Y[pl.row_lo:pl.row_hi]))
    torch.cuda.synchronize()
    handles = [None] * world
    dist.all_gather_object(handles, buf.handle())
    peers = [buf.ptr if r == rank else L.ipc_open(handles[r]) for r in range(world)]
    Z = torch.full((pl.row_hi - pl.row_lo, ld), float("nan"), device="cuda")
    M = torch.zeros(pl.row_hi - pl.row_lo, (F + 31) // 32, dtype=torch.int32, device="cuda")
    pl.forward_peer(peers, ld, Z, F, flags=L.IN_PRESCALED | L.RELU | L.MASK_OUT, mask=M)
    Zb = torch.full_like(Z, float("nan"))
    pl.backward_peer(peers, ld, Zb, F, flags=L.IN_PRESCALED)
    torch.cuda.synchronize()
    q.put((rank, pl.row_lo, pl.row_hi, Z.cpu().numpy(), M.cpu().numpy(), Zb.cpu().numpy(), row0.tolist()))
    dist.barrier()
    for r, ptr in enumerate(peers):
        if r != rank:
            L.ipc_close(ptr)
    buf.free()
    dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("wname,F,ld,theta", [("pl-small", 128, 128, 2.0), ("pl-small", 32, 32, 2.0),
                                              ("pubmed", 41, 48, 2.0)])
def test_peer_gather_matches_unsharded(wname, F, ld, theta):
    """pcgcn_forward_peer / pcgcn_backward_peer: each shard's
    selective pass reads every source row from the owner shard's own buffer
    (CUDA IPC mappings between two processes on this GPU; NVLink peer memory
    on a multi-GPU node) — no exchanged copy — and its rows (values, ReLU
    mask) are bitwise equal to the unsharded aggregation."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from synth import configs as C
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_peer_worker, args=(r, 2, port, q, wname, F, ld, theta)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=600) for _ in ps], key=lambda t: t[0])
    for p in ps:
        p.join(timeout=60)
    w = C.WORKLOADS[wname]
    g = C.graph(w)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, theta)
    Y = np.random.default_rng(5).standard_normal((g.n, ld)).astype(np.float32)
    Y[:, F:] = 0
    Yd = torch.from_numpy(Y).cuda()
    Z = torch.full((g.n, ld), float("nan"), device="cuda")
    M = torch.zeros(g.n, (F + 31) // 32, dtype=torch.int32, device="cuda")
    pl.forward(Yd, Z, F=F, flags=L.IN_PRESCALED | L.RELU | L.MASK_OUT, mask=M)
    Zb = torch.full_like(Z, float("nan"))
    pl.backward(Yd, Zb, F=F, flags=L.IN_PRESCALED)
    torch.cuda.synchronize()
    Z, M, Zb = Z.cpu().numpy(), M.cpu().numpy(), Zb.cpu().numpy()
    assert res[0][1] == 0 and res[-1][2] == g.n
    for rank, lo, hi, z, m, zb, row0 in res:
        assert np.array_equal(z[:, :F], Z[lo:hi, :F])
        assert np.array_equal(m, M[lo:hi])
        assert np.array_equal(zb[:, :F], Zb[lo:hi, :F])


def _peer_epoch_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.dist import PeerExchange
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    _init(rank, world, port)
    torch.cuda.set_device(0)
    w = C.PL_SMALL
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    y = C.labels(w, g)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, 2.0, rank=rank, world=world)
    perm = pl.perm()
    ex = PeerExchange(pl)
    model = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1, exchange=ex)
    assert model.peer and model.Y0.shape[0] == pl.row_hi - pl.row_lo
    model.epoch()
    torch.cuda.synchronize()
    q.put((rank, pl.row_lo, pl.row_hi, model.H1.cpu().numpy(), model.Lg.cpu().numpy(), model.G0.cpu().numpy(),
           model.loss.item(), model.grad.cpu().numpy(), model.theta.cpu().numpy()))
    ex.close()
    dist.destroy_process_group()


@pytest.mark.gpu
def test_sharded_peer_epoch_matches_unsharded():
    """A whole sharded 2-layer GCN epoch in peer mode (dist.PeerExchange: the
    aggregation inputs live in per-shard IPC buffers, every selective pass
    reads remote rows from their owners; no halo copies): rows bitwise equal
    to the unsharded epoch, gradients within the all-reduce tolerance."""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_tianmyd20_b200 import _lib as L
    from paper_conf_ipps_tianmyd20_b200.gcn import GCN2
    from synth import configs as C
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_peer_epoch_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=600) for _ in ps], key=lambda t: t[0])
    for p in ps:
        p.join(timeout=60)
    w = C.PL_SMALL
    g = C.graph(w)
    X = C.features(w, g.n)
    Th0, Th1 = C.thetas(w)
    T = C.train_mask(g.n, w.theta_seed)
    y = C.labels(w, g)
    pl = L.Plan(g.n, g.rowptr, g.col, w.P, 2.0)
    perm = pl.perm()
    ref = GCN2(pl, X[perm], y[perm], T[perm], Th0, Th1, optimizer="sgd", lr=0.1)
    ref.epoch()
    torch.cuda.synchronize()
    H1, Lg, G0, gr = ref.H1.cpu().numpy(), ref.Lg.cpu().numpy(), ref.G0.cpu().numpy(), ref.grad.cpu().numpy()
    for rank, lo, hi, h1, lg, g0, loss, grad, theta in res:
        assert np.array_equal(h1, H1[lo:hi])
        assert np.array_equal(lg, Lg[lo:hi])
        assert np.array_equal(g0, G0[lo:hi])
        assert abs(loss - ref.loss.item()) <= 1e-6 * abs(ref.loss.item())
        assert np.max(np.abs(grad - gr)) <= 1e-5 * np.max(np.abs(gr))
    assert np.array_equal(res[0][8], res[1][8])
