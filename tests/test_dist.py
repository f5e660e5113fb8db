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
