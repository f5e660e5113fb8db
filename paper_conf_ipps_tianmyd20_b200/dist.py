"""Multi-GPU plumbing for sharded plans.

Destination partitions are sharded over ranks in contiguous plan-row ranges
(the planner's cost-balanced split).  Each aggregation needs the prescaled
source rows of the partitions its blocks touch (§III-A.b):

* HaloExchange — the planner's halo lists (pcgcn_plan_halo_*): libpcgcn packs
  the rows each peer reads into one send buffer, one all-to-all with per-peer
  split sizes (NCCL grouped send/recv over NVLink) moves only those rows, and
  libpcgcn scatters the received rows into the full-height input.  When a
  plan's halo exceeds half of the remote rows on some rank (Reddit-shaped
  graphs touch ~100% of them) the exchange falls back to
* RowExchange — an all-gather of every owner's range (one broadcast per
  owner, ranges are uneven).

∇Θ (one flat buffer) and the loss are summed with one all-reduce each.
torch.distributed (NCCL on GPUs, gloo in the tests) is the transport; the
arithmetic and the row packing stay in libpcgcn.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def check_ranges(ranges, n=None):
    """The shard row ranges must tile [0, n) in rank order (contiguous
    partition ranges); raises ValueError otherwise."""
    if not ranges or ranges[0][0] != 0:
        raise ValueError(f"shard ranges must start at row 0: {ranges}")
    for a, b in ranges:
        if b < a:
            raise ValueError(f"empty-negative shard range {(a, b)}")
    for a, b in zip(ranges, ranges[1:]):
        if a[1] != b[0]:
            raise ValueError(f"shard ranges must tile the rows (gap/overlap at {a} -> {b})")
    if n is not None and ranges[-1][1] != n:
        raise ValueError(f"shard ranges end at {ranges[-1][1]}, not at n = {n}")


class RowExchange:
    def __init__(self, lo: int, hi: int, group=None, n: int | None = None):
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        ranges = [None] * self.world
        dist.all_gather_object(ranges, (int(lo), int(hi)), group=group)
        self.ranges = ranges
        assert ranges[self.rank] == (lo, hi)
        check_ranges(ranges, n)
        # broadcast() takes GLOBAL ranks; map the group-local owner index
        self.src = [q if group is None else dist.get_global_rank(group, q) for q in range(self.world)]

    def gather(self, full: torch.Tensor, lo: int = None, hi: int = None, plan=None):
        """full[lo_q:hi_q] of every rank q becomes visible on every rank."""
        if full.shape[0] != self.ranges[-1][1]:
            raise ValueError(f"full buffer has {full.shape[0]} rows, ranges cover {self.ranges[-1][1]}")
        for q, (a, b) in enumerate(self.ranges):
            if b > a:
                dist.broadcast(full[a:b], src=self.src[q], group=self.group)

    def allreduce(self, t: torch.Tensor):
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)


class HaloExchange:
    """Halo-only exchange (see the module doc).  ``plans``: the plans whose
    aggregations consume exchanged buffers (per-width plans have their own
    lists); ``gather(full, lo, hi, plan)`` refreshes the rows of ``full`` that
    ``plan``'s local rows read.  Falls back to the all-gather per plan when
    its halo exceeds ``threshold`` of the remote rows on any rank."""

    def __init__(self, plans, group=None, threshold: float = 0.5, transport: str = "torch"):
        """transport: "torch" — torch.distributed all_to_all_single (NCCL grouped
        send/recv on GPUs, gloo in the tests); "lib" — libpcgcn's own NCCL group
        (pcgcn_halo_exchange on a communicator bootstrapped here)."""
        self.group = group
        self.transport = transport
        self.comm = None
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.backend = dist.get_backend(group)
        p0 = plans[0]
        self.ranges = [(int(a), int(b)) for a, b in zip(p0.shard_rows(self.world)[:-1], p0.shard_rows(self.world)[1:])]
        check_ranges(self.ranges, p0.n)
        assert self.ranges[self.rank] == (p0.row_lo, p0.row_hi)
        self.rowx = RowExchange(p0.row_lo, p0.row_hi, group=group, n=p0.n)
        self.info = {}
        for pl in plans:
            recv = [len(pl.halo(q, False)) if q != self.rank else 0 for q in range(self.world)]
            send = [len(pl.halo(q, True)) if q != self.rank else 0 for q in range(self.world)]
            remote = pl.n - (pl.row_hi - pl.row_lo)
            frac = torch.tensor([sum(recv) / max(remote, 1)], dtype=torch.float64)
            dist.all_reduce(frac, op=dist.ReduceOp.MAX, group=group)
            mode = "allgather" if float(frac) > threshold else "halo"
            self.info[id(pl)] = dict(plan=pl, recv=recv, send=send, mode=mode, frac=float(frac))
        self._bufs = {}
        self.bytes_moved = 0   # rows x stride x 4 received by this rank, summed over gather calls
        if transport == "lib":
            from . import _lib as L
            uid = [L.nccl_unique_id() if self.rank == 0 else None]
            dist.broadcast_object_list(uid, src=0 if group is None else dist.get_global_rank(group, 0), group=group)
            self.comm = L.nccl_comm_init(uid[0], self.rank, self.world)

    def close(self):
        if self.comm is not None:
            from . import _lib as L
            L.nccl_comm_destroy(self.comm)
            self.comm = None

    def mode(self, plan):
        return self.info[id(plan)]["mode"]

    def _buf(self, key, rows, w, like):
        b = self._bufs.get(key)
        if b is None or b.shape[0] < rows or b.shape[1] != w:
            b = torch.empty(max(rows, 1), w, dtype=like.dtype, device=like.device)
            self._bufs[key] = b
        return b[:rows]

    def gather(self, full: torch.Tensor, lo: int = None, hi: int = None, plan=None):
        inf = self.info[id(plan)] if plan is not None else None
        if inf is None or inf["mode"] == "allgather":
            self.rowx.gather(full)
            self.bytes_moved += (full.shape[0] - (self.ranges[self.rank][1] - self.ranges[self.rank][0])) \
                * full.shape[1] * 4
            return
        pl, w = inf["plan"], full.shape[1]
        assert full.is_contiguous() and full.shape[0] == pl.n
        send = self._buf(("s", id(pl), w), sum(inf["send"]), w, full)
        recv = self._buf(("r", id(pl), w), sum(inf["recv"]), w, full)
        if self.comm is not None:
            pl.halo_exchange(full, send, recv, self.comm, w)
            self.bytes_moved += recv.shape[0] * w * 4
            return
        pl.halo_pack(full, send, w)
        if self.backend == "gloo" and full.is_cuda:   # gloo moves host tensors only (tests)
            r_h = torch.empty(recv.shape, dtype=recv.dtype)
            dist.all_to_all_single(r_h, send.cpu(), output_split_sizes=inf["recv"], input_split_sizes=inf["send"],
                                   group=self.group)
            recv.copy_(r_h)
        else:
            dist.all_to_all_single(recv, send, output_split_sizes=inf["recv"], input_split_sizes=inf["send"],
                                   group=self.group)
        pl.halo_unpack(recv, full, w)
        self.bytes_moved += recv.shape[0] * w * 4

    def allreduce(self, t: torch.Tensor):
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)


class PeerExchange:
    """Device-initiated peer gather: no rows are copied.
    Each shard keeps its aggregation inputs (Y0', Y1', dL', dP1') in buffers of
    its own rows that every other shard maps — NVLink peer memory across the
    GPUs of a node, CUDA IPC between processes — and the selective pass
    (pcgcn_forward_peer) reads each source row from its owner.  Before an
    aggregation the shards only synchronise (every producer must have written
    its rows): ``gather`` is a barrier.  Selective-only plans (the full mode's
    window split would need the remote rows)."""

    peer = True

    def __init__(self, plan, group=None):
        from . import _lib as L
        self.L = L
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        row0 = plan.shard_rows(self.world)
        self.ranges = [(int(a), int(b)) for a, b in zip(row0[:-1], row0[1:])]
        check_ranges(self.ranges, plan.n)
        self._bufs, self._peers, self._opened = {}, {}, []
        self._flag = torch.zeros(1, device="cuda") if dist.get_backend(group) == "nccl" else torch.zeros(1)

    def local_buffer(self, key, rows, cols):
        """This shard's buffer for input ``key`` (collective: all ranks call it
        in the same order); returns the torch view of its rows."""
        buf = self.L.IpcBuffer(rows, cols)
        handles = [None] * self.world
        dist.all_gather_object(handles, buf.handle(), group=self.group)
        peers = []
        for q in range(self.world):
            if q == self.rank:
                peers.append(buf.ptr)
            else:
                ptr = self.L.ipc_open(handles[q])
                self._opened.append(ptr)
                peers.append(ptr)
        self._bufs[key], self._peers[key] = buf, peers
        return buf.tensor

    def peers(self, key):
        return self._peers[key]

    def gather(self, full, lo=None, hi=None, plan=None):
        # the producers of every shard must be done before anyone reads: a
        # (stream-ordered, for NCCL) all-reduce of one float is the barrier
        if self._flag.is_cuda:
            dist.all_reduce(self._flag, group=self.group)
        else:
            torch.cuda.synchronize()
            dist.barrier(group=self.group)

    def allreduce(self, t: torch.Tensor):
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)

    def close(self):
        dist.barrier(group=self.group)
        for ptr in self._opened:
            self.L.ipc_close(ptr)
        for b in self._bufs.values():
            b.free()
        self._opened, self._bufs = [], {}
