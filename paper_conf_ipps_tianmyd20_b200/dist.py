"""Multi-GPU plumbing for sharded plans.

Destination partitions are sharded over ranks in contiguous plan-row ranges
(the planner's cost-balanced split).  Each aggregation needs the prescaled
source rows of every partition its blocks touch; Reddit-shaped graphs touch
all remote rows, so the exchange is an all-gather of the producer's output
rows into the full-height input buffer (one broadcast per owner into its row
range — ranges are uneven).  ∇Θ (one flat buffer) and the loss are summed
with one all-reduce each.  torch.distributed (NCCL on GPUs, gloo in the CPU
tests) is the transport; the arithmetic stays in libpcgcn.
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

    def gather(self, full: torch.Tensor, lo: int = None, hi: int = None):
        """full[lo_q:hi_q] of every rank q becomes visible on every rank."""
        if full.shape[0] != self.ranges[-1][1]:
            raise ValueError(f"full buffer has {full.shape[0]} rows, ranges cover {self.ranges[-1][1]}")
        for q, (a, b) in enumerate(self.ranges):
            if b > a:
                dist.broadcast(full[a:b], src=self.src[q], group=self.group)

    def allreduce(self, t: torch.Tensor):
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)
