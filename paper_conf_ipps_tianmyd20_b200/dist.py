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


class RowExchange:
    def __init__(self, lo: int, hi: int, group=None):
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        ranges = [None] * self.world
        dist.all_gather_object(ranges, (int(lo), int(hi)), group=group)
        self.ranges = ranges
        assert ranges[self.rank] == (lo, hi)
        for a, b in zip(ranges, ranges[1:]):
            assert a[1] == b[0], "shard ranges must tile the rows"

    def gather(self, full: torch.Tensor, lo: int = None, hi: int = None):
        """full[lo_q:hi_q] of every rank q becomes visible on every rank."""
        for q, (a, b) in enumerate(self.ranges):
            if b > a:
                dist.broadcast(full[a:b], src=q, group=self.group)

    def allreduce(self, t: torch.Tensor):
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)
