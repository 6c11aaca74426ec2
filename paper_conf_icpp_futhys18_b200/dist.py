"""Data-parallel plumbing of the hot path: batch sharding across ranks and
one all_reduce(SUM) of the flat dW||db buffer.  Host logic only — the per-rank compute is the
library's kernels; torch.distributed (NCCL on GPUs, gloo in the CPU tests) does the exchange.

Reading R10: dy already carries 1/N_global (batch-averaged loss), so summing the
per-rank gradients gives the full-batch gradient.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Sequence, Tuple


def shard_range(n_global: int, rank: int, world: int) -> Tuple[int, int]:
    """Samples [start, stop) of rank `rank` (contiguous, sizes differ by at most one)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    base, rem = divmod(n_global, world)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


@dataclass
class GradSlot:
    w_shape: Tuple[int, int, int, int]
    w_off: int
    b_off: int
    co: int


class FlatGrads:
    """One contiguous fp32 buffer [dW_1 | db_1 | ... | dW_L | db_L] with per-layer views, so the
    whole step's parameter gradients are exchanged by a single collective."""

    def __init__(self, w_shapes: Sequence[Tuple[int, int, int, int]], device="cpu", dtype=None):
        import torch
        self.slots: List[GradSlot] = []
        off = 0
        for s in w_shapes:
            n = s[0] * s[1] * s[2] * s[3]
            self.slots.append(GradSlot(tuple(s), off, off + n, s[0]))
            off += n + s[0]
        self.numel = off
        self.buf = torch.zeros(off, device=device, dtype=dtype or torch.float32)

    def dw(self, i):
        s = self.slots[i]
        return self.buf[s.w_off:s.b_off].view(s.w_shape)

    def db(self, i):
        s = self.slots[i]
        return self.buf[s.b_off:s.b_off + s.co]

    def allreduce(self, group=None):
        import torch.distributed as dist
        if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
            dist.all_reduce(self.buf, op=dist.ReduceOp.SUM, group=group)
        return self.buf
