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
            off = (off + 3) // 4 * 4   # every dW starts 16-byte aligned (the library checks)
        self.numel = off
        self.buf = torch.zeros(off, device=device, dtype=dtype or torch.float32)

    def dw(self, i):
        s = self.slots[i]
        return self.buf[s.w_off:s.b_off].view(s.w_shape)

    def db(self, i):
        s = self.slots[i]
        return self.buf[s.b_off:s.b_off + s.co]

    def bucket(self, idxs):
        """The contiguous slice [dW_i | db_i | ... ] of the slots `idxs` (consecutive): one unit's
        all-reduce bucket, issued as soon as that unit's filter gradient is reduced (bench.py
        overlaps the buckets with the remaining backward, in reverse layer order)."""
        lo = self.slots[min(idxs)].w_off
        hi = max(self.slots[j].b_off + self.slots[j].co for j in idxs)
        return self.buf[lo:hi]

    def allreduce(self, group=None):
        import torch.distributed as dist
        if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
            dist.all_reduce(self.buf, op=dist.ReduceOp.SUM, group=group)
        return self.buf


# ------------------------------------------------------------ deterministic exchange (NEXT-2) ---

LEAVES = 8   # fixed number of batch leaves: the tree (and so every dW bit) is the same for 1..8 ranks


def leaf_range(n_global: int, leaf: int, leaves: int = LEAVES) -> Tuple[int, int]:
    """Samples [start, stop) of batch leaf `leaf` (equal contiguous leaves; leaves | n_global)."""
    if n_global % leaves or not 0 <= leaf < leaves:
        raise ValueError("the global batch must split into equal leaves")
    n = n_global // leaves
    return leaf * n, (leaf + 1) * n


def rank_leaves(rank: int, world: int, leaves: int = LEAVES) -> List[int]:
    """The contiguous block of leaves rank `rank` computes (world must be a power of two <= leaves
    dividing it, so a rank's block is one subtree of the fixed tree)."""
    if world < 1 or leaves % world or world & (world - 1) or not 0 <= rank < world:
        raise ValueError("world must be a power of two dividing the leaf count")
    per = leaves // world
    return list(range(rank * per, (rank + 1) * per))


def tree_sum(parts, add):
    """Fixed balanced binary tree over `parts` (a power-of-two count, in leaf order): level by
    level, node = add(left, right).  Returns a new buffer (inputs are not modified)."""
    level = list(parts)
    if not level or len(level) & (len(level) - 1):
        raise ValueError("need a power-of-two number of parts")
    first = True
    while len(level) > 1:
        nxt = []
        for i in range(0, len(level), 2):
            a, b = level[i], level[i + 1]
            out = a.clone() if first else a   # never write into the caller's leaf buffers
            add(a, b, out)
            nxt.append(out)
        level = nxt
        first = False
    return level[0] if not first else level[0].clone()


def _default_add(a, b, out):
    if a.is_cuda:
        from . import sum2
        return sum2(a, b, out)
    import torch
    return torch.add(a, b, out=out)


class TreeAllreduce:
    """Deterministic all-reduce of per-leaf partial sums (include/glp.h "deterministic gradient
    exchange"): each rank holds the partials of its leaves (rank_leaves), sums them with the local
    subtree of a fixed binary tree over LEAVES leaves, then combines subtree sums by recursive
    doubling (log2(world) exchanges with partner rank ^ d; the lower-ranked subtree is always the
    left operand).  Every rank ends with the same bits, and the bits do not depend on the world
    size: every fp32 add is a node of the same tree, and a + b == b + a.  `add(a, b, out)` is the
    library's glp_sum2 on CUDA tensors (torch.add on CPU, for the gloo tests)."""

    def __init__(self, group=None, add=None):
        self.group = group
        self.add = add or _default_add

    def __call__(self, parts):
        import torch.distributed as dist
        acc = tree_sum(parts, self.add)
        if not (dist.is_available() and dist.is_initialized()):
            return acc
        if acc.is_cuda and dist.get_backend(self.group) == "gloo":
            # gloo moves host memory only: run the exchange on a host copy (IEEE fp32 adds are
            # correctly rounded on both sides, so the bits are those of the device adds)
            dev = acc.device
            out = TreeAllreduce(self.group, add=lambda a, b, o: __import__("torch").add(a, b, out=o))(
                [acc.cpu()])
            return out.to(dev)
        world = dist.get_world_size(self.group)
        rank = dist.get_rank(self.group)   # rank within the group
        recv = acc.clone()
        d = 1
        while d < world:
            partner = rank ^ d
            # P2POp takes the peer's GLOBAL rank: map the group rank (identity for the default group)
            peer = partner if self.group is None else dist.get_global_rank(self.group, partner)
            ops = [dist.P2POp(dist.isend, acc, peer, self.group),
                   dist.P2POp(dist.irecv, recv, peer, self.group)]
            for r in dist.batch_isend_irecv(ops):
                r.wait()
            if rank < partner:
                self.add(acc, recv, acc)
            else:
                self.add(recv, acc, acc)
            d <<= 1
        return acc


class LeafTreeExchange:
    """The deterministic gradient exchange as the library runs it (P264
    convergence invariance extended across GPU counts):

      1. the filter gradient of a leaf plan (glp_plan_options_t.wgrad_leaves = this rank's leaves)
         reduces its split partials per leaf into `leaves` ([L, numel], one flat dW||db buffer per
         leaf; glp_stage_reduce_leaves) -- the step packs x and dy once, only the reduction is split;
      2. glp_tree_sum sums the rank's leaves with its subtree of the fixed 8-leaf binary tree;
      3. world > 1: the top levels across ranks -- over torch symmetric memory, glp_tree_exchange
         (each rank computes a slice of the top tree with NVLink peer loads and stores it into every
         rank's buffer, between two symmetric-memory barriers), or, without symmetric memory,
         recursive doubling over torch.distributed point-to-point (TreeAllreduce).
    Every fp32 add is a node of the same tree, so the result is bitwise identical for 1, 2, 4 and
    8 ranks."""

    def __init__(self, numel, n_local_leaves, device, group=None, transport="auto"):
        import torch
        import torch.distributed as dist
        self.numel, self.L, self.group = int(numel), int(n_local_leaves), group
        self.leaves = torch.zeros(self.L, self.numel, device=device)
        self.world = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if self.world > 1 else 0
        self.transport = "local"
        if self.world > 1:
            self.transport = "p2p"
            if transport in ("auto", "symm") and torch.device(device).type == "cuda":
                try:
                    import torch.distributed._symmetric_memory as symm
                    name = (group or dist.group.WORLD).group_name
                    self.sub = symm.empty(self.numel, device=device)
                    self.out = symm.empty(self.numel, device=device)
                    self.hs = symm.rendezvous(self.sub, name)
                    self.ho = symm.rendezvous(self.out, name)
                    self.transport = "symm"
                except Exception:
                    if transport == "symm":
                        raise
        if self.transport != "symm":
            self.sub = torch.empty(self.numel, device=device)

    def __call__(self, flat):
        """flat <- the tree over every rank's leaves (all ranks get the same bits)."""
        from . import tree_sum
        tree_sum([self.leaves[l] for l in range(self.L)], self.sub)
        if self.transport == "local":
            flat.copy_(self.sub)
        elif self.transport == "symm":
            from . import tree_exchange
            self.hs.barrier(channel=0)
            tree_exchange(self.hs.buffer_ptrs, self.ho.buffer_ptrs, self.rank, self.numel)
            self.ho.barrier(channel=0)
            flat.copy_(self.out)
        else:
            flat.copy_(TreeAllreduce(self.group)([self.sub]))
        return flat
