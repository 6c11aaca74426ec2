"""CPU (gloo, world_size 2) tests of the multi-GPU path's host logic: batch sharding, the flat
dW||db buffer and its single all_reduce.  The per-rank compute is the oracle (a fake backend), so
the test checks sharding/ordering/scaling with no GPU."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from glp_workloads import gen_custom
from paper_conf_icpp_futhys18_b200.dist import FlatGrads, shard_range

LAYERS = [(4, 3, 9, 9, 5, 3, 1, 1), (4, 5, 7, 7, 6, 3, 2, 1)]   # N, C, H, W, Co, K, S, P


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _data():
    out = []
    for i, (N, C, H, W, Co, K, S, P) in enumerate(LAYERS):
        Ho = oracle.out_dim(H, K, S, P)
        out.append(gen_custom(N, C, H, W, Co, K, K, 40 + i, Ho=Ho, Wo=Ho))
    return out


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    data = _data()
    fg = FlatGrads([(L[4], L[1], L[5], L[5]) for L in LAYERS])
    for i, (N, C, H, W, Co, K, S, P) in enumerate(LAYERS):
        a, b = shard_range(N, rank, world)
        d = data[i]
        dw, db = oracle.conv_bwd_filter(d["x"][a:b], d["dy"][a:b], d["w"].shape, S, P)
        fg.dw(i).copy_(torch.from_numpy(dw.astype(np.float32)))
        fg.db(i).copy_(torch.from_numpy(db.astype(np.float32)))
    local = fg.buf.clone()
    fg.allreduce()
    q.put((rank, local.numpy(), fg.buf.numpy()))
    dist.barrier()
    dist.destroy_process_group()


def test_shard_range_partition():
    for n in (1, 7, 64, 256, 257):
        for w in (1, 2, 3, 4, 8):
            if w > n:
                continue
            rs = [shard_range(n, r, w) for r in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(w - 1))
            sizes = [b - a for a, b in rs]
            assert max(sizes) - min(sizes) <= 1


def test_flat_grads_views():
    fg = FlatGrads([(2, 3, 3, 3), (4, 2, 1, 1)])
    assert fg.numel == 2 * 27 + 2 + 4 * 2 + 4
    fg.dw(1).fill_(1.0)
    fg.db(0).fill_(2.0)
    assert float(fg.buf.sum()) == 8 * 1.0 + 2 * 2.0
    assert fg.dw(0).shape == (2, 3, 3, 3) and fg.db(1).shape == (4,)


def test_gloo_allreduce_equals_full_batch():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=240) for _ in range(world)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    locals_ = [r[1] for r in res]
    reduced = [r[2] for r in res]
    # every rank holds the same reduced buffer; for G = 2 it is the fp32 sum of the two halves
    np.testing.assert_array_equal(reduced[0], reduced[1])
    np.testing.assert_array_equal(reduced[0], (locals_[0] + locals_[1]).astype(np.float32))
    # and equals the full-batch oracle gradients (sum over the whole batch, R10)
    data = _data()
    off = 0
    for i, (N, C, H, W, Co, K, S, P) in enumerate(LAYERS):
        dw, db = oracle.conv_bwd_filter(data[i]["x"], data[i]["dy"], data[i]["w"].shape, S, P)
        n = dw.size
        assert oracle.normwise_err(reduced[0][off:off + n].reshape(dw.shape), dw) < 1e-6
        assert oracle.normwise_err(reduced[0][off + n:off + n + Co], db) < 1e-6
        off += n + Co


# ----------------------------------------------------------- deterministic tree exchange -----

from paper_conf_icpp_futhys18_b200.dist import LEAVES, TreeAllreduce, leaf_range, rank_leaves, tree_sum  # noqa: E402


def _leaf_parts(n=4099, seed=5):
    # partial sums spanning many magnitudes, so a different summation order changes bits
    r = np.random.default_rng(seed)
    return [(r.standard_normal(n) * 10.0 ** r.uniform(-6, 6, n)).astype(np.float32)
            for _ in range(LEAVES)]


def _tree_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    parts = _leaf_parts()
    mine = [torch.from_numpy(parts[j].copy()) for j in rank_leaves(rank, world)]
    out = TreeAllreduce()(mine)
    q.put((rank, out.numpy().copy()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_tree_allreduce_bitwise_invariant_across_world_sizes(world):
    """The tree all-reduce gives every rank the same bits, equal to the 1-process tree over all
    leaves, for 2, 4 and 8 ranks (gloo); plain left-to-right summation gives different bits."""
    ref = tree_sum([torch.from_numpy(p.copy()) for p in _leaf_parts()],
                   lambda a, b, o: torch.add(a, b, out=o)).numpy()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_tree_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        np.testing.assert_array_equal(res[r], ref)
    seq = np.zeros_like(ref)
    for p in _leaf_parts():
        seq = (seq + p).astype(np.float32)
    assert not np.array_equal(seq, ref)   # the order matters: the test can see a wrong tree
    np.testing.assert_allclose(ref, np.sum(np.stack(_leaf_parts()).astype(np.float64), 0),
                               rtol=1e-5, atol=1e-2)


def test_leaf_partition():
    assert [leaf_range(256, j) for j in (0, 7)] == [(0, 32), (224, 256)]
    assert rank_leaves(1, 4) == [2, 3] and rank_leaves(0, 1) == list(range(8))
    with pytest.raises(ValueError):
        rank_leaves(0, 3)
    with pytest.raises(ValueError):
        leaf_range(100, 0)


def _bucket_worker(rank, world, port, q):
    """bench.py's overlapped exchange: one all_reduce per unit bucket, issued in reverse layer
    order, must give the same buffer as the single whole-buffer all_reduce."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    shapes = [(4, 3, 3, 3), (6, 4, 1, 1), (5, 6, 5, 5)]
    a, b = FlatGrads(shapes), FlatGrads(shapes)
    g = torch.Generator().manual_seed(100 + rank)
    a.buf.copy_(torch.randn(a.numel, generator=g))
    pad = torch.ones(a.numel, dtype=torch.bool)   # the alignment padding between slots stays 0
    for sl in a.slots:
        pad[sl.w_off:sl.b_off + sl.co] = False
    a.buf[pad] = 0.0
    b.buf.copy_(a.buf)
    a.allreduce()
    works = [dist.all_reduce(b.bucket([i]), async_op=True) for i in reversed(range(len(shapes)))]
    for w in works:
        w.wait()
    q.put((rank, a.buf.numpy().copy(), b.buf.numpy().copy(),
           b.bucket([1, 2]).numel() == b.slots[2].b_off + b.slots[2].co - b.slots[1].w_off
           and all(sl.w_off % 4 == 0 for sl in b.slots)))
    dist.barrier()
    dist.destroy_process_group()


def test_bucketed_allreduce_equals_flat():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bucket_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for _, flat, buck, ok in res:
        assert ok
        np.testing.assert_array_equal(flat, buck)   # two-operand fp32 sums: bitwise
    np.testing.assert_array_equal(res[0][1], res[1][1])


def _subgroup_tree_worker(rank, world, port, q):
    """TreeAllreduce on a subgroup whose group ranks differ from the global ranks (global ranks
    1 and 3 of 4 form the group): the partner must be mapped to its global rank."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    grp = dist.new_group([1, 3])
    if rank in (1, 3):
        gr = dist.get_rank(grp)
        parts = _leaf_parts()
        mine = [torch.from_numpy(parts[j].copy()) for j in rank_leaves(gr, 2)]
        out = TreeAllreduce(group=grp)(mine)
        q.put((rank, out.numpy().copy()))
    dist.barrier()
    dist.destroy_process_group()


def test_tree_allreduce_on_subgroup():
    ref = tree_sum([torch.from_numpy(p.copy()) for p in _leaf_parts()],
                   lambda a, b, o: torch.add(a, b, out=o)).numpy()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_subgroup_tree_worker, args=(r, 4, port, q)) for r in range(4)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
    assert sorted(res) == [1, 3]
    for r in res:
        np.testing.assert_array_equal(res[r], ref)
