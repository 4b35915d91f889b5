"""World-size-2 gloo tests of the multi-GPU search path's host logic.

The device path shards candidate ids as [floor(rK/W), floor((r+1)K/W)) per rank, reduces the
packed (makespan << 24 | j) keys with a MIN allreduce, and every rank commits the same winner.
Here each rank scores its shard with the CPU oracle, the keys are MIN-reduced over gloo, and
the result must equal the unsharded step on every rank.
"""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from workloads import dag

MIX = (50, 20, 20, 10)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from oracle import oracle as O
    g = dag.random_dag(61, 80, 1.5, D=2, p_max=3000, max_bytes=100_000, beta0=300,
                       beta1_fs=20_000)
    P, K = 2, 1000
    xs = dag.random_placements(g, 3, P)
    orders = np.stack([dag.random_topo_order(g, 10 + b) for b in range(P)]).astype(np.int32)
    mk = np.asarray([O.makespan(g, xs[b], orders[b]) for b in range(P)], np.int64)
    for step in range(3):
        keys = np.zeros(P, np.uint64)
        lo, hi = K * rank // world, K * (rank + 1) // world
        for b in range(P):
            keys[b] = O.candidate_keys(g, P, b, xs, orders, lo, hi, 7, step, MIX, 1).min()
        t = torch.from_numpy(keys.view(np.int64).copy())
        # keys < 2^63 here (makespan << 24 fits), so signed MIN == unsigned MIN
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        red = t.numpy().view(np.uint64)
        xs1, or1, mk1 = xs.copy(), orders.copy(), mk.copy()
        ref = O.search_step(g, xs1, or1, mk1, K, 7, step, MIX, world=1, threads=1)
        assert (red == ref).all(), (rank, step, red, ref)
        # every rank commits the same winner from the reduced key
        for b in range(P):
            j = int(red[b]) & ((1 << 24) - 1)
            if j:
                ok, x, o = O.candidate(g, P, b, xs, orders, j, 7, step, MIX)
                xs[b], orders[b] = x, o
            mk[b] = int(red[b]) >> 24
        assert (xs == xs1).all() and (orders == or1).all() and (mk == mk1).all()
        h = torch.tensor([int(np.bitwise_xor.reduce(xs.ravel().astype(np.int64) * 131 +
                                                    np.arange(xs.size)))], dtype=torch.int64)
        hs = [torch.zeros_like(h) for _ in range(world)]
        dist.all_gather(hs, h)
        assert all(int(x) == int(hs[0]) for x in hs)              # bases identical on all ranks
    out[rank] = 1
    dist.destroy_process_group()


def test_two_rank_sharded_search_equals_single_rank():
    world = 2
    ctx = mp.get_context("spawn")
    out = ctx.Array("i", world)
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, out)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    assert list(out) == [1, 1]


def test_rank_ranges_partition_every_candidate():
    for K in (1, 7, 1000, 1 << 16):
        for W in (1, 2, 3, 8):
            ranges = [(K * r // W, K * (r + 1) // W) for r in range(W)]
            assert ranges[0][0] == 0 and ranges[-1][1] == K
            assert all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
