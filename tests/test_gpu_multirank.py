"""The library's multi-rank search path in two processes on ONE GPU.

Each rank builds its own pesto_graph / pesto_search (rank r of world 2, no NCCL comm: two ranks
cannot share one GPU in NCCL), evaluates its contiguous share of every base's candidate ids with
the timed kernels (pesto_search_eval), reads its per-base minima (pesto_search_keys), MIN-reduces
them with the other rank over gloo -- the exchange ncclAllReduce performs on a multi-GPU box --
writes the global minima back (pesto_search_set_keys) and commits (pesto_search_commit).  Bases
must be identical on both ranks after every step and equal to the oracle's world-2 reference
step (oracle_search_step, per-rank minima then the minimum)."""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from workloads import dag

pytestmark = pytest.mark.gpu

MIX = (40, 20, 20, 20)
K, STEPS, SEED = 8192, 5, 23


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _graph():
    return dag.random_dag(131, 1400, 1.6, D=2, p_max=4000, max_bytes=300_000, beta0=700,
                          beta1_fs=30_000)


def _bases(g):
    orders = np.stack([dag.random_topo_order(g, 40 + b) for b in range(3)]).astype(np.int32)
    return dag.random_placements(g, 77, 3), orders


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        from paper_conf_middleware_hafeezsg021_b200 import pesto as P
        g = _graph()
        xs, orders = _bases(g)
        G = P.Graph.from_arrays(g, device=0)
        S = P.Search(G, xs, orders, K, MIX, seed=SEED, rank=rank, world=world)
        hist = []
        for step in range(STEPS):
            S.eval()
            local = S.keys()
            # unsigned MIN through a signed MIN: flip the top bit (order preserving)
            t = torch.from_numpy((local ^ np.uint64(1 << 63)).view(np.int64).copy())
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            red = t.numpy().view(np.uint64) ^ np.uint64(1 << 63)
            S.set_keys(red)
            S.commit()
            state = [S.get(b) for b in range(3)]
            hist.append((local.copy(), red.copy(),
                         [(mk, x.copy(), o.copy()) for mk, x, o in state]))
        q.put((rank, hist))
        dist.destroy_process_group()
    except Exception as e:                                   # surface the failure to the parent
        q.put((rank, repr(e)))
        raise


def test_two_processes_one_gpu_equal_oracle_world2(O):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
    assert all(not isinstance(res[r], str) for r in range(world)), res
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    g = _graph()
    rx, ro = _bases(g)
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(3)], np.int64)
    for step in range(STEPS):
        # each rank's local minima are the oracle's minima over that rank's id range
        for r in range(world):
            lo, hi = K * r // world, K * (r + 1) // world
            want = [O.candidate_keys(g, 3, b, rx, ro, lo, hi, SEED, step, MIX).min()
                    for b in range(3)]
            assert [int(k) for k in res[r][step][0]] == [int(k) for k in want], (step, r)
        keys = O.search_step(g, rx, ro, rmk, K, SEED, step, MIX, world=world)
        for r in range(world):
            assert (res[r][step][1] == keys).all(), (step, r)
            for b in range(3):
                mk, x, o = res[r][step][2][b]
                assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, r, b)
