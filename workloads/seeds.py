"""Search incumbents as INPUTS, written in plain Python.

libpesto has the same seed generators in C++ (`pesto_seed_order`, `pesto_seed_placement`; row
a1).  This independent restatement lets the CPU reference arm of bench.py start from exactly the
bases the GPU arm searches without loading libpesto, and `tests/test_lib_host.py` checks that the
two agree op for op.  It holds none of the method's arithmetic (no makespan, no move decoding):
orders are Kahn traversals, placements are device codes.

  * critical-path order: Kahn by max bottom level (longest path to a sink counting p only),
    ties by smaller op id (Fig. 2b's list order);
  * FIFO order: Kahn with a FIFO queue, out-edges visited in edge-input order;
  * random order: Kahn with a seeded pick from the ready set (TF's default dispatch, L90):
    index = SplitMix64 next mod |ready|, the picked entry replaced by the last one;
  * expert placement: device floor(layer * D / n_layers) (contiguous layers, L308);
  * topological split: pi cut into D contiguous segments of about equal sum p (mTOPO-like,
    L320): op v goes to floor((2 * before + p_v) * D / (2 * total));
  * single device: every op on its lowest allowed device;
  * random placement: per op, the (next mod popcount)-th allowed device.
Ops whose mask forbids the chosen device take their lowest allowed one.
"""

from __future__ import annotations

import heapq

import numpy as np

from .rng import SplitMix64


def _csr(g):
    order = np.argsort(g.src, kind="stable")           # out-edges of each op in input order
    off = np.zeros(g.n + 1, np.int64)
    np.add.at(off, g.src.astype(np.int64) + 1, 1)
    off = np.cumsum(off)
    return off, g.dst[order].astype(np.int64)


def _allowed(g, v):
    return 0xFF if g.allowed is None else int(g.allowed[v])


def _lowest(g, v):
    a = _allowed(g, v)
    for d in range(g.D):
        if (a >> d) & 1:
            return d
    return 0


def order_critical_path(g) -> np.ndarray:
    off, dsts = _csr(g)
    indeg = np.bincount(g.dst, minlength=g.n).astype(np.int64)
    deg = indeg.copy()
    topo = [v for v in range(g.n) if deg[v] == 0]
    h = 0
    while h < len(topo):
        v = topo[h]
        h += 1
        for w in dsts[off[v]:off[v + 1]]:
            deg[w] -= 1
            if deg[w] == 0:
                topo.append(int(w))
    bl = np.zeros(g.n, np.int64)
    p = g.p.astype(np.int64)
    for v in reversed(topo):
        s = dsts[off[v]:off[v + 1]]
        bl[v] = p[v] + (int(bl[s].max()) if len(s) else 0)
    deg = indeg.copy()
    heap = [(-int(bl[v]), v) for v in range(g.n) if deg[v] == 0]
    heapq.heapify(heap)
    out = []
    while heap:
        _, v = heapq.heappop(heap)
        out.append(v)
        for w in dsts[off[v]:off[v + 1]]:
            deg[w] -= 1
            if deg[w] == 0:
                heapq.heappush(heap, (-int(bl[w]), int(w)))
    return np.asarray(out, np.int32)


def order_fifo(g) -> np.ndarray:
    off, dsts = _csr(g)
    deg = np.bincount(g.dst, minlength=g.n).astype(np.int64)
    out = [v for v in range(g.n) if deg[v] == 0]
    h = 0
    while h < len(out):
        v = out[h]
        h += 1
        for w in dsts[off[v]:off[v + 1]]:
            deg[w] -= 1
            if deg[w] == 0:
                out.append(int(w))
    return np.asarray(out, np.int32)


def order_random(g, seed: int) -> np.ndarray:
    off, dsts = _csr(g)
    deg = np.bincount(g.dst, minlength=g.n).astype(np.int64)
    rng = SplitMix64(seed)
    ready = [v for v in range(g.n) if deg[v] == 0]
    out = []
    while ready:
        i = rng.next_u64() % len(ready)
        v = ready[i]
        ready[i] = ready[-1]
        ready.pop()
        out.append(v)
        for w in dsts[off[v]:off[v + 1]]:
            deg[w] -= 1
            if deg[w] == 0:
                ready.append(int(w))
    return np.asarray(out, np.int32)


def _fix(g, v, d):
    return d if (_allowed(g, v) >> d) & 1 else _lowest(g, v)


def place_single(g) -> np.ndarray:
    return np.asarray([_lowest(g, v) for v in range(g.n)], np.uint8)


def place_expert(g, layer) -> np.ndarray:
    layer = np.asarray(layer, np.int64)
    nl = int(layer.max()) + 1
    return np.asarray([_fix(g, v, int(layer[v]) * g.D // nl) for v in range(g.n)], np.uint8)


def place_topo_split(g, order) -> np.ndarray:
    p = g.p.astype(np.int64)
    total = int(p.sum())
    x = np.zeros(g.n, np.uint8)
    before = 0
    for k, v in enumerate(np.asarray(order).tolist()):
        if total > 0:
            d = ((2 * before + int(p[v])) * g.D) // (2 * total)
        else:
            d = k * g.D // g.n
        x[v] = _fix(g, v, min(d, g.D - 1))
        before += int(p[v])
    return x


def place_random(g, seed: int) -> np.ndarray:
    rng = SplitMix64(seed)
    x = np.zeros(g.n, np.uint8)
    for v in range(g.n):
        a = _allowed(g, v) & ((1 << g.D) - 1) if g.allowed is not None else (1 << g.D) - 1
        ds = [d for d in range(g.D) if (a >> d) & 1]
        x[v] = ds[rng.next_u64() % len(ds)]
    return x


def bench_seeds(g, n_bases: int = 4, seed: int = 2021):
    """The bench's P = 4 incumbents (SURVEY §8(d) "Search"): expert (topological split when the
    graph has no layer tags) on the critical-path order, topological split on the critical-path
    order, single device on the FIFO order, random placement on a random order."""
    o_cp = order_critical_path(g)
    o_fifo = order_fifo(g)
    o_rand = order_random(g, seed)
    xs = [place_expert(g, g.layer) if getattr(g, "layer", None) is not None
          else place_topo_split(g, o_cp),
          place_topo_split(g, o_cp), place_single(g), place_random(g, seed)]
    os_ = [o_cp, o_cp, o_fifo, o_rand]
    return np.stack(xs[:n_bases]), np.stack(os_[:n_bases])
