"""Graph container, fixed fixtures and seeded random DAG / order / placement inputs.

Holds no arithmetic of the method: nothing here computes a start time, a
transfer time or a makespan. It builds the inputs of the problem statement
(§3.2.1): a DAG G=(V,E) with per-op compute time p_i, per-edge
transfer size in bytes (L138 §3.1), D devices, and the per-ordered-link linear
comm coefficients (beta0 ns, beta1 fs/byte).
"""

from __future__ import annotations

from dataclasses import dataclass, field
from typing import List, Optional

import numpy as np

from .rng import SplitMix64


@dataclass
class Graph:
    name: str
    n: int
    p: np.ndarray            # int64 [n], compute ns >= 0
    src: np.ndarray          # int32 [m]
    dst: np.ndarray          # int32 [m]
    nbytes: np.ndarray       # int64 [m], transfer size in bytes
    D: int = 2
    beta0: Optional[np.ndarray] = None   # int64 [D*D], ns (diagonal unused)
    beta1: Optional[np.ndarray] = None   # int64 [D*D], fs per byte (diagonal unused)
    allowed: Optional[np.ndarray] = None  # uint8 [n] device bitmask, None = all
    layer: Optional[np.ndarray] = None    # int32 [n] layer tag (expert seed only)
    roles: Optional[List[str]] = None
    meta: dict = field(default_factory=dict)

    @property
    def m(self) -> int:
        return int(self.src.shape[0])

    def with_comm(self, D: int, beta0: int, beta1_fs: int) -> "Graph":
        """Same graph with a homogeneous comm model on every ordered pair a != b."""
        b0 = np.full(D * D, beta0, dtype=np.int64)
        b1 = np.full(D * D, beta1_fs, dtype=np.int64)
        for d in range(D):
            b0[d * D + d] = 0
            b1[d * D + d] = 0
        g = Graph(self.name, self.n, self.p, self.src, self.dst, self.nbytes, D, b0, b1,
                  self.allowed, self.layer, self.roles, dict(self.meta))
        return g

    def preds(self):
        pr = [[] for _ in range(self.n)]
        for e in range(self.m):
            pr[int(self.dst[e])].append(e)
        return pr

    def succs(self):
        su = [[] for _ in range(self.n)]
        for e in range(self.m):
            su[int(self.src[e])].append(e)
        return su


def make_graph(name, p, edges, nbytes=None, D=2, beta0=0, beta1_fs=0, allowed=None,
               layer=None, roles=None) -> Graph:
    """Build a Graph from Python lists. `edges` is a list of (src, dst)."""
    p = np.asarray(p, dtype=np.int64)
    src = np.asarray([e[0] for e in edges], dtype=np.int32)
    dst = np.asarray([e[1] for e in edges], dtype=np.int32)
    if nbytes is None:
        nbytes = [0] * len(edges)
    g = Graph(name, int(p.shape[0]), p, src, dst, np.asarray(nbytes, dtype=np.int64),
              allowed=None if allowed is None else np.asarray(allowed, dtype=np.uint8),
              layer=None if layer is None else np.asarray(layer, dtype=np.int32),
              roles=roles)
    return g.with_comm(D, beta0, beta1_fs)


# ---------------------------------------------------------------------------------------
# tiny12 fixture: source 0, chain A = 1..5, chain B = 6..10,
# sink 11, cross edge 2 -> 8.  beta0 = 1000 ns, beta1 = 1e6 fs/B (1 ns/B).
# ---------------------------------------------------------------------------------------
TINY12_P = [2000, 5000, 3000, 8000, 2000, 4000, 6000, 1000, 7000, 3000, 5000, 1000]
TINY12_EDGES = [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5), (5, 11),
                (0, 6), (6, 7), (7, 8), (8, 9), (9, 10), (10, 11), (2, 8)]
TINY12_BYTES = [4096, 2048, 6144, 1024, 3072, 2048, 4096, 1024, 8192, 2048, 3072, 1024, 5120]


def tiny12() -> Graph:
    return make_graph("tiny12", TINY12_P, TINY12_EDGES, TINY12_BYTES, D=2,
                      beta0=1000, beta1_fs=1_000_000)


def all_linear_extensions(g: Graph) -> List[List[int]]:
    """Every topological order of a tiny DAG (plain recursive enumeration)."""
    preds = [set() for _ in range(g.n)]
    for s, d in zip(g.src.tolist(), g.dst.tolist()):
        preds[d].add(s)
    out: List[List[int]] = []
    cur: List[int] = []
    placed = [False] * g.n

    def rec():
        if len(cur) == g.n:
            out.append(list(cur))
            return
        for v in range(g.n):
            if not placed[v] and all(placed[u] for u in preds[v]):
                placed[v] = True
                cur.append(v)
                rec()
                cur.pop()
                placed[v] = False

    rec()
    return out


# ---------------------------------------------------------------------------------------
# Random inputs
# ---------------------------------------------------------------------------------------
def random_dag(seed: int, n: int, avg_out: float = 1.5, D: int = 2, *, max_bytes: int = 1 << 20,
               p_max: int = 10_000, zero_frac: float = 0.1, multi_frac: float = 0.05,
               fan_in_hub: int = 0, fan_out_hub: int = 0, locality: int = 0,
               allowed_frac: float = 0.0,
               beta0: Optional[int] = None, beta1_fs: Optional[int] = None,
               hetero_links: bool = False) -> Graph:
    """Random DAG on n ops: a hidden random rank order; edges go from lower to higher rank.

    zero_frac: fraction of zero-duration ops and zero-byte edges.
    multi_frac: fraction of edges duplicated as multi-edges (Q4).
    fan_in_hub: if > 0, one op receives that many extra in-edges (fan-in > 32 / > 1024 cases).
    fan_out_hub: if > 0, one op gets that many extra out-edges (out-of-line edge records).
    locality: if > 0, edge endpoints are at most `locality` ranks apart (long-lived slots rarer).
    allowed_frac: fraction of ops given a random non-full allowed-device mask.
    """
    r = SplitMix64(seed)
    rank = list(range(n))
    r.shuffle(rank)                      # op rank[i] is the i-th in the hidden order
    p = []
    for _ in range(n):
        if r.chance(zero_frac):
            p.append(0)
        else:
            p.append(r.log_uniform_int(1, p_max + 1))
    edges = []
    nb = []
    m_target = int(round(avg_out * n)) if n > 1 else 0
    for _ in range(m_target):
        a = r.below(n)
        if locality > 0:
            b = a + 1 + r.below(locality)
            if b >= n:
                continue
        else:
            b = r.below(n)
        if a == b:
            continue
        if a > b:
            a, b = b, a
        u, v = rank[a], rank[b]
        w = 0 if r.chance(zero_frac) else r.log_uniform_int(1, max_bytes + 1)
        edges.append((u, v))
        nb.append(w)
        if r.chance(multi_frac):
            edges.append((u, v))
            nb.append(r.log_uniform_int(1, max_bytes + 1))
    if fan_in_hub > 0 and n > 2:
        # the hub is the last op of the hidden order, fed by fan_in_hub random earlier ops
        hub = rank[n - 1]
        for _ in range(fan_in_hub):
            a = r.below(n - 1)
            edges.append((rank[a], hub))
            nb.append(r.log_uniform_int(1, max_bytes + 1))
    if fan_out_hub > 0 and n > 2:
        # the first op of the hidden order feeds fan_out_hub random later ops
        hub = rank[0]
        for _ in range(fan_out_hub):
            b = 1 + r.below(n - 1)
            edges.append((hub, rank[b]))
            nb.append(r.log_uniform_int(1, max_bytes + 1))
    allowed = None
    if allowed_frac > 0:
        full = (1 << D) - 1
        allowed = []
        for _ in range(n):
            if r.chance(allowed_frac):
                msk = 0
                while msk == 0:
                    msk = r.below(full + 1)
                allowed.append(msk)
            else:
                allowed.append(full)
    b0 = r.log_uniform_int(1, 20_000) if beta0 is None else beta0
    b1 = r.log_uniform_int(1, 100_000) if beta1_fs is None else beta1_fs
    g = make_graph(f"rand{seed}", p, edges, nb, D=D, beta0=b0, beta1_fs=b1, allowed=allowed)
    if hetero_links:
        for a in range(D):
            for b in range(D):
                if a != b:
                    g.beta0[a * D + b] = r.log_uniform_int(1, 20_000)
                    g.beta1[a * D + b] = r.log_uniform_int(1, 100_000)
    return g


def random_topo_order(g: Graph, seed: int) -> np.ndarray:
    """Kahn's algorithm with a seeded uniformly random pick from the ready set
    (the TensorFlow default ready-queue behaviour, §2.1)."""
    r = SplitMix64(seed)
    indeg = [0] * g.n
    succ = [[] for _ in range(g.n)]
    for s, d in zip(g.src.tolist(), g.dst.tolist()):
        indeg[d] += 1
        succ[s].append(d)
    ready = [v for v in range(g.n) if indeg[v] == 0]
    order = []
    while ready:
        i = r.below(len(ready))
        v = ready[i]
        ready[i] = ready[-1]
        ready.pop()
        order.append(v)
        for w in succ[v]:
            indeg[w] -= 1
            if indeg[w] == 0:
                ready.append(w)
    if len(order) != g.n:
        raise ValueError("graph has a cycle")
    return np.asarray(order, dtype=np.int32)


def random_placements(g: Graph, seed: int, count: int) -> np.ndarray:
    """[count, n] uint8 device codes, uniform over each op's allowed devices."""
    rng = np.random.default_rng(seed)
    x = rng.integers(0, g.D, size=(count, g.n), dtype=np.uint8)
    if g.allowed is not None:
        for v in range(g.n):
            devs = [d for d in range(g.D) if (int(g.allowed[v]) >> d) & 1]
            if len(devs) < g.D:
                x[:, v] = np.asarray(devs, dtype=np.uint8)[rng.integers(0, len(devs), size=count)]
    return x


def pack_placements(x: np.ndarray, D: int, row_stride: Optional[int] = None) -> np.ndarray:
    """Pack [count, n] device codes into rows of b bits/op, little-endian within each byte
    (op i occupies bits [b*i, b*i+b) of the row), rows padded to a multiple of 16 bytes.
    b = 1 (D <= 2), 2 (D <= 4), 4 (D <= 8).  This is the `pesto_eval_batch` row format."""
    count, n = x.shape
    b = 1 if D <= 2 else (2 if D <= 4 else 4)
    row_bytes = (n * b + 7) // 8
    if row_stride is None:
        row_stride = (row_bytes + 15) // 16 * 16
    out = np.zeros((count, row_stride), dtype=np.uint8)
    xs = x.astype(np.uint16)
    for k in range(b):
        bits = ((xs >> k) & 1).astype(np.uint8)           # [count, n]
        # bit position of (op i, plane k) = b*i + k
        pos = np.arange(n) * b + k
        byte_idx = pos // 8
        bit_idx = (pos % 8).astype(np.uint8)
        for i in range(8):
            sel = bit_idx == i
            if not sel.any():
                continue
            contrib = bits[:, sel] << i
            # each byte index appears once for a fixed bit index i, so fancy-index OR is exact
            out[:, byte_idx[sel]] |= contrib
    return out


def random_packed_rows(g: Graph, seed: int, count: int, chunk: int = 65536) -> np.ndarray:
    """[count, stride] packed rows (the `pesto_eval_batch` format of `pack_placements`) of
    placements uniform over all device codes, drawn directly as random bits so that 1M-row
    batches need no [count, n] intermediate.  For graphs whose every op allows all devices and
    D a power of two (every code < D) this is the distribution of `random_placements`."""
    if g.allowed is not None and (np.asarray(g.allowed) != (1 << g.D) - 1).any():
        raise ValueError("random_packed_rows needs all-allowed masks")
    if g.D & (g.D - 1):
        raise ValueError("random_packed_rows needs D a power of two")
    b = 1 if g.D <= 2 else (2 if g.D <= 4 else 4)
    nbits = g.n * b
    stride = ((nbits + 7) // 8 + 15) // 16 * 16
    out = np.empty((count, stride), dtype=np.uint8)
    rng = np.random.default_rng(seed)
    tail = np.zeros(stride, dtype=np.uint8)              # keep only the row's nbits
    tail[: nbits // 8] = 0xFF
    if nbits % 8:
        tail[nbits // 8] = (1 << (nbits % 8)) - 1
    for a in range(0, count, chunk):
        e = min(count, a + chunk)
        out[a:e] = rng.integers(0, 256, size=(e - a, stride), dtype=np.uint8) & tail
    return out
