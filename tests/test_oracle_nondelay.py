"""Pins of the oracle's non-delay dispatch variant (no GPU).

PAPER.md L90 (§2.1): "for each device, TensorFlow randomly picks an operation from the ready
queue (those whose predecessors have completed execution)".  Row f4(i) reads the pick as a
priority: whenever a device is idle it starts, among its ops whose inputs have all arrived, the
one earliest in pi (reading R24).  Links keep Pesto's FCFS queues (L144, L188-198).

Independent checks of `oracle_makespan_model(..., nondelay=1)`:
  * hand-computed worked examples (tests/golden/worked_examples.json, "nondelay" fields; WN2);
  * a discrete-time (tick-by-tick) simulator written below -- a different algorithm from the
    oracle's event heap -- on small integer instances with positive durations;
  * invariants read off the trace: precedence, no device/link overlap, FCFS link order, the
    non-delay property (a device never idles while one of its ops is ready) and the priority
    property (no ready op earlier in pi is passed over);
  * closed forms (one device = sum p; no edges = max device load) and the brute-force optimum
    as a lower bound.
"""

import numpy as np

from workloads import dag
from workloads.rng import SplitMix64


def tt(g, e, a, b):
    D = g.D
    b0, b1 = int(g.beta0[a * D + b]), int(g.beta1[a * D + b])
    return b0 + (int(g.nbytes[e]) * b1 + 999_999) // 1_000_000


def tick_sim(g, x, order, congestion=True):
    """Discrete-time simulation, one integer ns per tick (positive durations only).

    Each tick t: (1) ops and transfers finishing at t deliver their data; (2) every idle link
    starts its FCFS-first released transfer (key: release, pos producer, pos consumer, edge);
    (3) every idle device starts its ready op earliest in pi."""
    n, D = g.n, g.D
    pos = {int(v): k for k, v in enumerate(order)}
    ins = [[] for _ in range(n)]
    outs = [[] for _ in range(n)]
    for e in range(g.m):
        ins[int(g.dst[e])].append(e)
        outs[int(g.src[e])].append(e)
    arrived = [0] * n                  # inputs delivered so far
    ready_at = [None] * n
    S, Cc = [None] * n, [None] * n
    dev_until = [0] * D
    link_until = {}
    queue = {}
    flight = []                        # (arrival time, edge)
    done = 0
    t = 0
    for v in range(n):
        if not ins[v]:
            ready_at[v] = 0
    while done < n:
        # (1) completions at t
        for v in range(n):
            if Cc[v] == t:
                done += 1
                for e in outs[v]:
                    w = int(g.dst[e])
                    if x[w] == x[v]:
                        flight.append((t, e))
                    elif congestion:
                        L = (int(x[v]), int(x[w]))
                        queue.setdefault(L, []).append((t, pos[v], pos[w], e))
                    else:
                        flight.append((t + tt(g, e, int(x[v]), int(x[w])), e))
        # (2) links
        for L, q in queue.items():
            if q and link_until.get(L, 0) <= t:
                q.sort()
                rel, _, _, e = q.pop(0)
                assert rel <= t
                a = t + tt(g, e, L[0], L[1])
                link_until[L] = a
                flight.append((a, e))
        # deliveries at t (same-device data at C_u, transfers at their arrival)
        keep = []
        for a, e in flight:
            if a == t:
                w = int(g.dst[e])
                arrived[w] += 1
                if arrived[w] == len(ins[w]):
                    ready_at[w] = t
            else:
                keep.append((a, e))
        flight = keep
        # (3) devices
        for d in range(D):
            if dev_until[d] > t:
                continue
            cand = [v for v in range(n) if x[v] == d and S[v] is None and ready_at[v] is not None]
            if cand:
                v = min(cand, key=lambda v: pos[v])
                S[v], Cc[v] = t, t + int(g.p[v])
                dev_until[d] = Cc[v]
        t += 1
        assert t < 10 ** 6
    return max(Cc), S, Cc


def _positive_cases(count, seed0, hetero=False):
    r = SplitMix64(seed0)
    for s in range(count):
        n = 1 + r.below(22)
        D = 1 + r.below(4)
        g = dag.random_dag(seed0 + s, n, 0.5 + 2.0 * r.uniform(), D=D, zero_frac=0.0,
                           multi_frac=0.1, p_max=30, max_bytes=3000, allowed_frac=0.0,
                           hetero_links=hetero, beta0=1 + r.below(12), beta1_fs=r.below(6000))
        if (np.asarray(g.beta0)[~np.eye(D, dtype=bool).ravel()] < 1).any():
            continue                   # the variant's domain: every transfer takes >= 1 ns
        order = dag.random_topo_order(g, s)
        x = dag.random_placements(g, s, 1)[0]
        yield g, x, order


def test_tick_simulator_agrees(O):
    for g, x, order in _positive_cases(400, 9100):
        for cong in (True, False):
            mk, S, _ = tick_sim(g, x, order, congestion=cong)
            got, tr = O.makespan_model(g, x, order, congestion=cong, nondelay=True, trace=True)
            assert got == mk, (g.name, cong, got, mk)
            assert [int(v) for v in tr["S"]] == S


def test_tick_simulator_agrees_hetero_links(O):
    for g, x, order in _positive_cases(60, 9700, hetero=True):
        mk, _, _ = tick_sim(g, x, order)
        assert O.makespan_model(g, x, order, nondelay=True) == mk


def _ready_times(g, x, tr):
    rdy = np.zeros(g.n, np.int64)
    for e in range(g.m):
        u, v = int(g.src[e]), int(g.dst[e])
        a = tr["C"][u] if x[u] == x[v] else tr["XA"][e]
        rdy[v] = max(rdy[v], a)
    return rdy


def test_trace_invariants(O):
    for g, x, order in _positive_cases(300, 9400):
        mk, tr = O.makespan_model(g, x, order, nondelay=True, trace=True)
        pos = {int(v): k for k, v in enumerate(order)}
        S, Cc, XS, XA = tr["S"], tr["C"], tr["XS"], tr["XA"]
        assert mk == int(Cc.max())
        assert (Cc == S + g.p).all()
        rdy = _ready_times(g, x, tr)
        assert (S >= rdy).all()                                          # precedence (L144)
        links = {}
        for e in range(g.m):
            u, v = int(g.src[e]), int(g.dst[e])
            if x[u] != x[v]:
                assert XS[e] >= Cc[u] and XA[e] == XS[e] + tt(g, e, int(x[u]), int(x[v]))
                links.setdefault((int(x[u]), int(x[v])), []).append(e)
        for es in links.values():                                         # FCFS, no overlap
            es = sorted(es, key=lambda e: (Cc[int(g.src[e])], pos[int(g.src[e])],
                                           pos[int(g.dst[e])], e))
            for a, b in zip(es, es[1:]):
                assert XS[b] >= XA[a]
        for d in range(g.D):
            ops = sorted([v for v in range(g.n) if x[v] == d], key=lambda v: S[v])
            for a, b in zip(ops, ops[1:]):                                # no overlap (L146)
                assert S[b] >= Cc[a]
            busy = [(int(S[v]), int(Cc[v])) for v in ops]
            for w in ops:
                # non-delay: over [ready(w), S_w) the device is never idle
                t = int(rdy[w])
                while t < S[w]:
                    cover = [c for s, c in busy if s <= t < c]
                    assert cover, (g.name, d, w, t)
                    t = max(cover)
                # priority: an op started while w was ready and unstarted is earlier in pi
                for v in ops:
                    if rdy[w] <= S[v] < S[w]:
                        assert pos[v] < pos[w], (g.name, v, w)


def test_closed_forms(O):
    r = SplitMix64(5)
    for s in range(60):
        g = dag.random_dag(300 + s, 1 + r.below(30), 1.5, D=3, zero_frac=0.0, p_max=100,
                           beta0=1 + r.below(9), beta1_fs=r.below(5000))
        order = dag.random_topo_order(g, s)
        for d in range(3):                                   # one device: never idle, sum p
            x = np.full(g.n, d, np.uint8)
            assert O.makespan_model(g, x, order, nondelay=True) == int(g.p.sum())
        e0 = dag.make_graph("noedge", g.p, [], [], D=3, beta0=1, beta1_fs=0)
        x = dag.random_placements(e0, s, 1)[0]               # no edges: max device load
        load = max(int(g.p[x == d].sum()) for d in range(3))
        assert O.makespan_model(e0, x, np.arange(g.n), nondelay=True) == load


def test_bruteforce_is_a_lower_bound(O):
    r = SplitMix64(8)
    for s in range(25):
        g = dag.random_dag(800 + s, 2 + r.below(5), 1.2, D=2, zero_frac=0.0, p_max=20,
                           beta0=1 + r.below(5), beta1_fs=0)
        best = O.bruteforce(g)[0]
        for k in range(5):
            order = dag.random_topo_order(g, k)
            x = dag.random_placements(g, k, 1)[0]
            assert O.makespan_model(g, x, order, nondelay=True) >= best
