"""Pins of the CPU oracle against what PAPER.md and mathematics fix (no GPU).

Every check here is independent of the oracle's own code path: hand-computed worked
examples (tests/golden/worked_examples.json), closed forms, invariants I1-I10 read off the
event trace, agreement of three different formulations (event simulation, longest path in
the augmented DAG, a plain position-order recursion written below), and brute force.
"""

import itertools
import json
import os

import numpy as np
import pytest

from workloads import dag
from workloads.rng import SplitMix64, mix64 as py_mix64

GOLD = os.path.join(os.path.dirname(__file__), "golden")
INF = (1 << 63) - 1


def tt(g, e, a, b):
    """transfer time of edge e on link a->b, by the Q6 rule restated with Python ints."""
    D = g.D
    b0, b1 = int(g.beta0[a * D + b]), int(g.beta1[a * D + b])
    prod = int(g.nbytes[e]) * b1
    return b0 + (prod + 999_999) // 1_000_000


def recursion(g, x, order):
    """Plain recursion of SURVEY §8(c) (formulation #3): ops in pi order, a per-link
    free time advanced in producer order, transfers of one producer in (pos v, e) order."""
    n = g.n
    pos = {int(v): k for k, v in enumerate(order)}
    ins = [[] for _ in range(n)]
    outs = [[] for _ in range(n)]
    for e in range(g.m):
        ins[int(g.dst[e])].append(e)
        outs[int(g.src[e])].append(e)
    dev_free = [0] * g.D
    link_free = {}
    arr = {}
    C = [0] * n
    for v in order:
        v = int(v)
        r = max([arr[e] for e in ins[v]], default=0)
        d = int(x[v])
        s = max(r, dev_free[d])
        C[v] = s + int(g.p[v])
        dev_free[d] = C[v]
        for e in sorted(outs[v], key=lambda e: (pos[int(g.dst[e])], e)):
            w = int(g.dst[e])
            if int(x[w]) != d:
                L = (d, int(x[w]))
                st = max(C[v], link_free.get(L, 0))
                arr[e] = st + tt(g, e, d, int(x[w]))
                link_free[L] = arr[e]
            else:
                arr[e] = C[v]
    return max(C)


def critical_path_p(g):
    """Longest path counting p only (textbook DAG DP in a topological order)."""
    order = dag.random_topo_order(g, 1)
    fin = [0] * g.n
    ins = [[] for _ in range(g.n)]
    for e in range(g.m):
        ins[int(g.dst[e])].append(int(g.src[e]))
    for v in order:
        fin[v] = max([fin[u] for u in ins[v]], default=0) + int(g.p[v])
    return max(fin)


# ------------------------------------------------------------------------------------------
# worked examples and the comm-model rule
# ------------------------------------------------------------------------------------------
def _worked():
    data = json.load(open(os.path.join(GOLD, "worked_examples.json")))
    for ex in data["examples"]:
        yield ex


@pytest.mark.parametrize("ex", list(_worked()), ids=lambda ex: ex["name"])
def test_worked_examples(O, ex):
    g = dag.make_graph(ex["name"], ex["p"], [tuple(e) for e in ex["edges"]],
                       [1] * len(ex["edges"]), D=2, beta0=ex["t"], beta1_fs=0)
    for case in ex["cases"]:
        assert O.makespan(g, case["x"], case["order"]) == case["makespan"], (ex["name"], case)
        assert O.longest_path(g, case["x"], case["order"]) == case["makespan"]
        if "nocongest" in case:
            assert O.makespan_nocongest(g, case["x"], case["order"]) == case["nocongest"]
        if "nondelay" in case:                                    # row f4(i), reading R24
            assert O.makespan_model(g, case["x"], case["order"], nondelay=True) == case["nondelay"]
        assert O.makespan_model(g, case["x"], case["order"]) == case["makespan"]
    if "optimum" in ex:
        assert O.bruteforce(g)[0] == ex["optimum"]


def test_transfer_rule_table(O):
    for nbytes, b0, b1, expect in json.load(open(os.path.join(GOLD, "transfer_ns.json")))["cases"]:
        assert O.transfer_ns(nbytes, b0, b1) == expect, (nbytes, b0, b1)


def test_splitmix64_reference_values(O):
    # SplitMix64 (Steele, Lea, Flood 2014) from state 0: published first outputs
    r = SplitMix64(0)
    expect = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]
    got = [r.next_u64() for _ in range(3)]
    assert got == expect
    gamma = 0x9E3779B97F4A7C15
    for k in range(1, 4):
        z = (gamma * k) & ((1 << 64) - 1)
        assert O.mix64(z) == py_mix64(z) == expect[k - 1]


# ------------------------------------------------------------------------------------------
# closed forms and textbook reductions
# ------------------------------------------------------------------------------------------
def test_single_device_is_sum_p(O):
    for s in range(20):
        g = dag.random_dag(100 + s, 40, 1.5, D=3)
        order = dag.random_topo_order(g, s)
        for d in range(3):
            x = np.full(g.n, d, np.uint8)
            assert O.makespan(g, x, order) == int(g.p.sum())
        g1 = dag.random_dag(100 + s, 40, 1.5, D=1)
        assert O.makespan(g1, np.zeros(g1.n, np.uint8), dag.random_topo_order(g1, s)) == int(g1.p.sum())


def test_no_edges_is_max_load(O):
    r = SplitMix64(7)
    for s in range(30):
        n = 1 + r.below(12)
        p = [r.below(50) for _ in range(n)]
        g = dag.make_graph("noedge", p, [], [], D=3, beta0=5, beta1_fs=0)
        x = np.asarray([r.below(3) for _ in range(n)], np.uint8)
        load = [sum(p[v] for v in range(n) if x[v] == d) for d in range(3)]
        assert O.makespan(g, x, list(range(n))) == max(load)


def test_no_edges_optimum_is_partition(O):
    """optimum over x of max device load = P||Cmax, here by subset-sum DP for D=2."""
    r = SplitMix64(8)
    for s in range(10):
        n = 2 + r.below(7)
        p = [1 + r.below(30) for _ in range(n)]
        g = dag.make_graph("part", p, [], [], D=2, beta0=1, beta1_fs=0)
        total = sum(p)
        reach = {0}
        for w in p:
            reach |= {a + w for a in reach}
        best = min(max(a, total - a) for a in reach)
        assert O.bruteforce(g)[0] == best


def test_all_crossing_chain(O):
    """a chain alternating devices: every edge crosses, nothing overlaps -> sum p + sum t."""
    for s in range(10):
        n = 10
        r = SplitMix64(s)
        p = [r.below(1000) for _ in range(n)]
        edges = [(i, i + 1) for i in range(n - 1)]
        nb = [r.below(100000) for _ in range(n - 1)]
        g = dag.make_graph("chain", p, edges, nb, D=2, beta0=r.below(5000), beta1_fs=r.below(90000))
        x = np.asarray([i % 2 for i in range(n)], np.uint8)
        expect = sum(p) + sum(tt(g, e, i % 2, (i + 1) % 2) for e, i in enumerate(range(n - 1)))
        assert O.makespan(g, x, list(range(n))) == expect


def test_zero_comm_is_longest_path_with_device_edges(O):
    """beta = 0: makespan = longest p-weighted path in G plus sigma_d edges (textbook)."""
    for s in range(30):
        g = dag.random_dag(400 + s, 30, 1.6, D=3, beta0=0, beta1_fs=0)
        order = dag.random_topo_order(g, s)
        x = dag.random_placements(g, s, 1)[0]
        ins = [[] for _ in range(g.n)]
        for e in range(g.m):
            ins[int(g.dst[e])].append(int(g.src[e]))
        last = {}
        for v in order:
            v = int(v)
            if int(x[v]) in last:
                ins[v].append(last[int(x[v])])
            last[int(x[v])] = v
        fin = {}
        for v in order:
            v = int(v)
            fin[v] = max([fin[u] for u in ins[v]], default=0) + int(g.p[v])
        assert O.makespan(g, x, order) == max(fin.values())


# ------------------------------------------------------------------------------------------
# three formulations agree, on many random DAGs with ties, zeros, multi-edges, hubs
# ------------------------------------------------------------------------------------------
def _random_cases(count, seed0=1000):
    r = SplitMix64(seed0)
    for s in range(count):
        n = 1 + r.below(40)
        D = 2 + r.below(3)
        hub = [0, 0, 0, 40][r.below(4)]
        g = dag.random_dag(seed0 + s, n, 0.5 + 2.0 * r.uniform(), D=D, zero_frac=0.2,
                           multi_frac=0.1, fan_in_hub=hub, p_max=50, max_bytes=2000,
                           allowed_frac=0.0, hetero_links=bool(r.below(2)),
                           beta0=r.below(30), beta1_fs=r.below(20_000))
        order = dag.random_topo_order(g, s)
        x = dag.random_placements(g, s, 1)[0]
        yield g, x, order


def test_three_way_agreement(O):
    for g, x, order in _random_cases(1500):
        a = O.makespan(g, x, order)
        b = O.longest_path(g, x, order)
        c = recursion(g, x, order)
        assert a == b == c, (g.name, a, b, c)


def test_fan_in_over_1024(O):
    g = dag.random_dag(77, 60, 1.0, D=2, fan_in_hub=1500, p_max=100, max_bytes=5000,
                       beta0=3, beta1_fs=7000)
    for s in range(3):
        order = dag.random_topo_order(g, s)
        x = dag.random_placements(g, s, 1)[0]
        assert O.makespan(g, x, order) == O.longest_path(g, x, order) == recursion(g, x, order)


# ------------------------------------------------------------------------------------------
# invariants I1-I10 on the event trace
# ------------------------------------------------------------------------------------------
def check_trace(g, x, order, mk, tr):
    n, D = g.n, g.D
    pos = {int(v): k for k, v in enumerate(order)}
    S, Cc, XS, XA = tr["S"], tr["C"], tr["XS"], tr["XA"]
    assert mk == int(Cc.max())
    for v in range(n):
        assert Cc[v] == S[v] + g.p[v]
    link_items = {}
    for e in range(g.m):
        u, v = int(g.src[e]), int(g.dst[e])
        if x[u] == x[v]:
            assert XS[e] == -1 and S[v] >= Cc[u]                       # I1 same device
        else:
            t = tt(g, e, int(x[u]), int(x[v]))
            assert XS[e] >= Cc[u] and XA[e] == XS[e] + t and S[v] >= XA[e]   # I1 cross
            link_items.setdefault((int(x[u]), int(x[v])), []).append(e)
    for d in range(D):                                                    # I2
        ops = sorted([v for v in range(n) if x[v] == d], key=lambda v: pos[v])
        for a, b in zip(ops, ops[1:]):
            assert S[b] >= Cc[a]
    for L, es in link_items.items():                                      # I3
        es_fcfs = sorted(es, key=lambda e: (pos[int(g.src[e])], pos[int(g.dst[e])], e))
        for a, b in zip(es_fcfs, es_fcfs[1:]):
            assert XS[b] >= XA[a]
    # I6 semi-active: an op starts at 0, at its device predecessor's C, or at an arrival
    prev = {}
    for v in sorted(range(n), key=lambda v: pos[v]):
        cands = {0}
        if int(x[v]) in prev:
            cands.add(int(Cc[prev[int(x[v])]]))
        prev[int(x[v])] = v
        for e in range(g.m):
            if int(g.dst[e]) == v:
                u = int(g.src[e])
                cands.add(int(Cc[u]) if x[u] == x[v] else int(XA[e]))
        assert int(S[v]) in cands
    for L, es in link_items.items():
        es_fcfs = sorted(es, key=lambda e: (pos[int(g.src[e])], pos[int(g.dst[e])], e))
        for i, e in enumerate(es_fcfs):
            c = {int(Cc[int(g.src[e])])}
            if i:
                c.add(int(XA[es_fcfs[i - 1]]))
            assert int(XS[e]) in c
    # I4 lower bounds, I4' placement-aware bound, I5 upper bound
    load = [int(g.p[x == d].sum()) for d in range(D)]
    assert mk >= max(critical_path_p(g), max(load))
    assert mk >= -(-int(g.p.sum()) // D)
    fin = {}
    ins = [[] for _ in range(n)]
    for e in range(g.m):
        ins[int(g.dst[e])].append(e)
    for v in sorted(range(n), key=lambda v: pos[v]):
        best = 0
        for e in ins[v]:
            u = int(g.src[e])
            w = fin[u] + (tt(g, e, int(x[u]), int(x[v])) if x[u] != x[v] else 0)
            best = max(best, w)
        fin[v] = best + int(g.p[v])
    assert mk >= max(fin.values())
    cross_t = sum(tt(g, e, int(x[int(g.src[e])]), int(x[int(g.dst[e])]))
                  for e in range(g.m) if x[int(g.src[e])] != x[int(g.dst[e])])
    assert mk <= int(g.p.sum()) + cross_t


def test_invariants_I1_to_I6(O):
    for g, x, order in _random_cases(300, seed0=5000):
        mk, tr = O.makespan(g, x, order, trace=True)
        check_trace(g, x, order, mk, tr)


def test_I7_monotone(O):
    r = SplitMix64(11)
    for g, x, order in _random_cases(150, seed0=6000):
        mk = O.makespan(g, x, order)
        g2 = dag.Graph(g.name, g.n, g.p.copy(), g.src, g.dst, g.nbytes, g.D, g.beta0.copy(),
                       g.beta1.copy(), g.allowed)
        g2.p[r.below(g.n)] += 1 + r.below(100)
        assert O.makespan(g2, x, order) >= mk
        g3 = dag.Graph(g.name, g.n, g.p, g.src, g.dst, g.nbytes, g.D, g.beta0 + r.below(50),
                       g.beta1 + r.below(5000), g.allowed)
        for d in range(g.D):
            g3.beta0[d * g.D + d] = 0
            g3.beta1[d * g.D + d] = 0
        assert O.makespan(g3, x, order) >= mk


def test_I8_interleaving_invariance(O):
    """two orders with equal per-device restrictions give equal makespans."""
    for g, x, order in _random_cases(150, seed0=7000):
        edges = list(zip(g.src.tolist(), g.dst.tolist()))
        last = {}
        for v in order:
            v = int(v)
            if int(x[v]) in last:
                edges.append((last[int(x[v])], v))
            last[int(x[v])] = v
        aug = dag.make_graph("aug", g.p, edges, [0] * len(edges), D=g.D)
        order2 = dag.random_topo_order(aug, 99)
        assert O.makespan(g, x, order) == O.makespan(g, x, order2)


def test_I9_device_relabel_symmetry(O):
    for g, x, order in _random_cases(150, seed0=8000):
        g = g.with_comm(g.D, 13, 17_000)                                  # homogeneous links
        perm = list(range(g.D))
        SplitMix64(g.n).shuffle(perm)
        x2 = np.asarray([perm[int(d)] for d in x], np.uint8)
        assert O.makespan(g, x, order) == O.makespan(g, x2, order)


def test_I10_all_on_one_device(O):
    for g, x, order in _random_cases(50, seed0=9000):
        assert O.makespan(g, np.zeros(g.n, np.uint8), order) == int(g.p.sum())


# ------------------------------------------------------------------------------------------
# brute force (Thm 3.1's optimality analogue, L204-206)
# ------------------------------------------------------------------------------------------
def test_tiny12_bruteforce(O):
    g = dag.tiny12()
    exts = dag.all_linear_extensions(g)
    assert len(exts) == 186                       # 60+60+45+21
    best, bx, bo, count = O.bruteforce(g)
    assert count == 186 * 4096
    assert O.makespan(g, bx, bo) == best
    # the optimum is no worse than every single-device or alternating placement
    for d in range(2):
        assert best <= O.makespan(g, np.full(12, d, np.uint8), exts[0])
    golden = json.load(open(os.path.join(GOLD, "tiny12_optimum.json")))
    assert best == golden["optimum"]


def test_random_bruteforce_vs_python_enumeration(O):
    r = SplitMix64(21)
    for s in range(12):
        n = 2 + r.below(5)
        g = dag.random_dag(2000 + s, n, 1.2, D=2, p_max=30, max_bytes=3000,
                           beta0=r.below(20), beta1_fs=r.below(9000))
        best_py = INF
        for order in dag.all_linear_extensions(g):
            for x in itertools.product(range(2), repeat=n):
                best_py = min(best_py, recursion(g, np.asarray(x, np.uint8), order))
        assert O.bruteforce(g)[0] == best_py


# ------------------------------------------------------------------------------------------
# validation / error codes
# ------------------------------------------------------------------------------------------
def test_error_codes(O):
    g = dag.make_graph("cyc", [1, 1, 1], [(0, 1), (1, 2), (2, 0)], [1, 1, 1], D=2, beta0=1)
    assert O.makespan(g, [0, 0, 0], [0, 1, 2]) == O.ECYCLE
    g = dag.make_graph("ok", [1, 1, 1], [(0, 1), (1, 2)], [1, 1], D=2, beta0=1)
    assert O.makespan(g, [0, 0, 0], [1, 0, 2]) == O.ENOTTOPO
    assert O.makespan(g, [0, 0, 0], [0, 0, 2]) == O.ENOTTOPO
    assert O.makespan(g, [0, 2, 0], [0, 1, 2]) == O.INFEASIBLE
    bad = dag.make_graph("self", [1, 1], [(0, 0)], [1], D=2, beta0=1)
    assert O.makespan(bad, [0, 0], [0, 1]) == O.EINVAL
    neg = dag.make_graph("neg", [1, -1], [], [], D=2, beta0=1)
    assert O.makespan(neg, [0, 0], [0, 1]) == O.EINVAL
    big = dag.make_graph("big", [1 << 39, 1 << 39], [], [], D=2, beta0=1)
    assert O.makespan(big, [0, 1], [0, 1]) == O.EOVERFLOW
    ok = dag.make_graph("edge", [1 << 38, 1 << 38], [], [], D=2, beta0=1)
    assert O.makespan(ok, [0, 1], [0, 1]) == 1 << 38
    allowed = dag.make_graph("aff", [1, 1], [(0, 1)], [1], D=2, beta0=1, allowed=[1, 2])
    assert O.makespan(allowed, [1, 1], [0, 1]) == O.INFEASIBLE
    assert O.makespan(allowed, [0, 1], [0, 1]) == 3


# ---------------------------------------------------------------------------------------
# Row f3: memory footprint and colocation (L175) constraints
# ---------------------------------------------------------------------------------------
def _f3_graph():
    # a -> b carries 100 B, a -> c 50 B; footprints (input + output tensors, L202):
    # a = 150, b = 100, c = 50 (hand-computed)
    return dag.make_graph("f3", [1, 1, 1], [(0, 1), (0, 2)], [100, 50], D=2, beta0=3,
                          beta1_fs=0)


def test_f3_memory_caps_worked_example(O):
    """cap 200 B per device: feasible placements (x_a x_b x_c) are exactly 010, 011, 100, 101
    (hand-computed: e.g. 000 puts 300 B on device 0, 110 puts 250 B on device 1)."""
    g = _f3_graph()
    order = np.asarray([0, 1, 2], np.int32)
    feasible = {"010", "011", "100", "101"}
    with O.constraints(g, cap=[200, 200]) as c:
        for bits in itertools.product([0, 1], repeat=3):
            x = np.asarray(bits, np.uint8)
            key = "".join(map(str, bits))
            assert c.ok(x) == (key in feasible), key
            mk = O.makespan(g, x, order)
            assert (mk == INF) == (key not in feasible), key
    # the constraint is off again outside the block
    assert O.makespan(g, np.zeros(3, np.uint8), order) == 3


def test_f3_explicit_footprints_and_colocation(O):
    g = _f3_graph()
    order = np.asarray([0, 1, 2], np.int32)
    # explicit footprints: a = 10, b = 10, c = 100; cap [100, 1000]: c may not join a or b on 0
    with O.constraints(g, mem=[10, 10, 100], cap=[100, 1000]) as c:
        assert c.ok(np.asarray([0, 0, 1], np.uint8)) and not c.ok(np.asarray([1, 0, 0], np.uint8))
    # colocation {a, c}: x_a == x_c (L175)
    with O.constraints(g, coloc=[2, -1, 2]) as c:
        for bits in itertools.product([0, 1], repeat=3):
            x = np.asarray(bits, np.uint8)
            assert c.ok(x) == (bits[0] == bits[2])
            assert (O.makespan(g, x, order) == INF) == (bits[0] != bits[2])


def test_f3_search_respects_constraints(O):
    """the reference search never commits an infeasible candidate and its keys mark them."""
    g = dag.random_dag(77, 60, 1.5, D=2, p_max=3000, max_bytes=200_000, beta0=500,
                       beta1_fs=25_000)
    mem = np.zeros(g.n, np.int64)
    np.add.at(mem, g.src, g.nbytes)
    np.add.at(mem, g.dst, g.nbytes)
    cap = [int(mem.sum() * 0.6)] * 2
    coloc = np.full(g.n, -1, np.int32)
    coloc[[3, 9, 17]] = 4
    x0 = (np.arange(g.n) % 2).astype(np.uint8)
    x0[[3, 9, 17]] = 1
    orders = np.stack([dag.random_topo_order(g, 1)]).astype(np.int32)
    with O.constraints(g, cap=cap, coloc=coloc) as c:
        assert c.ok(x0)
        xs = x0[None].copy()
        mk = np.asarray([O.makespan(g, xs[0], orders[0])], np.int64)
        keys = O.candidate_keys(g, 1, 0, xs, orders, 0, 600, 5, 0, (50, 20, 20, 10))
        n_bad = 0
        for j in range(600):
            ok, x, o = O.candidate(g, 1, 0, xs, orders, j, 5, 0, (50, 20, 20, 10))
            if ok and not c.ok(x):
                assert keys[j] == (1 << 64) - 1
                n_bad += 1
        assert n_bad > 0
        for step in range(3):
            O.search_step(g, xs, orders, mk, 600, 5, step, (50, 20, 20, 10))
            assert c.ok(xs[0])
