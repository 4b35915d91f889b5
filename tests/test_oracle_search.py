"""Pins of the oracle's reference local-search step (no GPU).

The search is the north star's method, not a paper method, so its pins are the properties
its spec fixes: the counter-based draw, what each move type may change, the identity
candidate, the min/commit rule, and that W simulated ranks give the single-rank result.
"""

import numpy as np
import pytest

from workloads import dag
from workloads.rng import mix64

MIX = (50, 20, 20, 10)


def _setup(seed=5, n=60, D=2, allowed_frac=0.0, P=3):
    g = dag.random_dag(seed, n, 1.4, D=D, p_max=2000, max_bytes=50_000, beta0=300,
                       beta1_fs=20_000, allowed_frac=allowed_frac)
    orders = np.stack([dag.random_topo_order(g, 10 + b) for b in range(P)]).astype(np.int32)
    xs = dag.random_placements(g, 3, P)
    return g, xs, orders


def test_draw_matches_spec_text(O):
    for (seed, step, P, b, j, k) in [(2021, 0, 4, 0, 0, 0), (1, 7, 3, 2, 12345, 15),
                                     (2 ** 64 - 1, 2 ** 40, 4, 3, 2 ** 24 - 1, 9)]:
        ctr = ((((step * P + b) * (1 << 24) + j) * 16 + k)) & ((1 << 64) - 1)
        assert O.draw(seed, step, P, b, j, k) == mix64(seed ^ mix64(ctr))


def test_identity_and_move_shapes(O):
    g, xs, orders = _setup()
    edges = set(zip(g.src.tolist(), g.dst.tolist()))
    P, n = xs.shape
    seen = {"flip": 0, "window": 0, "swap": 0}
    mix = (50, 20, 20, 60)                                # swap-heavy (v6 blocks pairs on
    for b in range(P):                                    # different base devices)
        ok, x, o = O.candidate(g, P, b, xs, orders, 0, 2021, 3, mix)
        assert ok and (x == xs[b]).all() and (o == orders[b]).all()
        W = mix[0] + mix[1] + mix[2]
        b2 = (128 * (mix[0] + mix[1])) // W
        for j in range(1, 2048):
            ok, x, o = O.candidate(g, P, b, xs, orders, j, 2021, 3, mix)
            if not ok:
                # no masks here: only a WINDOW lane can be invalid (v7: fewer than two eligible
                # ops from its start, or every window length of that start already used)
                assert j % 128 >= b2
                continue
            diff_pos = np.nonzero(o != orders[b])[0]
            if len(diff_pos):
                seen["swap"] += 1
                k = int(diff_pos[0])
                assert list(diff_pos) == [k, k + 1]
                assert o[k] == orders[b][k + 1] and o[k + 1] == orders[b][k]
                a, c = int(orders[b][k]), int(orders[b][k + 1])
                assert (a, c) not in edges
                # S3: swapped ops share no producer and no consumer, fan-out <= 64
                preds = lambda v: {s for s, d in edges if d == v}
                succs = lambda v: {d for s, d in edges if s == v}
                assert not (preds(a) & preds(c)) and not (succs(a) & succs(c))
                assert len(succs(a)) <= 64 and len(succs(c)) <= 64
                assert xs[b][a] == xs[b][c]                  # same base device (v6)
                assert O.makespan(g, x, o) >= 0           # still topological
                if j % 128 == 0:
                    assert (x == xs[b]).all()              # lane 0 of a swap group: pure swap
            changed = np.nonzero(x != xs[b])[0]
            if len(changed) == 0:
                continue
            dev = set(x[changed].tolist())
            pos_changed = sorted(int(np.nonzero(orders[b] == v)[0][0]) for v in changed)
            if len(changed) <= 4:
                seen["flip"] += 1
            if len(dev) == 1 and pos_changed[-1] - pos_changed[0] < 64:
                seen["window"] += 1
            assert len(changed) <= 4 or (len(dev) == 1 and pos_changed[-1] - pos_changed[0] < 64)
    assert seen["flip"] > 0 and seen["window"] > 0 and seen["swap"] > 0


def test_group_changes_stay_in_its_region(O):
    """every change a group of 128 candidates makes lies in its region [c_g, c_g + 64), the
    regions of consecutive groups tile the order (DESIGN §4 S2, v6)."""
    g, xs, orders = _setup(seed=6, n=300)
    P = xs.shape[0]
    R = (g.n + 63) // 64
    for b in range(P):
        rot = O.draw(2021, 2, P, b, 0, 13) % R
        for grp in range(1, 12):
            c = 64 * ((grp + rot) % R)
            hi = min(g.n, c + 64)
            for lane in range(128):
                j = 128 * grp + lane
                ok, x, o = O.candidate(g, P, b, xs, orders, j, 2021, 2, MIX)
                changed = np.nonzero(x != xs[b])[0]
                pos = [int(np.nonzero(orders[b] == v)[0][0]) for v in changed]
                assert all(c <= q < hi for q in pos), (grp, lane, c, pos)
                diff = np.nonzero(o != orders[b])[0]
                if len(diff):
                    assert c <= diff[0] < hi or diff[0] == g.n - 2


def test_moves_respect_allowed(O):
    g, xs, orders = _setup(seed=9, n=50, D=4, allowed_frac=0.6)
    for v in range(g.n):                                  # make the bases feasible
        if not (int(g.allowed[v]) >> int(xs[0][v])) & 1:
            xs[:, v] = [d for d in range(4) if (int(g.allowed[v]) >> d) & 1][0]
    P = xs.shape[0]
    for b in range(P):
        for j in range(1, 800):
            ok, x, o = O.candidate(g, P, b, xs, orders, j, 77, 1, MIX)
            if ok:
                for v in range(g.n):
                    assert (int(g.allowed[v]) >> int(x[v])) & 1


def test_flip_without_movable_ops_is_invalid(O):
    g, xs, orders = _setup(seed=4, n=20)
    g.allowed = np.ones(g.n, np.uint8)                    # every op pinned to device 0
    xs[:] = 0
    keys = O.candidate_keys(g, 3, 0, xs, orders, 0, 256, 5, 0, (1, 0, 0, 0))
    assert keys[0] != O.KEY_INVALID
    assert all(k == O.KEY_INVALID for k in keys[1:])


def test_step_min_commit_and_sharding(O):
    g, xs, orders = _setup(seed=12, n=40)
    P = xs.shape[0]
    K = 300
    mk = np.asarray([O.makespan(g, xs[b], orders[b]) for b in range(P)], np.int64)
    for step in range(4):
        keys_all = [O.candidate_keys(g, P, b, xs, orders, 0, K, 2021, step, MIX) for b in range(P)]
        xs1, or1, mk1 = xs.copy(), orders.copy(), mk.copy()
        keys1 = O.search_step(g, xs1, or1, mk1, K, 2021, step, MIX, world=1)
        xs3, or3, mk3 = xs.copy(), orders.copy(), mk.copy()
        keys3 = O.search_step(g, xs3, or3, mk3, K, 2021, step, MIX, world=3)
        assert (keys1 == keys3).all() and (xs1 == xs3).all() and (or1 == or3).all()
        for b in range(P):
            assert int(keys1[b]) == int(keys_all[b].min())
            assert int(keys_all[b][0]) == (int(mk[b]) << 24)      # j=0 is the base itself
            assert mk1[b] <= mk[b]
            assert O.makespan(g, xs1[b], or1[b]) == mk1[b]        # committed base re-evaluates
        xs, orders, mk = xs1, or1, mk1


def test_keys_equal_makespan_of_decoded_candidate(O):
    g, xs, orders = _setup(seed=13, n=30)
    keys = O.candidate_keys(g, 3, 1, xs, orders, 0, 200, 42, 9, MIX)
    valid = 0
    for j in range(200):
        ok, x, o = O.candidate(g, 3, 1, xs, orders, j, 42, 9, MIX)
        if not ok:                                  # an invalid (v7 WINDOW) lane: no key
            assert int(keys[j]) == 2**64 - 1
            continue
        valid += 1
        assert int(keys[j]) == (O.makespan(g, x, o) << 24) | j
    assert valid > 150


def test_coarse_group_moves_spec(O):
    """S9 (row f2): in a coarse group every candidate moves exactly the ops of one merged
    vertex that allow the drawn device -- the vertex and device restated from the spec text --
    with the order unchanged; other groups decode exactly as without coarse moves."""
    g, xs, orders = _setup(seed=9, n=80, D=3, allowed_frac=0.3)
    P, n = xs.shape
    coarse_of = (np.arange(n) * 7 % 5).astype(np.int32)      # 5 merged vertices, interleaved
    pct, seed, step = 40, 77, 2
    plain = {}
    for b in range(P):
        for j in range(0, 1536):
            plain[(b, j)] = O.candidate(g, P, b, xs, orders, j, seed, step, MIX)
    n_coarse_groups = 0
    with O.coarse_moves(g, coarse_of, 5, pct):
        for b in range(P):
            for j in range(0, 1536):
                ok, x, o = O.candidate(g, P, b, xs, orders, j, seed, step, MIX)
                grp = j >> 7
                coarse = grp != 0 and O.draw(seed, step, P, b, 128 * grp, 12) % 100 < pct
                if not coarse:
                    pok, px, po = plain[(b, j)]
                    assert ok == pok and (x == px).all() and (o == po).all()
                    continue
                n_coarse_groups += (j & 127) == 0
                assert ok and (o == orders[b]).all()
                k = O.draw(seed, step, P, b, j, 10) % 5
                d = O.draw(seed, step, P, b, j, 11) % 3
                want = xs[b].copy()
                for v in range(n):
                    if coarse_of[v] == k and (g.allowed is None or (g.allowed[v] >> d) & 1):
                        want[v] = d
                assert (x == want).all(), (b, j)
    assert n_coarse_groups > 0


def test_coarse_search_step_commits_best(O):
    """a whole step with coarse groups: the committed base is the argmin candidate."""
    g, xs, orders = _setup(seed=12, n=60, D=2)
    coarse_of = (np.arange(g.n) // 12).astype(np.int32)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(3)], np.int64)
    with O.coarse_moves(g, coarse_of, 5, 60):
        keys_all = [O.candidate_keys(g, 3, b, xs, orders, 0, 1024, 4, 0, MIX) for b in range(3)]
        keys = O.search_step(g, rx, ro, rmk, 1024, 4, 0, MIX)
        for b in range(3):
            assert keys[b] == keys_all[b].min()
            ok, x, o = O.candidate(g, 3, b, xs, orders, int(keys[b]) & ((1 << 24) - 1), 4, 0, MIX)
            assert (rx[b] == x).all() and (ro[b] == o).all()
            assert rmk[b] == int(keys[b]) >> 24 == O.makespan(g, x, o)


# ---------------------------------------------------------------------------------------------
# Exact restatement of DESIGN.md §4 S2-S4 (spec v7) in plain Python, written from the text and
# compared element by element with the oracle's decode (oracle_candidate).
# ---------------------------------------------------------------------------------------------
def _py_draw(seed, step, P, b, j, k):
    ctr = (((step * P + b) * (1 << 24) + j) * 16 + k) & ((1 << 64) - 1)
    return mix64(seed ^ mix64(ctr))


def _py_candidate(g, P, b, xs, orders, j, seed, step, mix, edges, preds, succs):
    n, D = g.n, g.D
    bx, bo = xs[b], orders[b]
    x, o = bx.copy(), bo.copy()
    dr = lambda jj, k: _py_draw(seed, step, P, b, jj, k)
    allowed = lambda v: [d for d in range(D)
                         if g.allowed is None or (int(g.allowed[v]) >> d) & 1]
    A = lambda q: [d for d in allowed(int(bo[q])) if d != int(bx[bo[q]])]
    grp, lane = j // 128, j % 128
    R = (n + 63) // 64                                         # S2
    r = (grp + dr(0, 13) % R) % R
    c, ln, ps = 64 * r, min(64, n - 64 * r), grp // R
    swap = False                                               # S3
    if grp != 0 and mix[3] > 0 and n >= 2 and dr(128 * grp, 15) % 100 < mix[3]:
        k = min(c + dr(128 * grp, 14) % ln, n - 2)
        a, cc = int(bo[k]), int(bo[k + 1])
        blocked = ((a, cc) in edges or (cc, a) in edges or (preds[a] & preds[cc]) or
                   (succs[a] & succs[cc]) or len(succs[a]) > 64 or len(succs[cc]) > 64 or
                   bx[a] != bx[cc])
        if not blocked:
            o[k], o[k + 1] = cc, a
            swap = True
    if j == 0 or (swap and lane == 0):                         # S4
        return True, x, o
    W = mix[0] + mix[1] + mix[2]
    if W <= 0:
        return True, x, o
    b1, b2 = (128 * mix[0]) // W, (128 * (mix[0] + mix[1])) // W
    kind = "flip1" if lane < b1 else ("flipk" if lane < b2 else "window")
    if kind == "flip1":
        t = ps * b1 + lane
        if t < ln * (D - 1):
            q = c + t % ln
            aq = A(q)
            if t // ln >= len(aq):
                return False, x, o
            x[bo[q]] = aq[t // ln]
            return True, x, o
        kind = "flipk"
    if kind == "flipk":
        f = min(2 + dr(j, 1) % 3, ln)
        taken = []
        for i in range(f):
            free = [q for q in range(c, c + ln) if q not in taken]
            q = free[dr(j, 2 + 2 * i) % (ln - i)]
            taken.append(q)
            aq = A(q)
            if not aq:
                return False, x, o
            x[bo[q]] = aq[dr(j, 3 + 2 * i) % len(aq)]
        return True, x, o
    i, nw = lane - b2, 128 - b2                                # WINDOW (v7)
    w = ps * nw + i
    s, visit = c + w % ln, w // ln
    aq = A(s)
    if not aq:
        return False, x, o
    d = aq[dr(j, 4) % len(aq)]
    elig = [q for q in range(s, c + ln) if d in allowed(int(bo[q])) and int(bx[bo[q]]) != d]
    if len(elig) < 2 or visit >= len(elig) - 1:
        return False, x, o
    L = 2 + (visit + dr(s, 0)) % (len(elig) - 1)
    for q in elig[:L]:
        x[bo[q]] = d
    return True, x, o


@pytest.mark.parametrize("seed,n,D,allowed_frac,mix,P", [
    (21, 150, 2, 0.0, (50, 20, 20, 10), 3),          # R = 3 regions: passes 0..10 in 4096 ids
    (22, 333, 2, 0.0, (40, 20, 20, 60), 2),          # swap-heavy, clipped last region (13)
    (23, 200, 3, 0.4, (50, 20, 20, 30), 2),          # masks: invalid and used-up flips
    (24, 260, 4, 0.0, (10, 30, 60, 20), 2),          # D = 4, window-heavy
    (25, 90, 4, 0.5, (80, 0, 0, 50), 1),             # FLIP1 only: enumerations run out
    (26, 70, 2, 0.0, (0, 0, 1, 0), 2)])              # WINDOW only
def test_decode_equals_spec_restatement(O, seed, n, D, allowed_frac, mix, P):
    """oracle_candidate (C) = the plain-Python restatement of DESIGN §4 S2-S4, x and order
    element by element, for 4096 ids per base (groups of every pass, swap groups, lane 0)."""
    g = dag.random_dag(seed, n, 1.5, D=D, p_max=2000, max_bytes=50_000, beta0=300,
                       beta1_fs=20_000, allowed_frac=allowed_frac)
    orders = np.stack([dag.random_topo_order(g, 5 + b) for b in range(P)]).astype(np.int32)
    xs = dag.random_placements(g, 9, P)
    edges = set(zip(g.src.tolist(), g.dst.tolist()))
    preds = [set() for _ in range(n)]
    succs = [set() for _ in range(n)]
    for s_, d_ in edges:
        preds[d_].add(s_)
        succs[s_].add(d_)
    for s_ in range(n):                       # S3 counts out-edges (parallel edges included)
        if int((g.src == s_).sum()) > 64:
            succs[s_] = succs[s_] | {-1 - k for k in range(65)}
    counts = {"valid": 0, "invalid": 0, "swapped": 0}
    for step in (0, 3):
        for b in range(P):
            for j in range(4096):
                ok, x, o = O.candidate(g, P, b, xs, orders, j, 77, step, mix)
                pok, px, po = _py_candidate(g, P, b, xs, orders, j, 77, step, mix, edges, preds,
                                            succs)
                assert ok == pok, (step, b, j)
                if ok:
                    assert (x == px).all() and (o == po).all(), (step, b, j)
                counts["valid" if ok else "invalid"] += 1
                counts["swapped"] += int((o != orders[b]).any())
    assert counts["valid"] > 0
    if mix[3]:
        assert counts["swapped"] > 0
    if allowed_frac:
        assert counts["invalid"] > 0
