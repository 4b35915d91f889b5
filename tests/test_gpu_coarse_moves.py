"""Search spec S9 on the GPU (row f2 group moves over merged vertices, DESIGN.md §4 S9): every
candidate key, whole steps (eval32 fast path + K4 commit of a vertex move) and committed swaps
that must carry the per-position merged-vertex arrays along -- all bit-exact against the oracle's
decode (`oracle_candidate` under `oracle.coarse_moves`), which `test_oracle_search.py` pins to
the spec text.  PAPER.md L269: every op of a merged vertex takes the vertex's device."""

import numpy as np
import pytest

from workloads import configs, dag

pytestmark = pytest.mark.gpu

KEY_INVALID = (1 << 64) - 1


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_middleware_hafeezsg021_b200 import pesto
    return pesto


def _bases(g, n_bases, seed):
    orders = np.stack([dag.random_topo_order(g, seed + b) for b in range(n_bases)]).astype(np.int32)
    return dag.random_placements(g, seed + 50, n_bases), orders


def _coarse_groups(O, seed, step, n_bases, b, K, pct):
    return [grp for grp in range(1, (K + 127) // 128)
            if O.draw(seed, step, n_bases, b, 128 * grp, 12) % 100 < pct]


@pytest.mark.parametrize("D,allowed_frac,kind", [(2, 0.0, "coarsen"), (4, 0.5, "coarsen"),
                                                 (3, 0.3, "interleaved")])
def test_coarse_candidate_keys(P, O, D, allowed_frac, kind):
    """every key of K candidates per base (eval64) equals the oracle's, coarse groups included"""
    g = dag.random_dag(201 + D, 300, 1.5, D=D, p_max=3000, max_bytes=200_000, beta0=500,
                       beta1_fs=25_000, allowed_frac=allowed_frac)
    G = P.Graph.from_arrays(g)
    if kind == "coarsen":
        co, nc = G.coarsen(12)
    else:                                    # vertices spread over the whole order
        nc = 7
        co = (np.arange(g.n) * 5 % nc).astype(np.int32)
    xs, orders = _bases(g, 3, seed=4)
    K, mix, pct, seed = 1536, (40, 20, 20, 20), 50, 61
    S = P.Search(G, xs, orders, K, mix, seed=seed)
    S.set_coarse_moves(co, nc, pct)
    with O.coarse_moves(g, co, nc, pct):
        for b in range(3):
            assert _coarse_groups(O, seed, 0, 3, b, K, pct)
            gk = S.candidate_keys(b, 0, K)
            ok = O.candidate_keys(g, 3, b, xs, orders, 0, K, seed, 0, mix)
            assert (gk == ok).all(), (b, np.nonzero(gk != ok)[0][:5])
        gk = S.candidate_keys(2, 201, 1111)                  # unaligned range
        ok = O.candidate_keys(g, 3, 2, xs, orders, 201, 1111, seed, 0, mix)
        assert (gk == ok).all()


@pytest.mark.parametrize("D,mix,pct,need_win", [(2, (40, 10, 10, 40), 40, True),
                                                (4, (30, 10, 10, 50), 30, False),
                                                (2, (0, 0, 0, 0), 100, True)])
def test_coarse_search_steps(P, O, D, mix, pct, need_win):
    """whole steps on a multi-tile graph (eval32 argmin, K4 vertex commit, swaps patched in place
    with the merged-vertex positions) match the oracle's steps; afterwards every candidate key of
    the evolved bases matches too"""
    g = dag.random_dag(231 + D, 1400, 1.6, D=D, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    G = P.Graph.from_arrays(g)
    co, nc = G.coarsen(40)
    xs, orders = _bases(g, 2, seed=19)
    K, seed, steps = 4096, 23, 10
    S = P.Search(G, xs, orders, K, mix, seed=seed)
    S.set_coarse_moves(co, nc, pct)
    rx, ro = xs.copy(), orders.copy()
    coarse_wins = 0
    with O.coarse_moves(g, co, nc, pct):
        rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
        for step in range(steps):
            keys = O.search_step(g, rx, ro, rmk, K, seed, step, mix)
            S.step()
            for b in range(2):
                j = int(keys[b]) & ((1 << 24) - 1)
                grp = j >> 7
                coarse_wins += int(j != 0 and grp in _coarse_groups(O, seed, step, 2, b, K, pct))
                mk, x, o = S.get(b)
                assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)
        for b in range(2):
            gk = S.candidate_keys(b, 0, K)
            ok = O.candidate_keys(g, 2, b, rx, ro, 0, K, seed, steps, mix)
            assert (gk == ok).all(), (b, np.nonzero(gk != ok)[0][:5])
    assert coarse_wins > 0 or not need_win              # a vertex move was committed
    if mix[3]:
        assert sum(S.swap_stats()) > 0


def test_coarse_moves_nondelay(P, O):
    """S9 under non-delay dispatch (row f4(i) kernel): candidate keys and one committed step"""
    g = dag.random_dag(241, 400, 1.5, D=2, zero_frac=0.0, p_max=3000, max_bytes=200_000,
                       beta0=500, beta1_fs=25_000)
    G = P.Graph.from_arrays(g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    co, nc = G.coarsen(10)
    xs, orders = _bases(g, 2, seed=8)
    K, mix, pct, seed = 768, (40, 20, 20, 20), 60, 5
    S = P.Search(G, xs, orders, K, mix, seed=seed)
    S.set_coarse_moves(co, nc, pct)
    with O.coarse_moves(g, co, nc, pct):
        rows = []
        for b in range(2):
            gk = S.candidate_keys(b, 0, K)
            ok = O.candidate_keys_model(g, 2, b, xs, orders, 0, K, seed, 0, mix, nondelay=True)
            assert (gk == ok).all(), (b, np.nonzero(gk != ok)[0][:5])
            rows.append(ok)
        S.step()
        for b in range(2):
            k = int(rows[b].min())
            j = k & ((1 << 24) - 1)
            ok_, x, o = O.candidate(g, 2, b, xs, orders, j, seed, 0, mix)
            mk, gx, go = S.get(b)
            assert mk == k >> 24 and (gx == x).all() and (go == o).all()


def test_coarse_moves_argument_checks(P, O):
    g = dag.random_dag(251, 60, 1.5, D=2)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 1, seed=1)
    S = P.Search(G, xs, orders, 256, (50, 20, 20, 10), seed=1)
    co = np.zeros(g.n, np.int32)
    for bad in [(co, 0, 10), (co, 256, 10), (co, 1, 101), (co + 3, 3, 10), (co - 1, 1, 10)]:
        with pytest.raises(Exception):
            S.set_coarse_moves(*bad)
    S.set_coarse_moves(co, 1, 0)                             # off: accepted, nothing changes
    G.set_constraints(cap=np.full(2, 1 << 40, np.int64))    # row f3 cannot be combined
    with pytest.raises(Exception):
        S.set_coarse_moves(co, 1, 50)


def test_coarse_moves_full_size_sampled(P, O):
    """inception-shaped graph coarsened to ~200 vertices (the paper's size, L267): one fast step
    of 4 x 16,384 candidates; each winner is re-decoded and re-scored by the oracle, and sampled
    coarse-group candidates' keys (eval64) equal the oracle's"""
    g = configs.graph_for(configs.CONFIGS["inception_v3_2dev"])
    G = P.Graph.from_arrays(g)
    co, nc = G.coarsen(200)
    assert nc <= 255
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    xs = np.stack([G.seed_placement(P.PLACE_TOPO_SPLIT, order=order),
                   G.seed_placement(P.PLACE_RANDOM, seed=3)])
    orders = np.stack([order, order])
    K, mix, pct, seed = 16384, (50, 20, 20, 10), 30, 7
    S = P.Search(G, xs, orders, K, mix, seed=seed)
    S.set_coarse_moves(co, nc, pct)
    S.eval()
    keys = S.keys()
    with O.coarse_moves(g, co, nc, pct):
        for b in range(2):
            j = int(keys[b]) & ((1 << 24) - 1)
            ok, x, o = O.candidate(g, 2, b, xs, orders, j, seed, 0, mix)
            assert ok and O.makespan(g, x, o) == int(keys[b]) >> 24
            grp = _coarse_groups(O, seed, 0, 2, b, K, pct)[:3]
            js = [128 * gg + l for gg in grp for l in (0, 77)]
            for jj in js:
                gk = S.candidate_keys(b, jj, jj + 1)
                ok_ = O.candidate_keys(g, 2, b, xs, orders, jj, jj + 1, seed, 0, mix)
                assert (gk == ok_).all(), (b, jj)
