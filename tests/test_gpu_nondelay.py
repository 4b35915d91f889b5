"""Row f4(i): the non-delay dispatch kernel through the C ABI vs the oracle's
non-delay event simulator (`oracle_makespan_model(..., nondelay=1)`, pinned in
tests/test_oracle_nondelay.py), element by element, bit-exact (int64 ns)."""

import json
import os

import numpy as np
import pytest

from workloads import configs, dag

pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden")
MIX = (50, 20, 20, 10)
KEY_INVALID = (1 << 64) - 1
INF = (1 << 63) - 1


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_middleware_hafeezsg021_b200 import pesto
    return pesto


def _gpu_eval(P, G, g, order, x):
    import torch
    rows = torch.from_numpy(dag.pack_placements(x, g.D)).cuda()
    out = G.eval(order, rows)
    torch.cuda.synchronize()
    return out.cpu().numpy()


def _ref(O, g, x, order, congestion=True):
    return np.asarray([O.makespan_model(g, x[i], order, congestion=congestion, nondelay=True)
                       for i in range(len(x))], np.int64)


def test_worked_examples(P, O):
    data = json.load(open(os.path.join(GOLD, "worked_examples.json")))
    for ex in data["examples"]:
        g = dag.make_graph(ex["name"], ex["p"], [tuple(e) for e in ex["edges"]],
                           [1] * len(ex["edges"]), D=2, beta0=ex["t"], beta1_fs=0)
        G = P.Graph.from_arrays(g)
        G.set_dispatch(P.DISPATCH_NONDELAY)
        for case in ex["cases"]:
            x = np.asarray([case["x"]], np.uint8)
            if min(ex["p"]) == 0:                           # outside the variant's domain (R24)
                with pytest.raises(P.PestoError):
                    _gpu_eval(P, G, g, case["order"], x)
                continue
            assert _gpu_eval(P, G, g, case["order"], x)[0] == case["nondelay"], (ex["name"], case)


CASES = [
    # (seed, n, avg_out, D, kwargs)
    (1, 1, 0.0, 2, {}),
    (2, 2, 1.0, 2, {}),
    (3, 40, 1.5, 2, {}),
    (4, 300, 1.6, 2, {"multi_frac": 0.2}),
    (5, 1200, 1.5, 2, {"fan_in_hub": 1500}),                # fan-in > 1024
    (6, 1500, 1.4, 2, {"fan_out_hub": 700}),                # out-degree >> 32 lanes
    (7, 400, 1.5, 3, {"allowed_frac": 0.4}),                # D = 3: codes 3 are infeasible
    (8, 500, 1.5, 4, {"hetero_links": True}),               # several link classes
    (9, 300, 2.0, 8, {"allowed_frac": 0.3}),                # D = 8: 64 links, 4 planes
    (10, 2100, 1.5, 2, {"locality": 8}),                    # n > 2048: several bitmap words
]


@pytest.mark.parametrize("case", CASES, ids=lambda c: f"s{c[0]}n{c[1]}D{c[3]}")
def test_random_dags(P, O, case):
    seed, n, avg, D, kw = case
    g = dag.random_dag(seed, n, avg, D=D, zero_frac=0.0, p_max=5000, max_bytes=300_000,
                       beta0=900, beta1_fs=35_000, **kw)
    G = P.Graph.from_arrays(g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    for k in range(2):
        order = dag.random_topo_order(g, seed + k)
        x = dag.random_placements(g, seed + 10 * k, 70)
        if D == 3:
            x[5, 0] = 3                                     # an infeasible code
        gpu = _gpu_eval(P, G, g, order, x)
        ref = _ref(O, g, x, order)
        assert (gpu == ref).all(), (k, np.nonzero(gpu != ref)[0][:5], gpu[:4], ref[:4])
        if D == 3:
            assert gpu[5] == INF


def test_congestion_free_and_fixed_still_exact(P, O):
    """non-delay x congestion-free links; switching back restores the fixed-sequence kernels."""
    g = dag.random_dag(44, 800, 1.6, D=2, zero_frac=0.0, p_max=4000, max_bytes=300_000,
                       beta0=700, beta1_fs=40_000)
    G = P.Graph.from_arrays(g)
    order = dag.random_topo_order(g, 4)
    x = dag.random_placements(g, 4, 64)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    G.set_link_model(P.LINKS_UNLIMITED)
    assert (_gpu_eval(P, G, g, order, x) == _ref(O, g, x, order, congestion=False)).all()
    G.set_link_model(P.LINKS_FCFS)
    nd = _gpu_eval(P, G, g, order, x)
    assert (nd == _ref(O, g, x, order)).all()
    G.set_dispatch(P.DISPATCH_FIXED)
    fixed = _gpu_eval(P, G, g, order, x)
    assert (fixed == O.makespan_batch(g, x, order)[0]).all()
    assert (nd != fixed).any()                              # the variant changes schedules


def test_zero_durations_rejected(P, O):
    g = dag.random_dag(3, 50, 1.5, D=2, zero_frac=0.3, p_max=100, beta0=5, beta1_fs=0)
    G = P.Graph.from_arrays(g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    with pytest.raises(P.PestoError):
        _gpu_eval(P, G, g, dag.random_topo_order(g, 0), dag.random_placements(g, 0, 2))


def _nd_search_step(O, g, rx, ro, rmk, K, seed, step, mix):
    """reference step under non-delay dispatch: DESIGN.md §4 S1-S8 with the variant's keys."""
    Pn = rx.shape[0]
    for b in range(Pn):
        keys = O.candidate_keys_model(g, Pn, b, rx, ro, 0, K, seed, step, mix, nondelay=True)
        k = int(keys.min())
        if k == KEY_INVALID:
            continue
        j = k & ((1 << 24) - 1)
        if j:
            ok, x, o = O.candidate(g, Pn, b, rx, ro, j, seed, step, mix)
            assert ok
            rx[b], ro[b] = x, o
        rmk[b] = k >> 24


@pytest.mark.parametrize("D,allowed_frac", [(2, 0.0), (4, 0.5)])
def test_search_candidate_keys(P, O, D, allowed_frac):
    g = dag.random_dag(21, 150, 1.5, D=D, zero_frac=0.0, p_max=3000, max_bytes=200_000,
                       beta0=500, beta1_fs=25_000, allowed_frac=allowed_frac)
    G = P.Graph.from_arrays(g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    orders = np.stack([dag.random_topo_order(g, b) for b in range(3)]).astype(np.int32)
    xs = dag.random_placements(g, 50, 3)
    K = 1200
    S = P.Search(G, xs, orders, K, (40, 20, 20, 30), seed=99)
    for b in range(3):
        gk = S.candidate_keys(b, 0, K)
        ok = O.candidate_keys_model(g, 3, b, xs, orders, 0, K, 99, 0, (40, 20, 20, 30),
                                    nondelay=True)
        assert (gk == ok).all(), (b, np.nonzero(gk != ok)[0][:5])


def test_search_steps_match_reference(P, O):
    """whole steps (argmin, commit, committed swaps patched in place) under non-delay dispatch."""
    g = dag.random_dag(31, 700, 1.5, D=2, zero_frac=0.0, p_max=3000, max_bytes=200_000,
                       beta0=500, beta1_fs=25_000)
    G = P.Graph.from_arrays(g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    orders = np.stack([dag.random_topo_order(g, 7 + b) for b in range(2)]).astype(np.int32)
    xs = dag.random_placements(g, 57, 2)
    K, mix = 1024, (30, 10, 10, 50)
    S = P.Search(G, xs, orders, K, mix, seed=5)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan_model(g, rx[b], ro[b], nondelay=True) for b in range(2)],
                     np.int64)
    for b in range(2):
        assert S.get(b)[0] == rmk[b]
    for step in range(5):
        S.step()
        _nd_search_step(O, g, rx, ro, rmk, K, 5, step, mix)
        for b in range(2):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)


@pytest.mark.parametrize("name", ["inception_v3_2dev", "transformer_4dev_8gpu"])
def test_full_size_sampled(P, O, name):
    """BASELINE-size shaped graphs: 1024 rows on the GPU, a sample checked one by one."""
    cfg = configs.CONFIGS[name]
    g = configs.graph_for(cfg)
    G = P.Graph.from_arrays(g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    seeds = [G.seed_placement(P.PLACE_EXPERT, layer=g.layer),
             G.seed_placement(P.PLACE_TOPO_SPLIT, order=order),
             G.seed_placement(P.PLACE_SINGLE)]
    x = np.concatenate([np.stack(seeds), dag.random_placements(g, 5, 1021)])
    gpu = _gpu_eval(P, G, g, order, x)
    idx = [0, 1, 2, 3, 500, 1023]
    ref = _ref(O, g, x[idx], order)
    assert (gpu[idx] == ref).all(), (gpu[idx], ref)
    assert gpu[2] == int(g.p.sum())                           # one device: never idle
