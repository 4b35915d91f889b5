"""CUDA path (through the C ABI) vs the CPU oracle, element by element, bit-exact (int64 ns).

North star tolerance: "GPU makespans must match the oracle bit-exactly (all times are integer
nanoseconds)" -- every comparison below is exact equality.
"""

import json
import os

import numpy as np
import pytest

from workloads import configs, dag

pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden")
MIX = (50, 20, 20, 10)


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


def test_tiny12_exhaustive(P, O):
    """all 4096 placements x 186 orders = 761,856 schedules, each bit-exact; min = optimum."""
    g = dag.tiny12()
    G = P.Graph.from_arrays(g)
    xs = np.asarray([[(c >> i) & 1 for i in range(12)] for c in range(4096)], np.uint8)
    best = None
    for order in dag.all_linear_extensions(g):
        gpu = _gpu_eval(P, G, g, order, xs)
        ref, _ = O.makespan_batch(g, xs, np.asarray(order, np.int32))
        assert (gpu == ref).all(), order
        best = gpu.min() if best is None else min(best, gpu.min())
    assert best == json.load(open(os.path.join(GOLD, "tiny12_optimum.json")))["optimum"]


CASES = [
    # (seed, n, avg_out, D, extra kwargs)
    (1, 1, 0.0, 2, {}),
    (2, 2, 1.0, 2, {}),
    (3, 37, 1.5, 2, {}),
    (4, 300, 1.6, 2, {"multi_frac": 0.2, "zero_frac": 0.3}),
    (5, 2500, 1.5, 2, {"fan_in_hub": 1500}),                     # fan-in > 1024, many tiles
    (6, 2000, 1.4, 2, {"fan_out_hub": 700}),                     # out-of-line edge records
    (7, 400, 1.5, 3, {"allowed_frac": 0.4}),                      # D=3: invalid codes exist
    (8, 800, 1.5, 4, {"hetero_links": True}),                     # several link classes
    (9, 500, 1.5, 4, {"allowed_frac": 0.5, "hetero_links": True}),
    (10, 300, 1.5, 8, {"hetero_links": True}),
    (11, 3000, 1.7, 2, {"locality": 40}),
    (12, 600, 1.5, 1, {}),
]


@pytest.mark.parametrize("case", CASES, ids=lambda c: f"seed{c[0]}_n{c[1]}_D{c[3]}")
def test_random_dags(P, O, case):
    seed, n, avg, D, kw = case
    g = dag.random_dag(seed, n, avg, D=D, p_max=5000, max_bytes=400_000, beta0=700,
                       beta1_fs=30_000, **kw)
    G = P.Graph.from_arrays(g)
    for s, n_cand in [(0, 1), (1, 33), (2, 517)]:          # ragged candidate counts
        order = dag.random_topo_order(g, 100 + s)
        x = dag.random_placements(g, 200 + s, n_cand)
        if D == 3 or kw.get("allowed_frac"):
            # include infeasible rows: codes >= D or disallowed devices
            rng = np.random.default_rng(s)
            bad = rng.random(n_cand) < 0.1
            x[bad, 0] = (1 << (1 if D <= 2 else (2 if D <= 4 else 3))) - 1
        gpu = _gpu_eval(P, G, g, order, x)
        ref, _ = O.makespan_batch(g, x, order)
        assert (gpu == ref).all(), (s, np.nonzero(gpu != ref)[0][:5], gpu[:3], ref[:3])


def test_saturated_rows_take_the_64bit_path(P, O):
    """makespans above the 32-bit kernel's saturation (4.03 s) are re-evaluated in int64."""
    g = dag.random_dag(51, 60, 1.5, D=2, p_max=250_000_000, zero_frac=0.0, max_bytes=1 << 20,
                       beta0=1000, beta1_fs=40_000)
    g.p[:] = np.maximum(g.p, 170_000_000)                    # every op 170-250 ms: sum p >> 4 s
    G = P.Graph.from_arrays(g)
    order = dag.random_topo_order(g, 1)
    x = dag.random_placements(g, 2, 300)
    x[0] = 0                                                 # single device: sum p (saturated)
    gpu = _gpu_eval(P, G, g, order, x)
    ref, _ = O.makespan_batch(g, x, order)
    assert (gpu == ref).all()
    assert (ref > 0xF0000000).mean() > 0.5


def test_ineligible_durations_use_64bit_path(P, O):
    """a transfer >= 2^28 ns makes the graph ineligible for the 32-bit kernel."""
    g = dag.random_dag(52, 200, 1.5, D=2, p_max=5000, max_bytes=1 << 20, beta0=10,
                       beta1_fs=300_000_000)                 # 1 MB -> 300 ms transfers
    G = P.Graph.from_arrays(g)
    order = dag.random_topo_order(g, 3)
    x = dag.random_placements(g, 4, 100)
    gpu = _gpu_eval(P, G, g, order, x)
    ref, _ = O.makespan_batch(g, x, order)
    assert (gpu == ref).all()


def test_search_with_bases_above_saturation(P, O):
    """bases whose makespan exceeds 4.03 s run on the 64-bit kernel until they drop below."""
    g = dag.random_dag(53, 50, 1.4, D=2, p_max=200_000_000, zero_frac=0.0, max_bytes=1 << 20,
                       beta0=1000, beta1_fs=40_000)
    g.p[:] = np.maximum(g.p, 150_000_000)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=11)
    xs[0] = 0                                                # base 0: sum p > 4.03 s
    mix = (50, 20, 20, 10)
    S = P.Search(G, xs, orders, 512, mix, seed=4)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
    assert rmk[0] > 0xF0000000
    for step in range(4):
        S.step()
        O.search_step(g, rx, ro, rmk, 512, 4, step, mix)
        for b in range(2):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)


@pytest.mark.parametrize("D,mix", [(2, (50, 20, 20, 10)), (4, (30, 10, 10, 50))])
def test_wide_eval32_bases_above_saturation(P, O, D, mix):
    """bases above 4.03 s run on the wide (exact 64-bit) eval32 instance: each step's argmin key
    equals the minimum of the oracle's keys over every candidate, over several steps."""
    g = dag.random_dag(57 + D, 900, 1.5, D=D, p_max=30_000_000, zero_frac=0.0, max_bytes=1 << 22,
                       beta0=20_000, beta1_fs=400_000)
    g.p[:] = np.maximum(g.p, 5_000_000 * D)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=21)
    K = 1024
    S = P.Search(G, xs, orders, K, mix, seed=6)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
    assert (rmk > 0xF0000000).all()
    for step in range(3):
        S.eval()
        got = S.keys()
        keys = O.search_step(g, rx, ro, rmk, K, 6, step, mix)
        assert (got == keys).all(), (step, got, keys)
        S.commit()
        for b in range(2):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)


@pytest.mark.parametrize("name", ["inception_v3_2dev", "nmt4_2dev_commheavy",
                                  "transformer_2dev", "transformer_4dev_8gpu"])
def test_full_size_sampled(P, O, name):
    """full BASELINE-size graphs: 4096 candidates on the GPU, a sample checked one by one."""
    cfg = configs.CONFIGS[name]
    g = configs.graph_for(cfg)
    G = P.Graph.from_arrays(g)
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    seeds = [G.seed_placement(P.PLACE_EXPERT, layer=g.layer),
             G.seed_placement(P.PLACE_TOPO_SPLIT, order=order),
             G.seed_placement(P.PLACE_SINGLE)]
    x = np.concatenate([np.stack(seeds), dag.random_placements(g, 5, 4093)])
    gpu = _gpu_eval(P, G, g, order, x)
    ref, _ = O.makespan_batch(g, x, order, threads=os.cpu_count())
    assert (gpu == ref).all(), np.nonzero(gpu != ref)[0][:5]  # all 4096 rows
    assert gpu[2] == int(g.p.sum())                           # single device = sum p


def _search_graph(seed=21, n=150, D=2, allowed_frac=0.0):
    g = dag.random_dag(seed, n, 1.5, D=D, p_max=3000, max_bytes=200_000, beta0=500,
                       beta1_fs=25_000, allowed_frac=allowed_frac)
    return g


def _bases(g, P_, seed=0):
    orders = np.stack([dag.random_topo_order(g, seed + b) for b in range(P_)]).astype(np.int32)
    xs = dag.random_placements(g, seed + 50, P_)
    return xs, orders


SAT32 = np.uint64(0xF0000000)


def _check_raw(P, raw, ok):
    """the timed kernel's own keys: exact where its 32-bit walk did not saturate; a clamped walk
    (makespan field 0xF0000000) must belong to a candidate whose exact makespan is >= the clamp"""
    sat = (raw != np.uint64(P.KEY_INVALID)) & ((raw >> np.uint64(24)) >= SAT32)
    assert (raw[~sat] == ok[~sat]).all(), np.nonzero((raw != ok) & ~sat)[0][:5]
    assert ((ok[sat] >> np.uint64(24)) >= SAT32).all()
    return int(sat.sum())


@pytest.mark.parametrize("D,allowed_frac", [(2, 0.0), (4, 0.5)])
def test_search_candidate_keys(P, O, D, allowed_frac):
    """per-candidate keys of the timed eval32 instantiation, of its raw output and of the
    independent 64-bit kernel, each equal to the oracle's decode + makespan"""
    g = _search_graph(D=D, allowed_frac=allowed_frac)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 3)
    K = 1500
    S = P.Search(G, xs, orders, K, MIX, seed=99)
    for b in range(3):
        ok = O.candidate_keys(g, 3, b, xs, orders, 0, K, 99, 0, MIX)
        for kern in (P.KEYS_TIMED, P.KEYS_EVAL64):
            gk = S.candidate_keys(b, 0, K, kernel=kern)
            assert (gk == ok).all(), (kern, b, np.nonzero(gk != ok)[0][:5])
        _check_raw(P, S.candidate_keys(b, 0, K, kernel=P.KEYS_TIMED_RAW), ok)
    ok = O.candidate_keys(g, 3, 1, xs, orders, 77, 1013, 99, 0, MIX)
    for kern in (P.KEYS_TIMED, P.KEYS_EVAL64):               # unaligned range
        assert (S.candidate_keys(1, 77, 1013, kernel=kern) == ok).all(), kern


def test_search_steps_match_reference(P, O):
    g = _search_graph(seed=31, n=120)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 4, seed=7)
    K = 2048
    mix = (40, 20, 20, 30)                                   # many swaps: exercise rebuilds
    S = P.Search(G, xs, orders, K, mix, seed=5)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(4)], np.int64)
    for b in range(4):
        assert S.get(b)[0] == rmk[b]
    for step in range(6):
        S.step()
        keys = O.search_step(g, rx, ro, rmk, K, 5, step, mix)
        for b in range(4):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)
        assert S.step_count == step + 1
        del keys


@pytest.mark.parametrize("D", [2, 4])
def test_async_workspaces_double_buffered(P, O, D):
    """pesto_eval_batch_host_async: four batches on two workspaces / two streams in flight at
    once (the e2e pattern of bench.py); every makespan equals the oracle's"""
    import torch
    g = dag.random_dag(321 + D, 900, 1.5, D=D, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000, allowed_frac=0.3)
    G = P.Graph.from_arrays(g)
    order = dag.random_topo_order(g, 5)
    xs = [dag.random_placements(g, 40 + i, 700 + 37 * i) for i in range(4)]
    rows = [torch.from_numpy(P.pack_rows(x, g.D)).pin_memory().numpy() for x in xs]
    outs = [torch.empty(len(x), dtype=torch.int64).pin_memory().numpy() for x in xs]
    wss = [G.workspace(), G.workspace()]
    sts = [torch.cuda.Stream(), torch.cuda.Stream()]
    got = []
    for i in range(4):
        k = i & 1
        if i >= 2:
            sts[k].synchronize()
            got.append(outs[i - 2].copy())
        wss[k].eval_host_async(order, rows[i], outs[i], stream=sts[k])
    for st in sts:
        st.synchronize()
    got += [outs[2].copy(), outs[3].copy()]
    for i in range(4):
        ref, _ = O.makespan_batch(g, xs[i], order)
        assert (got[i] == ref).all(), i


@pytest.mark.parametrize("D", [2, 4])
def test_multiwave_search_steps(P, O, D):
    """search launches of more than one wave (2 x 131,072 candidates = 1,024 eval32 tasks: the
    multi-candidate-per-lane instances): each step's keys equal the oracle's
    reference step, and the per-base minimum of the independent eval64 kernel's keys"""
    g = dag.random_dag(301 + D, 1500, 1.6, D=D, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=29)
    K, mix, seed = 131072, (40, 20, 20, 20), 8
    S = P.Search(G, xs, orders, K, mix, seed=seed)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
    for step in range(3):
        S.eval()
        gkeys = S.keys()
        for b in range(2):
            # every candidate of the step from the timed instantiation (CPL 2 here) vs the oracle
            tk = S.candidate_keys(b, 0, K, kernel=P.KEYS_TIMED)
            ok = O.candidate_keys(g, 2, b, rx, ro, 0, K, seed, step, mix, os.cpu_count())
            assert (tk == ok).all(), (step, b, np.nonzero(tk != ok)[0][:5])
            _check_raw(P, S.candidate_keys(b, 0, K, kernel=P.KEYS_TIMED_RAW), ok)
            assert int(gkeys[b]) == int(tk.min()), (step, b)
            assert int(gkeys[b]) == int(S.candidate_keys(b, 0, K, kernel=P.KEYS_EVAL64).min())
        keys = O.search_step(g, rx, ro, rmk, K, seed, step, mix)
        assert [int(k) for k in gkeys] == [int(k) for k in keys], step
        S.commit()
        for b in range(2):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)


@pytest.mark.parametrize("D,mix,steps", [(2, (0, 0, 0, 100), 24), (2, (30, 10, 10, 50), 12),
                                         (4, (20, 10, 10, 60), 10)])
def test_committed_swaps_patch_layouts(P, O, D, mix, steps):
    """swap-heavy search on a multi-tile graph: committed swaps are patched into the device
    layouts in place or rebuilt; either way every step matches the oracle, and
    afterwards every candidate key of the patched bases matches too (eval64 layouts)."""
    g = dag.random_dag(61 + D, 1400, 1.6, D=D, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=13)
    K = 4096
    S = P.Search(G, xs, orders, K, mix, seed=17)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
    swaps = 0
    for step in range(steps):
        before = ro.copy()
        S.step()
        O.search_step(g, rx, ro, rmk, K, 17, step, mix)
        swaps += int(sum((before[b] != ro[b]).any() for b in range(2)))
        for b in range(2):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)
    in_place, rebuilt = S.swap_stats()
    assert in_place + rebuilt == swaps and swaps > 0
    assert in_place > 0
    for b in range(2):
        gk = S.candidate_keys(b, 0, K)
        ok = O.candidate_keys(g, 2, b, rx, ro, 0, K, 17, steps, mix)
        assert (gk == ok).all(), (b, np.nonzero(gk != ok)[0][:5])


@pytest.mark.parametrize("seed,n,D,kw", [(91, 700, 2, {}), (92, 500, 4, {"hetero_links": True}),
                                          (93, 2500, 2, {"fan_out_hub": 300})])
def test_congestion_free_links_match_oracle(P, O, seed, n, D, kw):
    """row f4(ii): PESTO_LINKS_UNLIMITED vs the oracle's congestion-free simulator (W2 pin)."""
    g = dag.random_dag(seed, n, 1.5, D=D, p_max=5000, max_bytes=400_000, beta0=700,
                       beta1_fs=30_000, **kw)
    G = P.Graph.from_arrays(g)
    G.set_link_model(P.LINKS_UNLIMITED)
    order = dag.random_topo_order(g, seed)
    x = dag.random_placements(g, seed + 1, 300)
    gpu = _gpu_eval(P, G, g, order, x)
    ref = np.asarray([O.makespan_nocongest(g, x[i], order) for i in range(len(x))], np.int64)
    assert (gpu == ref).all(), np.nonzero(gpu != ref)[0][:5]
    fcfs, _ = O.makespan_batch(g, x, order)
    assert (ref <= fcfs).all() and (ref < fcfs).any()        # queues only ever delay
    G.set_link_model(P.LINKS_FCFS)
    assert (_gpu_eval(P, G, g, order, x) == fcfs).all()


def test_congestion_free_search_keys(P, O):
    """the search kernels under PESTO_LINKS_UNLIMITED: every key of a step (eval32 argmin and
    the eval64 per-candidate keys) equals the oracle's decode + congestion-free makespan."""
    g = _search_graph(seed=95, n=160)
    G = P.Graph.from_arrays(g)
    G.set_link_model(P.LINKS_UNLIMITED)
    xs, orders = _bases(g, 2, seed=9)
    K = 700
    S = P.Search(G, xs, orders, K, MIX, seed=12)
    keys = np.empty((2, K), np.uint64)
    for b in range(2):
        for j in range(K):
            ok, x, o = O.candidate(g, 2, b, xs, orders, j, 12, 0, MIX)
            keys[b, j] = ((O.makespan_nocongest(g, x, o) << 24) | j) if ok else (1 << 64) - 1
        assert (S.candidate_keys(b, 0, K) == keys[b]).all(), b
    S.eval()
    assert (S.keys() == keys.min(axis=1)).all()


def test_fake_sharding_equals_single_rank(P, O):
    """W rank ranges evaluated one after another on one GPU, minima reduced on the host."""
    g = _search_graph(seed=41, n=90)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=3)
    K, W = 3000, 3
    single = P.Search(G, xs, orders, K, MIX, seed=8)
    shards = [P.Search(G, xs, orders, K, MIX, seed=8, rank=r, world=W) for r in range(W)]
    for step in range(3):
        single.eval()
        k1 = single.keys()
        per = []
        for s in shards:
            s.eval()
            per.append(s.keys())
        kmin = np.minimum.reduce(per)
        assert (kmin == k1).all()
        single.commit()
        for s in shards:
            s.set_keys(kmin)
            s.commit()
        for b in range(2):
            a, s0 = single.get(b), shards[0].get(b)
            assert a[0] == s0[0] and (a[1] == s0[1]).all() and (a[2] == s0[2]).all()


def test_nccl_allreduce_path_single_rank(P, O):
    """the NCCL comm + allreduce-MIN path (1-rank comm) commits the same bases as no comm."""
    g = _search_graph(seed=71, n=100)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 3, seed=5)
    plain = P.Search(G, xs, orders, 1024, MIX, seed=3)
    nccl = P.Search(G, xs, orders, 1024, MIX, seed=3, rank=0, world=1,
                    nccl_id=P.nccl_unique_id())
    for _ in range(3):
        plain.step()
        nccl.step()
        for b in range(3):
            a, c = plain.get(b), nccl.get(b)
            assert a[0] == c[0] and (a[1] == c[1]).all() and (a[2] == c[2]).all()


def _full_size_ids(K):
    """>= 4,096 candidate ids of one base: the first 2,048 (16 whole 128-id groups, group 0's
    identity included) and 16 whole groups spread over [0, K) (swap groups among them)"""
    spread = np.linspace(16, K // 128 - 1, 16).astype(np.int64)
    return np.unique(np.concatenate([np.arange(2048)] +
                                    [np.arange(128 * g, 128 * g + 128) for g in spread]))


@pytest.mark.parametrize("name", ["inception_v3_2dev", "nmt4_2dev_commheavy",
                                  "transformer_2dev", "transformer_4dev_8gpu"])
def test_search_full_size_parity(P, O, name):
    """every BASELINE config at full size, the bench's four seeds (nmt4 includes bases above the
    32-bit saturation, walked by the wide instance), the full step's K per base: per-candidate
    keys of the timed instantiation over all K ids of each base, the >= 4,096-id sample of each
    base compared element by element with the oracle; the step's argmin equals their minimum"""
    from workloads import seeds
    cfg = configs.CONFIGS[name]
    g = configs.graph_for(cfg)
    G = P.Graph.from_arrays(g)
    xs, orders = seeds.bench_seeds(g, cfg.bases, configs.SEARCH_SEED)
    K = cfg.candidates_per_gpu // cfg.bases
    S = P.Search(G, xs, orders, K, configs.MOVE_MIX, configs.SEARCH_SEED)
    S.eval()
    gkeys = S.keys()
    ids = _full_size_ids(K)
    for b in range(cfg.bases):
        tk = S.candidate_keys(b, 0, K, kernel=P.KEYS_TIMED)
        assert int(gkeys[b]) == int(tk.min()), b
        ok = np.empty(len(ids), np.uint64)
        for lo in range(0, len(ids), 128):                  # whole groups, contiguous ids
            j0 = int(ids[lo])
            ok[lo:lo + 128] = O.candidate_keys(g, cfg.bases, b, xs, orders, j0, j0 + 128,
                                               configs.SEARCH_SEED, 0, configs.MOVE_MIX,
                                               os.cpu_count())
        assert (tk[ids] == ok).all(), (b, ids[np.nonzero(tk[ids] != ok)[0][:5]])
        raw = S.candidate_keys(b, 0, K, kernel=P.KEYS_TIMED_RAW)
        _check_raw(P, raw[ids], ok)


# ---------------------------------------------------------------------------------------------
# Row f3: memory caps (L202) and colocation (L175)
# ---------------------------------------------------------------------------------------------
def _f3_constraints(g, frac=0.58, n_groups=6, size=3, seed=0):
    rng = np.random.default_rng(seed)
    mem = np.zeros(g.n, np.int64)
    np.add.at(mem, g.src, g.nbytes)
    np.add.at(mem, g.dst, g.nbytes)
    cap = np.full(g.D, int(mem.sum() * frac), np.int64)
    coloc = np.full(g.n, -1, np.int32)
    ops = rng.choice(g.n, n_groups * size, replace=False)
    for k in range(n_groups):
        coloc[ops[k * size:(k + 1) * size]] = k
    return mem, cap, coloc


@pytest.mark.parametrize("D", [2, 4])
def test_constraints_explicit_rows(P, O, D):
    """explicit rows under memory caps and colocation: infeasible rows -> INT64_MAX, others
    bit-exact, both equal to the oracle under the same constraints."""
    g = dag.random_dag(101 + D, 900, 1.5, D=D, p_max=5000, max_bytes=400_000, beta0=700,
                       beta1_fs=30_000)
    mem, cap, coloc = _f3_constraints(g, frac=0.55 if D == 2 else 0.3)
    G = P.Graph.from_arrays(g)
    G.set_constraints(cap=cap, coloc=coloc)
    order = dag.random_topo_order(g, 5)
    x = dag.random_placements(g, 6, 700)
    # make a third of the rows colocation-feasible so both outcomes occur
    for i in range(0, len(x), 3):
        for k in range(6):
            x[i, coloc == k] = x[i, np.nonzero(coloc == k)[0][0]]
    gpu = _gpu_eval(P, G, g, order, x)
    with O.constraints(g, cap=cap, coloc=coloc) as c:
        ok = np.asarray([c.ok(r) for r in x])
        ref, _ = O.makespan_batch(g, x, order)
    assert (gpu == ref).all(), np.nonzero(gpu != ref)[0][:5]
    assert ok.any() and (~ok).any()
    assert (gpu[~ok] == (1 << 63) - 1).all()
    G.set_constraints()                                      # cleared: plain makespans
    plain, _ = O.makespan_batch(g, x, order)
    assert (_gpu_eval(P, G, g, order, x) == plain).all()


@pytest.mark.parametrize("D", [2, 4])
def test_constraints_search(P, O, D):
    """search under caps + colocation: every candidate key (eval64) and each step's commits
    (eval32 argmin, K4 footprint update) match the oracle's constrained search."""
    g = dag.random_dag(111 + D, 400, 1.5, D=D, p_max=4000, max_bytes=300_000, beta0=600,
                       beta1_fs=30_000)
    mem, cap, coloc = _f3_constraints(g, frac=0.56 if D == 2 else 0.32, n_groups=5, seed=1)
    xs, orders = _bases(g, 2, seed=21)
    for b in range(2):                                       # feasible bases: groups together,
        for k in range(5):                                   # then balance the footprint
            xs[b, coloc == k] = 0
        xs[b] = np.where(coloc >= 0, 0, np.arange(g.n) % D).astype(np.uint8)
    G = P.Graph.from_arrays(g)
    G.set_constraints(cap=cap, coloc=coloc)
    mix = (40, 20, 20, 20)
    K = 1024
    S = P.Search(G, xs, orders, K, mix, seed=44)
    rx, ro = xs.copy(), orders.copy()
    with O.constraints(g, cap=cap, coloc=coloc) as c:
        assert all(c.ok(rx[b]) for b in range(2))
        rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
        for b in range(2):
            gk = S.candidate_keys(b, 0, K)
            ok = O.candidate_keys(g, 2, b, rx, ro, 0, K, 44, 0, mix)
            assert (gk == ok).all(), (b, np.nonzero(gk != ok)[0][:5])
            assert (ok == (1 << 64) - 1).sum() > 0
        for step in range(5):
            S.step()
            O.search_step(g, rx, ro, rmk, K, 44, step, mix)
            for b in range(2):
                mk, x, o = S.get(b)
                assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (step, b)
                assert c.ok(x)


# ---------------------------------------------------------------------------------------------
# Row f2: coarsening + exhaustive evaluation of the coarse placements
# ---------------------------------------------------------------------------------------------
@pytest.mark.parametrize("n,target,D", [(120, 10, 2), (300, 16, 2), (150, 6, 4)])
def test_exhaustive_coarse_search(P, O, n, target, D):
    """every coarse placement on the GPU (eval32 mode 4) vs the oracle's brute force over the
    same D^n_coarse expanded placements: best makespan and smallest best index, bit-exact."""
    from oracle import coarsen as OC
    g = dag.random_dag(120 + n, n, 1.5, D=D, p_max=4000, max_bytes=200_000, beta0=500,
                       beta1_fs=25_000)
    G = P.Graph.from_arrays(g)
    co, nc = G.coarsen(target)
    assert nc == target
    order = dag.random_topo_order(g, 3)
    mk, idx, x = G.eval_coarse_exhaustive(order, co, nc)
    best, bidx, allmk = OC.exhaustive(O, g, order, co, nc)
    assert (mk, idx) == (best, bidx)
    assert (x == OC.expand(co, D, idx)).all()


def test_exhaustive_coarse_search_inception(P, O):
    """PAPER.md §3.3 on the inception-shaped graph: coarsened to 20 vertices, all 2^20 coarse
    placements evaluated on the GPU; the winner's makespan is re-checked by the oracle and no
    sampled coarse placement beats it."""
    from oracle import coarsen as OC
    g = configs.graph_for(configs.CONFIGS["inception_v3_2dev"])
    G = P.Graph.from_arrays(g)
    co, nc = G.coarsen(20)
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    mk, idx, x = G.eval_coarse_exhaustive(order, co, nc)
    assert O.makespan(g, x, order) == mk
    rng = np.random.default_rng(0)
    sample = rng.choice(1 << nc, 24, replace=False)
    xs = np.stack([OC.expand(co, 2, int(c)) for c in sample])
    ref, _ = O.makespan_batch(g, xs, order)
    assert (ref >= mk).all()


def test_roofs_microbenchmarks(P):
    """pesto_measure_roofs: positive, physically plausible ceilings on a B200"""
    r = P.measure_roofs(0, 2)
    assert 1e12 < r["int_ops_per_s"] < 1e14
    assert abs(r["int_ops_per_s"] - 3 * r["int_chain_steps_per_s"]) < 1e-6 * r["int_ops_per_s"]
    assert 1e3 < r["l2_read_gbs"] < 1e5 and 1e3 < r["l2_rmw_gbs"] < 1e5
    assert 1e3 < r["hbm_copy_gbs"] < 1e4
    assert r["l2_buffer_bytes"] > 0


@pytest.mark.parametrize("D,allowed_frac,mix", [(2, 0.0, (50, 20, 20, 10)),
                                                 (3, 0.4, (40, 20, 20, 40))])
def test_move_stats_count_distinct_candidates(P, O, D, allowed_frac, mix):
    """pesto_search_move_stats (host decode by the product's spec code) counts the same
    invalid / identical-to-base / distinct (placement, order) candidates as the oracle's decode,
    over several passes of the region tiling (n = 300: 5 regions, K = 2048: 16 groups)"""
    g = dag.random_dag(140 + D, 300, 1.5, D=D, p_max=3000, max_bytes=100_000, beta0=500,
                       beta1_fs=25_000, allowed_frac=allowed_frac)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=3)
    K = 2048
    S = P.Search(G, xs, orders, K, mix, seed=31)
    for step in range(2):
        for b in range(2):
            st = S.move_stats(b)
            seen, inval, ident = set(), 0, 0
            cur_x, cur_o = _cur(S)
            for j in range(K):
                ok, x, o = O.candidate(g, 2, b, cur_x, cur_o, j, 31, step, mix)
                if not ok:
                    inval += 1
                    continue
                ident += int((x == cur_x[b]).all() and (o == cur_o[b]).all())
                seen.add((x.tobytes(), o.tobytes()))
            assert st == {"candidates": K, "invalid": inval, "identical_to_base": ident,
                          "distinct": len(seen)}, (step, b, st)
        S.step()


def _cur(S):
    xs, os_ = [], []
    for b in range(S.P):
        _, x, o = S.get(b)
        xs.append(x)
        os_.append(o)
    return np.stack(xs), np.stack(os_)


def test_checkpoint_resume_continues_exactly(P, O, tmp_path):
    """SURVEY §5 checkpoint/resume: a search saved after 3 steps (incumbents, step counter, K,
    mix, seed) and resumed in a fresh search object takes exactly the steps the uninterrupted
    search takes (every draw is a function of (seed, step, base, j)), swaps included; both equal
    the oracle's reference steps."""
    g = dag.random_dag(401, 900, 1.6, D=2, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    G = P.Graph.from_arrays(g)
    xs, orders = _bases(g, 2, seed=41)
    K, mix, seed = 4096, (40, 20, 20, 30), 12
    A = P.Search(G, xs, orders, K, mix, seed=seed)
    for _ in range(3):
        A.step()
    ck = A.checkpoint()
    np.savez(tmp_path / "ck.npz", **ck)
    for _ in range(3):
        A.step()
    B = P.Search.resume(G, dict(np.load(tmp_path / "ck.npz")))
    assert B.step_count == 3
    for _ in range(3):
        B.step()
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
    for step in range(6):
        O.search_step(g, rx, ro, rmk, K, seed, step, mix)
    for b in range(2):
        ma, xa, oa = A.get(b)
        mb, xb, ob = B.get(b)
        assert ma == mb == rmk[b] and (xa == xb).all() and (oa == ob).all()
        assert (xa == rx[b]).all() and (oa == ro[b]).all()
