"""libpesto.so without a GPU: it loads, exports every symbol include/pesto.h declares, and its
host-only paths (validation, comm guard, layouts, seeds) behave as the header states."""

import os
import re
import subprocess

import numpy as np
import pytest

from workloads import configs, dag

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def P():
    from paper_conf_middleware_hafeezsg021_b200 import build
    build.build()
    from paper_conf_middleware_hafeezsg021_b200 import pesto
    return pesto


def test_exports_every_declared_symbol(P):
    hdr = open(os.path.join(ROOT, "include", "pesto.h")).read()
    declared = set(re.findall(r"\b(pesto_[a-z0-9_]+)\s*\(", hdr))
    assert len(declared) >= 20
    out = subprocess.run(["nm", "-D", "--defined-only", P.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (pesto_[a-z0-9_]+)", out))
    assert declared <= exported, declared - exported
    assert declared == set(P.SIGNATURES)            # the binding covers the whole ABI
    assert P.lib().pesto_version() == 100


def _host_graph(P, g):
    return P.Graph.from_arrays(g, device=-1)


def test_validation_errors(P):
    with pytest.raises(P.PestoError) as e:
        P.Graph([1, 1, 1], [0, 1, 2], [1, 2, 0], [1, 1, 1], 2, device=-1)
    assert e.value.status == P.ECYCLE
    with pytest.raises(P.PestoError) as e:
        P.Graph([1, 1], [0], [0], [1], 2, device=-1)
    assert e.value.status == P.EINVAL
    with pytest.raises(P.PestoError) as e:
        P.Graph([1, -1], [], [], [], 2, device=-1)
    assert e.value.status == P.EINVAL
    with pytest.raises(P.PestoError) as e:
        P.Graph([1, 1], [0], [5], [1], 2, device=-1)
    assert e.value.status == P.EINVAL
    with pytest.raises(P.PestoError) as e:
        P.Graph([1, 1], [0], [1], [1], 9, device=-1)
    assert e.value.status == P.EINVAL
    with pytest.raises(P.PestoError) as e:
        P.Graph([1, 1], [0], [1], [1], 2, allowed=[1, 4], device=-1)   # op 1 allows nothing
    assert e.value.status == P.EINVAL
    with pytest.raises(P.PestoError) as e:
        P.Graph([1 << 39, 1 << 39], [], [], [], 2, device=-1)
    assert e.value.status == P.EOVERFLOW


def test_comm_model_guard_and_state(P):
    G = P.Graph([10, 10], [0], [1], [1 << 40], 2, device=-1)
    with pytest.raises(P.PestoError) as e:
        G.stats([0, 1])                                       # comm model unset
    assert e.value.status == P.ESTATE
    with pytest.raises(P.PestoError) as e:
        G.comm_model(-1, -1, 0, 1_000_000)                     # 2^40 ns transfer
    assert e.value.status == P.EOVERFLOW
    with pytest.raises(P.PestoError) as e:
        G.comm_model(0, 0, 1, 1)
    assert e.value.status == P.EINVAL
    with pytest.raises(P.PestoError) as e:
        G.comm_model(0, 1, -1, 1)
    assert e.value.status == P.EINVAL
    G.comm_model(0, 1, 5, 1)
    with pytest.raises(P.PestoError):
        G.stats([0, 1])                                        # 1 -> 0 still unset
    G.comm_model(1, 0, 5, 1)
    st = G.stats([0, 1])
    assert st["live_slots"] == 1 and st["link_classes"] == 1
    with pytest.raises(P.PestoError) as e:
        G.stats([1, 0])
    assert e.value.status == P.ENOTTOPO
    rc = P.lib().pesto_eval_batch(G.handle, np.asarray([0, 1], np.int32).ctypes.data, None, 16, 1,
                                  None, None)
    assert rc == P.ESTATE


def _is_topological(g, order):
    pos = np.empty(g.n, np.int64)
    pos[np.asarray(order)] = np.arange(g.n)
    return sorted(order) == list(range(g.n)) and bool((pos[g.src] < pos[g.dst]).all())


def test_seed_orders(P):
    g = configs.graph_for(configs.CONFIGS["inception_v3_2dev"])
    G = _host_graph(P, g)
    for kind in (P.ORDER_CRITICAL_PATH, P.ORDER_FIFO, P.ORDER_RANDOM):
        o = G.seed_order(kind, 5)
        assert _is_topological(g, o.tolist())
    assert (G.seed_order(P.ORDER_RANDOM, 5) == G.seed_order(P.ORDER_RANDOM, 5)).all()
    assert (G.seed_order(P.ORDER_RANDOM, 5) != G.seed_order(P.ORDER_RANDOM, 6)).any()
    # critical-path order: whenever two ops are both ready, the larger bottom level goes first;
    # in particular the first op is a source with maximal bottom level
    small = dag.random_dag(3, 60, 1.5, D=2, beta0=1, beta1_fs=1)
    Gs = _host_graph(P, small)
    o = Gs.seed_order(P.ORDER_CRITICAL_PATH)
    succ = small.succs()
    bl = np.zeros(small.n, np.int64)
    for v in reversed(dag.random_topo_order(small, 0).tolist()):
        bl[v] = small.p[v] + max([bl[int(small.dst[e])] for e in succ[v]], default=0)
    sources = [v for v in range(small.n) if not any(int(d) == v for d in small.dst)]
    assert bl[o[0]] == max(bl[s] for s in sources)


def test_seed_placements(P):
    g = configs.graph_for(configs.CONFIGS["transformer_4dev_8gpu"])
    G = _host_graph(P, g)
    o = G.seed_order(P.ORDER_CRITICAL_PATH)
    x = G.seed_placement(P.PLACE_TOPO_SPLIT, order=o)
    assert (np.diff(x[o].astype(int)) >= 0).all()             # contiguous segments along pi
    loads = [int(g.p[x == d].sum()) for d in range(4)]
    assert max(loads) - min(loads) <= 2 * int(g.p.max())      # about equal sum p
    xe = G.seed_placement(P.PLACE_EXPERT, layer=g.layer)
    nl = int(g.layer.max()) + 1
    assert (xe == (g.layer * 4 // nl)).all()
    assert (G.seed_placement(P.PLACE_SINGLE) == 0).all()
    xr = G.seed_placement(P.PLACE_RANDOM, seed=1)
    assert set(np.unique(xr)) == {0, 1, 2, 3}
    aff = dag.random_dag(4, 50, 1.2, D=4, allowed_frac=0.7, beta0=1, beta1_fs=1)
    Ga = _host_graph(P, aff)
    for kind in (P.PLACE_SINGLE, P.PLACE_RANDOM):
        xa = Ga.seed_placement(kind, seed=3)
        assert all((int(aff.allowed[v]) >> int(xa[v])) & 1 for v in range(aff.n))


def test_pack_rows_matches_generator_packing(P):
    for D in (2, 3, 4, 8):
        g = dag.random_dag(D, 77, 1.0, D=D)
        x = dag.random_placements(g, 1, 9)
        assert (P.pack_rows(x, D) == dag.pack_placements(x, D)).all()


def test_layout_live_slots_bounds(P):
    g = configs.graph_for(configs.CONFIGS["transformer_2dev"])
    G = _host_graph(P, g)
    for kind in (P.ORDER_CRITICAL_PATH, P.ORDER_FIFO):
        st = G.stats(G.seed_order(kind))
        assert 1 <= st["live_slots"] <= g.n
        assert st["n_tiles"] >= 1 and st["layout_bytes"] >= 16 * (g.n + g.m)
        assert st["max_in_degree"] == int(np.bincount(g.dst).max())


def test_coarsen_matches_oracle(P):
    """row f2 host code (§3.3 coarsening) equals the oracle's plain-Python coarsening
    exactly, on random DAGs and on a shaped training-step graph."""
    from oracle import coarsen as OC
    cases = [dag.random_dag(800 + s, 50 + 23 * s, 1.5, D=2, max_bytes=50_000) for s in range(12)]
    cases.append(dag.random_dag(900, 400, 1.6, D=2, max_bytes=50_000, fan_out_hub=60))
    for g in cases:
        G = _host_graph(P, g)
        for target in (1, 5, 20, 64):
            co, nc = G.coarsen(target)
            ro, rn = OC.coarsen(g.n, g.src, g.dst, g.nbytes, target)
            assert nc == rn and (co == ro).all(), (g.n, target)
    # the shaped inception graph through its first, largest batches (the plain-Python oracle
    # takes minutes to go all the way down; the random DAGs above reach the small targets)
    g = configs.graph_for(configs.CONFIGS["inception_v3_2dev"])
    co, nc = _host_graph(P, g).coarsen(8000)
    ro, rn = OC.coarsen(g.n, g.src, g.dst, g.nbytes, 8000)
    assert nc == rn == 8000 and (co == ro).all()
    with pytest.raises(P.PestoError):
        _host_graph(P, g).coarsen(0)


def test_dispatch_and_link_model_validation(P):
    """pesto_graph_set_dispatch / set_link_model accept their enums only (pesto.h)."""
    g = dag.random_dag(5, 30, 1.5, D=2, beta0=10, beta1_fs=100)
    G = _host_graph(P, g)
    G.set_dispatch(P.DISPATCH_NONDELAY)
    G.set_dispatch(P.DISPATCH_FIXED)
    with pytest.raises(P.PestoError):
        G.set_dispatch(2)
    with pytest.raises(P.PestoError):
        G.set_link_model(5)


def test_workspace_and_async_validation(P):
    """pesto.h: a workspace needs a device graph (ESTATE on a host-only handle); NULL -> EINVAL;
    the async call validates like pesto_eval_batch_host before touching a GPU."""
    import ctypes as C
    g = dag.random_dag(3, 20, 1.5, D=2)
    G = _host_graph(P, g)
    h = C.c_void_p()
    assert P.lib().pesto_workspace_create(G.handle, C.byref(h)) == P.ESTATE
    assert not h.value
    assert P.lib().pesto_workspace_create(None, C.byref(h)) == P.EINVAL
    assert P.lib().pesto_eval_batch_host_async(None, None, None, 16, 1, None, None) == P.EINVAL
    P.lib().pesto_workspace_destroy(None)                      # NULL-safe


@pytest.mark.parametrize("name", ["inception_v3_2dev", "nmt4_2dev_commheavy",
                                  "transformer_4dev_8gpu", "random_masked"])
def test_python_seeds_equal_library_seeds(P, name):
    """workloads/seeds.py (the CPU reference arm's incumbents) restates libpesto's row-a1 seed
    generators: every order and placement agrees op for op."""
    from workloads import seeds
    if name == "random_masked":
        g = dag.random_dag(77, 500, 1.5, D=3, p_max=3000, max_bytes=10_000, beta0=100,
                           beta1_fs=1000, allowed_frac=0.4)
        g.layer = (np.arange(g.n) * 7) // g.n
    else:
        g = configs.graph_for(configs.CONFIGS[name])
    G = _host_graph(P, g)
    o_cp = G.seed_order(P.ORDER_CRITICAL_PATH)
    assert (o_cp == seeds.order_critical_path(g)).all()
    assert (G.seed_order(P.ORDER_FIFO) == seeds.order_fifo(g)).all()
    assert (G.seed_order(P.ORDER_RANDOM, 2021) == seeds.order_random(g, 2021)).all()
    assert (G.seed_placement(P.PLACE_SINGLE) == seeds.place_single(g)).all()
    assert (G.seed_placement(P.PLACE_EXPERT, layer=g.layer) == seeds.place_expert(g, g.layer)).all()
    assert (G.seed_placement(P.PLACE_TOPO_SPLIT, order=o_cp) ==
            seeds.place_topo_split(g, o_cp)).all()
    assert (G.seed_placement(P.PLACE_RANDOM, seed=2021) == seeds.place_random(g, 2021)).all()
