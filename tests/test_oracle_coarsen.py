"""Row f2 oracle: PAPER.md §3.3 coarsening (Def 3.4, Thm 3.5) and the exhaustive coarse
search, pinned by hand examples, Figure 6, and properties of every result."""

import itertools

import numpy as np

from oracle import coarsen as C
from workloads import dag


def _coarse_edges(g, coarse_of):
    return {(int(coarse_of[a]), int(coarse_of[b])) for a, b in zip(g.src, g.dst)
            if coarse_of[a] != coarse_of[b]}


def test_heights_definition_3_4():
    # a->b->c, a->c, d isolated: H = 1, 2, 3, 1 (longest root path in vertices)
    assert C.heights(4, [(0, 1), (1, 2), (0, 2)]) == [1, 2, 3, 1]
    assert C.heights(2, [(0, 1), (1, 0)]) is None                 # cycle


def test_figure6_double_merge_is_refused():
    """Figure 6 (L236-240): A->C and B->D each satisfy Thm 3.2, but merging both makes a cycle
    (with A->D and B->C).  Under reading R21 of Thm 3.5 (iii) the batch takes only one."""
    A, B, Cc, Dd = 0, 1, 2, 3
    g = dag.make_graph("fig6", [1, 1, 1, 1], [(A, Cc), (B, Dd), (A, Dd), (B, Cc)],
                       [100, 90, 10, 10])
    before = C.FALLBACKS[0]
    co, nc = C.coarsen(g.n, g.src, g.dst, g.nbytes, 2)
    assert C.FALLBACKS[0] == before                              # no defensive shrink needed
    assert not (co[A] == co[Cc] and co[B] == co[Dd] and co[A] != co[B])
    assert C.heights(nc, list(_coarse_edges(g, co))) is not None
    # the heaviest edge A->C is merged first
    assert co[A] == co[Cc]


def test_second_path_blocks_a_merge():
    """u->w->v and u->v: merging (u, v) alone would close a cycle (Thm 3.2); (ii) refuses it
    while w is separate, so u and v only meet after w has joined one of them."""
    u, w, v = 0, 1, 2
    g = dag.make_graph("tri", [1, 1, 1], [(u, w), (w, v), (u, v)], [1, 1, 1000])
    co, nc = C.coarsen(g.n, g.src, g.dst, g.nbytes, 2)
    assert nc == 2 and co[u] != co[v]
    co1, nc1 = C.coarsen(g.n, g.src, g.dst, g.nbytes, 1)
    assert nc1 == 1


def test_random_dags_stay_acyclic_and_reach_the_target():
    fallbacks = C.FALLBACKS[0]
    for s in range(40):
        g = dag.random_dag(700 + s, 30 + 7 * s, 1.5, D=2, max_bytes=10_000)
        for target in (1, 4, 12):
            co, nc = C.coarsen(g.n, g.src, g.dst, g.nbytes, target)
            assert sorted(set(co.tolist())) == list(range(nc))
            assert C.heights(nc, list(_coarse_edges(g, co))) is not None
            assert nc >= min(target, g.n) or nc == 1
            # dense ids ordered by the smallest op of each vertex
            firsts = [int(np.nonzero(co == k)[0][0]) for k in range(nc)]
            assert firsts == sorted(firsts)
    assert C.FALLBACKS[0] == fallbacks          # Thm 3.5 under R21 never produced a cycle


def test_exhaustive_matches_brute_force(O):
    g = dag.random_dag(9, 40, 1.5, D=2, p_max=3000, max_bytes=100_000, beta0=400,
                       beta1_fs=20_000)
    co, nc = C.coarsen(g.n, g.src, g.dst, g.nbytes, 6)
    order = dag.random_topo_order(g, 1)
    best, idx, mk = C.exhaustive(O, g, order, co, nc)
    # brute force by hand over the 2^6 placements
    vals = []
    for bits in itertools.product([0, 1], repeat=nc):
        c = sum(b << k for k, b in enumerate(bits))
        vals.append((O.makespan(g, C.expand(co, 2, c), order), c))
    assert (best, idx) == min(vals)
    assert mk.shape == (2 ** nc,)
