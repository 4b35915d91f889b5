"""TEST INFRASTRUCTURE ONLY: reference graph coarsening (row f2) and exhaustive coarse search.

Follows PAPER.md §3.3 in its order and notation, plain Python, no shared code with the CUDA path:

* Definition 3.4 (L245-247): height H(v) = number of vertices on the longest root-to-v path,
  roots have H = 1, computed level by level (the modified Kahn sort of footnote 1).
* Theorem 3.5 (L249-253): a set M of edges (u_i, v_i) may be merged in one batch if
  (i)   M is a matching;
  (ii)  |succ(u_i)| = 1 or |prec(v_i)| = 1 or H(v_i) = H(u_i) + 1 or
        H(w) > H(u_i) + d_i for every w in succ(u_i), w != v_i   (d_i = H(v_i) - H(u_i));
  (iii) for i != j: h(u_i) != h(v_j) - d_j  or  (u_i, v_j) not in E      -- reading R21.
* "Our coarsening algorithm" (L265-267): each iteration merges all feasible edges, prioritised
  by the size of the connecting edge (the comm estimate, L263), until the DAG reaches the target
  size or no feasible edge is left.  Ops of a merged vertex inherit its device (L269).

Readings (R21-R23):
  R21 (iii) as extracted reads "h(u_i) != h(v_j) + d_j", which is always true for an edge
      (u_i, v_j) (H(v_j) > H(u_i)) and would accept Figure 6's cyclic double merge; with
      h(v_j) - d_j = h(u_j) it forbids exactly Figure 6's case (A->D with H(A) = H(B)).  We use
      that reading and, defensively, check the merged graph for a cycle (Kahn) and drop the later
      half of the batch until it is acyclic.
  R22 priority = the bytes of all original edges between the two merged vertices (ties: smaller
      u, then smaller v); the batch stops early so the graph does not go below the target.
  R23 merged vertex id = the smaller id of the pair; final ids are dense, ordered by the smallest
      op in each merged vertex.
"""

from __future__ import annotations

import numpy as np

FALLBACKS = [0]          # times the defensive cycle check had to shrink a batch (R21)


def heights(nv, edges):
    """Definition 3.4 by level-wise Kahn: roots 1, else 1 + max over predecessors."""
    pred = [[] for _ in range(nv)]
    succ = [[] for _ in range(nv)]
    indeg = [0] * nv
    for u, v in edges:
        succ[u].append(v)
        pred[v].append(u)
        indeg[v] += 1
    H = [0] * nv
    level = [v for v in range(nv) if indeg[v] == 0]
    h = 1
    seen = 0
    while level:
        nxt = []
        for v in level:
            H[v] = h
            seen += 1
            for w in succ[v]:
                indeg[w] -= 1
                if indeg[w] == 0:
                    nxt.append(w)
        level = nxt
        h += 1
    return H if seen == nv else None          # None: not a DAG


def _acyclic(nv, edges):
    return heights(nv, edges) is not None


def coarsen(n, src, dst, nbytes, target):
    """Returns coarse_of [n] (dense ids) and the number of coarse vertices."""
    rep = list(range(n))                       # op -> current vertex id (an op id)

    def find(a):
        r = a
        while rep[r] != r:
            r = rep[r]
        while rep[a] != r:                     # path compression (roots are unchanged)
            rep[a], a = r, rep[a]
        return r

    while True:
        ids = sorted({find(a) for a in range(n)})
        if len(ids) <= target:
            break
        idx = {v: k for k, v in enumerate(ids)}
        w = {}
        for a, b, by in zip(src, dst, nbytes):
            ra, rb = find(int(a)), find(int(b))
            if ra != rb:
                w[(idx[ra], idx[rb])] = w.get((idx[ra], idx[rb]), 0) + int(by)
        nv = len(ids)
        E = set(w)
        H = heights(nv, list(E))
        succ = [set() for _ in range(nv)]
        pred = [set() for _ in range(nv)]
        for u, v in E:
            succ[u].add(v)
            pred[v].add(u)
        cand = sorted(E, key=lambda e: (-w[e], e[0], e[1]))
        M = []
        matched = set()
        acc_v = {}                             # accepted v_j -> u_j
        acc_u = {}                             # accepted u_j -> v_j
        for u, v in cand:
            if u in matched or v in matched:                                    # (i)
                continue
            d = H[v] - H[u]
            ok = (len(succ[u]) == 1 or len(pred[v]) == 1 or d == 1 or
                  all(H[x] > H[u] + d for x in succ[u] if x != v))             # (ii)
            if not ok:
                continue
            # (iii), reading R21: no accepted pair j with (u, v_j) in E and H(u) == H(u_j),
            # nor (u_j, v) in E and H(u_j) == H(u)
            if any(x in acc_v and H[acc_v[x]] == H[u] for x in succ[u]):
                continue
            if any(p in acc_u and H[p] == H[u] for p in pred[v]):
                continue
            M.append((u, v))
            matched |= {u, v}
            acc_v[v] = u
            acc_u[u] = v
            if nv - len(M) <= target:
                break
        while M:
            comp = list(range(nv))
            for u, v in M:
                comp[v] = u
            merged = {(comp[a], comp[b]) for a, b in E if comp[a] != comp[b]}
            # dense relabel for the acyclicity check
            keep = sorted(set(comp))
            kid = {c: k for k, c in enumerate(keep)}
            if _acyclic(len(keep), [(kid[a], kid[b]) for a, b in merged]):
                break
            M = M[:len(M) // 2]                # defensive (R21): drop the later half
            FALLBACKS[0] += 1
        if not M:
            break
        for u, v in M:                          # the merged vertex keeps the smaller op id
            ru, rv = ids[u], ids[v]
            lo, hi = min(ru, rv), max(ru, rv)
            rep[hi] = lo
    roots = sorted({find(a) for a in range(n)})          # smallest op of each vertex, ordered
    dense = {r: k for k, r in enumerate(roots)}
    coarse_of = np.asarray([dense[find(a)] for a in range(n)], np.int32)
    return coarse_of, len(roots)


def expand(coarse_of, D, index):
    """Placement of candidate `index`: coarse vertex k gets digit k of index in base D."""
    b = {2: 1, 4: 2, 8: 3}[D]
    return ((int(index) >> (b * coarse_of.astype(np.int64))) & (D - 1)).astype(np.uint8)


def exhaustive(O, g, order, coarse_of, n_coarse):
    """Brute force over every coarse placement: (best makespan, smallest best index)."""
    total = g.D ** n_coarse
    xs = np.stack([expand(coarse_of, g.D, c) for c in range(total)])
    mk, _ = O.makespan_batch(g, xs, np.asarray(order, np.int32))
    best = int(mk.min())
    return best, int(np.nonzero(mk == best)[0][0]), mk
