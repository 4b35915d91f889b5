"""A small workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

Exercises every eval32 path the bench times, at a size the sanitizers finish in minutes:
  * explicit rows (K5 transpose + eval32 mode 0) on a multi-tile graph, D = 2 and D = 4;
  * search steps (eval32 mode 1, the TMA/mbarrier ring) with a swap-heavy mix, so that swapped
    pairs straddle tile boundaries (the walk then waits on the next stage before releasing the
    current one, eval32.cu), committed swaps patched in place (patch kernel) and K4 commits;
  * both candidates-per-lane instances (PESTO_EVAL32_CPL=1 / 2 set by the caller) and the wide
    64-bit instance (a base above the 32-bit saturation point).
Every result is checked against the oracle (bit-exact), so a run that the sanitizer passes is
also a correct run.  Exit code 0 = all equal.

usage: PESTO_EVAL32_CPL=2 compute-sanitizer --tool racecheck python tests/tools/sanitize_run.py
(test infrastructure: it uses oracle/)
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
from oracle import oracle as O  # noqa: E402
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402
from workloads import dag  # noqa: E402


def rows_check(seed, n, D):
    import torch
    g = dag.random_dag(seed, n, 1.6, D=D, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    G = P.Graph.from_arrays(g)
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    x = dag.random_placements(g, seed + 1, 96)
    rows = torch.from_numpy(P.pack_rows(x, D)).cuda()
    got = G.eval(order, rows).cpu().numpy()
    ref, _ = O.makespan_batch(g, x, order)
    assert (got == ref).all(), ("rows", seed, n, D)
    return len(x)


def search_check(seed, n, D, mix, steps, K, sat_base=False):
    g = dag.random_dag(seed, n, 1.6, D=D, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    if sat_base:
        g.p[: n // 2] += 9_000_000        # single-device sum above 4.03 s: one wide base
    G = P.Graph.from_arrays(g)
    orders = np.stack([dag.random_topo_order(g, seed + b) for b in range(2)]).astype(np.int32)
    xs = dag.random_placements(g, seed + 50, 2)
    if sat_base:
        xs[1][:] = 0
    S = P.Search(G, xs, orders, K, mix, seed=seed)
    rx, ro = xs.copy(), orders.copy()
    rmk = np.asarray([O.makespan(g, rx[b], ro[b]) for b in range(2)], np.int64)
    for step in range(steps):
        S.step()
        O.search_step(g, rx, ro, rmk, K, seed, step, mix)
        for b in range(2):
            mk, x, o = S.get(b)
            assert mk == rmk[b] and (x == rx[b]).all() and (o == ro[b]).all(), (seed, step, b)
    return S.swap_stats()


def main():
    # SAN_D4=0 skips the D = 4 cases (under memcheck the instrumented two-candidates-per-lane
    # D = 4 kernel no longer fits its launch bounds)
    d4 = os.environ.get("SAN_D4", "1") != "0"
    n_rows = rows_check(3, 1200, 2) + (rows_check(4, 900, 4) if d4 else 0)
    sw = search_check(11, 1400, 2, (30, 10, 10, 50), 4, 2048)
    sw4 = search_check(12, 1000, 4, (20, 10, 10, 60), 3, 2048) if d4 else None
    wide = search_check(13, 900, 2, (50, 20, 20, 10), 2, 1024, sat_base=True)
    print(f"sanitize_run ok: {n_rows} rows, swaps (in place, rebuilt) D2 {sw} D4 {sw4}, "
          f"wide {wide}; CPL env {os.environ.get('PESTO_EVAL32_CPL', 'auto')}")


if __name__ == "__main__":
    main()
