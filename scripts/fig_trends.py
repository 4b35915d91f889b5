#!/usr/bin/env python
"""Qualitative PAPER.md Fig. 5 / Fig. 8 trends on the synthetic graphs (SURVEY §8(f) row f4:
"reproduce the qualitative Fig. 5 / Fig. 8 trends on synthetic graphs by scaling p and beta",
L378-380).  GPU only; writes gpurun_out/fig_trends.json.

* Fig. 8(a) analogue: compute speed s x (every p_i -> max(1, p_i // s)), NVLink-like comm: the
  makespan reduction of the search's best schedule over the expert seed (L308).
* Fig. 8(b) analogue: communication speed c x (beta0, beta1 -> beta / c) at 1x compute.
* Fig. 5 analogue (L200): the search run with congestion-free links (a planner that ignores
  link congestion, L113) and its result replayed with FCFS links, against the search run with
  FCFS links (congestion-aware), both judged under FCFS.

The search is the north star's (default mix) with 20% S9 coarse groups over a
200-vertex PAPER.md §3.3 coarsening, from the bench seeds (expert, topological split, single
device, random).  The paper's own numbers need its profiles and V100 testbed (not reproduced).

  python scripts/fig_trends.py [--config nmt4_2dev_commheavy] [--steps 100]
"""

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from workloads import configs  # noqa: E402

NVLINK_B0, NVLINK_B1 = 10_000, 40_000      # SURVEY §8(d) NVLink-V100-like comm model


def run_search(P, G, g, cfg, steps, coarse):
    xs, orders = bench.seeds_for(P, G, g, cfg.bases)
    S = P.Search(G, xs, orders, cfg.candidates_per_gpu // cfg.bases, configs.MOVE_MIX,
                 configs.SEARCH_SEED)
    if coarse is not None:
        S.set_coarse_moves(*coarse)
    seed_mk = [S.get(b)[0] for b in range(cfg.bases)]
    for _ in range(steps):
        S.step()
    res = [S.get(b) for b in range(cfg.bases)]
    best = int(np.argmin([r[0] for r in res]))
    return seed_mk, res[best]


def scaled_graph(P, base, s_compute, c_comm):
    g = base.with_comm(base.D, max(1, int(round(NVLINK_B0 / c_comm))),
                       max(1, int(round(NVLINK_B1 / c_comm))))
    g.p = np.maximum(1, base.p // s_compute).astype(np.int64)
    return g, P.Graph.from_arrays(g)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="nmt4_2dev_commheavy")
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "fig_trends.json"))
    a = ap.parse_args()
    import torch
    from paper_conf_middleware_hafeezsg021_b200 import pesto as P
    cfg = configs.CONFIGS[a.config]
    base = configs.graph_for(cfg)
    out = {"config": a.config, "steps": a.steps, "k_per_step": cfg.candidates_per_gpu,
           "comm_1x": {"beta0_ns": NVLINK_B0, "beta1_fs_per_byte": NVLINK_B1},
           "fig8a": [], "fig8b": []}
    coarse_of = None
    for key, settings in (("fig8a", [(s, 1.0) for s in (1, 2, 4, 8)]),
                          ("fig8b", [(1, c) for c in (0.1, 0.25, 0.5, 1.0, 2.0)])):
        for s, c in settings:
            g, G = scaled_graph(P, base, s, c)
            if coarse_of is None:
                coarse_of = G.coarsen(200)            # the graph's structure: same for all scales
            t0 = time.perf_counter()
            seed_mk, (mk, x, o) = run_search(P, G, g, cfg, a.steps, (*coarse_of, 20))
            torch.cuda.synchronize()
            rec = {"compute_speed": s, "comm_speed": c, "expert_ms": seed_mk[0] / 1e6,
                   "seeds_ms": [v / 1e6 for v in seed_mk], "search_ms": mk / 1e6,
                   "reduction_vs_expert": 1.0 - mk / seed_mk[0],
                   "cross_edges": int((x[g.src] != x[g.dst]).sum()),
                   "ops_per_device": np.bincount(x, minlength=g.D).tolist(),
                   "wall_s": time.perf_counter() - t0}
            out[key].append(rec)
            print(key, json.dumps(rec), flush=True)
    # Fig. 5: planning with and without congestion, both executed with FCFS links (1x, 1x)
    g, G = scaled_graph(P, base, 1, 1.0)
    _, (mk_fcfs, x_f, o_f) = run_search(P, G, g, cfg, a.steps, (*coarse_of, 20))
    G.set_link_model(P.LINKS_UNLIMITED)
    _, (mk_free_plan, x_u, o_u) = run_search(P, G, g, cfg, a.steps, (*coarse_of, 20))
    rows = torch.from_numpy(P.pack_rows(np.stack([x_u, x_f]), g.D)).cuda()
    free_of_f = int(G.eval(o_f, rows[1:2]).cpu()[0])        # FCFS plan without congestion
    G.set_link_model(P.LINKS_FCFS)
    replay = int(G.eval(o_u, rows[0:1]).cpu()[0])            # congestion-free plan, real links
    out["fig5"] = {"fcfs_planned_ms": mk_fcfs / 1e6,
                   "congestion_free_planned_ms_as_planned": mk_free_plan / 1e6,
                   "congestion_free_planned_ms_with_fcfs_links": replay / 1e6,
                   "fcfs_plan_without_congestion_ms": free_of_f / 1e6,
                   "slowdown_of_congestion_oblivious_plan": replay / mk_fcfs,
                   "cross_edges_fcfs_plan": int((x_f[g.src] != x_f[g.dst]).sum()),
                   "cross_edges_free_plan": int((x_u[g.src] != x_u[g.dst]).sum())}
    print("fig5", json.dumps(out["fig5"]), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(out, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
