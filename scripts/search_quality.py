#!/usr/bin/env python
"""Search quality with and without S9 coarse-group moves (row f2, DESIGN.md §4 S9).

Runs the bench's search (same seeds, K, move mix) for a number of steps at several coarse-group
percentages and records each base's incumbent makespan along the way.  GPU only; writes one JSON
document (default gpurun_out/search_quality.json).

  python scripts/search_quality.py [--configs a,b] [--steps 300] [--pcts 0,20] [--target 200]
"""

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from workloads import configs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="inception_v3_2dev,transformer_2dev,nmt4_2dev_commheavy")
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--pcts", default="0,20")
    ap.add_argument("--target", type=int, default=200)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "search_quality.json"))
    a = ap.parse_args()
    import torch
    from paper_conf_middleware_hafeezsg021_b200 import pesto as P
    res = []
    for name in a.configs.split(","):
        cfg = configs.CONFIGS[name]
        g = configs.graph_for(cfg)
        G = P.Graph.from_arrays(g)
        t0 = time.perf_counter()
        co, nc = G.coarsen(a.target)
        t_coarsen = time.perf_counter() - t0
        xs, orders = bench.seeds_for(P, G, g, cfg.bases)
        k_per_base = cfg.candidates_per_gpu // cfg.bases
        for pct in [int(x) for x in a.pcts.split(",")]:
            S = P.Search(G, xs, orders, k_per_base, configs.MOVE_MIX, configs.SEARCH_SEED)
            if pct:
                S.set_coarse_moves(co, nc, pct)
            traj = {0: [S.get(b)[0] for b in range(cfg.bases)]}
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for s in range(1, a.steps + 1):
                S.step()
                if s in (10, 30, 100, 300, 1000, 2000, a.steps):
                    traj[s] = [S.get(b)[0] for b in range(cfg.bases)]
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            res.append({"config": name, "coarse_pct": pct, "n_coarse": nc, "coarsen_s": t_coarsen,
                        "steps": a.steps, "k_per_base": k_per_base, "bases": cfg.bases,
                        "wall_s": dt, "makespans_by_step": traj,
                        "swap_stats": list(S.swap_stats())})
            print(json.dumps(res[-1]), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
