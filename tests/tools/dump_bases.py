"""Run the bench's search (same graph, seeds, K, mix, seed) for S steps on the GPU and save the
bases after each requested step count, for CPU-side studies (tests/tools/f1_early_exit.py).

usage: python tests/tools/dump_bases.py CONFIG OUT.npz [STEPS ...]   (default steps: 0 100)
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402
from workloads import configs, seeds  # noqa: E402


def main():
    name, out = sys.argv[1], sys.argv[2]
    want = sorted(int(s) for s in sys.argv[3:]) or [0, 100]
    cfg = configs.CONFIGS[name]
    g = configs.graph_for(cfg)
    G = P.Graph.from_arrays(g)
    xs, orders = seeds.bench_seeds(g, cfg.bases, configs.SEARCH_SEED)
    K = cfg.candidates_per_gpu // cfg.bases
    S = P.Search(G, xs, orders, K, configs.MOVE_MIX, configs.SEARCH_SEED)
    saved = {}
    step = 0
    for w in want:
        while step < w:
            S.step()
            step += 1
        bx, bo, bm = [], [], []
        for b in range(cfg.bases):
            mk, x, o = S.get(b)
            bx.append(x), bo.append(o), bm.append(mk)
        saved[f"x_{w}"] = np.stack(bx)
        saved[f"order_{w}"] = np.stack(bo)
        saved[f"mk_{w}"] = np.asarray(bm, np.int64)
        print(name, "step", w, "makespans", bm, flush=True)
    np.savez_compressed(out, steps=np.asarray(want), **saved)


if __name__ == "__main__":
    main()
