"""Row f2 on the shaped graphs: coarsen to T vertices, evaluate all D^T coarse placements on the
GPU, compare the best with the expert / topological-split seeds.  Prints one JSON line per config."""
import json, sys, time
import numpy as np
import torch
sys.path.insert(0, '.')
from workloads import configs  # noqa: E402
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402

T = int(sys.argv[1]) if len(sys.argv) > 1 else 20
for name in ['inception_v3_2dev', 'nmt4_2dev_commheavy', 'transformer_2dev']:
    g = configs.graph_for(configs.CONFIGS[name])
    G = P.Graph.from_arrays(g)
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    t0 = time.perf_counter()
    co, nc = G.coarsen(T)
    t_coarsen = time.perf_counter() - t0
    G.eval_coarse_exhaustive(order, co, nc)                     # warm-up (layout, state)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    mk, idx, x = G.eval_coarse_exhaustive(order, co, nc)
    t_exh = time.perf_counter() - t0
    seeds = {'expert': G.seed_placement(P.PLACE_EXPERT, layer=g.layer),
             'topo_split': G.seed_placement(P.PLACE_TOPO_SPLIT, order=order),
             'single': G.seed_placement(P.PLACE_SINGLE)}
    rows = torch.from_numpy(P.pack_rows(np.stack(list(seeds.values())), g.D)).cuda()
    smk = G.eval(order, rows).cpu().numpy()
    print(json.dumps({'config': name, 'n_coarse': nc, 'coarsen_s': round(t_coarsen, 3),
                      'candidates': 2 ** nc, 'exhaustive_s': round(t_exh, 4),
                      'cand_per_s': round(2 ** nc / t_exh), 'best_ms': mk / 1e6,
                      'seeds_ms': {k: int(v) / 1e6 for k, v in zip(seeds, smk)}}))
