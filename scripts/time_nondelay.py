"""Time the row f4(i) non-delay kernel on a shaped config (explicit rows, device-resident)."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402
from workloads import configs, dag  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "inception_v3_2dev"
count = int(sys.argv[2]) if len(sys.argv) > 2 else 8192
g = configs.graph_for(configs.CONFIGS[name])
G = P.Graph.from_arrays(g)
order = G.seed_order(P.ORDER_CRITICAL_PATH)
x = dag.random_placements(g, 3, count)
rows = torch.from_numpy(dag.pack_placements(x, g.D)).cuda()
for mode in (P.DISPATCH_FIXED, P.DISPATCH_NONDELAY):
    G.set_dispatch(mode)
    out = G.eval(order, rows)
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    reps = 3
    for _ in range(reps):
        out = G.eval(order, rows)
    ev1.record()
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1) / reps
    print(f"{name} dispatch={mode} rows={count} {ms:.2f} ms  {count / ms * 1e3:.3e} cand/s  "
          f"mean makespan {out.double().mean().item():.4e}")
