"""Device time of the explicit-row path (K5 + eval32 + fixup) and of its H2D/D2H, per batch."""
import sys, time
import numpy as np
import torch
sys.path.insert(0, '.')
from workloads import configs, dag
from paper_conf_middleware_hafeezsg021_b200 import pesto as P

name = sys.argv[1] if len(sys.argv) > 1 else 'inception_v3_2dev'
cfg = configs.CONFIGS[name]
g = configs.graph_for(cfg)
G = P.Graph.from_arrays(g)
k = cfg.candidates_per_gpu if cfg.candidates_per_gpu <= 65536 else 65536
rows = P.pack_rows(dag.random_placements(g, 11, k), g.D)
order = G.seed_order(P.ORDER_CRITICAL_PATH)
d_rows = torch.from_numpy(rows).cuda()
out = torch.empty(k, dtype=torch.int64, device='cuda')
for _ in range(3):
    G.eval(order, d_rows, out)
torch.cuda.synchronize()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
ev[0].record()
for _ in range(5):
    G.eval(order, d_rows, out)
ev[1].record()
torch.cuda.synchronize()
print(name, 'explicit eval ms', ev[0].elapsed_time(ev[1]) / 5, 'rows MB', rows.nbytes / 1e6)
pin = torch.from_numpy(rows).pin_memory()
torch.cuda.synchronize()
ev[0].record()
for _ in range(5):
    d_rows.copy_(pin, non_blocking=True)
ev[1].record()
torch.cuda.synchronize()
print('H2D ms', ev[0].elapsed_time(ev[1]) / 5)
rh = pin.numpy()
oh = torch.empty(k, dtype=torch.int64).pin_memory().numpy()
G.eval_host(order, rh, oh)
t = time.perf_counter()
for _ in range(5):
    G.eval_host(order, rh, oh)
print('eval_host ms', (time.perf_counter() - t) / 5 * 1e3)
