"""Device time of the explicit-row path at a config's full per-GPU batch (K5 + eval32 mode 0 +
fixup; the e2e leg's kernels), plus the host-buffer API time of one batch.

usage: python scripts/time_rows.py [config] [rows]   (PESTO_LIB selects a variant build)
"""
import json
import sys
import time

import torch

sys.path.insert(0, '.')
from workloads import configs, dag  # noqa: E402
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else 'transformer_2dev'
cfg = configs.CONFIGS[name]
g = configs.graph_for(cfg)
G = P.Graph.from_arrays(g)
k = int(sys.argv[2]) if len(sys.argv) > 2 else cfg.candidates_per_gpu
rows = dag.random_packed_rows(g, 11, k)
order = G.seed_order(P.ORDER_CRITICAL_PATH)
d_rows = torch.from_numpy(rows).cuda()
out = torch.empty(k, dtype=torch.int64, device='cuda')
for _ in range(2):
    G.eval(order, d_rows, out)
torch.cuda.synchronize()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
reps = 4
ev[0].record()
for _ in range(reps):
    G.eval(order, d_rows, out)
ev[1].record()
torch.cuda.synchronize()
dev_ms = ev[0].elapsed_time(ev[1]) / reps
first = out[:4096].cpu().numpy()
print(json.dumps({"config": name, "rows": k, "device_ms": dev_ms,
                  "cand_per_s": k / dev_ms * 1e3, "rows_MB": rows.nbytes / 1e6,
                  "checksum": int(first.sum() % (1 << 61))}), flush=True)
