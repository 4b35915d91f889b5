"""Row f2: wall time of the host coarsening (pesto_coarsen, §3.3) on the BASELINE graphs,
for the DESIGN §3.7d descoping note (GPU coarsening is not built: this is a one-off cost)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402
from workloads import configs  # noqa: E402

out = {}
for name in ["inception_v3_2dev", "nmt4_2dev_commheavy", "transformer_2dev", "transformer_4dev_8gpu"]:
    cfg = configs.CONFIGS[name]
    g = configs.graph_for(cfg)
    G = P.Graph.from_arrays(g)
    for target in (20, 200):
        t0 = time.perf_counter()
        _, nc = G.coarsen(target)
        dt = time.perf_counter() - t0
        out[f"{name}/target{target}"] = {"n": g.n, "m": int(len(g.src)), "n_coarse": nc,
                                         "host_s": round(dt, 4)}
        print(name, target, nc, round(dt, 4), flush=True)
json.dump(out, open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/coarsen_time.json", "w"),
          indent=1)
