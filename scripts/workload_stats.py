"""SURVEY §8(d) structural report of the BASELINE configs (host only, no GPU).

For each config: n, m, m/n, max in/out degree, height H (Def. 3.4), Σp, the Table 1
bucket mix, live ready-time slots W (eval64) and cold slots W32 (eval32) under the
critical-path and FIFO orders, the crossing fraction f_x at the four search seeds, and whether
the 32-bit time path is eligible.  Writes profiles/r1_workload_stats.json and prints a table.
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_middleware_hafeezsg021_b200 import pesto as P  # noqa: E402
from workloads import configs, shaped  # noqa: E402

out = {}
for name, cfg in configs.CONFIGS.items():
    g = configs.graph_for(cfg)
    st = shaped.stats(g)
    G = P.Graph.from_arrays(g, device=-1)
    o_cp = G.seed_order(P.ORDER_CRITICAL_PATH)
    o_fifo = G.seed_order(P.ORDER_FIFO)
    lay_cp, lay_fifo = G.stats(o_cp), G.stats(o_fifo)
    seeds = {"single": G.seed_placement(P.PLACE_SINGLE),
             "topo_split": G.seed_placement(P.PLACE_TOPO_SPLIT, order=o_cp),
             "random": G.seed_placement(P.PLACE_RANDOM, seed=2021)}
    if getattr(g, "layer", None) is not None:
        seeds["expert"] = G.seed_placement(P.PLACE_EXPERT, layer=g.layer)
    fx = {k: round(float((x[g.src] != x[g.dst]).mean()), 4) if g.m else 0.0
          for k, x in seeds.items()}
    out[name] = {**st, "W_cp": lay_cp["live_slots"], "W_fifo": lay_fifo["live_slots"],
                 "time32_exact": lay_cp["time32_exact"], "link_classes": lay_cp["link_classes"],
                 "crossing_fraction": fx, "D": g.D}
    print(f"{name:24s} n={st['n']:6d} m/n={st['m_over_n']:.2f} in<={st['max_in']:5d} "
          f"H={st['height']:5d} sum_p={st['sum_p_ns'] / 1e9:.3f}s mix={st['mix_pct']} "
          f"W cp/fifo={lay_cp['live_slots']}/{lay_fifo['live_slots']} f_x={fx}")
json.dump(out, open(os.path.join(ROOT, "profiles", "r1_workload_stats.json"), "w"), indent=1)
