"""Row f1 (delta evaluation) bound: how much of each candidate walk a base snapshot could skip.

A candidate equals its base only before the first op whose computation reads a moved device:
the region's ops themselves AND every producer of a region op (the producer's push needs the
successor's device to decide cross / link).  The resume point of a group is therefore
min(c, min over region ops of their first producer position), rounded down to a checkpoint.
Prints the mean fraction of the walk that must still run, for the shaped graphs and two orders.
"""
import sys

import numpy as np

sys.path.insert(0, '.')
from workloads import configs  # noqa: E402
import paper_conf_middleware_hafeezsg021_b200.pesto as P  # noqa: E402

for name in ['inception_v3_2dev', 'transformer_2dev', 'nmt4_2dev_commheavy']:
    g = configs.graph_for(configs.CONFIGS[name])
    G = P.Graph.from_arrays(g, device=-1)
    for oname, o in [('critical-path', G.seed_order(P.ORDER_CRITICAL_PATH)),
                     ('random', G.seed_order(P.ORDER_RANDOM, 2021))]:
        n = len(o)
        pos = np.empty(n, np.int64)
        pos[o] = np.arange(n)
        src, dst = np.asarray(g.src), np.asarray(g.dst)
        first = np.full(n, n, np.int64)
        np.minimum.at(first, pos[dst], pos[src])          # first producer, by position
        cs = np.random.default_rng(0).integers(0, n, 4000)
        lim = np.array([min(c, first[c:min(n, c + 64)].min()) for c in cs])
        for delta in (256, 512):
            print(f"{name:22s} {oname:13s} delta {delta}: walk fraction with snapshots "
                  f"{np.mean(n - (lim // delta) * delta) / n:.3f} (region start only, which is "
                  f"wrong: {np.mean(n - (cs // delta) * delta) / n:.3f})")
