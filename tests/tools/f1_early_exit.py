"""Row f1, second half: how much of K1's walk an early exit could skip (measure before building).

A candidate whose makespan will be >= its base's makespan M_b can never win the step's argmin
(j = 0, the base itself, wins every tie), so its walk may stop as soon as a lower bound on its
makespan reaches M_b.  A warp (32 x CPL candidates of one group) can stop only when every lane
has.  Lower bounds after the op at position v of the candidate's order (all monotone in v):
  LB1 = max over started ops of C_u                          (a device's free time)
  LB2 = max_d (free time of d + sum of p of d's ops after v)  (device load still to run)
  LB3 = max over started ops u of C_u + tail(u), tail(u) = longest p-path from u to a sink
        without u itself (its successors still have to run, transfers >= 0)
Prints, per config and base, the mean fraction of warp walks (positions) an exit at the first
position where all lanes' max(LB1, LB2, LB3) >= M_b would skip, from the oracle's trace.

usage: python tests/tools/f1_early_exit.py [config ...] [config=bases.npz ...]\n(CPU, test infrastructure: uses oracle/; bases.npz from tests/tools/dump_bases.py on the GPU)
"""
import json
import sys

import numpy as np

sys.path.insert(0, '.')
from oracle import oracle as O  # noqa: E402
from workloads import configs, seeds  # noqa: E402


def tails(g):
    n = g.n
    order = seeds.order_fifo(g)
    succ = [[] for _ in range(n)]
    for s, d in zip(g.src.tolist(), g.dst.tolist()):
        succ[s].append(d)
    bl = np.zeros(n, np.int64)
    for v in reversed(order.tolist()):
        bl[v] = int(g.p[v]) + (max(bl[w] for w in succ[v]) if succ[v] else 0)
    return bl - g.p.astype(np.int64)


def exit_position(g, tail, x, order, mk_base):
    mk, t = O.makespan(g, x, order, trace=True)
    if mk >= (1 << 62):
        return 0, mk                              # invalid: exits at once
    C = t["C"][order]                             # by position
    p = g.p.astype(np.int64)[order]
    xd = x[order].astype(np.int64)
    lb = np.maximum.accumulate(C + tail[order])   # LB3 (>= LB1)
    free = np.zeros((g.D, g.n), np.int64)
    for d in range(g.D):
        on = xd == d
        cd = np.where(on, C, 0)
        free[d] = np.maximum.accumulate(cd)
        rem = np.cumsum((p * on)[::-1])[::-1]     # load of d at positions >= v
        rem_after = np.concatenate([rem[1:], [0]])
        lb = np.maximum(lb, free[d] + rem_after)  # LB2
    hit = np.nonzero(lb >= mk_base)[0]
    return (int(hit[0]) + 1 if len(hit) else g.n), mk


def main(names, bases_npz=None, out_name="profiles/r2_f1_early_exit.json"):
    """bases_npz: {config: file written by tests/tools/dump_bases.py} -- the bases after s steps
    of the GPU search (key "x_s"/"order_s"), else the step-0 seeds"""
    out = {}
    for name in names:
        cfg = configs.CONFIGS[name]
        g = configs.graph_for(cfg)
        tail = tails(g)
        K = cfg.candidates_per_gpu // cfg.bases
        stages = [(0, seeds.bench_seeds(g, cfg.bases, configs.SEARCH_SEED))]
        if bases_npz and name in bases_npz:
            z = np.load(bases_npz[name])
            stages = [(int(s), (z[f"x_{int(s)}"], z[f"order_{int(s)}"])) for s in z["steps"]]
        res = {}
        for step, (xs, orders) in stages:
          rng = np.random.default_rng(0)
          for b in range(cfg.bases):
            mk_b = O.makespan(g, xs[b], orders[b])
            fr, worse = [], 0
            groups = rng.choice(np.arange(1, K // 128), 6, replace=False)
            for grp in groups:
                for w in range(2):                # two 64-candidate warps (CPL 2) per group
                    pos = []
                    for j in range(128 * grp + 64 * w, 128 * grp + 64 * w + 64):
                        ok, x, o = O.candidate(g, cfg.bases, b, xs, orders, int(j),
                                               configs.SEARCH_SEED, step, configs.MOVE_MIX)
                        if not ok:
                            pos.append(0)
                            continue
                        e, mk = exit_position(g, tail, x, o, mk_b)
                        worse += mk >= mk_b
                        pos.append(e)
                    fr.append(1.0 - max(pos) / g.n)
            res[f"step{step}_base{b}"] = {
                "step": step, "base": b, "base_mk": int(mk_b),
                "skippable_warp_fraction": float(np.mean(fr)), "warps": len(fr),
                "lanes_not_better": worse / (len(fr) * 64)}
            print(name, step, b, res[f"step{step}_base{b}"], flush=True)
        out[name] = res
    json.dump(out, open(out_name, "w"), indent=1)


if __name__ == "__main__":
    args = sys.argv[1:]
    npz = {}
    for a in list(args):
        if a.endswith(".npz"):          # CONFIG=FILE.npz
            k, v = a.split("=", 1)
            npz[k] = v
            args.remove(a)
    main(args or ["inception_v3_2dev", "transformer_2dev"], npz,
         "profiles/r2_f1_early_exit_steps.json" if npz else "profiles/r2_f1_early_exit.json")
