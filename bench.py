#!/usr/bin/env python
"""Benchmark: placement candidates evaluated/sec (and op-relaxations/sec) of the Pesto search
step on B200 (BASELINE.json metric).  One JSON line on rank 0.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config NAME] [--impl pesto|reference]

A step = one pass of the whole hot path over one batch: K2 neighbour decode + K1 makespan of
every candidate + K3 argmin (one kernel) -> N1 allreduce-MIN over ranks -> K4 commit.  Per-GPU work
is fixed as N grows (weak scaling).  `--impl reference` times the CPU oracle on the same
workload (the reference arm of this tier).

Default workload: transformer_2dev (BASELINE.json configs[3], 1,048,576 candidates per step, the
largest single-GPU config; Table 1's Transformer-6 row).
"""

from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from workloads import configs, dag, seeds  # noqa: E402

METRIC = "placement candidates evaluated/sec (and op-relaxations/sec) at 1/2/4/8 B200"
DEFAULT_CONFIG = "transformer_2dev"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default=DEFAULT_CONFIG, choices=sorted(configs.CONFIGS))
    ap.add_argument("--impl", default="pesto", choices=["pesto", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--dispatch", default="fixed", choices=["fixed", "nondelay"],
                    help="row f4(i): nondelay = TF-style ready-queue dispatch by pi priority")
    ap.add_argument("--coarse-pct", type=int, default=0,
                    help="search spec S9 (row f2): %% of candidate groups that move merged "
                         "vertices of a PAPER.md 3.3 coarsening (0 = off, the default mix)")
    ap.add_argument("--coarse-target", type=int, default=200,
                    help="merged vertices of that coarsening (L267: ~200)")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = None

    def __enter__(self):
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        # nvidia-smi takes a few hundred ms to start: wait for its first sample so that a short
        # timed region (10 inception steps are ~50 ms) is sampled too
        t0 = time.perf_counter()
        while self.proc is not None and time.perf_counter() - t0 < 5.0:
            if os.path.getsize(self.path) > 0 or self.proc.poll() is not None:
                break
            time.sleep(0.02)
        return self

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        out = {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        try:
            rows = [r.split(",") for r in open(self.path).read().strip().splitlines() if r.strip()]
        except Exception:
            return out
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            r = [x.strip() for x in r]
            if len(r) < 9:
                continue
            try:
                sm.append(float(r[1]))
                smax.append(float(r[2]))
            except ValueError:
                continue
            for nm, val in zip(names, r[5:9]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        if sm:
            out.update(sm_mhz=statistics.median(sm), sm_max_mhz=max(smax), samples=len(sm))
        out["reasons"] = sorted(reasons)
        return out


def seeds_for(P, G, g, n_bases: int):
    """Search incumbents (row a1) from libpesto's generators: expert, topological split,
    single-device, random.  They must equal workloads/seeds.py's plain-Python restatement, which
    the CPU reference arm starts from (so both arms search the same four bases)."""
    o_cp = G.seed_order(P.ORDER_CRITICAL_PATH)
    o_fifo = G.seed_order(P.ORDER_FIFO)
    o_rand = G.seed_order(P.ORDER_RANDOM, configs.SEARCH_SEED)
    xs = [G.seed_placement(P.PLACE_EXPERT, layer=g.layer) if g.layer is not None
          else G.seed_placement(P.PLACE_TOPO_SPLIT, order=o_cp),
          G.seed_placement(P.PLACE_TOPO_SPLIT, order=o_cp),
          G.seed_placement(P.PLACE_SINGLE),
          G.seed_placement(P.PLACE_RANDOM, seed=configs.SEARCH_SEED)]
    os_ = [o_cp, o_cp, o_fifo, o_rand]
    xs, os_ = np.stack(xs[:n_bases]), np.stack(os_[:n_bases])
    px, po = seeds.bench_seeds(g, n_bases, configs.SEARCH_SEED)
    assert (px == xs).all() and (po == os_).all(), "library seeds differ from workloads/seeds.py"
    return xs, os_


def common_config(args, cfg, g, world):
    """The `config` object both arms print (same keys and values, so the driver can match them)."""
    k_gpu = cfg.candidates_per_gpu
    return {"workload": args.config, "n_ops": g.n, "n_edges": g.m, "D": g.D,
            "candidates_per_step": k_gpu * world, "candidates_per_gpu": k_gpu,
            "bases": cfg.bases, "k_per_base": (k_gpu * world) // cfg.bases,
            "move_mix": list(configs.MOVE_MIX), "search_seed": configs.SEARCH_SEED,
            "seeds": "expert / topological split on the critical-path order, single device on "
                     "the FIFO order, random placement on a random order (workloads/seeds.py)",
            "l2": "GPU arm: flushed (256 MiB write) between timed steps",
            "parallelism": f"candidate-dp{world}", "dispatch": args.dispatch,
            "coarse_groups_pct": args.coarse_pct}


def oracle_rate(g, xs, orders, k_per_base, seconds, threads, nondelay=False, coarse=None):
    """Oracle (as it stands) on a bounded sample of this workload's step-0 candidates: the
    first ids of every base (they span whole 128-id groups, swap groups included)."""
    from oracle import oracle as O
    if coarse is not None:                   # the same S9 coarse groups as the timed search
        with O.coarse_moves(g, *coarse):
            return oracle_rate(g, xs, orders, k_per_base, seconds, threads, nondelay)
    P_ = xs.shape[0]
    mix = configs.MOVE_MIX

    def keys(b, j1):
        if nondelay:
            return O.candidate_keys_model(g, P_, b, xs, orders, 0, j1, configs.SEARCH_SEED, 0,
                                          mix, nondelay=True, threads=threads)
        return O.candidate_keys(g, P_, b, xs, orders, 0, j1, configs.SEARCH_SEED, 0, mix,
                                threads)
    # calibrate a sample size that takes about `seconds` on `threads` threads
    t0 = time.perf_counter()
    probe = max(threads, 8)
    keys(0, probe)
    dt = time.perf_counter() - t0
    per = dt / probe
    sample = int(max(probe * P_, min(k_per_base * P_, seconds / max(per, 1e-9))))
    t0 = time.perf_counter()
    done = 0
    sample_keys = []
    for b in range(P_):
        cnt = sample // P_
        sample_keys.append(keys(b, cnt))
        done += cnt
    dt = time.perf_counter() - t0
    oracle_rate.sample_keys = sample_keys           # the timed sample's keys, for parity
    return done / dt, done, dt


def run_reference(args, rank, world):
    """This tier's reference arm: the CPU oracle as it stands, on the same workload, the same
    four bases (workloads/seeds.py) and the same step-0 candidates; each step is a bounded
    sample, timed on the wall clock (ms_per_step is the measured sample step)."""
    if rank != 0:
        return
    cfg = configs.CONFIGS[args.config]
    g = configs.graph_for(cfg)
    from oracle import oracle as O  # noqa: F401  (TEST INFRASTRUCTURE: the reference arm)
    threads = len(os.sched_getaffinity(0))
    xs, orders = seeds.bench_seeds(g, cfg.bases, configs.SEARCH_SEED)
    k_per_base = cfg.candidates_per_gpu // cfg.bases
    per_step_budget = max(0.5, args.cpu_seconds / max(1, args.steps + args.warmup))
    rates, times, counts = [], [], []
    nd = args.dispatch == "nondelay"
    for i in range(args.warmup + args.steps):
        rate, done, dt = oracle_rate(g, xs, orders, k_per_base, per_step_budget, threads,
                                     nondelay=nd)
        if i >= args.warmup:
            rates.append(rate)
            times.append(dt)
            counts.append(done)
    value = sum(counts) / sum(times)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "candidates/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * statistics.median(times), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "config": common_config(args, cfg, g, 1),
            "op_relaxations_per_s": value * g.n,
            "cpu_baseline": {"value": value, "unit": "candidates/s", "cores": threads,
                             "kind": "oracle",
                             "sample": f"each step: the first {counts[0] // cfg.bases} step-0 "
                                       f"neighbour ids of each of the {cfg.bases} bases "
                                       f"({counts[0]} candidates, ~{per_step_budget:.1f} s), "
                                       "event-driven simulator; ms_per_step is that sample's "
                                       "measured wall time"},
            "e2e": {"value": value, "unit": "candidates/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_pesto(args, rank, world, local):
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_hafeezsg021_b200 import pesto as P

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cfg = configs.CONFIGS[args.config]
    # SURVEY 8(d) roof microbenchmarks on this GPU (integer issue, L2, HBM), before anything else
    roofs = P.measure_roofs(local, 5)
    g = configs.graph_for(cfg)
    G = P.Graph.from_arrays(g, device=local)
    nd = args.dispatch == "nondelay"
    if nd:
        G.set_dispatch(P.DISPATCH_NONDELAY)                 # row f4(i)
    n_bases = cfg.bases
    xs, orders = seeds_for(P, G, g, n_bases)
    k_gpu = cfg.candidates_per_gpu
    k_per_base = (k_gpu * world) // n_bases          # global K per base; each rank gets 1/world
    nid = None
    if world > 1:
        obj = [P.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nid = obj[0]
    S = P.Search(G, xs, orders, k_per_base, configs.MOVE_MIX, configs.SEARCH_SEED, rank, world,
                 nid)
    coarse = None
    if args.coarse_pct > 0:                          # S9 group moves (host coarsening, untimed)
        co, nc = G.coarsen(args.coarse_target)
        S.set_coarse_moves(co, nc, args.coarse_pct)
        coarse = (co, nc, args.coarse_pct)
    seed_mk = [S.get(b)[0] for b in range(n_bases)]
    stream = torch.cuda.current_stream()
    # L2 flush buffer (> 126 MB L2) written between timed steps
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def one_step(ev=None):
        if ev is not None:
            ev[0].record(stream)
        S.eval(stream)
        if ev is not None:
            ev[1].record(stream)
        S.reduce(stream)
        S.commit(stream)
        if ev is not None:
            ev[2].record(stream)

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    launches0 = P.launch_count()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        wall0 = time.perf_counter()
        for i in range(args.steps):
            flush.fill_(i & 0xFF)                    # evict L2 between timed steps (not timed)
            one_step(evs[i])
        torch.cuda.synchronize()
        wall = time.perf_counter() - wall0
    if world > 1:
        dist.barrier()
    launches = P.launch_count() - launches0
    step_ms = [e[0].elapsed_time(e[2]) for e in evs]
    eval_ms = [e[0].elapsed_time(e[1]) for e in evs]
    tot_ms = sum(step_ms)
    t = torch.tensor([tot_ms, sum(eval_ms)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    tot_ms, tot_eval_ms = float(t[0]), float(t[1])
    total_cands = k_gpu * world * args.steps
    value = total_cands / (tot_ms / 1e3)
    best_mk = [S.get(b)[0] for b in range(n_bases)]
    swap_stats = S.swap_stats()
    # the neighbourhood the next step evaluates (DESIGN §4 v6): distinct (placement, order)
    # pairs among this rank's candidates, decoded on the host by the kernels' spec code
    ms = [S.move_stats(b, k_per_base * rank // world, k_per_base * (rank + 1) // world)
          for b in range(n_bases)]
    tot = {k: sum(m[k] for m in ms) for k in ms[0]}
    move_stats = dict(tot, step=S.step_count,
                      distinct_fraction=tot["distinct"] / tot["candidates"],
                      duplicate_fraction=1.0 - (tot["distinct"] + tot["invalid"]) / tot["candidates"])

    # ---- end to end through the public API with host buffers ----
    # every step copies its batch of explicit placement rows in from pinned host memory,
    # evaluates it and copies the makespans out; four workspaces on four streams keep four steps
    # in flight (pesto_eval_batch_host_async), so copies overlap kernels and the kernels of
    # consecutive batches overlap each other
    e2e = None
    if not args.no_e2e:
        rows_h = []
        # two distinct input batches, alternating (one per rank under torchrun: at 8 ranks two
        # 1 M-row batches each would pin 41 GB of host memory)
        for r in range(2 if world == 1 else 1):
            rows = dag.random_packed_rows(g, 11 + 2 * rank + r, k_gpu)
            rows_h.append(torch.from_numpy(rows).pin_memory().numpy())
            del rows
        # batches in flight: 4 for one-wave batches (inception's 64 K rows: their kernels overlap
        # each other), 2 for multi-wave ones (1 M rows: the copy-in of one batch overlaps the
        # evaluation of the other; each workspace holds ~14 GB of scratch at that size)
        nbuf = int(os.environ.get("PESTO_E2E_BUFFERS",
                                  "4" if rows_h[0].nbytes < (1 << 30) else "2"))
        outs = [torch.empty(k_gpu, dtype=torch.int64).pin_memory().numpy() for _ in range(nbuf)]
        wss = [G.workspace() for _ in range(nbuf)]
        sts = [torch.cuda.Stream() for _ in range(nbuf)]
        o = orders[0]

        def e2e_run(n):
            for i in range(n):
                k = i % nbuf
                if i >= nbuf:
                    sts[k].synchronize()             # batch i-nbuf is done and its makespans read
                wss[k].eval_host_async(o, rows_h[i % len(rows_h)], outs[k], stream=sts[k])
            for st_ in sts:
                st_.synchronize()
        nw = max(nbuf, args.warmup)
        e2e_run(nw)
        last0 = max(i for i in range(nw) if i % nbuf == 0)   # the batch buffer 0 holds
        ref0 = G.eval_host(o, rows_h[last0 % len(rows_h)])   # the synchronous API agrees
        assert (ref0 == outs[0]).all(), "async host-buffer evaluation disagrees"
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        e2e_steps = max(4, min(args.steps, 10))
        e2e_run(e2e_steps)
        e2e_s = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(e2e_s, op=dist.ReduceOp.MAX)
        e2e = {"value": k_gpu * world * e2e_steps / float(e2e_s[0]), "unit": "candidates/s",
               "h2d_bytes_per_step": int(rows_h[0].nbytes), "d2h_bytes_per_step": int(8 * k_gpu),
               "api": "pesto_eval_batch_host_async (explicit placement rows from pinned host "
                      f"memory, makespans back to pinned host memory; {nbuf} workspaces on "
                      f"{nbuf} streams, {nbuf} batches in flight)"}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    # ---- roofline of the dominant kernel (K1 eval), DESIGN.md §5 ----
    # K1 is bound by integer issue and latency, not by HBM (the ncu capture in profiles/ shows
    # DRAM at ~12% of peak).  Algorithmic work per candidate: per op one max + one add (C_v), per
    # edge one max (the arrival push), per crossing edge one more max + add (the link queue):
    # 2n + m + 2*cross integer ops; cross is counted at the base placements.
    pk = peaks()
    sm_mhz = pk.get("sm_max_mhz") or 1965.0
    peak_note = ("148 SMs x 128 int32 lanes/clk (4 SMSPs x 32 lanes, one integer warp-instr per "
                 f"clk per SMSP) x {sm_mhz:.0f} MHz (MEASURED_PEAKS.json sm_max_mhz)")
    peak_tops = 148 * 128 * sm_mhz * 1e6 / 1e12
    cross = float(np.mean([int((xs[b][g.src] != xs[b][g.dst]).sum()) for b in range(n_bases)]))
    alg_ops_launch = (2.0 * g.n + g.m + 2.0 * cross) * k_gpu
    eval_avg_s = (tot_eval_ms / args.steps) / 1e3
    achieved = alg_ops_launch / eval_avg_s / 1e12
    traffic = None
    issue = None
    prof = None
    for cand in (f"r2_eval32_{args.config}_ncu.json",
                 f"r1_eval32_{args.config.split('_')[0]}_ncu.json"):
        if os.path.exists(os.path.join(ROOT, "profiles", cand)):
            prof = os.path.join(ROOT, "profiles", cand)
            break
    if prof and world == 1 and not nd:
        try:
            pj = json.load(open(prof))
            if pj.get("config") == args.config:
                traffic = pj["dram_bytes_per_launch"]
                m = pj["metrics"]
                inst = m["smsp__inst_executed.sum"]["value"]
                issue = {"issue_slots_busy_pct": m["smsp__issue_active.avg.pct_of_peak_sustained_active"]["value"],
                         "warps_per_smsp": m["smsp__warps_active.avg.per_cycle_active"]["value"],
                         "dram_GBps": pj.get("dram_GBps"),
                         "l2_bytes_per_launch": pj.get("lts_bytes_per_launch"),
                         "warp_instr_per_op_relax": inst / (k_gpu * g.n),
                         "source": os.path.relpath(prof, ROOT),
                         "note": "ncu capture of the same kernel on the same config (cold cache, "
                                 "one launch); its duration is not this run's"}
        except Exception:
            traffic = None
    st = G.stats(orders[0])
    line = {"metric": METRIC, "value": value, "unit": "candidates/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_ms / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            # the arithmetic the timed kernel computes in: uint32 ns saturating at 4.03 s (exact
            # below it; bases above it run the exact 64-bit instance), keys int64
            "dtype": "u32" if not nd else "int64",
            "data": "synthetic",
            "config": common_config(args, cfg, g, world),
            "workload_details": {
                "live_slots": st["live_slots"],
                "f_x_seeds": [round(float((xs[b][g.src] != xs[b][g.dst]).mean()), 4)
                              for b in range(n_bases)],
                "time_t": "uint32 saturating at 4.03 s (eval32), exact 64-bit for bases "
                          "above it (wide eval32 / eval64)",
                "state_tier": "near ring + far staging in shared memory, cold slots in global "
                              "memory (L2/HBM), device/link state in registers (D = 2) or "
                              "shared memory (D > 2)",
                "n_coarse": int(coarse[1]) if coarse else None},
            "op_relaxations_per_s": value * g.n, "edge_relaxations_per_s": value * g.m,
            "eval_kernel_ms": tot_eval_ms / args.steps,
            "roofline": {"bound": "alu", "achieved": achieved, "peak": peak_tops,
                         "unit": "TOP/s (int32)", "frac": achieved / peak_tops,
                         "traffic": traffic, "peak_source": peak_note,
                         "ops_per_candidate": 2.0 * g.n + g.m + 2.0 * cross,
                         "ncu": issue,
                         "kernel": "nondelay_kernel (row f4(i))" if nd else "eval32_kernel (K1)",
                         "note": "algorithmic int ops (2n+m+2*cross per candidate) / K1 time; "
                                 "traffic = ncu DRAM bytes per K1 launch (profiles/)"},
            "roofs": dict(roofs, source="pesto_measure_roofs (csrc/roofs.cu): K1's max/add/"
                          "saturate chains on all SMs, L2-resident sweeps, 1 GiB copy; best of 5",
                          k1_frac_of_measured_int_roof=achieved * 1e12 / roofs["int_ops_per_s"]),
            "gpu_launches": int(launches),
            "wall_s_timed_region": wall,
            "candidates": move_stats,
            "search": {"seed_makespans": seed_mk, "best_makespans": best_mk,
                       "swaps_patched_in_place": swap_stats[0], "swaps_rebuilt": swap_stats[1]},
            "e2e": e2e}
    line["clocks"] = clk.summary()
    if not args.no_cpu_baseline and world == 1:
        threads = len(os.sched_getaffinity(0))
        rate, done, dt = oracle_rate(g, xs, orders, k_per_base, args.cpu_seconds, threads,
                                     nondelay=nd, coarse=coarse)
        line["cpu_baseline"] = {"value": rate, "unit": "candidates/s", "cores": threads,
                                "kind": "oracle",
                                "sample": f"{done} step-0 neighbour candidates of the same "
                                          f"{n_bases} bases ({dt:.1f}s)"}
        # the same sample on the GPU (a fresh search at step 0): every candidate's key from the
        # kernel instantiation the timed step launches (pesto_search_candidate_keys_ex,
        # PESTO_KEYS_TIMED), compared key by key with the oracle's; saturated 32-bit walks are
        # re-run by the 64-bit kernel there, and the raw timed output is checked on the rest
        S0 = P.Search(G, xs, orders, k_per_base, configs.MOVE_MIX, configs.SEARCH_SEED)
        if coarse is not None:
            S0.set_coarse_moves(*coarse)
        mism = mism_raw = n_sat = 0
        for b, ok in enumerate(oracle_rate.sample_keys):
            if len(ok):
                gk = S0.candidate_keys(b, 0, len(ok), kernel=P.KEYS_TIMED)
                raw = S0.candidate_keys(b, 0, len(ok), kernel=P.KEYS_TIMED_RAW)
                mism += int((gk != ok).sum())
                sat = (raw != P.KEY_INVALID) & ((raw >> np.uint64(24)) >= np.uint64(0xF0000000))
                n_sat += int(sat.sum())
                mism_raw += int((raw[~sat] != ok[~sat]).sum())
                # a clamped walk's exact makespan is at least the clamp
                mism_raw += int(((ok[sat] >> np.uint64(24)) < np.uint64(0xF0000000)).sum())
        line["parity"] = {"checked": int(done), "mismatches": mism,
                          "raw_mismatches": mism_raw, "saturated_walks": n_sat,
                          "what": "keys (makespan << 24 | j) of the cpu_baseline sample from the "
                                  "timed eval32 instantiation (pesto_search_candidate_keys_ex "
                                  "PESTO_KEYS_TIMED: same kernel, CPL and 32-bit/wide split as "
                                  "the step) vs the oracle, bit-exact"}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    rank, world, local = dist_env()
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    run_pesto(args, rank, world, local)


if __name__ == "__main__":
    main()
