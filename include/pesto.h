/*
 * pesto.h -- C ABI of libpesto.so: batched makespan evaluation and parallel local search over
 * operation-level placements and schedules of a DNN op DAG, on B200 (sm_100a).
 *
 * The operation every entry point computes is Pesto's objective (Hafeez et al., Middleware'21,
 * PAPER.md): the makespan C_max (L159-162 eq. (3); "time between the first task arrival and
 * the last task completion", L111) of a DAG G=(V,E) whose ops have compute times p_i
 * (L142 §3.2.1), under
 *   - precedence: op j starts only after op i completed and its data transfer completed (L144);
 *   - a transfer only when producer and consumer sit on different devices, taking
 *     T = beta0 + beta1 * bytes (L138 §3.1) on the directed link between them (L144);
 *   - no overlap on each device and on each link, no pre-emption (L146);
 *   - one First-Come-First-Served queue per directed link (L144, L188-198 §3.2.2);
 *   - a schedule given as a priority order pi: each device runs its ops in pi order (the
 *     per-device order TF enforces with control dependencies, L279; the simulator's "adds
 *     precedence constraints", L374).
 * Readings of points PAPER.md leaves open are listed in DESIGN.md §2 (R1-R17).  All times are
 * int64 nanoseconds, so results are exact and reproducible bit for bit.
 *
 * Conventions
 *   - Host arrays passed to *_create / pesto_comm_model are COPIED; the caller may free them
 *     on return.  Device pointers (placements, makespans, keys) are BORROWED and must stay
 *     alive until the work enqueued on `cuda_stream` completes.  Streams are borrowed
 *     (cudaStream_t passed as void*; NULL = the legacy default stream).
 *   - Every call returns a pesto_status; no C++ exception crosses the ABI.  Validation
 *     failures return before any GPU work.  Asynchronous CUDA/NCCL errors surface on the next
 *     call that synchronises.  pesto_last_error() gives a thread-local description.
 *   - Per-candidate infeasibility (a device code >= D, a device the op's mask forbids, an
 *     invalid search move) is data, not an error: makespan INT64_MAX / key UINT64_MAX.
 *   - Handles are not thread-safe.  Destroy a handle only after synchronising the streams
 *     that used it.
 */
#ifndef PESTO_H
#define PESTO_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct pesto_graph pesto_graph;     /* opaque: host copies + device buffers, one GPU */
typedef struct pesto_search pesto_search;   /* opaque: population, keys, optional NCCL comm   */

typedef enum {
    PESTO_OK = 0,
    PESTO_EINVAL = 1,      /* bad argument: index out of range, self loop, negative size ...  */
    PESTO_ECYCLE = 2,      /* G is not a DAG (L142)                                            */
    PESTO_ENOTTOPO = 3,    /* order is not a permutation / not a linear extension of G         */
    PESTO_EOVERFLOW = 4,   /* sum p + sum_e max_L t_e >= 2^40 ns, or a t_e overflows int64     */
    PESTO_ENOMEM = 5,      /* host or device allocation failed                                 */
    PESTO_ECUDA = 6,       /* CUDA runtime error (see pesto_last_error)                        */
    PESTO_ENCCL = 7,       /* NCCL unavailable or failed                                       */
    PESTO_ESTATE = 8       /* call not valid in this state (comm model unset, host-only ...)   */
} pesto_status;

#define PESTO_INFEASIBLE INT64_MAX
#define PESTO_KEY_INVALID UINT64_MAX
#define PESTO_MAX_OPS (1 << 24)
#define PESTO_MAX_DEVICES 8

/* ------------------------------------------------------------------------------------------ */
/* Graph ingest                                                              */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
    int32_t n_ops;              /* 1 .. 2^24                                                  */
    const int64_t *compute_ns;  /* [n_ops] p_i >= 0 (L142)                                     */
    int64_t n_edges;            /* >= 0; multi-edges allowed, each its own tensor (R4)         */
    const int32_t *src;         /* [n_edges] producer op id                                    */
    const int32_t *dst;         /* [n_edges] consumer op id; src != dst; G acyclic              */
    const int64_t *bytes;       /* [n_edges] >= 0, tensor size for the comm model (L138)       */
    int32_t n_devices;          /* D in 1..8; placement rows use b = 1 (D<=2), 2 (D<=4), 4 bits */
    const uint8_t *allowed;     /* [n_ops] device bitmask (device affinity, L121/L175) or NULL  */
    int32_t cuda_device;        /* ordinal for device buffers; -1 = host-only handle (ingest,    */
                                /* layout, seeds; eval/search then return PESTO_ESTATE)         */
} pesto_graph_desc;

/* Validates (indices, self loops, Kahn cycle check) and copies G.  Errors: EINVAL, ECYCLE,
 * ENOMEM, ECUDA. */
pesto_status pesto_graph_create(const pesto_graph_desc *desc, pesto_graph **out);
void pesto_graph_destroy(pesto_graph *g);                          /* NULL-safe */

/* Linear comm model of the directed link src_dev -> dst_dev (L138 §3.1; per ordered pair,
 * L188-198): t_e = beta0_ns + ceil(bytes_e * beta1_fs_per_byte / 10^6) (reading R6, exact via
 * a 128-bit product).  src_dev/dst_dev = -1 is a wildcard (all pairs a != b).  Both
 * coefficients >= 0.  Errors: EINVAL, EOVERFLOW (the 2^40 guard is checked here, over all
 * links set so far). */
pesto_status pesto_comm_model(pesto_graph *g, int32_t src_dev, int32_t dst_dev,
                              int64_t beta0_ns, int64_t beta1_fs_per_byte);

/* Link model.  PESTO_LINKS_FCFS (the default, Pesto's model): each
 * directed link is one serial FCFS queue, a transfer starts at
 * max(producer completion, link free).  PESTO_LINKS_UNLIMITED: transfers never queue and start
 * at the producer's completion -- the "unlimited bandwidth" assumption of prior work that
 * PAPER.md L113 / L200 (Fig. 5) contrasts with.  Applies to every later pesto_eval_batch* and
 * search step on g; evaluations under PESTO_LINKS_UNLIMITED run on the exact 64-bit kernel
 * (a modelling variant, not the throughput path).  Errors: EINVAL. */
typedef enum { PESTO_LINKS_FCFS = 0, PESTO_LINKS_UNLIMITED = 1 } pesto_link_model;
pesto_status pesto_graph_set_link_model(pesto_graph *g, int32_t model);

/* Dispatch.  PESTO_DISPATCH_FIXED (the default, Pesto's schedule): each
 * device runs its ops in pi order (L279 control dependencies, L374).  PESTO_DISPATCH_NONDELAY:
 * TensorFlow's per-device ready queue ("picks an operation from the ready queue")
 * with pi as the pick priority -- whenever a device is idle it starts, among its ops whose
 * inputs have all arrived, the one earliest in pi (reading R24).  Links keep
 * the link model.  Applies to every later pesto_eval_batch* and search step on g; runs on the
 * exact 64-bit non-delay kernel (one warp per candidate; a modelling variant, not the
 * throughput path).  Those calls return PESTO_ESTATE unless every p_i >= 1 ns, every transfer
 * on every link >= 1 ns (R24: simultaneous zero-length events have no TF-defined order) and
 * n_ops <= 2^20.  pesto_eval_coarse_exhaustive requires PESTO_DISPATCH_FIXED.  Errors: EINVAL. */
typedef enum { PESTO_DISPATCH_FIXED = 0, PESTO_DISPATCH_NONDELAY = 1 } pesto_dispatch;
pesto_status pesto_graph_set_dispatch(pesto_graph *g, int32_t mode);

/* Feasibility constraints: per-device memory footprint and
 * colocation groups (L175).  A candidate violating one is infeasible: makespan INT64_MAX,
 * search key UINT64_MAX.  All arrays HOST, copied:
 *   mem_bytes:  [n_ops] footprint of each op, >= 0; NULL = the sum of its input and output
 *               tensor bytes (every edge into or out of the op, L202);
 *   cap_bytes:  [n_devices] cap on the summed footprint of the ops on each device, >= 0;
 *               NULL = no memory constraint;
 *   coloc:      [n_ops] colocation group of each op in [0, n_ops), -1 = none; ops of one
 *               group must share a device; NULL = no colocation.
 * Both NULL (cap_bytes and coloc) clears the constraints.  Search bases must satisfy them
 * (pesto_search_create fails with EINVAL otherwise; a later change is checked at the next
 * step: ESTATE).  Errors: EINVAL. */
pesto_status pesto_graph_set_constraints(pesto_graph *g, const int64_t *mem_bytes,
                                         const int64_t *cap_bytes, const int32_t *coloc);

/* Row f2: Pesto's graph coarsening (§3.3): heights (Def. 3.4), batch merges
 * under Theorem 3.5 (reading R21 of (iii)), prioritised by the bytes between the merged
 * vertices, repeated until at most `target` vertices remain or nothing can be merged.
 *   coarse_of: HOST [n_ops] out, merged vertex of each op in [0, *n_coarse), numbered by each
 *              vertex's smallest op id.   Host-only (works on a host-only handle).
 * Errors: EINVAL (target < 1), ECYCLE (internal). */
pesto_status pesto_coarsen(pesto_graph *g, int32_t target, int32_t *coarse_of, int32_t *n_coarse);

/* Row f2: every placement of the merged vertices, each op on its vertex's device (L269),
 * evaluated under order pi on the GPU: D^n_coarse candidates, candidate j giving vertex k the
 * device (j >> (b*k)) & (D-1), b = log2 D.  Requires D in {1, 2, 4, 8}, b*n_coarse <= 24, the
 * FCFS link model, fixed dispatch, no row-f3 constraints, an eval32-eligible graph and a best makespan below
 * 4.03 s (else ESTATE).  Candidates with a vertex on a device some member may not use are
 * skipped.  Outputs (HOST): the best makespan (INT64_MAX if none is feasible), the smallest
 * best index, and its placement by op id [n_ops].  Synchronises.  Errors: EINVAL, ESTATE,
 * ECUDA. */
pesto_status pesto_eval_coarse_exhaustive(pesto_graph *g, const int32_t *order,
                                          const int32_t *coarse_of, int32_t n_coarse,
                                          int64_t *best_makespan, int64_t *best_index,
                                          uint8_t *best_x, void *cuda_stream);

typedef struct {
    int32_t n_ops, n_devices;
    int64_t n_edges;
    int32_t live_slots;         /* W: ready-time slots per candidate for this order           */
    int32_t n_tiles;            /* DAG tiles streamed by TMA per candidate group               */
    int64_t layout_bytes;       /* position-space record stream size                            */
    int32_t max_in_degree, max_out_degree;
    int32_t link_classes;       /* distinct (beta0, beta1) among the directed links              */
    int32_t time32_exact;       /* 1 if every makespan fits int32 (worst-case guard < 2^31)      */
} pesto_graph_stats;

/* Builds (or fetches from the per-graph cache) the position-space layout for `order` and
 * reports its statistics.  order: host [n_ops], a topological order.  Errors: ENOTTOPO. */
pesto_status pesto_graph_stats_for(pesto_graph *g, const int32_t *order, pesto_graph_stats *st);

/* ------------------------------------------------------------------------------------------ */
/* Seeds (host, once)                                                         */
/* ------------------------------------------------------------------------------------------ */
enum { PESTO_ORDER_CRITICAL_PATH = 0,  /* Kahn, max-heap on bottom level (p only), ties by op id;
                                          the naive critical-path list order of L98 */
       PESTO_ORDER_FIFO = 1,           /* Kahn with a FIFO queue in op-id order                  */
       PESTO_ORDER_RANDOM = 2 };       /* Kahn with a seeded random pick (TF ready queue, L90)    */
pesto_status pesto_seed_order(pesto_graph *g, int32_t kind, uint64_t seed, int32_t *order_out);

enum { PESTO_PLACE_SINGLE = 0,         /* every op on its lowest allowed device                  */
       PESTO_PLACE_EXPERT = 1,         /* contiguous layers per device: floor(layer*D/n_layers)  */
                                       /* (L308; the caller's layer tags carry the colocations)  */
       PESTO_PLACE_TOPO_SPLIT = 2,     /* `order` cut into D contiguous segments of ~equal sum p  */
                                       /* (an mTOPO-like split, L320)                             */
       PESTO_PLACE_RANDOM = 3 };       /* seeded uniform over allowed devices                     */
/* x_out: host [n_ops], one device code per op.  layer_tags needed only for EXPERT, order only
 * for TOPO_SPLIT.  Ops whose mask forbids the chosen device take their lowest allowed one. */
pesto_status pesto_seed_placement(pesto_graph *g, int32_t kind, const int32_t *order,
                                  const int32_t *layer_tags, uint64_t seed, uint8_t *x_out);

/* ------------------------------------------------------------------------------------------ */
/* Batched evaluation of explicit candidates (SURVEY §8(a) a3 + a4, call stack C4)             */
/* ------------------------------------------------------------------------------------------ */
/* Makespan of n_cand candidates sharing one schedule order pi.
 *   order:      HOST [n_ops] topological order (layout cached by content).
 *   placements: DEVICE, 16-byte aligned, n_cand rows; row c holds op i's device code in bits
 *               [b*i, b*i+b) of the row (little-endian bytes), b = 1 (D<=2), 2 (D<=4), 4 (D<=8).
 *   row_stride_bytes: >= ceil(n_ops*b/8), a multiple of 16.
 *   makespans:  DEVICE [n_cand] int64 out; INT64_MAX for an infeasible row.
 * Enqueued on cuda_stream; returns without synchronising.  Errors: EINVAL, ENOTTOPO, ESTATE
 * (comm model missing for a link, or host-only handle), ENOMEM, ECUDA. */
pesto_status pesto_eval_batch(pesto_graph *g, const int32_t *order, const void *placements,
                              int64_t row_stride_bytes, int64_t n_cand, int64_t *makespans,
                              void *cuda_stream);

/* Same with HOST buffers (ideally pinned): copies the rows in, evaluates, copies makespans
 * out, and synchronises the stream before returning (the end-to-end entry point). */
pesto_status pesto_eval_batch_host(pesto_graph *g, const int32_t *order,
                                   const void *placements_host, int64_t row_stride_bytes,
                                   int64_t n_cand, int64_t *makespans_host, void *cuda_stream);

/* Asynchronous host-buffer evaluation.  A workspace owns a private set of evaluation scratch
 * (rows and makespans staging, bit-sliced rows, slot state) on the graph's GPU, so calls on
 * different workspaces (on different streams) may be in flight at once -- e.g. the host->device
 * copy of one batch overlapping the evaluation of the previous one (double buffering).
 * pesto_eval_batch_host_async = pesto_eval_batch_host on the workspace's scratch, enqueued on
 * cuda_stream WITHOUT synchronising: the caller synchronises that stream before reading
 * makespans_host, before reusing placements_host, and before the next call on the same
 * workspace from another stream.  placements_host should be pinned (else the copy is
 * synchronous).  The graph and its layouts are shared (not thread-safe: one host thread).
 * A workspace must be destroyed before its graph.  (pesto_eval_batch, pesto_eval_batch_host and
 * the search steps share the graph's own scratch: calls of those on different streams must be
 * ordered by the caller.)
 * Errors as pesto_eval_batch_host; create: EINVAL, ESTATE (host-only graph), ENOMEM. */
typedef struct pesto_workspace pesto_workspace;
pesto_status pesto_workspace_create(pesto_graph *g, pesto_workspace **out);
void pesto_workspace_destroy(pesto_workspace *w);                      /* NULL-safe */
pesto_status pesto_eval_batch_host_async(pesto_workspace *w, const int32_t *order,
                                         const void *placements_host, int64_t row_stride_bytes,
                                         int64_t n_cand, int64_t *makespans_host,
                                         void *cuda_stream);

/* ------------------------------------------------------------------------------------------ */
/* Parallel local search (DESIGN.md §4 for the move spec)         */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
    int32_t n_bases;            /* P >= 1 independent incumbents                               */
    const uint8_t *base_x;      /* HOST [P * n_ops] device code per op (must be feasible)      */
    const int32_t *base_order;  /* HOST [P * n_ops] topological orders                          */
    int64_t k_per_base;         /* K: global neighbours per base per step, 1 .. 2^24            */
    int32_t mix[4];             /* FLIP1, FLIPk, WINDOW lane-move weights; SWAP % of groups      */
    uint64_t seed;
    int32_t rank, world;        /* candidate ids of base b split as [floor(rK/W), floor((r+1)K/W)) */
    const uint8_t *nccl_unique_id;  /* 128 bytes (ncclUniqueId) when world > 1, else NULL; with  */
                                    /* NULL and world > 1 the caller reduces keys itself          */
} pesto_search_desc;

/* The search snapshots the graph's comm model (its layouts hold the transfer times): a later
 * pesto_comm_model on the same graph makes pesto_search_eval / _commit / _step /
 * _candidate_keys return PESTO_ESTATE -- create a new search after changing the comm model. */
pesto_status pesto_search_create(pesto_graph *g, const pesto_search_desc *desc,
                                 pesto_search **out);

/* One step: neighbour decode + makespan + CTA argmin (K1) -> ncclAllReduce MIN over ranks
 * (N1, only with an NCCL comm) -> commit (K4) on every rank.  Enqueued on cuda_stream.  When
 * SWAP moves are enabled it synchronises once to learn whether an order changed. */
pesto_status pesto_search_step(pesto_search *s, void *cuda_stream);

/* The three phases of a step, for callers that reduce keys themselves (tests, fake shards). */
pesto_status pesto_search_eval(pesto_search *s, void *cuda_stream);   /* keys = local minima */
pesto_status pesto_search_reduce(pesto_search *s, void *cuda_stream); /* NCCL MIN (no-op w/o) */
pesto_status pesto_search_keys(pesto_search *s, uint64_t *keys_host, void *cuda_stream); /*syncs*/
pesto_status pesto_search_set_keys(pesto_search *s, const uint64_t *keys_host, void *cuda_stream);
pesto_status pesto_search_commit(pesto_search *s, void *cuda_stream); /* K4 + step += 1        */

/* Per-candidate keys (makespan << 24 | j, UINT64_MAX if invalid) of candidates j in [j0, j1)
 * of `base` at the current step, into DEVICE keys_out[j1 - j0] (parity/debug; ignores
 * rank/world).  `kernel` says which kernel computes them:
 *   PESTO_KEYS_TIMED     the instantiation pesto_search_eval launches for this step (same
 *                        kernel, candidates per lane, 32-bit / wide split), each walk storing
 *                        its own key after the argmin epilogue; walks that saturated the 32-bit
 *                        time (makespan field >= 0xF0000000) are re-run by the exact 64-bit
 *                        kernel, so every key is exact.  Synchronises the stream.
 *   PESTO_KEYS_EVAL64    the independent exact 64-bit kernel (eval64) for every candidate.
 *   PESTO_KEYS_TIMED_RAW the timed instantiation's own output, saturated walks left clamped
 *                        (makespan field 0xF0000000).
 * pesto_search_candidate_keys = _ex with PESTO_KEYS_TIMED.  Errors: EINVAL (range outside
 * [0, K], unknown kernel), ESTATE, ECUDA. */
enum { PESTO_KEYS_TIMED = 0, PESTO_KEYS_EVAL64 = 1, PESTO_KEYS_TIMED_RAW = 2 };
pesto_status pesto_search_candidate_keys_ex(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                            uint64_t *keys_out, int32_t kernel, void *cuda_stream);
pesto_status pesto_search_candidate_keys(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                         uint64_t *keys_out, void *cuda_stream);

/* Search spec S9: group moves over merged vertices -- the
 * placement unit of PAPER.md L269 ("all vertices that were merged ... to form v will be placed
 * on GPU-0").  From the next step on, group g != 0 of every base is a coarse group iff
 * draw(128g, 12) mod 100 < pct; its candidate j moves every op of merged vertex
 * draw(j, 10) mod n_coarse whose mask allows device draw(j, 11) mod D to that device, with no
 * order move and no region move.  Other groups decode as before.  All ranks must make the same
 * call before the same step.
 *   coarse_of: HOST [n_ops] merged vertex of each op in [0, n_coarse) (e.g. pesto_coarsen), copied;
 *   n_coarse:  1 .. 255;   pct: 0 .. 100 (0 turns the moves off; coarse_of is then ignored).
 * Synchronises.  Errors: EINVAL; ESTATE when the graph has row-f3 constraints (their local
 * check does not cover a vertex spread over the whole order; constraints set later make the next
 * step fail with ESTATE). */
pesto_status pesto_search_set_coarse_moves(pesto_search *s, const int32_t *coarse_of,
                                          int32_t n_coarse, int32_t pct);

/* Neighbourhood statistics of candidates j in [j0, j1) of `base` at the current step, decoded
 * on the host by the same spec code the kernels use: how many are invalid, how
 * many valid ones are identical to the base (no placement change, no order move; j = 0
 * included) and how many distinct (placement, order) pairs the valid ones form.  Synchronises.
 * Errors: EINVAL. */
typedef struct {
    int64_t candidates, invalid, identical_to_base, distinct;
} pesto_move_stats;
pesto_status pesto_search_move_stats(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                     pesto_move_stats *out);

/* Current incumbent of `base` (synchronises): makespan, x (host [n_ops]) and order. */
pesto_status pesto_search_get(pesto_search *s, int32_t base, int64_t *makespan,
                              uint8_t *x_host, int32_t *order_host);
int64_t pesto_search_step_count(const pesto_search *s);

/* Checkpoint / resume: every draw of the search is a function of (seed, step, base,
 * candidate id) (DESIGN.md §4 S1), so a search is fully described by its incumbents
 * (pesto_search_get), its step counter and its creation parameters (K, mix, seed, rank/world;
 * S9 coarse moves are re-applied by the caller).  To resume, create a search from the saved
 * incumbents with the same parameters and set its step counter: the next step draws exactly the
 * candidates the original would have.  step >= 0; call before the first step of the new
 * search (synchronises).  Errors: EINVAL. */
pesto_status pesto_search_set_step(pesto_search *s, int64_t step);

/* Committed adjacent swaps so far: patched in place on the device (in_place)
 * or handled by a host rebuild of that base's layout (rebuilt).  Either pointer may be NULL.
 * Errors: EINVAL if s is NULL. */
pesto_status pesto_search_swap_stats(const pesto_search *s, int64_t *in_place, int64_t *rebuilt);

/* ncclGetUniqueId through the process's libnccl.so.2 (rank 0 calls it and broadcasts the 128
 * bytes over its own process group).  Errors: ENCCL if NCCL cannot be loaded. */
pesto_status pesto_nccl_unique_id(uint8_t *out128);
void pesto_search_destroy(pesto_search *s);                        /* NULL-safe */

/* Roof microbenchmarks on `device`, best of `reps` CUDA-event-timed runs each:
 * the ceilings K1 is reported against, measured on the box that runs the bench.  Synchronises;
 * ~1 s.  Errors: EINVAL (NULL out, reps < 1), ESTATE (no such device), ECUDA. */
typedef struct {
    double int_ops_per_s;          /* K1's per-op arithmetic c = min(max(r, d) + p, sat) on 8
                                      independent uint32 chains per thread, all SMs full:
                                      algorithmic ops (max, add, saturate) per second          */
    double int_chain_steps_per_s;  /* the same in chain steps (3 ops each) per second           */
    double l2_read_gbs;            /* L2-resident buffer (a quarter of the L2), 128-bit reads   */
    double l2_rmw_gbs;             /* same buffer, 4-byte lanes read + written (K1's cold slots)*/
    int64_t l2_buffer_bytes;
    double hbm_copy_gbs;           /* 1 GiB copy kernel, read + write bytes                     */
} pesto_roofs;
pesto_status pesto_measure_roofs(int32_t device, int32_t reps, pesto_roofs *out);

/* ------------------------------------------------------------------------------------------ */
const char *pesto_last_error(void);       /* thread-local detail of the last failure */
const char *pesto_status_str(pesto_status s);
int32_t pesto_version(void);              /* major*10000 + minor*100 + patch */
/* Number of kernel launches this process has enqueued through libpesto (bench evidence). */
int64_t pesto_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif
