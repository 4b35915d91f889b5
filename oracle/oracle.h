/*
 * oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what the Pesto hot path
 * computes: the makespan of one (placement, schedule) candidate under PAPER.md's
 * problem statement (L142-146 §3.2.1), evaluated the way the paper's simulator does
 * it (L374 §5.4): precedence edges + device orders + a linear comm model per ordered
 * device pair (L138 §3.1) + one FCFS queue per directed link (L144, L188-198 §3.2.2).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load this library.  It shares no code, header, table or helper with the
 * CUDA path (paper_conf_middleware_hafeezsg021_b200/csrc) and never includes it.
 *
 * Conventions (all arrays host memory, caller-owned, indexed by op id / edge index):
 *   n ops, p[n] >= 0 ns; m edges src[e] -> dst[e] with bytes[e] >= 0;
 *   D devices; beta0[a*D+b] ns and beta1[a*D+b] fs/byte for the link a -> b (a != b);
 *   allowed[n] device bitmask (NULL = all D devices); x[n] device per op;
 *   order[n] = pi, the op at each position (a topological order of G).
 * Return values of the makespan functions:
 *   >= 0        the makespan C_max in ns (eq. (3));
 *   INT64_MAX   the placement is infeasible (x_v >= D or not allowed) -- data, not error;
 *   < 0         ORACLE_E* error code for invalid input.
 */
#ifndef PESTO_ORACLE_H
#define PESTO_ORACLE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORACLE_EINVAL    (-1)   /* bad index, negative size, self loop, bad D        */
#define ORACLE_ECYCLE    (-2)   /* G is not a DAG                                     */
#define ORACLE_ENOTTOPO  (-3)   /* order is not a permutation / not topological        */
#define ORACLE_EOVERFLOW (-4)   /* sum p + sum_e max_L t_e >= 2^40, or t_e overflow    */
#define ORACLE_ENOMEM    (-5)

typedef struct {
    int64_t *S, *C;     /* [n] start / completion of each op (by op id)                  */
    int64_t *XS, *XA;   /* [m] transfer start / arrival per edge; -1 if not cross-device  */
} oracle_trace;

/* t = beta0 + ceil(bytes * beta1_fs / 10^6) with a 128-bit product;
 * returns -1 on overflow of int64 or on negative inputs. */
int64_t oracle_transfer_ns(int64_t bytes, int64_t beta0, int64_t beta1_fs);

/* Event-driven simulator (oracle #1, SURVEY §8(c) "Oracle algorithm"). */
int64_t oracle_makespan(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                        const int32_t *dst, const int64_t *bytes, int32_t D,
                        const int64_t *beta0, const int64_t *beta1,
                        const uint8_t *allowed, const uint8_t *x, const int32_t *order,
                        oracle_trace *trace);

/* Longest node-weighted path in the augmented DAG (oracle #2): PAPER.md L152-154 comm
 * vertices + device-sequence arcs + link-sequence arcs (L374 "adds precedence"). */
int64_t oracle_longest_path(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                            const int32_t *dst, const int64_t *bytes, int32_t D,
                            const int64_t *beta0, const int64_t *beta1,
                            const uint8_t *allowed, const uint8_t *x, const int32_t *order);

/* Congestion-free variant: transfers never queue.  f4 row / W2. */
int64_t oracle_makespan_nocongest(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                                  const int32_t *dst, const int64_t *bytes, int32_t D,
                                  const int64_t *beta0, const int64_t *beta1,
                                  const uint8_t *allowed, const uint8_t *x,
                                  const int32_t *order);

/* Row f4 evaluator variants in one entry point (event simulator, oracle #1):
 *   congestion = 1: FCFS link queues (L144, L188-198); 0: congestion-free links (L113, L200);
 *   nondelay   = 0: fixed per-device sequences sigma_d in pi order (reading Q1, L279, L374);
 *                1: non-delay dispatch (row f4(i)): whenever a device is idle it starts, among
 *                   its ops whose inputs have all arrived, the one earliest in pi -- TF's
 *                   per-device ready queue (L90) with pi as the pick priority.
 * oracle_makespan(...) == oracle_makespan_model(..., 1, 0, trace). */
int64_t oracle_makespan_model(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                              const int32_t *dst, const int64_t *bytes, int32_t D,
                              const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                              const uint8_t *x, const int32_t *order, int32_t congestion,
                              int32_t nondelay, oracle_trace *trace);

/* Feasibility constraints, row f3 (PAPER.md L202 memory, L175 colocation).  While set, every
 * makespan / key function of this library treats a placement that violates them as infeasible
 * (INT64_MAX, key UINT64_MAX).  For the graph (n, m, src, dst, bytes, D):
 *   mem  [n] footprint of each op in bytes; NULL: the sum of its input and output tensor sizes
 *        (L202), i.e. the bytes of every edge into or out of the op;
 *   cap  [D] per-device cap on the summed footprint of the ops placed there; NULL: none;
 *   coloc[n] colocation group of each op in [0, n), -1 = none (L175: x equal within a group);
 *        NULL: none.
 * Global state (test infrastructure, not thread-safe against concurrent set/clear); applies
 * only to calls with the same n.  Returns 0 or ORACLE_EINVAL. */
int oracle_set_constraints(int32_t n, int64_t m, const int32_t *src, const int32_t *dst,
                           const int64_t *bytes, int32_t D, const int64_t *mem,
                           const int64_t *cap, const int32_t *coloc);
void oracle_clear_constraints(void);
/* 1 if x satisfies the constraints set (or none are set), else 0. */
int oracle_constraints_ok(int32_t n, const uint8_t *x);

/* Batch: out[c] = oracle_makespan(x + c*n, order) for c < count, `threads` pthreads
 * (threads <= 0: 1).  Returns wall seconds, or a negative error code. */
double oracle_makespan_batch(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                             const int32_t *dst, const int64_t *bytes, int32_t D,
                             const int64_t *beta0, const int64_t *beta1,
                             const uint8_t *allowed, int64_t count, const uint8_t *xs,
                             const int32_t *orders, int32_t per_candidate_order,
                             int32_t threads, int64_t *out);

/* Exhaustive minimum over every placement in allowed^n and every linear extension
 * (oracle #3, the analogue of Thm 3.1's optimality, L204-206).  Tiny graphs only.
 * Writes an optimal (x, order) and the number of schedules enumerated. */
int64_t oracle_bruteforce(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                          const int32_t *dst, const int64_t *bytes, int32_t D,
                          const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                          uint8_t *best_x, int32_t *best_order, int64_t *n_schedules);

/* ----- reference local-search step (the north star's method; spec in DESIGN.md §4) ----- */
uint64_t oracle_mix64(uint64_t z);
uint64_t oracle_draw(uint64_t seed, uint64_t step, int32_t P, int32_t b, int64_t j, int32_t k);

/* Group moves over merged vertices (row f2; DESIGN.md §4 S9): while set, a coarse group of the
 * search (draw(128g, 12) mod 100 < pct, g != 0) moves, per candidate j, every op of merged vertex
 * draw(j, 10) mod n_coarse that allows device draw(j, 11) mod D to that device, and nothing
 * else.  coarse_of [n] in [0, n_coarse), n_coarse <= 255.  Global (test infrastructure); applies
 * to calls with the same n.  Returns 0 or ORACLE_EINVAL. */
int oracle_set_coarse_moves(int32_t n, const int32_t *coarse_of, int32_t n_coarse, int32_t pct);
void oracle_clear_coarse_moves(void);

/* Decode candidate j of base b into (x_out, order_out); returns 1 valid, 0 invalid. */
int oracle_candidate(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, int32_t D,
                     const uint8_t *allowed, int32_t P, int32_t b, const uint8_t *base_x,
                     const int32_t *base_order, int64_t j, uint64_t seed, uint64_t step,
                     const int32_t mix[4], uint8_t *x_out, int32_t *order_out);

/* Keys of candidates j in [j0, j1) of base b: (makespan << 24) | j, UINT64_MAX if invalid. */
int oracle_candidate_keys(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                          const int32_t *dst, const int64_t *bytes, int32_t D,
                          const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                          int32_t P, int32_t b, const uint8_t *base_x, const int32_t *base_order,
                          int64_t j0, int64_t j1, uint64_t seed, uint64_t step,
                          const int32_t mix[4], int32_t threads, uint64_t *keys_out);

/* The same under an evaluator variant (see oracle_makespan_model). */
int oracle_candidate_keys_model(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                                const int32_t *dst, const int64_t *bytes, int32_t D,
                                const int64_t *beta0, const int64_t *beta1,
                                const uint8_t *allowed, int32_t P, int32_t b,
                                const uint8_t *base_x, const int32_t *base_order, int64_t j0,
                                int64_t j1, uint64_t seed, uint64_t step, const int32_t mix[4],
                                int32_t congestion, int32_t nondelay, int32_t threads,
                                uint64_t *keys_out);

/* One full step over P bases (in/out), K neighbours per base, W simulated ranks:
 * per-rank minima over [floor(rK/W), floor((r+1)K/W)) then the min of minima; commit. */
int oracle_search_step(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                       const int32_t *dst, const int64_t *bytes, int32_t D,
                       const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                       int32_t P, uint8_t *base_x, int32_t *base_order, int64_t *base_mk,
                       int64_t K, uint64_t seed, uint64_t step, const int32_t mix[4],
                       int32_t world, int32_t threads, uint64_t *keys);

#ifdef __cplusplus
}
#endif
#endif
