/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).  Plain C11, no CUDA, no code shared
 * with the product.  Written for a reader checking it against PAPER.md by eye, not for speed.
 *
 * Citations: PAPER.md line numbers (Lnnn) with the section; SURVEY.md §8(c) for the readings
 * Q1-Q17 of points the paper leaves open (restated in DESIGN.md §2).
 */
#include "oracle.h"

#include <pthread.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

#define GUARD_2_40 ((int64_t)1 << 40)
#define ORACLE_EINTERNAL (-6)

/* ------------------------------------------------------------------------------------- */
/* comm model: T_comm = beta0 + beta1 * data (§3.1), integerised per Q6.     */
/* ------------------------------------------------------------------------------------- */
int64_t oracle_transfer_ns(int64_t bytes, int64_t beta0, int64_t beta1_fs) {
    if (bytes < 0 || beta0 < 0 || beta1_fs < 0) return -1;
    unsigned __int128 prod = (unsigned __int128)(uint64_t)bytes * (uint64_t)beta1_fs;
    unsigned __int128 q = prod / 1000000u;
    if (prod % 1000000u != 0) q += 1;                       /* ceil */
    unsigned __int128 t = q + (uint64_t)beta0;
    if (t > (unsigned __int128)INT64_MAX) return -1;
    return (int64_t)t;
}

/* ------------------------------------------------------------------------------------- */
/* input validation                                                                       */
/* ------------------------------------------------------------------------------------- */
static int popcount8(unsigned v) {
    int c = 0;
    while (v) { c += (int)(v & 1u); v >>= 1; }
    return c;
}

static int allowed_dev(const uint8_t *allowed, int32_t v, int32_t d) {
    if (allowed == NULL) return 1;
    return (allowed[v] >> d) & 1;
}

/* G must be a DAG (L142 "We represent the DNN model as a DAG").  Kahn's algorithm. */
static int64_t check_graph(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                           const int32_t *dst, const int64_t *bytes, int32_t D,
                           const int64_t *beta0, const int64_t *beta1) {
    if (n < 1 || m < 0 || D < 1 || D > 8) return ORACLE_EINVAL;
    for (int32_t v = 0; v < n; v++)
        if (p[v] < 0) return ORACLE_EINVAL;
    for (int32_t a = 0; a < D; a++)
        for (int32_t b = 0; b < D; b++)
            if (a != b && (beta0[a * D + b] < 0 || beta1[a * D + b] < 0)) return ORACLE_EINVAL;
    for (int64_t e = 0; e < m; e++) {
        if (src[e] < 0 || src[e] >= n || dst[e] < 0 || dst[e] >= n) return ORACLE_EINVAL;
        if (src[e] == dst[e] || bytes[e] < 0) return ORACLE_EINVAL;
    }
    /* overflow guard: every makespan is a longest path over
       distinct op and transfer weights, so it is at most sum p + sum_e max_L t_e. */
    int64_t total = 0;
    for (int32_t v = 0; v < n; v++) {
        total += p[v];
        if (total >= GUARD_2_40) return ORACLE_EOVERFLOW;
    }
    for (int64_t e = 0; e < m; e++) {
        int64_t worst = 0;
        for (int32_t a = 0; a < D; a++)
            for (int32_t b = 0; b < D; b++) {
                if (a == b) continue;
                int64_t t = oracle_transfer_ns(bytes[e], beta0[a * D + b], beta1[a * D + b]);
                if (t < 0) return ORACLE_EOVERFLOW;
                if (t > worst) worst = t;
            }
        if (worst >= GUARD_2_40) return ORACLE_EOVERFLOW;
        total += worst;
        if (total >= GUARD_2_40) return ORACLE_EOVERFLOW;
    }
    int32_t *indeg = calloc((size_t)n, sizeof(int32_t));
    int32_t *queue = malloc((size_t)n * sizeof(int32_t));
    if (!indeg || !queue) { free(indeg); free(queue); return ORACLE_ENOMEM; }
    for (int64_t e = 0; e < m; e++) indeg[dst[e]]++;
    int32_t head = 0, tail = 0;
    for (int32_t v = 0; v < n; v++)
        if (indeg[v] == 0) queue[tail++] = v;
    /* Kahn: pop a source, delete its out-edges (per-call CSR of out-edges) */
    int64_t *off = calloc((size_t)n + 1, sizeof(int64_t));
    int64_t *adj = malloc((size_t)(m > 0 ? m : 1) * sizeof(int64_t));
    if (!off || !adj) { free(indeg); free(queue); free(off); free(adj); return ORACLE_ENOMEM; }
    for (int64_t e = 0; e < m; e++) off[src[e] + 1]++;
    for (int32_t v = 0; v < n; v++) off[v + 1] += off[v];
    int64_t *fill = malloc((size_t)n * sizeof(int64_t));
    if (!fill) { free(indeg); free(queue); free(off); free(adj); return ORACLE_ENOMEM; }
    for (int32_t v = 0; v < n; v++) fill[v] = off[v];
    for (int64_t e = 0; e < m; e++) adj[fill[src[e]]++] = e;
    while (head < tail) {
        int32_t v = queue[head++];
        for (int64_t i = off[v]; i < off[v + 1]; i++) {
            int32_t w = dst[adj[i]];
            if (--indeg[w] == 0) queue[tail++] = w;
        }
    }
    free(indeg); free(queue); free(off); free(adj); free(fill);
    return tail == n ? 0 : ORACLE_ECYCLE;
}

/* order must be a permutation of the ops and a linear extension of G. */
static int64_t check_order(int32_t n, int64_t m, const int32_t *src, const int32_t *dst,
                           const int32_t *order, int32_t *pos) {
    for (int32_t v = 0; v < n; v++) pos[v] = -1;
    for (int32_t k = 0; k < n; k++) {
        int32_t v = order[k];
        if (v < 0 || v >= n || pos[v] != -1) return ORACLE_ENOTTOPO;
        pos[v] = k;
    }
    for (int64_t e = 0; e < m; e++)
        if (pos[src[e]] >= pos[dst[e]]) return ORACLE_ENOTTOPO;
    return 0;
}

/* a placement is feasible iff every op sits on an existing device its mask allows (Q16) */
/* ------------------------------------------------------------------------------------- */
/* row f3: memory footprint per device (L202) and colocation groups (L175)                 */
/* ------------------------------------------------------------------------------------- */
static struct {
    int active;
    int32_t n, D;
    int64_t *mem;        /* [n] footprint of each op */
    int64_t *cap;        /* [D] or NULL */
    int32_t *coloc;      /* [n] or NULL */
} g_cons;

void oracle_clear_constraints(void) {
    free(g_cons.mem);
    free(g_cons.cap);
    free(g_cons.coloc);
    memset(&g_cons, 0, sizeof g_cons);
}

int oracle_set_constraints(int32_t n, int64_t m, const int32_t *src, const int32_t *dst,
                           const int64_t *bytes, int32_t D, const int64_t *mem,
                           const int64_t *cap, const int32_t *coloc) {
    oracle_clear_constraints();
    if (n < 1 || m < 0 || D < 1 || D > 8) return ORACLE_EINVAL;
    g_cons.mem = calloc((size_t)n, sizeof(int64_t));
    if (!g_cons.mem) return ORACLE_ENOMEM;
    if (mem) {
        for (int32_t v = 0; v < n; v++) {
            if (mem[v] < 0) { oracle_clear_constraints(); return ORACLE_EINVAL; }
            g_cons.mem[v] = mem[v];
        }
    } else {                                 /* L202: input + output tensor sizes of the op */
        for (int64_t e = 0; e < m; e++) {
            g_cons.mem[src[e]] += bytes[e];
            g_cons.mem[dst[e]] += bytes[e];
        }
    }
    if (cap) {
        g_cons.cap = malloc((size_t)D * sizeof(int64_t));
        for (int32_t d = 0; d < D; d++) g_cons.cap[d] = cap[d];
    }
    if (coloc) {
        g_cons.coloc = malloc((size_t)n * sizeof(int32_t));
        for (int32_t v = 0; v < n; v++) {
            if (coloc[v] < -1 || coloc[v] >= n) { oracle_clear_constraints(); return ORACLE_EINVAL; }
            g_cons.coloc[v] = coloc[v];
        }
    }
    g_cons.n = n;
    g_cons.D = D;
    g_cons.active = 1;
    return 0;
}

int oracle_constraints_ok(int32_t n, const uint8_t *x) {
    if (!g_cons.active || n != g_cons.n) return 1;
    if (g_cons.cap) {                        /* footprint of the ops on each device <= cap */
        int64_t F[8] = {0};
        for (int32_t v = 0; v < n; v++) F[x[v]] += g_cons.mem[v];
        for (int32_t d = 0; d < g_cons.D; d++)
            if (F[d] > g_cons.cap[d]) return 0;
    }
    if (g_cons.coloc) {                      /* every op of a group on one device */
        int32_t *dev = malloc((size_t)n * sizeof(int32_t));
        int ok = 1;
        for (int32_t v = 0; v < n; v++) dev[v] = -1;
        for (int32_t v = 0; v < n && ok; v++) {
            const int32_t grp = g_cons.coloc[v];
            if (grp < 0) continue;
            if (dev[grp] < 0) dev[grp] = x[v];
            else if (dev[grp] != x[v]) ok = 0;
        }
        free(dev);
        if (!ok) return 0;
    }
    return 1;
}

static int feasible(int32_t n, int32_t D, const uint8_t *allowed, const uint8_t *x) {
    for (int32_t v = 0; v < n; v++) {
        if (x[v] >= D) return 0;
        if (!allowed_dev(allowed, v, x[v])) return 0;
    }
    return oracle_constraints_ok(n, x);
}

/* ------------------------------------------------------------------------------------- */
/* a binary min-heap of 4-tuples (lexicographic), used for events and link queues          */
/* ------------------------------------------------------------------------------------- */
typedef struct { int64_t k[4]; } hkey;
typedef struct { hkey *a; int64_t len, cap; } heap;

static int hless(const hkey *x, const hkey *y) {
    for (int i = 0; i < 4; i++)
        if (x->k[i] != y->k[i]) return x->k[i] < y->k[i];
    return 0;
}

static int hpush(heap *h, hkey v) {
    if (h->len == h->cap) {
        int64_t nc = h->cap ? 2 * h->cap : 16;
        hkey *na = realloc(h->a, (size_t)nc * sizeof(hkey));
        if (!na) return -1;
        h->a = na;
        h->cap = nc;
    }
    int64_t i = h->len++;
    h->a[i] = v;
    while (i > 0) {
        int64_t parent = (i - 1) / 2;
        if (!hless(&h->a[i], &h->a[parent])) break;
        hkey t = h->a[i]; h->a[i] = h->a[parent]; h->a[parent] = t;
        i = parent;
    }
    return 0;
}

static hkey hpop(heap *h) {
    hkey top = h->a[0];
    h->a[0] = h->a[--h->len];
    int64_t i = 0;
    for (;;) {
        int64_t l = 2 * i + 1, r = l + 1, s = i;
        if (l < h->len && hless(&h->a[l], &h->a[s])) s = l;
        if (r < h->len && hless(&h->a[r], &h->a[s])) s = r;
        if (s == i) break;
        hkey t = h->a[i]; h->a[i] = h->a[s]; h->a[s] = t;
        i = s;
    }
    return top;
}

/* ------------------------------------------------------------------------------------- */
/* oracle #1: event-driven simulation (§5.4)         */
/* ------------------------------------------------------------------------------------- */
enum { EV_OP_DONE = 0, EV_XFER_DONE = 1 };

static int64_t simulate(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                        const int32_t *dst, const int64_t *bytes, int32_t D,
                        const int64_t *beta0, const int64_t *beta1, const uint8_t *x,
                        const int32_t *order, const int32_t *pos, int congestion,
                        int nondelay, oracle_trace *trace) {
    int64_t ret = 0;
    int32_t L = D * D;
    /* out-edge lists (by producer) */
    int64_t *off = calloc((size_t)n + 1, sizeof(int64_t));
    int64_t *adj = malloc((size_t)(m > 0 ? m : 1) * sizeof(int64_t));
    int64_t *fill = malloc((size_t)n * sizeof(int64_t));
    int64_t *tx = malloc((size_t)(m > 0 ? m : 1) * sizeof(int64_t));
    int32_t *pending = calloc((size_t)n, sizeof(int32_t));
    int32_t *seq = malloc((size_t)n * sizeof(int32_t));     /* sigma_d, concatenated */
    int32_t *seq_off = calloc((size_t)D + 1, sizeof(int32_t));
    int32_t *head = calloc((size_t)D, sizeof(int32_t));
    int *dbusy = calloc((size_t)D, sizeof(int));
    int *lbusy = calloc((size_t)L, sizeof(int));
    int64_t *S = malloc((size_t)n * sizeof(int64_t));
    int64_t *C = malloc((size_t)n * sizeof(int64_t));
    heap ev = {0}, *lq = calloc((size_t)L, sizeof(heap));
    if (!off || !adj || !fill || !tx || !pending || !seq || !seq_off || !head || !dbusy ||
        !lbusy || !S || !C || !lq) { ret = ORACLE_ENOMEM; goto out; }

    for (int64_t e = 0; e < m; e++) off[src[e] + 1]++;
    for (int32_t v = 0; v < n; v++) off[v + 1] += off[v];
    for (int32_t v = 0; v < n; v++) fill[v] = off[v];
    for (int64_t e = 0; e < m; e++) adj[fill[src[e]]++] = e;

    /* transfer only when producer and consumer sit on different devices
       (L144 "if the operations are placed on the same device, the transfer time is
       negligible and is ignored"; eq. (5)-(6), L164-165) */
    for (int64_t e = 0; e < m; e++) {
        int32_t a = x[src[e]], b = x[dst[e]];
        tx[e] = (a == b) ? -1 : oracle_transfer_ns(bytes[e], beta0[a * D + b], beta1[a * D + b]);
        pending[dst[e]]++;
    }
    /* device sequences sigma_d = ops placed on d, in pi order (schedule = per-device order,
       L279 control dependencies, L374 precedence; reading Q1) */
    for (int32_t k = 0; k < n; k++) seq_off[x[order[k]] + 1]++;
    for (int32_t d = 0; d < D; d++) seq_off[d + 1] += seq_off[d];
    for (int32_t d = 0; d < D; d++) head[d] = seq_off[d];
    {
        int32_t *f2 = malloc((size_t)D * sizeof(int32_t));
        if (!f2) { ret = ORACLE_ENOMEM; goto out; }
        for (int32_t d = 0; d < D; d++) f2[d] = seq_off[d];
        for (int32_t k = 0; k < n; k++) seq[f2[x[order[k]]]++] = order[k];
        free(f2);
    }
    for (int32_t v = 0; v < n; v++) { S[v] = -1; C[v] = -1; }
    if (trace) for (int64_t e = 0; e < m; e++) { trace->XS[e] = -1; trace->XA[e] = -1; }

    int64_t now = 0, done = 0;
    for (;;) {
        /* start everything that can start at `now`, to a fixpoint (step 6) */
        int progress = 1;
        while (progress) {
            progress = 0;
            /* links: one transfer at a time per ordered device pair, FCFS (L144, L188-198) */
            for (int32_t l = 0; l < L; l++) {
                if (lbusy[l] || lq[l].len == 0) continue;
                hkey it = hpop(&lq[l]);
                int64_t e = it.k[3];
                if (trace) { trace->XS[e] = now; trace->XA[e] = now + tx[e]; }
                lbusy[l] = 1;
                hkey evk = {{now + tx[e], EV_XFER_DONE, e, 0}};
                if (hpush(&ev, evk)) { ret = ORACLE_ENOMEM; goto out; }
                progress = 1;
            }
            /* devices: no pre-emption, one op at a time (L146).  Fixed sequences (reading
               Q1): the next op of sigma_d only, once its inputs are in.  Non-delay dispatch
               (row f4(i), L90 "for each device, TensorFlow ... picks an operation from the
               ready queue", with pi as the pick priority): the first op of sigma_d, in pi
               order, that has not started and whose inputs are all in. */
            for (int32_t d = 0; d < D; d++) {
                if (dbusy[d] || head[d] >= seq_off[d + 1]) continue;
                int32_t v = -1;
                if (!nondelay) {
                    if (pending[seq[head[d]]] == 0) v = seq[head[d]];
                } else {
                    while (head[d] < seq_off[d + 1] && S[seq[head[d]]] >= 0) head[d]++;
                    for (int32_t i = head[d]; i < seq_off[d + 1]; i++) {
                        int32_t u = seq[i];
                        if (S[u] < 0 && pending[u] == 0) { v = u; break; }
                    }
                }
                if (v < 0) continue;
                S[v] = now;
                C[v] = now + p[v];
                if (!nondelay) head[d]++;
                dbusy[d] = 1;
                hkey evk = {{C[v], EV_OP_DONE, v, 0}};
                if (hpush(&ev, evk)) { ret = ORACLE_ENOMEM; goto out; }
                progress = 1;
            }
        }
        if (ev.len == 0) break;
        /* pop every event at the minimum time (step 5) */
        now = ev.a[0].k[0];
        while (ev.len > 0 && ev.a[0].k[0] == now) {
            hkey it = hpop(&ev);
            if (it.k[1] == EV_OP_DONE) {
                int32_t u = (int32_t)it.k[2];
                dbusy[x[u]] = 0;
                done++;
                for (int64_t i = off[u]; i < off[u + 1]; i++) {
                    int64_t e = adj[i];
                    int32_t v = dst[e];
                    if (tx[e] < 0) {
                        pending[v]--;                       /* same device: C_u suffices */
                    } else if (!congestion) {
                        if (trace) { trace->XS[e] = now; trace->XA[e] = now + tx[e]; }
                        hkey evk = {{now + tx[e], EV_XFER_DONE, e, 0}};
                        if (hpush(&ev, evk)) { ret = ORACLE_ENOMEM; goto out; }
                    } else {
                        /* FCFS key (release, pos u, pos v, e): reading Q3 */
                        int32_t l = x[u] * D + x[v];
                        hkey q = {{now, pos[u], pos[v], e}};
                        if (hpush(&lq[l], q)) { ret = ORACLE_ENOMEM; goto out; }
                    }
                }
            } else {
                int64_t e = it.k[2];
                if (congestion) lbusy[x[src[e]] * D + x[dst[e]]] = 0;
                pending[dst[e]]--;
            }
        }
    }
    if (done != n) { ret = ORACLE_EINTERNAL; goto out; }
    /* C_max = max_i C_i (L159-162 eq. (3); makespan definition) */
    for (int32_t v = 0; v < n; v++)
        if (C[v] > ret) ret = C[v];
    if (trace) {
        memcpy(trace->S, S, (size_t)n * sizeof(int64_t));
        memcpy(trace->C, C, (size_t)n * sizeof(int64_t));
    }
out:
    free(off); free(adj); free(fill); free(tx); free(pending); free(seq); free(seq_off);
    free(head); free(dbusy); free(lbusy); free(S); free(C); free(ev.a);
    if (lq) { for (int32_t l = 0; l < L; l++) free(lq[l].a); free(lq); }
    return ret;
}

static int64_t makespan_common(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                               const int32_t *dst, const int64_t *bytes, int32_t D,
                               const int64_t *beta0, const int64_t *beta1,
                               const uint8_t *allowed, const uint8_t *x, const int32_t *order,
                               int congestion, int nondelay, oracle_trace *trace) {
    int64_t rc = check_graph(n, p, m, src, dst, bytes, D, beta0, beta1);
    if (rc) return rc;
    int32_t *pos = malloc((size_t)n * sizeof(int32_t));
    if (!pos) return ORACLE_ENOMEM;
    rc = check_order(n, m, src, dst, order, pos);
    if (rc == 0) {
        if (!feasible(n, D, allowed, x)) rc = INT64_MAX;
        else rc = simulate(n, p, m, src, dst, bytes, D, beta0, beta1, x, order, pos,
                           congestion, nondelay, trace);
    }
    free(pos);
    return rc;
}

int64_t oracle_makespan(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                        const int32_t *dst, const int64_t *bytes, int32_t D,
                        const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                        const uint8_t *x, const int32_t *order, oracle_trace *trace) {
    return makespan_common(n, p, m, src, dst, bytes, D, beta0, beta1, allowed, x, order, 1, 0,
                           trace);
}

int64_t oracle_makespan_nocongest(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                                  const int32_t *dst, const int64_t *bytes, int32_t D,
                                  const int64_t *beta0, const int64_t *beta1,
                                  const uint8_t *allowed, const uint8_t *x,
                                  const int32_t *order) {
    return makespan_common(n, p, m, src, dst, bytes, D, beta0, beta1, allowed, x, order, 0, 0,
                           NULL);
}

int64_t oracle_makespan_model(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                              const int32_t *dst, const int64_t *bytes, int32_t D,
                              const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                              const uint8_t *x, const int32_t *order, int32_t congestion,
                              int32_t nondelay, oracle_trace *trace) {
    return makespan_common(n, p, m, src, dst, bytes, D, beta0, beta1, allowed, x, order,
                           congestion != 0, nondelay != 0, trace);
}

/* ------------------------------------------------------------------------------------- */
/* oracle #2: longest path in the augmented disjunctive DAG                                */
/*   vertices: ops (weight p_i) and one comm vertex per edge (L152-154, weight z_k p_k,     */
/*   eq. (6)); arcs: (i,k),(k,j) per edge; consecutive ops of sigma_d; consecutive comm     */
/*   vertices of each directed link, in FCFS order (pos u, pos v, e) -- Q3 / Lemma 1.      */
/* ------------------------------------------------------------------------------------- */
typedef struct { const int32_t *pos; const int32_t *src; const int32_t *dst; } lk_ctx;

static int lk_less(const lk_ctx *c, int64_t a, int64_t b) {
    int32_t pa = c->pos[c->src[a]], pb = c->pos[c->src[b]];
    if (pa != pb) return pa < pb;
    pa = c->pos[c->dst[a]]; pb = c->pos[c->dst[b]];
    if (pa != pb) return pa < pb;
    return a < b;
}

static void lk_sort(const lk_ctx *c, int64_t *v, int64_t *tmp, int64_t len) {  /* merge sort */
    if (len < 2) return;
    int64_t h = len / 2;
    lk_sort(c, v, tmp, h);
    lk_sort(c, v + h, tmp, len - h);
    int64_t i = 0, j = h, k = 0;
    while (i < h && j < len) tmp[k++] = lk_less(c, v[j], v[i]) ? v[j++] : v[i++];
    while (i < h) tmp[k++] = v[i++];
    while (j < len) tmp[k++] = v[j++];
    memcpy(v, tmp, (size_t)len * sizeof(int64_t));
}

int64_t oracle_longest_path(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                            const int32_t *dst, const int64_t *bytes, int32_t D,
                            const int64_t *beta0, const int64_t *beta1,
                            const uint8_t *allowed, const uint8_t *x, const int32_t *order) {
    int64_t rc = check_graph(n, p, m, src, dst, bytes, D, beta0, beta1);
    if (rc) return rc;
    int32_t *pos = malloc((size_t)n * sizeof(int32_t));
    if (!pos) return ORACLE_ENOMEM;
    rc = check_order(n, m, src, dst, order, pos);
    if (rc) { free(pos); return rc; }
    if (!feasible(n, D, allowed, x)) { free(pos); return INT64_MAX; }

    int64_t V = (int64_t)n + m;
    int64_t A_cap = 2 * m + n + m + 1;               /* arcs: 2 per edge + sigma + tau */
    int64_t *as = malloc((size_t)A_cap * sizeof(int64_t));
    int64_t *ad = malloc((size_t)A_cap * sizeof(int64_t));
    int64_t *w = malloc((size_t)V * sizeof(int64_t));
    int64_t *cross = malloc((size_t)(m > 0 ? m : 1) * sizeof(int64_t));
    int64_t *tmp = malloc((size_t)(m > 0 ? m : 1) * sizeof(int64_t));
    int32_t *last_on_dev = malloc((size_t)D * sizeof(int32_t));
    if (!as || !ad || !w || !cross || !tmp || !last_on_dev) { rc = ORACLE_ENOMEM; goto out2; }
    int64_t na = 0;
    for (int32_t v = 0; v < n; v++) w[v] = p[v];
    for (int64_t e = 0; e < m; e++) {
        int32_t a = x[src[e]], b = x[dst[e]];
        w[n + e] = (a == b) ? 0 : oracle_transfer_ns(bytes[e], beta0[a * D + b], beta1[a * D + b]);
        as[na] = src[e]; ad[na++] = n + e;
        as[na] = n + e;  ad[na++] = dst[e];
    }
    for (int32_t d = 0; d < D; d++) last_on_dev[d] = -1;
    for (int32_t k = 0; k < n; k++) {
        int32_t v = order[k], d = x[v];
        if (last_on_dev[d] >= 0) { as[na] = last_on_dev[d]; ad[na++] = v; }
        last_on_dev[d] = v;
    }
    lk_ctx ctx = {pos, src, dst};
    for (int32_t a = 0; a < D; a++)
        for (int32_t b = 0; b < D; b++) {
            if (a == b) continue;
            int64_t c = 0;
            for (int64_t e = 0; e < m; e++)
                if (x[src[e]] == a && x[dst[e]] == b) cross[c++] = e;
            lk_sort(&ctx, cross, tmp, c);
            for (int64_t i = 1; i < c; i++) { as[na] = n + cross[i - 1]; ad[na++] = n + cross[i]; }
        }
    /* Kahn over the augmented graph, finish(k) = max_pred finish + w(k) */
    {
        int64_t *indeg = calloc((size_t)V, sizeof(int64_t));
        int64_t *off = calloc((size_t)V + 1, sizeof(int64_t));
        int64_t *adj = malloc((size_t)(na > 0 ? na : 1) * sizeof(int64_t));
        int64_t *fill = malloc((size_t)V * sizeof(int64_t));
        int64_t *fin = calloc((size_t)V, sizeof(int64_t));
        int64_t *start = calloc((size_t)V, sizeof(int64_t));
        int64_t *queue = malloc((size_t)V * sizeof(int64_t));
        if (!indeg || !off || !adj || !fill || !fin || !start || !queue) rc = ORACLE_ENOMEM;
        else {
            for (int64_t i = 0; i < na; i++) { indeg[ad[i]]++; off[as[i] + 1]++; }
            for (int64_t v = 0; v < V; v++) off[v + 1] += off[v];
            for (int64_t v = 0; v < V; v++) fill[v] = off[v];
            for (int64_t i = 0; i < na; i++) adj[fill[as[i]]++] = ad[i];
            int64_t hd = 0, tl = 0;
            for (int64_t v = 0; v < V; v++) if (indeg[v] == 0) queue[tl++] = v;
            while (hd < tl) {
                int64_t v = queue[hd++];
                fin[v] = start[v] + w[v];
                for (int64_t i = off[v]; i < off[v + 1]; i++) {
                    int64_t u = adj[i];
                    if (fin[v] > start[u]) start[u] = fin[v];
                    if (--indeg[u] == 0) queue[tl++] = u;
                }
            }
            if (tl != V) rc = ORACLE_EINTERNAL;
            else {
                rc = 0;
                for (int32_t v = 0; v < n; v++) if (fin[v] > rc) rc = fin[v];
            }
        }
        free(indeg); free(off); free(adj); free(fill); free(fin); free(start); free(queue);
    }
out2:
    free(pos); free(as); free(ad); free(w); free(cross); free(tmp); free(last_on_dev);
    return rc;
}

/* ------------------------------------------------------------------------------------- */
/* batch evaluation on a pthread pool (used for the CPU baseline and for parity tests)     */
/* ------------------------------------------------------------------------------------- */
typedef struct {
    int32_t n; const int64_t *p; int64_t m; const int32_t *src, *dst; const int64_t *bytes;
    int32_t D; const int64_t *beta0, *beta1; const uint8_t *allowed;
    const uint8_t *xs; const int32_t *orders; int32_t per_cand_order;
    int64_t begin, end; int64_t *out;
} batch_job;

static void *batch_worker(void *arg) {
    batch_job *j = (batch_job *)arg;
    for (int64_t c = j->begin; c < j->end; c++) {
        const int32_t *ord = j->orders + (j->per_cand_order ? c * j->n : 0);
        j->out[c] = oracle_makespan(j->n, j->p, j->m, j->src, j->dst, j->bytes, j->D, j->beta0,
                                    j->beta1, j->allowed, j->xs + c * j->n, ord, NULL);
    }
    return NULL;
}

static double now_s(void) {
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (double)ts.tv_sec + 1e-9 * (double)ts.tv_nsec;
}

double oracle_makespan_batch(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                             const int32_t *dst, const int64_t *bytes, int32_t D,
                             const int64_t *beta0, const int64_t *beta1,
                             const uint8_t *allowed, int64_t count, const uint8_t *xs,
                             const int32_t *orders, int32_t per_candidate_order,
                             int32_t threads, int64_t *out) {
    if (threads <= 0) threads = 1;
    if (threads > count && count > 0) threads = (int32_t)count;
    pthread_t *th = malloc((size_t)threads * sizeof(pthread_t));
    batch_job *jobs = malloc((size_t)threads * sizeof(batch_job));
    if (!th || !jobs) { free(th); free(jobs); return ORACLE_ENOMEM; }
    double t0 = now_s();
    for (int32_t t = 0; t < threads; t++) {
        batch_job j = {n, p, m, src, dst, bytes, D, beta0, beta1, allowed, xs, orders,
                       per_candidate_order, count * t / threads, count * (t + 1) / threads, out};
        jobs[t] = j;
        pthread_create(&th[t], NULL, batch_worker, &jobs[t]);
    }
    for (int32_t t = 0; t < threads; t++) pthread_join(th[t], NULL);
    double dt = now_s() - t0;
    free(th); free(jobs);
    return dt;
}

/* ------------------------------------------------------------------------------------- */
/* oracle #3: brute force over allowed^n x linear extensions (tiny graphs)                  */
/* ------------------------------------------------------------------------------------- */
typedef struct {
    int32_t n; const int64_t *p; int64_t m; const int32_t *src, *dst; const int64_t *bytes;
    int32_t D; const int64_t *beta0, *beta1; const uint8_t *allowed;
    int32_t *order, *pos, *placed, *npred_left;
    uint8_t *x; uint8_t *best_x; int32_t *best_order; int64_t best, count;
} bf_ctx;

static void bf_all_placements(bf_ctx *c) {
    int32_t n = c->n;
    for (int32_t v = 0; v < n; v++) {           /* first allowed device of every op */
        c->x[v] = 0;
        while (!allowed_dev(c->allowed, v, c->x[v])) c->x[v]++;
    }
    for (;;) {
        int64_t mk = simulate(n, c->p, c->m, c->src, c->dst, c->bytes, c->D, c->beta0,
                              c->beta1, c->x, c->order, c->pos, 1, 0, NULL);
        c->count++;
        if (mk < c->best) {
            c->best = mk;
            memcpy(c->best_x, c->x, (size_t)n);
            memcpy(c->best_order, c->order, (size_t)n * sizeof(int32_t));
        }
        /* odometer over allowed devices */
        int32_t v = 0;
        for (; v < n; v++) {
            int32_t d = c->x[v] + 1;
            while (d < c->D && !allowed_dev(c->allowed, v, d)) d++;
            if (d < c->D) { c->x[v] = (uint8_t)d; break; }
            d = 0;
            while (!allowed_dev(c->allowed, v, d)) d++;
            c->x[v] = (uint8_t)d;
        }
        if (v == n) return;
    }
}

static void bf_orders(bf_ctx *c, int32_t k) {
    if (k == c->n) { bf_all_placements(c); return; }
    for (int32_t v = 0; v < c->n; v++) {
        if (c->placed[v] || c->npred_left[v] != 0) continue;
        c->placed[v] = 1;
        c->order[k] = v;
        c->pos[v] = k;
        for (int64_t e = 0; e < c->m; e++) if (c->src[e] == v) c->npred_left[c->dst[e]]--;
        bf_orders(c, k + 1);
        for (int64_t e = 0; e < c->m; e++) if (c->src[e] == v) c->npred_left[c->dst[e]]++;
        c->placed[v] = 0;
    }
}

int64_t oracle_bruteforce(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                          const int32_t *dst, const int64_t *bytes, int32_t D,
                          const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                          uint8_t *best_x, int32_t *best_order, int64_t *n_schedules) {
    int64_t rc = check_graph(n, p, m, src, dst, bytes, D, beta0, beta1);
    if (rc) return rc;
    for (int32_t v = 0; v < n; v++)
        if (allowed && (allowed[v] & ((1u << D) - 1u)) == 0) return INT64_MAX;
    bf_ctx c = {n, p, m, src, dst, bytes, D, beta0, beta1, allowed,
                calloc((size_t)n, 4), calloc((size_t)n, 4), calloc((size_t)n, 4),
                calloc((size_t)n, 4), calloc((size_t)n, 1), best_x, best_order, INT64_MAX, 0};
    for (int64_t e = 0; e < m; e++) c.npred_left[dst[e]]++;
    bf_orders(&c, 0);
    free(c.order); free(c.pos); free(c.placed); free(c.npred_left); free(c.x);
    if (n_schedules) *n_schedules = c.count;
    return c.best;
}

/* ------------------------------------------------------------------------------------- */
/* reference search step.  Restates DESIGN.md §4 (the north star's local search; not a     */
/* paper method) with no code shared with the CUDA path.                                   */
/* ------------------------------------------------------------------------------------- */
uint64_t oracle_mix64(uint64_t z) {          /* SplitMix64 finaliser */
    z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27; z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

uint64_t oracle_draw(uint64_t seed, uint64_t step, int32_t P, int32_t b, int64_t j, int32_t k) {
    uint64_t ctr = ((step * (uint64_t)P + (uint64_t)b) * (1ull << 24) + (uint64_t)j) * 16ull
                   + (uint64_t)k;
    return oracle_mix64(seed ^ oracle_mix64(ctr));
}

/* devices op v may move to from device `cur`, ascending (the set A_i of DESIGN §4) */
static int32_t alt_devices(const uint8_t *allowed, int32_t D, int32_t v, int32_t cur,
                           int32_t *out) {
    int32_t c = 0;
    for (int32_t d = 0; d < D; d++)
        if (d != cur && allowed_dev(allowed, v, d)) out[c++] = d;
    return c;
}

/* group moves over merged vertices (row f2, DESIGN §4 S9): global, test infrastructure */
static struct {
    int active;
    int32_t n, n_coarse, pct;
    int32_t *coarse_of;
} g_coarse;

void oracle_clear_coarse_moves(void) {
    free(g_coarse.coarse_of);
    memset(&g_coarse, 0, sizeof g_coarse);
}

int oracle_set_coarse_moves(int32_t n, const int32_t *coarse_of, int32_t n_coarse, int32_t pct) {
    oracle_clear_coarse_moves();
    if (n < 1 || n_coarse < 1 || n_coarse > 255 || pct < 0 || pct > 100 || !coarse_of)
        return ORACLE_EINVAL;
    g_coarse.coarse_of = malloc((size_t)n * sizeof(int32_t));
    if (!g_coarse.coarse_of) return ORACLE_ENOMEM;
    for (int32_t v = 0; v < n; v++) {
        if (coarse_of[v] < 0 || coarse_of[v] >= n_coarse) { oracle_clear_coarse_moves(); return ORACLE_EINVAL; }
        g_coarse.coarse_of[v] = coarse_of[v];
    }
    g_coarse.n = n;
    g_coarse.n_coarse = n_coarse;
    g_coarse.pct = pct;
    g_coarse.active = 1;
    return 0;
}

int oracle_candidate(int32_t n, int64_t m, const int32_t *src, const int32_t *dst, int32_t D,
                     const uint8_t *allowed, int32_t P, int32_t b, const uint8_t *base_x,
                     const int32_t *base_order, int64_t j, uint64_t seed, uint64_t step,
                     const int32_t mix[4], uint8_t *x_out, int32_t *order_out) {
    const uint8_t *bx = base_x + (int64_t)b * n;
    const int32_t *bo = base_order + (int64_t)b * n;
    memcpy(x_out, bx, (size_t)n);
    memcpy(order_out, bo, (size_t)n * sizeof(int32_t));
    int64_t g = j >> 7, lane = j & 127;      /* groups of 128 candidate ids (DESIGN §4 S2) */
    /* S9: a coarse group moves one merged vertex per candidate and nothing else: vertex
       k = draw(j, 10) mod n_coarse goes to device d = draw(j, 11) mod D (each of its ops whose
       mask allows d); no order move, no region moves */
    if (g_coarse.active && g_coarse.n == n && g != 0 && g_coarse.pct > 0 &&
        (int64_t)(oracle_draw(seed, step, P, b, 128 * g, 12) % 100u) < g_coarse.pct) {
        int32_t k = (int32_t)(oracle_draw(seed, step, P, b, j, 10) % (uint64_t)g_coarse.n_coarse);
        int32_t d = (int32_t)(oracle_draw(seed, step, P, b, j, 11) % (uint64_t)D);
        for (int32_t v = 0; v < n; v++)
            if (g_coarse.coarse_of[v] == k && allowed_dev(allowed, v, d)) x_out[v] = (uint8_t)d;
        return 1;
    }
    int swap = 0;
    /* S2 (v6): the regions tile the base order, R = ceil(n/64), rotated by o = draw(0, 13)
       mod R; group g takes region (g + o) mod R = positions [c, c + len), in pass g / R */
    int64_t R = ((int64_t)n + 63) / 64;
    int64_t rot = (int64_t)(oracle_draw(seed, step, P, b, 0, 13) % (uint64_t)R);
    int64_t c0 = 64 * ((g + rot) % R);
    int64_t rlen = n - c0 < 64 ? n - c0 : 64;
    int64_t pass = g / R;
    /* S3: order move, one adjacent swap per group */
    if (g != 0 && mix[3] > 0 && n >= 2) {
        uint64_t u = oracle_draw(seed, step, P, b, 128 * g, 15);
        if ((int64_t)(u % 100u) < mix[3]) {
            int64_t k = c0 + (int64_t)(oracle_draw(seed, step, P, b, 128 * g, 14) % (uint64_t)rlen);
            if (k > n - 2) k = n - 2;
            int32_t a = bo[k], c = bo[k + 1];
            /* blocked: an edge joins them, they share a producer or a consumer, either has more
               than 64 out-edges, or their base devices differ */
            int joined = bx[a] != bx[c];
            int64_t out_a = 0, out_c = 0;
            for (int64_t e = 0; e < m; e++) {
                if ((src[e] == a && dst[e] == c) || (src[e] == c && dst[e] == a)) joined = 1;
                if (src[e] == a) out_a++;
                if (src[e] == c) out_c++;
            }
            uint8_t *mark = calloc((size_t)n, 2);   /* [n] preds of a, [n] succs of a */
            for (int64_t e = 0; e < m; e++) {
                if (dst[e] == a) mark[src[e]] = 1;
                if (src[e] == a) mark[n + dst[e]] = 1;
            }
            for (int64_t e = 0; e < m; e++) {
                if (dst[e] == c && mark[src[e]]) joined = 1;       /* common producer */
                if (src[e] == c && mark[n + dst[e]]) joined = 1;   /* common consumer */
            }
            free(mark);
            if (out_a > 64 || out_c > 64) joined = 1;
            if (!joined) {
                order_out[k] = c;
                order_out[k + 1] = a;
                swap = 1;
            }
        }
    }
    /* S4: placement move */
    if (j == 0 || (swap && lane == 0)) return 1;
    int32_t wsum = mix[0] + mix[1] + mix[2];
    if (wsum <= 0) return 1;
    int64_t b1 = (128 * (int64_t)mix[0]) / wsum, b2 = (128 * (int64_t)(mix[0] + mix[1])) / wsum;
    int32_t alts[8];
    if (lane < b1) {                                         /* FLIP1: enumerated */
        int64_t t = pass * b1 + lane;
        if (t < rlen * (D - 1)) {
            int64_t q = c0 + t % rlen, a = t / rlen;
            int32_t v = bo[q];
            int32_t na = alt_devices(allowed, D, v, bx[v], alts);
            if (a >= na) return 0;                           /* no such alternative: invalid */
            x_out[v] = (uint8_t)alts[a];
            return 1;
        }
        /* the region's single-op moves are used up: a FLIPk lane */
    }
    if (lane < b2) {                                         /* FLIPk: distinct positions */
        int64_t f = 2 + (int64_t)(oracle_draw(seed, step, P, b, j, 1) % 3u);
        if (f > rlen) f = rlen;
        int64_t taken[4];
        for (int64_t i = 0; i < f; i++) {
            int64_t r = (int64_t)(oracle_draw(seed, step, P, b, j, 2 + 2 * i) % (uint64_t)(rlen - i));
            int64_t q = -1;                                  /* r-th free position, ascending */
            for (int64_t cand = c0; cand < c0 + rlen; cand++) {
                int used = 0;
                for (int64_t u = 0; u < i; u++) used |= taken[u] == cand;
                if (used) continue;
                if (r == 0) { q = cand; break; }
                r--;
            }
            taken[i] = q;
            int32_t v = bo[q];
            int32_t na = alt_devices(allowed, D, v, bx[v], alts);
            if (na == 0) return 0;                           /* op cannot move: invalid */
            x_out[v] = (uint8_t)alts[oracle_draw(seed, step, P, b, j, 3 + 2 * i) % (uint64_t)na];
        }
        return 1;
    }
    {   /* WINDOW (v7): start s enumerated over the region (visit = how many times the
           enumeration has passed s); device d = A_s[draw(j, 4) mod |A_s|]; the window moves
           the first L ops from s that allow d and are not on d in the base (the "eligible"
           ops, M of them in [s, c + len)), L = 2 + (visit + draw(s, 0)) mod (M - 1): distinct
           for every visit of s; invalid if M < 2 or every length is used */
        int64_t i = lane - b2, nw = 128 - b2;
        int64_t w = pass * nw + i;
        int64_t s = c0 + w % rlen, visit = w / rlen;
        int32_t na = alt_devices(allowed, D, bo[s], bx[bo[s]], alts);
        if (na == 0) return 0;
        int32_t d = alts[oracle_draw(seed, step, P, b, j, 4) % (uint64_t)na];
        int64_t M = 0;
        for (int64_t q = s; q < c0 + rlen; q++)
            if (allowed_dev(allowed, bo[q], d) && bx[bo[q]] != d) M++;
        if (M < 2 || visit >= M - 1) return 0;
        int64_t L = 2 + (int64_t)(((uint64_t)visit + oracle_draw(seed, step, P, b, s, 0)) %
                                  (uint64_t)(M - 1));
        for (int64_t q = s; L > 0; q++) {
            int32_t v = bo[q];
            if (allowed_dev(allowed, v, d) && bx[v] != d) {
                x_out[v] = (uint8_t)d;
                L--;
            }
        }
    }
    return 1;
}

typedef struct {
    int32_t n; const int64_t *p; int64_t m; const int32_t *src, *dst; const int64_t *bytes;
    int32_t D; const int64_t *beta0, *beta1; const uint8_t *allowed;
    int32_t P, b; const uint8_t *base_x; const int32_t *base_order;
    uint64_t seed, step; const int32_t *mix;
    int64_t j0, j1, base_j; uint64_t *out;
    int32_t congestion, nondelay;
} key_job;

static void *key_worker(void *arg) {
    key_job *k = (key_job *)arg;
    uint8_t *x = malloc((size_t)k->n);
    int32_t *ord = malloc((size_t)k->n * sizeof(int32_t));
    for (int64_t j = k->j0; j < k->j1; j++) {
        uint64_t key = UINT64_MAX;
        if (oracle_candidate(k->n, k->m, k->src, k->dst, k->D, k->allowed, k->P, k->b, k->base_x,
                             k->base_order, j, k->seed, k->step, k->mix, x, ord)) {
            int64_t mk = oracle_makespan_model(k->n, k->p, k->m, k->src, k->dst, k->bytes, k->D,
                                               k->beta0, k->beta1, k->allowed, x, ord,
                                               k->congestion, k->nondelay, NULL);
            if (mk >= 0 && mk != INT64_MAX) key = ((uint64_t)mk << 24) | (uint64_t)j;
        }
        k->out[j - k->base_j] = key;
    }
    free(x); free(ord);
    return NULL;
}

int oracle_candidate_keys(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                          const int32_t *dst, const int64_t *bytes, int32_t D,
                          const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                          int32_t P, int32_t b, const uint8_t *base_x, const int32_t *base_order,
                          int64_t j0, int64_t j1, uint64_t seed, uint64_t step,
                          const int32_t mix[4], int32_t threads, uint64_t *keys_out) {
    return oracle_candidate_keys_model(n, p, m, src, dst, bytes, D, beta0, beta1, allowed, P, b,
                                       base_x, base_order, j0, j1, seed, step, mix, 1, 0,
                                       threads, keys_out);
}

int oracle_candidate_keys_model(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                                const int32_t *dst, const int64_t *bytes, int32_t D,
                                const int64_t *beta0, const int64_t *beta1,
                                const uint8_t *allowed, int32_t P, int32_t b,
                                const uint8_t *base_x, const int32_t *base_order, int64_t j0,
                                int64_t j1, uint64_t seed, uint64_t step, const int32_t mix[4],
                                int32_t congestion, int32_t nondelay, int32_t threads,
                                uint64_t *keys_out) {
    int64_t rc = check_graph(n, p, m, src, dst, bytes, D, beta0, beta1);
    if (rc) return (int)rc;
    if (j0 < 0 || j1 < j0 || j1 > (1ll << 24)) return ORACLE_EINVAL;
    int64_t cnt = j1 - j0;
    if (threads <= 0) threads = 1;
    if (cnt < threads) threads = cnt > 0 ? (int32_t)cnt : 1;
    pthread_t *th = malloc((size_t)threads * sizeof(pthread_t));
    key_job *jobs = malloc((size_t)threads * sizeof(key_job));
    for (int32_t t = 0; t < threads; t++) {
        key_job kj = {n, p, m, src, dst, bytes, D, beta0, beta1, allowed, P, b, base_x,
                      base_order, seed, step, mix, j0 + cnt * t / threads,
                      j0 + cnt * (t + 1) / threads, j0, keys_out, congestion, nondelay};
        jobs[t] = kj;
        pthread_create(&th[t], NULL, key_worker, &jobs[t]);
    }
    for (int32_t t = 0; t < threads; t++) pthread_join(th[t], NULL);
    free(th); free(jobs);
    return 0;
}

int oracle_search_step(int32_t n, const int64_t *p, int64_t m, const int32_t *src,
                       const int32_t *dst, const int64_t *bytes, int32_t D,
                       const int64_t *beta0, const int64_t *beta1, const uint8_t *allowed,
                       int32_t P, uint8_t *base_x, int32_t *base_order, int64_t *base_mk,
                       int64_t K, uint64_t seed, uint64_t step, const int32_t mix[4],
                       int32_t world, int32_t threads, uint64_t *keys) {
    if (P < 1 || K < 1 || K > (1ll << 24) || world < 1) return ORACLE_EINVAL;
    uint64_t *buf = malloc((size_t)K * sizeof(uint64_t));
    uint8_t *x = malloc((size_t)n);
    int32_t *ord = malloc((size_t)n * sizeof(int32_t));
    if (!buf || !x || !ord) { free(buf); free(x); free(ord); return ORACLE_ENOMEM; }
    int rc = 0;
    for (int32_t b = 0; b < P && rc == 0; b++) {
        uint64_t best = UINT64_MAX;
        for (int32_t r = 0; r < world && rc == 0; r++) {
            int64_t j0 = K * r / world, j1 = K * (r + 1) / world;
            rc = oracle_candidate_keys(n, p, m, src, dst, bytes, D, beta0, beta1, allowed, P, b,
                                       base_x, base_order, j0, j1, seed, step, mix, threads,
                                       buf);
            uint64_t rank_min = UINT64_MAX;          /* per-rank minimum ... */
            for (int64_t j = 0; j < j1 - j0; j++) if (buf[j] < rank_min) rank_min = buf[j];
            if (rank_min < best) best = rank_min;    /* ... then the min of minima */
        }
        keys[b] = best;
        if (rc || best == UINT64_MAX) continue;
        int64_t jstar = (int64_t)(best & ((1ull << 24) - 1));
        if (jstar != 0) {
            oracle_candidate(n, m, src, dst, D, allowed, P, b, base_x, base_order, jstar, seed,
                             step, mix, x, ord);
            memcpy(base_x + (int64_t)b * n, x, (size_t)n);
            memcpy(base_order + (int64_t)b * n, ord, (size_t)n * sizeof(int32_t));
        }
        base_mk[b] = (int64_t)(best >> 24);
    }
    free(buf); free(x); free(ord);
    return rc;
}
