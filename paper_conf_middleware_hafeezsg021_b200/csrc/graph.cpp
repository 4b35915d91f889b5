// graph.cpp -- graph ingest, comm model, position-space layout, seeds and batched evaluation
// (SURVEY §8(a) rows a0, a1, a3/a4 host side; C ABI in include/pesto.h).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <new>
#include <queue>
#include <string>

#include "host.h"
#include "moves.cuh"

using namespace pesto;

namespace pesto {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }
pesto_status fail(pesto_status s, const std::string &msg) {
    g_err = msg;
    return s;
}
pesto_status cuda_fail(cudaError_t e, const char *what) {
    g_err = std::string(what) + ": " + cudaGetErrorString(e);
    return e == cudaErrorMemoryAllocation ? PESTO_ENOMEM : PESTO_ECUDA;
}

static constexpr int64_t kGuard40 = int64_t(1) << 40;

// t = beta0 + ceil(bytes * beta1_fs / 10^6) (PAPER.md L138 linear model, reading R6); -1 overflow
static int64_t transfer_ns(int64_t bytes, int64_t beta0, int64_t beta1) {
    unsigned __int128 prod = (unsigned __int128)(uint64_t)bytes * (uint64_t)beta1;
    unsigned __int128 q = (prod + 999999u) / 1000000u;
    unsigned __int128 t = q + (uint64_t)beta0;
    if (t > (unsigned __int128)INT64_MAX) return -1;
    return (int64_t)t;
}

static int planes_for(int D) { return D <= 2 ? 1 : (D <= 4 ? 2 : 4); }

// worst-case makespan bound over the links set so far: sum p + sum_e max_L t_e (a0 step 3)
static int64_t worst_total(const pesto_graph *g, const std::vector<int64_t> &b0,
                           const std::vector<int64_t> &b1, const std::vector<uint8_t> &set) {
    int64_t total = 0;
    for (int32_t v = 0; v < g->n; v++) {
        total += g->p[v];
        if (total >= kGuard40) return -1;
    }
    for (int64_t e = 0; e < g->m; e++) {
        int64_t worst = 0;
        for (int L = 0; L < g->D * g->D; L++) {
            if (!set[L]) continue;
            int64_t t = transfer_ns(g->bytes[e], b0[L], b1[L]);
            if (t < 0) return -1;
            worst = std::max(worst, t);
        }
        total += worst;
        if (total >= kGuard40) return -1;
    }
    return total;
}

pesto_status ensure_comm_tables(pesto_graph *g) {
    const int D = g->D;
    for (int a = 0; a < D; a++)
        for (int b = 0; b < D; b++)
            if (a != b && !g->link_set[a * D + b])
                return fail(PESTO_ESTATE, "comm model not set for link " + std::to_string(a) +
                                              "->" + std::to_string(b));
    if (g->t_gen == g->comm_gen) return PESTO_OK;
    // link classes: distinct (beta0, beta1) in order of first appearance
    std::vector<std::pair<int64_t, int64_t>> cls;
    std::memset(g->link_class, 0, sizeof(g->link_class));
    for (int a = 0; a < D; a++)
        for (int b = 0; b < D; b++) {
            if (a == b) continue;
            const int L = a * D + b;
            std::pair<int64_t, int64_t> k{g->beta0[L], g->beta1[L]};
            int c = -1;
            for (size_t i = 0; i < cls.size(); i++)
                if (cls[i] == k) c = (int)i;
            if (c < 0) { c = (int)cls.size(); cls.push_back(k); }
            g->link_class[L] = (uint8_t)c;
        }
    if (cls.empty()) cls.push_back({0, 0});                 // D == 1: no links at all
    g->n_classes = (int32_t)cls.size();
    g->t_class.assign((size_t)g->m * g->n_classes, 0);
    for (int64_t e = 0; e < g->m; e++)
        for (int c = 0; c < g->n_classes; c++)
            g->t_class[(size_t)e * g->n_classes + c] = transfer_ns(g->bytes[e], cls[c].first, cls[c].second);
    g->t_gen = g->comm_gen;
    g->eligible32 = true;                                    // eval32: all durations < 2^28 ns
    for (int32_t v = 0; v < g->n; v++)
        if (g->p[v] >= (int64_t)kMaxDur32) g->eligible32 = false;
    for (int64_t t : g->t_class)
        if (t >= (int64_t)kMaxDur32) g->eligible32 = false;
    g->cache.clear();                                        // layouts embed t
    return PESTO_OK;
}

template <class T>
static cudaError_t upload_vec(DevBuf &d, const std::vector<T> &v) {
    cudaError_t e = d.ensure(std::max<size_t>(v.size() * sizeof(T), 16));
    if (e != cudaSuccess) return e;
    if (!v.empty()) e = cudaMemcpy(d.ptr, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice);
    return e;
}

pesto_status upload_layout(pesto_graph *g, Layout &L) {
    if (L.on_device) return PESTO_OK;
    DeviceGuard guard(g->device);
    cudaError_t e;
    if ((e = upload_vec(L.d_blob, L.blob)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_heavy, L.heavy)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_tiles, L.tiles)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_pos, L.pos)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_adj, L.swap_blocked)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_allowed_pos, L.allowed_pos)) != cudaSuccess)
        return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_blob32, L.blob32)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_heavy32, L.heavy32)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_tiles32, L.tiles32)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_order, L.order)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_op_off32, L.op_off32)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_pin_off, L.pin_off)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_pin_ref, L.pin_ref)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_slot_succ, L.slot_succ)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_spec_off, L.spec_off)) != cudaSuccess) return cuda_fail(e, "upload layout");
    if ((e = upload_vec(L.d_spec_pos, L.spec_pos)) != cudaSuccess) return cuda_fail(e, "upload layout");
    L.on_device = true;
    std::vector<BaseLayoutDev> view{layout_view(L)};
    if ((e = upload_vec(L.d_view, view)) != cudaSuccess) return cuda_fail(e, "upload layout");
    return PESTO_OK;
}

BaseLayoutDev layout_view(const Layout &L) {
    BaseLayoutDev v{};
    v.blob = L.d_blob.as<uint8_t>();
    v.tiles = L.d_tiles.as<TileDesc>();
    v.heavy = L.d_heavy.as<uint8_t>();
    v.pos_of = L.d_pos.as<int32_t>();
    v.allowed_pos = L.d_allowed_pos.as<uint8_t>();
    v.swap_blocked = L.d_adj.as<uint8_t>();
    v.bits = nullptr;
    v.n_tiles = (int32_t)L.tiles.size();
    v.W = L.W;
    v.blob32 = L.d_blob32.as<uint8_t>();
    v.tiles32 = L.d_tiles32.as<TileDesc>();
    v.heavy32 = L.d_heavy32.as<uint8_t>();
    v.n_tiles32 = (int32_t)L.tiles32.size();
    v.W32 = L.W32;
    v.order = L.d_order.as<int32_t>();
    v.op_off32 = L.d_op_off32.as<uint32_t>();
    v.pin_off = L.d_pin_off.as<uint32_t>();
    v.pin_ref = L.d_pin_ref.as<uint32_t>();
    v.nd_dst = L.d_nd_dst.as<int32_t>();
    v.nd_t = L.d_nd_t.as<int64_t>();
    v.spec_off = L.spec_off.empty() ? nullptr : L.d_spec_off.as<uint32_t>();
    v.spec_pos = L.spec_pos.empty() ? nullptr : L.d_spec_pos.as<int32_t>();
    return v;
}

// ---------------------------------------------------------------------------------------------
// row f4(i): non-delay dispatch (reading R24)
// ---------------------------------------------------------------------------------------------
pesto_status nd_check(pesto_graph *g) {
    pesto_status s = ensure_comm_tables(g);
    if (s) return s;
    if (g->n > (1 << 20)) return fail(PESTO_ESTATE, "non-delay dispatch supports n_ops <= 2^20");
    for (int32_t v = 0; v < g->n; v++)
        if (g->p[v] < 1)
            return fail(PESTO_ESTATE, "non-delay dispatch needs every p_i >= 1 ns (reading R24); op " +
                                          std::to_string(v) + " has p = 0");
    if (g->D > 1)
        for (int64_t t : g->t_class)
            if (t < 1) return fail(PESTO_ESTATE, "non-delay dispatch needs every transfer >= 1 ns (reading R24)");
    if (!g->nd_graph_ready) {
        cudaError_t e;
        if ((e = upload_vec(g->d_nd_p, g->p)) != cudaSuccess || (e = upload_vec(g->d_nd_indeg, g->indeg)) != cudaSuccess ||
            (e = upload_vec(g->d_nd_off, g->out_off)) != cudaSuccess)
            return cuda_fail(e, "upload non-delay graph arrays");
        g->nd_graph_ready = true;
    }
    return PESTO_OK;
}

pesto_status nd_ensure_layout(pesto_graph *g, Layout &L) {
    if (L.nd_gen == g->t_gen && L.d_nd_dst.ptr) return PESTO_OK;
    const int NC = g->n_classes;
    std::vector<int32_t> dst((size_t)g->m);
    std::vector<int64_t> t((size_t)g->m * NC);
    std::vector<int64_t> es;
    for (int32_t v = 0; v < g->n; v++) {
        es.assign(g->out_edges.begin() + g->out_off[v], g->out_edges.begin() + g->out_off[v + 1]);
        std::sort(es.begin(), es.end(), [&](int64_t a, int64_t b) {   // FCFS ties: (pos w, e), R3
            const int32_t pa = L.pos[g->dst[a]], pb = L.pos[g->dst[b]];
            return pa != pb ? pa < pb : a < b;
        });
        for (size_t k = 0; k < es.size(); k++) {
            const int64_t i = g->out_off[v] + (int64_t)k;
            dst[i] = g->dst[es[k]];
            for (int c = 0; c < NC; c++) t[(size_t)i * NC + c] = g->t_class[(size_t)es[k] * NC + c];
        }
    }
    cudaError_t e;
    if ((e = upload_vec(L.d_nd_dst, dst)) != cudaSuccess || (e = upload_vec(L.d_nd_t, t)) != cudaSuccess)
        return cuda_fail(e, "upload non-delay edge order");
    L.nd_gen = g->t_gen;
    return PESTO_OK;
}

pesto_status nd_fill(pesto_graph *g, Scratch &ws, NdParams &p, int64_t n_tasks, int *grid_out) {
    std::memset(&p, 0, sizeof p);
    p.n = g->n;
    p.D = g->D;
    p.planes = g->planes;
    p.words = g->words;
    p.nw1 = (p.words + 31) / 32;
    p.nw2 = (p.nw1 + 31) / 32;
    p.rb = p.words + p.nw1 + p.nw2;
    p.n_classes = g->n_classes;
    p.link_queue = g->link_model == PESTO_LINKS_FCFS ? 1 : 0;
    p.all_allowed = g->all_allowed ? 1 : 0;
    std::memcpy(p.link_class, g->link_class, 64);
    p.p = g->d_nd_p.as<int64_t>();
    p.indeg = g->d_nd_indeg.as<int32_t>();
    p.out_off = g->d_nd_off.as<int64_t>();
    p.feas = feasibility_view(g);
    p.warps_per_cta = nondelay_warps_per_cta(p);
    if (p.warps_per_cta == 0)
        return fail(PESTO_ESTATE, "non-delay kernel: the graph's per-warp state exceeds shared memory");
    const int per_sm = nondelay_max_ctas_per_sm(p);
    if (per_sm <= 0) return fail(PESTO_ECUDA, "non-delay kernel does not fit on an SM");
    int64_t grid = std::min<int64_t>((n_tasks + p.warps_per_cta - 1) / p.warps_per_cta,
                                     (int64_t)g->sms * per_sm);
    if (const char *e = std::getenv("PESTO_ND_MAX_WARPS")) {     // tuning experiments
        const int64_t w = std::atoll(e);
        if (w > 0) grid = std::min<int64_t>(grid, std::max<int64_t>(1, w / p.warps_per_cta));
    }
    grid = std::max<int64_t>(grid, 1);
    const size_t slots = (size_t)grid * p.warps_per_cta;
    cudaError_t e;
    if ((e = ws.nd_rem.ensure(slots * g->n * 4)) != cudaSuccess ||
        (e = ws.nd_rdy.ensure(slots * g->n * 8)) != cudaSuccess ||
        (e = ws.nd_pend.ensure(slots * g->n * g->D * 8)) != cudaSuccess)
        return cuda_fail(e, "allocate non-delay scratch");
    p.rem = ws.nd_rem.as<int32_t>();
    p.rdy = ws.nd_rdy.as<int64_t>();
    p.pend = ws.nd_pend.as<uint64_t>();
    *grid_out = (int)grid;
    return PESTO_OK;
}

void fill_eval_common(const pesto_graph *g, EvalParams &p) {
    std::memset(&p, 0, sizeof p);
    p.n = g->n;
    p.D = g->D;
    p.planes = g->planes;
    p.words = g->words;
    p.edge_stride = edge_stride_for(g->n_classes);
    p.edge_stride32 = edge_stride32_for(g->n_classes);
    p.n_classes = g->n_classes;
    p.link_queue = g->link_model == PESTO_LINKS_FCFS ? 1 : 0;
    p.feas = feasibility_view(g);
    std::memcpy(p.link_class, g->link_class, 64);
    p.all_allowed = g->all_allowed ? 1 : 0;
}

pesto_status ensure_state(pesto_graph *g, Scratch &ws, const EvalParams &p, int search_mode,
                          int64_t n_tasks, int *grid_out) {
    int per_sm = eval_max_ctas_per_sm(p, search_mode);
    if (per_sm <= 0)
        return fail(PESTO_ECUDA, "eval kernel does not fit on an SM (smem " +
                                     std::to_string(eval_smem_bytes(p, search_mode)) + " B)");
    int64_t grid = std::min<int64_t>(n_tasks, (int64_t)g->sms * per_sm);
    grid = std::max<int64_t>(grid, 1);
    size_t bytes = (size_t)grid * kWarps * (size_t)std::max(p.max_W, 1) * 32 * sizeof(int64_t);
    cudaError_t e = ws.state.ensure(bytes);
    if (e != cudaSuccess) return cuda_fail(e, "allocate slot state");
    *grid_out = (int)grid;
    return PESTO_OK;
}

int choose_cpl32(const pesto_graph *g, int64_t n_tasks) {
    static const int forced = [] {
        const char *e = std::getenv("PESTO_EVAL32_CPL");
        return e ? std::atoi(e) : 0;
    }();
    if (forced == 1 || forced == 2) return forced;
    return n_tasks <= 2 * (int64_t)g->sms ? 1 : 2;
}

void plan_eval32(const pesto_graph *g, EvalParams &p, int64_t j0, int64_t j1, int n_bases) {
    // CPL 1 when its tasks fit in one wave of 2 CTAs per SM (latency-bound: more warps), else 2
    const int64_t ts1 = eval32_task_size(1);
    const int64_t t1 = (j1 - (j0 - j0 % ts1) + ts1 - 1) / ts1 * n_bases;
    p.cpl32 = choose_cpl32(g, t1);
    const int64_t ts = eval32_task_size(p.cpl32);
    p.tasks_per_base = (j1 - (j0 - j0 % ts) + ts - 1) / ts;
    p.n_tasks = p.tasks_per_base * n_bases;
}

pesto_status ensure_state32(pesto_graph *g, Scratch &ws, const EvalParams &p, int search_mode,
                            int64_t n_tasks, int *grid_out, bool wide_buf) {
    int per_sm = eval32_max_ctas_per_sm(p, search_mode);
    if (per_sm <= 0)
        return fail(PESTO_ECUDA, "eval32 kernel does not fit on an SM (smem " +
                                     std::to_string(eval32_smem_bytes(p, search_mode)) + " B)");
    int64_t grid = std::min<int64_t>(n_tasks, (int64_t)g->sms * per_sm);
    grid = std::max<int64_t>(grid, 1);
    size_t bytes = (size_t)grid * eval32_task_size(p.cpl32) * (size_t)std::max(p.max_W32, 1) *
                   (p.wide32 ? sizeof(uint64_t) : sizeof(uint32_t));
    cudaError_t e = (wide_buf ? ws.state32w : ws.state32).ensure(bytes);
    if (e != cudaSuccess) return cuda_fail(e, "allocate cold slot state");
    *grid_out = (int)grid;
    return PESTO_OK;
}

Feasibility feasibility_view(const pesto_graph *g) {
    Feasibility f{};
    f.has_cap = g->has_cap ? 1 : 0;
    f.has_coloc = g->has_coloc ? 1 : 0;
    if (!f.has_cap && !f.has_coloc) return f;
    f.mem = g->d_mem.as<int64_t>();
    f.cap = g->d_cap.as<int64_t>();
    f.coloc = g->d_coloc.as<int32_t>();
    f.coloc_size = g->d_coloc_size.as<int32_t>();
    f.coloc_pairs = g->d_coloc_pairs.as<int2>();
    f.n_pairs = (int32_t)g->coloc_pairs.size();
    return f;
}

bool placement_feasible(const pesto_graph *g, const uint8_t *x, int64_t *footprint8) {
    int64_t F[8] = {0};
    for (int32_t v = 0; v < g->n; v++)
        if (!g->mem.empty()) F[x[v] & 7] += g->mem[v];
    if (footprint8) std::copy(F, F + 8, footprint8);
    if (g->has_cap)
        for (int d = 0; d < g->D; d++)
            if (F[d] > g->cap[d]) return false;
    if (g->has_coloc) {
        std::vector<int32_t> dev(g->n, -1);
        for (int32_t v = 0; v < g->n; v++) {
            const int32_t c = g->coloc[v];
            if (c < 0) continue;
            if (dev[c] < 0) dev[c] = x[v];
            else if (dev[c] != x[v]) return false;
        }
    }
    return true;
}

static uint64_t splitmix_next(uint64_t &s) {
    s += 0x9E3779B97F4A7C15ull;
    return mix64(s);
}

}  // namespace pesto

// =============================================================================================
// C ABI
// =============================================================================================
extern "C" {

const char *pesto_last_error(void) { return g_err.c_str(); }

const char *pesto_status_str(pesto_status s) {
    switch (s) {
        case PESTO_OK: return "PESTO_OK";
        case PESTO_EINVAL: return "PESTO_EINVAL";
        case PESTO_ECYCLE: return "PESTO_ECYCLE";
        case PESTO_ENOTTOPO: return "PESTO_ENOTTOPO";
        case PESTO_EOVERFLOW: return "PESTO_EOVERFLOW";
        case PESTO_ENOMEM: return "PESTO_ENOMEM";
        case PESTO_ECUDA: return "PESTO_ECUDA";
        case PESTO_ENCCL: return "PESTO_ENCCL";
        case PESTO_ESTATE: return "PESTO_ESTATE";
    }
    return "PESTO_?";
}

int32_t pesto_version(void) { return 100; }
int64_t pesto_launch_count(void) { return launch_count_value(); }

pesto_status pesto_graph_create(const pesto_graph_desc *d, pesto_graph **out) {
    if (!d || !out) return fail(PESTO_EINVAL, "NULL argument");
    *out = nullptr;
    if (d->n_ops < 1 || d->n_ops > PESTO_MAX_OPS) return fail(PESTO_EINVAL, "n_ops out of range");
    if (d->n_edges < 0) return fail(PESTO_EINVAL, "n_edges < 0");
    if (d->n_devices < 1 || d->n_devices > PESTO_MAX_DEVICES)
        return fail(PESTO_EINVAL, "n_devices out of range");
    if (!d->compute_ns) return fail(PESTO_EINVAL, "compute_ns is NULL");
    if (d->n_edges > 0 && (!d->src || !d->dst || !d->bytes))
        return fail(PESTO_EINVAL, "edge arrays are NULL");
    std::unique_ptr<pesto_graph> g(new (std::nothrow) pesto_graph());
    if (!g) return fail(PESTO_ENOMEM, "host allocation");
    const int32_t n = d->n_ops;
    const int64_t m = d->n_edges;
    g->n = n;
    g->m = m;
    g->D = d->n_devices;
    g->planes = planes_for(g->D);
    g->words = (n + 31) / 32;
    g->device = d->cuda_device;
    try {
        g->p.assign(d->compute_ns, d->compute_ns + n);
        if (m) {
            g->src.assign(d->src, d->src + m);
            g->dst.assign(d->dst, d->dst + m);
            g->bytes.assign(d->bytes, d->bytes + m);
        }
    } catch (...) {
        return fail(PESTO_ENOMEM, "host allocation");
    }
    for (int32_t v = 0; v < n; v++)
        if (g->p[v] < 0) return fail(PESTO_EINVAL, "compute_ns[" + std::to_string(v) + "] < 0");
    for (int64_t e = 0; e < m; e++) {
        if (g->src[e] < 0 || g->src[e] >= n || g->dst[e] < 0 || g->dst[e] >= n)
            return fail(PESTO_EINVAL, "edge " + std::to_string(e) + " index out of range");
        if (g->src[e] == g->dst[e]) return fail(PESTO_EINVAL, "self loop at edge " + std::to_string(e));
        if (g->bytes[e] < 0) return fail(PESTO_EINVAL, "bytes[" + std::to_string(e) + "] < 0");
    }
    const unsigned full = (1u << g->D) - 1u;
    g->allowed.assign(n, (uint8_t)full);
    if (d->allowed) {
        for (int32_t v = 0; v < n; v++) {
            const unsigned msk = d->allowed[v] & full;
            if (!msk) return fail(PESTO_EINVAL, "op " + std::to_string(v) + " allows no device");
            g->allowed[v] = (uint8_t)msk;
            if (msk != full) g->all_allowed = false;
        }
    }
    // out-edge CSR + Kahn cycle check (L142: G is a DAG)
    g->out_off.assign((size_t)n + 1, 0);
    g->indeg.assign(n, 0);
    for (int64_t e = 0; e < m; e++) { g->out_off[g->src[e] + 1]++; g->indeg[g->dst[e]]++; }
    for (int32_t v = 0; v < n; v++) g->out_off[v + 1] += g->out_off[v];
    g->out_edges.resize(m);
    {
        std::vector<int64_t> fill(g->out_off.begin(), g->out_off.end() - 1);
        for (int64_t e = 0; e < m; e++) g->out_edges[fill[g->src[e]]++] = e;
        std::vector<int32_t> deg(g->indeg), q;
        q.reserve(n);
        for (int32_t v = 0; v < n; v++) if (!deg[v]) q.push_back(v);
        for (size_t h = 0; h < q.size(); h++)
            for (int64_t i = g->out_off[q[h]]; i < g->out_off[q[h] + 1]; i++)
                if (--deg[g->dst[g->out_edges[i]]] == 0) q.push_back(g->dst[g->out_edges[i]]);
        if ((int32_t)q.size() != n) return fail(PESTO_ECYCLE, "graph has a cycle");
    }
    g->in_off.assign((size_t)n + 1, 0);
    for (int64_t e = 0; e < m; e++) g->in_off[g->dst[e] + 1]++;
    for (int32_t v = 0; v < n; v++) g->in_off[v + 1] += g->in_off[v];
    g->in_edges.resize(m);
    {
        std::vector<int64_t> fill(g->in_off.begin(), g->in_off.end() - 1);
        for (int64_t e = 0; e < m; e++) g->in_edges[fill[g->dst[e]]++] = e;
    }
    {
        int64_t total = 0;
        for (int32_t v = 0; v < n; v++) {
            total += g->p[v];
            if (total >= kGuard40) return fail(PESTO_EOVERFLOW, "sum of compute times >= 2^40 ns");
        }
        g->worst_total = total;
    }
    g->beta0.assign((size_t)g->D * g->D, 0);
    g->beta1.assign((size_t)g->D * g->D, 0);
    g->link_set.assign((size_t)g->D * g->D, 0);
    for (int32_t v = 0; v < n; v++)
        if (popc32(g->allowed[v]) >= 2) g->movable.push_back(v);
    const int P = g->planes;
    g->fmask.assign(n, 0);
    for (int32_t v = 0; v < n; v++)
        for (int c = 0; c < (1 << P); c++)
            if (c >= g->D || !((g->allowed[v] >> c) & 1)) g->fmask[v] |= (uint16_t)(1u << c);
    if (g->device >= 0) {
        DeviceGuard guard(g->device);
        cudaError_t e = cudaDeviceGetAttribute(&g->sms, cudaDevAttrMultiProcessorCount, g->device);
        if (e != cudaSuccess) return cuda_fail(e, "query device");
        if ((e = upload_vec(g->d_fmask, g->fmask)) != cudaSuccess) return cuda_fail(e, "upload");
        if ((e = upload_vec(g->d_movable, g->movable)) != cudaSuccess) return cuda_fail(e, "upload");
        if ((e = upload_vec(g->d_allowed, g->allowed)) != cudaSuccess) return cuda_fail(e, "upload");
    }
    *out = g.release();
    return PESTO_OK;
}

void pesto_graph_destroy(pesto_graph *g) {
    if (!g) return;
    DeviceGuard guard(g->device);
    delete g;
}

pesto_status pesto_graph_set_constraints(pesto_graph *g, const int64_t *mem, const int64_t *cap,
                                         const int32_t *coloc) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    const int32_t n = g->n;
    if (mem)
        for (int32_t v = 0; v < n; v++)
            if (mem[v] < 0) return fail(PESTO_EINVAL, "negative footprint");
    if (cap)
        for (int d = 0; d < g->D; d++)
            if (cap[d] < 0) return fail(PESTO_EINVAL, "negative cap");
    if (coloc)
        for (int32_t v = 0; v < n; v++)
            if (coloc[v] < -1 || coloc[v] >= n) return fail(PESTO_EINVAL, "colocation group out of [-1, n)");
    DeviceGuard guard(g->device);
    g->has_cap = cap != nullptr;
    g->has_coloc = coloc != nullptr;
    g->mem.assign(n, 0);
    if (mem) {
        std::copy(mem, mem + n, g->mem.begin());
    } else {                                      // L202: input + output tensor sizes
        for (int64_t e = 0; e < g->m; e++) {
            g->mem[g->src[e]] += g->bytes[e];
            g->mem[g->dst[e]] += g->bytes[e];
        }
    }
    g->cap.assign(8, 0);
    if (cap) std::copy(cap, cap + g->D, g->cap.begin());
    g->coloc.assign(n, -1);
    g->coloc_size.assign(n, 0);
    g->coloc_pairs.clear();
    if (coloc) {
        std::vector<int32_t> rep(n, -1);
        for (int32_t v = 0; v < n; v++) {
            const int32_t c = coloc[v];
            g->coloc[v] = c;
            if (c < 0) continue;
            g->coloc_size[c]++;
            if (rep[c] < 0) rep[c] = v;
            else g->coloc_pairs.push_back(make_int2(v, rep[c]));
        }
    }
    g->cons_gen++;
    if (g->device < 0) return PESTO_OK;
    cudaError_t e;
    if ((e = upload_vec(g->d_mem, g->mem)) != cudaSuccess || (e = upload_vec(g->d_cap, g->cap)) != cudaSuccess ||
        (e = upload_vec(g->d_coloc, g->coloc)) != cudaSuccess ||
        (e = upload_vec(g->d_coloc_size, g->coloc_size)) != cudaSuccess ||
        (e = upload_vec(g->d_coloc_pairs, g->coloc_pairs)) != cudaSuccess)
        return cuda_fail(e, "upload constraints");
    return PESTO_OK;
}

pesto_status pesto_graph_set_dispatch(pesto_graph *g, int32_t mode) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    if (mode != PESTO_DISPATCH_FIXED && mode != PESTO_DISPATCH_NONDELAY) return fail(PESTO_EINVAL, "unknown dispatch mode");
    g->dispatch = mode;
    return PESTO_OK;
}

pesto_status pesto_graph_set_link_model(pesto_graph *g, int32_t model) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    if (model != PESTO_LINKS_FCFS && model != PESTO_LINKS_UNLIMITED) return fail(PESTO_EINVAL, "unknown link model");
    g->link_model = model;
    return PESTO_OK;
}

pesto_status pesto_comm_model(pesto_graph *g, int32_t a, int32_t b, int64_t beta0,
                              int64_t beta1) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    if (beta0 < 0 || beta1 < 0) return fail(PESTO_EINVAL, "negative comm coefficient");
    if (a < -1 || a >= g->D || b < -1 || b >= g->D) return fail(PESTO_EINVAL, "device out of range");
    if (a >= 0 && a == b) return fail(PESTO_EINVAL, "a link joins two different devices");
    std::vector<int64_t> b0 = g->beta0, b1 = g->beta1;
    std::vector<uint8_t> set = g->link_set;
    for (int x = 0; x < g->D; x++)
        for (int y = 0; y < g->D; y++) {
            if (x == y || (a >= 0 && x != a) || (b >= 0 && y != b)) continue;
            b0[x * g->D + y] = beta0;
            b1[x * g->D + y] = beta1;
            set[x * g->D + y] = 1;
        }
    const int64_t tot = worst_total(g, b0, b1, set);
    if (tot < 0) return fail(PESTO_EOVERFLOW, "sum p + sum_e max_L t_e >= 2^40 ns");
    g->beta0 = b0;
    g->beta1 = b1;
    g->link_set = set;
    g->worst_total = tot;
    g->comm_gen++;
    return PESTO_OK;
}

pesto_status pesto_graph_stats_for(pesto_graph *g, const int32_t *order, pesto_graph_stats *st) {
    if (!g || !st) return fail(PESTO_EINVAL, "NULL argument");
    std::shared_ptr<Layout> L;
    pesto_status s = build_layout(g, order, L, true);
    if (s) return s;
    st->n_ops = g->n;
    st->n_devices = g->D;
    st->n_edges = g->m;
    st->live_slots = L->W;
    st->n_tiles = (int32_t)L->tiles.size();
    st->layout_bytes = (int64_t)(L->blob.size() + L->heavy.size());
    int32_t mi = 0, mo = 0;
    for (int32_t v = 0; v < g->n; v++) {
        mi = std::max(mi, g->indeg[v]);
        mo = std::max<int32_t>(mo, (int32_t)(g->out_off[v + 1] - g->out_off[v]));
    }
    st->max_in_degree = mi;
    st->max_out_degree = mo;
    st->link_classes = g->n_classes;
    st->time32_exact = g->worst_total < (int64_t(1) << 31) ? 1 : 0;
    return PESTO_OK;
}

pesto_status pesto_seed_order(pesto_graph *g, int32_t kind, uint64_t seed, int32_t *order_out) {
    if (!g || !order_out) return fail(PESTO_EINVAL, "NULL argument");
    const int32_t n = g->n;
    std::vector<int32_t> deg(g->indeg);
    std::vector<int32_t> out;
    out.reserve(n);
    if (kind == PESTO_ORDER_CRITICAL_PATH) {
        // bottom level (longest path to a sink counting p only), then Kahn by max bottom level,
        // ties by smaller op id: the critical-path list order of PAPER.md L98 (Fig. 2b)
        std::vector<int32_t> topo;
        {
            std::vector<int32_t> d2(g->indeg);
            for (int32_t v = 0; v < n; v++) if (!d2[v]) topo.push_back(v);
            for (size_t h = 0; h < topo.size(); h++)
                for (int64_t i = g->out_off[topo[h]]; i < g->out_off[topo[h] + 1]; i++)
                    if (--d2[g->dst[g->out_edges[i]]] == 0) topo.push_back(g->dst[g->out_edges[i]]);
        }
        std::vector<int64_t> bl(n, 0);
        for (int32_t k = n - 1; k >= 0; k--) {
            const int32_t v = topo[k];
            int64_t best = 0;
            for (int64_t i = g->out_off[v]; i < g->out_off[v + 1]; i++)
                best = std::max(best, bl[g->dst[g->out_edges[i]]]);
            bl[v] = g->p[v] + best;
        }
        auto cmp = [&](int32_t a, int32_t b) { return bl[a] != bl[b] ? bl[a] < bl[b] : a > b; };
        std::priority_queue<int32_t, std::vector<int32_t>, decltype(cmp)> pq(cmp);
        for (int32_t v = 0; v < n; v++) if (!deg[v]) pq.push(v);
        while (!pq.empty()) {
            const int32_t v = pq.top();
            pq.pop();
            out.push_back(v);
            for (int64_t i = g->out_off[v]; i < g->out_off[v + 1]; i++)
                if (--deg[g->dst[g->out_edges[i]]] == 0) pq.push(g->dst[g->out_edges[i]]);
        }
    } else if (kind == PESTO_ORDER_FIFO) {
        for (int32_t v = 0; v < n; v++) if (!deg[v]) out.push_back(v);
        for (size_t h = 0; h < out.size(); h++)
            for (int64_t i = g->out_off[out[h]]; i < g->out_off[out[h] + 1]; i++)
                if (--deg[g->dst[g->out_edges[i]]] == 0) out.push_back(g->dst[g->out_edges[i]]);
    } else if (kind == PESTO_ORDER_RANDOM) {
        // seeded random pick from the ready set: TF's default dispatch
        uint64_t s = seed;
        std::vector<int32_t> ready;
        for (int32_t v = 0; v < n; v++) if (!deg[v]) ready.push_back(v);
        while (!ready.empty()) {
            const size_t i = (size_t)(splitmix_next(s) % ready.size());
            const int32_t v = ready[i];
            ready[i] = ready.back();
            ready.pop_back();
            out.push_back(v);
            for (int64_t k = g->out_off[v]; k < g->out_off[v + 1]; k++)
                if (--deg[g->dst[g->out_edges[k]]] == 0) ready.push_back(g->dst[g->out_edges[k]]);
        }
    } else {
        return fail(PESTO_EINVAL, "unknown order kind");
    }
    std::copy(out.begin(), out.end(), order_out);
    return PESTO_OK;
}

pesto_status pesto_seed_placement(pesto_graph *g, int32_t kind, const int32_t *order,
                                  const int32_t *layer, uint64_t seed, uint8_t *x) {
    if (!g || !x) return fail(PESTO_EINVAL, "NULL argument");
    const int32_t n = g->n, D = g->D;
    auto lowest = [&](int32_t v) {
        for (int d = 0; d < D; d++) if ((g->allowed[v] >> d) & 1) return d;
        return 0;
    };
    auto fix = [&](int32_t v, int d) { return ((g->allowed[v] >> d) & 1) ? d : lowest(v); };
    if (kind == PESTO_PLACE_SINGLE) {
        for (int32_t v = 0; v < n; v++) x[v] = (uint8_t)lowest(v);
    } else if (kind == PESTO_PLACE_EXPERT) {
        // contiguous layers per device ("Expert"): floor(layer * D / n_layers)
        if (!layer) return fail(PESTO_EINVAL, "EXPERT needs layer tags");
        int32_t nl = 0;
        for (int32_t v = 0; v < n; v++) {
            if (layer[v] < 0) return fail(PESTO_EINVAL, "negative layer tag");
            nl = std::max(nl, layer[v] + 1);
        }
        for (int32_t v = 0; v < n; v++)
            x[v] = (uint8_t)fix(v, (int)((int64_t)layer[v] * D / nl));
    } else if (kind == PESTO_PLACE_TOPO_SPLIT) {
        // pi cut into D contiguous segments of about equal sum p (mTOPO-like)
        if (!order) return fail(PESTO_EINVAL, "TOPO_SPLIT needs an order");
        int64_t total = 0;
        for (int32_t v = 0; v < n; v++) total += g->p[v];
        int64_t before = 0;
        for (int32_t k = 0; k < n; k++) {
            const int32_t v = order[k];
            if (v < 0 || v >= n) return fail(PESTO_EINVAL, "order entry out of range");
            int d;
            if (total > 0) d = (int)(((__int128)(2 * before + g->p[v]) * D) / (2 * (__int128)total));
            else d = (int)((int64_t)k * D / n);
            x[v] = (uint8_t)fix(v, std::min(d, D - 1));
            before += g->p[v];
        }
    } else if (kind == PESTO_PLACE_RANDOM) {
        uint64_t s = seed;
        for (int32_t v = 0; v < n; v++) {
            const int na = popc32(g->allowed[v]);
            int pick = (int)(splitmix_next(s) % (uint64_t)na);
            for (int d = 0; d < D; d++)
                if ((g->allowed[v] >> d) & 1) {
                    if (pick == 0) { x[v] = (uint8_t)d; break; }
                    pick--;
                }
        }
    } else {
        return fail(PESTO_EINVAL, "unknown placement kind");
    }
    return PESTO_OK;
}

}  // extern "C"

namespace {

// pesto_eval_batch on the scratch set ws (the graph's own, or a workspace's)
pesto_status eval_batch_ws(pesto_graph *g, Scratch &ws, const int32_t *order, const void *placements,
                           int64_t stride, int64_t n_cand, int64_t *makespans, void *stream) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    if (g->device < 0) return fail(PESTO_ESTATE, "host-only graph handle");
    if (n_cand < 0) return fail(PESTO_EINVAL, "n_cand < 0");
    const int64_t row_bytes = ((int64_t)g->n * g->planes + 7) / 8;
    if (stride < row_bytes || stride % 16) return fail(PESTO_EINVAL, "row_stride_bytes must be >= ceil(n*b/8) and a multiple of 16");
    if (n_cand == 0) return PESTO_OK;
    if (!placements || !makespans) return fail(PESTO_EINVAL, "NULL buffer");
    if ((reinterpret_cast<uintptr_t>(placements) & 15) != 0) return fail(PESTO_EINVAL, "placements must be 16-byte aligned");
    DeviceGuard guard(g->device);
    std::shared_ptr<Layout> L;
    pesto_status s = build_layout(g, order, L, true);
    if (s) return s;
    if ((s = upload_layout(g, *L))) return s;
    cudaStream_t st = (cudaStream_t)stream;
    const int64_t n_groups = (n_cand + 31) / 32;
    // kStreamPad zeroed bytes past both word streams: the explicit-row walk reads the next
    // op's and the next step's words one step ahead (eval32.cu fast_rows)
    const size_t planes_bytes = (size_t)n_groups * g->n * g->planes * 4;
    cudaError_t e = ws.planes.ensure(planes_bytes + kStreamPad);
    if (e != cudaSuccess) return cuda_fail(e, "allocate bit-sliced placements");
    if ((e = cudaMemsetAsync(ws.planes.as<uint8_t>() + planes_bytes, 0, kStreamPad,
                             (cudaStream_t)stream)) != cudaSuccess)
        return cuda_fail(e, "clear stream padding");
    if ((e = ws.invalid.ensure((size_t)n_groups * 4)) != cudaSuccess) return cuda_fail(e, "allocate");
    TransposeParams tp{};
    tp.rows = static_cast<const uint8_t *>(placements);
    tp.stride = stride;
    tp.n_cand = n_cand;
    tp.n_groups = n_groups;
    tp.n = g->n;
    tp.planes = g->planes;
    tp.pos_of = L->d_pos.as<int32_t>();
    tp.fmask = g->d_fmask.as<uint16_t>();
    tp.planes_out = ws.planes.as<uint32_t>();
    tp.invalid_out = ws.invalid.as<uint32_t>();
    // the successors' codes in eval32 walk order (edge slots), for the explicit-row walk
    const bool nondelay = g->dispatch == PESTO_DISPATCH_NONDELAY;
    if (nondelay) {
        if ((s = nd_check(g))) return s;
        if ((s = nd_ensure_layout(g, *L))) return s;
    }
    const bool ystream = !nondelay && g->eligible32 && L->W32 > 0 && g->link_model == PESTO_LINKS_FCFS;
    if (ystream) {
        tp.slot_succ = L->d_slot_succ.as<int32_t>();
        tp.n_slots = (int64_t)L->slot_succ.size();
        const size_t ybytes = (size_t)n_groups * tp.n_slots * g->planes * 4;
        if ((e = ws.yplanes.ensure(ybytes + kStreamPad)) != cudaSuccess)
            return cuda_fail(e, "allocate edge-slot stream");
        if ((e = cudaMemsetAsync(ws.yplanes.as<uint8_t>() + ybytes, 0, kStreamPad, st)) != cudaSuccess)
            return cuda_fail(e, "clear stream padding");
        tp.yplanes_out = ws.yplanes.as<uint32_t>();
    }
    if ((e = launch_transpose(tp, st)) != cudaSuccess) return cuda_fail(e, "launch transpose");
    if (g->has_cap || g->has_coloc) {                 // row f3: mark infeasible rows
        FeasParams fp{};
        fp.planes = ws.planes.as<uint32_t>();
        fp.invalid = ws.invalid.as<uint32_t>();
        fp.n_groups = n_groups;
        fp.n = g->n;
        fp.D = g->D;
        fp.planes_n = g->planes;
        fp.order = L->d_order.as<int32_t>();
        fp.pos_of = L->d_pos.as<int32_t>();
        fp.feas = feasibility_view(g);
        if ((e = launch_feasibility(fp, st)) != cudaSuccess) return cuda_fail(e, "launch feasibility");
    }
    if (nondelay) {                                   // row f4(i): one warp per row
        NdParams np;
        int grid = 0;
        if ((s = nd_fill(g, ws, np, n_cand, &grid))) return s;
        np.rows = tp.rows;
        np.stride = stride;
        np.n_cand = n_cand;
        np.invalid = ws.invalid.as<uint32_t>();
        np.makespans = makespans;
        np.nd_dst = L->d_nd_dst.as<int32_t>();
        np.nd_t = L->d_nd_t.as<int64_t>();
        np.pos_of = L->d_pos.as<int32_t>();
        np.order = L->d_order.as<int32_t>();
        if ((e = launch_nondelay(np, 0, grid, st)) != cudaSuccess) return cuda_fail(e, "launch non-delay");
        return PESTO_OK;
    }
    EvalParams p;
    fill_eval_common(g, p);
    p.stage_bytes = L->stage_bytes;
    p.max_W = L->W;
    p.stage_bytes32 = L->stage_bytes32;
    p.max_W32 = L->W32;
    p.planes_in = ws.planes.as<uint32_t>();
    p.yplanes = ws.yplanes.as<uint32_t>();
    p.n_slots = (int64_t)L->slot_succ.size();
    p.invalid = ws.invalid.as<uint32_t>();
    p.n_cand = n_cand;
    p.makespans = makespans;
    p.bases = L->d_view.as<BaseLayoutDev>();
    p.group_begin = 0;
    p.groups_per_base = n_groups;
    p.tasks_per_base = (n_groups + kWarps - 1) / kWarps;
    p.n_tasks = p.tasks_per_base;
    int grid = 0;
    // 64-bit path for every row: ineligible durations, no eval32 stream, or congestion-free
    // links (row f4(ii) is a modelling variant; eval32 carries only the FCFS link queues)
    if (!g->eligible32 || L->W32 == 0 || g->link_model != PESTO_LINKS_FCFS) {
        if ((s = ensure_state(g, ws, p, 0, p.n_tasks, &grid))) return s;
        p.state = ws.state.as<int64_t>();
        if ((e = launch_eval(p, 0, grid, st)) != cudaSuccess) return cuda_fail(e, "launch eval");
        return PESTO_OK;
    }
    // fast path: 32-bit saturating K1; rows that saturate are listed and re-run in 64-bit
    if ((e = ws.flags.ensure((size_t)(n_cand + 4) * 4)) != cudaSuccess) return cuda_fail(e, "allocate");
    if ((e = cudaMemsetAsync(ws.flags.ptr, 0, 4, st)) != cudaSuccess) return cuda_fail(e, "reset flags");
    p.flag_count = ws.flags.as<int32_t>();
    p.flag_list = ws.flags.as<int32_t>() + 4;
    {
        EvalParams p32 = p;
        plan_eval32(g, p32, 0, n_cand, 1);
        // a workspace's batches are meant to overlap each other (several in flight on their own
        // streams): two candidates per lane (4 CTAs/SM) leaves room on the SMs for the next
        // batch's CTAs, where one per lane (2 CTAs/SM, the fastest for a lone batch) does not
        // (e2e with 4 buffers 10.8 -> 11.9 M cand/s)
        if (&ws != &g->ws && !std::getenv("PESTO_EVAL32_CPL")) {
            p32.cpl32 = 2;
            const int64_t ts = eval32_task_size(2);
            p32.tasks_per_base = (n_cand + ts - 1) / ts;
            p32.n_tasks = p32.tasks_per_base;
        }
        // many-wave batches (>= 4 waves at five CTAs per SM) of two candidates per lane run the
        // no-producer instance at five CTAs per SM (PESTO_E32_NP=0 disables it);
        // one-wave batches keep room on the SMs for the next batch in flight
        static const bool np_on = [] {
            const char *v = std::getenv("PESTO_E32_NP");
            return !(v && std::atoi(v) == 0);
        }();
        p32.np32 = (np_on && p32.cpl32 == 2 && g->planes == 1 &&
                    p32.n_tasks >= 4 * 5 * (int64_t)g->sms) ? 1 : 0;
        if ((s = ensure_state32(g, ws, p32, 0, p32.n_tasks, &grid))) return s;
        p32.state32 = ws.state32.as<uint32_t>();
        if ((e = launch_eval32(p32, 0, grid, st)) != cudaSuccess) return cuda_fail(e, "launch eval32");
    }
    p.list = p.flag_list;
    p.list_count = p.flag_count;
    const int64_t fix_tasks = std::min<int64_t>(p.n_tasks, g->sms);
    if ((s = ensure_state(g, ws, p, 2, fix_tasks, &grid))) return s;
    p.state = ws.state.as<int64_t>();
    if ((e = launch_eval(p, 2, grid, st)) != cudaSuccess) return cuda_fail(e, "launch eval fixup");
    return PESTO_OK;
}

// rows copied in from host memory, evaluated, makespans copied out -- all enqueued on stream
pesto_status eval_batch_host_ws(pesto_graph *g, Scratch &ws, const int32_t *order, const void *rows,
                                int64_t stride, int64_t n_cand, int64_t *mk_host, void *stream) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    if (g->device < 0) return fail(PESTO_ESTATE, "host-only graph handle");
    if (n_cand <= 0) return n_cand == 0 ? PESTO_OK : fail(PESTO_EINVAL, "n_cand < 0");
    if (!rows || !mk_host) return fail(PESTO_EINVAL, "NULL buffer");
    DeviceGuard guard(g->device);
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e = ws.rows.ensure((size_t)n_cand * stride);
    if (e != cudaSuccess) return cuda_fail(e, "allocate rows");
    if ((e = ws.out.ensure((size_t)n_cand * 8)) != cudaSuccess) return cuda_fail(e, "allocate out");
    if ((e = cudaMemcpyAsync(ws.rows.ptr, rows, (size_t)n_cand * stride, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_fail(e, "copy rows in");
    pesto_status s = eval_batch_ws(g, ws, order, ws.rows.ptr, stride, n_cand, ws.out.as<int64_t>(), stream);
    if (s) return s;
    if ((e = cudaMemcpyAsync(mk_host, ws.out.ptr, (size_t)n_cand * 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
        return cuda_fail(e, "copy makespans out");
    return PESTO_OK;
}

}  // namespace

struct pesto_workspace {
    pesto_graph *g = nullptr;
    Scratch ws;
};

extern "C" {

pesto_status pesto_eval_batch(pesto_graph *g, const int32_t *order, const void *placements,
                              int64_t stride, int64_t n_cand, int64_t *makespans, void *stream) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    NvtxRange nvtx("pesto_eval_batch (K5 + K1)");
    return eval_batch_ws(g, g->ws, order, placements, stride, n_cand, makespans, stream);
}

pesto_status pesto_eval_batch_host(pesto_graph *g, const int32_t *order, const void *rows,
                                   int64_t stride, int64_t n_cand, int64_t *mk_host, void *stream) {
    if (!g) return fail(PESTO_EINVAL, "NULL graph");
    NvtxRange nvtx("pesto_eval_batch_host (H2D + K5 + K1 + D2H)");
    pesto_status s = eval_batch_host_ws(g, g->ws, order, rows, stride, n_cand, mk_host, stream);
    if (s || n_cand == 0) return s;
    DeviceGuard guard(g->device);
    cudaError_t e = cudaStreamSynchronize((cudaStream_t)stream);
    return e == cudaSuccess ? PESTO_OK : cuda_fail(e, "eval_batch_host");
}

pesto_status pesto_workspace_create(pesto_graph *g, pesto_workspace **out) {
    if (!g || !out) return fail(PESTO_EINVAL, "NULL argument");
    *out = nullptr;
    if (g->device < 0) return fail(PESTO_ESTATE, "host-only graph handle");
    pesto_workspace *w = new (std::nothrow) pesto_workspace();
    if (!w) return fail(PESTO_ENOMEM, "workspace");
    w->g = g;
    *out = w;
    return PESTO_OK;
}

void pesto_workspace_destroy(pesto_workspace *w) {
    if (!w) return;
    DeviceGuard guard(w->g->device);
    delete w;                           // DevBuf frees synchronise with the device
}

pesto_status pesto_eval_batch_host_async(pesto_workspace *w, const int32_t *order, const void *rows,
                                         int64_t stride, int64_t n_cand, int64_t *mk_host,
                                         void *stream) {
    if (!w) return fail(PESTO_EINVAL, "NULL workspace");
    NvtxRange nvtx("pesto_eval_batch_host_async");
    return eval_batch_host_ws(w->g, w->ws, order, rows, stride, n_cand, mk_host, stream);
}

}  // extern "C"
