// search.cpp -- parallel local search over placements and orders.
//
// One step = K1 (neighbour decode + makespan + warp argmin, this rank's share of candidate ids)
// -> ncclAllReduce MIN of the packed (makespan << 24 | j) keys across ranks (the only exchange)
// -> K4 commit on every rank (each regenerates the winner from the counter, so bases stay equal).
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "host.h"
#include "moves.cuh"

using namespace pesto;

namespace {

struct NcclApi {
    void *h = nullptr;
    ncclResult_t (*get_unique_id)(ncclUniqueId *) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*all_reduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t,
                               ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    const char *(*error_string)(ncclResult_t) = nullptr;
    bool ok = false;
};

NcclApi &nccl() {
    static NcclApi api;
    static bool tried = false;
    if (tried) return api;
    tried = true;
    // prefer the copy already loaded by the process (torch's), matched by SONAME
    api.h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!api.h) return api;
    api.get_unique_id = (decltype(api.get_unique_id))dlsym(api.h, "ncclGetUniqueId");
    api.comm_init_rank = (decltype(api.comm_init_rank))dlsym(api.h, "ncclCommInitRank");
    api.all_reduce = (decltype(api.all_reduce))dlsym(api.h, "ncclAllReduce");
    api.comm_destroy = (decltype(api.comm_destroy))dlsym(api.h, "ncclCommDestroy");
    api.error_string = (decltype(api.error_string))dlsym(api.h, "ncclGetErrorString");
    api.ok = api.get_unique_id && api.comm_init_rank && api.all_reduce && api.comm_destroy;
    return api;
}

pesto_status nccl_fail(ncclResult_t r, const char *what) {
    const char *s = nccl().error_string ? nccl().error_string(r) : "?";
    return fail(PESTO_ENCCL, std::string(what) + ": " + s);
}

}  // namespace

struct pesto_search {
    pesto_graph *g = nullptr;
    int32_t P = 0;
    int64_t K = 0;
    int32_t mix[4] = {0, 0, 0, 0};
    uint64_t seed = 0;
    int32_t rank = 0, world = 1;
    int64_t j_begin = 0, j_end = 0;
    int32_t tile32 = 0;            // eval32 tile budget of the bases' layouts (0 = automatic)
    int64_t step = 0;
    std::vector<std::vector<int32_t>> order;
    std::vector<std::shared_ptr<Layout>> layouts;
    std::vector<BaseLayoutDev> views;
    DevBuf d_views, d_bits, d_keys, d_mk, d_swap, d_dbg_key;
    int32_t *h_swap = nullptr;
    uint64_t *h_keys = nullptr;
    ncclComm_t comm = nullptr;
    cudaStream_t last_stream = nullptr;
    int32_t max_W = 1, stage_bytes = 16, max_W32 = 1, stage_bytes32 = 16;
    // upper bounds of the base makespans known on the host (they never increase): once all are
    // below kSat32 every base runs on eval32 and the 64-bit kernel is not launched at all
    std::vector<int64_t> h_mk;
    bool all_below = false;
    bool use32 = false;            // eval32 records exist for every base
    // row f3: footprint of each base per device ([P][8]), for the constraints of cons_gen
    DevBuf d_fbase;
    int64_t cons_gen = -1;
    // the comm model the bases' layouts were built with (their edge records hold the transfer
    // times); a later pesto_comm_model makes the search fail with ESTATE instead of walking
    // stale records
    int64_t comm_gen = -1;
    // committed swaps: patched in place on the device vs. layout rebuilt on the host
    DevBuf d_patch;
    int64_t n_swap_inplace = 0, n_swap_rebuilt = 0;
    // search spec S9 (row f2 group moves): merged vertex of every op, and per base the merged
    // vertex of the op at each position ([P][n], kept in step with committed swaps)
    int32_t n_coarse = 0, coarse_pct = 0;
    std::vector<int32_t> coarse_of;
    std::vector<uint8_t> cpos;
    DevBuf d_cpos;
    // the wide eval32 launch (bases at or above saturation) runs on `aux`, forked from and
    // joined back into the caller's stream, beside the 32-bit launch
    cudaStream_t aux = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    // bases whose special-position lists overflowed during an in-place swap patch
    std::vector<int> spec_rebuild;
    // without swap moves a commit does not read the base makespans back synchronously: it
    // copies them into pinned h_mk_async and the next eval picks them up once the copy is done
    // (the device gates every base itself; this only stops the wide launch when none needs it)
    int64_t *h_mk_async = nullptr;
    cudaEvent_t ev_mk = nullptr;
    bool mk_pending = false;
};

namespace {

void refresh_views(pesto_search *s) {
    s->max_W = 1;
    s->stage_bytes = 16;
    s->max_W32 = 1;
    s->stage_bytes32 = 16;
    s->use32 = s->g->eligible32;
    for (int b = 0; b < s->P; b++) {
        if (s->layouts[b]->W32 == 0) s->use32 = false;
        s->views[b] = layout_view(*s->layouts[b]);
        s->views[b].bits = s->d_bits.as<uint32_t>() + (size_t)b * s->g->planes * s->g->words;
        s->views[b].coarse_pos = s->cpos.empty() ? nullptr : s->d_cpos.as<uint8_t>() + (size_t)b * s->g->n;
        s->max_W = std::max(s->max_W, s->layouts[b]->W);
        s->stage_bytes = std::max(s->stage_bytes, s->layouts[b]->stage_bytes);
        s->max_W32 = std::max(s->max_W32, s->layouts[b]->W32);
        s->stage_bytes32 = std::max(s->stage_bytes32, s->layouts[b]->stage_bytes32);
    }
}

void update_all_below(pesto_search *s) {
    s->all_below = s->use32;
    for (int64_t mk : s->h_mk)
        if (mk >= (int64_t)kSat32) s->all_below = false;
}

pesto_status download_x(pesto_search *s, int b, uint8_t *x_op);

// row f3: (re)compute the bases' footprints when the graph's constraints changed; the bases
// must satisfy the new constraints
pesto_status sync_constraints(pesto_search *s) {
    pesto_graph *g = s->g;
    if (s->cons_gen == g->cons_gen) return PESTO_OK;
    std::vector<int64_t> fb((size_t)s->P * 8, 0);
    std::vector<uint8_t> x(g->n);
    for (int b = 0; b < s->P; b++) {
        pesto_status rc = download_x(s, b, x.data());
        if (rc) return rc;
        if (!placement_feasible(g, x.data(), fb.data() + (size_t)b * 8))
            return fail(PESTO_ESTATE, "search base " + std::to_string(b) + " violates the constraints");
    }
    cudaError_t e;
    if ((e = s->d_fbase.ensure(fb.size() * 8)) != cudaSuccess ||
        (e = cudaMemcpy(s->d_fbase.ptr, fb.data(), fb.size() * 8, cudaMemcpyHostToDevice)) != cudaSuccess)
        return cuda_fail(e, "upload base footprints");
    s->cons_gen = g->cons_gen;
    return PESTO_OK;
}

// row f4(i): every candidate on the non-delay kernel (one warp each); the bases' producer-grouped
// edge orders are built on demand (a committed swap never reorders a producer's consumers: the
// S3 rule blocks pairs that share a producer)
pesto_status launch_search_nondelay(pesto_search *s, int b_first, int n_bases, int64_t j0, int64_t j1,
                                    uint64_t *keys, uint64_t *keys_dbg, cudaStream_t st) {
    pesto_graph *g = s->g;
    pesto_status rc = nd_check(g);
    if (rc) return rc;
    bool changed = false;
    for (int b = 0; b < s->P; b++) {
        void *before = s->layouts[b]->d_nd_dst.ptr;
        const int64_t gen = s->layouts[b]->nd_gen;
        if ((rc = nd_ensure_layout(g, *s->layouts[b]))) return rc;
        changed |= before != s->layouts[b]->d_nd_dst.ptr || gen != s->layouts[b]->nd_gen;
    }
    cudaError_t e;
    if (changed) {
        refresh_views(s);
        if ((e = cudaMemcpyAsync(s->d_views.ptr, s->views.data(), sizeof(BaseLayoutDev) * s->P,
                                 cudaMemcpyHostToDevice, st)) != cudaSuccess)
            return cuda_fail(e, "upload views");
        if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_fail(e, "upload views");
    }
    NdParams p;
    int grid = 0;
    const int64_t n_tasks = (int64_t)n_bases * (j1 - j0);
    if ((rc = nd_fill(g, g->ws, p, n_tasks, &grid))) return rc;
    p.feas.fbase = s->d_fbase.as<int64_t>() + (size_t)b_first * 8;
    p.bases = s->d_views.as<BaseLayoutDev>() + b_first;
    p.n_bases = n_bases;
    p.b_offset = b_first;
    p.P_total = s->P;
    p.j_begin = j0;
    p.j_end = j1;
    p.seed = s->seed;
    p.step = (uint64_t)s->step;
    std::memcpy(p.mix, s->mix, sizeof p.mix);
    p.allowed_op = g->d_allowed.as<uint8_t>();
    p.keys = keys;
    p.keys_dbg = keys_dbg;
    p.n_coarse = s->n_coarse;
    p.coarse_pct = s->coarse_pct;
    if ((e = launch_nondelay(p, 1, grid, st)) != cudaSuccess) return cuda_fail(e, "launch non-delay search");
    return PESTO_OK;
}

// fast: eval32 for the bases below saturation (+ eval64 for the others while any may exist);
// otherwise (debug keys, initial makespans, ineligible graphs) eval64 for all candidates
// cpl_force (1 or 2): the candidates-per-lane instance to launch instead of the one this range
// alone would choose -- the parity path runs the instance the full step launches
pesto_status launch_search_eval(pesto_search *s, int b_first, int n_bases, int64_t j0, int64_t j1,
                                uint64_t *keys, uint64_t *keys_dbg, cudaStream_t st,
                                bool fast = false, int cpl_force = 0, bool wide_all = false) {
    pesto_graph *g = s->g;
    if (j1 <= j0) return PESTO_OK;
    if (s->comm_gen >= 0 && s->comm_gen != g->comm_gen)
        return fail(PESTO_ESTATE, "the comm model changed after the search was created");
    pesto_status rc0 = sync_constraints(s);
    if (rc0) return rc0;
    if (s->coarse_pct > 0 && (g->has_cap || g->has_coloc))
        return fail(PESTO_ESTATE, "coarse group moves (S9) cannot be combined with row-f3 constraints");
    if (g->dispatch == PESTO_DISPATCH_NONDELAY)
        return launch_search_nondelay(s, b_first, n_bases, j0, j1, keys, keys_dbg, st);
    EvalParams p;
    fill_eval_common(g, p);
    p.feas.fbase = s->d_fbase.as<int64_t>() + (size_t)b_first * 8;
    p.stage_bytes = s->stage_bytes;
    p.max_W = s->max_W;
    p.stage_bytes32 = s->stage_bytes32;
    p.max_W32 = s->max_W32;
    p.base_mk = s->d_mk.as<int64_t>() + b_first;
    p.bases = s->d_views.as<BaseLayoutDev>() + b_first;
    p.b_offset = b_first;
    p.P_total = s->P;
    p.j_begin = j0;
    p.j_end = j1;
    p.seed = s->seed;
    p.step = (uint64_t)s->step;
    std::memcpy(p.mix, s->mix, sizeof p.mix);
    p.movable = g->d_movable.as<int32_t>();
    p.n_movable = (int32_t)g->movable.size();
    p.allowed_op = g->d_allowed.as<uint8_t>();
    p.keys = keys;
    p.keys_dbg = keys_dbg;
    p.n_coarse = s->n_coarse;
    p.coarse_pct = s->coarse_pct;
    p.coarse_pos = s->cpos.empty() ? nullptr : s->d_cpos.as<uint8_t>() + (size_t)b_first * g->n;
    p.group_begin = j0 >> 5;
    p.groups_per_base = ((j1 - 1) >> 5) - p.group_begin + 1;
    p.tasks_per_base = (p.groups_per_base + kWarps - 1) / kWarps;
    p.n_tasks = p.tasks_per_base * n_bases;
    int grid = 0;
    pesto_status rc;
    cudaError_t e;
    if (s->mk_pending && cudaEventQuery(s->ev_mk) == cudaSuccess) {   // non-blocking refresh
        std::memcpy(s->h_mk.data(), s->h_mk_async, 8 * s->P);
        s->mk_pending = false;
        update_all_below(s);
    }
    const bool use32 = fast && s->use32 && g->link_model == PESTO_LINKS_FCFS;   // f4(ii): eval64
    if (use32) {
        // eval32 tasks: consecutive ids from a multiple of the task size
        EvalParams p32 = p;
        p32.gate = 1;
        plan_eval32(g, p32, j0, j1, n_bases);
        if (cpl_force == 1 || cpl_force == 2) {
            p32.cpl32 = cpl_force;
            const int64_t ts = eval32_task_size(cpl_force);
            p32.tasks_per_base = (j1 - (j0 - j0 % ts) + ts - 1) / ts;
            p32.n_tasks = p32.tasks_per_base * n_bases;
        }
        if (wide_all) {
            // every candidate of the range on the wide (exact 64-bit) instance, whatever its
            // base's makespan: the parity path's exact keys of saturated 32-bit walks
            p32.gate = 0;
            p32.wide32 = 1;
            p32.cpl32 = 1;
            const int64_t ts = eval32_task_size(1);
            p32.tasks_per_base = (j1 - (j0 - j0 % ts) + ts - 1) / ts;
            p32.n_tasks = p32.tasks_per_base * n_bases;
            if ((rc = ensure_state32(g, g->ws, p32, 1, p32.n_tasks, &grid, true))) return rc;
            p32.state32 = g->ws.state32w.as<uint32_t>();
            if ((e = launch_eval32(p32, 1, grid, st)) != cudaSuccess) return cuda_fail(e, "launch wide eval32");
            return PESTO_OK;
        }
        // launched alone (no wide launch beside it), the two-candidates-per-lane 32-bit walk
        // runs without a producer warp at five CTAs per SM (PESTO_E32_NP=0
        // keeps the producer warp): transformer_2dev 35.9 -> 35.0 ms per step.  Beside a wide
        // launch (nmt4's saturated bases) the producer instance is faster (29.0 vs 31.7 ms).
        static const bool np_on = [] {
            const char *e = std::getenv("PESTO_E32_NP");
            return !(e && std::atoi(e) == 0);
        }();
        p32.np32 = (np_on && s->all_below && p32.cpl32 == 2 && g->planes == 1) ? 1 : 0;
        if ((rc = ensure_state32(g, g->ws, p32, 1, p32.n_tasks, &grid))) return rc;
        p32.state32 = g->ws.state32.as<uint32_t>();
        if (s->all_below) {
            if ((e = launch_eval32(p32, 1, grid, st)) != cudaSuccess) return cuda_fail(e, "launch eval32");
            return PESTO_OK;
        }
        // some bases are at or above saturation: their wide launch runs on the auxiliary
        // stream beside this one (own cold-slot buffer; disjoint bases, so disjoint keys)
        if (!s->aux) {
            if ((e = cudaStreamCreateWithFlags(&s->aux, cudaStreamNonBlocking)) != cudaSuccess ||
                (e = cudaEventCreateWithFlags(&s->ev_fork, cudaEventDisableTiming)) != cudaSuccess ||
                (e = cudaEventCreateWithFlags(&s->ev_join, cudaEventDisableTiming)) != cudaSuccess)
                return cuda_fail(e, "auxiliary stream");
        }
        if ((e = cudaEventRecord(s->ev_fork, st)) != cudaSuccess ||
            (e = cudaStreamWaitEvent(s->aux, s->ev_fork, 0)) != cudaSuccess)
            return cuda_fail(e, "fork");
        if ((e = launch_eval32(p32, 1, grid, st)) != cudaSuccess) return cuda_fail(e, "launch eval32");
        // bases at or above saturation: the wide eval32 instance (exact 64-bit times, the
        // same step records) -- about 2x the throughput of eval64 there
        p32.gate = 2;
        p32.wide32 = 1;
        // one candidate per lane: the 64-bit state of two would spill at 4 CTAs/SM (measured on
        // nmt4: CPL 1 5.17 vs CPL 2 4.96 M cand/s); PESTO_WIDE_CPL overrides for experiments
        {
            const char *w = std::getenv("PESTO_WIDE_CPL");
            const int c = (w && std::atoi(w) == 2) ? 2 : 1;
            p32.cpl32 = c;
            const int64_t ts = eval32_task_size(c);
            p32.tasks_per_base = (j1 - (j0 - j0 % ts) + ts - 1) / ts;
            p32.n_tasks = p32.tasks_per_base * n_bases;
        }
        if ((rc = ensure_state32(g, g->ws, p32, 1, p32.n_tasks, &grid, true))) return rc;
        p32.state32 = g->ws.state32w.as<uint32_t>();
        if ((e = launch_eval32(p32, 1, grid, s->aux)) != cudaSuccess) return cuda_fail(e, "launch wide eval32");
        if ((e = cudaEventRecord(s->ev_join, s->aux)) != cudaSuccess ||
            (e = cudaStreamWaitEvent(st, s->ev_join, 0)) != cudaSuccess)
            return cuda_fail(e, "join");
        return PESTO_OK;
    }
    if ((rc = ensure_state(g, g->ws, p, 1, p.n_tasks, &grid))) return rc;
    p.state = g->ws.state.as<int64_t>();
    if ((e = launch_eval(p, 1, grid, st)) != cudaSuccess) return cuda_fail(e, "launch search eval");
    return PESTO_OK;
}

pesto_status upload_bits(pesto_search *s, int b, const uint8_t *x_op) {
    pesto_graph *g = s->g;
    std::vector<uint32_t> bits((size_t)g->planes * g->words, 0);
    const Layout &L = *s->layouts[b];
    for (int32_t q = 0; q < g->n; q++) {
        const int x = x_op[L.order[q]];
        for (int k = 0; k < g->planes; k++)
            if ((x >> k) & 1) bits[(size_t)k * g->words + (q >> 5)] |= 1u << (q & 31);
    }
    cudaError_t e = cudaMemcpy(s->d_bits.as<uint32_t>() + (size_t)b * bits.size(), bits.data(),
                               bits.size() * 4, cudaMemcpyHostToDevice);
    return e == cudaSuccess ? PESTO_OK : cuda_fail(e, "upload base placement");
}

// the base placement by op id, from the device bit planes (position space of order[b])
pesto_status download_x(pesto_search *s, int b, uint8_t *x_op) {
    pesto_graph *g = s->g;
    std::vector<uint32_t> bits((size_t)g->planes * g->words);
    cudaError_t e = cudaMemcpy(bits.data(), s->d_bits.as<uint32_t>() + (size_t)b * bits.size(),
                               bits.size() * 4, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_fail(e, "read placement");
    for (int32_t q = 0; q < g->n; q++) {
        int x = 0;
        for (int k = 0; k < g->planes; k++)
            x |= (int)((bits[(size_t)k * g->words + (q >> 5)] >> (q & 31)) & 1u) << k;
        x_op[s->order[b][q]] = (uint8_t)x;
    }
    return PESTO_OK;
}

// ---------------------------------------------------------------------------------------------
// In-place patch of a committed adjacent swap (k, k+1) of base b.
// Under the v4 rule (§4 S3) the two ops share no edge, producer or consumer, so only local
// records change: the two ops' record blocks exchange places inside their tile, their in-edge
// records get the new successor positions (and, in eval32, targets), the eval32 heads that name
// their cold slots for prefetch are re-pointed, and the position-indexed arrays are updated.
// The slot colourings are kept; the swap is refused (-> full rebuild) when that would break the
// padded-interval invariant of §3.3, when an edge would change between near and far, or when
// the pair spans two tiles.  The host copies are patched the same way; the device copies are
// patched by one kernel (their embedded base codes are newer than the host's and are kept).
// ---------------------------------------------------------------------------------------------
struct Patcher {
    std::vector<PatchOp> ops;
    int max_block = 0;
    void set32(const DevBuf &d, uint8_t *host, size_t off, uint32_t mask, uint32_t val) {
        uint32_t w;
        std::memcpy(&w, host + off, 4);
        w = (w & ~mask) | (val & mask);
        std::memcpy(host + off, &w, 4);
        ops.push_back(PatchOp{(uint64_t)(uintptr_t)(d.as<uint8_t>() + off), kPatchSet32, 0, 0, mask, val, 0});
    }
    template <class T>
    void set_elem(const DevBuf &d, std::vector<T> &host, size_t i, T val) {
        static_assert(sizeof(T) == 4 || sizeof(T) == 1, "4- or 1-byte elements");
        host[i] = val;
        uint32_t v = 0;
        std::memcpy(&v, &val, sizeof(T));
        ops.push_back(PatchOp{(uint64_t)(uintptr_t)(d.as<uint8_t>() + i * sizeof(T)),
                              sizeof(T) == 4 ? (uint32_t)kPatchSet32 : (uint32_t)kPatchSet8, 0, 0,
                              ~0u, v, 0});
    }
    void rotate(const DevBuf &d, std::vector<uint8_t> &host, size_t off, uint32_t a, uint32_t b) {
        std::rotate(host.begin() + off, host.begin() + off + a, host.begin() + off + a + b);
        ops.push_back(PatchOp{(uint64_t)(uintptr_t)(d.as<uint8_t>() + off), kPatchRotate, a, b, 0, 0, 0});
        max_block = std::max(max_block, (int)(a + b));
    }
};

bool swap_in_place(pesto_search *s, int b, int32_t k, Patcher &pt) {
    pesto_graph *g = s->g;
    Layout &L = *s->layouts[b];
    const int32_t n = g->n;
    if (k < 0 || k + 1 >= n || L.slot64.empty()) return false;
    const int32_t a = L.order[k], c = L.order[k + 1];
    const bool has32 = L.W32 > 0;
    const int C = g->n_classes;
    const int es = edge_stride_for(C);
    auto nout = [&](int32_t op) { return g->out_off[op + 1] - g->out_off[op]; };
    auto heavy64 = [&](int32_t op) { return nout(op) * es > kMaxInlineBytes; };
    auto size64 = [&](int32_t op) { return (uint32_t)(heavy64(op) ? 32 : 16 + nout(op) * es); };
    auto nst = [&](int32_t op) { return (uint32_t)std::max<int64_t>(1, (nout(op) + 1) / 2); };
    auto npos = [&](int32_t op) { return op == a ? k + 1 : (op == c ? k : L.pos[op]); };
    auto cls = [](int32_t d) { return d == 1 ? 0 : (d <= kNearDelta ? 1 : 2); };
    const int32_t prev = k >= 1 ? L.order[k - 1] : -1;
    const int32_t p2 = k + 2 < n ? L.order[k + 2] : -1;

    // ---- checks (nothing is modified before all pass) ----
    if (L.tile64_of[k] != L.tile64_of[k + 1]) return false;
    if (size64(a) + size64(c) > (uint32_t)kPatchMaxBlock) return false;
    if (has32) {
        if (L.tile32_of[k] != L.tile32_of[k + 1]) return false;
        if ((nst(a) + nst(c)) * kStepBytes > (uint32_t)kPatchMaxBlock) return false;
        for (int32_t op : {a, c}) {
            for (int64_t i = g->in_off[op]; i < g->in_off[op + 1]; i++) {
                const int64_t e = g->in_edges[i];
                const int32_t u = g->src[e];
                if ((cls(L.pos[op] - L.pos[u]) == 2) != (cls(npos(op) - npos(u)) == 2)) return false;
            }
            for (int64_t i = g->out_off[op]; i < g->out_off[op + 1]; i++) {
                const int32_t w = g->dst[g->out_edges[i]];
                if ((cls(L.pos[w] - L.pos[op]) == 2) != (cls(npos(w) - npos(op)) == 2)) return false;
            }
        }
    }
    // padded intervals (§3.3): a's interval now ends at k+2; consumers first fed by c now start at k
    auto intervals_ok = [&](const std::vector<int32_t> &first, const std::vector<int32_t> &slot,
                            bool far_only) {
        auto counts = [&](int32_t u, int32_t w) {       // does edge u -> w open w's interval?
            return !far_only || cls(npos(w) - npos(u)) == 2;
        };
        if (slot[a] >= 0 && first[a] >= 0 && p2 >= 0) {
            for (int64_t i = g->out_off[p2]; i < g->out_off[p2 + 1]; i++) {
                const int32_t u = g->dst[g->out_edges[i]];
                if (counts(p2, u) && first[u] == k + 2 && slot[u] == slot[a]) return false;
            }
        }
        if (prev >= 0 && first[prev] >= 0 && slot[prev] >= 0) {
            for (int64_t i = g->out_off[c]; i < g->out_off[c + 1]; i++) {
                const int32_t u = g->dst[g->out_edges[i]];
                if (counts(c, u) && first[u] == k + 1 && slot[u] == slot[prev]) return false;
            }
        }
        return true;
    };
    if (!intervals_ok(L.first64, L.slot64, false)) return false;
    if (has32 && !intervals_ok(L.first_far, L.cslot, true)) return false;

    // ---- order, positions, per-position arrays ----
    std::swap(L.order[k], L.order[k + 1]);
    L.pos[a] = k + 1;
    L.pos[c] = k;
    pt.set_elem(L.d_order, L.order, k, c);
    pt.set_elem(L.d_order, L.order, k + 1, a);
    pt.set_elem(L.d_pos, L.pos, a, k + 1);
    pt.set_elem(L.d_pos, L.pos, c, k);
    pt.set_elem(L.d_allowed_pos, L.allowed_pos, k, g->allowed[c]);
    pt.set_elem(L.d_allowed_pos, L.allowed_pos, k + 1, g->allowed[a]);
    for (int32_t q = std::max(0, k - 1); q <= k + 1 && q + 1 < n; q++)
        pt.set_elem(L.d_adj, L.swap_blocked, q, (uint8_t)(pair_blocked(g, L.order[q], L.order[q + 1]) ? 1 : 0));
    // first producer positions of the consumers of a and c
    auto refirst = [&](int32_t u, std::vector<int32_t> &first, bool far_only) {
        int32_t f = -1;
        for (int64_t i = g->in_off[u]; i < g->in_off[u + 1]; i++) {
            const int32_t p = L.pos[g->src[g->in_edges[i]]];
            if (far_only && cls(L.pos[u] - p) != 2) continue;
            if (f < 0 || p < f) f = p;
        }
        first[u] = f;
    };

    // ---- eval64 stream ----
    {
        const uint32_t off = L.op_off64[k], A = size64(a), B = size64(c);
        pt.rotate(L.d_blob, L.blob, off, A, B);
        L.op_off64[k] = off;
        L.op_off64[k + 1] = off + B;
        if (!heavy64(a))
            for (int64_t i = g->out_off[a]; i < g->out_off[a + 1]; i++) L.eloc64[g->out_edges[i]] += B;
        if (!heavy64(c))
            for (int64_t i = g->out_off[c]; i < g->out_off[c + 1]; i++) L.eloc64[g->out_edges[i]] -= A;
        for (int32_t op : {a, c}) {
            for (int64_t i = g->in_off[op]; i < g->in_off[op + 1]; i++) {
                const uint32_t loc = L.eloc64[g->in_edges[i]];
                const bool hv = (loc & kPinHeavy) != 0;
                pt.set32(hv ? L.d_heavy : L.d_blob, hv ? L.heavy.data() : L.blob.data(),
                         (loc & ~kPinHeavy) + 8, ~0u, (uint32_t)L.pos[op]);
            }
            for (int64_t i = g->out_off[op]; i < g->out_off[op + 1]; i++)
                refirst(g->dst[g->out_edges[i]], L.first64, false);
        }
    }

    // ---- eval32 stream ----
    if (has32) {
        const uint32_t off = L.op_off32[k], A = nst(a) * kStepBytes, B = nst(c) * kStepBytes;
        pt.rotate(L.d_blob32, L.blob32, off, A, B);
        pt.set_elem(L.d_op_off32, L.op_off32, k, off);
        pt.set_elem(L.d_op_off32, L.op_off32, k + 1, off + B);
        // records of the out-edges of a and c moved: their locations and patch-index entries
        // (one pass per successor over its entries, old -> new, so parallel edges stay exact)
        for (int32_t op : {a, c}) {
            const uint32_t base = op == a ? off : off + A, len = op == a ? A : B;   // old block
            const uint32_t shift = op == a ? B : (uint32_t)(0u - A);       // mod 2^32
            std::vector<int32_t> succ_q;
            for (int64_t i = g->out_off[op]; i < g->out_off[op + 1]; i++)
                succ_q.push_back(L.pos[g->dst[g->out_edges[i]]]);
            std::sort(succ_q.begin(), succ_q.end());
            succ_q.erase(std::unique(succ_q.begin(), succ_q.end()), succ_q.end());
            for (int32_t q : succ_q)                  // entries into op's old block move with it
                for (uint32_t r = L.pin_off[q]; r < L.pin_off[q + 1]; r++)
                    if ((L.pin_ref[r] & kPinOffMask) >= base && (L.pin_ref[r] & kPinOffMask) < base + len)
                        pt.set_elem(L.d_pin_ref, L.pin_ref, r, L.pin_ref[r] + shift);
            for (int64_t i = g->out_off[op]; i < g->out_off[op + 1]; i++)
                L.eloc32[g->out_edges[i]] += shift;
        }
        // patch index of positions k (now c) and k+1 (now a)
        {
            uint32_t r = L.pin_off[k];
            for (int64_t i = g->in_off[c]; i < g->in_off[c + 1]; i++)
                pt.set_elem(L.d_pin_ref, L.pin_ref, r++, L.eloc32[g->in_edges[i]]);
            pt.set_elem(L.d_pin_off, L.pin_off, k + 1, r);
            for (int64_t i = g->in_off[a]; i < g->in_off[a + 1]; i++)
                pt.set_elem(L.d_pin_ref, L.pin_ref, r++, L.eloc32[g->in_edges[i]]);
        }
        for (int32_t op : {a, c})
            for (int64_t i = g->out_off[op]; i < g->out_off[op + 1]; i++)
                refirst(g->dst[g->out_edges[i]], L.first_far, true);
        // targets of every in-edge of a, c and the op after them (NEXT <-> NEAR may change there)
        auto retarget = [&](int32_t w) {
            const int32_t q = L.pos[w];
            int64_t near_first = -1, far_first = -1;
            int32_t near_p = 0, far_p = 0;
            for (int64_t i = g->in_off[w]; i < g->in_off[w + 1]; i++) {   // ascending edge id
                const int64_t e = g->in_edges[i];
                const int32_t p = L.pos[g->src[e]];
                const int cl = cls(q - p);
                if (cl == 1 && (near_first < 0 || p < near_p)) { near_first = e; near_p = p; }
                if (cl == 2 && (far_first < 0 || p < far_p)) { far_first = e; far_p = p; }
            }
            for (int64_t i = g->in_off[w]; i < g->in_off[w + 1]; i++) {
                const int64_t e = g->in_edges[i];
                const int cl = cls(q - L.pos[g->src[e]]);
                const uint32_t tgt = cl == 0 ? kT32Next
                                   : cl == 1 ? (kT32Near | (uint32_t)(q & (kRing - 1)) * 128u |
                                                (e == near_first ? kT32First : 0u))
                                             : ((uint32_t)L.cslot[w] * 128u | (e == far_first ? kT32First : 0u));
                const uint32_t loc = L.eloc32[e] & kPinOffMask;
                const uint32_t slot = (L.eloc32[e] & kPinSlot) ? 1u : 0u;
                pt.set32(L.d_blob32, L.blob32.data(), loc + 4, kSuccPosMask | kSuccTcMask,
                         (uint32_t)q | (target_class32(tgt) << kSuccTcShift));
                pt.set32(L.d_blob32, L.blob32.data(), loc + 8, ~0u, tgt);
                if (g->D <= 4)        // the fast walk's dispatch entry of the slot: class bits
                    pt.set32(L.d_blob32, L.blob32.data(), loc - 16 * (slot + 1) + 4,
                             (7u << kind_cshift(g->D)) << (8 * slot),
                             (target_class32(tgt) << kind_cshift(g->D)) << (8 * slot));
            }
            pt.set32(L.d_blob32, L.blob32.data(), L.op_off32[q] + 12, kStHasNear,
                     near_first >= 0 ? kStHasNear : 0u);
        };
        retarget(a);
        retarget(c);
        if (p2 >= 0) retarget(p2);
        // heads that name a cold slot for prefetch: q names the op at q + kPrefetchDist
        for (int32_t q : {k - kPrefetchDist, k + 1 - kPrefetchDist, k, k + 1}) {
            if (q < 0 || q >= n) continue;
            const int32_t ahead = q + kPrefetchDist;
            const int32_t pf = ahead < n ? L.cslot[L.order[ahead]] : -1;
            pt.set32(L.d_blob32, L.blob32.data(), L.op_off32[q] + 8, ~0u, (uint32_t)pf);
        }
        // special positions of the regions the swap can touch: the regions of k and k+1 (a and c
        // change region when they straddle a boundary) and those of every successor of a or c
        // (their producer positions changed); rewritten in place within each list's capacity
        if (!L.spec_off.empty()) {
            std::vector<int32_t> regs{k / kRegion, (k + 1) / kRegion};
            for (int32_t op : {a, c})
                for (int64_t i = g->out_off[op]; i < g->out_off[op + 1]; i++)
                    regs.push_back(L.pos[g->dst[g->out_edges[i]]] / kRegion);
            std::sort(regs.begin(), regs.end());
            regs.erase(std::unique(regs.begin(), regs.end()), regs.end());
            std::vector<int32_t> lst;
            bool fits = true;
            for (int32_t r : regs) {
                spec_region(g, L, r, lst);
                if (lst.size() + 1 > (size_t)(L.spec_off[r + 1] - L.spec_off[r])) fits = false;
            }
            if (!fits) {                     // rare: rebuild this base's lists (host + upload)
                s->spec_rebuild.push_back(b);
            } else {
                for (int32_t r : regs) {
                    spec_region(g, L, r, lst);
                    const uint32_t o = L.spec_off[r], cap = L.spec_off[r + 1] - o;
                    for (uint32_t i = 0; i < cap; i++) {
                        const int32_t val = i < lst.size() ? lst[i] : INT32_MAX;
                        if (L.spec_pos[o + i] != val) pt.set_elem(L.d_spec_pos, L.spec_pos, o + i, val);
                    }
                }
            }
        }
    }
    return true;
}

// rebuild the special-position lists of a layout whose in-place rewrite overflowed a region's
// capacity (fresh slack everywhere), and upload them
pesto_status rebuild_spec(pesto_graph *g, Layout &L) {
    const int32_t n = g->n, R = (n + kRegion - 1) / kRegion;
    L.spec_off.assign((size_t)R + 1, 0);
    L.spec_pos.clear();
    std::vector<int32_t> lst;
    for (int32_t r = 0; r < R; r++) {
        L.spec_off[r] = (uint32_t)L.spec_pos.size();
        spec_region(g, L, r, lst);
        L.spec_pos.insert(L.spec_pos.end(), lst.begin(), lst.end());
        L.spec_pos.insert(L.spec_pos.end(), (size_t)kSpecSlack, INT32_MAX);
    }
    L.spec_off[R] = (uint32_t)L.spec_pos.size();
    cudaError_t e;
    if ((e = L.d_spec_off.ensure(L.spec_off.size() * 4)) != cudaSuccess ||
        (e = cudaMemcpy(L.d_spec_off.ptr, L.spec_off.data(), L.spec_off.size() * 4,
                        cudaMemcpyHostToDevice)) != cudaSuccess ||
        (e = L.d_spec_pos.ensure(L.spec_pos.size() * 4)) != cudaSuccess ||
        (e = cudaMemcpy(L.d_spec_pos.ptr, L.spec_pos.data(), L.spec_pos.size() * 4,
                        cudaMemcpyHostToDevice)) != cudaSuccess)
        return cuda_fail(e, "upload special positions");
    return PESTO_OK;
}

}  // namespace

extern "C" {

pesto_status pesto_nccl_unique_id(uint8_t *out128) {
    if (!out128) return fail(PESTO_EINVAL, "NULL argument");
    if (!nccl().ok) return fail(PESTO_ENCCL, "libnccl.so.2 not loadable");
    ncclUniqueId id;
    ncclResult_t r = nccl().get_unique_id(&id);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    std::memcpy(out128, &id, sizeof id);
    return PESTO_OK;
}

pesto_status pesto_search_create(pesto_graph *g, const pesto_search_desc *d, pesto_search **out) {
    if (!g || !d || !out) return fail(PESTO_EINVAL, "NULL argument");
    *out = nullptr;
    if (g->device < 0) return fail(PESTO_ESTATE, "host-only graph handle");
    if (d->n_bases < 1 || d->n_bases > 1024) return fail(PESTO_EINVAL, "n_bases out of range");
    if (d->k_per_base < 1 || d->k_per_base > (int64_t(1) << 24))
        return fail(PESTO_EINVAL, "k_per_base must be in 1..2^24");
    if (!d->base_x || !d->base_order) return fail(PESTO_EINVAL, "NULL base arrays");
    for (int i = 0; i < 4; i++)
        if (d->mix[i] < 0) return fail(PESTO_EINVAL, "negative move weight");
    if (d->mix[3] > 100) return fail(PESTO_EINVAL, "swap percentage > 100");
    if (d->world < 1 || d->rank < 0 || d->rank >= d->world) return fail(PESTO_EINVAL, "bad rank/world");
    const int32_t n = g->n;
    for (int64_t i = 0; i < (int64_t)d->n_bases * n; i++) {
        const int32_t v = (int32_t)(i % n);
        if (d->base_x[i] >= g->D || !((g->allowed[v] >> d->base_x[i]) & 1))
            return fail(PESTO_EINVAL, "infeasible base placement at op " + std::to_string(v));
    }
    for (int b = 0; b < d->n_bases; b++)                  // row f3 constraints
        if (!placement_feasible(g, d->base_x + (size_t)b * n, nullptr))
            return fail(PESTO_EINVAL, "base " + std::to_string(b) + " violates the graph's constraints");
    DeviceGuard guard(g->device);
    std::unique_ptr<pesto_search> s(new pesto_search());
    s->g = g;
    s->P = d->n_bases;
    s->K = d->k_per_base;
    std::memcpy(s->mix, d->mix, sizeof s->mix);
    s->seed = d->seed;
    s->rank = d->rank;
    s->world = d->world;
    s->j_begin = s->K * d->rank / d->world;
    s->j_end = s->K * (d->rank + 1) / d->world;
    s->order.resize(s->P);
    s->layouts.resize(s->P);
    s->views.resize(s->P);
    cudaError_t e;
    if ((e = s->d_bits.ensure((size_t)s->P * g->planes * g->words * 4)) != cudaSuccess)
        return cuda_fail(e, "allocate");
    {
        // a search whose launches run one candidate per lane (one wave: inception's 64 K) keeps
        // 8 KB tiles; the 6 KB tiles of D = 2 layouts serve the five-CTA instance of the
        // two-per-lane launches (inception with 6 KB tiles: 4.10 -> 4.12 ms)
        EvalParams plan;
        fill_eval_common(g, plan);
        plan_eval32(g, plan, s->j_begin, s->j_end, s->P);
        s->tile32 = plan.cpl32 == 1 ? kTileTarget : 0;
    }
    for (int b = 0; b < s->P; b++) {
        s->order[b].assign(d->base_order + (size_t)b * n, d->base_order + (size_t)(b + 1) * n);
        pesto_status rc = build_layout(g, s->order[b].data(), s->layouts[b], false,
                                       d->base_x + (size_t)b * n, s->tile32);
        if (rc) return rc;
        if ((rc = upload_layout(g, *s->layouts[b]))) return rc;
        if ((rc = upload_bits(s.get(), b, d->base_x + (size_t)b * n))) return rc;
    }
    s->comm_gen = g->comm_gen;
    if ((e = s->d_views.ensure(sizeof(BaseLayoutDev) * s->P)) != cudaSuccess) return cuda_fail(e, "allocate");
    refresh_views(s.get());
    if ((e = cudaMemcpy(s->d_views.ptr, s->views.data(), sizeof(BaseLayoutDev) * s->P,
                        cudaMemcpyHostToDevice)) != cudaSuccess)
        return cuda_fail(e, "upload views");
    if ((e = s->d_keys.ensure(8 * s->P)) != cudaSuccess) return cuda_fail(e, "allocate");
    if ((e = s->d_mk.ensure(8 * s->P)) != cudaSuccess) return cuda_fail(e, "allocate");
    if ((e = s->d_swap.ensure(4 * s->P)) != cudaSuccess) return cuda_fail(e, "allocate");
    if ((e = s->d_dbg_key.ensure(8)) != cudaSuccess) return cuda_fail(e, "allocate");
    if ((e = cudaMallocHost((void **)&s->h_swap, 4 * s->P)) != cudaSuccess) return cuda_fail(e, "pinned");
    if ((e = cudaMallocHost((void **)&s->h_keys, 8 * s->P)) != cudaSuccess) return cuda_fail(e, "pinned");
    // initial base makespans: candidate j = 0 of every base is the base itself (exact, eval64,
    // one launch for all bases)
    if ((e = cudaMemset(s->d_keys.ptr, 0xFF, 8 * s->P)) != cudaSuccess) return cuda_fail(e, "reset keys");
    {
        pesto_status rc = launch_search_eval(s.get(), 0, s->P, 0, 1, s->d_keys.as<uint64_t>(),
                                             nullptr, nullptr);
        if (rc) return rc;
    }
    if ((e = cudaDeviceSynchronize()) != cudaSuccess) return cuda_fail(e, "initial evaluation");
    std::vector<uint64_t> k0(s->P);
    cudaMemcpy(k0.data(), s->d_keys.ptr, 8 * s->P, cudaMemcpyDeviceToHost);
    std::vector<int64_t> mk0(s->P);
    for (int b = 0; b < s->P; b++) mk0[b] = (int64_t)(k0[b] >> 24);
    cudaMemcpy(s->d_mk.ptr, mk0.data(), 8 * s->P, cudaMemcpyHostToDevice);
    s->h_mk = mk0;
    update_all_below(s.get());
    if (d->nccl_unique_id) {                 // (a 1-rank comm is allowed: exercises the path)
        if (!nccl().ok) return fail(PESTO_ENCCL, "libnccl.so.2 not loadable");
        ncclUniqueId id;
        std::memcpy(&id, d->nccl_unique_id, sizeof id);
        ncclResult_t r = nccl().comm_init_rank(&s->comm, s->world, id, s->rank);
        if (r != ncclSuccess) return nccl_fail(r, "ncclCommInitRank");
    }
    *out = s.release();
    return PESTO_OK;
}

pesto_status pesto_search_eval(pesto_search *s, void *stream) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    NvtxRange nvtx("pesto_search_eval (K1)");
    DeviceGuard guard(s->g->device);
    cudaStream_t st = (cudaStream_t)stream;
    s->last_stream = st;
    cudaError_t e = cudaMemsetAsync(s->d_keys.ptr, 0xFF, 8 * s->P, st);
    if (e != cudaSuccess) return cuda_fail(e, "reset keys");
    return launch_search_eval(s, 0, s->P, s->j_begin, s->j_end, s->d_keys.as<uint64_t>(), nullptr, st,
                              true);
}

pesto_status pesto_search_keys(pesto_search *s, uint64_t *keys_host, void *stream) {
    if (!s || !keys_host) return fail(PESTO_EINVAL, "NULL argument");
    DeviceGuard guard(s->g->device);
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e = cudaMemcpyAsync(s->h_keys, s->d_keys.ptr, 8 * s->P, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_fail(e, "read keys");
    std::memcpy(keys_host, s->h_keys, 8 * s->P);
    return PESTO_OK;
}

pesto_status pesto_search_set_keys(pesto_search *s, const uint64_t *keys_host, void *stream) {
    if (!s || !keys_host) return fail(PESTO_EINVAL, "NULL argument");
    DeviceGuard guard(s->g->device);
    cudaStream_t st = (cudaStream_t)stream;
    std::memcpy(s->h_keys, keys_host, 8 * s->P);
    cudaError_t e = cudaMemcpyAsync(s->d_keys.ptr, s->h_keys, 8 * s->P, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    return e == cudaSuccess ? PESTO_OK : cuda_fail(e, "write keys");
}

pesto_status pesto_search_commit(pesto_search *s, void *stream) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    NvtxRange nvtx("pesto_search_commit (K4)");
    pesto_graph *g = s->g;
    if (s->comm_gen != g->comm_gen)
        return fail(PESTO_ESTATE, "the comm model changed after the search was created");
    DeviceGuard guard(g->device);
    cudaStream_t st = (cudaStream_t)stream;
    s->last_stream = st;
    CommitParams cp{};
    cp.bases = s->d_views.as<BaseLayoutDev>();
    cp.bits = s->d_bits.as<uint32_t>();
    cp.n = g->n;
    cp.D = g->D;
    cp.planes = g->planes;
    cp.words = g->words;
    cp.P = s->P;
    cp.seed = s->seed;
    cp.step = (uint64_t)s->step;
    std::memcpy(cp.mix, s->mix, sizeof cp.mix);
    cp.movable = g->d_movable.as<int32_t>();
    cp.n_movable = (int32_t)g->movable.size();
    cp.allowed_op = g->d_allowed.as<uint8_t>();
    cp.keys = s->d_keys.as<uint64_t>();
    cp.base_mk = s->d_mk.as<int64_t>();
    cp.swap_out = s->d_swap.as<int32_t>();
    cp.feas = feasibility_view(g);
    cp.feas.fbase = s->d_fbase.as<int64_t>();
    cp.n_coarse = s->n_coarse;
    cp.coarse_pct = s->coarse_pct;
    cudaError_t e = launch_commit(cp, st);
    if (e != cudaSuccess) return cuda_fail(e, "launch commit");
    s->step++;
    if (s->mix[3] == 0 && !s->all_below) {
        // bases may have dropped below the 32-bit saturation point: read their makespans back
        // asynchronously (without this the wide launch ran every step)
        if (!s->ev_mk && (e = cudaEventCreateWithFlags(&s->ev_mk, cudaEventDisableTiming)) != cudaSuccess)
            return cuda_fail(e, "event");
        if (!s->h_mk_async && (e = cudaMallocHost((void **)&s->h_mk_async, 8 * s->P)) != cudaSuccess)
            return cuda_fail(e, "pinned");
        if ((e = cudaMemcpyAsync(s->h_mk_async, s->d_mk.ptr, 8 * s->P, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
            (e = cudaEventRecord(s->ev_mk, st)) != cudaSuccess)
            return cuda_fail(e, "read base makespans");
        s->mk_pending = true;
    }
    if (s->mix[3] > 0) {
        // a committed adjacent swap changes a base's order: rebuild its position-space layout
        if ((e = cudaMemcpyAsync(s->h_swap, s->d_swap.ptr, 4 * s->P, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
            (e = cudaMemcpyAsync(s->h_keys, s->d_mk.ptr, 8 * s->P, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
            (e = cudaStreamSynchronize(st)) != cudaSuccess)
            return cuda_fail(e, "read committed swaps");
        std::memcpy(s->h_mk.data(), s->h_keys, 8 * s->P);   // h_keys doubles as a staging buffer
        update_all_below(s);
        bool changed = false;
        Patcher pt;
        for (int b = 0; b < s->P; b++) {
            const int32_t k = s->h_swap[b];
            if (k < 0) continue;
            std::swap(s->order[b][k], s->order[b][k + 1]);
            if (!s->cpos.empty()) {           // S9 merged vertices by position follow the order
                const size_t r = (size_t)b * g->n;
                pt.set_elem(s->d_cpos, s->cpos, r + k, (uint8_t)s->coarse_of[s->order[b][k]]);
                pt.set_elem(s->d_cpos, s->cpos, r + k + 1, (uint8_t)s->coarse_of[s->order[b][k + 1]]);
            }
            if (swap_in_place(s, b, k, pt)) {
                s->n_swap_inplace++;
                continue;
            }
            s->n_swap_rebuilt++;
            std::vector<uint8_t> x_op(g->n);
            pesto_status rc = download_x(s, b, x_op.data());      // K4 already swapped the bits
            if (rc) return rc;
            if ((rc = build_layout(g, s->order[b].data(), s->layouts[b], false, x_op.data(),
                                   s->tile32))) return rc;
            if ((rc = upload_layout(g, *s->layouts[b]))) return rc;
            changed = true;
        }
        for (int b : s->spec_rebuild) {
            pesto_status rc = rebuild_spec(g, *s->layouts[b]);
            if (rc) return rc;
            changed = true;                  // the list buffers may have moved: refresh views
        }
        s->spec_rebuild.clear();
        if (!pt.ops.empty()) {
            const size_t bytes = pt.ops.size() * sizeof(PatchOp);
            if ((e = s->d_patch.ensure(bytes)) != cudaSuccess ||
                (e = cudaMemcpyAsync(s->d_patch.ptr, pt.ops.data(), bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess ||
                (e = launch_patch(s->d_patch.as<PatchOp>(), (int)pt.ops.size(), pt.max_block, st)) != cudaSuccess ||
                (e = cudaStreamSynchronize(st)) != cudaSuccess)
                return cuda_fail(e, "patch swapped layouts");
        }
        if (changed) {
            refresh_views(s);
            if ((e = cudaMemcpyAsync(s->d_views.ptr, s->views.data(), sizeof(BaseLayoutDev) * s->P,
                                     cudaMemcpyHostToDevice, st)) != cudaSuccess ||
                (e = cudaStreamSynchronize(st)) != cudaSuccess)
                return cuda_fail(e, "upload views");
        }
    }
    return PESTO_OK;
}

pesto_status pesto_search_set_coarse_moves(pesto_search *s, const int32_t *coarse_of, int32_t n_coarse,
                                          int32_t pct) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    pesto_graph *g = s->g;
    if (pct < 0 || pct > 100) return fail(PESTO_EINVAL, "coarse percentage out of 0..100");
    if (pct == 0) {                       // off; the position arrays are kept (cheap) but unused
        s->coarse_pct = 0;
        return PESTO_OK;
    }
    if (!coarse_of) return fail(PESTO_EINVAL, "NULL coarse_of");
    if (n_coarse < 1 || n_coarse > 255) return fail(PESTO_EINVAL, "n_coarse must be in 1..255");
    for (int32_t v = 0; v < g->n; v++)
        if (coarse_of[v] < 0 || coarse_of[v] >= n_coarse)
            return fail(PESTO_EINVAL, "coarse_of[" + std::to_string(v) + "] out of range");
    if (g->has_cap || g->has_coloc)
        return fail(PESTO_ESTATE, "coarse group moves (S9) cannot be combined with row-f3 constraints");
    DeviceGuard guard(g->device);
    cudaError_t e;
    if (s->last_stream && (e = cudaStreamSynchronize(s->last_stream)) != cudaSuccess)
        return cuda_fail(e, "synchronise");
    s->coarse_of.assign(coarse_of, coarse_of + g->n);
    s->cpos.resize((size_t)s->P * g->n);
    for (int b = 0; b < s->P; b++)
        for (int32_t q = 0; q < g->n; q++)
            s->cpos[(size_t)b * g->n + q] = (uint8_t)coarse_of[s->order[b][q]];
    if ((e = s->d_cpos.ensure(s->cpos.size())) != cudaSuccess ||
        (e = cudaMemcpy(s->d_cpos.ptr, s->cpos.data(), s->cpos.size(), cudaMemcpyHostToDevice)) != cudaSuccess)
        return cuda_fail(e, "upload merged vertices");
    refresh_views(s);
    if ((e = cudaMemcpy(s->d_views.ptr, s->views.data(), sizeof(BaseLayoutDev) * s->P,
                        cudaMemcpyHostToDevice)) != cudaSuccess)
        return cuda_fail(e, "upload views");
    s->n_coarse = n_coarse;
    s->coarse_pct = pct;
    return PESTO_OK;
}

pesto_status pesto_search_reduce(pesto_search *s, void *stream) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    NvtxRange nvtx("pesto_search_reduce (allreduce-MIN)");
    if (s->comm) {
        DeviceGuard guard(s->g->device);
        // the step's only cross-GPU exchange: global best (makespan, candidate id) per base
        ncclResult_t r = nccl().all_reduce(s->d_keys.ptr, s->d_keys.ptr, (size_t)s->P, ncclUint64,
                                           ncclMin, s->comm, (cudaStream_t)stream);
        if (r != ncclSuccess) return nccl_fail(r, "ncclAllReduce");
    }
    return PESTO_OK;
}

pesto_status pesto_search_step(pesto_search *s, void *stream) {
    NvtxRange nvtx("pesto_search_step");
    pesto_status rc = pesto_search_eval(s, stream);
    if (rc) return rc;
    if ((rc = pesto_search_reduce(s, stream))) return rc;
    return pesto_search_commit(s, stream);
}

pesto_status pesto_search_candidate_keys_ex(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                            uint64_t *keys_out, int32_t kernel, void *stream) {
    if (!s || !keys_out) return fail(PESTO_EINVAL, "NULL argument");
    if (base < 0 || base >= s->P) return fail(PESTO_EINVAL, "base out of range");
    if (j0 < 0 || j1 < j0 || j1 > s->K) return fail(PESTO_EINVAL, "candidate range out of [0, K]");
    if (kernel < PESTO_KEYS_TIMED || kernel > PESTO_KEYS_TIMED_RAW)
        return fail(PESTO_EINVAL, "unknown key kernel");
    if (j1 == j0) return PESTO_OK;
    pesto_graph *g = s->g;
    DeviceGuard guard(g->device);
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e = cudaMemsetAsync(s->d_dbg_key.ptr, 0xFF, 8, st);
    if (e != cudaSuccess) return cuda_fail(e, "reset");
    if (kernel == PESTO_KEYS_EVAL64)
        return launch_search_eval(s, base, 1, j0, j1, s->d_dbg_key.as<uint64_t>(), keys_out, st);
    // the instance the timed step launches: its candidates-per-lane choice is the full step's
    EvalParams plan;
    fill_eval_common(g, plan);
    plan_eval32(g, plan, s->j_begin, s->j_end, s->P);
    pesto_status rc = launch_search_eval(s, base, 1, j0, j1, s->d_dbg_key.as<uint64_t>(), keys_out,
                                         st, true, plan.cpl32);
    if (rc || kernel == PESTO_KEYS_TIMED_RAW || !s->use32 || g->dispatch != PESTO_DISPATCH_FIXED ||
        g->link_model != PESTO_LINKS_FCFS)
        return rc;                                   // (those paths are exact 64-bit already)
    // saturated 32-bit walks (makespan field kSat32): exact keys from one launch of the wide
    // (exact 64-bit) instance over the range (round 1 re-ran each on eval64: ~1 launch per
    // saturated id, 33 minutes on nmt4's full K)
    std::vector<uint64_t> h((size_t)(j1 - j0));
    if ((e = cudaMemcpyAsync(h.data(), keys_out, h.size() * 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
        (e = cudaStreamSynchronize(st)) != cudaSuccess)
        return cuda_fail(e, "read keys");
    bool any = false;
    for (size_t i = 0; i < h.size() && !any; i++)
        any = h[i] != ~0ull && (h[i] >> 24) >= (uint64_t)kSat32;
    if (!any) return PESTO_OK;
    DevBuf wide;
    if ((e = wide.ensure(h.size() * 8)) != cudaSuccess) return cuda_fail(e, "alloc");
    if ((rc = launch_search_eval(s, base, 1, j0, j1, s->d_dbg_key.as<uint64_t>(), wide.as<uint64_t>(), st,
                                 true, 0, true)))
        return rc;
    std::vector<uint64_t> hw(h.size());
    if ((e = cudaMemcpyAsync(hw.data(), wide.ptr, hw.size() * 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
        (e = cudaStreamSynchronize(st)) != cudaSuccess)
        return cuda_fail(e, "read keys");
    for (size_t i = 0; i < h.size(); i++)
        if (h[i] != ~0ull && (h[i] >> 24) >= (uint64_t)kSat32) h[i] = hw[i];
    if ((e = cudaMemcpyAsync(keys_out, h.data(), h.size() * 8, cudaMemcpyHostToDevice, st)) != cudaSuccess ||
        (e = cudaStreamSynchronize(st)) != cudaSuccess)
        return cuda_fail(e, "write keys");
    return PESTO_OK;
}

pesto_status pesto_search_candidate_keys(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                         uint64_t *keys_out, void *stream) {
    return pesto_search_candidate_keys_ex(s, base, j0, j1, keys_out, PESTO_KEYS_TIMED, stream);
}

pesto_status pesto_search_move_stats(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                     pesto_move_stats *out) {
    if (!s || !out) return fail(PESTO_EINVAL, "NULL argument");
    if (base < 0 || base >= s->P) return fail(PESTO_EINVAL, "base out of range");
    if (j0 < 0 || j1 < j0 || j1 > s->K) return fail(PESTO_EINVAL, "candidate range out of [0, K]");
    pesto_graph *g = s->g;
    DeviceGuard guard(g->device);
    cudaError_t e = s->last_stream ? cudaStreamSynchronize(s->last_stream) : cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(e, "synchronise");
    const int32_t n = g->n;
    std::vector<uint8_t> x_op(n), xq(n);
    pesto_status rc = download_x(s, base, x_op.data());
    if (rc) return rc;
    const std::vector<int32_t> &ord = s->order[base];
    for (int32_t q = 0; q < n; q++) xq[q] = x_op[ord[q]];
    const std::vector<uint8_t> &blocked = s->layouts[base]->swap_blocked;
    const uint64_t cb = ctr_base_of((uint64_t)s->step, s->P, base);
    // a candidate's signature: its order move and every (position, new device) that differs
    // from the base, hashed; equal signatures = identical (placement, order) pairs
    std::vector<uint64_t> sig;
    sig.reserve((size_t)(j1 - j0));
    pesto_move_stats st{};
    for (int64_t j = j0; j < j1; j++) {
        const int64_t grp = j >> kGroupShift;
        const bool coarse = coarse_group(s->seed, cb, grp, s->coarse_pct, s->n_coarse);
        const Region rg = decode_region(s->seed, cb, grp, n);
        const int32_t ks = coarse ? -1
            : decode_swap(s->seed, cb, grp, n, s->mix[3], rg,
                          [&](int32_t k) { return blocked[k] != 0; },
                          [&](int32_t q) { return (int)xq[q]; });
        const LaneMove mv = j == 0 ? LaneMove{kMoveNone, 0, {-1, -1, -1, -1}, {0, 0, 0, 0}, 0, 0, 0}
            : coarse ? decode_coarse_lane(s->seed, cb, j, s->n_coarse, g->D)
            : decode_lane(s->seed, cb, j, ks >= 0 && (j & (kGroup - 1)) == 0, g->D, s->mix, rg,
                          [&](int32_t q) { return ord[q]; }, [&](int32_t q) { return (int)xq[q]; },
                          [&](int32_t op) { return (unsigned)g->allowed[op]; });
        st.candidates++;
        if (mv.kind == kMoveInvalid) { st.invalid++; continue; }
        uint64_t h = mix64(0x5045535430ull + (uint64_t)(ks + 1));
        int changed = 0;
        auto add = [&](int32_t q, int d) {
            if (d == (int)xq[q]) return;
            h = mix64(h ^ mix64(((uint64_t)q << 8) | (uint64_t)d));
            changed++;
        };
        if (mv.kind == kMoveFlip) {
            int32_t qs[4];
            int m = 0;
            for (int f = 0; f < mv.nflip; f++) {           // a later flip of a position wins
                bool last = true;
                for (int f2 = f + 1; f2 < mv.nflip; f2++) last = last && mv.fpos[f2] != mv.fpos[f];
                if (last) qs[m++] = f;
            }
            for (int a = 1; a < m; a++)                      // ascending position
                for (int b = a; b > 0 && mv.fpos[qs[b]] < mv.fpos[qs[b - 1]]; b--) std::swap(qs[b], qs[b - 1]);
            for (int i = 0; i < m; i++) add(mv.fpos[qs[i]], mv.fdev[qs[i]]);
        } else if (mv.kind == kMoveWindow) {
            for (int32_t q = mv.ws; q < mv.ws + mv.wl; q++)
                if ((g->allowed[ord[q]] >> mv.wd) & 1) add(q, mv.wd);
        } else if (mv.kind == kMoveCoarse) {
            for (int32_t q = 0; q < n; q++)
                if (s->coarse_of[ord[q]] == mv.ws && ((g->allowed[ord[q]] >> mv.wd) & 1)) add(q, mv.wd);
        }
        if (changed == 0 && ks < 0) st.identical_to_base++;
        sig.push_back(h);
    }
    std::sort(sig.begin(), sig.end());
    st.distinct = (int64_t)(std::unique(sig.begin(), sig.end()) - sig.begin());
    *out = st;
    return PESTO_OK;
}

pesto_status pesto_search_get(pesto_search *s, int32_t base, int64_t *mk, uint8_t *x_host,
                              int32_t *order_host) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    if (base < 0 || base >= s->P) return fail(PESTO_EINVAL, "base out of range");
    pesto_graph *g = s->g;
    DeviceGuard guard(g->device);
    cudaError_t e = s->last_stream ? cudaStreamSynchronize(s->last_stream) : cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(e, "synchronise");
    if (mk && (e = cudaMemcpy(mk, s->d_mk.as<int64_t>() + base, 8, cudaMemcpyDeviceToHost)) != cudaSuccess)
        return cuda_fail(e, "read makespan");
    if (x_host) {
        pesto_status rc = download_x(s, base, x_host);
        if (rc) return rc;
    }
    if (order_host) std::copy(s->order[base].begin(), s->order[base].end(), order_host);
    return PESTO_OK;
}

int64_t pesto_search_step_count(const pesto_search *s) { return s ? s->step : -1; }

pesto_status pesto_search_set_step(pesto_search *s, int64_t step) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    if (step < 0) return fail(PESTO_EINVAL, "step must be >= 0");
    DeviceGuard guard(s->g->device);
    cudaError_t e = s->last_stream ? cudaStreamSynchronize(s->last_stream) : cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(e, "synchronise");
    s->step = step;
    return PESTO_OK;
}

pesto_status pesto_search_swap_stats(const pesto_search *s, int64_t *in_place, int64_t *rebuilt) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
    if (in_place) *in_place = s->n_swap_inplace;
    if (rebuilt) *rebuilt = s->n_swap_rebuilt;
    return PESTO_OK;
}

void pesto_search_destroy(pesto_search *s) {
    if (!s) return;
    DeviceGuard guard(s->g->device);
    if (s->comm && nccl().comm_destroy) nccl().comm_destroy(s->comm);
    if (s->aux) cudaStreamSynchronize(s->aux);
    if (s->ev_fork) cudaEventDestroy(s->ev_fork);
    if (s->ev_join) cudaEventDestroy(s->ev_join);
    if (s->aux) cudaStreamDestroy(s->aux);
    if (s->h_swap) cudaFreeHost(s->h_swap);
    if (s->h_keys) cudaFreeHost(s->h_keys);
    if (s->h_mk_async) cudaFreeHost(s->h_mk_async);
    if (s->ev_mk) cudaEventDestroy(s->ev_mk);
    delete s;
}

}  // extern "C"
