// search.cpp -- parallel local search over placements and orders.
//
// One step = K1 (neighbour decode + makespan + warp argmin, this rank's share of candidate ids)
// -> ncclAllReduce MIN of the packed (makespan << 24 | j) keys across ranks (the only exchange)
// -> K4 commit on every rank (each regenerates the winner from the counter, so bases stay equal).
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
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

// fast: eval32 for the bases below saturation (+ eval64 for the others while any may exist);
// otherwise (debug keys, initial makespans, ineligible graphs) eval64 for all candidates
pesto_status launch_search_eval(pesto_search *s, int b_first, int n_bases, int64_t j0, int64_t j1,
                                uint64_t *keys, uint64_t *keys_dbg, cudaStream_t st,
                                bool fast = false) {
    pesto_graph *g = s->g;
    if (j1 <= j0) return PESTO_OK;
    EvalParams p;
    fill_eval_common(g, p);
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
    p.group_begin = j0 >> 5;
    p.groups_per_base = ((j1 - 1) >> 5) - p.group_begin + 1;
    p.tasks_per_base = (p.groups_per_base + kWarps - 1) / kWarps;
    p.n_tasks = p.tasks_per_base * n_bases;
    int grid = 0;
    pesto_status rc;
    cudaError_t e;
    const bool use32 = fast && s->use32 && keys_dbg == nullptr;
    if (use32) {
        // eval32 tasks: 256 consecutive ids starting at a multiple of 256
        EvalParams p32 = p;
        p32.gate = 1;
        p32.tasks_per_base = (j1 - (j0 & ~(int64_t)255) + 255) / 256;
        p32.n_tasks = p32.tasks_per_base * n_bases;
        if ((rc = ensure_state32(g, p32, 1, p32.n_tasks, &grid))) return rc;
        p32.state32 = g->d_state32.as<uint32_t>();
        if ((e = launch_eval32(p32, 1, grid, st)) != cudaSuccess) return cuda_fail(e, "launch eval32");
        if (s->all_below) return PESTO_OK;
        p.gate = 2;
    }
    if ((rc = ensure_state(g, p, 1, p.n_tasks, &grid))) return rc;
    p.state = g->d_state.as<int64_t>();
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
    for (int b = 0; b < s->P; b++) {
        s->order[b].assign(d->base_order + (size_t)b * n, d->base_order + (size_t)(b + 1) * n);
        pesto_status rc = build_layout(g, s->order[b].data(), s->layouts[b], false,
                                       d->base_x + (size_t)b * n);
        if (rc) return rc;
        if ((rc = upload_layout(g, *s->layouts[b]))) return rc;
        if ((rc = upload_bits(s.get(), b, d->base_x + (size_t)b * n))) return rc;
    }
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
    pesto_graph *g = s->g;
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
    cp.patch32 = s->use32 ? 1 : 0;
    cudaError_t e = launch_commit(cp, st);
    if (e != cudaSuccess) return cuda_fail(e, "launch commit");
    s->step++;
    if (s->mix[3] > 0) {
        // a committed adjacent swap changes a base's order: rebuild its position-space layout
        if ((e = cudaMemcpyAsync(s->h_swap, s->d_swap.ptr, 4 * s->P, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
            (e = cudaMemcpyAsync(s->h_keys, s->d_mk.ptr, 8 * s->P, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
            (e = cudaStreamSynchronize(st)) != cudaSuccess)
            return cuda_fail(e, "read committed swaps");
        std::memcpy(s->h_mk.data(), s->h_keys, 8 * s->P);   // h_keys doubles as a staging buffer
        update_all_below(s);
        bool changed = false;
        for (int b = 0; b < s->P; b++) {
            const int32_t k = s->h_swap[b];
            if (k < 0) continue;
            std::swap(s->order[b][k], s->order[b][k + 1]);
            std::vector<uint8_t> x_op(g->n);
            pesto_status rc = download_x(s, b, x_op.data());      // K4 already swapped the bits
            if (rc) return rc;
            if ((rc = build_layout(g, s->order[b].data(), s->layouts[b], false, x_op.data()))) return rc;
            if ((rc = upload_layout(g, *s->layouts[b]))) return rc;
            changed = true;
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

pesto_status pesto_search_reduce(pesto_search *s, void *stream) {
    if (!s) return fail(PESTO_EINVAL, "NULL search");
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
    pesto_status rc = pesto_search_eval(s, stream);
    if (rc) return rc;
    if ((rc = pesto_search_reduce(s, stream))) return rc;
    return pesto_search_commit(s, stream);
}

pesto_status pesto_search_candidate_keys(pesto_search *s, int32_t base, int64_t j0, int64_t j1,
                                         uint64_t *keys_out, void *stream) {
    if (!s || !keys_out) return fail(PESTO_EINVAL, "NULL argument");
    if (base < 0 || base >= s->P) return fail(PESTO_EINVAL, "base out of range");
    if (j0 < 0 || j1 < j0 || j1 > s->K) return fail(PESTO_EINVAL, "candidate range out of [0, K]");
    DeviceGuard guard(s->g->device);
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e = cudaMemsetAsync(s->d_dbg_key.ptr, 0xFF, 8, st);
    if (e != cudaSuccess) return cuda_fail(e, "reset");
    return launch_search_eval(s, base, 1, j0, j1, s->d_dbg_key.as<uint64_t>(), keys_out, st);
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

void pesto_search_destroy(pesto_search *s) {
    if (!s) return;
    DeviceGuard guard(s->g->device);
    if (s->comm && nccl().comm_destroy) nccl().comm_destroy(s->comm);
    if (s->h_swap) cudaFreeHost(s->h_swap);
    if (s->h_keys) cudaFreeHost(s->h_keys);
    delete s;
}

}  // extern "C"
