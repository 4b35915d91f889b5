// coarsen.cpp -- row f2: graph coarsening of PAPER.md §3.3 (product code, host).
//
// Each iteration (L265-267): heights by level-wise Kahn (Definition 3.4, footnote 1);
// the coarse edges sorted by the bytes they carry (the comm estimate, L263; reading R22); a
// matching of the edges that satisfy Theorem 3.5 (L249-253) under reading R21 of condition
// (iii), taken greedily in that order; a defensive Kahn check of the merged graph (the batch is
// halved until acyclic); the merge (the merged vertex keeps the smaller op id, R23).  Stops at
// the target size or when no edge can be merged.  O(m log m) per iteration; each iteration at
// least halves nothing in the worst case but in practice removes 30-70% of the vertices.
#include <algorithm>
#include <numeric>
#include <string>
#include <vector>

#include "host.h"

namespace pesto {
namespace {

struct CEdge {
    int32_t u, v;
    int64_t w;
};

// level-wise Kahn over nv vertices: heights (roots 1); false if the graph has a cycle
bool heights(int32_t nv, const std::vector<CEdge> &E, std::vector<int32_t> &H) {
    std::vector<int32_t> indeg(nv, 0), off(nv + 1, 0), adj(E.size());
    for (const CEdge &e : E) {
        indeg[e.v]++;
        off[e.u + 1]++;
    }
    for (int32_t k = 0; k < nv; k++) off[k + 1] += off[k];
    {
        std::vector<int32_t> fill(off.begin(), off.end() - 1);
        for (const CEdge &e : E) adj[fill[e.u]++] = e.v;
    }
    H.assign(nv, 0);
    std::vector<int32_t> level, next;
    for (int32_t k = 0; k < nv; k++)
        if (indeg[k] == 0) level.push_back(k);
    int32_t h = 1, seen = 0;
    while (!level.empty()) {
        next.clear();
        for (int32_t k : level) {
            H[k] = h;
            seen++;
            for (int32_t i = off[k]; i < off[k + 1]; i++)
                if (--indeg[adj[i]] == 0) next.push_back(adj[i]);
        }
        level.swap(next);
        h++;
    }
    return seen == nv;
}

}  // namespace

pesto_status coarsen_graph(const pesto_graph *g, int32_t target, std::vector<int32_t> &coarse_of,
                           int32_t &n_coarse) {
    const int32_t n = g->n;
    std::vector<int32_t> rep(n);
    std::iota(rep.begin(), rep.end(), 0);
    auto find = [&](int32_t a) {
        int32_t r = a;
        while (rep[r] != r) r = rep[r];
        while (rep[a] != r) {                     // path compression: roots are unchanged
            const int32_t nx = rep[a];
            rep[a] = r;
            a = nx;
        }
        return r;
    };
    std::vector<int32_t> idx(n, -1), ids;
    std::vector<CEdge> raw, E;
    std::vector<int32_t> H;
    for (;;) {
        ids.clear();
        for (int32_t a = 0; a < n; a++)
            if (find(a) == a) ids.push_back(a);   // ascending
        const int32_t nv = (int32_t)ids.size();
        if (nv <= target) break;
        for (int32_t k = 0; k < nv; k++) idx[ids[k]] = k;
        // coarse edges: parallel edges merged, bytes summed
        raw.clear();
        for (int64_t e = 0; e < g->m; e++) {
            const int32_t ra = find(g->src[e]), rb = find(g->dst[e]);
            if (ra != rb) raw.push_back({idx[ra], idx[rb], g->bytes[e]});
        }
        std::sort(raw.begin(), raw.end(), [](const CEdge &a, const CEdge &b) {
            return a.u != b.u ? a.u < b.u : a.v < b.v;
        });
        E.clear();
        for (const CEdge &e : raw) {
            if (!E.empty() && E.back().u == e.u && E.back().v == e.v) E.back().w += e.w;
            else E.push_back(e);
        }
        if (!heights(nv, E, H)) return fail(PESTO_ECYCLE, "coarsening produced a cycle");
        // distinct successor / predecessor lists (E is sorted by (u, v) and deduplicated)
        std::vector<int32_t> soff(nv + 1, 0), poff(nv + 1, 0), sadj(E.size()), padj(E.size());
        for (const CEdge &e : E) {
            soff[e.u + 1]++;
            poff[e.v + 1]++;
        }
        for (int32_t k = 0; k < nv; k++) {
            soff[k + 1] += soff[k];
            poff[k + 1] += poff[k];
        }
        {
            std::vector<int32_t> sf(soff.begin(), soff.end() - 1), pf(poff.begin(), poff.end() - 1);
            for (const CEdge &e : E) {
                sadj[sf[e.u]++] = e.v;
                padj[pf[e.v]++] = e.u;
            }
        }
        std::vector<int32_t> cand(E.size());
        std::iota(cand.begin(), cand.end(), 0);
        std::sort(cand.begin(), cand.end(), [&](int32_t a, int32_t b) {
            const CEdge &x = E[a], &y = E[b];
            if (x.w != y.w) return x.w > y.w;
            return x.u != y.u ? x.u < y.u : x.v < y.v;
        });
        std::vector<uint8_t> matched(nv, 0);
        std::vector<int32_t> acc_u_of_v(nv, -1), acc_v_of_u(nv, -1);
        std::vector<std::pair<int32_t, int32_t>> M;
        for (int32_t ci : cand) {
            const int32_t u = E[ci].u, v = E[ci].v;
            if (matched[u] || matched[v]) continue;                               // (i)
            const int32_t d = H[v] - H[u];
            bool ok = soff[u + 1] - soff[u] == 1 || poff[v + 1] - poff[v] == 1 || d == 1;
            if (!ok) {                                                              // (ii)
                ok = true;
                for (int32_t i = soff[u]; i < soff[u + 1] && ok; i++)
                    if (sadj[i] != v && H[sadj[i]] <= H[u] + d) ok = false;
            }
            if (!ok) continue;
            // (iii), reading R21: no accepted pair j with (u, v_j) in E and H(u_j) == H(u),
            // nor (u_j, v) in E and H(u_j) == H(u)
            for (int32_t i = soff[u]; i < soff[u + 1] && ok; i++) {
                const int32_t uj = acc_u_of_v[sadj[i]];
                if (uj >= 0 && H[uj] == H[u]) ok = false;
            }
            for (int32_t i = poff[v]; i < poff[v + 1] && ok; i++) {
                const int32_t p = padj[i];
                if (acc_v_of_u[p] >= 0 && H[p] == H[u]) ok = false;
            }
            if (!ok) continue;
            M.push_back({u, v});
            matched[u] = matched[v] = 1;
            acc_u_of_v[v] = u;
            acc_v_of_u[u] = v;
            if (nv - (int32_t)M.size() <= target) break;
        }
        // defensive: the merged graph must be acyclic (R21); halve the batch until it is
        while (!M.empty()) {
            std::vector<int32_t> comp(nv);
            std::iota(comp.begin(), comp.end(), 0);
            for (auto &pr : M) comp[pr.second] = pr.first;
            std::vector<int32_t> kid(nv, -1);
            int32_t nk = 0;
            for (int32_t k = 0; k < nv; k++)
                if (comp[k] == k) kid[k] = nk++;
            std::vector<CEdge> merged;
            for (const CEdge &e : E)
                if (comp[e.u] != comp[e.v]) merged.push_back({kid[comp[e.u]], kid[comp[e.v]], 0});
            std::vector<int32_t> Hm;
            if (heights(nk, merged, Hm)) break;
            M.resize(M.size() / 2);
        }
        if (M.empty()) break;
        for (auto &pr : M) {                       // the merged vertex keeps the smaller op id
            const int32_t ru = ids[pr.first], rv = ids[pr.second];
            rep[std::max(ru, rv)] = std::min(ru, rv);
        }
    }
    // dense ids ordered by the smallest op of each merged vertex (R23)
    std::vector<int32_t> dense(n, -1);
    n_coarse = 0;
    coarse_of.assign(n, 0);
    for (int32_t a = 0; a < n; a++) {
        const int32_t r = find(a);
        if (dense[r] < 0) dense[r] = n_coarse++;
        coarse_of[a] = dense[r];
    }
    return PESTO_OK;
}

}  // namespace pesto

// =============================================================================================
// C ABI (include/pesto.h)
// =============================================================================================
using namespace pesto;

extern "C" {

pesto_status pesto_coarsen(pesto_graph *g, int32_t target, int32_t *coarse_of, int32_t *n_coarse) {
    if (!g || !coarse_of || !n_coarse) return fail(PESTO_EINVAL, "NULL argument");
    if (target < 1) return fail(PESTO_EINVAL, "target must be >= 1");
    std::vector<int32_t> co;
    int32_t nc = 0;
    pesto_status s = coarsen_graph(g, target, co, nc);
    if (s) return s;
    std::copy(co.begin(), co.end(), coarse_of);
    *n_coarse = nc;
    return PESTO_OK;
}

pesto_status pesto_eval_coarse_exhaustive(pesto_graph *g, const int32_t *order,
                                          const int32_t *coarse_of, int32_t n_coarse,
                                          int64_t *best_makespan, int64_t *best_index,
                                          uint8_t *best_x, void *stream) {
    if (!g || !order || !coarse_of || !best_makespan || !best_index || !best_x)
        return fail(PESTO_EINVAL, "NULL argument");
    if (g->device < 0) return fail(PESTO_ESTATE, "host-only graph handle");
    const int32_t n = g->n;
    if (n_coarse < 1 || n_coarse > n || n_coarse > 32) return fail(PESTO_EINVAL, "n_coarse out of [1, min(n_ops, 32)]");
    for (int32_t v = 0; v < n; v++)
        if (coarse_of[v] < 0 || coarse_of[v] >= n_coarse) return fail(PESTO_EINVAL, "coarse id out of range");
    const int D = g->D;
    const int b = D == 1 ? 0 : D == 2 ? 1 : D == 4 ? 2 : D == 8 ? 3 : -1;
    if (b < 0) return fail(PESTO_EINVAL, "exhaustive coarse search needs D in {1, 2, 4, 8}");
    if (b * n_coarse > 24) return fail(PESTO_EINVAL, "D^n_coarse exceeds 2^24 candidates");
    if (g->link_model != PESTO_LINKS_FCFS || g->dispatch != PESTO_DISPATCH_FIXED || g->has_cap || g->has_coloc)
        return fail(PESTO_ESTATE, "exhaustive coarse search supports the FCFS fixed-sequence model without constraints");
    DeviceGuard guard(g->device);
    cudaStream_t st = (cudaStream_t)stream;
    std::shared_ptr<Layout> L;
    pesto_status s = build_layout(g, order, L, true);
    if (s) return s;
    if ((s = upload_layout(g, *L))) return s;
    if (!g->eligible32 || L->W32 == 0)
        return fail(PESTO_ESTATE, "exhaustive coarse search needs an eval32-eligible graph");
    const int64_t total = int64_t(1) << (b * n_coarse);
    // the merged vertices by position, and the devices every member of a vertex allows
    std::vector<uint8_t> cpos(n);
    for (int32_t q = 0; q < n; q++) cpos[q] = (uint8_t)coarse_of[order[q]];
    std::vector<uint8_t> cmask(32, 0xFF);
    for (int32_t v = 0; v < n; v++) cmask[coarse_of[v]] &= g->allowed[v];
    cudaError_t e;
    if ((e = g->d_cpos.ensure(n)) != cudaSuccess ||
        (e = cudaMemcpyAsync(g->d_cpos.ptr, cpos.data(), n, cudaMemcpyHostToDevice, st)) != cudaSuccess ||
        (e = g->d_ckey.ensure(8)) != cudaSuccess ||
        (e = cudaMemsetAsync(g->d_ckey.ptr, 0xFF, 8, st)) != cudaSuccess)
        return cuda_fail(e, "stage exhaustive coarse search");
    EvalParams p;
    fill_eval_common(g, p);
    p.stage_bytes = L->stage_bytes;
    p.max_W = L->W;
    p.stage_bytes32 = L->stage_bytes32;
    p.max_W32 = L->W32;
    p.bases = L->d_view.as<BaseLayoutDev>();
    p.n_cand = total;

    p.keys = g->d_ckey.as<uint64_t>();
    p.coarse_pos = g->d_cpos.as<uint8_t>();
    p.coarse_bits = b;
    p.n_coarse = n_coarse;
    std::copy(cmask.begin(), cmask.end(), p.coarse_allowed);
    plan_eval32(g, p, 0, total, 1);
    int grid = 0;
    if ((s = ensure_state32(g, g->ws, p, 4, p.n_tasks, &grid))) return s;
    p.state32 = g->ws.state32.as<uint32_t>();
    if ((e = launch_eval32(p, 4, grid, st)) != cudaSuccess) return cuda_fail(e, "launch exhaustive coarse search");
    uint64_t key = ~0ull;
    if ((e = cudaMemcpyAsync(&key, g->d_ckey.ptr, 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
        (e = cudaStreamSynchronize(st)) != cudaSuccess)
        return cuda_fail(e, "exhaustive coarse search");
    if (key == ~0ull) {                                  // no feasible coarse placement
        *best_makespan = INT64_MAX;
        *best_index = -1;
        std::fill(best_x, best_x + n, 0);
        return PESTO_OK;
    }
    const int64_t mk = (int64_t)(key >> 24);
    if (mk >= (int64_t)kSat32) return fail(PESTO_ESTATE, "best makespan beyond the 32-bit kernel's 4.03 s");
    const int64_t j = (int64_t)(key & ((1ull << 24) - 1));
    *best_makespan = mk;
    *best_index = j;
    for (int32_t v = 0; v < n; v++) best_x[v] = (uint8_t)((j >> (b * coarse_of[v])) & (D - 1));
    return PESTO_OK;
}

}  // extern "C"
