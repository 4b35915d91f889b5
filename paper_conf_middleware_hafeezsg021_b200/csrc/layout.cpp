// layout.cpp -- position-space layouts of one schedule order.
//
// For an order pi (the per-device op order) every op is relabelled by its
// position.  Two record streams are emitted, one per kernel:
//   eval64: ready-time slots in global memory, interval-coloured (one slot per consumer, live
//           from its first producer to one position past itself -- DESIGN.md §3.3);
//   eval32: near/far split with the base placement embedded in the records
//           (search bases only; patched in place by K4 when a placement move is committed).
// Everything is O(n + m): counting sorts by position, flat CSR arrays, one pass per field.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "host.h"
#include "moves.cuh"

namespace pesto {

namespace {

// LIFO interval colouring: interval of consumer w is [start[w], end[w]] (end = pos(w) + 1),
// w without interval has start < 0.  Returns the slot count.
int32_t colour_intervals(int32_t n, const std::vector<int32_t> &start, const std::vector<int32_t> &pos,
                         std::vector<int32_t> &slot) {
    std::vector<int32_t> s_off(n + 1, 0), f_off(n + 1, 0);
    for (int32_t w = 0; w < n; w++) {
        if (start[w] < 0) continue;
        s_off[start[w] + 1]++;
        if (pos[w] + 2 < n) f_off[pos[w] + 2 + 1]++;
    }
    for (int32_t k = 0; k < n; k++) { s_off[k + 1] += s_off[k]; f_off[k + 1] += f_off[k]; }
    std::vector<int32_t> s_list(s_off[n]), f_list(f_off[n]);
    {
        std::vector<int32_t> sf(s_off.begin(), s_off.end() - 1), ff(f_off.begin(), f_off.end() - 1);
        // consumers in position order so the colouring is deterministic
        for (int32_t w = 0; w < n; w++) {
            if (start[w] < 0) continue;
            s_list[sf[start[w]]++] = w;
            if (pos[w] + 2 < n) f_list[ff[pos[w] + 2]++] = w;
        }
    }
    slot.assign(n, -1);
    std::vector<int32_t> stack;
    stack.reserve(1024);
    int32_t W = 0;
    for (int32_t k = 0; k < n; k++) {
        for (int32_t i = f_off[k]; i < f_off[k + 1]; i++) stack.push_back(slot[f_list[i]]);
        for (int32_t i = s_off[k]; i < s_off[k + 1]; i++) {
            const int32_t w = s_list[i];
            if (!stack.empty()) { slot[w] = stack.back(); stack.pop_back(); }
            else slot[w] = W++;
        }
    }
    return W;
}

struct TileWriter {
    std::vector<uint8_t> &blob;
    std::vector<TileDesc> &tiles;
    int32_t &stage_bytes;
    size_t start = 0;
    int32_t pos0 = 0;
    TileWriter(std::vector<uint8_t> &b, std::vector<TileDesc> &t, int32_t &sb) : blob(b), tiles(t), stage_bytes(sb) {}
    void open(int32_t k) {
        start = blob.size();
        pos0 = k;
        blob.resize(start + kTileHeader, 0);
    }
    void close(int32_t k_end) {
        TileDesc td{};
        td.byte_off = (int64_t)start;
        td.bytes = (int32_t)(blob.size() - start);
        td.pos_begin = pos0;
        td.pos_end = k_end;
        const int32_t hdr[4] = {pos0, k_end, td.bytes, 0};
        std::memcpy(blob.data() + start, hdr, 16);
        tiles.push_back(td);
        stage_bytes = std::max(stage_bytes, td.bytes);
    }
    // start a new tile before an op whose records take `rec_bytes` if the current one is full
    void maybe_cut(int32_t k, size_t rec_bytes) {
        if (k > pos0 && blob.size() - start + rec_bytes > (size_t)kTileTarget) {
            close(k);
            open(k);
        }
    }
};

template <class T>
void append(std::vector<uint8_t> &buf, const T &v) {
    const size_t at = buf.size();
    buf.resize(at + sizeof(T));
    std::memcpy(buf.data() + at, &v, sizeof(T));
}

}  // namespace

pesto_status build_layout(pesto_graph *g, const int32_t *order, std::shared_ptr<Layout> &out,
                          bool use_cache, const uint8_t *x_op, int32_t tile32) {
    pesto_status s = ensure_comm_tables(g);
    if (s) return s;
    const int32_t n = g->n;
    const int64_t m = g->m;
    if (!order) return fail(PESTO_EINVAL, "order is NULL");
    if (use_cache && !x_op) {
        for (auto it = g->cache.begin(); it != g->cache.end(); ++it) {
            if ((*it)->comm_gen == g->comm_gen &&
                std::memcmp((*it)->order.data(), order, (size_t)n * 4) == 0) {
                out = *it;
                g->cache.splice(g->cache.begin(), g->cache, it);
                return PESTO_OK;
            }
        }
    }
    // a search base rebuilt after a committed swap reuses its layout object, so the device
    // buffers are recycled instead of freed (cudaFree synchronises the device) and reallocated
    std::shared_ptr<Layout> L = (x_op && out && out.use_count() == 1) ? out : std::make_shared<Layout>();
    L->on_device = false;
    L->stage_bytes = 0;
    L->comm_gen = g->comm_gen;
    L->order.assign(order, order + n);
    L->pos.assign(n, -1);
    std::vector<int32_t> &pos = L->pos;
    for (int32_t k = 0; k < n; k++) {
        const int32_t v = order[k];
        if (v < 0 || v >= n || pos[v] != -1) return fail(PESTO_ENOTTOPO, "order is not a permutation");
        pos[v] = k;
    }
    for (int64_t e = 0; e < m; e++)
        if (pos[g->src[e]] >= pos[g->dst[e]])
            return fail(PESTO_ENOTTOPO, "order violates edge " + std::to_string(e));

    // out-edges of every producer sorted by (successor position, edge index) -- the FCFS tie
    // order of reading R3 -- by one pass over consumers in position order (in-edges of a
    // consumer are listed by edge index)
    std::vector<int64_t> sorted(m);
    {
        std::vector<int64_t> fill(g->out_off.begin(), g->out_off.end() - 1);
        for (int32_t q = 0; q < n; q++) {
            const int32_t w = order[q];
            for (int64_t i = g->in_off[w]; i < g->in_off[w + 1]; i++) {
                const int64_t e = g->in_edges[i];
                sorted[fill[g->src[e]]++] = e;
            }
        }
    }
    auto succ_pos = [&](int64_t e) { return pos[g->dst[e]]; };
    const int C = g->n_classes;

    // ---------------- eval64 stream ----------------
    {
        std::vector<int32_t> &first = L->first64;
        first.assign(n, -1);
        for (int64_t e = 0; e < m; e++) {
            const int32_t w = g->dst[e], ps = pos[g->src[e]];
            if (first[w] < 0 || ps < first[w]) first[w] = ps;
        }
        std::vector<int32_t> &slot = L->slot64;
        L->W = std::max(colour_intervals(n, first, pos, slot), 1);
        std::vector<uint8_t> seen(n, 0), first_flag(m, 0);
        for (int32_t k = 0; k < n; k++) {
            const int32_t u = order[k];
            for (int64_t i = g->out_off[u]; i < g->out_off[u + 1]; i++) {
                const int64_t e = sorted[i];
                if (!seen[g->dst[e]]) { seen[g->dst[e]] = 1; first_flag[e] = 1; }
            }
        }
        const int es = edge_stride_for(C);
        L->blob.clear();
        L->heavy.clear();
        L->tiles.clear();
        L->blob.reserve((size_t)n * 16 + (size_t)m * es + 64 * kTileHeader);
        L->op_off64.assign(n, 0);
        L->tile64_of.assign(n, 0);
        L->eloc64.assign(m, 0);
        auto put_edge = [&](std::vector<uint8_t> &buf, int64_t e) {
            const size_t at = buf.size();
            L->eloc64[e] = (uint32_t)at | (&buf == &L->heavy ? kPinHeavy : 0u);
            buf.resize(at + es, 0);
            EdgeRec r;
            r.t0 = g->t_class[(size_t)e * C];
            r.succ_pos = succ_pos(e);
            r.slot = (uint32_t)slot[g->dst[e]] | (first_flag[e] ? kEdgeFirst : 0u);
            std::memcpy(buf.data() + at, &r, sizeof r);
            for (int c = 1; c < C; c++)
                std::memcpy(buf.data() + at + 16 + 8 * (c - 1), &g->t_class[(size_t)e * C + c], 8);
        };
        TileWriter tw(L->blob, L->tiles, L->stage_bytes);
        tw.open(0);
        for (int32_t k = 0; k < n; k++) {
            const int32_t u = order[k];
            const int64_t nout = g->out_off[u + 1] - g->out_off[u];
            const bool heavy = nout * es > kMaxInlineBytes;
            tw.maybe_cut(k, 16 + (heavy ? 16 : (size_t)nout * es));
            L->op_off64[k] = (uint32_t)L->blob.size();
            L->tile64_of[k] = (int32_t)L->tiles.size();
            OpRec op;
            op.p = g->p[u];
            op.in_slot = slot[u];
            op.nout = heavy ? kOpHeavy : (uint32_t)nout;
            append(L->blob, op);
            if (heavy) {
                append(L->blob, ExtRec{(int64_t)L->heavy.size(), nout});
                for (int64_t i = g->out_off[u]; i < g->out_off[u + 1]; i++) put_edge(L->heavy, sorted[i]);
            } else {
                for (int64_t i = g->out_off[u]; i < g->out_off[u + 1]; i++) put_edge(L->blob, sorted[i]);
            }
        }
        tw.close(n);
    }

    // ---------------- eval32 stream ----------------
    // distance 1: the next op's forwarding register; 2..kNearDelta: the ring; farther: cold slot
    auto next_edge = [&](int64_t e) { return pos[g->dst[e]] - pos[g->src[e]] == 1; };
    auto near_edge = [&](int64_t e) { return pos[g->dst[e]] - pos[g->src[e]] <= kNearDelta; };
    std::vector<int32_t> &first_far = L->first_far, &cslot = L->cslot;
    first_far.clear();
    cslot.clear();
    std::vector<uint8_t> has_near;
    L->W32 = 0;
    if (g->eligible32) {
        first_far.assign(n, -1);
        has_near.assign(n, 0);
        for (int64_t e = 0; e < m; e++) {
            const int32_t w = g->dst[e];
            if (next_edge(e)) continue;                       // register-forwarded
            if (near_edge(e)) { has_near[w] = 1; continue; }  // shared-memory ring
            const int32_t ps = pos[g->src[e]];
            if (first_far[w] < 0 || ps < first_far[w]) first_far[w] = ps;
        }
        L->W32 = std::max(colour_intervals(n, first_far, pos, cslot), 1);
        if (L->W32 >= (1 << 22)) L->W32 = 0;  // slot byte offsets must fit 29 bits: 64-bit path
    }
    if (L->W32 > 0 && C > 2) L->W32 = 0;     // the step format carries two link classes
    if (L->W32 > 0) {
        std::vector<uint8_t> seen_near(n, 0), seen_far(n, 0), first32(m, 0);
        for (int32_t k = 0; k < n; k++) {
            const int32_t u = order[k];
            for (int64_t i = g->out_off[u]; i < g->out_off[u + 1]; i++) {
                const int64_t e = sorted[i];
                const int32_t w = g->dst[e];
                if (next_edge(e)) continue;
                uint8_t &seen = near_edge(e) ? seen_near[w] : seen_far[w];
                if (!seen) { seen = 1; first32[e] = 1; }
            }
        }
        auto t32 = [&](int64_t e, int c) { return (uint32_t)g->t_class[(size_t)e * C + c]; };
        auto xcode = [&](int32_t op) { return x_op ? (uint32_t)(x_op[op] & 7u) : 0u; };
        L->blob32.clear();
        L->heavy32.clear();
        L->tiles32.clear();
        L->stage_bytes32 = 0;
        L->blob32.reserve((size_t)(n + m / 2 + 64) * kStepBytes + 64 * kTileHeader);
        L->op_off32.assign(n, 0);
        L->tile32_of.assign(n, 0);
        L->slot_succ.clear();
        L->eloc32.assign(m, 0);
        // patch index: locations of every edge record by successor position
        L->pin_off.assign((size_t)n + 1, 0);
        L->pin_ref.assign(m, 0);
        for (int64_t e = 0; e < m; e++) L->pin_off[pos[g->dst[e]] + 1]++;
        for (int32_t q = 0; q < n; q++) L->pin_off[q + 1] += L->pin_off[q];
        std::vector<uint32_t> pfill(L->pin_off.begin(), L->pin_off.end() - 1);
        auto edge_rec = [&](int64_t e, size_t at, uint32_t slot) {
            EdgeRec32 r;
            if (g->D == 2) {             // by direction: t0 on link 0 -> 1, t1 on link 1 -> 0
                r.t0 = t32(e, g->link_class[1]);
                r.t1 = t32(e, g->link_class[2]);
            } else {                     // by link class (D > 2: at most two classes here)
                r.t0 = t32(e, 0);
                r.t1 = C > 1 ? t32(e, 1) : 0u;
            }
            const int32_t w = g->dst[e];
            r.succ_pos = (int32_t)((uint32_t)pos[w] | (xcode(w) << kSuccXShift));
            // byte offset of the lane's slot column: ring slot (pos & 15) or cold slot, x 128
            r.target = next_edge(e) ? kT32Next
                     : (near_edge(e) ? (kT32Near | (uint32_t)(pos[w] & (kRing - 1)) * 128u)
                                     : (uint32_t)cslot[w] * 128u) |
                       (first32[e] ? kT32First : 0u);
            r.succ_pos = (int32_t)((uint32_t)r.succ_pos | (target_class32(r.target) << kSuccTcShift));
            L->pin_ref[pfill[pos[w]]++] = (uint32_t)at | (slot ? kPinSlot : 0u);
            L->eloc32[e] = (uint32_t)at | (slot ? kPinSlot : 0u);
            return r;
        };
        // tiles hold whole ops, except an op larger than a tile, which continues in the next
        std::vector<uint8_t> &blob = L->blob32;
        size_t t_start = 0;
        int32_t t_steps = 0;
        auto open = [&]() { t_start = blob.size(); t_steps = 0; blob.resize(t_start + kTileHeader, 0); };
        auto close = [&]() {
            TileDesc td{};
            td.byte_off = (int64_t)t_start;
            td.bytes = (int32_t)(blob.size() - t_start);
            td.pos_begin = t_steps;                  // (steps in the tile)
            // {steps, blob offset of the tile (the walk locates a swapped pair with it), bytes, 0}
            const int32_t hdr[4] = {t_steps, (int32_t)(uint32_t)t_start, td.bytes, 0};
            std::memcpy(blob.data() + t_start, hdr, 16);
            L->tiles32.push_back(td);
            L->stage_bytes32 = std::max(L->stage_bytes32, td.bytes);
        };
        // eval32 tile budget: kTileTarget, or PESTO_TILE32_BYTES (occupancy experiments: a smaller
        // tile lets more CTAs' stages fit in shared memory)
        // eval32 layouts of D = 2 graphs (search and explicit rows) use 6 KB tiles, so that five
        // CTAs of the no-producer instance fit in shared memory (measured neutral for the
        // producer instance: transformer_2dev 35.93 / 35.95 ms, nmt4 29.02 / 28.92 ms at 8 / 6 KB)
        static const size_t env_budget = [] {
            const char *e = std::getenv("PESTO_TILE32_BYTES");
            const long v = e ? std::atol(e) : 0;
            return (size_t)(v >= 1024 && v <= 65536 ? (v & ~15L) : 0);
        }();
        const size_t budget = env_budget ? env_budget
                            : tile32 > 0 ? (size_t)tile32
                            : (g->planes == 1 ? (size_t)kTileTarget32Search : (size_t)kTileTarget);
        open();
        for (int32_t k = 0; k < n; k++) {
            const int32_t u = order[k];
            const int64_t b0 = g->out_off[u], b1 = g->out_off[u + 1];
            const int64_t nout = b1 - b0;
            const int64_t nsteps = std::max<int64_t>(1, (nout + 1) / 2);
            const size_t op_bytes = (size_t)nsteps * kStepBytes;
            if (t_steps > 0 && blob.size() - t_start + op_bytes > budget) { close(); open(); }
            L->op_off32[k] = (uint32_t)blob.size();
            L->tile32_of[k] = (int32_t)L->tiles32.size();
            for (int64_t s = 0; s < nsteps; s++) {
                if (t_steps > 0 && blob.size() - t_start + kStepBytes > budget) { close(); open(); }
                const size_t at = blob.size();
                blob.resize(at + kStepBytes, 0);
                StepHead h{};
                const int64_t ne = std::min<int64_t>(2, nout - 2 * s);
                if (s == 0) {
                    h.p = (uint32_t)g->p[u];
                    const int32_t ahead = k + kPrefetchDist;
                    h.pf_slot = ahead < n ? cslot[order[ahead]] : -1;
                    h.flags = xcode(u) | (has_near[u] ? kStHasNear : 0u) |
                              ((uint32_t)std::max<int64_t>(ne, 0) << kStEdgeShift) |
                              ((uint32_t)nsteps << kStStepsShift);
                } else {
                    h.p = 0;
                    h.pf_slot = -1;
                    h.flags = kStCont | ((uint32_t)ne << kStEdgeShift);
                }
                std::memcpy(blob.data() + at, &h, 16);
                uint32_t kinds = 0;
                for (int64_t q = 0; q < 2; q++) {
                    const size_t eo = at + 16 + 16 * q;
                    EdgeRec32 r{};
                    if (q < ne) r = edge_rec(sorted[b0 + 2 * s + q], eo, (uint32_t)q);
                    else r.succ_pos = (int32_t)(kSuccClassNone << kSuccTcShift);   // empty slot
                    std::memcpy(blob.data() + eo, &r, 16);
                    // the fast walk's dispatch entry of this slot (D <= 4)
                    const uint32_t yu = ((uint32_t)r.succ_pos >> kSuccXShift) & kind_code_mask(g->D);
                    const uint32_t cls = ((uint32_t)r.succ_pos >> kSuccTcShift) & 7u;
                    kinds |= kind_byte(g->D, yu, cls, xcode(u)) << (8 * q);
                }
                std::memcpy(blob.data() + at + 4, &kinds, 4);
                for (int64_t q = 0; q < 2; q++)       // explicit rows: successor of each slot
                    L->slot_succ.push_back(q < ne ? pos[g->dst[sorted[b0 + 2 * s + q]]] : -1);
                t_steps++;
            }
        }
        close();
        if ((int64_t)blob.size() >= ((int64_t)1 << 31)) return fail(PESTO_ENOMEM, "layout too large");
    }

    // order moves: positions (k, k+1) may be swapped unless an edge joins them, they share a
    // producer or a consumer, or either has more than kSwapMaxOut successors (DESIGN §4 S3)
    L->swap_blocked.assign(n, 1);
    {
        std::vector<int32_t> mark_pred(n, -1), mark_succ(n, -1);
        for (int32_t k = 0; k + 1 < n; k++) {
            const int32_t a = order[k], c = order[k + 1];
            bool blocked = g->out_off[a + 1] - g->out_off[a] > kSwapMaxOut ||
                           g->out_off[c + 1] - g->out_off[c] > kSwapMaxOut;
            for (int64_t i = g->in_off[a]; i < g->in_off[a + 1]; i++) mark_pred[g->src[g->in_edges[i]]] = k;
            for (int64_t i = g->out_off[a]; i < g->out_off[a + 1]; i++) {
                const int32_t w = g->dst[g->out_edges[i]];
                if (w == c) blocked = true;
                mark_succ[w] = k;
            }
            for (int64_t i = g->in_off[c]; i < g->in_off[c + 1] && !blocked; i++)
                if (mark_pred[g->src[g->in_edges[i]]] == k) blocked = true;
            for (int64_t i = g->out_off[c]; i < g->out_off[c + 1] && !blocked; i++)
                if (mark_succ[g->dst[g->out_edges[i]]] == k) blocked = true;
            L->swap_blocked[k] = blocked ? 1 : 0;
        }
    }
    if (L->W32 > 0) {
        const int32_t R = (n + kRegion - 1) / kRegion;
        L->spec_off.assign((size_t)R + 1, 0);
        L->spec_pos.clear();
        std::vector<int32_t> lst;
        for (int32_t r = 0; r < R; r++) {
            L->spec_off[r] = (uint32_t)L->spec_pos.size();
            spec_region(g, *L, r, lst);
            L->spec_pos.insert(L->spec_pos.end(), lst.begin(), lst.end());
            L->spec_pos.insert(L->spec_pos.end(), (size_t)kSpecSlack, INT32_MAX);
        }
        L->spec_off[R] = (uint32_t)L->spec_pos.size();
    }
    L->allowed_pos.resize(n);
    for (int32_t k = 0; k < n; k++) L->allowed_pos[k] = g->allowed[order[k]];
    if (use_cache && !x_op) {
        g->cache.push_front(L);
        while (g->cache.size() > 8) g->cache.pop_back();
    }
    out = L;
    return PESTO_OK;
}

void spec_region(const pesto_graph *g, const Layout &L, int32_t r, std::vector<int32_t> &out) {
    const int32_t c = r * kRegion, e = std::min(g->n, c + kRegion);
    out.clear();
    for (int32_t q = c; q < e; q++) {
        out.push_back(q);
        const int32_t w = L.order[q];
        for (int64_t i = g->in_off[w]; i < g->in_off[w + 1]; i++) {
            const int32_t pq = L.pos[g->src[g->in_edges[i]]];
            if (pq < c) out.push_back(pq);
        }
    }
    std::sort(out.begin(), out.end());
    out.erase(std::unique(out.begin(), out.end()), out.end());
}

bool pair_blocked(const pesto_graph *g, int32_t a, int32_t c) {
    if (g->out_off[a + 1] - g->out_off[a] > kSwapMaxOut || g->out_off[c + 1] - g->out_off[c] > kSwapMaxOut)
        return true;
    for (int64_t i = g->out_off[a]; i < g->out_off[a + 1]; i++) {
        const int32_t w = g->dst[g->out_edges[i]];
        if (w == c) return true;
        for (int64_t j = g->out_off[c]; j < g->out_off[c + 1]; j++)
            if (g->dst[g->out_edges[j]] == w) return true;        // common consumer
    }
    for (int64_t i = g->in_off[a]; i < g->in_off[a + 1]; i++) {
        const int32_t u = g->src[g->in_edges[i]];
        for (int64_t j = g->in_off[c]; j < g->in_off[c + 1]; j++)
            if (g->src[g->in_edges[j]] == u) return true;         // common producer
    }
    return false;
}

}  // namespace pesto
