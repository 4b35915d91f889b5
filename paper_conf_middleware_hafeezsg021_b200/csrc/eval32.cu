// eval32.cu -- K1 fast path: the makespan recursion in 32-bit saturating time (product code).
//
// Same recursion as eval64 (kernels.cu; PAPER.md L142-146, L188-198, L374 -- DESIGN.md §3):
//   S_v = max(max_in arrival, dev_free[x_v]);  C_v = S_v + p_v;  dev_free[x_v] = C_v
//   cross e=(v,w): A_e = max(C_v, link_free[x_v->x_w]) + t_e;  link_free = A_e
// Layout of the work:
//   * one warp walks the DAG record stream once for 32 x CPL candidates: every lane carries
//     CPL candidates, so the warp-uniform work (records, flags, loop control, region checks)
//     is paid once per CPL candidates;
//   * the stream is TMA-staged (cp.async.bulk + mbarrier ring) by a producer warp and shared by
//     all consumer warps of the CTA;
//   * ready-time state by producer distance: distance 1 -> a register (`fwd`), 2..kNearDelta ->
//     the warp's shared-memory ring (slot = pos & 15), farther -> a global cold slot written
//     with fire-and-forget STG / RED.MAX and staged back by cp.async kPrefetchDist positions
//     before the consumer runs;
//   * search candidates differ from their base only inside their group's 64-position region
//     (DESIGN.md §4), so outside it a lane's device is the base code embedded in the record.
#include <algorithm>
#include <type_traits>

#include "device_common.cuh"
#include "internal.h"

namespace pesto {
namespace {

using namespace dev;

__device__ __forceinline__ uint32_t add_sat(uint32_t a, uint32_t b) {
    return min(a + b, kSat32);                 // a <= kSat32, b < kMaxDur32: never wraps
}

__host__ __device__ constexpr int warps_for(int cpl) { return cpl == 1 ? 8 : (cpl == 2 ? 4 : 2); }

// per-candidate device / link free times
template <int CPL>
struct RegState32 {          // D <= 2
    uint32_t d0[CPL], d1[CPL], l01[CPL], l10[CPL];
    __device__ __forceinline__ void init() {
#pragma unroll
        for (int c = 0; c < CPL; c++) d0[c] = d1[c] = l01[c] = l10[c] = 0u;
    }
    __device__ __forceinline__ uint32_t dev(int c, int x) const { return x ? d1[c] : d0[c]; }
    __device__ __forceinline__ void set_dev(int c, int x, uint32_t v) {
        if (x) d1[c] = v; else d0[c] = v;
    }
    __device__ __forceinline__ uint32_t link(int c, int x, int) const { return x ? l10[c] : l01[c]; }
    __device__ __forceinline__ void set_link_if(int c, int x, int, bool cond, uint32_t v) {
        l10[c] = (cond && x) ? v : l10[c];
        l01[c] = (cond && !x) ? v : l01[c];
    }
    __device__ __forceinline__ uint32_t makespan(int c) const { return max(d0[c], d1[c]); }
};

template <int CPL>
struct SmemState32 {         // D <= 8: [column][CPL][32] in shared memory (shared addresses)
    uint32_t d, l;           // + lane * 4
    int D;
    __device__ __forceinline__ uint32_t at(uint32_t base, int col, int c) const {
        return base + (uint32_t)(col * CPL + c) * 128;
    }
    __device__ __forceinline__ void init() {
        for (int x = 0; x < D; x++)
            for (int c = 0; c < CPL; c++) sts_u32(at(d, x, c), 0u);
        for (int x = 0; x < D * D; x++)
            for (int c = 0; c < CPL; c++) sts_u32(at(l, x, c), 0u);
    }
    __device__ __forceinline__ uint32_t dev(int c, int x) const { return lds_u32(at(d, x, c)); }
    __device__ __forceinline__ void set_dev(int c, int x, uint32_t v) { sts_u32(at(d, x, c), v); }
    __device__ __forceinline__ uint32_t link(int c, int x, int y) const {
        return lds_u32(at(l, x * D + y, c));
    }
    __device__ __forceinline__ void set_link_if(int c, int x, int y, bool cond, uint32_t v) {
        if (cond) sts_u32(at(l, x * D + y, c), v);
    }
    __device__ __forceinline__ uint32_t makespan(int c) const {
        uint32_t m = 0;
        for (int x = 0; x < D; x++) m = max(m, lds_u32(at(d, x, c)));
        return m;
    }
};

// devices of the lane's CPL candidates at position q; xb = the base code of the record naming q
template <int MODE, int PL, int CPL>
struct Place32 {
    const uint32_t *pl;          // MODE 0: words of the warp's first 32-row group
    int64_t pl_stride;           // MODE 0: words between consecutive 32-row groups
    const uint8_t *allowed_pos;  // MODE 1: masks by position (window moves)
    int32_t rc, rlen;            // MODE 1: the group's region [rc, rc + rlen)
    int all_allowed, lane, dmax;
    LaneMove mv[CPL];
    __device__ __forceinline__ void at(int32_t q, int xb, int (&x)[CPL]) const {
        if (MODE == 0) {
#pragma unroll
            for (int c = 0; c < CPL; c++) x[c] = planes_dev_at<PL>(pl + c * pl_stride, q, lane, dmax);
            return;
        }
#pragma unroll
        for (int c = 0; c < CPL; c++) x[c] = xb;
        if ((uint32_t)(q - rc) < (uint32_t)rlen) {             // warp-uniform branch
            const unsigned aq = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q);
#pragma unroll
            for (int c = 0; c < CPL; c++) x[c] = apply_lane(mv[c], q, xb, aq);
        }
    }
};

struct Ctx32 {
    uint32_t smem;               // shared address of the CTA's dynamic shared memory (records)
    uint32_t ring;               // shared address of ring[0][0][lane]; slot s, cand c: + (s*CPL+c)*128
    uint8_t *cold;               // global byte address of cold[0][0][lane]; same layout
    uint32_t lclass;             // shared address of the link-class table
    int edge_stride, D;
    bool two_classes;            // a second link class exists (its t is EdgeRec32.t1)
};

template <bool GLOBAL>
__device__ __forceinline__ uint4 rec_at(const Ctx32 &cx, const uint8_t *heavy, uint32_t off) {
    if (GLOBAL) return __ldg(reinterpret_cast<const uint4 *>(heavy + off));
    return lds_v4(cx.smem + off);
}

template <bool MULTI>
__device__ __forceinline__ int stride32(const Ctx32 &cx) { return MULTI ? cx.edge_stride : 16; }

// one out-edge, for the lane's CPL candidates
template <int CPL, bool MULTI, bool GLOBAL, bool ALL_MAX, class PlaceT, class StateT>
__device__ __forceinline__ void push32(const Ctx32 &cx, const uint8_t *heavy, uint32_t off,
                                       const uint4 rec, const int (&x)[CPL],
                                       const uint32_t (&cc)[CPL], const PlaceT &place,
                                       StateT &st, uint32_t (&fwd)[CPL]) {
    const int32_t succ = (int32_t)(rec.y & kSuccPosMask);
    const uint32_t tgt = rec.z;
    int y[CPL];
    place.at(succ, (int)((rec.y >> kSuccXShift) & 7u), y);
    uint32_t a[CPL];
#pragma unroll
    for (int c = 0; c < CPL; c++) {
        const bool cross = y[c] != x[c];                     // cross: FCFS link x -> y
        uint32_t t = rec.x;
        if ((MULTI || cx.two_classes) && cross) {
            const int cls = (int)lds_u8(cx.lclass + (uint32_t)(x[c] * cx.D + y[c]));
            if (cls == 1) t = rec.w;
            else if (MULTI && cls > 1) {
                const uint32_t eo = off + 16 + 4 * (cls - 2);
                t = GLOBAL ? __ldg(reinterpret_cast<const uint32_t *>(heavy + eo))
                           : lds_u32(cx.smem + eo);
            }
        }
        // branch-free: the transfer's arrival when crossing, C_v (L144) when not
        const uint32_t ac = add_sat(max(cc[c], st.link(c, x[c], y[c])), t);
        a[c] = cross ? ac : cc[c];
        st.set_link_if(c, x[c], y[c], cross, ac);
    }
    if (tgt & kT32Next) {                                    // consumer is the next position
#pragma unroll
        for (int c = 0; c < CPL; c++) fwd[c] = max(fwd[c], a[c]);
        return;
    }
    const uint32_t bytes = (tgt & kT32SlotMask) * CPL;
    if (tgt & kT32Near) {
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            const uint32_t slot = cx.ring + bytes + c * 128;
            uint32_t v = a[c];
            if (ALL_MAX || !(tgt & kT32First)) v = max(v, lds_u32(slot));
            sts_u32(slot, v);
        }
    } else {
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            uint32_t *slot = reinterpret_cast<uint32_t *>(cx.cold + bytes + c * 128);
            if (!ALL_MAX && (tgt & kT32First)) *slot = a[c];     // first far push: plain store
            else atomicMax(slot, a[c]);                          // RED.MAX, no reply awaited
        }
    }
}

// out-edges of one producer in record order.  Only a producer feeding two adjacent positions
// (kOpAdj) can see its order change under a swap (ks, ks+1): then the run of edges to ks+1 is
// pushed before the run to ks (the swapped order's consumer order).
template <int CPL, bool MULTI, bool GLOBAL, bool ALL_MAX, class PlaceT, class StateT>
__device__ __forceinline__ void push_all32(const Ctx32 &cx, const uint8_t *heavy, uint32_t ep,
                                           uint32_t nout, bool adj, int32_t ks,
                                           const int (&x)[CPL], const uint32_t (&cc)[CPL],
                                           const PlaceT &place, StateT &st, uint32_t (&fwd)[CPL]) {
    const int es = stride32<MULTI>(cx);
    auto push_i = [&](uint32_t i) {
        const uint32_t off = ep + i * es;
        push32<CPL, MULTI, GLOBAL, ALL_MAX>(cx, heavy, off, rec_at<GLOBAL>(cx, heavy, off), x, cc,
                                            place, st, fwd);
    };
    if (!adj || ks < 0) {
        for (uint32_t i = 0; i < nout; i++) push_i(i);
        return;
    }
    auto spos = [&](uint32_t i) {
        return (int32_t)(rec_at<GLOBAL>(cx, heavy, ep + i * es).y & kSuccPosMask);
    };
    for (uint32_t i = 0; i < nout;) {
        if (spos(i) != ks) {
            push_i(i);
            i++;
            continue;
        }
        uint32_t a_end = i;
        while (a_end < nout && spos(a_end) == ks) a_end++;
        uint32_t b_end = a_end;
        while (b_end < nout && spos(b_end) == ks + 1) b_end++;
        for (uint32_t e = a_end; e < b_end; e++) push_i(e);
        for (uint32_t e = i; e < a_end; e++) push_i(e);
        i = b_end;
    }
}

// Relax the op at position v (record o at shared offset rp) whose arrivals are r[c].
// Returns, in fwd[c], the forwarded arrivals for position v + 1.
template <int CPL, bool MULTI, bool ALL_MAX, class PlaceT, class StateT>
__device__ __forceinline__ void relax32(const Ctx32 &cx, uint32_t rp, const uint4 o, int32_t v,
                                        int32_t ks, const uint8_t *heavy, const PlaceT &place,
                                        StateT &st, const uint32_t (&r)[CPL], uint32_t (&fwd)[CPL]) {
    int x[CPL];
    place.at(v, (int)((o.w >> kOpXShift) & 7u), x);
    uint32_t cc[CPL];
#pragma unroll
    for (int c = 0; c < CPL; c++) {
        cc[c] = add_sat(max(r[c], st.dev(c, x[c])), o.x);    // C_v = S_v + p_v
        st.set_dev(c, x[c], cc[c]);
        fwd[c] = 0u;
    }
    const bool adj = (o.w & kOpAdj) != 0;
    if (!(o.w & kOpHeavy)) {
        push_all32<CPL, MULTI, false, ALL_MAX>(cx, heavy, rp + 16, o.w & kOpNoutMask, adj, ks, x, cc,
                                               place, st, fwd);
        return;
    }
    const uint4 ext = lds_v4(cx.smem + rp + 16);             // ExtRec
    push_all32<CPL, MULTI, true, ALL_MAX>(cx, heavy, ext.x, ext.z, adj, ks, x, cc, place, st, fwd);
}

template <bool MULTI>
__device__ __forceinline__ uint32_t next_rp(const Ctx32 &cx, uint32_t rp, uint32_t nout) {
    if (nout & kOpHeavy) return rp + 32;
    return rp + 16 + (nout & kOpNoutMask) * stride32<MULTI>(cx);
}

// zero the slots an op opens with a first push (swap pairs only; times are >= 0)
template <int CPL, bool MULTI>
__device__ __forceinline__ void clear_first32(const Ctx32 &cx, uint32_t rp, const uint8_t *heavy) {
    const uint4 o = lds_v4(cx.smem + rp);
    const bool global = (o.w & kOpHeavy) != 0;
    uint32_t ep = rp + 16, nout = o.w & kOpNoutMask;
    if (global) {
        const uint4 ext = lds_v4(cx.smem + rp + 16);
        ep = ext.x;
        nout = ext.z;
    }
    const int es = stride32<MULTI>(cx);
    for (uint32_t i = 0; i < nout; i++) {
        const uint4 rec = global ? rec_at<true>(cx, heavy, ep + i * es)
                                 : rec_at<false>(cx, heavy, ep + i * es);
        if (!(rec.z & kT32First) || (rec.z & kT32Next)) continue;
        const uint32_t bytes = (rec.z & kT32SlotMask) * CPL;
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            if (rec.z & kT32Near) sts_u32(cx.ring + bytes + c * 128, 0u);
            else *reinterpret_cast<uint32_t *>(cx.cold + bytes + c * 128) = 0u;
        }
    }
}

template <int MODE, int PL, bool MULTI, int CPL>
__global__ void __launch_bounds__((warps_for(CPL) + 1) * 32, 2)
eval32_kernel(const EvalParams P) {
    constexpr int NW = warps_for(CPL);          // consumer warps per CTA (256 candidates)
    constexpr int CW = 32 * CPL;                // candidates per warp
    extern __shared__ __align__(128) uint8_t smem[];
    const int sb = P.stage_bytes32;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)kStages * sb);
    uint64_t *empty = full + kStages;
    uint8_t *cur = align16(reinterpret_cast<uint8_t *>(empty + kStages));
    uint8_t *lclass = cur;
    cur = align16(cur + 64);
    uint32_t *ring_all = reinterpret_cast<uint32_t *>(cur);
    cur = align16(cur + (size_t)NW * kRing * CW * 4);
    uint32_t *stage_all = reinterpret_cast<uint32_t *>(cur);          // far-arrival staging
    cur = align16(cur + (size_t)NW * kRing * CW * 4);
    uint32_t *dstate = reinterpret_cast<uint32_t *>(cur);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], NW);
        }
        mbar_fence_init();
    }
    if (threadIdx.x < 64) lclass[threadIdx.x] = P.link_class[threadIdx.x];
    __syncthreads();

    auto runs_here = [&](int bl) {           // search: this kernel owns bases below saturation
        return MODE != 1 || P.gate == 0 || P.base_mk[bl] < (int64_t)kSat32;
    };

    if (warp == NW) {
        if (lane == 0) {
            uint32_t it = 0;
            for (int64_t task = blockIdx.x; task < P.n_tasks; task += gridDim.x) {
                const int bl = MODE ? (int)(task / P.tasks_per_base) : 0;
                if (!runs_here(bl)) continue;
                const BaseLayoutDev *B = &P.bases[bl];
                const int nt = B->n_tiles32;
                for (int t = 0; t < nt; t++, it++) {
                    const int s = it % kStages;
                    if (it >= (uint32_t)kStages) mbar_wait(&empty[s], ((it / kStages) - 1) & 1);
                    const TileDesc td = B->tiles32[t];
                    mbar_expect_tx(&full[s], (uint32_t)td.bytes);
                    bulk_g2s(smem + (size_t)s * sb, B->blob32 + td.byte_off, (uint32_t)td.bytes,
                             &full[s]);
                }
            }
        }
        return;
    }

    Ctx32 cx;
    cx.smem = su32_reg(smem);
    cx.ring = su32_reg(ring_all + (size_t)warp * kRing * CW + lane);
    cx.cold = reinterpret_cast<uint8_t *>(P.state32 + ((size_t)(blockIdx.x * NW + warp) * P.max_W32) * CW + lane);
    cx.lclass = su32_reg(lclass);
    cx.edge_stride = P.edge_stride32;
    cx.D = P.D;
    cx.two_classes = P.n_classes > 1;
    const uint32_t stage = su32_reg(stage_all + (size_t)warp * kRing * CW + lane);

    using StateT = typename std::conditional<PL == 1, RegState32<CPL>, SmemState32<CPL>>::type;
    StateT st;
    if constexpr (PL != 1) {
        st.D = P.D;
        st.d = su32_reg(dstate + (size_t)warp * (P.D + P.D * P.D) * CW + lane);
        st.l = st.d + (uint32_t)(P.D * CPL) * 128;
    }

    // Far arrivals of position q arrive by cp.async into stage[q & 15], issued while position
    // q - kPrefetchDist is relaxed (its record names the slot); one commit group per position,
    // so waiting for all but kPrefetchDist groups makes position q's values visible.  The first
    // kPrefetchDist positions of a task load them directly.
    auto issue_far = [&](const uint4 o, int32_t v) {
        const uint32_t dst = stage + (uint32_t)(((v + kPrefetchDist) & (kRing - 1)) * CPL) * 128;
        const bool have = (int32_t)o.z >= 0;
        const uint8_t *src = cx.cold + (size_t)(have ? o.z : 0) * CW * 4;
#pragma unroll
        for (int c = 0; c < CPL; c++) cp_async4(dst + c * 128, src + c * 128, have);
        cp_async_commit();
    };
    auto far_of = [&](const uint4 o, int32_t v, uint32_t (&f)[CPL]) {
#pragma unroll
        for (int c = 0; c < CPL; c++) f[c] = 0u;
        if ((int32_t)o.y < 0) return;
        if (v < kPrefetchDist) {
#pragma unroll
            for (int c = 0; c < CPL; c++)
                f[c] = *reinterpret_cast<const uint32_t *>(cx.cold + (size_t)o.y * CW * 4 + c * 128);
            return;
        }
        const uint32_t src = stage + (uint32_t)((v & (kRing - 1)) * CPL) * 128;
#pragma unroll
        for (int c = 0; c < CPL; c++) f[c] = lds_u32(src + c * 128);
    };
    auto ring_of = [&](const uint4 o, int32_t v, uint32_t (&f)[CPL]) {
        const uint32_t src = cx.ring + (uint32_t)((v & (kRing - 1)) * CPL) * 128;
#pragma unroll
        for (int c = 0; c < CPL; c++) f[c] = (o.w & kOp32HasNear) ? lds_u32(src + c * 128) : 0u;
    };

    uint32_t it = 0;
    for (int64_t task = blockIdx.x; task < P.n_tasks; task += gridDim.x) {
        const int bl = MODE ? (int)(task / P.tasks_per_base) : 0;
        if (!runs_here(bl)) continue;
        const int64_t local = MODE ? task % P.tasks_per_base : task;
        const BaseLayoutDev *B = &P.bases[bl];
        const int nt = B->n_tiles32;
        const uint8_t *heavy = B->heavy32;
        // a task = 256 consecutive candidate ids starting at a multiple of 256; a warp = CW of them
        const int64_t j0 = (P.j_begin & ~(int64_t)255) + local * 256 + warp * CW;
        const int64_t gw = j0 >> 5;                                 // first 32-row group

        Place32<MODE, PL, CPL> place;
        place.lane = lane;
        place.dmax = P.D - 1;
        place.all_allowed = P.all_allowed;
        place.rc = 0;
        place.rlen = 0;
        bool active;
        bool valid[CPL];
        int32_t ks = -1;
        if (MODE == 0) {
            active = j0 < P.n_cand;
            place.pl = P.planes_in + (size_t)gw * P.n * PL;
            place.pl_stride = (int64_t)P.n * PL;
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const int64_t j = j0 + c * 32 + lane;
                valid[c] = j < P.n_cand && !((__ldg(P.invalid + gw + c) >> lane) & 1u);
            }
        } else {
            active = j0 < P.j_end;
            const int breal = P.b_offset + bl;
            const uint64_t cb = ctr_base_of(P.step, P.P_total, breal);
            const int64_t grp = j0 >> kGroupShift;
            const Region rg = decode_region(P.seed, cb, grp, P.n);
            place.rc = rg.c;
            place.rlen = rg.len;
            place.allowed_pos = B->allowed_pos;
            const uint8_t *adj = B->adj_next;
            ks = active ? decode_swap(P.seed, cb, grp, P.n, P.mix[3], rg,
                                      [&](int32_t k) { return __ldg(adj + k) != 0; })
                        : -1;
            const int32_t *ord = B->order;
            const uint32_t *bits = B->bits;
            const uint8_t *aop = P.allowed_op;
            const int words = P.words;
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const int64_t j = j0 + c * 32 + lane;
                const bool in_range = active && j >= P.j_begin && j < P.j_end;
                place.mv[c] = in_range
                    ? decode_lane(P.seed, cb, j, ks >= 0 && (j & (kGroup - 1)) == 0, P.D, P.mix, rg,
                                  [&](int32_t q) { return __ldg(ord + q); },
                                  [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); },
                                  [&](int32_t op) { return (unsigned)__ldg(aop + op); })
                    : no_move();
                valid[c] = in_range && place.mv[c].kind != kMoveInvalid;
                if (place.mv[c].kind == kMoveInvalid) place.mv[c] = no_move();
            }
        }
        st.init();

        bool skip_first = false;
        uint32_t fwd[CPL];
#pragma unroll
        for (int c = 0; c < CPL; c++) fwd[c] = 0u;
        for (int t = 0; t < nt; t++, it++) {
            const int s = it % kStages;
            mbar_wait(&full[s], (it / kStages) & 1);
            if (active) {
                const uint32_t tile = (uint32_t)s * sb;
                const uint4 hdr = lds_v4(cx.smem + tile);
                const int32_t pos_end = (int32_t)hdr.y;
                int32_t v = (int32_t)hdr.x;
                uint32_t rp = tile + kTileHeader;
                if (skip_first) {
                    rp = next_rp<MULTI>(cx, rp, lds_v4(cx.smem + rp).w);
                    v++;
                    skip_first = false;
                }
                uint4 o = lds_v4(cx.smem + rp);
                while (v < pos_end) {
                    if (v != ks) {
                        const uint32_t rp_n = next_rp<MULTI>(cx, rp, o.w);
                        const uint4 o_n = (v + 1 < pos_end) ? lds_v4(cx.smem + rp_n) : o;
                        issue_far(o, v);
                        cp_async_wait<kPrefetchDist>();
                        uint32_t r[CPL], f[CPL], rg[CPL];
                        far_of(o, v, f);
                        ring_of(o, v, rg);
#pragma unroll
                        for (int c = 0; c < CPL; c++) r[c] = max(max(f[c], rg[c]), fwd[c]);
                        relax32<CPL, MULTI, false>(cx, rp, o, v, ks, heavy, place, st, r, fwd);
                        rp = rp_n;
                        v++;
                        o = o_n;
                        continue;
                    }
                    // swapped pair: ops at ks+1 then ks
                    const uint32_t rk = rp;
                    const uint4 o_k = o;
                    uint32_t rk1;
                    const bool straddle = (v + 1 == pos_end);
                    if (straddle) {
                        const int s2 = (it + 1) % kStages;
                        mbar_wait(&full[s2], ((it + 1) / kStages) & 1);
                        rk1 = (uint32_t)s2 * sb + kTileHeader;
                    } else {
                        rk1 = next_rp<MULTI>(cx, rk, o_k.w);
                    }
                    const uint4 o_k1 = lds_v4(cx.smem + rk1);
                    issue_far(o_k, v);
                    issue_far(o_k1, v + 1);
                    cp_async_wait<kPrefetchDist>();
                    uint32_t f0[CPL], g0[CPL], f1[CPL], g1[CPL], r0[CPL], r1[CPL], fwd_k2[CPL], dummy[CPL];
                    far_of(o_k, v, f0);
                    ring_of(o_k, v, g0);
                    far_of(o_k1, v + 1, f1);
                    ring_of(o_k1, v + 1, g1);
#pragma unroll
                    for (int c = 0; c < CPL; c++) {
                        r0[c] = max(max(f0[c], g0[c]), fwd[c]);
                        r1[c] = max(f1[c], g1[c]);     // k+1's only distance-1 producer is k: none
                    }
                    clear_first32<CPL, MULTI>(cx, rk, heavy);
                    relax32<CPL, MULTI, false>(cx, rk1, o_k1, v + 1, ks, heavy, place, st, r1, fwd_k2);
                    relax32<CPL, MULTI, true>(cx, rk, o_k, v, ks, heavy, place, st, r0, dummy);
#pragma unroll
                    for (int c = 0; c < CPL; c++) fwd[c] = fwd_k2[c];
                    if (straddle) {
                        skip_first = true;
                        v = pos_end;
                    } else {
                        rp = next_rp<MULTI>(cx, rk1, o_k1.w);
                        v += 2;
                        if (v < pos_end) o = lds_v4(cx.smem + rp);
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }
        cp_async_wait<0>();

        if (!active) continue;
        if (MODE == 0) {
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const int64_t j = j0 + c * 32 + lane;
                if (j >= P.n_cand) continue;
                const uint32_t mk = st.makespan(c);
                if (!valid[c]) {
                    P.makespans[j] = INT64_MAX;
                } else if (mk < kSat32) {
                    P.makespans[j] = (int64_t)mk;
                } else {                             // saturated: exact value from eval64
                    P.makespans[j] = INT64_MAX;
                    P.flag_list[atomicAdd(P.flag_count, 1)] = (int32_t)j;
                }
            }
        } else {
            // a saturated candidate's true makespan is >= kSat32 > this base's makespan, so it
            // never wins the argmin; its clamped key still sorts after the base's (exact) key
            uint64_t key = ~0ull;
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const int64_t j = j0 + c * 32 + lane;
                const uint64_t kc = valid[c] ? (((uint64_t)st.makespan(c) << 24) | (uint64_t)j) : ~0ull;
                key = kc < key ? kc : key;
            }
            key = warp_min_u64(key);
            if (lane == 0 && key != ~0ull)
                atomicMin(reinterpret_cast<unsigned long long *>(P.keys + bl), (unsigned long long)key);
        }
    }
}

template <int MODE, int PL, bool MULTI, int CPL>
cudaError_t launch_one32(const EvalParams &p, int grid, cudaStream_t st) {
    const int smem = eval32_smem_bytes(p, MODE);
    auto kern = eval32_kernel<MODE, PL, MULTI, CPL>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    kern<<<grid, (warps_for(CPL) + 1) * 32, smem, st>>>(p);
    return cudaGetLastError();
}

template <int MODE, int PL, bool MULTI, int CPL>
int occupancy_one32(const EvalParams &p) {
    const int smem = eval32_smem_bytes(p, MODE);
    auto kern = eval32_kernel<MODE, PL, MULTI, CPL>;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
        return 0;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, (warps_for(CPL) + 1) * 32, smem) !=
        cudaSuccess)
        return 0;
    return n;
}

int planes_of32(int D) { return D <= 2 ? 1 : (D <= 4 ? 2 : 4); }

}  // namespace

int eval32_cpl() { return kEval32Cpl; }

int eval32_smem_bytes(const EvalParams &p, int search_mode) {
    (void)search_mode;
    const int cpl = kEval32Cpl;
    const int nw = warps_for(cpl);
    const int pl = planes_of32(p.D);
    size_t b = (size_t)kStages * p.stage_bytes32 + 2 * kStages * 8;
    b = (b + 15) & ~size_t(15);
    b += 64;
    b = (b + 15) & ~size_t(15);
    b += (size_t)nw * kRing * 32 * cpl * 4;        // near ring
    b = (b + 15) & ~size_t(15);
    b += (size_t)nw * kRing * 32 * cpl * 4;        // far-arrival staging
    b = (b + 15) & ~size_t(15);
    if (pl != 1) b += (size_t)nw * (p.D + p.D * p.D) * 32 * cpl * 4;
    return (int)b + 128;
}

// the edge stride is a compile-time 16 bytes unless some link class beyond the second exists
#define PESTO_DISPATCH32(FN, ...)                                                          \
    do {                                                                                   \
        constexpr int C = kEval32Cpl;                                                      \
        const int pl = planes_of32(p.D);                                                   \
        const bool multi = p.n_classes > 2;                                                \
        if (search_mode) {                                                                 \
            if (pl == 1) return multi ? FN<1, 1, true, C>(__VA_ARGS__) : FN<1, 1, false, C>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<1, 2, true, C>(__VA_ARGS__) : FN<1, 2, false, C>(__VA_ARGS__); \
            return multi ? FN<1, 4, true, C>(__VA_ARGS__) : FN<1, 4, false, C>(__VA_ARGS__); \
        } else {                                                                           \
            if (pl == 1) return multi ? FN<0, 1, true, C>(__VA_ARGS__) : FN<0, 1, false, C>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<0, 2, true, C>(__VA_ARGS__) : FN<0, 2, false, C>(__VA_ARGS__); \
            return multi ? FN<0, 4, true, C>(__VA_ARGS__) : FN<0, 4, false, C>(__VA_ARGS__); \
        }                                                                                  \
    } while (0)

cudaError_t launch_eval32(const EvalParams &p, int search_mode, int grid, cudaStream_t st) {
    note_launch();
    PESTO_DISPATCH32(launch_one32, p, grid, st);
}

int eval32_max_ctas_per_sm(const EvalParams &p, int search_mode) {
    PESTO_DISPATCH32(occupancy_one32, p);
}

}  // namespace pesto
