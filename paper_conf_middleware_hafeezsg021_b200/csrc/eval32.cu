// eval32.cu -- K1 fast path: the makespan recursion in 32-bit saturating time (product code).
//
// Same recursion as eval64 (kernels.cu; PAPER.md L142-146, L188-198, L374 -- DESIGN.md §3):
//   S_v = max(max_in arrival, dev_free[x_v]);  C_v = S_v + p_v;  dev_free[x_v] = C_v
//   cross e=(v,w): A_e = max(C_v, link_free[x_v->x_w]) + t_e;  link_free = A_e
// with the ready-time state split by producer distance:
//   near (consumer within kNearDelta positions): the warp's shared-memory ring, slot = pos & 15
//   far:  a global cold slot written with fire-and-forget STG (first push) / RED.MAX, and
//         copied into a shared staging ring with cp.async kPrefetchDist positions ahead.
// One lane = one candidate, 32 candidates per warp share every DAG tile, which the producer
// warp streams into shared memory with cp.async.bulk (TMA) through an mbarrier ring.
// Search candidates differ from their base only inside their group's 64-position region
// (DESIGN.md §4), so outside it a lane's device is the base code embedded in the record, and
// once the walk is past the region no lookup needs the check at all (successors come later).
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

struct RegState32 {          // D <= 2
    uint32_t d0, d1, l01, l10;
    __device__ void init() { d0 = d1 = l01 = l10 = 0u; }
    __device__ uint32_t dev(int x) const { return x ? d1 : d0; }
    __device__ void set_dev(int x, uint32_t v) { if (x) d1 = v; else d0 = v; }
    __device__ uint32_t link(int x, int) const { return x ? l10 : l01; }
    __device__ void set_link(int x, int, uint32_t v) { if (x) l10 = v; else l01 = v; }
    __device__ uint32_t makespan() const { return max(d0, d1); }
};

struct SmemState32 {         // D <= 8: [column][lane] in shared memory (shared addresses)
    uint32_t d, l;
    int D;
    __device__ void init() {
        for (int x = 0; x < D; x++) sts_u32(d + x * 128, 0u);
        for (int x = 0; x < D * D; x++) sts_u32(l + x * 128, 0u);
    }
    __device__ uint32_t dev(int x) const { return lds_u32(d + x * 128); }
    __device__ void set_dev(int x, uint32_t v) { sts_u32(d + x * 128, v); }
    __device__ uint32_t link(int x, int y) const { return lds_u32(l + (x * D + y) * 128); }
    __device__ void set_link(int x, int y, uint32_t v) { sts_u32(l + (x * D + y) * 128, v); }
    __device__ uint32_t makespan() const {
        uint32_t m = 0;
        for (int x = 0; x < D; x++) m = max(m, lds_u32(d + x * 128));
        return m;
    }
};

// lane's device at position q; xb = the base code carried by the record that names q.
// CHECK = false once the walk is past the group's region (no lookup can fall inside it).
template <int MODE, int PL>
struct Place32 {
    const uint32_t *pl;          // MODE 0: this group's bit-sliced words
    const uint8_t *allowed_pos;  // MODE 1: masks by position (window moves)
    int32_t rc, rlen;            // MODE 1: the group's region [rc, rc + rlen)
    int all_allowed, lane, dmax;
    LaneMove mv;
    template <bool CHECK>
    __device__ __forceinline__ int at(int32_t q, int xb) const {
        if (MODE == 0) return planes_dev_at<PL>(pl, q, lane, dmax);
        if (CHECK && (uint32_t)(q - rc) < (uint32_t)rlen) {  // warp-uniform branch
            const unsigned aq = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q);
            return apply_lane(mv, q, xb, aq);
        }
        return xb;
    }
};

struct Ctx32 {
    uint32_t smem;               // shared address of the CTA's dynamic shared memory (records)
    uint32_t ring;               // shared address of ring[0][lane]; slot bytes from the record
    uint32_t *cold;              // global: cold[slot * 32 + lane]
    uint32_t lclass;             // shared address of the link-class table
    int edge_stride, D;
    bool two_classes;            // a second link class exists (its t is EdgeRec32.t1)
};

__device__ __forceinline__ void prefetch_l1(const void *p) {
    asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
}

// record at byte offset `off` of shared memory (GLOBAL: of the out-of-line array)
template <bool GLOBAL>
__device__ __forceinline__ uint4 rec_at(const Ctx32 &cx, const uint8_t *heavy, uint32_t off) {
    if (GLOBAL) return __ldg(reinterpret_cast<const uint4 *>(heavy + off));
    return lds_v4(cx.smem + off);
}

template <bool MULTI>
__device__ __forceinline__ int stride32(const Ctx32 &cx) { return MULTI ? cx.edge_stride : 16; }

template <bool MULTI, bool GLOBAL, bool ALL_MAX, bool CHECK, class PlaceT, class StateT>
__device__ __forceinline__ void push32(const Ctx32 &cx, const uint8_t *heavy, uint32_t off,
                                       const uint4 rec, int x, uint32_t c, const PlaceT &place,
                                       StateT &st, uint32_t &fwd) {
    const int32_t succ = (int32_t)(rec.y & kSuccPosMask);
    const uint32_t tgt = rec.z;
    const int y = place.template at<CHECK>(succ, (int)((rec.y >> kSuccXShift) & 7u));
    uint32_t a = c;                                          // same device: C_v (L144)
    if (y != x) {                                            // cross: FCFS link x -> y
        uint32_t t = rec.x;
        if (MULTI || cx.two_classes) {
            const int cls = (int)lds_u8(cx.lclass + (uint32_t)(x * cx.D + y));
            if (cls == 1) t = rec.w;
            else if (MULTI && cls > 1) {
                const uint32_t eo = off + 16 + 4 * (cls - 2);
                t = GLOBAL ? __ldg(reinterpret_cast<const uint32_t *>(heavy + eo))
                           : lds_u32(cx.smem + eo);
            }
        }
        a = add_sat(max(c, st.link(x, y)), t);
        st.set_link(x, y, a);
    }
    if (tgt & kT32Next) {                                    // consumer is the next position
        fwd = max(fwd, a);
        return;
    }
    const uint32_t bytes = tgt & kT32SlotMask;
    if (tgt & kT32Near) {
        const uint32_t slot = cx.ring + bytes;
        if (ALL_MAX || !(tgt & kT32First)) a = max(a, lds_u32(slot));
        sts_u32(slot, a);
    } else {
        uint32_t *slot = reinterpret_cast<uint32_t *>(reinterpret_cast<uint8_t *>(cx.cold) + bytes);
        if (!ALL_MAX && (tgt & kT32First)) *slot = a;        // first far push: plain store
        else atomicMax(slot, a);                             // RED.MAX, no wait for a reply
    }
}

// out-edges of one producer in record order.  Only a producer feeding two adjacent positions
// (kOpAdj) can see its order change under a swap (ks, ks+1): then the run of edges to ks+1 is
// pushed before the run to ks (the swapped order's consumer order).
template <bool MULTI, bool GLOBAL, bool ALL_MAX, bool CHECK, class PlaceT, class StateT>
__device__ __forceinline__ uint32_t push_all32(const Ctx32 &cx, const uint8_t *heavy, uint32_t ep,
                                               uint32_t nout, bool adj, int32_t ks, int x,
                                               uint32_t c, const PlaceT &place, StateT &st) {
    const int es = stride32<MULTI>(cx);
    uint32_t fwd = 0;
    if (!adj || ks < 0) {
        for (uint32_t i = 0; i < nout; i++) {
            const uint32_t off = ep + i * es;
            push32<MULTI, GLOBAL, ALL_MAX, CHECK>(cx, heavy, off, rec_at<GLOBAL>(cx, heavy, off), x, c,
                                                  place, st, fwd);
        }
        return fwd;
    }
    auto spos = [&](uint32_t i) {
        return (int32_t)(rec_at<GLOBAL>(cx, heavy, ep + i * es).y & kSuccPosMask);
    };
    auto push_i = [&](uint32_t i) {
        const uint32_t off = ep + i * es;
        push32<MULTI, GLOBAL, ALL_MAX, CHECK>(cx, heavy, off, rec_at<GLOBAL>(cx, heavy, off), x, c,
                                              place, st, fwd);
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
    return fwd;
}

// Relax the op at position v (record o at shared offset rp) whose arrivals are r (the max of
// its far, ring and forwarded arrivals).  Returns the forwarded arrival for position v + 1.
template <bool MULTI, bool ALL_MAX, bool CHECK, class PlaceT, class StateT>
__device__ __forceinline__ uint32_t relax32(const Ctx32 &cx, uint32_t rp, const uint4 o, int32_t v,
                                            int32_t ks, const uint8_t *heavy, const PlaceT &place,
                                            StateT &st, uint32_t r) {
    const int x = place.template at<CHECK>(v, (int)((o.w >> kOpXShift) & 7u));
    const uint32_t c = add_sat(max(r, st.dev(x)), o.x);    // C_v = S_v + p_v
    st.set_dev(x, c);
    const bool adj = (o.w & kOpAdj) != 0;
    if (!(o.w & kOpHeavy))
        return push_all32<MULTI, false, ALL_MAX, CHECK>(cx, heavy, rp + 16, o.w & kOpNoutMask, adj,
                                                        ks, x, c, place, st);
    const uint4 ext = lds_v4(cx.smem + rp + 16);   // ExtRec
    return push_all32<MULTI, true, ALL_MAX, CHECK>(cx, heavy, ext.x, ext.z, adj, ks, x, c, place, st);
}

template <bool MULTI>
__device__ __forceinline__ uint32_t next_rp(const Ctx32 &cx, uint32_t rp, uint32_t nout) {
    if (nout & kOpHeavy) return rp + 32;
    return rp + 16 + (nout & kOpNoutMask) * stride32<MULTI>(cx);
}

__device__ __forceinline__ uint4 op_at(const Ctx32 &cx, uint32_t rp) {
    return lds_v4(cx.smem + rp);
}
__device__ __forceinline__ uint32_t ring_at(const Ctx32 &cx, int32_t v) {
    return lds_u32(cx.ring + (uint32_t)(v & (kRing - 1)) * 128);
}
__device__ __forceinline__ uint32_t cold_at(const Ctx32 &cx, int32_t slot) {
    return slot >= 0 ? cx.cold[(size_t)slot * 32] : 0u;
}
__device__ __forceinline__ uint32_t arrivals(const uint4 o, uint32_t ring, uint32_t cold, uint32_t fwd) {
    uint32_t r = max(cold, fwd);
    return (o.w & kOp32HasNear) ? max(r, ring) : r;
}

// zero the slots an op opens with a first push (swap pairs only; times are >= 0)
template <bool MULTI>
__device__ __forceinline__ void clear_first32(const Ctx32 &cx, uint32_t rp, const uint8_t *heavy) {
    const uint4 o = op_at(cx, rp);
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
        const uint32_t bytes = rec.z & kT32SlotMask;
        if (rec.z & kT32Near) sts_u32(cx.ring + bytes, 0u);
        else *reinterpret_cast<uint32_t *>(reinterpret_cast<uint8_t *>(cx.cold) + bytes) = 0u;
    }
}

template <int MODE, int PL, bool MULTI>
__global__ void __launch_bounds__((kWarps + 1) * 32, 2)
eval32_kernel(const EvalParams P) {
    extern __shared__ __align__(128) uint8_t smem[];
    const int sb = P.stage_bytes32;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)kStages * sb);
    uint64_t *empty = full + kStages;
    uint8_t *cur = align16(reinterpret_cast<uint8_t *>(empty + kStages));
    uint8_t *lclass = cur;
    cur = align16(cur + 64);
    uint32_t *ring_all = reinterpret_cast<uint32_t *>(cur);
    cur = align16(cur + (size_t)kWarps * kRing * 32 * 4);
    uint32_t *stage_all = reinterpret_cast<uint32_t *>(cur);          // far-arrival staging
    cur = align16(cur + (size_t)kWarps * kRing * 32 * 4);
    uint32_t *dstate = reinterpret_cast<uint32_t *>(cur);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kWarps);
        }
        mbar_fence_init();
    }
    if (threadIdx.x < 64) lclass[threadIdx.x] = P.link_class[threadIdx.x];
    __syncthreads();

    auto runs_here = [&](int bl) {           // search: this kernel owns bases below saturation
        return MODE != 1 || P.gate == 0 || P.base_mk[bl] < (int64_t)kSat32;
    };

    if (warp == kWarps) {
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
    cx.smem = su32(smem);
    cx.ring = su32(ring_all + (size_t)warp * kRing * 32 + lane);
    cx.cold = P.state32 + ((size_t)(blockIdx.x * kWarps + warp) * P.max_W32) * 32 + lane;
    cx.lclass = su32(lclass);
    cx.edge_stride = P.edge_stride32;
    cx.D = P.D;
    cx.two_classes = P.n_classes > 1;
    const uint32_t stage = su32(stage_all + (size_t)warp * kRing * 32 + lane);

    using StateT = typename std::conditional<PL == 1, RegState32, SmemState32>::type;
    StateT st;
    if constexpr (PL != 1) {
        st.D = P.D;
        st.d = su32(dstate + (size_t)warp * (P.D + P.D * P.D) * 32 + lane);
        st.l = st.d + (uint32_t)P.D * 128;
    }

    // Far arrivals of position q arrive by cp.async into stage[q & 15], issued while position
    // q - kPrefetchDist is relaxed (its record names the slot); one commit group per position,
    // so waiting for all but kPrefetchDist groups makes position q's value visible.  The first
    // kPrefetchDist positions of a task load it directly.
    auto issue_far = [&](const uint4 o, int32_t v) {
        cp_async4(stage + (uint32_t)((v + kPrefetchDist) & (kRing - 1)) * 128,
                  cx.cold + (size_t)(int32_t)o.z * 32, (int32_t)o.z >= 0);
        cp_async_commit();
    };
    auto far_of = [&](const uint4 o, int32_t v) -> uint32_t {
        if ((int32_t)o.y < 0) return 0u;
        if (v < kPrefetchDist) return cx.cold[(size_t)(int32_t)o.y * 32];
        return lds_u32(stage + (uint32_t)(v & (kRing - 1)) * 128);
    };

    uint32_t it = 0;
    for (int64_t task = blockIdx.x; task < P.n_tasks; task += gridDim.x) {
        const int bl = MODE ? (int)(task / P.tasks_per_base) : 0;
        if (!runs_here(bl)) continue;
        const int64_t local = MODE ? task % P.tasks_per_base : task;
        const BaseLayoutDev *B = &P.bases[bl];
        const int nt = B->n_tiles32;
        const uint8_t *heavy = B->heavy32;
        const int64_t g = P.group_begin + local * kWarps + warp;

        Place32<MODE, PL> place;
        place.lane = lane;
        place.dmax = P.D - 1;
        place.all_allowed = P.all_allowed;
        place.rc = 0;
        place.rlen = 0;
        bool active, valid = true;
        const int64_t j = g * 32 + lane;
        int32_t ks = -1;
        int32_t check_end = P.n;                     // positions from here on need no check
        if (MODE == 0) {
            active = g * 32 < P.n_cand;
            place.pl = P.planes_in + (size_t)g * P.n * PL;
            if (active) valid = !((__ldg(P.invalid + g) >> lane) & 1u);
        } else {
            active = g < P.group_begin + P.groups_per_base;
            const int breal = P.b_offset + bl;
            const uint64_t cb = ctr_base_of(P.step, P.P_total, breal);
            const Region rg = decode_region(P.seed, cb, g, P.n);
            place.rc = rg.c;
            place.rlen = rg.len;
            check_end = rg.c + rg.len;
            place.allowed_pos = B->allowed_pos;
            const uint8_t *adj = B->adj_next;
            ks = active ? decode_swap(P.seed, cb, g, P.n, P.mix[3], rg,
                                      [&](int32_t k) { return __ldg(adj + k) != 0; })
                        : -1;
            const bool in_range = active && j >= P.j_begin && j < P.j_end;
            const int32_t *ord = B->order;
            const uint32_t *bits = B->bits;
            const uint8_t *aop = P.allowed_op;
            const int words = P.words;
            place.mv = in_range
                ? decode_lane(P.seed, cb, j, ks >= 0 && lane == 0, P.D, P.mix, rg,
                              [&](int32_t q) { return __ldg(ord + q); },
                              [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); },
                              [&](int32_t op) { return (unsigned)__ldg(aop + op); })
                : no_move();
            valid = in_range && place.mv.kind != kMoveInvalid;
            if (place.mv.kind == kMoveInvalid) place.mv = no_move();
        }
        st.init();

        // While op v is relaxed, op v+1's record and ring value are already loaded; its
        // distance-1 arrival is forwarded in `fwd`; far arrivals come through the staging ring.
        bool skip_first = false;
        uint32_t fwd = 0;
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
                    rp = next_rp<MULTI>(cx, rp, op_at(cx, rp).w);
                    v++;
                    skip_first = false;
                }
                uint4 o = op_at(cx, rp);
                uint32_t ringv = ring_at(cx, v);
                while (v < pos_end) {
                    const bool plain = MODE == 0 || (v >= check_end && ks < v);
                    if (plain || v != ks) {
                        const uint32_t rp_n = next_rp<MULTI>(cx, rp, o.w);
                        uint4 o_n = o;
                        uint32_t ring_n = 0;
                        if (v + 1 < pos_end) { o_n = op_at(cx, rp_n); ring_n = ring_at(cx, v + 1); }
                        issue_far(o, v);
                        cp_async_wait<kPrefetchDist>();
                        const uint32_t r = arrivals(o, ringv, far_of(o, v), fwd);
                        if (plain)
                            fwd = relax32<MULTI, false, false>(cx, rp, o, v, -1, heavy, place, st, r);
                        else
                            fwd = relax32<MULTI, false, true>(cx, rp, o, v, ks, heavy, place, st, r);
                        rp = rp_n; o = o_n; ringv = ring_n; v++;
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
                    const uint4 o_k1 = op_at(cx, rk1);
                    const uint32_t ring_k1 = ring_at(cx, v + 1);
                    issue_far(o_k, v);
                    issue_far(o_k1, v + 1);
                    cp_async_wait<kPrefetchDist>();
                    const uint32_t far_k = far_of(o_k, v), far_k1 = far_of(o_k1, v + 1);
                    clear_first32<MULTI>(cx, rk, heavy);
                    // k+1 first: its only distance-1 producer would be k, which it does not use
                    const uint32_t fwd_k2 = relax32<MULTI, false, true>(
                        cx, rk1, o_k1, v + 1, ks, heavy, place, st, arrivals(o_k1, ring_k1, far_k1, 0u));
                    relax32<MULTI, true, true>(cx, rk, o_k, v, ks, heavy, place, st,
                                               arrivals(o_k, ringv, far_k, fwd));
                    fwd = fwd_k2;
                    if (straddle) {
                        skip_first = true;
                        v = pos_end;
                    } else {
                        rp = next_rp<MULTI>(cx, rk1, o_k1.w);
                        v += 2;
                        if (v < pos_end) { o = op_at(cx, rp); ringv = ring_at(cx, v); }
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }
        cp_async_wait<0>();

        if (!active) continue;
        const uint32_t mk = st.makespan();
        if (MODE == 0) {
            if (j < P.n_cand) {
                if (!valid) {
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
            uint64_t key = valid ? (((uint64_t)mk << 24) | (uint64_t)j) : ~0ull;
            key = warp_min_u64(key);
            if (lane == 0 && key != ~0ull)
                atomicMin(reinterpret_cast<unsigned long long *>(P.keys + bl), (unsigned long long)key);
        }
    }
}

template <int MODE, int PL, bool MULTI>
cudaError_t launch_one32(const EvalParams &p, int grid, cudaStream_t st) {
    const int smem = eval32_smem_bytes(p, MODE);
    auto kern = eval32_kernel<MODE, PL, MULTI>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    kern<<<grid, (kWarps + 1) * 32, smem, st>>>(p);
    return cudaGetLastError();
}

template <int MODE, int PL, bool MULTI>
int occupancy_one32(const EvalParams &p) {
    const int smem = eval32_smem_bytes(p, MODE);
    auto kern = eval32_kernel<MODE, PL, MULTI>;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
        return 0;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, (kWarps + 1) * 32, smem) != cudaSuccess)
        return 0;
    return n;
}

int planes_of32(int D) { return D <= 2 ? 1 : (D <= 4 ? 2 : 4); }

}  // namespace

int eval32_smem_bytes(const EvalParams &p, int search_mode) {
    (void)search_mode;
    const int pl = planes_of32(p.D);
    size_t b = (size_t)kStages * p.stage_bytes32 + 2 * kStages * 8;
    b = (b + 15) & ~size_t(15);
    b += 64;
    b = (b + 15) & ~size_t(15);
    b += (size_t)kWarps * kRing * 32 * 4;          // near ring
    b = (b + 15) & ~size_t(15);
    b += (size_t)kWarps * kRing * 32 * 4;          // far-arrival staging
    b = (b + 15) & ~size_t(15);
    if (pl != 1) b += (size_t)kWarps * (p.D + p.D * p.D) * 32 * 4;
    return (int)b + 128;
}

// the edge stride is a compile-time 16 bytes unless some link class beyond the second exists
#define PESTO_DISPATCH32(FN, ...)                                                          \
    do {                                                                                   \
        const int pl = planes_of32(p.D);                                                   \
        const bool multi = p.n_classes > 2;                                                \
        if (search_mode) {                                                                 \
            if (pl == 1) return multi ? FN<1, 1, true>(__VA_ARGS__) : FN<1, 1, false>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<1, 2, true>(__VA_ARGS__) : FN<1, 2, false>(__VA_ARGS__); \
            return multi ? FN<1, 4, true>(__VA_ARGS__) : FN<1, 4, false>(__VA_ARGS__);     \
        } else {                                                                           \
            if (pl == 1) return multi ? FN<0, 1, true>(__VA_ARGS__) : FN<0, 1, false>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<0, 2, true>(__VA_ARGS__) : FN<0, 2, false>(__VA_ARGS__); \
            return multi ? FN<0, 4, true>(__VA_ARGS__) : FN<0, 4, false>(__VA_ARGS__);     \
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
