// kernels.cu -- sm_100a kernels of the Pesto hot path (product code).
//
//   K1 eval_kernel      makespan of 32 candidates per warp (one lane = one candidate), the DAG
//                       record stream TMA-staged (cp.async.bulk + mbarrier ring) into shared
//                       memory and shared by every warp of the CTA; neighbour moves (K2) decoded
//                       in the prologue; warp argmin + atomicMin epilogue (K3).
//   K5 transpose_kernel explicit placement rows -> bit-sliced [group][pos][plane] words.
//   K4 commit_kernel    apply each base's winning move.
//
// What K1 computes per lane is PAPER.md's objective for one (placement, order) candidate:
// ops run in pi order per device with no overlap (L146, L279, L374), an op starts after every
// input arrived (L144), a cross-device input arrives after its transfer, which waits for the
// directed link in FCFS order (L144, L188-198) and takes t_e = beta0 + beta1*bytes (L138);
// makespan = max completion (L159-162 eq. (3)).  Recursion:
//   S_v = max(max_in arrival, dev_free[x_v]);  C_v = S_v + p_v;  dev_free[x_v] = C_v
//   cross e=(v,w): A_e = max(C_v, link_free[x_v->x_w]) + t_e;  link_free[..] = A_e
//   arrival pushed (max) into w's ready-time slot, read when w is processed.
#include <algorithm>
#include <cstdio>
#include <type_traits>

#include "device_common.cuh"
#include "feasibility.cuh"
#include "internal.h"

namespace pesto {
namespace {

constexpr int64_t kInf64 = INT64_MAX;
using namespace dev;

// ---------------------------------------------------------------------------------------------
// per-lane device / link state
// ---------------------------------------------------------------------------------------------
struct RegState {            // D <= 2: two devices, two directed links, in registers
    int64_t d0, d1, l01, l10;
    __device__ void init(int) { d0 = d1 = l01 = l10 = 0; }
    __device__ int64_t dev(int x) const { return x ? d1 : d0; }
    __device__ void set_dev(int x, int64_t v) { if (x) d1 = v; else d0 = v; }
    __device__ int64_t link(int x, int) const { return x ? l10 : l01; }
    __device__ void set_link(int x, int, int64_t v) { if (x) l10 = v; else l01 = v; }
    __device__ int64_t makespan(int) const { return max(d0, d1); }
};

struct SmemState {           // D <= 8: [slot][lane] columns in shared memory (shared addresses)
    uint32_t d;              // [D][32] + lane
    uint32_t l;              // [D*D][32] + lane
    int D;
    __device__ void init(int) {
        for (int x = 0; x < D; x++) sts_u64(d + x * 256, 0);
        for (int x = 0; x < D * D; x++) sts_u64(l + x * 256, 0);
    }
    __device__ int64_t dev(int x) const { return (int64_t)lds_u64(d + x * 256); }
    __device__ void set_dev(int x, int64_t v) { sts_u64(d + x * 256, (uint64_t)v); }
    __device__ int64_t link(int x, int y) const { return (int64_t)lds_u64(l + (x * D + y) * 256); }
    __device__ void set_link(int x, int y, int64_t v) { sts_u64(l + (x * D + y) * 256, (uint64_t)v); }
    __device__ int64_t makespan(int) const {
        int64_t m = 0;
        for (int x = 0; x < D; x++) m = max(m, (int64_t)lds_u64(d + x * 256));
        return m;
    }
};

// ---------------------------------------------------------------------------------------------
// placement sources: each lane's device code for any position q (q is warp-uniform)
// ---------------------------------------------------------------------------------------------
template <int MODE, int PL>
struct Placement {
    // explicit rows (MODE 0): bit-sliced words of this warp's 32 candidates
    const uint32_t *pl;
    // search (MODE 1): base bits + the group's region + this lane's move
    const uint32_t *bits;
    const uint8_t *allowed_pos;
    int32_t rc, rlen;
    int words;
    int all_allowed;
    LaneMove mv;
    int lane;
    int dmax;
    const uint8_t *cpos;         // S9 coarse group: merged vertex by position (else unused)
    bool coarse;

    __device__ __forceinline__ int operator()(int32_t q) const {
        // MODE 0: this warp's group words, bit `lane`; MODE 2 (fixup list): each lane's own
        // candidate, i.e. its group's words (per-lane pointer) and bit (lane field = bit index)
        if (MODE != 1) return planes_dev_at<PL>(pl, q, lane, dmax);
        int x = ldg_bits_dev_at<PL>(bits, words, q);
        if ((uint32_t)(q - rc) < (uint32_t)rlen) {            // warp-uniform branch
            unsigned aq = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q);
            x = coarse ? apply_coarse(mv.ws, mv.wd, (int)__ldg(cpos + q), x, aq)
                       : apply_lane(mv, q, x, aq);
        }
        return x;
    }
};

// ---------------------------------------------------------------------------------------------
// the relaxation of one op and its pushes
// ---------------------------------------------------------------------------------------------
struct Ctx {
    int64_t *R;                  // this lane's ready-time slots: R[slot * 32]
    const uint8_t *lclass;       // shared-memory copy of the link-class table
    int edge_stride;
    int D;
    bool queue;                  // FCFS link queues; false: congestion-free links (f4)
};

template <bool GLOBAL>
__device__ __forceinline__ uint4 load_rec(const uint8_t *p) {
    if (GLOBAL) return __ldg(reinterpret_cast<const uint4 *>(p));
    return *reinterpret_cast<const uint4 *>(p);
}

template <bool MULTI, bool GLOBAL, bool ALL_MAX, class PlaceT, class StateT>
__device__ __forceinline__ void push_edge(const uint8_t *ep, const uint4 rec, int x, int64_t c,
                                          const PlaceT &place, StateT &st, const Ctx &cx) {
    const int64_t t0 = (int64_t)(((uint64_t)rec.y << 32) | rec.x);
    const int32_t succ = (int32_t)rec.z;
    const uint32_t sl = rec.w;
    const int y = place(succ);
    int64_t a = c;                                           // same device: C_v (L144)
    if (y != x) {                                            // cross: FCFS link x -> y
        int64_t t = t0;
        if (MULTI) {
            int cls = cx.lclass[x * cx.D + y];
            if (cls) {
                const int64_t *ext = reinterpret_cast<const int64_t *>(ep + 16) + (cls - 1);
                t = GLOBAL ? (int64_t)__ldg(reinterpret_cast<const long long *>(ext)) : *ext;
            }
        }
        a = max(c, st.link(x, y)) + t;                       // link state stays 0 if free
        if (cx.queue) st.set_link(x, y, a);
    }
    int64_t *slot = cx.R + (int64_t)(sl & kEdgeSlotMask) * 32;
    if (ALL_MAX || !(sl & kEdgeFirst)) a = max(a, *slot);
    *slot = a;
}

// out-edges of one producer, in record order except that under an active swap (ks, ks+1) the
// run of edges to ks+1 is pushed before the run to ks (the swapped order's consumer order).
template <bool MULTI, bool GLOBAL, bool ALL_MAX, class PlaceT, class StateT>
__device__ __forceinline__ void push_edges(const uint8_t *ep, uint32_t nout, int32_t ks, int x,
                                           int64_t c, const PlaceT &place, StateT &st,
                                           const Ctx &cx) {
    const int es = cx.edge_stride;
    for (uint32_t i = 0; i < nout;) {
        const uint4 rec = load_rec<GLOBAL>(ep + (size_t)i * es);
        if ((int32_t)rec.z != ks) {
            push_edge<MULTI, GLOBAL, ALL_MAX>(ep + (size_t)i * es, rec, x, c, place, st, cx);
            i++;
            continue;
        }
        uint32_t a_end = i;
        while (a_end < nout && (int32_t)load_rec<GLOBAL>(ep + (size_t)a_end * es).z == ks) a_end++;
        uint32_t b_end = a_end;
        while (b_end < nout && (int32_t)load_rec<GLOBAL>(ep + (size_t)b_end * es).z == ks + 1) b_end++;
        for (uint32_t e = a_end; e < b_end; e++)
            push_edge<MULTI, GLOBAL, ALL_MAX>(ep + (size_t)e * es, load_rec<GLOBAL>(ep + (size_t)e * es),
                                              x, c, place, st, cx);
        for (uint32_t e = i; e < a_end; e++)
            push_edge<MULTI, GLOBAL, ALL_MAX>(ep + (size_t)e * es, load_rec<GLOBAL>(ep + (size_t)e * es),
                                              x, c, place, st, cx);
        i = b_end;
    }
}

__device__ __forceinline__ const uint8_t *skip_op(const uint8_t *rp, int es) {
    const OpRec op = *reinterpret_cast<const OpRec *>(rp);
    if (op.nout & kOpHeavy) return rp + 32;
    return rp + 16 + (size_t)(op.nout & kOpNoutMask) * es;
}

// relax the op whose record starts at rp (shared memory), at position v
template <bool MULTI, bool ALL_MAX, class PlaceT, class StateT>
__device__ __forceinline__ void relax_op(const uint8_t *rp, int32_t v, int32_t ks,
                                         const uint8_t *heavy, const PlaceT &place, StateT &st,
                                         const Ctx &cx) {
    const OpRec op = *reinterpret_cast<const OpRec *>(rp);
    const int x = place(v);
    int64_t r = 0;
    if (op.in_slot >= 0) r = cx.R[(int64_t)op.in_slot * 32];
    const int64_t c = max(r, st.dev(x)) + op.p;              // S_v + p_v
    st.set_dev(x, c);
    if (!(op.nout & kOpHeavy)) {
        push_edges<MULTI, false, ALL_MAX>(rp + 16, op.nout & kOpNoutMask, ks, x, c, place, st, cx);
    } else {
        const ExtRec ext = *reinterpret_cast<const ExtRec *>(rp + 16);
        push_edges<MULTI, true, ALL_MAX>(heavy + ext.edge_off, (uint32_t)ext.nout, ks, x, c, place,
                                         st, cx);
    }
}

// zero the slots an op opens with a first push (swap pairs only; times are >= 0)
__device__ __forceinline__ void clear_first_targets(const uint8_t *rp, const uint8_t *heavy,
                                                    const Ctx &cx) {
    const OpRec op = *reinterpret_cast<const OpRec *>(rp);
    const uint8_t *ep;
    uint32_t nout;
    bool global = (op.nout & kOpHeavy) != 0;
    if (global) {
        const ExtRec ext = *reinterpret_cast<const ExtRec *>(rp + 16);
        ep = heavy + ext.edge_off;
        nout = (uint32_t)ext.nout;
    } else {
        ep = rp + 16;
        nout = op.nout & kOpNoutMask;
    }
    for (uint32_t i = 0; i < nout; i++) {
        uint4 rec = global ? load_rec<true>(ep + (size_t)i * cx.edge_stride)
                           : load_rec<false>(ep + (size_t)i * cx.edge_stride);
        if (rec.w & kEdgeFirst) cx.R[(int64_t)(rec.w & kEdgeSlotMask) * 32] = 0;
    }
}

// ---------------------------------------------------------------------------------------------
// K1
// ---------------------------------------------------------------------------------------------
template <int MODE, int PL, bool MULTI>
__global__ void __launch_bounds__((kWarps + 1) * 32, 2)
eval_kernel(const EvalParams P) {
    extern __shared__ __align__(128) uint8_t smem[];
    uint8_t *stage_buf = smem;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)kStages * P.stage_bytes);
    uint64_t *empty = full + kStages;
    uint8_t *cur = align16(reinterpret_cast<uint8_t *>(empty + kStages));
    uint8_t *lclass = cur;
    cur = align16(cur + 64);
    int64_t *dstate = reinterpret_cast<int64_t *>(cur);

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

    // MODE 2 (fixup list) sizes its work from the device-side count; search bases may be
    // gated to eval32 (gate 1 there) and only the saturated ones run here (gate 2)
    const int64_t n_tasks = (MODE == 2) ? ((int64_t)*(volatile const int32_t *)P.list_count +
                                           kWarps * 32 - 1) / (kWarps * 32)
                                        : P.n_tasks;
    auto runs_here = [&](int bl) {
        return MODE != 1 || P.gate != 2 || P.base_mk[bl] >= (int64_t)kSat32;
    };

    if (warp == kWarps) {
        // ---- producer: stream every task's tiles through the ring ----
        if (lane == 0) {
            uint32_t it = 0;
            for (int64_t task = blockIdx.x; task < n_tasks; task += gridDim.x) {
                const int bl = MODE == 1 ? (int)(task / P.tasks_per_base) : 0;
                if (!runs_here(bl)) continue;
                const BaseLayoutDev *B = &P.bases[bl];
                const int nt = B->n_tiles;
                for (int t = 0; t < nt; t++, it++) {
                    const int s = it % kStages;
                    if (it >= (uint32_t)kStages) mbar_wait(&empty[s], ((it / kStages) - 1) & 1);
                    const TileDesc td = B->tiles[t];
                    mbar_expect_tx(&full[s], (uint32_t)td.bytes);
                    bulk_g2s(stage_buf + (size_t)s * P.stage_bytes, B->blob + td.byte_off,
                             (uint32_t)td.bytes, &full[s]);
                }
            }
        }
        return;
    }

    // ---- consumers ----
    Ctx cx;
    cx.lclass = lclass;
    cx.edge_stride = P.edge_stride;
    cx.D = P.D;
    cx.queue = P.link_queue != 0;
    cx.R = P.state + ((int64_t)(blockIdx.x * kWarps + warp) * P.max_W) * 32 + lane;

    using StateT = typename std::conditional<PL == 1, RegState, SmemState>::type;
    StateT st;
    if constexpr (PL != 1) {
        st.D = P.D;
        st.d = su32(dstate + (size_t)warp * (P.D + P.D * P.D) * 32 + lane);
        st.l = st.d + (uint32_t)P.D * 256;
    }

    uint32_t it = 0;
    for (int64_t task = blockIdx.x; task < n_tasks; task += gridDim.x) {
        const int bl = MODE == 1 ? (int)(task / P.tasks_per_base) : 0;
        if (!runs_here(bl)) continue;
        const int64_t local = MODE == 1 ? task % P.tasks_per_base : task;
        const BaseLayoutDev *B = &P.bases[bl];
        const int nt = B->n_tiles;
        const uint8_t *heavy = B->heavy;
        const int64_t g = P.group_begin + local * kWarps + warp;

        Placement<MODE, PL> place;
        place.lane = lane;
        place.dmax = P.D - 1;
        place.words = P.words;
        place.all_allowed = P.all_allowed;
        place.coarse = false;
        place.cpos = nullptr;
        bool active, valid = true;
        int64_t j = g * 32 + lane;
        int32_t ks = -1;
        if (MODE == 0) {
            active = g * 32 < P.n_cand;
            place.pl = P.planes_in + (size_t)g * P.n * PL;
            if (active) valid = !((__ldg(P.invalid + g) >> lane) & 1u);
        } else if (MODE == 2) {
            const int32_t count = *(volatile const int32_t *)P.list_count;
            active = g * 32 < count;
            valid = j < count;
            const int32_t c = valid ? P.list[j] : 0;      // this lane's candidate
            place.pl = P.planes_in + (size_t)(c >> 5) * P.n * PL;
            place.lane = c & 31;
            j = c;
        } else {
            active = g < P.group_begin + P.groups_per_base;
            const int breal = P.b_offset + bl;
            const uint64_t cb = ctr_base_of(P.step, P.P_total, breal);
            const int64_t grp = (g * 32) >> kGroupShift;          // spec group of this warp
            const Region rg = decode_region(P.seed, cb, grp, P.n);
            place.coarse = coarse_group(P.seed, cb, grp, P.coarse_pct, P.n_coarse);
            place.rc = place.coarse ? 0 : rg.c;          // S9: a coarse group may move any op
            place.rlen = place.coarse ? P.n : rg.len;
            place.cpos = B->coarse_pos;
            place.bits = B->bits;
            place.allowed_pos = B->allowed_pos;
            const uint8_t *adj = B->swap_blocked;
            const int32_t *ord = B->order;
            const uint32_t *bits = B->bits;
            const uint8_t *aop = P.allowed_op;
            const int words = P.words;
            ks = active && !place.coarse
                     ? decode_swap(P.seed, cb, grp, P.n, P.mix[3], rg,
                                   [&](int32_t k) { return __ldg(adj + k) != 0; },
                                   [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); })
                     : -1;
            const bool in_range = active && j >= P.j_begin && j < P.j_end;
            if (place.coarse)
                place.mv = decode_coarse_lane(P.seed, cb, j, P.n_coarse, P.D);
            else place.mv = in_range
                ? decode_lane(P.seed, cb, j, ks >= 0 && (j & (kGroup - 1)) == 0, P.D, P.mix, rg,
                              [&](int32_t q) { return __ldg(ord + q); },
                              [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); },
                              [&](int32_t op) { return (unsigned)__ldg(aop + op); })
                : no_move();
            valid = in_range && place.mv.kind != kMoveInvalid;
            if (place.mv.kind == kMoveInvalid) place.mv = no_move();
            if (valid && (P.feas.has_cap || P.feas.has_coloc))    // row f3
                valid = move_feasible<PL>(place.mv, rg, P.D, bits, words, ord, B->allowed_pos,
                                          P.all_allowed, P.feas, P.feas.fbase + (size_t)bl * 8);
        }
        st.init(P.D);

        bool skip_first = false;
        for (int t = 0; t < nt; t++, it++) {
            const int s = it % kStages;
            mbar_wait(&full[s], (it / kStages) & 1);
            if (active) {
                const uint8_t *tile = stage_buf + (size_t)s * P.stage_bytes;
                const int32_t pos_begin = reinterpret_cast<const int32_t *>(tile)[0];
                const int32_t pos_end = reinterpret_cast<const int32_t *>(tile)[1];
                const uint8_t *rp = tile + kTileHeader;
                int32_t v = pos_begin;
                if (skip_first) {
                    rp = skip_op(rp, P.edge_stride);
                    v++;
                    skip_first = false;
                }
                while (v < pos_end) {
                    if (v != ks) {
                        relax_op<MULTI, false>(rp, v, ks, heavy, place, st, cx);
                        rp = skip_op(rp, P.edge_stride);
                        v++;
                        continue;
                    }
                    // swapped pair: ops at ks+1 then ks
                    const uint8_t *rk = rp;
                    const uint8_t *rk1;
                    const bool straddle = (v + 1 == pos_end);
                    if (straddle) {
                        const int s2 = (it + 1) % kStages;
                        mbar_wait(&full[s2], ((it + 1) / kStages) & 1);
                        rk1 = stage_buf + (size_t)s2 * P.stage_bytes + kTileHeader;
                    } else {
                        rk1 = skip_op(rk, P.edge_stride);
                    }
                    clear_first_targets(rk, heavy, cx);
                    relax_op<MULTI, false>(rk1, v + 1, ks, heavy, place, st, cx);
                    relax_op<MULTI, true>(rk, v, ks, heavy, place, st, cx);
                    if (straddle) {
                        skip_first = true;
                        v = pos_end;
                    } else {
                        rp = skip_op(rk1, P.edge_stride);
                        v += 2;
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
        }

        if (!active) continue;
        const int64_t mk = st.makespan(P.D);                 // C_max = max_d dev_free[d]
        if (MODE == 0) {
            if (j < P.n_cand) P.makespans[j] = valid ? mk : kInf64;
        } else if (MODE == 2) {
            if (valid) P.makespans[j] = mk;                  // listed rows are feasible
        } else {
            uint64_t key = valid ? (((uint64_t)mk << 24) | (uint64_t)j) : ~0ull;
            if (P.keys_dbg && j >= P.j_begin && j < P.j_end) P.keys_dbg[j - P.j_begin] = key;
            key = warp_min_u64(key);
            if (lane == 0 && key != ~0ull)
                atomicMin(reinterpret_cast<unsigned long long *>(P.keys + bl),
                          (unsigned long long)key);
        }
    }
}

// ---------------------------------------------------------------------------------------------
// K5: rows of b-bit codes (op-id order) -> per group of 32 rows, [pos][plane] words whose bit l
// is candidate l's bit; plus the mask of rows holding an infeasible code.
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t compress2(uint32_t w) {  // even bits -> low 16
    w &= 0x55555555u;
    w = (w | (w >> 1)) & 0x33333333u;
    w = (w | (w >> 2)) & 0x0F0F0F0Fu;
    w = (w | (w >> 4)) & 0x00FF00FFu;
    w = (w | (w >> 8)) & 0x0000FFFFu;
    return w;
}
__device__ __forceinline__ uint32_t compress4(uint32_t w) {  // every 4th bit -> low 8
    w &= 0x11111111u;
    w = (w | (w >> 3)) & 0x03030303u;
    w = (w | (w >> 6)) & 0x000F000Fu;
    w = (w | (w >> 12)) & 0x000000FFu;
    return w;
}
__device__ __forceinline__ uint32_t transpose32(uint32_t w, int lane) {
    const uint32_t masks[5] = {0x0000FFFFu, 0x00FF00FFu, 0x0F0F0F0Fu, 0x33333333u, 0x55555555u};
#pragma unroll
    for (int s = 0; s < 5; s++) {
        const int j = 16 >> s;
        const uint32_t m = masks[s];
        const uint32_t o = __shfl_xor_sync(0xffffffffu, w, j);
        w = (lane & j) ? ((w & ~m) | ((o & ~m) >> j)) : ((w & m) | ((o & m) << j));
    }
    return w;
}

template <int PL>
__global__ void __launch_bounds__(256) transpose_kernel(const TransposeParams P) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t g = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); g < P.n_groups;
         g += warps) {
        const int64_t row = g * 32 + lane;
        const uint8_t *rp = P.rows + row * P.stride;
        const bool have = row < P.n_cand;
        uint32_t bad = 0;
        const int chunks = (P.n + 31) >> 5;
        for (int c = 0; c < chunks; c++) {
            uint32_t pw[PL];
            if (PL == 1) {
                pw[0] = have ? __ldg(reinterpret_cast<const uint32_t *>(rp) + c) : 0u;
            } else if (PL == 2) {
                uint2 w = have ? __ldg(reinterpret_cast<const uint2 *>(rp) + c) : make_uint2(0, 0);
                pw[0] = compress2(w.x) | (compress2(w.y) << 16);
                pw[1] = compress2(w.x >> 1) | (compress2(w.y >> 1) << 16);
            } else {
                uint4 w = have ? __ldg(reinterpret_cast<const uint4 *>(rp) + c) : make_uint4(0, 0, 0, 0);
#pragma unroll
                for (int k = 0; k < PL; k++)
                    pw[k] = compress4(w.x >> k) | (compress4(w.y >> k) << 8) |
                            (compress4(w.z >> k) << 16) | (compress4(w.w >> k) << 24);
            }
#pragma unroll
            for (int k = 0; k < PL; k++) pw[k] = transpose32(pw[k], lane);
            const int op = c * 32 + lane;                     // lane now holds op's 32 codes
            if (op < P.n) {
                const unsigned fm = __ldg(P.fmask + op);
                if (fm) {
                    for (int code = 0; code < (1 << PL); code++) {
                        if (!((fm >> code) & 1u)) continue;
                        uint32_t match = 0xffffffffu;
#pragma unroll
                        for (int k = 0; k < PL; k++) match &= ((code >> k) & 1) ? pw[k] : ~pw[k];
                        bad |= match;
                    }
                }
                uint32_t *out = P.planes_out + ((size_t)g * P.n + __ldg(P.pos_of + op)) * PL;
                if (PL == 1) out[0] = pw[0];
                else if (PL == 2) *reinterpret_cast<uint2 *>(out) = make_uint2(pw[0], pw[1]);
                else *reinterpret_cast<uint4 *>(out) = make_uint4(pw[0], pw[1], pw[2], pw[3]);
            }
        }
        bad = __reduce_or_sync(0xffffffffu, bad);
        if (lane == 0) P.invalid_out[g] = bad;
    }
}

// K5, shared-memory variant: one CTA per 32-row group.  The rows are read once with 16-byte
// loads (a row's sectors are reused from L1 by the following loads), the permutation to
// position order is applied in shared memory, and the group's n*PL words leave with coalesced
// stores -- the global-scatter variant above wrote 4 bytes per 32-byte sector.
#ifndef PESTO_T16
#define PESTO_T16 4
#endif
constexpr int kT16 = PESTO_T16;
// successor positions per thread in flight in K5's edge-slot gather: 24 where shared memory
// allows two CTAs per SM anyway (large graphs: 106 registers fit), 8 where three fit (80
// registers) -- transformer_2dev, 1 M rows: 6.89 (8) -> 5.69 (16) -> 5.50 ms (24); inception at
// 16 would drop to two CTAs per SM; 8 row chunks per lane in flight instead of 4: 5.93 ms
#ifndef PESTO_YU
#define PESTO_YU 8
#endif
#ifndef PESTO_YU_BIG
#define PESTO_YU_BIG 24
#endif
template <int PL, int kYU = PESTO_YU>
__global__ void __launch_bounds__(256) transpose_smem_kernel(const TransposeParams P) {
    extern __shared__ uint4 tsm[];
    uint32_t *out_s = reinterpret_cast<uint32_t *>(tsm);
    __shared__ uint32_t bad_s;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int n16 = (P.n * PL + 127) / 128;             // 16-byte chunks of a row
    const int nw = P.n * PL;                            // output words of a group
    for (int64_t g = blockIdx.x; g < P.n_groups; g += gridDim.x) {
        if (threadIdx.x == 0) bad_s = 0;
        const int64_t row = g * 32 + lane;
        const bool have = row < P.n_cand;
        const uint4 *rp = reinterpret_cast<const uint4 *>(P.rows + row * P.stride);
        uint32_t bad = 0;
        // chunk c = ops [32c, 32c + 32); fm, q: the lane's op's forbidden codes and position
        auto emit = [&](int c, uint32_t (&pw)[PL], unsigned fm, int q) {
#pragma unroll
            for (int k = 0; k < PL; k++) pw[k] = transpose32(pw[k], lane);
            const int op = c * 32 + lane;
            if (op >= P.n) return;
            if (fm) {
                for (int code = 0; code < (1 << PL); code++) {
                    if (!((fm >> code) & 1u)) continue;
                    uint32_t match = 0xffffffffu;
#pragma unroll
                    for (int k = 0; k < PL; k++) match &= ((code >> k) & 1) ? pw[k] : ~pw[k];
                    bad |= match;
                }
            }
#pragma unroll
            for (int k = 0; k < PL; k++) out_s[q * PL + k] = pw[k];
        };
        constexpr int CPK = 4 / PL;                     // 32-op chunks per 16-byte row chunk
        __syncthreads();
        // kT16 of the row's 16-byte chunks per lane are loaded before any is used: with one
        // load in flight per warp (16 warps per SM) the load phase ran at ~1 TB/s
        for (int kb = warp; kb < n16; kb += 8 * kT16) {
          uint4 wv[kT16];
#pragma unroll
          for (int u = 0; u < kT16; u++) {
              const int k16 = kb + 8 * u;
              wv[u] = (have && k16 < n16) ? __ldg(rp + k16) : make_uint4(0, 0, 0, 0);
          }
          // the ops' masks and positions, also loaded before first use
          unsigned fmv[kT16 * CPK];
          int qv[kT16 * CPK];
#pragma unroll
          for (int u = 0; u < kT16; u++) {
#pragma unroll
              for (int j = 0; j < CPK; j++) {
                  const int op = (CPK * (kb + 8 * u) + j) * 32 + lane;
                  const bool in = op < P.n;
                  fmv[u * CPK + j] = in ? __ldg(P.fmask + op) : 0u;
                  qv[u * CPK + j] = in ? __ldg(P.pos_of + op) : 0;
              }
          }
#pragma unroll
          for (int u = 0; u < kT16; u++) {
            const int k16 = kb + 8 * u;
            if (k16 >= n16) break;
            const uint4 w = wv[u];
            if (PL == 1) {
                const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
                for (int j = 0; j < 4; j++) {
                    uint32_t pw[PL];
                    pw[0] = ws[j];
                    emit(4 * k16 + j, pw, fmv[u * CPK + j], qv[u * CPK + j]);
                }
            } else if (PL == 2) {
                const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
                for (int j = 0; j < 2; j++) {
                    uint32_t pw[PL];
                    const uint32_t lo = ws[2 * j], hi = ws[2 * j + 1];
                    pw[0] = compress2(lo) | (compress2(hi) << 16);
                    pw[1] = compress2(lo >> 1) | (compress2(hi >> 1) << 16);
                    emit(2 * k16 + j, pw, fmv[u * CPK + j], qv[u * CPK + j]);
                }
            } else {
                uint32_t pw[PL];
#pragma unroll
                for (int k = 0; k < PL; k++)
                    pw[k] = compress4(w.x >> k) | (compress4(w.y >> k) << 8) |
                            (compress4(w.z >> k) << 16) | (compress4(w.w >> k) << 24);
                emit(k16, pw, fmv[u], qv[u]);
            }
          }
        }
        bad = __reduce_or_sync(0xffffffffu, bad);
        if (lane == 0 && bad) atomicOr(&bad_s, bad);
        __syncthreads();
        uint32_t *dst = P.planes_out + (size_t)g * nw;
        for (int i = threadIdx.x; i < nw; i += blockDim.x) dst[i] = out_s[i];
        if (P.yplanes_out) {                   // the edge-slot stream of the eval32 walk
            // kYU successor positions per thread in flight (one dependent L2 load per slot
            // left K5 waiting on long scoreboards)
            uint32_t *ydst = P.yplanes_out + (size_t)g * P.n_slots * PL;
            for (int64_t i0 = threadIdx.x; i0 < P.n_slots; i0 += (int64_t)blockDim.x * kYU) {
                int32_t qv[kYU];
#pragma unroll
                for (int u = 0; u < kYU; u++) {
                    const int64_t i = i0 + (int64_t)u * blockDim.x;
                    qv[u] = i < P.n_slots ? __ldg(P.slot_succ + i) : -1;
                }
#pragma unroll
                for (int u = 0; u < kYU; u++) {
                    const int64_t i = i0 + (int64_t)u * blockDim.x;
                    if (i >= P.n_slots) break;
#pragma unroll
                    for (int k = 0; k < PL; k++)
                        ydst[i * PL + k] = qv[u] >= 0 ? out_s[qv[u] * PL + k] : 0u;
                }
            }
        }
        if (threadIdx.x == 0) P.invalid_out[g] = bad_s;
    }
}

// the edge-slot stream from plane words in global memory (used after the global-scatter K5)
template <int PL>
__global__ void __launch_bounds__(256) ystream_kernel(const TransposeParams P) {
    const int64_t total = P.n_groups * P.n_slots;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t g = t / P.n_slots, i = t % P.n_slots;
        const int32_t q = __ldg(P.slot_succ + i);
        const uint32_t *src = P.planes_out + ((size_t)g * P.n + (q >= 0 ? q : 0)) * PL;
#pragma unroll
        for (int k = 0; k < PL; k++) P.yplanes_out[t * PL + k] = q >= 0 ? src[k] : 0u;
    }
}

// ---------------------------------------------------------------------------------------------
// K4: commit the winner of every base (one warp per base: the lanes share the move's positions)
// ---------------------------------------------------------------------------------------------
template <int PL>
__device__ void set_dev_at(uint32_t *bits, int words, int32_t q, int x) {   // lanes may share words
#pragma unroll
    for (int k = 0; k < PL; k++) {
        uint32_t *w = bits + k * words + (q >> 5);
        const uint32_t m = 1u << (q & 31);
        if ((x >> k) & 1) atomicOr(w, m);
        else atomicAnd(w, ~m);
    }
}
template <int PL>
__device__ int get_dev_at(const uint32_t *bits, int words, int32_t q) {
    int x = 0;
#pragma unroll
    for (int k = 0; k < PL; k++) x |= (int)((bits[k * words + (q >> 5)] >> (q & 31)) & 1u) << k;
    return x;
}

template <int PL>
__global__ void commit_kernel(const CommitParams P) {
    const int b = blockIdx.x, lane = threadIdx.x;
    const uint64_t key = P.keys[b];
    if (key == ~0ull) {
        if (lane == 0) P.swap_out[b] = -1;
        return;
    }
    const int64_t j = (int64_t)(key & ((1ull << 24) - 1));
    const BaseLayoutDev &B = P.bases[b];
    uint32_t *bits = P.bits + (size_t)b * PL * P.words;
    const uint64_t cb = ctr_base_of(P.step, P.P, b);
    const uint8_t *adj = B.swap_blocked;
    const Region rg = decode_region(P.seed, cb, j >> kGroupShift, P.n);
    const bool coarse = coarse_group(P.seed, cb, j >> kGroupShift, P.coarse_pct, P.n_coarse);
    const int32_t ks = j == 0 || coarse ? -1
                              : decode_swap(P.seed, cb, j >> kGroupShift, P.n, P.mix[3], rg,
                                            [&](int32_t k) { return adj[k] != 0; },
                                            [&](int32_t q) { return get_dev_at<PL>(bits, P.words, q); });
    const int words = P.words;
    const LaneMove mv = j == 0 ? no_move()
        : coarse ? decode_coarse_lane(P.seed, cb, j, P.n_coarse, P.D)
        : decode_lane(P.seed, cb, j, ks >= 0 && (j & (kGroup - 1)) == 0, P.D, P.mix, rg,
                      [&](int32_t q) { return B.order[q]; },
                      [&](int32_t q) { return get_dev_at<PL>(bits, words, q); },
                      [&](int32_t op) { return (unsigned)P.allowed_op[op]; });
    __syncwarp();                       // every lane decoded from the unmodified base
    if (lane == 0) {
        P.base_mk[b] = (int64_t)(key >> 24);
        P.swap_out[b] = ks;
    }
    if (j == 0) return;
    // the base code is also embedded in the eval32 records that name position q: the op's
    // own record and every edge record whose successor sits at q
    uint8_t *blob32 = const_cast<uint8_t *>(B.blob32);
    uint8_t *heavy32 = const_cast<uint8_t *>(B.heavy32);
    auto set_dev = [&](int32_t q, int x) {
        if (P.feas.has_cap) {                 // row f3: the base's footprint per device
            const int old = get_dev_at<PL>(bits, words, q);
            const long long m = (long long)P.feas.mem[B.order[q]];
            atomicAdd(reinterpret_cast<unsigned long long *>(P.feas.fbase + (size_t)b * 8 + old),
                      (unsigned long long)(-m));
            atomicAdd(reinterpret_cast<unsigned long long *>(P.feas.fbase + (size_t)b * 8 + x),
                      (unsigned long long)m);
        }
        set_dev_at<PL>(bits, words, q, x);
        if (B.W32 == 0) return;           // this base has no eval32 records (per base)
        uint32_t *flags = reinterpret_cast<uint32_t *>(blob32 + B.op_off32[q]) + 3;   // StepHead
        *flags = (*flags & ~kStXMask) | (uint32_t)x;
        if (PL <= 2) {
            // the fast walk's dispatch entries (StepHead.kinds, D <= 4): xu of every step of the
            // op (atomics: another lane may set a yu bit of the same word)
            const uint32_t nst = *flags >> kStStepsShift;
            constexpr int xs = PL == 1 ? kind_xshift(2) : kind_xshift(4);
            constexpr uint32_t cm = kind_code_mask(PL == 1 ? 2 : 4);
            const uint32_t xm = (cm << xs) * 0x101u;
            const uint32_t xv = ((uint32_t)x << xs) * 0x101u;
            for (uint32_t k = 0; k < nst; k++) {
                uint32_t *kinds = reinterpret_cast<uint32_t *>(blob32 + B.op_off32[q] + k * kStepBytes) + 1;
                atomicAnd(kinds, ~xm);
                if (xv) atomicOr(kinds, xv);
            }
        }
        for (uint32_t i = B.pin_off[q]; i < B.pin_off[q + 1]; i++) {
            const uint32_t ref = B.pin_ref[i];
            uint8_t *base = (ref & kPinHeavy) ? heavy32 : blob32;
            uint32_t *succ = reinterpret_cast<uint32_t *>(base + (ref & kPinOffMask)) + 1;
            *succ = (*succ & ~(7u << kSuccXShift)) | ((uint32_t)x << kSuccXShift);
            if (PL <= 2 && !(ref & kPinHeavy)) {      // yu of this slot in its step's kinds
                const uint32_t slot = (ref & kPinSlot) ? 1u : 0u;
                uint32_t *kinds = reinterpret_cast<uint32_t *>(blob32 + (ref & kPinOffMask) -
                                                               16u * (slot + 1u)) + 1;
                constexpr uint32_t cm = kind_code_mask(PL == 1 ? 2 : 4);
                const uint32_t ym = cm << (8 * slot);
                atomicAnd(kinds, ~ym);
                if (x) atomicOr(kinds, (uint32_t)x << (8 * slot));
            }
        }
    };
    if (mv.kind == kMoveFlip) {
        // flips apply in sequence; a position flipped twice keeps its last device
        if (lane < mv.nflip) {
            bool last = true;
            for (int f = lane + 1; f < mv.nflip; f++) last = last && mv.fpos[f] != mv.fpos[lane];
            if (last) set_dev(mv.fpos[lane], mv.fdev[lane]);
        }
    } else if (mv.kind == kMoveWindow) {
        for (int32_t q = mv.ws + lane; q < mv.ws + mv.wl; q += 32)
            if ((B.allowed_pos[q] >> mv.wd) & 1u) set_dev(q, mv.wd);
    } else if (mv.kind == kMoveCoarse) {       // S9: every op of merged vertex ws that allows wd
        for (int32_t q = lane; q < P.n; q += 32)
            if (B.coarse_pos[q] == mv.ws && ((B.allowed_pos[q] >> mv.wd) & 1u)) set_dev(q, mv.wd);
    }
    __threadfence();                     // every lane's bit updates are performed ...
    __syncwarp();                        // ... before lane 0 reads the planes for the swap
    if (ks >= 0 && lane == 0) {          // ops at ks and ks+1 exchange positions
        const int a = get_dev_at<PL>(bits, words, ks), c = get_dev_at<PL>(bits, words, ks + 1);
        set_dev_at<PL>(bits, words, ks, c);
        set_dev_at<PL>(bits, words, ks + 1, a);
    }
}

template <int MODE, int PL, bool MULTI>
cudaError_t launch_one(const EvalParams &p, int grid, cudaStream_t st) {
    const int smem = eval_smem_bytes(p, MODE);
    auto kern = eval_kernel<MODE, PL, MULTI>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    kern<<<grid, (kWarps + 1) * 32, smem, st>>>(p);
    return cudaGetLastError();
}

template <int MODE, int PL, bool MULTI>
int occupancy_one(const EvalParams &p) {
    const int smem = eval_smem_bytes(p, MODE);
    auto kern = eval_kernel<MODE, PL, MULTI>;
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
        return 0;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, (kWarps + 1) * 32, smem) != cudaSuccess)
        return 0;
    return n;
}

int planes_of(int D) { return D <= 2 ? 1 : (D <= 4 ? 2 : 4); }

}  // namespace

static int64_t g_launches = 0;
void note_launch() { __atomic_add_fetch(&g_launches, 1, __ATOMIC_RELAXED); }
int64_t launch_count_value() { return __atomic_load_n(&g_launches, __ATOMIC_RELAXED); }

int eval_smem_bytes(const EvalParams &p, int search_mode) {
    size_t b = (size_t)kStages * p.stage_bytes + 2 * kStages * 8;
    b = (b + 15) & ~size_t(15);
    b += 64;
    b = (b + 15) & ~size_t(15);
    if (search_mode) b += (size_t)kWarps * p.words * 4;
    b = (b + 15) & ~size_t(15);
    if (planes_of(p.D) != 1) b += (size_t)kWarps * (p.D + p.D * p.D) * 32 * 8;
    return (int)b + 128;
}

#define PESTO_DISPATCH(FN, ...)                                                            \
    do {                                                                                   \
        const int pl = planes_of(p.D);                                                     \
        const bool multi = p.n_classes > 1;                                                \
        if (search_mode == 2) {                                                            \
            if (pl == 1) return multi ? FN<2, 1, true>(__VA_ARGS__) : FN<2, 1, false>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<2, 2, true>(__VA_ARGS__) : FN<2, 2, false>(__VA_ARGS__); \
            return multi ? FN<2, 4, true>(__VA_ARGS__) : FN<2, 4, false>(__VA_ARGS__);     \
        } else if (search_mode) {                                                          \
            if (pl == 1) return multi ? FN<1, 1, true>(__VA_ARGS__) : FN<1, 1, false>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<1, 2, true>(__VA_ARGS__) : FN<1, 2, false>(__VA_ARGS__); \
            return multi ? FN<1, 4, true>(__VA_ARGS__) : FN<1, 4, false>(__VA_ARGS__);     \
        } else {                                                                           \
            if (pl == 1) return multi ? FN<0, 1, true>(__VA_ARGS__) : FN<0, 1, false>(__VA_ARGS__); \
            if (pl == 2) return multi ? FN<0, 2, true>(__VA_ARGS__) : FN<0, 2, false>(__VA_ARGS__); \
            return multi ? FN<0, 4, true>(__VA_ARGS__) : FN<0, 4, false>(__VA_ARGS__);     \
        }                                                                                  \
    } while (0)

cudaError_t launch_eval(const EvalParams &p, int search_mode, int grid, cudaStream_t st) {
    note_launch();
    PESTO_DISPATCH(launch_one, p, grid, st);
}

int eval_max_ctas_per_sm(const EvalParams &p, int search_mode) {
    PESTO_DISPATCH(occupancy_one, p);
}

cudaError_t launch_transpose(const TransposeParams &p, cudaStream_t st) {
    note_launch();
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (p.n_groups <= 0) return cudaSuccess;
    const size_t smem = (size_t)p.n * p.planes * 4;
    if (smem <= (size_t)kTransposeSmemMax) {          // one CTA per group, output staged in smem
        auto set = [&](const void *f) {
            return cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        };
        // two CTAs per SM at most (by shared memory): the deeper gather (more registers)
        const bool big = 3 * (smem + 1024) > 228 * 1024;
        cudaError_t e = p.planes == 1 ? (big ? set((const void *)transpose_smem_kernel<1, PESTO_YU_BIG>)
                                             : set((const void *)transpose_smem_kernel<1>))
                      : p.planes == 2 ? set((const void *)transpose_smem_kernel<2>)
                                      : set((const void *)transpose_smem_kernel<4>);
        if (e != cudaSuccess) return e;
        const int per_sm = std::max(1, (int)(200 * 1024 / std::max<size_t>(smem, 1)));
        const int grid = (int)std::min<int64_t>(p.n_groups, (int64_t)sms * std::min(per_sm, 8));
        if (p.planes == 1 && big) transpose_smem_kernel<1, PESTO_YU_BIG><<<grid, 256, smem, st>>>(p);
        else if (p.planes == 1) transpose_smem_kernel<1><<<grid, 256, smem, st>>>(p);
        else if (p.planes == 2) transpose_smem_kernel<2><<<grid, 256, smem, st>>>(p);
        else transpose_smem_kernel<4><<<grid, 256, smem, st>>>(p);
        return cudaGetLastError();
    }
    const int64_t blocks_needed = (p.n_groups + 7) / 8;
    const int grid = (int)std::min<int64_t>(blocks_needed, (int64_t)sms * 8);
    if (p.planes == 1) transpose_kernel<1><<<grid, 256, 0, st>>>(p);
    else if (p.planes == 2) transpose_kernel<2><<<grid, 256, 0, st>>>(p);
    else transpose_kernel<4><<<grid, 256, 0, st>>>(p);
    if (p.yplanes_out) {
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        const int yg = sms * 8;
        if (p.planes == 1) ystream_kernel<1><<<yg, 256, 0, st>>>(p);
        else if (p.planes == 2) ystream_kernel<2><<<yg, 256, 0, st>>>(p);
        else ystream_kernel<4><<<yg, 256, 0, st>>>(p);
    }
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------------
// Layout patch for committed swaps (search.cpp swap_in_place): one CTA applies the host's list.
// ---------------------------------------------------------------------------------------------
static __global__ void patch_kernel(const PatchOp *ops, int n_ops) {
    extern __shared__ uint4 pbuf[];
    for (int i = 0; i < n_ops; i++) {
        const PatchOp op = ops[i];
        if (op.kind != kPatchRotate) continue;
        uint4 *p = reinterpret_cast<uint4 *>(op.ptr);
        const int na = (int)(op.a / 16), nb = (int)(op.b / 16);
        for (int t = threadIdx.x; t < na + nb; t += blockDim.x) pbuf[t] = p[t];
        __syncthreads();
        for (int t = threadIdx.x; t < na + nb; t += blockDim.x) p[t] = t < nb ? pbuf[na + t] : pbuf[t - nb];
        __syncthreads();
    }
    if (threadIdx.x != 0) return;
    for (int i = 0; i < n_ops; i++) {            // in order: later stores win
        const PatchOp op = ops[i];
        if (op.kind == kPatchSet32) {
            uint32_t *w = reinterpret_cast<uint32_t *>(op.ptr);
            *w = (*w & ~op.mask) | (op.val & op.mask);
        } else if (op.kind == kPatchSet8) {
            *reinterpret_cast<uint8_t *>(op.ptr) = (uint8_t)op.val;
        }
    }
}

cudaError_t launch_patch(const PatchOp *ops_dev, int n_ops, int max_block, cudaStream_t st) {
    note_launch();
    patch_kernel<<<1, 256, (size_t)std::max(max_block, 16), st>>>(ops_dev, n_ops);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------------
// Row f3 for explicit rows: one CTA per 32-row group marks the rows whose per-device footprint
// exceeds its cap (L202) or whose colocation groups are split (L175).  Lane = row; the 8 warps
// share the positions, then warp 0 adds their partial footprints.
// ---------------------------------------------------------------------------------------------
template <int PL>
__global__ void __launch_bounds__(256) feasibility_kernel(const FeasParams P) {
    __shared__ long long part[8][8][32];             // [warp][device][lane]
    __shared__ uint32_t bad_s;
    const int lane = threadIdx.x & 31, wq = threadIdx.x >> 5;
    const Feasibility &F = P.feas;
    for (int64_t g = blockIdx.x; g < P.n_groups; g += gridDim.x) {
        if (threadIdx.x == 0) bad_s = 0;
        const uint32_t *pl = P.planes + (size_t)g * P.n * PL;
        __syncthreads();
        if (F.has_cap) {
            long long f[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            for (int32_t q = wq; q < P.n; q += 8) {
                int code = 0;
#pragma unroll
                for (int k = 0; k < PL; k++) code |= (int)((__ldg(pl + (size_t)q * PL + k) >> lane) & 1u) << k;
                const long long m = __ldg(reinterpret_cast<const long long *>(F.mem) + __ldg(P.order + q));
#pragma unroll
                for (int d = 0; d < 8; d++) f[d] += d == code ? m : 0;
            }
#pragma unroll
            for (int d = 0; d < 8; d++) part[wq][d][lane] = f[d];
        }
        uint32_t bad = 0;
        if (F.has_coloc) {
            for (int i = threadIdx.x; i < F.n_pairs; i += blockDim.x) {
                const int2 pr = F.coloc_pairs[i];
                const int32_t qa = __ldg(P.pos_of + pr.x), qb = __ldg(P.pos_of + pr.y);
#pragma unroll
                for (int k = 0; k < PL; k++) bad |= __ldg(pl + (size_t)qa * PL + k) ^ __ldg(pl + (size_t)qb * PL + k);
            }
        }
        __syncthreads();
        if (F.has_cap && wq == 0) {
            bool over = false;
            for (int d = 0; d < P.D; d++) {
                long long tot = 0;
#pragma unroll
                for (int w = 0; w < 8; w++) tot += part[w][d][lane];
                over = over || tot > __ldg(reinterpret_cast<const long long *>(F.cap) + d);
            }
            bad |= __ballot_sync(0xffffffffu, over);
        }
        if (bad) atomicOr(&bad_s, bad);
        __syncthreads();
        if (threadIdx.x == 0 && bad_s) P.invalid[g] |= bad_s;
        __syncthreads();
    }
}

cudaError_t launch_feasibility(const FeasParams &p, cudaStream_t st) {
    note_launch();
    if (p.n_groups <= 0) return cudaSuccess;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = (int)std::min<int64_t>(p.n_groups, (int64_t)sms * 4);
    if (p.planes_n == 1) feasibility_kernel<1><<<grid, 256, 0, st>>>(p);
    else if (p.planes_n == 2) feasibility_kernel<2><<<grid, 256, 0, st>>>(p);
    else feasibility_kernel<4><<<grid, 256, 0, st>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_commit(const CommitParams &p, cudaStream_t st) {
    note_launch();
    if (p.planes == 1) commit_kernel<1><<<p.P, 32, 0, st>>>(p);
    else if (p.planes == 2) commit_kernel<2><<<p.P, 32, 0, st>>>(p);
    else commit_kernel<4><<<p.P, 32, 0, st>>>(p);
    return cudaGetLastError();
}

}  // namespace pesto
