// eval32.cu -- K1 fast path: the makespan recursion in 32-bit saturating time (product code).
//
// Same recursion as eval64 (kernels.cu; PAPER.md L142-146, L188-198, L374 -- DESIGN.md §3):
//   S_v = max(max_in arrival, dev_free[x_v]);  C_v = S_v + p_v;  dev_free[x_v] = C_v
//   cross e=(v,w): A_e = max(C_v, link_free[x_v->x_w]) + t_e;  link_free = A_e
// Layout of the work:
//   * one warp walks the DAG record stream once for 32 x CPL candidates: every lane carries
//     CPL candidates, so the warp-uniform work (records, flags, loop control, region checks)
//     is paid once per CPL candidates;
//   * the stream is a run of fixed 48-byte steps (a head + two out-edge records; an op with
//     more out-edges continues in CONT steps), so the walk is one straight-line loop; it is
//     TMA-staged (cp.async.bulk + mbarrier ring) by a producer warp and shared by all consumer
//     warps of the CTA;
//   * ready-time state by producer distance: distance 1 -> a register (`fwd`), 2..kNearDelta ->
//     the warp's shared-memory ring (slot = pos & 15), farther -> a global cold slot written
//     with fire-and-forget STG / RED.MAX and staged back by cp.async kPrefetchDist positions
//     before the consumer runs;
//   * search candidates differ from their base only inside their group's 64-position region
//     (DESIGN.md §4), so outside it a lane's device is the base code embedded in the record.
#include <algorithm>
#include <type_traits>

#include "device_common.cuh"
#include "feasibility.cuh"
#include "internal.h"

namespace pesto {
namespace {

using namespace dev;

__device__ __forceinline__ uint32_t add_sat(uint32_t a, uint32_t b) {
    return min(a + b, kSat32);                 // a <= kSat32, b < kMaxDur32: never wraps
}
// The walk's time type T: uint32 saturating at kSat32 (the fast path) or uint64 exact (the
// "wide" instance, for search bases whose makespan is >= kSat32: same records, same kernel,
// 8-byte state; exact because every time is < 2^40, the ingest guard).
__device__ __forceinline__ uint64_t add_sat(uint64_t a, uint64_t b) { return a + b; }
template <class T> __device__ __forceinline__ T lds_t(uint32_t addr);
template <> __device__ __forceinline__ uint32_t lds_t<uint32_t>(uint32_t addr) { return lds_u32(addr); }
template <> __device__ __forceinline__ uint64_t lds_t<uint64_t>(uint32_t addr) { return lds_u64(addr); }
__device__ __forceinline__ void sts_t(uint32_t addr, uint32_t v) { sts_u32(addr, v); }
__device__ __forceinline__ void sts_t(uint32_t addr, uint64_t v) { sts_u64(addr, v); }
// bytes of one 32-lane column of T; record slot offsets are written for 4-byte columns
template <class T> constexpr uint32_t kColB = 32u * sizeof(T);
// slot layout of the ring, the staging ring and the cold slots: a slot holds 32 lanes x CPL
// values; with two candidates per lane in 32-bit time the lane's pair sits side by side
// (interleaved: lane base lane x 8, candidate c at +4c) so the fast walk moves the pair with one
// 8-byte access; otherwise one 32-lane column per candidate (lane base lane x sizeof(T),
// candidate c at +c x kColB).  A slot's byte size is CPL x kColB either way, so the records'
// slot offsets are the same.
constexpr bool kInterleave2 = true;
template <int CPL, class T> constexpr bool kIL = kInterleave2 && CPL == 2 && sizeof(T) == 4;
template <int CPL, class T> constexpr uint32_t kCandB = kIL<CPL, T> ? (uint32_t)sizeof(T) : kColB<T>;
template <int CPL, class T> constexpr uint32_t kLaneMul = kIL<CPL, T> ? (uint32_t)CPL : 1u;
template <class T> constexpr uint32_t kSc = sizeof(T) / 4u;

// consumer warps per CTA: 256 candidates either way.  (Measured: 2-warp CTAs for CPL = 1, to
// spread inception's 2,048 warps evenly over the SMs, fit only 6 CTAs per SM by registers and
// shared memory, so the launch needed two waves: 5.84 -> 10.14 ms.)
#ifndef PESTO_E32_W1
#define PESTO_E32_W1 8
#endif
#ifndef PESTO_E32_W2
#define PESTO_E32_W2 4
#endif
__host__ __device__ constexpr int warps_for(int cpl) { return cpl == 1 ? PESTO_E32_W1 : PESTO_E32_W2; }

// TMA ring depth and the occupancy target (resident CTAs per SM the register allocation aims
// for), per candidates-per-lane
#ifndef PESTO_E32_STAGES
#define PESTO_E32_STAGES 2
#endif
#ifndef PESTO_E32_MINB1
#define PESTO_E32_MINB1 2
#endif
#ifndef PESTO_E32_MINB2
#define PESTO_E32_MINB2 4
#endif

constexpr int kStages32 = PESTO_E32_STAGES;
#ifndef PESTO_UNI_SWITCH
#define PESTO_UNI_SWITCH 2
#endif
// CPL = 2 reads the next step's head one step ahead (1) or its own head at the step's top (0)
#ifndef PESTO_HEAD_AHEAD2
#define PESTO_HEAD_AHEAD2 1
#endif
constexpr bool kHeadAhead = PESTO_HEAD_AHEAD2 != 0;
// search walk, D = 2, two candidates per lane, uint32 time: uniform steps run in the PTX fast
// segment (fast_walk_ptx.inc), special positions in the C++ step below
#ifndef PESTO_FAST_WALK
#define PESTO_FAST_WALK 1
#endif
#ifndef PESTO_FAST_D4
#define PESTO_FAST_D4 1
#endif
#ifndef PESTO_FAST_ROWS
#define PESTO_FAST_ROWS 1
#endif
constexpr bool kUniSwitch = PESTO_UNI_SWITCH != 0;
// the no-producer instance (np: the consumer that releases a stage last issues its next load)
// targets five CTAs per SM: 128 threads, no warp slot or registers spent on a mostly sleeping
// producer
#ifndef PESTO_E32_MINB_NP
#define PESTO_E32_MINB_NP 5
#endif
__host__ __device__ constexpr int min_blocks_for(int cpl, bool np = false) {
    return np ? PESTO_E32_MINB_NP : (cpl == 1 ? PESTO_E32_MINB1 : PESTO_E32_MINB2);
}
// tile loads: a producer warp per CTA (0), or issued by the consumer warp that releases a stage
// last (1: no warp slot and no registers spent on a warp that mostly sleeps)
#ifndef PESTO_E32_NOPROD
#define PESTO_E32_NOPROD 0
#endif
constexpr bool kProducerWarp = PESTO_E32_NOPROD == 0;
__host__ __device__ constexpr int threads_for(int cpl, bool np = false) {
    return (warps_for(cpl) + (kProducerWarp && !np ? 1 : 0)) * 32;
}

// per-candidate device / link free times
template <int CPL, class T>
struct RegState32 {          // D <= 2
    T d0[CPL], d1[CPL], l01[CPL], l10[CPL];
    __device__ __forceinline__ void init() {
#pragma unroll
        for (int c = 0; c < CPL; c++) d0[c] = d1[c] = l01[c] = l10[c] = 0u;
    }
    __device__ __forceinline__ T dev(int c, int x) const { return x ? d1[c] : d0[c]; }
    __device__ __forceinline__ void set_dev(int c, int x, T v) {
        if (x) d1[c] = v; else d0[c] = v;
    }
    __device__ __forceinline__ T link(int c, int x, int) const { return x ? l10[c] : l01[c]; }
    __device__ __forceinline__ void set_link_if(int c, int x, int, bool cond, T v) {
        l10[c] = (cond && x) ? v : l10[c];
        l01[c] = (cond && !x) ? v : l01[c];
    }
    __device__ __forceinline__ T makespan(int c) const { return max(d0[c], d1[c]); }
    // warp-uniform device codes (search positions outside the group's region): branches on a
    // uniform value instead of per-lane selects
    __device__ __forceinline__ void begin_u(int xu, uint32_t p, const T (&r)[CPL], T (&cc)[CPL]) {
        if (xu) {
#pragma unroll
            for (int c = 0; c < CPL; c++) { cc[c] = add_sat(max(r[c], d1[c]), (T)p); d1[c] = cc[c]; }
        } else {
#pragma unroll
            for (int c = 0; c < CPL; c++) { cc[c] = add_sat(max(r[c], d0[c]), (T)p); d0[c] = cc[c]; }
        }
    }
    __device__ __forceinline__ void link_u(int xu, int, uint32_t t, const T (&cc)[CPL], T (&a)[CPL]) {
        if (xu) {
#pragma unroll
            for (int c = 0; c < CPL; c++) { a[c] = add_sat(max(cc[c], l10[c]), (T)t); l10[c] = a[c]; }
        } else {
#pragma unroll
            for (int c = 0; c < CPL; c++) { a[c] = add_sat(max(cc[c], l01[c]), (T)t); l01[c] = a[c]; }
        }
    }
};

// link columns of device x: x * DS + y; DS = 4 for D <= 4 (a fixed stride the D <= 4 fast walk
// addresses at compile time), D for D <= 8
__host__ __device__ constexpr int link_stride32(int pl, int D) { return pl == 2 ? 4 : D; }

template <int CPL, class T>
struct SmemState32 {         // D <= 8: per column (device, then link x * DS + y) one slot of
    uint32_t d, l;           // 32 lanes x CPL (lane pair interleaved like the rings)
    int D, DS;
    __device__ __forceinline__ uint32_t at(uint32_t base, int col, int c) const {
        return base + (uint32_t)(col * CPL) * kColB<T> + (uint32_t)c * kCandB<CPL, T>;
    }
    __device__ __forceinline__ void init() {
        for (int x = 0; x < D; x++)
            for (int c = 0; c < CPL; c++) sts_t(at(d, x, c), (T)0);
        for (int x = 0; x < D * DS; x++)
            for (int c = 0; c < CPL; c++) sts_t(at(l, x, c), (T)0);
    }
    __device__ __forceinline__ T dev(int c, int x) const { return lds_t<T>(at(d, x, c)); }
    __device__ __forceinline__ void set_dev(int c, int x, T v) { sts_t(at(d, x, c), v); }
    __device__ __forceinline__ T link(int c, int x, int y) const {
        return lds_t<T>(at(l, x * DS + y, c));
    }
    __device__ __forceinline__ void set_link_if(int c, int x, int y, bool cond, T v) {
        if (cond) sts_t(at(l, x * DS + y, c), v);
    }
    __device__ __forceinline__ T makespan(int c) const {
        T m = 0;
        for (int x = 0; x < D; x++) m = max(m, lds_t<T>(at(d, x, c)));
        return m;
    }
    __device__ __forceinline__ void begin_u(int xu, uint32_t p, const T (&r)[CPL], T (&cc)[CPL]) {
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            const uint32_t a = at(d, xu, c);
            cc[c] = add_sat(max(r[c], lds_t<T>(a)), (T)p);
            sts_t(a, cc[c]);
        }
    }
    __device__ __forceinline__ void link_u(int xu, int yu, uint32_t t, const T (&cc)[CPL], T (&a)[CPL]) {
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            const uint32_t ad = at(l, xu * DS + yu, c);
            a[c] = add_sat(max(cc[c], lds_t<T>(ad)), (T)t);
            sts_t(ad, a[c]);
        }
    }
};

// A lane move packed into two registers (the walk reads it only inside the 64-position region,
// so the 13 words of a LaneMove need not stay live; for CPL = 2 that is 22 registers fewer).
// Positions are offsets from the region start (0..63):
//   w0: flip offsets 4 x 6 bits | nflip << 24 | kind << 27
//   w1: flip devices 4 x 3 bits | window offset << 12 | window length << 18 | window device << 25
struct PackedMove {
    uint32_t w0, w1;
};
__device__ __forceinline__ PackedMove pack_move(const LaneMove &mv, int32_t rc) {
    PackedMove p;
    p.w0 = ((uint32_t)mv.nflip << 24) | ((uint32_t)mv.kind << 27);
    p.w1 = 0u;
#pragma unroll
    for (int f = 0; f < 4; f++) {
        if (f < mv.nflip) {
            p.w0 |= (uint32_t)(mv.fpos[f] - rc) << (6 * f);
            p.w1 |= (uint32_t)mv.fdev[f] << (3 * f);
        }
    }
    if (mv.kind == kMoveWindow)
        p.w1 |= ((uint32_t)(mv.ws - rc) << 12) | ((uint32_t)mv.wl << 18) | ((uint32_t)mv.wd << 25);
    return p;
}
// S9 coarse move (merged vertex k -> device d): w1 = k | d << 8 (w0 holds only the kind)
__device__ __forceinline__ PackedMove pack_coarse(const LaneMove &mv) {
    PackedMove p;
    p.w0 = (uint32_t)kMoveCoarse << 27;
    p.w1 = (uint32_t)mv.ws | ((uint32_t)mv.wd << 8);
    return p;
}
__device__ __forceinline__ int coarse_apply_kept(const LaneMove &mv, int cq, int xb, unsigned aq) {
    return apply_coarse(mv.ws, mv.wd, cq, xb, aq);
}
__device__ __forceinline__ int coarse_apply_kept(const PackedMove &mv, int cq, int xb, unsigned aq) {
    return apply_coarse((int32_t)(mv.w1 & 255u), (int32_t)(mv.w1 >> 8), cq, xb, aq);
}
__device__ __forceinline__ int coarse_k(const LaneMove &mv) { return mv.ws; }
__device__ __forceinline__ int coarse_k(const PackedMove &mv) { return (int)(mv.w1 & 255u); }
__device__ __forceinline__ void keep_coarse(LaneMove &dst, const LaneMove &mv) { dst = mv; }
__device__ __forceinline__ void keep_coarse(PackedMove &dst, const LaneMove &mv) { dst = pack_coarse(mv); }

// = apply_lane (moves.cuh) for offset o = q - rc of a position inside the region
__device__ __forceinline__ int apply_packed(const PackedMove &p, uint32_t o, int xb, unsigned aq) {
    int x = xb;
    const uint32_t kind = p.w0 >> 27;
    if (kind == kMoveWindow) {
        const uint32_t ws = (p.w1 >> 12) & 63u, wl = (p.w1 >> 18) & 127u, wd = (p.w1 >> 25) & 7u;
        if (o - ws < wl && ((aq >> wd) & 1u)) x = (int)wd;
    } else if (kind == kMoveFlip) {
        const uint32_t nf = (p.w0 >> 24) & 7u;
#pragma unroll
        for (uint32_t f = 0; f < 4; f++)
            if (f < nf && o == ((p.w0 >> (6 * f)) & 63u)) x = (int)((p.w1 >> (3 * f)) & 7u);
    }
    return x;
}

// the move as the walk keeps it: unpacked with one candidate per lane (registers are not the
// limit there and the unpacked form applies with fewer instructions), packed with two
__device__ __forceinline__ int apply_kept(const LaneMove &mv, int32_t q, int32_t, int xb, unsigned aq) {
    return apply_lane(mv, q, xb, aq);
}
__device__ __forceinline__ int apply_kept(const PackedMove &mv, int32_t q, int32_t rc, int xb,
                                          unsigned aq) {
    return apply_packed(mv, (uint32_t)(q - rc), xb, aq);
}
__device__ __forceinline__ void keep_move(LaneMove &dst, const LaneMove &mv, int32_t) { dst = mv; }
__device__ __forceinline__ void keep_move(PackedMove &dst, const LaneMove &mv, int32_t rc) {
    dst = pack_move(mv, rc);
}

// devices of the lane's CPL candidates at position q; xb = the base code of the record naming q
template <int MODE, int PL, int CPL>
struct Place32 {
    const uint32_t *pl;          // MODE 0: words of the warp's first 32-row group
    int64_t pl_stride;           // MODE 0: words between consecutive 32-row groups
    const uint8_t *allowed_pos;  // MODE 1: masks by position (window moves)
    int32_t rc, rlen;            // MODE 1: the group's region [rc, rc + rlen)
    int all_allowed, lane, dmax;
    typename std::conditional<CPL == 1, LaneMove, PackedMove>::type mv[CPL];
    const uint8_t *cpos;         // MODE 4: merged vertex by position
    int cbits;                   // MODE 4: bits per merged vertex in the candidate index
    uint32_t jc[CPL];            // MODE 4: the lane's candidate indices
    // MODE 5 (search with S9 coarse groups), coarse group: the region is the whole order, marked by a negative rlen (the
    // unsigned range test still admits every position), so no flag register stays live
    __device__ __forceinline__ bool coarse() const { return rlen < 0; }
    // cfn(q): merged vertex of the op at position q (MODE 5 coarse groups only).  Returns true
    // when every lane keeps the base code xb (search: outside the region; a coarse group: no
    // lane moves the op's merged vertex -- a warp vote), false otherwise or when unknown.
    template <class CFn>
    __device__ __forceinline__ bool at(int32_t q, int xb, int (&x)[CPL], const CFn &cfn) const {
        if (MODE == 0) {
#pragma unroll
            for (int c = 0; c < CPL; c++) x[c] = planes_dev_at<PL>(pl + c * pl_stride, q, lane, dmax);
            return false;
        }
        if (MODE == 4) {                                       // digit of the merged vertex
            const int sh = cbits * (int)__ldg(cpos + q);
#pragma unroll
            for (int c = 0; c < CPL; c++) x[c] = (int)((jc[c] >> sh) & (uint32_t)dmax);
            return false;
        }
#pragma unroll
        for (int c = 0; c < CPL; c++) x[c] = xb;
        if ((uint32_t)(q - rc) < (uint32_t)rlen) {             // warp-uniform branch
            if (MODE == 5 && coarse()) {                       // S9: one merged vertex per lane
                const int cq = cfn(q);
                bool hit = false;
#pragma unroll
                for (int c = 0; c < CPL; c++) hit = hit || coarse_k(mv[c]) == cq;
                if (!__any_sync(0xffffffffu, hit)) return true;   // no lane moves this vertex
                const unsigned aq = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q);
#pragma unroll
                for (int c = 0; c < CPL; c++) x[c] = coarse_apply_kept(mv[c], cq, xb, aq);
                return false;
            }
            const unsigned aq = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q);
#pragma unroll
            for (int c = 0; c < CPL; c++) x[c] = apply_kept(mv[c], q, rc, xb, aq);
            return false;
        }
        return true;
    }
};

// explicit rows: one 32-row group's bit-sliced plane words at a position (K5 layout)
template <int PL>
struct PlaneWords {
    uint32_t w[PL];
};
template <int PL>
__device__ __forceinline__ PlaneWords<PL> ldg_planes(const uint32_t *pl, int32_t q) {
    PlaneWords<PL> r;
    if constexpr (PL == 1) {
        r.w[0] = __ldg(pl + q);
    } else if constexpr (PL == 2) {
        const uint2 t = __ldg(reinterpret_cast<const uint2 *>(pl) + q);
        r.w[0] = t.x;
        r.w[1] = t.y;
    } else {
        const uint4 t = __ldg(reinterpret_cast<const uint4 *>(pl) + q);
        r.w[0] = t.x;
        r.w[1] = t.y;
        r.w[2] = t.z;
        r.w[3] = t.w;
    }
    return r;
}
// codes >= D belong to rows K5 flagged infeasible: clamped so the lane stays in its columns
template <int PL>
__device__ __forceinline__ int plane_dev(const PlaneWords<PL> &p, int lane, int dmax) {
    int x = 0;
#pragma unroll
    for (int k = 0; k < PL; k++) x |= (int)((p.w[k] >> lane) & 1u) << k;
    return PL == 1 ? x : min(x, dmax);
}

struct Ctx32 {
    uint32_t smem;               // shared address of the CTA's dynamic shared memory (records)
    uint32_t ring;               // shared address of ring[0][0][lane]; slot s, cand c: + (s*CPL+c)*128
    uint8_t *cold;               // global byte address of cold[0][0][lane]; same layout
    uint64_t cls1;               // bit a*D+b: directed link a -> b is in link class 1 (t = t1)
    int D;
};

template <int CPL, class T>
__device__ __forceinline__ void push_tail(const Ctx32 &cx, const uint32_t tgt, const T (&a)[CPL],
                                          T (&fwd)[CPL]);

// one out-edge record, for the lane's CPL candidates (FCFS link of L144 / L188-198)
template <int PL, int CPL, class T, class StateT>
__device__ __forceinline__ void push32(const Ctx32 &cx, const uint4 rec, const int (&x)[CPL],
                                       const int (&y)[CPL], const T (&cc)[CPL],
                                       StateT &st, T (&fwd)[CPL]) {
    const uint32_t tgt = rec.z;
    T a[CPL];
#pragma unroll
    for (int c = 0; c < CPL; c++) {
        const bool cross = y[c] != x[c];                     // cross: FCFS link x -> y
        uint32_t t;
        if constexpr (PL == 1) t = x[c] ? rec.w : rec.x;     // D = 2: t by direction
        else t = ((cx.cls1 >> (x[c] * cx.D + y[c])) & 1u) ? rec.w : rec.x;
        // branch-free: the transfer's arrival when crossing, C_v (L144) when not
        const T ac = add_sat(max(cc[c], st.link(c, x[c], y[c])), (T)t);
        a[c] = cross ? ac : cc[c];
        st.set_link_if(c, x[c], y[c], cross, ac);
    }
    push_tail<CPL, T>(cx, tgt, a, fwd);
}

// deliver the arrivals a[] of one edge: register (next position), near ring or cold slot
template <int CPL, class T>
__device__ __forceinline__ void push_tail(const Ctx32 &cx, const uint32_t tgt, const T (&a)[CPL],
                                          T (&fwd)[CPL]) {
    if (tgt & kT32Next) {                                    // consumer is the next position
#pragma unroll
        for (int c = 0; c < CPL; c++) fwd[c] = max(fwd[c], a[c]);
        return;
    }
    const uint32_t bytes = (tgt & kT32SlotMask) * CPL * kSc<T>;
    if (tgt & kT32Near) {
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            const uint32_t slot = cx.ring + bytes + c * kCandB<CPL, T>;
            T v = a[c];
            if (!(tgt & kT32First)) v = max(v, lds_t<T>(slot));
            sts_t(slot, v);
        }
    } else {
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            T *slot = reinterpret_cast<T *>(cx.cold + bytes + c * kCandB<CPL, T>);
            if (tgt & kT32First) *slot = a[c];                   // first far push: plain store
            else if constexpr (sizeof(T) == 4) atomicMax(slot, a[c]);   // RED.MAX, no reply
            else atomicMax(reinterpret_cast<unsigned long long *>(slot), (unsigned long long)a[c]);
        }
    }
}

// one out-edge whose producer and consumer devices are warp-uniform (xu, yu): a same-device
// edge skips the link entirely (uniform branch), a crossing edge updates the one link xu -> yu
template <int PL, int CPL, class T, class StateT>
__device__ __forceinline__ void push32_u(const Ctx32 &cx, const uint4 rec, int xu, int yu,
                                         const T (&cc)[CPL], StateT &st, T (&fwd)[CPL]) {
    T a[CPL];
    if (xu != yu) {
        uint32_t t;
        if constexpr (PL == 1) t = xu ? rec.w : rec.x;
        else t = ((cx.cls1 >> (xu * cx.D + yu)) & 1u) ? rec.w : rec.x;
        st.link_u(xu, yu, t, cc, a);
    } else {
#pragma unroll
        for (int c = 0; c < CPL; c++) a[c] = cc[c];
    }
    push_tail<CPL, T>(cx, rec.z, a, fwd);
}

// D = 2 (register state), both devices warp-uniform: the edge's whole path -- link or not, which
// direction, register / ring / cold slot, first push or max -- is selected by one jump-table
// dispatch on idx = target class << 2 | xu << 1 | (xu != yu), taken from one record word
// (succ_pos: successor code at bit 24, class code at bits 27-29) and xm = xu * 3
template <uint32_t TC, int XU, int CROSS, int CPL, class T>
__device__ __forceinline__ void uni_edge(const Ctx32 &cx, const uint4 rec, const T (&cc)[CPL],
                                         RegState32<CPL, T> &st, T (&fwd)[CPL]) {
    T a[CPL];
#pragma unroll
    for (int c = 0; c < CPL; c++) {
        if constexpr (CROSS) {                               // FCFS link xu -> 1 - xu
            T &l = XU ? st.l10[c] : st.l01[c];
            a[c] = add_sat(max(cc[c], l), (T)(XU ? rec.w : rec.x));
            l = a[c];
        } else {
            a[c] = cc[c];                                    // same device: C_v (L144)
        }
    }
    constexpr uint32_t F = TC << 29;
    if constexpr ((F & kT32Next) != 0) {
#pragma unroll
        for (int c = 0; c < CPL; c++) fwd[c] = max(fwd[c], a[c]);
    } else {
        const uint32_t bytes = (rec.z & kT32SlotMask) * CPL * kSc<T>;
        if constexpr ((F & kT32Near) != 0) {
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const uint32_t slot = cx.ring + bytes + c * kCandB<CPL, T>;
                T v = a[c];
                if constexpr ((F & kT32First) == 0) v = max(v, lds_t<T>(slot));
                sts_t(slot, v);
            }
        } else {
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                T *slot = reinterpret_cast<T *>(cx.cold + bytes + c * kCandB<CPL, T>);
                if constexpr ((F & kT32First) != 0) *slot = a[c];
                else if constexpr (sizeof(T) == 4) atomicMax(slot, a[c]);
                else atomicMax(reinterpret_cast<unsigned long long *>(slot), (unsigned long long)a[c]);
            }
        }
    }
}
#include "uni_push_ptx.inc"
#include "fast_walk_ptx.inc"
// the fast segment reads the next step's head one step ahead (1) or at the step's top (0)
#ifndef PESTO_FAST_RA
#define PESTO_FAST_RA 0
#endif
#ifndef PESTO_FAST_DT
#define PESTO_FAST_DT 0
#endif
#if PESTO_FAST_DT
#define PESTO_FW1 PESTO_FAST_WALK_PTX1_DT
#define PESTO_FW2 PESTO_FAST_WALK_PTX2_DT
#define PESTO_FW1W PESTO_FAST_WALK_PTX1W_DT
#elif PESTO_FAST_RA
#define PESTO_FW1 PESTO_FAST_WALK_PTX1_RA
#define PESTO_FW2 PESTO_FAST_WALK_PTX2_RA
#define PESTO_FW1W PESTO_FAST_WALK_PTX1W_RA
#else
#define PESTO_FW1 PESTO_FAST_WALK_PTX1
#define PESTO_FW2 PESTO_FAST_WALK_PTX2
#define PESTO_FW1W PESTO_FAST_WALK_PTX1W
#endif
// the far-arrival copy of the two-candidates-per-lane fast walk as one 16-byte cp.async.cg per
// even lane (gen_fast_walk.py segment ce)
#ifndef PESTO_FAST_CE
#define PESTO_FAST_CE 1
#endif
#ifndef PESTO_FAST_KS
#define PESTO_FAST_KS 0
#endif
#if PESTO_FAST_CE && PESTO_FAST_KS
#undef PESTO_FW2
#define PESTO_FW2 PESTO_FAST_WALK_PTX2_CEKS
#elif PESTO_FAST_CE
#undef PESTO_FW2
#define PESTO_FW2 PESTO_FAST_WALK_PTX2_CE
#endif

// the uniform steps from sp on (until lim or the first step of the special position nspec),
// state in registers; returns with sp at the first step it did not take
__device__ __forceinline__ void fast_segment(uint32_t &sp, int32_t &v,
                                             RegState32<2, uint32_t> &st,
                                             uint32_t (&fwd)[2], uint32_t (&nfar)[2],
                                             uint32_t (&nnear)[2], uint32_t lim,
                                             uint32_t ring, uint32_t stage, const uint8_t *cold) {
    asm volatile(PESTO_FW2
                 : "+r"(sp), "+r"(v), "+r"(st.d0[0]), "+r"(st.d0[1]), "+r"(st.d1[0]), "+r"(st.d1[1]),
                   "+r"(st.l01[0]), "+r"(st.l01[1]), "+r"(st.l10[0]), "+r"(st.l10[1]),
                   "+r"(fwd[0]), "+r"(fwd[1]), "+r"(nfar[0]), "+r"(nfar[1]), "+r"(nnear[0]),
                   "+r"(nnear[1])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold)
                 : "memory");
}
__device__ __forceinline__ void fast_segment(uint32_t &sp, int32_t &v,
                                             RegState32<1, uint32_t> &st,
                                             uint32_t (&fwd)[1], uint32_t (&nfar)[1],
                                             uint32_t (&nnear)[1], uint32_t lim,
                                             uint32_t ring, uint32_t stage, const uint8_t *cold) {
    asm volatile(PESTO_FW1
                 : "+r"(sp), "+r"(v), "+r"(st.d0[0]), "+r"(st.d1[0]), "+r"(st.l01[0]),
                   "+r"(st.l10[0]), "+r"(fwd[0]), "+r"(nfar[0]), "+r"(nnear[0])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold)
                 : "memory");
}
__device__ __forceinline__ void fast_segment(uint32_t &sp, int32_t &v,
                                             RegState32<1, uint64_t> &st,
                                             uint64_t (&fwd)[1], uint64_t (&nfar)[1],
                                             uint64_t (&nnear)[1], uint32_t lim,
                                             uint32_t ring, uint32_t stage, const uint8_t *cold) {
    asm volatile(PESTO_FW1W
                 : "+r"(sp), "+r"(v), "+l"(st.d0[0]), "+l"(st.d1[0]), "+l"(st.l01[0]),
                   "+l"(st.l10[0]), "+l"(fwd[0]), "+l"(nfar[0]), "+l"(nnear[0])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold)
                 : "memory");
}
// explicit rows (mode 0), D = 2: per-lane devices from K5's words, control by class tables
#ifndef PESTO_ROWS_PF
#define PESTO_ROWS_PF 0
#endif
// PESTO_ROWS_V2 selects the explicit-row segment (scripts/gen_fast_walk.py segment_rows):
// 0 round-2 first version, 1 lane-mask tests, 3 + register read-ahead, 4 + windowed shuffles,
// 5: 4 for two candidates per lane, 3 for one; 6: the same with the successor-word window
// switch folded into the step's dispatch (segment_rows fold); 7 (default): both switches folded
// (foldx).  Measured (B200, K1 of 1 M random rows, transformer_2dev, CPL 2): 74.5 (0) -> 69.0 (3)
// -> 66.4 (4) -> 65.3 ms (fold); K5 + K1 with the five-CTA instance 65.85 -> 64.99 ms (foldx);
// inception 65,536 rows (CPL 1): 6.30 (0) -> 5.91 (3) / 6.47 ms (4)
#ifndef PESTO_ROWS_V2
#define PESTO_ROWS_V2 7
#endif
#if PESTO_ROWS_V2 == 7
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V3
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V6
#elif PESTO_ROWS_V2 == 6
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V3
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V5
#elif PESTO_ROWS_V2 == 5
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V3
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V4
#elif PESTO_ROWS_V2 >= 4
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V4
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V4
#elif PESTO_ROWS_V2 >= 3
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V3
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V3
#elif PESTO_ROWS_V2 && PESTO_ROWS_PF
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V2PF
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V2PF
#elif PESTO_ROWS_V2
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_V2
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_V2
#elif PESTO_ROWS_PF
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1_PF
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2_PF
#else
#define PESTO_FR1 PESTO_FAST_ROWS_PTX1
#define PESTO_FR2 PESTO_FAST_ROWS_PTX2
#endif
__device__ __forceinline__ void fast_rows(uint32_t &sp, int32_t &v, uint32_t &ys,
                                          RegState32<2, uint32_t> &st, uint32_t (&fwd)[2],
                                          uint32_t (&nfar)[2], uint32_t (&nnear)[2],
                                          uint32_t (&xr)[2], uint32_t lim, uint32_t ring,
                                          uint32_t stage, const uint8_t *cold, uint32_t lane,
                                          const uint32_t *const (&xb)[2],
                                          const uint32_t *const (&yb)[2]) {
    asm volatile(PESTO_FR2
                 : "+r"(sp), "+r"(v), "+r"(ys), "+r"(st.d0[0]), "+r"(st.d0[1]), "+r"(st.d1[0]),
                   "+r"(st.d1[1]), "+r"(st.l01[0]), "+r"(st.l01[1]), "+r"(st.l10[0]),
                   "+r"(st.l10[1]), "+r"(fwd[0]), "+r"(fwd[1]), "+r"(nfar[0]), "+r"(nfar[1]),
                   "+r"(nnear[0]), "+r"(nnear[1]), "+r"(xr[0]), "+r"(xr[1])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold), "r"(lane), "l"(xb[0]), "l"(xb[1]),
                   "l"(yb[0]), "l"(yb[1])
                 : "memory");
}
__device__ __forceinline__ void fast_rows(uint32_t &sp, int32_t &v, uint32_t &ys,
                                          RegState32<1, uint32_t> &st, uint32_t (&fwd)[1],
                                          uint32_t (&nfar)[1], uint32_t (&nnear)[1],
                                          uint32_t (&xr)[1], uint32_t lim, uint32_t ring,
                                          uint32_t stage, const uint8_t *cold, uint32_t lane,
                                          const uint32_t *const (&xb)[1],
                                          const uint32_t *const (&yb)[1]) {
    asm volatile(PESTO_FR1
                 : "+r"(sp), "+r"(v), "+r"(ys), "+r"(st.d0[0]), "+r"(st.d1[0]), "+r"(st.l01[0]),
                   "+r"(st.l10[0]), "+r"(fwd[0]), "+r"(nfar[0]), "+r"(nnear[0]), "+r"(xr[0])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold), "r"(lane), "l"(xb[0]), "l"(yb[0])
                 : "memory");
}
template <int CPL, class T, class ST>
__device__ __forceinline__ void fast_rows(uint32_t &, int32_t &, uint32_t &, ST &, T (&)[CPL],
                                          T (&)[CPL], T (&)[CPL], uint32_t (&)[CPL], uint32_t,
                                          uint32_t, uint32_t, const uint8_t *, uint32_t,
                                          const uint32_t *const (&)[CPL],
                                          const uint32_t *const (&)[CPL]) {}

// D = 3..4: device / link state stays in shared memory (SmemState32), the walk's control is
// the same jump-table loop (fast_walk_ptx.inc PESTO_FAST_WALK_PTX{1,2}_D4)
__device__ __forceinline__ void fast_segment(uint32_t &sp, int32_t &v, SmemState32<2, uint32_t> &st,
                                             uint32_t (&fwd)[2], uint32_t (&nfar)[2],
                                             uint32_t (&nnear)[2], uint32_t lim, uint32_t ring,
                                             uint32_t stage, const uint8_t *cold, uint32_t cls4) {
    asm volatile(PESTO_FAST_WALK_PTX2_D4
                 : "+r"(sp), "+r"(v), "+r"(fwd[0]), "+r"(fwd[1]), "+r"(nfar[0]), "+r"(nfar[1]),
                   "+r"(nnear[0]), "+r"(nnear[1])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold), "r"(st.d), "r"(st.l), "r"(cls4)
                 : "memory");
}
__device__ __forceinline__ void fast_segment(uint32_t &sp, int32_t &v, SmemState32<1, uint32_t> &st,
                                             uint32_t (&fwd)[1], uint32_t (&nfar)[1],
                                             uint32_t (&nnear)[1], uint32_t lim, uint32_t ring,
                                             uint32_t stage, const uint8_t *cold, uint32_t cls4) {
    asm volatile(PESTO_FAST_WALK_PTX1_D4
                 : "+r"(sp), "+r"(v), "+r"(fwd[0]), "+r"(nfar[0]), "+r"(nnear[0])
                 : "r"(lim), "r"(ring), "r"(stage), "l"(cold), "r"(st.d), "r"(st.l), "r"(cls4)
                 : "memory");
}
// D = 2: the link class is the direction (records hold t per direction); cls4 unused
template <class ST, class T, int N>
__device__ __forceinline__ void fast_segment(uint32_t &sp, int32_t &v, ST &st, T (&fwd)[N],
                                             T (&nfar)[N], T (&nnear)[N], uint32_t lim,
                                             uint32_t ring, uint32_t stage, const uint8_t *cold,
                                             uint32_t) {
    fast_segment(sp, v, st, fwd, nfar, nnear, lim, ring, stage, cold);
}
template <int CPL, class T, class ST>
__device__ __forceinline__ void fast_segment(uint32_t &, int32_t &, ST &, T (&)[CPL], T (&)[CPL],
                                             T (&)[CPL], uint32_t, uint32_t, uint32_t,
                                             const uint8_t *) {}
template <int CPL, class T>
__device__ __forceinline__ void push_uni(const Ctx32 &cx, const uint4 rec, uint32_t xm,
                                         const T (&cc)[CPL], RegState32<CPL, T> &st, T (&fwd)[CPL]) {
    if constexpr (PESTO_UNI_SWITCH == 2 && CPL == 2 && sizeof(T) == 4) {
        const uint32_t idx = ((((rec.y >> (kSuccTcShift - 2)) & 0x1Cu) | ((rec.y >> kSuccXShift) & 1u)) ^ xm);
        asm volatile(PESTO_UNI_PUSH_PTX
                     : "+r"(st.l01[0]), "+r"(st.l01[1]), "+r"(st.l10[0]), "+r"(st.l10[1]),
                       "+r"(fwd[0]), "+r"(fwd[1])
                     : "r"(idx), "r"(rec.x), "r"(rec.w), "r"(rec.z), "r"(cc[0]), "r"(cc[1]),
                       "r"(cx.ring), "l"(cx.cold)
                     : "memory");
        return;
    }
    // idx = class << 2 | xu << 1 | (xu != yu): 20 dense entries, one jump table
    const uint32_t idx = ((((rec.y >> (kSuccTcShift - 2)) & 0x1Cu) | ((rec.y >> kSuccXShift) & 1u)) ^ xm);
    switch (idx) {
#define PESTO_UNI_CASES(TC, FL)                                                          \
    case (TC) * 4 + 0: uni_edge<FL, 0, 0, CPL, T>(cx, rec, cc, st, fwd); break;          \
    case (TC) * 4 + 1: uni_edge<FL, 0, 1, CPL, T>(cx, rec, cc, st, fwd); break;          \
    case (TC) * 4 + 2: uni_edge<FL, 1, 0, CPL, T>(cx, rec, cc, st, fwd); break;          \
    case (TC) * 4 + 3: uni_edge<FL, 1, 1, CPL, T>(cx, rec, cc, st, fwd); break;
        PESTO_UNI_CASES(0u, 0u)      // far, later push: RED.MAX
        PESTO_UNI_CASES(1u, 4u)      // far, first push: STG
        PESTO_UNI_CASES(2u, 2u)      // near ring, later push
        PESTO_UNI_CASES(3u, 6u)      // near ring, first push
        PESTO_UNI_CASES(4u, 1u)      // next position: register
#undef PESTO_UNI_CASES
        default: __builtin_unreachable();
    }
}
template <int CPL, class T>
__device__ __forceinline__ void push_uni(const Ctx32 &, const uint4, uint32_t, const T (&)[CPL],
                                         SmemState32<CPL, T> &, T (&)[CPL]) {}

// the (up to two) out-edges of one step, records already in registers; yfn(k, rec, y) gives
// the successor's devices of edge k
template <int PL, int CPL, class T, class YFn, class StateT>
__device__ __forceinline__ void edges32(const Ctx32 &cx, uint32_t flags, const uint4 e0,
                                        const uint4 e1, const int (&x)[CPL],
                                        const T (&cc)[CPL], const YFn &yfn,
                                        StateT &st, T (&fwd)[CPL]) {
    const uint32_t ne = (flags >> kStEdgeShift) & 3u;
    if (ne >= 1) {
        int y[CPL];
        yfn(0, e0, y);
        push32<PL, CPL, T>(cx, e0, x, y, cc, st, fwd);
    }
    if (ne >= 2) {
        int y[CPL];
        yfn(1, e1, y);
        push32<PL, CPL, T>(cx, e1, x, y, cc, st, fwd);
    }
}

// start the op at position v (head h, devices x) whose arrivals are r[c]: S_v, C_v (L142-146)
template <int CPL, class T, class StateT>
__device__ __forceinline__ void begin32(const uint4 h, StateT &st, const T (&r)[CPL],
                                        const int (&x)[CPL], T (&cc)[CPL]) {
#pragma unroll
    for (int c = 0; c < CPL; c++) {
        cc[c] = add_sat(max(r[c], st.dev(c, x[c])), (T)h.x);  // C_v = S_v + p_v
        st.set_dev(c, x[c], cc[c]);
    }
}

template <int MODE, int PL, int CPL, class T, bool NP = false>
__global__ void __launch_bounds__(threads_for(CPL, NP), min_blocks_for(CPL, NP))
eval32_kernel(const EvalParams P) {
    constexpr bool kProd = kProducerWarp && !NP;       // a producer warp loads the tiles
    constexpr bool kSearch = MODE == 1 || MODE == 5;   // 5: search with S9 coarse groups
    // uniform steps through the PTX fast segment (D = 2, CPL 2, 32-bit time, search)
    // explicit rows, D = 2, 32-bit time: every step through the PTX rows segment
    constexpr bool kFastRows = PESTO_FAST_ROWS != 0 && MODE == 0 && PL == 1 && sizeof(T) == 4;
    constexpr bool kFast = PESTO_FAST_WALK != 0 && MODE == 1 &&
                           ((PL == 1 && (sizeof(T) == 4 || CPL == 1)) ||
                            (PL == 2 && sizeof(T) == 4 && PESTO_FAST_D4 != 0));
    constexpr int NW = warps_for(CPL);          // consumer warps per CTA (256 candidates)
    constexpr int CW = 32 * CPL;                // candidates per warp
    extern __shared__ __align__(128) uint8_t smem[];
    // stage stride: the largest tile + one step of padding, so the walk may read the records of
    // the step after a tile's last one without leaving its own stage
    const int sb = P.stage_bytes32 + kStepBytes;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + (size_t)kStages32 * sb);
    uint64_t *empty = full + kStages32;
    uint8_t *cur = align16(reinterpret_cast<uint8_t *>(empty + kStages32));
    T *ring_all = reinterpret_cast<T *>(cur);
    cur = align16(cur + (size_t)NW * kRing * CW * sizeof(T));
    T *stage_all = reinterpret_cast<T *>(cur);                        // far-arrival staging
    cur = align16(cur + (size_t)NW * kRing * CW * sizeof(T));
    T *dstate = reinterpret_cast<T *>(cur);
    // MODE 5, CPL 1: the merged vertex of every position of the current task's base in shared
    // memory (S9 coarse groups look one up per op and per successor; from global memory those
    // lookups missed L1 behind the cold-slot traffic and made a coarse warp ~1.7x slower).  Not
    // for CPL 2: n more bytes per CTA cost a resident CTA per SM there (measured slower).
    constexpr bool kCposSmem = MODE == 5 && CPL == 1;
    const uint32_t cpos_s = su32_reg(align16(cur + (PL != 1 ? (size_t)NW * (P.D + P.D * link_stride32(PL, P.D)) * CW * sizeof(T) : 0)));

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    auto runs_here = [&](int bl) {           // search: this kernel owns bases below saturation
        // (the wide instance, gate 2, owns the bases at or above saturation)
        return !kSearch || P.gate == 0 ||
               (P.gate == 1 ? P.base_mk[bl] < (int64_t)kSat32 : P.base_mk[bl] >= (int64_t)kSat32);
    };
    // the CTA's tile sequence: (task, tile) over its tasks, tiles in order (no-producer mode)
    auto first_task = [&](int64_t task) {
        for (; task < P.n_tasks; task += gridDim.x)
            if (runs_here(kSearch ? (int)(task / P.tasks_per_base) : 0)) break;
        return task;
    };
    auto advance = [&](int64_t &task, int &t) {
        if (task >= P.n_tasks) return;
        const int bl = kSearch ? (int)(task / P.tasks_per_base) : 0;
        if (++t < P.bases[bl].n_tiles32) return;
        t = 0;
        task = first_task(task + gridDim.x);
    };
    auto load_tile = [&](int64_t task, int t, int s) {      // one lane
        if (task >= P.n_tasks) return;
        const BaseLayoutDev *B = &P.bases[kSearch ? (int)(task / P.tasks_per_base) : 0];
        const TileDesc td = B->tiles32[t];
        mbar_expect_tx(&full[s], (uint32_t)td.bytes);
        bulk_g2s(smem + (size_t)s * sb, B->blob32 + td.byte_off, (uint32_t)td.bytes, &full[s]);
    };
    // stage release counters (no-producer mode), in the space of the empty barriers
    const uint32_t rel0 = su32(empty);
    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages32; s++) {
            mbar_init(&full[s], 1);
            if constexpr (kProd) mbar_init(&empty[s], NW);
            else empty[s] = 0;
        }
        mbar_fence_init();
        if constexpr (!kProd) {
            int64_t task = first_task(blockIdx.x);
            int t = 0;
            for (int s = 0; s < kStages32; s++) {
                load_tile(task, t, s);
                advance(task, t);
            }
        }
    }
    __syncthreads();

    if (kProd && warp == NW) {
        if (lane == 0) {
            uint32_t it = 0;
            for (int64_t task = blockIdx.x; task < P.n_tasks; task += gridDim.x) {
                const int bl = kSearch ? (int)(task / P.tasks_per_base) : 0;
                if (!runs_here(bl)) continue;
                const BaseLayoutDev *B = &P.bases[bl];
                const int nt = B->n_tiles32;
                for (int t = 0; t < nt; t++, it++) {
                    const int s = it % kStages32;
                    if (it >= (uint32_t)kStages32) {
                        mbar_wait(&empty[s], ((it / kStages32) - 1) & 1);
                        // the consumers' generic-proxy reads of the stage (released through the
                        // empty barrier) before the async-proxy (TMA) write that reuses it
                        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    }
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
    cx.ring = su32_reg(ring_all + (size_t)warp * kRing * CW + lane * kLaneMul<CPL, T>);
    cx.cold = reinterpret_cast<uint8_t *>(reinterpret_cast<T *>(P.state32) +
                                          ((size_t)(blockIdx.x * NW + warp) * P.max_W32) * CW +
                                          lane * kLaneMul<CPL, T>);
    cx.D = P.D;
    cx.cls1 = 0;
    for (int i = 0; i < P.D * P.D; i++)
        if (P.link_class[i] == 1) cx.cls1 |= 1ull << i;
    // D <= 4 fast walk: link x -> y in class 1 at bit x * 4 + y
    uint32_t cls4 = 0;
    if (PL == 2)
        for (int i = 0; i < P.D * P.D; i++)
            if (P.link_class[i] == 1) cls4 |= 1u << ((i / P.D) * 4 + i % P.D);
    // the staging ring sits a compile-time distance after the near ring (both NW x kRing x CW
    // times, 16-byte multiples): derived from cx.ring so that the pair of loads per position
    // shares one address register (the second load takes an immediate offset)
    static_assert((NW * kRing * CW * sizeof(T)) % 16 == 0, "ring and staging are adjacent");
    const uint32_t stage = cx.ring + (uint32_t)(NW * kRing * CW * sizeof(T));
    (void)stage_all;

    using StateT = typename std::conditional<PL == 1, RegState32<CPL, T>, SmemState32<CPL, T>>::type;
    StateT st;
    if constexpr (PL != 1) {
        st.D = P.D;
        st.DS = link_stride32(PL, P.D);
        st.d = su32_reg(dstate + (size_t)warp * (P.D + P.D * st.DS) * CW + lane * kLaneMul<CPL, T>);
        st.l = st.d + (uint32_t)(P.D * CPL) * kColB<T>;
    }

    // Far arrivals of position q arrive by cp.async into stage[q & 15] (zero when q has no far
    // producer), issued while position q - kPrefetchDist starts (its head names the slot); one
    // commit group per position.  Only positions > kNearDelta have far producers, so the first
    // positions of a task need no prefetch.
    auto issue_far = [&](const uint4 h, int32_t v) {
        const uint32_t dst = stage + (uint32_t)(((v + kPrefetchDist) & (kRing - 1)) * CPL) * kColB<T>;
        const bool have = (int32_t)h.z >= 0;
        const uint8_t *src = cx.cold + (size_t)(have ? h.z : 0) * CW * sizeof(T);
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            if constexpr (sizeof(T) == 4) cp_async4_zfill(dst + c * kCandB<CPL, T>, src + c * kCandB<CPL, T>, have);
            else cp_async8_zfill(dst + c * kCandB<CPL, T>, src + c * kCandB<CPL, T>, have);
        }
        cp_async_commit();
    };
    // The arrivals of position q from far producers (stage) and near producers (ring) are final
    // once the op at q - 1 starts (a distance-1 producer forwards in `fwd`), so they are read one
    // op ahead, off the critical path: nfar/nnear hold them for the next position.
    auto load_next = [&](int32_t q, T (&nfar)[CPL], T (&nnear)[CPL]) {
        const uint32_t o = (uint32_t)((q & (kRing - 1)) * CPL) * kColB<T>;
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            nfar[c] = lds_t<T>(stage + o + c * kCandB<CPL, T>);
            nnear[c] = lds_t<T>(cx.ring + o + c * kCandB<CPL, T>);
        }
    };
    auto arrivals = [&](uint32_t flags, const T (&nfar)[CPL], const T (&nnear)[CPL],
                        const T (&fwd)[CPL], T (&r)[CPL]) {
        const bool near = (flags & kStHasNear) != 0;          // else the ring slot is stale
#pragma unroll
        for (int c = 0; c < CPL; c++) r[c] = max(max(nfar[c], fwd[c]), near ? nnear[c] : (T)0);
    };

    uint32_t it = 0;
    int prev_bl = -1;
    for (int64_t task = blockIdx.x; task < P.n_tasks; task += gridDim.x) {
        const int bl = kSearch ? (int)(task / P.tasks_per_base) : 0;
        if (!runs_here(bl)) continue;
        if constexpr (kCposSmem) {
            if (bl != prev_bl) {         // the consumer warps copy the base's merged vertices
                named_bar_sync(1, NW * 32);                   // previous walks are done
                const uint8_t *src = P.coarse_pos + (size_t)bl * P.n;
                for (int q = threadIdx.x; q < P.n; q += NW * 32) sts_u8(cpos_s + q, __ldg(src + q));
                named_bar_sync(1, NW * 32);
                prev_bl = bl;
            }
        }
        const int64_t local = kSearch ? task % P.tasks_per_base : task;
        const BaseLayoutDev *B = &P.bases[bl];
        const int nt = B->n_tiles32;
        // a task = TS consecutive candidate ids starting at a multiple of TS; a warp = CW of them
        constexpr int64_t TS = (int64_t)NW * CW;
        const int64_t j0 = (kSearch ? P.j_begin - P.j_begin % TS : 0) + local * TS + warp * CW;
        const int64_t gw = j0 >> 5;                                 // first 32-row group

        Place32<MODE, PL, CPL> place;
        place.lane = lane;
        place.dmax = P.D - 1;
        place.all_allowed = P.all_allowed;
        place.rc = 0;
        place.rlen = 0;
        bool active;
        bool valid[CPL];
        // fast walk: the group's next special position (spec_pos list of its region)
        int32_t nspec = INT32_MAX;
        uint32_t spi = 0;
        bool fast_ok = false, gen_op = false;
        int32_t ks = -1;
        uint32_t off_ks = 0;         // search: byte offset of the op at ks in the step stream
        if (MODE == 4) {
            // exhaustive coarse placements (row f2): candidate j is its own placement code
            active = j0 < P.n_cand;
            place.cpos = P.coarse_pos;
            place.cbits = P.coarse_bits;
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const int64_t j = j0 + c * 32 + lane;
                place.jc[c] = (uint32_t)j;
                bool ok = j < P.n_cand;
                if (!P.all_allowed)
                    for (int k = 0; k < P.n_coarse; k++)
                        ok = ok && ((P.coarse_allowed[k] >> ((j >> (P.coarse_bits * k)) & (P.D - 1))) & 1u);
                valid[c] = ok;
            }
        } else if (MODE == 0) {
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
            place.allowed_pos = B->allowed_pos;
            const bool coarse = MODE == 5 && coarse_group(P.seed, cb, grp, P.coarse_pct, P.n_coarse);
            if (coarse) {
                // S9: every lane moves one merged vertex, anywhere in the order; no order move
                place.rc = 0;
                place.rlen = (int32_t)(0x80000000u | (uint32_t)P.n);
#pragma unroll
                for (int c = 0; c < CPL; c++) {
                    const int64_t j = j0 + c * 32 + lane;
                    valid[c] = active && j >= P.j_begin && j < P.j_end;
                    keep_coarse(place.mv[c], decode_coarse_lane(P.seed, cb, j, P.n_coarse, P.D));
                }
            }
            const Region rg = decode_region(P.seed, cb, grp, P.n);
            if (!coarse) {
                place.rc = rg.c;
                place.rlen = rg.len;
            }
            if constexpr (kFast) {
                fast_ok = B->spec_pos != nullptr;
                if (fast_ok) {
                    spi = __ldg(B->spec_off + rg.c / kRegion);
                    nspec = __ldg(B->spec_pos + spi);
                }
            }
            const uint8_t *blocked = B->swap_blocked;
            const int32_t *ord = B->order;
            const uint32_t *bits = B->bits;
            const uint8_t *aop = P.allowed_op;
            const int words = P.words;
            ks = active && !coarse
                     ? decode_swap(P.seed, cb, grp, P.n, P.mix[3], rg,
                                   [&](int32_t k) { return __ldg(blocked + k) != 0; },
                                   [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); })
                     : -1;
            if (ks >= 0) off_ks = __ldg(B->op_off32 + ks);
            if (!coarse) {
#pragma unroll
                for (int c = 0; c < CPL; c++) {
                    const int64_t j = j0 + c * 32 + lane;
                    const bool in_range = active && j >= P.j_begin && j < P.j_end;
                    LaneMove mv = in_range
                        ? decode_lane(P.seed, cb, j, ks >= 0 && (j & (kGroup - 1)) == 0, P.D, P.mix, rg,
                                      [&](int32_t q) { return __ldg(ord + q); },
                                      [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); },
                                      [&](int32_t op) { return (unsigned)__ldg(aop + op); })
                        : no_move();
                    valid[c] = in_range && mv.kind != kMoveInvalid;
                    if (mv.kind == kMoveInvalid) mv = no_move();
                    if (valid[c] && (P.feas.has_cap || P.feas.has_coloc))   // row f3
                        valid[c] = move_feasible<PL>(mv, rg, P.D, bits, words, ord,
                                                     B->allowed_pos, P.all_allowed, P.feas,
                                                     P.feas.fbase + (size_t)bl * 8);
                    keep_move(place.mv[c], mv, rg.c);
                }
            }
        }
        st.init();
        // positions 0 .. kPrefetchDist - 1 are never prefetched (they have no far producer)
#pragma unroll
        for (int q = 0; q < kRing; q++)
#pragma unroll
            for (int c = 0; c < CPL; c++) sts_t(stage + (q * CPL) * kColB<T> + c * kCandB<CPL, T>, (T)0);

        // the op being walked (its devices and C_v), the arrivals it forwards to v + 1, and the
        // far / near arrivals of v + 1 read ahead
        int x[CPL];
        T cc[CPL], fwd[CPL], nfar[CPL], nnear[CPL];
#pragma unroll
        for (int c = 0; c < CPL; c++) { x[c] = 0; cc[c] = 0u; fwd[c] = 0u; nfar[c] = 0u; nnear[c] = 0u; }
        // devices by direct lookup (search: base code + region moves; rows: plane words)
        // S9 merged vertices by position of this base (shared copy of P.coarse_pos[bl][.])
        // (a non-volatile shared load: the compiler may issue it early)
        auto cpos_at = [&](int32_t q) {
            if constexpr (kCposSmem) return (int)lds_u8_nv(cpos_s + (uint32_t)q);
            else return (int)__ldg(P.coarse_pos + (size_t)bl * P.n + q);
        };
        auto place_y = [&](int, const uint4 rec, int (&y)[CPL]) {
            place.at((int32_t)(rec.y & kSuccPosMask), (int)((rec.y >> kSuccXShift) & 7u), y, cpos_at);
        };
        // explicit rows: the plane words of the next op are loaded one step ahead (consecutive
        // positions share cache lines); the successors' words come from K5's edge-slot stream
        // (DESIGN.md §3.4), read sequentially 32 words per lane-coalesced load, one window
        // ahead, and handed out by shuffles -- no random lookups into the 139 MB of plane words
        // the op's own word likewise: position windows of 32 / PL positions
        const int64_t xwords = (int64_t)P.n * PL;
        uint32_t xw[CPL], xn[CPL];
        int32_t xwb = 0;
        // explicit rows: the warp's 32-row groups that exist (a warp's second group past the last
        // row reads its first group's words instead: never out of bounds, results unused --
        // compute-sanitizer memcheck / initcheck, round 2)
        const int64_t cgrp = (MODE == 0 && CPL > 1 && ((gw + 1) << 5) >= P.n_cand) ? 0 : 1;
        auto x_load = [&](int32_t q, uint32_t (&w)[CPL]) {
            const int64_t wi = (int64_t)q * PL + lane;
#pragma unroll
            for (int c = 0; c < CPL; c++)
                w[c] = wi < xwords ? __ldg(place.pl + c * cgrp * place.pl_stride + wi) : 0u;
        };
        constexpr int SW = 32 / PL;                    // edge slots per 32-word window
        const int64_t ywords = P.n_slots * PL;         // words of one group's slot stream
        uint32_t yw[CPL], yn[CPL];                     // this window / the next, per candidate
        int32_t ywb = 0;                               // first slot of this window
        int32_t slot0 = 0;                             // first slot of the current step
        auto y_load = [&](int32_t slot, uint32_t (&w)[CPL]) {
            const int64_t wi = (int64_t)slot * PL + lane;
#pragma unroll
            for (int c = 0; c < CPL; c++)
                w[c] = wi < ywords ? __ldg(P.yplanes + (size_t)(gw + c * cgrp) * ywords + wi) : 0u;
        };
        // the codes of a position's / an edge slot's word, by shuffle from a window
        auto shfl_dev = [&](const uint32_t (&win)[CPL], int base, int (&out)[CPL]) {
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                PlaneWords<PL> w;
#pragma unroll
                for (int p = 0; p < PL; p++) w.w[p] = __shfl_sync(0xffffffffu, win[c], base + p);
                out[c] = plane_dev<PL>(w, lane, place.dmax);
            }
        };
        // both successor slots of a step are shuffled at the step's top (off the edges' chains;
        // slot0 is even and a window holds an even number of slots, so both are in window yw)
        int ys[2][CPL];
        auto pw_y = [&](int k, const uint4, int (&y)[CPL]) {
#pragma unroll
            for (int c = 0; c < CPL; c++) y[c] = ys[k][c];
        };
        // the next op's codes, shuffled one op ahead
        int xnext[CPL];
        if constexpr (MODE == 0 && !kFastRows) {
            if (active) {
                x_load(0, xw);
                x_load(SW, xn);
                y_load(0, yw);
                y_load(SW, yn);
            }
            shfl_dev(xw, 0, xnext);
        }
        // rows segment state: the op's device per candidate, the walk's edge-slot counter, and
        // the words of the warp's 32-row groups (a missing second group reads the first's)
        uint32_t xr[CPL], yslot = 0;
        const uint32_t *xbp[CPL], *ybp[CPL];
#pragma unroll
        for (int c = 0; c < CPL; c++) {
            xr[c] = 0;
            if constexpr (kFastRows) {
                xbp[c] = place.pl + c * cgrp * place.pl_stride;
                ybp[c] = P.yplanes + (size_t)(gw + c * cgrp) * ywords;
            } else {
                xbp[c] = ybp[c] = nullptr;
            }
        }
        int32_t v = -1;
        int xu = -1;                 // search: the walked op's device if warp-uniform, else -1
        int32_t skip = 0;            // steps of the next tile already walked (swap pair)
        for (int t = 0; t < nt; t++, it++) {
            const int s = it % kStages32;
            mbar_wait(&full[s], (it / kStages32) & 1);
            if (active) {
                const uint32_t tile = (uint32_t)s * sb;
                const int32_t nsteps = (int32_t)lds_u32(cx.smem + tile);
                uint32_t sp = cx.smem + tile + kTileHeader + (uint32_t)skip * kStepBytes;
                // the tile's steps end at spe: the walk compares step addresses (no step counter)
                const uint32_t spe = cx.smem + tile + kTileHeader + (uint32_t)nsteps * kStepBytes;
                skip = 0;
                uint4 h = lds_v4(sp), e0 = lds_v4(sp + 16), e1 = lds_v4(sp + 32);
                // the search group's swapped pair (ks, ks+1): when the op at ks starts in this
                // tile the walk's step limit is its first step, where the pair is walked in
                // swapped order -- no per-op position test in the loop
                uint32_t lim = spe;
                if (kSearch && ks >= 0) {
                    const uint32_t rel = off_ks - lds_u32(cx.smem + tile + 4);   // tile's blob offset
                    if (rel < lds_u32(cx.smem + tile + 8)) lim = min(spe, cx.smem + tile + rel);
                }
                for (;;) {
                    while (sp < lim) {
                        if constexpr (kFastRows) {
                            fast_rows(sp, v, yslot, st, fwd, nfar, nnear, xr, lim, cx.ring, stage,
                                      cx.cold, (uint32_t)lane, xbp, ybp);
                            continue;
                        }
                        if constexpr (kFast) {
                            // uniform steps: the PTX segment; a special position's first step
                            // (and its continuation steps) take the C++ step below
                            if (fast_ok) {
                                const bool is_cont = (lds_u32(sp + 12) & kStCont) != 0;
                                if (is_cont ? !gen_op : (v + 1 != nspec)) {
                                    // stop at the first step of the next special position when
                                    // it starts in this tile (found by address, like the pair)
                                    uint32_t flim = lim;
                                    if (nspec < P.n) {
                                        const uint32_t rel = __ldg(P.bases[bl].op_off32 + nspec) -
                                                             lds_u32(cx.smem + tile + 4);
                                        if (rel < lds_u32(cx.smem + tile + 8))
                                            flim = min(flim, cx.smem + tile + rel);
                                    }
                                    fast_segment(sp, v, st, fwd, nfar, nnear, flim, cx.ring,
                                                 stage, cx.cold, cls4);
                                    gen_op = false;
                                    continue;
                                }
                                gen_op = true;
                            }
                        }
                        // the next step's head (past the tile's end: padding, never used); this
                        // step's edge records (their first use is after the head's work)
                        // (CPL = 1 reads its own head here: the read-ahead copy costs more than the
                        // LDS latency it hides there -- measured 5.86 vs 5.77 ms on inception)
                        uint4 hn;
                        if constexpr (CPL == 1 || !kHeadAhead || kFast) h = lds_v4(sp);
                        else hn = lds_v4(sp + 48);
                        e0 = lds_v4(sp + 16);
                        e1 = lds_v4(sp + 32);
                        if constexpr (MODE == 0) {
                            if (slot0 >= ywb + SW) {               // next window; prefetch the one after
#pragma unroll
                                for (int c = 0; c < CPL; c++) yw[c] = yn[c];
                                ywb += SW;
                                y_load(ywb + SW, yn);
                            }
                            shfl_dev(yw, (slot0 - ywb) * PL, ys[0]);
                            shfl_dev(yw, (slot0 + 1 - ywb) * PL, ys[1]);
                        }
                        if (!(h.w & kStCont)) {
                            v++;
                            if constexpr (kFast) {
                                if (fast_ok)
                                    while (nspec <= v) nspec = __ldg(P.bases[bl].spec_pos + ++spi);
                            }
                            issue_far(h, v);
                            cp_async_wait<kPrefetchDist - 1>();      // v+1 has landed
                            T r[CPL];
                            arrivals(h.w, nfar, nnear, fwd, r);
                            load_next(v + 1, nfar, nnear);
#pragma unroll
                            for (int c = 0; c < CPL; c++) fwd[c] = 0u;
                            if constexpr (MODE == 0) {
#pragma unroll
                                for (int c = 0; c < CPL; c++) x[c] = xnext[c];
                                if (v + 1 >= xwb + SW) {           // next window; prefetch the one after
#pragma unroll
                                    for (int c = 0; c < CPL; c++) xw[c] = xn[c];
                                    xwb += SW;
                                    x_load(xwb + SW, xn);
                                }
                                shfl_dev(xw, (v + 1 - xwb) * PL, xnext);
                            } else {
                                // outside the group's region every lane has the base device
                                // (CPL = 2 only: with one candidate per lane the launch is
                                // latency-bound and the branch-free selects schedule better)
                                if constexpr (MODE == 5) {
                                    // coarse groups: uniform wherever no lane moves the op's merged vertex
                                    const bool uni = place.at(v, (int)(h.w & kStXMask), x, cpos_at);
                                    xu = (CPL == 2 && uni) ? (int)(h.w & kStXMask) : -1;
                                } else {
                                    xu = (kSearch && CPL == 2 &&
                                          (uint32_t)(v - place.rc) >= (uint32_t)place.rlen)
                                             ? (int)(h.w & kStXMask) : -1;
                                    place.at(v, (int)(h.w & kStXMask), x, cpos_at);
                                }
                            }
                            if (MODE != 0 && xu >= 0) st.begin_u(xu, h.x, r, cc);
                            else begin32<CPL, T>(h, st, r, x, cc);
                        }
                        if constexpr (MODE == 0) {
                            edges32<PL, CPL, T>(cx, h.w, e0, e1, x, cc, pw_y, st, fwd);
                            slot0 += 2;
                        } else {
                            const uint32_t ne = (h.w >> kStEdgeShift) & 3u;
                            if (MODE == 5 && xu >= 0) {
                                // successors: the uniform push wherever no lane moves them
                                if (ne >= 1) {
                                    int y[CPL];
                                    const int yb = (int)((e0.y >> kSuccXShift) & 7u);
                                    if (place.at((int32_t)(e0.y & kSuccPosMask), yb, y, cpos_at))
                                        push32_u<PL, CPL, T>(cx, e0, xu, yb, cc, st, fwd);
                                    else push32<PL, CPL, T>(cx, e0, x, y, cc, st, fwd);
                                }
                                if (ne >= 2) {
                                    int y[CPL];
                                    const int yb = (int)((e1.y >> kSuccXShift) & 7u);
                                    if (place.at((int32_t)(e1.y & kSuccPosMask), yb, y, cpos_at))
                                        push32_u<PL, CPL, T>(cx, e1, xu, yb, cc, st, fwd);
                                    else push32<PL, CPL, T>(cx, e1, x, y, cc, st, fwd);
                                }
                            } else if (xu >= 0) {
                                const uint32_t xm = (uint32_t)xu * 3u;
                                if (ne >= 1) {
                                    const int32_t q0 = (int32_t)(e0.y & kSuccPosMask);
                                    if ((uint32_t)(q0 - place.rc) >= (uint32_t)place.rlen) {
                                        if constexpr (PL == 1 && kUniSwitch) push_uni<CPL, T>(cx, e0, xm, cc, st, fwd);
                                        else push32_u<PL, CPL, T>(cx, e0, xu, (int)((e0.y >> kSuccXShift) & 7u), cc, st, fwd);
                                    } else { int y[CPL]; place_y(0, e0, y); push32<PL, CPL, T>(cx, e0, x, y, cc, st, fwd); }
                                }
                                if (ne >= 2) {
                                    const int32_t q1 = (int32_t)(e1.y & kSuccPosMask);
                                    if ((uint32_t)(q1 - place.rc) >= (uint32_t)place.rlen) {
                                        if constexpr (PL == 1 && kUniSwitch) push_uni<CPL, T>(cx, e1, xm, cc, st, fwd);
                                        else push32_u<PL, CPL, T>(cx, e1, xu, (int)((e1.y >> kSuccXShift) & 7u), cc, st, fwd);
                                    } else { int y[CPL]; place_y(1, e1, y); push32<PL, CPL, T>(cx, e1, x, y, cc, st, fwd); }
                                }
                            } else {
                                edges32<PL, CPL, T>(cx, h.w, e0, e1, x, cc, place_y, st, fwd);
                            }
                        }
                        sp += kStepBytes;
                        if constexpr (CPL != 1 && kHeadAhead && !kFast) h = hn;
                    }
                    if (!kSearch || sp >= spe) break;
                    // sp = the first step of the op at ks (a walk stops there only for ks)
                    lim = spe;
                    if constexpr (CPL == 1 || !kHeadAhead || kFast) h = lds_v4(sp);
                    e0 = lds_v4(sp + 16);
                    e1 = lds_v4(sp + 32);
                    v++;
                    {
                        // swapped pair: the op at ks+1 runs first, then the op at ks.  They
                        // share no producer, no consumer and no edge (DESIGN.md §4 S3), so
                        // every slot's first push is unchanged; only device and link queues
                        // see the new order.
                        const int32_t nk = (int32_t)(h.w >> kStStepsShift);
                        const bool straddle = sp + (uint32_t)nk * kStepBytes >= spe;
                        uint32_t sp1;
                        if (straddle) {
                            const int s2 = (it + 1) % kStages32;
                            mbar_wait(&full[s2], ((it + 1) / kStages32) & 1);
                            sp1 = cx.smem + (uint32_t)s2 * sb + kTileHeader;
                        } else {
                            sp1 = sp + (uint32_t)nk * kStepBytes;
                        }
                        const uint4 h1 = lds_v4(sp1);
                        const int32_t n1 = (int32_t)(h1.w >> kStStepsShift);
                        issue_far(h, v);
                        issue_far(h1, v + 1);
                        cp_async_wait<kPrefetchDist - 1>();  // v+1 and v+2 have landed
                        T r0[CPL], r1[CPL], f1[CPL], g1[CPL], zero[CPL];
#pragma unroll
                        for (int c = 0; c < CPL; c++) zero[c] = 0u;
                        arrivals(h.w, nfar, nnear, fwd, r0);
                        load_next(v + 1, f1, g1);
                        arrivals(h1.w, f1, g1, zero, r1);   // ks+1's distance-1 producer is ks: none
#pragma unroll
                        for (int c = 0; c < CPL; c++) fwd[c] = 0u;
                        place.at(v + 1, (int)(h1.w & kStXMask), x, cpos_at);
                        begin32<CPL, T>(h1, st, r1, x, cc);
                        for (int32_t q = 0; q < n1; q++) {
                            const uint32_t a = sp1 + q * kStepBytes;
                            edges32<PL, CPL, T>(cx, lds_u32(a + 12), lds_v4(a + 16), lds_v4(a + 32), x,
                                             cc, place_y, st, fwd);
                        }
                        place.at(v, (int)(h.w & kStXMask), x, cpos_at);
                        begin32<CPL, T>(h, st, r0, x, cc);
                        edges32<PL, CPL, T>(cx, h.w, e0, e1, x, cc, place_y, st, fwd);
                        for (int32_t q = 1; q < nk; q++) {
                            const uint32_t a = sp + q * kStepBytes;
                            edges32<PL, CPL, T>(cx, lds_u32(a + 12), lds_v4(a + 16), lds_v4(a + 32), x,
                                             cc, place_y, st, fwd);
                        }
                        v++;
                        xu = -1;
                        load_next(v + 1, nfar, nnear);
                        if constexpr (kFast) {
                            if (fast_ok)
                                while (nspec <= v) nspec = __ldg(P.bases[bl].spec_pos + ++spi);
                            gen_op = false;       // the walk continues at a first step
                        }
                        if (straddle) {
                            skip = n1;
                            break;
                        }
                        sp = sp1 + (uint32_t)n1 * kStepBytes;
                        h = lds_v4(sp);
                        e0 = lds_v4(sp + 16);
                        e1 = lds_v4(sp + 32);
                        continue;
                    }
                }
            }
            __syncwarp();
            if constexpr (kProd) {
                if (lane == 0) mbar_arrive(&empty[s]);
            } else if (lane == 0) {
                // the warp that releases stage s last loads the CTA's tile kStages32 iterations
                // ahead into it (acq_rel: every warp's reads of the stage precede the load)
                uint32_t old;
                asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], 1;"
                             : "=r"(old) : "r"(rel0 + 8u * (uint32_t)s) : "memory");
                if ((old + 1u) % (uint32_t)NW == 0u) {
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    int64_t nt_task = task;
                    int nt_t = t;
                    for (int k = 0; k < kStages32; k++) advance(nt_task, nt_t);
                    load_tile(nt_task, nt_t, s);
                }
            }
        }
        cp_async_wait<0>();

        if (!active) continue;
        if (MODE == 0) {
#pragma unroll
            for (int c = 0; c < CPL; c++) {
                const int64_t j = j0 + c * 32 + lane;
                if (j >= P.n_cand) continue;
                const uint64_t mk = (uint64_t)st.makespan(c);
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
                // parity output (pesto_search_candidate_keys): this walk's own key of every
                // candidate, after the walk -- a saturated one carries kSat32 as its makespan
                if (P.keys_dbg && j >= P.j_begin && j < P.j_end) P.keys_dbg[j - P.j_begin] = kc;
            }
            key = warp_min_u64(key);
            if (lane == 0 && key != ~0ull)
                atomicMin(reinterpret_cast<unsigned long long *>(P.keys + bl), (unsigned long long)key);
        }
    }
}

// the no-producer five-CTA instance: search, D = 2, two candidates per lane, 32-bit time
template <int MODE, int PL, int CPL>
constexpr bool kHasNp = (MODE == 1 || MODE == 0) && PL == 1 && CPL == 2;
template <int MODE, int PL, int CPL>
bool use_np(const EvalParams &p) { return kHasNp<MODE, PL, CPL> && p.np32 && !p.wide32; }

template <int MODE, int PL, int CPL>
auto kernel_for(const EvalParams &p) {
    // the wide (exact 64-bit) instance serves search bases at or above saturation only
    if constexpr (MODE == 1 || MODE == 5) {
        if (p.wide32) return eval32_kernel<MODE, PL, CPL, uint64_t>;
    }
    if constexpr (kHasNp<MODE, PL, CPL>) {
        if (use_np<MODE, PL, CPL>(p)) return eval32_kernel<MODE, PL, CPL, uint32_t, true>;
    }
    return eval32_kernel<MODE, PL, CPL, uint32_t>;
}

template <int MODE, int PL, int CPL>
cudaError_t launch_one32(const EvalParams &p, int grid, cudaStream_t st) {
    const int smem = eval32_smem_bytes(p, MODE);
    auto kern = kernel_for<MODE, PL, CPL>(p);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    // explicit rows: the largest shared-memory carveout, so that the next batch's K5 (double-
    // buffered host batches on another stream) can be resident beside this launch's CTAs; with
    // the default carveout it waited for them (e2e 9.19 -> 9.68 M candidates/s)
    if (MODE == 0 &&
        (e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout,
                                  cudaSharedmemCarveoutMaxShared)) != cudaSuccess)
        return e;
    kern<<<grid, threads_for(CPL, use_np<MODE, PL, CPL>(p)), smem, st>>>(p);
    return cudaGetLastError();
}

template <int MODE, int PL, int CPL>
int occupancy_one32(const EvalParams &p) {
    const int smem = eval32_smem_bytes(p, MODE);
    auto kern = kernel_for<MODE, PL, CPL>(p);
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
        return 0;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, threads_for(CPL, use_np<MODE, PL, CPL>(p)), smem) !=
        cudaSuccess)
        return 0;
    return n;
}

int planes_of32(int D) { return D <= 2 ? 1 : (D <= 4 ? 2 : 4); }

}  // namespace

int eval32_task_size(int cpl) { return warps_for(cpl) * 32 * cpl; }

int eval32_smem_bytes(const EvalParams &p, int search_mode) {
    const int cpl = p.cpl32 == 1 ? 1 : 2;
    const int nw = warps_for(cpl);
    const int pl = planes_of32(p.D);
    const size_t tb = ((search_mode == 1 || search_mode == 5) && p.wide32) ? 8 : 4;   // bytes per time value
    size_t b = (size_t)kStages32 * (p.stage_bytes32 + kStepBytes) + 2 * kStages32 * 8;
    b = (b + 15) & ~size_t(15);
    b += (size_t)nw * kRing * 32 * cpl * tb;       // near ring
    b = (b + 15) & ~size_t(15);
    b += (size_t)nw * kRing * 32 * cpl * tb;       // far-arrival staging
    b = (b + 15) & ~size_t(15);
    if (pl != 1) b += (size_t)nw * (p.D + p.D * link_stride32(pl, p.D)) * 32 * cpl * tb;
    b = (b + 15) & ~size_t(15);
    if (search_mode == 5 && cpl == 1) b += (size_t)p.n;   // merged vertex per position (S9)
    return (int)b + 128;
}

// eval32 runs graphs with at most two link classes (layout.cpp emits no stream otherwise);
// candidates per lane: p.cpl32 (1 or 2, chosen by the host: choose_cpl32)
#define PESTO_DISPATCH32_C(FN, C, ...)                                                     \
    do {                                                                                   \
        const int pl = planes_of32(p.D);                                                   \
        if (search_mode == 4) {                                                            \
            if (pl == 1) return FN<4, 1, C>(__VA_ARGS__);                                  \
            if (pl == 2) return FN<4, 2, C>(__VA_ARGS__);                                  \
            return FN<4, 4, C>(__VA_ARGS__);                                               \
        } else if (search_mode && p.coarse_pct > 0) {   /* S9 coarse groups: own instance */ \
            if (pl == 1) return FN<5, 1, C>(__VA_ARGS__);                                  \
            if (pl == 2) return FN<5, 2, C>(__VA_ARGS__);                                  \
            return FN<5, 4, C>(__VA_ARGS__);                                               \
        } else if (search_mode) {                                                          \
            if (pl == 1) return FN<1, 1, C>(__VA_ARGS__);                                  \
            if (pl == 2) return FN<1, 2, C>(__VA_ARGS__);                                  \
            return FN<1, 4, C>(__VA_ARGS__);                                               \
        } else {                                                                           \
            if (pl == 1) return FN<0, 1, C>(__VA_ARGS__);                                  \
            if (pl == 2) return FN<0, 2, C>(__VA_ARGS__);                                  \
            return FN<0, 4, C>(__VA_ARGS__);                                               \
        }                                                                                  \
    } while (0)
#define PESTO_DISPATCH32(FN, ...)                                                          \
    do {                                                                                   \
        if (p.cpl32 == 1) PESTO_DISPATCH32_C(FN, 1, __VA_ARGS__);                          \
        PESTO_DISPATCH32_C(FN, 2, __VA_ARGS__);                                            \
    } while (0)

cudaError_t launch_eval32(const EvalParams &p, int search_mode, int grid, cudaStream_t st) {
    note_launch();
    PESTO_DISPATCH32(launch_one32, p, grid, st);
}

int eval32_max_ctas_per_sm(const EvalParams &p, int search_mode) {
    PESTO_DISPATCH32(occupancy_one32, p);
}

}  // namespace pesto
