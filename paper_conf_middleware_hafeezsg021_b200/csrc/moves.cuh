// moves.cuh -- counter-based neighbour moves of the local search (rows a2/a7).
//
// The search is the north star's method (not a PAPER.md method); it explores the two decision
// variables of the Pesto problem: the placement x_i (L175, L208 for >2 devices) and the
// schedule order (L171, L279).  Everything is integer and derived from the counter
// (seed, step, base, candidate j, draw k), so any rank can regenerate any candidate.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define PESTO_HD __host__ __device__ __forceinline__
#else
#define PESTO_HD inline
#endif

namespace pesto {

PESTO_HD uint64_t mix64(uint64_t z) {            // SplitMix64 finaliser
    z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27; z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}

// draw_k(j) = mix64(seed ^ mix64(((step*P + b) * 2^24 + j) * 16 + k))
PESTO_HD uint64_t draw(uint64_t seed, uint64_t ctr_base, int64_t j, int k) {
    return mix64(seed ^ mix64((ctr_base + (uint64_t)j) * 16ull + (uint64_t)k));
}
PESTO_HD uint64_t ctr_base_of(uint64_t step, int P, int b) {
    return (step * (uint64_t)P + (uint64_t)b) << 24;
}

PESTO_HD int popc32(unsigned v) {
#ifdef __CUDA_ARCH__
    return __popc(v);
#else
    return __builtin_popcount(v);
#endif
}

enum MoveKind : int { kMoveNone = 0, kMoveFlip = 1, kMoveWindow = 2, kMoveInvalid = 3, kMoveCoarse = 4 };

struct LaneMove {
    int kind;
    int nflip;
    int32_t fpos[4];     // flipped positions (in the base order), applied in sequence
    int32_t fdev[4];
    int32_t ws, wl, wd;  // window: positions [ws, ws + wl) move to wd where allowed
                         // coarse (S9): merged vertex ws moves to wd where allowed (wl = 0)
};

constexpr int kRegion = 64;     // positions a group of candidates may change (DESIGN §4 S2)
constexpr int kGroupShift = 7;  // a group = 128 consecutive candidate ids
constexpr int kGroup = 1 << kGroupShift;

// The group's region [c, c + len) of the base order and its pass over the regions.
struct Region {
    int32_t c, len, pass;
};
// S2 (v6): the regions tile the order (R = ceil(n/64)); group g takes region (g + o) mod R with
// the per-(step, base) rotation o = draw(0, 13) mod R, in pass g / R
PESTO_HD Region decode_region(uint64_t seed, uint64_t cb, int64_t group, int n) {
    const int64_t R = ((int64_t)n + kRegion - 1) / kRegion;
    const int64_t rot = (int64_t)(draw(seed, cb, 0, 13) % (uint64_t)R);
    Region r;
    r.c = (int32_t)(kRegion * ((group + rot) % R));
    r.len = n - r.c < kRegion ? n - r.c : kRegion;
    r.pass = (int32_t)(group / R);
    return r;
}

// Group order move (S3): adjacent swap of positions (k, k+1) of the base order, or -1.
// blocked(k) says whether (k, k+1) may not be swapped for structural reasons (an edge joins
// them, they share a producer or a consumer, or either has more than kSwapMaxOut out-edges);
// base_dev(q) is the base device at q -- a pair on different devices is blocked too (v6).
constexpr int kSwapMaxOut = 64;
template <class Blocked, class BaseDev>
PESTO_HD int32_t decode_swap(uint64_t seed, uint64_t cb, int64_t group, int n, int swap_pct,
                             Region rg, Blocked blocked, BaseDev base_dev) {
    if (group == 0 || swap_pct <= 0 || n < 2) return -1;
    int64_t j0 = group * kGroup;
    if ((int)(draw(seed, cb, j0, 15) % 100u) >= swap_pct) return -1;
    int32_t k = rg.c + (int32_t)(draw(seed, cb, j0, 14) % (uint64_t)rg.len);
    if (k > n - 2) k = n - 2;
    return (blocked(k) || base_dev(k) != base_dev(k + 1)) ? -1 : k;
}

// the a-th (0-based, ascending) device of mask msk, or -1
PESTO_HD int nth_device(unsigned msk, int a, int D) {
    for (int d = 0; d < D; d++) {
        if ((msk >> d) & 1u) {
            if (a == 0) return d;
            a--;
        }
    }
    return -1;
}

// Lane placement move of candidate j inside region rg (S4, v6).  Callbacks:
//   op_at(pos) -> op id at a position of the base order;  base_dev(pos) -> base device there;
//   allowed(op) -> device mask.
template <class OpAt, class BaseDev, class Allowed>
PESTO_HD LaneMove decode_lane(uint64_t seed, uint64_t cb, int64_t j, bool pure_swap, int D,
                              const int32_t mix[4], Region rg, OpAt op_at, BaseDev base_dev,
                              Allowed allowed) {
    LaneMove mv;
    mv.kind = kMoveNone;
    mv.nflip = 0;
    mv.ws = 0; mv.wl = 0; mv.wd = 0;
    for (int q = 0; q < 4; q++) { mv.fpos[q] = -1; mv.fdev[q] = 0; }
    if (j == 0 || pure_swap) return mv;
    const int wsum = mix[0] + mix[1] + mix[2];
    if (wsum <= 0) return mv;
    const int lane = (int)(j & (kGroup - 1));
    const int b1 = (kGroup * mix[0]) / wsum, b2 = (kGroup * (mix[0] + mix[1])) / wsum;
    const unsigned dmask = (1u << D) - 1u;
    // A_q: allowed devices of the op at q without its base device
    auto alts = [&](int32_t q) { return allowed(op_at(q)) & dmask & ~(1u << base_dev(q)); };
    if (lane < b1) {                                   // FLIP1: enumerated single-op moves
        const int64_t t = (int64_t)rg.pass * b1 + lane;
        if (t < (int64_t)rg.len * (D - 1)) {
            const int32_t q = rg.c + (int32_t)(t % rg.len);
            const int a = (int)(t / rg.len);
            const unsigned am = alts(q);
            if (a >= popc32(am)) { mv.kind = kMoveInvalid; return mv; }
            mv.kind = kMoveFlip;
            mv.nflip = 1;
            mv.fpos[0] = q;
            mv.fdev[0] = nth_device(am, a, D);
            return mv;
        }
        // the region's single-op moves are used up: a FLIPk lane
    }
    if (lane < b2) {                                   // FLIPk (or a used-up FLIP1 lane)
        int f = 2 + (int)(draw(seed, cb, j, 1) % 3u);
        if (f > rg.len) f = rg.len;
        mv.kind = kMoveFlip;
        mv.nflip = f;
        for (int i = 0; i < f; i++) {
            int r = (int)(draw(seed, cb, j, 2 + 2 * i) % (uint64_t)(rg.len - i));
            // the r-th free offset of the region: the least fixed point of
            // off = r + #{taken offsets <= off} (at most i <= 3 increases)
            int32_t off = r;
            for (int it = 0; it < 4; it++) {
                int32_t cnt = 0;
                for (int e = 0; e < i; e++) cnt += (mv.fpos[e] - rg.c) <= off ? 1 : 0;
                if (r + cnt == off) break;
                off = r + cnt;
            }
            const int32_t q = rg.c + off;
            const unsigned am = alts(q);
            const int na = popc32(am);
            if (na == 0) { mv.kind = kMoveInvalid; return mv; }
            mv.fpos[i] = q;
            mv.fdev[i] = nth_device(am, (int)(draw(seed, cb, j, 3 + 2 * i) % (uint64_t)na), D);
        }
        return mv;
    }
    // WINDOW (v7): enumerated starts s, the visit of s = how many times the enumeration has
    // passed it; the window moves the first L "eligible" ops from s (allow d, not on d in the
    // base; M of them in [s, c + len)), L = 2 + (visit + draw(s, 0)) mod (M - 1): every visit
    // of s changes a different number of ops, so no two WINDOW candidates coincide (v6 drew the
    // length in positions and clipped it at the region's end: 7% duplicates at 1 M per step)
    const int i = lane - b2, nw = kGroup - b2;
    const int64_t w = (int64_t)rg.pass * nw + i;
    const int32_t s = rg.c + (int32_t)(w % rg.len);
    const int64_t visit = w / rg.len;
    const unsigned am = alts(s);
    const int na = popc32(am);
    if (na == 0) { mv.kind = kMoveInvalid; return mv; }
    const int d = nth_device(am, (int)(draw(seed, cb, j, 4) % (uint64_t)na), D);
    auto eligible = [&](int32_t q) {
        return ((allowed(op_at(q)) >> d) & 1u) != 0 && base_dev(q) != d;
    };
    int32_t M = 0;
    for (int32_t q = s; q < rg.c + rg.len; q++) M += eligible(q) ? 1 : 0;
    if (M < 2 || visit >= M - 1) { mv.kind = kMoveInvalid; return mv; }
    int32_t L = 2 + (int32_t)(((uint64_t)visit + draw(seed, cb, s, 0)) % (uint64_t)(M - 1));
    int32_t e = s;
    while (L > 0) L -= eligible(e++) ? 1 : 0;
    mv.kind = kMoveWindow;
    mv.ws = s;
    mv.wl = e - s;
    mv.wd = d;
    return mv;
}

// S9 (row f2): group g != 0 is a coarse group iff draw(128g, 12) mod 100 < pct.
// A coarse group has no region, no order move and no region moves.
PESTO_HD bool coarse_group(uint64_t seed, uint64_t cb, int64_t group, int pct, int n_coarse) {
    return group != 0 && pct > 0 && n_coarse > 0 &&
           (int)(draw(seed, cb, group * kGroup, 12) % 100u) < pct;
}
// candidate j of a coarse group: merged vertex draw(j, 10) mod n_coarse to device draw(j, 11) mod D
PESTO_HD LaneMove decode_coarse_lane(uint64_t seed, uint64_t cb, int64_t j, int n_coarse, int D) {
    LaneMove mv;
    mv.kind = kMoveCoarse;
    mv.nflip = 0;
    for (int q = 0; q < 4; q++) { mv.fpos[q] = -1; mv.fdev[q] = 0; }
    mv.ws = (int32_t)(draw(seed, cb, j, 10) % (uint64_t)n_coarse);
    mv.wl = 0;
    mv.wd = (int32_t)(draw(seed, cb, j, 11) % (uint64_t)D);
    return mv;
}
// device of an op of merged vertex cq (base device xb, mask aq) under a coarse move
PESTO_HD int apply_coarse(int32_t k, int32_t d, int cq, int xb, unsigned aq) {
    return (cq == k && ((aq >> d) & 1u)) ? d : xb;
}

// device of position q under move mv (base device xb, op mask at q for the window check)
PESTO_HD int apply_lane(const LaneMove &mv, int32_t q, int xb, unsigned allowed_q) {
    int x = xb;
    if ((uint32_t)(q - mv.ws) < (uint32_t)mv.wl && ((allowed_q >> mv.wd) & 1u)) x = mv.wd;
#pragma unroll
    for (int f = 0; f < 4; f++)
        if (q == mv.fpos[f]) x = mv.fdev[f];
    return x;
}

}  // namespace pesto
