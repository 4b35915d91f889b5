// nondelay.cu -- row f4(i): makespan under non-delay dispatch (product code).
//
// PAPER.md L90 (§2.1): "for each device, TensorFlow randomly picks an operation from the ready
// queue (those whose predecessors have completed execution)".  Reading R24: the
// pick is by priority pi -- whenever a device is idle it starts, among its ops whose inputs
// have all arrived, the one earliest in pi.  Links stay Pesto's FCFS queues (L144, L188-198)
// or, under PESTO_LINKS_UNLIMITED, congestion-free (L113).  Domain: every p_i >= 1 and every
// transfer >= 1 ns (R24; the host checks it), which makes the schedule below equal to the
// event-driven one.
//
// One warp owns one candidate (the dispatch decisions are a serial chain; the warp spreads each
// op's out-edges, the FCFS prefix sums and the ready-set searches over its lanes).  The
// schedule is generated op by op in non-decreasing start time: each step starts, over all
// devices, the op with the smallest (earliest start, pi position), where a device's earliest
// start is its free time if some op of it is ready by then, else the earliest arrival among its
// eligible ops (all producers started).  Per warp:
//   * shared memory: the candidate's placement (bit planes by op id) and, per device, a
//     three-level bitmap over pi positions of the ops ready by the device's free time
//     ("released"), so the first ready op in pi is three warp-uniform LDS + FFS;
//   * registers: lane d holds device d's free time, lanes hold the D*D link free times;
//   * global scratch (the warp's slot): inputs still missing and the latest arrival per op
//     (atomics, so multi-edges of one producer resolve inside a chunk of lanes), and per device
//     a 32-ary min-heap of the eligible ops whose inputs arrive after the device's free time
//     ("pending"), as keys (time << 23 | position << 3 | device) ordered like the selection.
//     (A first version kept one unsorted list and rescanned it every step: with random
//     placements ~450 entries were pending on inception, and the rescans dominated.)
#include <cstdio>

#include "device_common.cuh"
#include "feasibility.cuh"
#include "internal.h"

namespace pesto {
namespace {

using namespace dev;

constexpr int kNdMaxWarps = 8;
constexpr uint64_t kNone = ~0ull;
constexpr uint32_t kFull = 0xffffffffu;
constexpr uint32_t kPrioMask = (1u << 20) - 1;

__device__ __forceinline__ uint64_t nd_key(int64_t t, uint32_t prio, int d) {
    return ((uint64_t)t << 23) | ((uint64_t)prio << 3) | (uint64_t)d;
}

// three-level bitmap over positions q < 2^20: L0 bit q, L1 bit q>>5, L2 bit q>>10; a level's
// bit is set iff the word below it is non-zero
struct Bitmap {
    uint32_t *w;
    int words, nw1, nw2;
    __device__ __forceinline__ void set(uint32_t q) const {     // any lanes, concurrently
        atomicOr(&w[q >> 5], 1u << (q & 31));
        atomicOr(&w[words + (q >> 10)], 1u << ((q >> 5) & 31));
        atomicOr(&w[words + nw1 + (q >> 15)], 1u << ((q >> 10) & 31));
    }
    __device__ __forceinline__ void clear(uint32_t q) const {   // one lane
        const uint32_t w0 = w[q >> 5] & ~(1u << (q & 31));
        w[q >> 5] = w0;
        if (w0) return;
        uint32_t *p1 = &w[words + (q >> 10)];
        const uint32_t w1 = *p1 & ~(1u << ((q >> 5) & 31));
        *p1 = w1;
        if (w1) return;
        w[words + nw1 + (q >> 15)] &= ~(1u << ((q >> 10) & 31));
    }
    __device__ __forceinline__ bool any() const {
        for (int i = 0; i < nw2; i++)
            if (w[words + nw1 + i]) return true;
        return false;
    }
    __device__ __forceinline__ uint32_t first() const {         // requires any()
        int i = 0;
        while (!w[words + nw1 + i]) i++;
        const int i1 = i * 32 + __ffs(w[words + nw1 + i]) - 1;
        const int i0 = i1 * 32 + __ffs(w[words + i1]) - 1;
        return (uint32_t)(i0 * 32 + __ffs(w[i0]) - 1);
    }
};

template <int PL>
__device__ __forceinline__ int dev_of(const uint32_t *X, int words, int32_t v) {
    return bits_dev_at<PL>(X, words, v);
}

template <int MODE, int PL>
__global__ void __launch_bounds__(kNdMaxWarps * 32, 3) nondelay_kernel(const NdParams P) {
    extern __shared__ __align__(16) uint32_t nsm[];
    uint8_t *lclass = reinterpret_cast<uint8_t *>(nsm);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x < 64) lclass[threadIdx.x] = P.link_class[threadIdx.x];
    __syncthreads();
    if (warp >= P.warps_per_cta) return;
    const int n = P.n, D = P.D, words = P.words;
    const int per_warp = PL * words + D * P.rb;
    uint32_t *X = nsm + 16 + (size_t)warp * per_warp;          // [PL][words] by op id
    uint32_t *Rw = X + PL * words;                             // [D][rb]
    const int64_t slot = (int64_t)blockIdx.x * P.warps_per_cta + warp;
    int32_t *rem = P.rem + slot * n;
    int64_t *rdy = P.rdy + slot * n;
    uint64_t *pend = P.pend + slot * n * D;
    const int64_t nj = P.j_end - P.j_begin;
    const int64_t total = MODE == 0 ? P.n_cand : (int64_t)P.n_bases * nj;
    const int64_t nslots = (int64_t)gridDim.x * P.warps_per_cta;
    auto bm = [&](int d) {
        Bitmap b;
        b.w = Rw + d * P.rb;
        b.words = words;
        b.nw1 = P.nw1;
        b.nw2 = P.nw2;
        return b;
    };

    for (int64_t task = slot; task < total; task += nslots) {
        // ---- the candidate: placement into X, its priority order (base order + swap) ----
        const int32_t *pos_of, *order, *edst;
        const int64_t *et;
        int32_t ks = -1;
        bool valid = true;
        int bl = 0;
        int64_t j = task;
        if (MODE == 0) {
            pos_of = P.pos_of;
            order = P.order;
            edst = P.nd_dst;
            et = P.nd_t;
            valid = !((__ldg(P.invalid + (task >> 5)) >> (task & 31)) & 1u);
            if (valid) {
                const uint8_t *row = P.rows + task * P.stride;
                for (int w = 0; w < words; w++) {
                    const int32_t v = w * 32 + lane;
                    int x = 0;
                    if (v < n) {
                        const int64_t bit = (int64_t)v * PL;
                        x = (int)((__ldg(row + (bit >> 3)) >> (bit & 7)) & ((1u << PL) - 1u));
                    }
#pragma unroll
                    for (int k = 0; k < PL; k++) {
                        const uint32_t b = __ballot_sync(kFull, (x >> k) & 1);
                        if (lane == 0) X[k * words + w] = b;
                    }
                }
            }
        } else {
            bl = (int)(task / nj);
            j = P.j_begin + task % nj;
            const BaseLayoutDev *B = &P.bases[bl];
            pos_of = B->pos_of;
            order = B->order;
            edst = B->nd_dst;
            et = B->nd_t;
            const uint64_t cb = ctr_base_of(P.step, P.P_total, P.b_offset + bl);
            const int64_t grp = j >> kGroupShift;
            const bool coarse = coarse_group(P.seed, cb, grp, P.coarse_pct, P.n_coarse);   // S9
            Region rg = decode_region(P.seed, cb, grp, n);
            const uint8_t *adj = B->swap_blocked;
            const uint32_t *bits = B->bits;
            ks = coarse ? -1
                        : decode_swap(P.seed, cb, grp, n, P.mix[3], rg,
                                      [&](int32_t k) { return __ldg(adj + k) != 0; },
                                      [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); });
            const uint8_t *aop = P.allowed_op;
            LaneMove mv = coarse ? decode_coarse_lane(P.seed, cb, j, P.n_coarse, D) : decode_lane(P.seed, cb, j, ks >= 0 && (j & (kGroup - 1)) == 0, D, P.mix,
                                      rg, [&](int32_t q) { return __ldg(order + q); },
                                      [&](int32_t q) { return ldg_bits_dev_at<PL>(bits, words, q); },
                                      [&](int32_t op) { return (unsigned)__ldg(aop + op); });
            valid = mv.kind != kMoveInvalid;
            if (!valid) mv = no_move();
            if (coarse) rg = Region{0, n, 0};                        // any op may move
            if (valid && (P.feas.has_cap || P.feas.has_coloc))    // row f3
                valid = move_feasible<PL>(mv, rg, D, bits, words, order, B->allowed_pos,
                                          P.all_allowed, P.feas, P.feas.fbase + (size_t)bl * 8);
            if (valid) {
                for (int w = 0; w < words; w++) {
                    const int32_t v = w * 32 + lane;
                    int x = 0;
                    if (v < n) {
                        const int32_t q = __ldg(pos_of + v);
                        x = ldg_bits_dev_at<PL>(bits, words, q);
                        if ((uint32_t)(q - rg.c) < (uint32_t)rg.len) {
                            const unsigned aq = P.all_allowed ? 0xFFu : (unsigned)__ldg(B->allowed_pos + q);
                            x = coarse ? apply_coarse(mv.ws, mv.wd, (int)__ldg(B->coarse_pos + q), x, aq)
                                       : apply_lane(mv, q, x, aq);
                        }
                    }
#pragma unroll
                    for (int k = 0; k < PL; k++) {
                        const uint32_t b = __ballot_sync(kFull, (x >> k) & 1);
                        if (lane == 0) X[k * words + w] = b;
                    }
                }
            }
        }
        if (!valid) {
            if (lane == 0) {
                if (MODE == 0) P.makespans[task] = INT64_MAX;
                else if (P.keys_dbg) P.keys_dbg[j - P.j_begin] = kNone;
            }
            continue;
        }
        // the swap (ks, ks+1) exchanges two priorities
        auto prio_of = [&](int32_t v) -> uint32_t {
            int32_t q = __ldg(pos_of + v);
            if (ks >= 0) q = q == ks ? ks + 1 : (q == ks + 1 ? ks : q);
            return (uint32_t)q;
        };
        auto op_at = [&](uint32_t q) -> int32_t {
            int32_t k = (int32_t)q;
            if (ks >= 0) k = k == ks ? ks + 1 : (k == ks + 1 ? ks : k);
            return __ldg(order + k);
        };

        // ---- initial state: every op's missing inputs, sources released at time 0 ----
        for (int i = lane; i < D * P.rb; i += 32) Rw[i] = 0u;
        __syncwarp();
        for (int32_t v = lane; v < n; v += 32) {
            const int32_t dg = __ldg(P.indeg + v);
            __stcg(rem + v, dg);
            __stcg(reinterpret_cast<long long *>(rdy + v), 0ll);
            if (dg == 0) bm(dev_of<PL>(X, words, v)).set(prio_of(v));
        }
        __syncwarp();

        int64_t f = 0, lk0 = 0, lk1 = 0;       // lane d: device d free; lane l: links l, l+32
        int32_t hc = 0;                         // lane d: entries in device d's pending heap
        // pending heaps: one 32-ary min-heap of keys per device (node i's children are
        // 32i+1 .. 32i+32: a level is one coalesced warp load + a shuffle argmin)
        auto heap_pop = [&](int d) {
            uint64_t *h = pend + (size_t)d * n;
            const int32_t c = __shfl_sync(kFull, hc, d) - 1;
            if (lane == d) hc = c;
            if (c > 0) {
                const uint64_t lastk = h[c];
                int32_t i = 0;
                while (true) {
                    const int32_t c0 = 32 * i + 1;
                    if (c0 >= c) break;
                    const uint64_t kv = c0 + lane < c ? h[c0 + lane] : kNone;
                    const uint64_t mn = warp_min_u64(kv);
                    if (mn >= lastk) break;
                    const int l = __ffs(__ballot_sync(kFull, kv == mn)) - 1;
                    if (lane == 0) h[i] = mn;
                    i = c0 + l;
                }
                if (lane == 0) h[i] = lastk;
            }
            __syncwarp();
        };
        auto heap_push = [&](int d, uint64_t k) {
            uint64_t *h = pend + (size_t)d * n;
            const int32_t c = __shfl_sync(kFull, hc, d);
            if (lane == 0) {
                int32_t i = c;
                while (i > 0) {
                    const int32_t par = (i - 1) >> 5;
                    const uint64_t pk = h[par];
                    if (pk <= k) break;
                    h[i] = pk;
                    i = par;
                }
                h[i] = k;
            }
            if (lane == d) hc = c + 1;
            __syncwarp();
        };
        bool ok = true;
        for (int32_t step = 0; step < n; step++) {
            // each device's earliest start: its free time if an op is ready by then (first in
            // pi from the bitmap), else its pending heap's top (earliest arrival, then pi)
            uint64_t cand = kNone;
            bool has = false;
            if (lane < D) {
                has = bm(lane).any();
                if (has) cand = nd_key(f, bm(lane).first(), lane);
                else if (hc > 0) cand = pend[(size_t)lane * n];
            }
            const uint32_t hasmask = __ballot_sync(kFull, has);
            const uint64_t K = warp_min_u64(cand);
            if (K == kNone) { ok = false; break; }              // unreachable for a DAG
            const int d = (int)(K & 7u);
            const uint32_t pr = (uint32_t)(K >> 3) & kPrioMask;
            const int64_t S = (int64_t)(K >> 23);
            if ((hasmask >> d) & 1u) {
                if (lane == 0) bm(d).clear(pr);
                __syncwarp();
            } else {
                heap_pop(d);
            }
            const int32_t v = op_at(pr);
            const int64_t C = S + __ldg(reinterpret_cast<const long long *>(P.p) + v);
            if (lane == d) f = C;
            // pending ops of d whose inputs are in by its new free time become ready
            while (__shfl_sync(kFull, hc, d) > 0) {
                const uint64_t top = pend[(size_t)d * n];
                if ((int64_t)(top >> 23) > C) break;
                heap_pop(d);
                if (lane == 0) bm(d).set((uint32_t)(top >> 3) & kPrioMask);
                __syncwarp();
            }

            // ---- out-edges: FCFS prefix sums per link, arrivals, newly eligible ops ----
            const int64_t e0 = __ldg(reinterpret_cast<const long long *>(P.out_off) + v);
            const int64_t e1 = __ldg(reinterpret_cast<const long long *>(P.out_off) + v + 1);
            if (e1 - e0 == 1) {
                // a single out-edge (most ops): every lane computes the same values and lane 0
                // stores them -- one edge cannot race, so no atomics, no ballots, no scan
                const int32_t w = __ldg(edst + e0);
                const int y = dev_of<PL>(X, words, w);
                int64_t A = C;                                   // same device: C_v (L144)
                if (y != d) {
                    const int64_t t = __ldg(reinterpret_cast<const long long *>(et) +
                                            e0 * P.n_classes + lclass[d * D + y]);
                    if (P.link_queue) {                          // FCFS link d -> y
                        const int li = d * D + y;
                        const int64_t lf = __shfl_sync(kFull, li < 32 ? lk0 : lk1, li & 31);
                        A = max(C, lf) + t;
                        if (lane == (li & 31)) {
                            if (li < 32) lk0 = A;
                            else lk1 = A;
                        }
                    } else {
                        A = C + t;                               // congestion-free (L113)
                    }
                }
                const int64_t r = max((int64_t)__ldcg(reinterpret_cast<const long long *>(rdy + w)), A);
                const int32_t rm = __ldcg(rem + w) - 1;
                if (lane == 0) {
                    __stcg(reinterpret_cast<long long *>(rdy + w), (long long)r);
                    __stcg(rem + w, rm);
                }
                const int64_t fy = __shfl_sync(kFull, f, y & 31);
                if (rm == 0) {
                    const uint32_t pw = prio_of(w);
                    if (r <= fy) {
                        if (lane == 0) bm(y).set(pw);
                    } else {
                        heap_push(y, nd_key(r, pw, y));
                    }
                }
                __syncwarp();
                continue;
            }
            for (int64_t b0 = e0; b0 < e1; b0 += 32) {
                const int64_t i = b0 + lane;
                const bool in = i < e1;
                const int32_t w = in ? __ldg(edst + i) : 0;
                const int y = in ? dev_of<PL>(X, words, w) : d;
                const bool cross = in && y != d;
                int64_t t = 0;
                if (cross)
                    t = __ldg(reinterpret_cast<const long long *>(et) + i * P.n_classes +
                              lclass[d * D + y]);
                int64_t A = C;                                   // same device: C_v (L144)
                if (P.link_queue) {
                    uint32_t cm = __ballot_sync(kFull, cross);
                    while (cm) {                                 // one FCFS link d -> yy at a time
                        const int yy = __shfl_sync(kFull, y, __ffs(cm) - 1);
                        const bool gsel = cross && y == yy;
                        const uint32_t gm = __ballot_sync(kFull, gsel);
                        int64_t s = gsel ? t : 0;
#pragma unroll
                        for (int o = 1; o < 32; o <<= 1) {
                            const int64_t u = __shfl_up_sync(kFull, s, o);
                            if (lane >= o) s += u;
                        }
                        const int li = d * D + yy;
                        const int64_t lf = __shfl_sync(kFull, li < 32 ? lk0 : lk1, li & 31);
                        const int64_t start = max(C, lf);
                        if (gsel) A = start + s;
                        const int64_t tot = __shfl_sync(kFull, s, 31);
                        if (lane == (li & 31)) {
                            if (li < 32) lk0 = start + tot;
                            else lk1 = start + tot;
                        }
                        cm &= ~gm;
                    }
                } else if (cross) {
                    A = C + t;                                   // congestion-free (L113)
                }
                if (in) atomicMax(reinterpret_cast<unsigned long long *>(rdy + w),
                                  (unsigned long long)A);
                __syncwarp();
                bool elig = false;
                if (in) elig = atomicSub(rem + w, 1) == 1;
                int64_t r = 0;
                uint32_t pw = 0;
                if (elig) {
                    r = (int64_t)__ldcg(reinterpret_cast<const long long *>(rdy + w));
                    pw = prio_of(w);
                }
                const int64_t fy = __shfl_sync(kFull, f, y & 31);
                const bool topend = elig && r > fy;
                if (elig && !topend) bm(y).set(pw);
                uint32_t pm = __ballot_sync(kFull, topend);
                const uint64_t mykey = nd_key(r, pw, y);
                while (pm) {                                     // pushes, one at a time
                    const int l = __ffs(pm) - 1;
                    pm &= pm - 1;
                    heap_push(__shfl_sync(kFull, y, l), __shfl_sync(kFull, mykey, l));
                }
                __syncwarp();
            }
        }
        // C_max = max_d device free time (L159-162 eq. (3))
        int64_t mk = lane < D ? f : 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) mk = max(mk, __shfl_xor_sync(kFull, mk, o));
        if (!ok) mk = -1;                                        // surfaces as a parity failure
        if (lane == 0) {
            if (MODE == 0) {
                P.makespans[task] = mk;
            } else {
                const uint64_t key = ok ? (((uint64_t)mk << 24) | (uint64_t)j) : kNone;
                if (P.keys_dbg) P.keys_dbg[j - P.j_begin] = key;
                if (key != kNone)
                    atomicMin(reinterpret_cast<unsigned long long *>(P.keys + bl),
                              (unsigned long long)key);
            }
        }
        __syncwarp();
    }
}

size_t nd_smem(const NdParams &p, int warps) {
    return 64 + (size_t)warps * (p.planes * p.words + p.D * p.rb) * 4;
}

template <int MODE, int PL>
cudaError_t launch_t(const NdParams &p, int grid, cudaStream_t st) {
    const size_t smem = nd_smem(p, p.warps_per_cta);
    cudaError_t e = cudaFuncSetAttribute(nondelay_kernel<MODE, PL>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    nondelay_kernel<MODE, PL><<<grid, p.warps_per_cta * 32, smem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace

int nondelay_warps_per_cta(const NdParams &p) {
    const size_t budget = 220 * 1024;
    for (int w = kNdMaxWarps; w >= 1; w--)
        if (nd_smem(p, w) <= budget) return w;
    return 0;
}

int nondelay_max_ctas_per_sm(const NdParams &p) {
    int per_sm = 0;
    const size_t smem = nd_smem(p, p.warps_per_cta);
    auto k = p.planes == 1 ? nondelay_kernel<1, 1> : (p.planes == 2 ? nondelay_kernel<1, 2> : nondelay_kernel<1, 4>);
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, p.warps_per_cta * 32, smem) !=
        cudaSuccess)
        return 0;
    return per_sm;
}

cudaError_t launch_nondelay(const NdParams &p, int mode, int grid, cudaStream_t st) {
    note_launch();
    if (mode == 0) {
        if (p.planes == 1) return launch_t<0, 1>(p, grid, st);
        if (p.planes == 2) return launch_t<0, 2>(p, grid, st);
        return launch_t<0, 4>(p, grid, st);
    }
    if (p.planes == 1) return launch_t<1, 1>(p, grid, st);
    if (p.planes == 2) return launch_t<1, 2>(p, grid, st);
    return launch_t<1, 4>(p, grid, st);
}

}  // namespace pesto
