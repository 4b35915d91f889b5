// device_common.cuh -- TMA bulk copy / mbarrier helpers and placement sources shared by the
// 64-bit (eval64) and 32-bit saturating (eval32) makespan kernels (product code).
#pragma once
#include <stdint.h>

#include "moves.cuh"

namespace pesto {
namespace dev {

__device__ __forceinline__ uint32_t su32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
// a shared address the compiler keeps in a register instead of rematerialising it from
// SR_CgaCtaId before every access
__device__ __forceinline__ uint32_t su32_reg(const void *p) {
    uint32_t a;
    asm volatile("mov.b32 %0, %1;" : "=r"(a) : "r"(su32(p)));
    return a;
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(bar)),
                 "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(bar)) : "memory");
}
// blocking wait for the phase with the given parity; the hint lets the warp sleep in hardware
// instead of spinning on issue slots (the producer warp waits most of the time)
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n"
            " selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(ok) : "r"(su32(bar)), "r"(parity), "r"(1000000u) : "memory");
    }
}
// one TMA bulk copy global -> shared, completion counted on `bar` (bytes % 16 == 0)
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(su32(dst)), "l"(src), "r"(bytes), "r"(su32(bar)) : "memory");
}

// explicit shared-space accesses: a pointer kept in a struct loses its address space and the
// compiler falls back to generic LD/ST (long-scoreboard latency).  volatile + "memory" keeps
// program order with the other state accesses (read-after-write through a slot).
__device__ __forceinline__ uint32_t lds_u32(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
    return v;
}
__device__ __forceinline__ void sts_u32(uint32_t addr, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
// records written by TMA: volatile keeps them after the mbarrier wait (also volatile asm)
__device__ __forceinline__ uint4 lds_v4(uint32_t addr) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
    return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}
// read-only data staged before a barrier: not volatile, so it may be scheduled freely
__device__ __forceinline__ uint32_t lds_u8_nv(uint32_t addr) {
    uint32_t v;
    asm("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}
__device__ __forceinline__ void sts_u8(uint32_t addr, uint32_t v) {
    asm volatile("st.shared.u8 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
// barrier among the first `threads` threads of the CTA (the consumer warps), id >= 1
__device__ __forceinline__ void named_bar_sync(int id, int threads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(threads) : "memory");
}
__device__ __forceinline__ uint64_t lds_u64(uint32_t addr) {
    uint64_t v;
    asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(addr) : "memory");
    return v;
}
__device__ __forceinline__ void sts_u64(uint32_t addr, uint64_t v) {
    asm volatile("st.shared.u64 [%0], %1;" ::"r"(addr), "l"(v) : "memory");
}

// per-thread async copy of 4 bytes global -> shared (LDGSTS), in commit groups
__device__ __forceinline__ void cp_async4(uint32_t smem_addr, const void *gptr, bool pred) {
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %2, 0;\n"
        " @p cp.async.ca.shared.global [%0], [%1], 4;\n}\n"
        ::"r"(smem_addr), "l"(gptr), "r"((int)pred) : "memory");
}
// predicated forms (a guard predicate, not a branch): the walk's per-edge pushes stay in one
// basic block so the scheduler can interleave the lane's independent candidate chains
__device__ __forceinline__ uint32_t lds_u32_if(uint32_t addr, bool p) {
    uint32_t v = 0;
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n @q ld.shared.u32 %0, [%1];\n}\n"
                 : "+r"(v) : "r"(addr), "r"((int)p) : "memory");
    return v;
}
__device__ __forceinline__ void sts_u32_if(uint32_t addr, uint32_t v, bool p) {
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n @q st.shared.u32 [%0], %1;\n}\n"
                 ::"r"(addr), "r"(v), "r"((int)p) : "memory");
}
__device__ __forceinline__ void stg_u32_if(void *ptr, uint32_t v, bool p) {
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n @q st.global.u32 [%0], %1;\n}\n"
                 ::"l"(ptr), "r"(v), "r"((int)p) : "memory");
}
__device__ __forceinline__ void redmax_u32_if(void *ptr, uint32_t v, bool p) {
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n @q red.relaxed.gpu.global.max.u32 [%0], %1;\n}\n"
                 ::"l"(ptr), "r"(v), "r"((int)p) : "memory");
}
// 4-byte async copy that writes zero when `have` is false (src-size 0: nothing is read)
__device__ __forceinline__ void cp_async4_zfill(uint32_t smem_addr, const void *gptr, bool have) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n"
                 ::"r"(smem_addr), "l"(gptr), "r"(have ? 4 : 0) : "memory");
}
__device__ __forceinline__ void cp_async8_zfill(uint32_t smem_addr, const void *gptr, bool have) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n"
                 ::"r"(smem_addr), "l"(gptr), "r"(have ? 8 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() {
    asm volatile("cp.async.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

template <int PL>
__device__ __forceinline__ int bits_dev_at(const uint32_t *bits, int words, int32_t q) {
    int x = 0;
#pragma unroll
    for (int k = 0; k < PL; k++) x |= (int)((bits[k * words + (q >> 5)] >> (q & 31)) & 1u) << k;
    return x;
}

template <int PL>
__device__ __forceinline__ int ldg_bits_dev_at(const uint32_t *bits, int words, int32_t q) {
    int x = 0;
#pragma unroll
    for (int k = 0; k < PL; k++) x |= (int)((__ldg(bits + k * words + (q >> 5)) >> (q & 31)) & 1u) << k;
    return x;
}

// explicit rows: lane's code at position q from the bit-sliced words of its group
template <int PL>
__device__ __forceinline__ int planes_dev_at(const uint32_t *pl, int32_t q, int lane, int dmax) {
    if (PL == 1) return (int)((__ldg(pl + q) >> lane) & 1u);
    // codes >= D belong to rows K5 flagged infeasible; clamp so the discarded lane still
    // indexes inside its state columns
    if (PL == 2) {
        uint2 w = __ldg(reinterpret_cast<const uint2 *>(pl) + q);
        return min((int)(((w.x >> lane) & 1u) | (((w.y >> lane) & 1u) << 1)), dmax);
    }
    uint4 w = __ldg(reinterpret_cast<const uint4 *>(pl) + q);
    return min((int)(((w.x >> lane) & 1u) | (((w.y >> lane) & 1u) << 1) |
                     (((w.z >> lane) & 1u) << 2) | (((w.w >> lane) & 1u) << 3)), dmax);
}

__device__ __forceinline__ uint64_t warp_min_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
        v = w < v ? w : v;
    }
    return v;
}

__device__ __forceinline__ uint8_t *align16(uint8_t *p) {
    return reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(p) + 15) & ~uintptr_t(15));
}

// warp-private bitmap of the positions where any lane's placement differs from the base
__device__ __forceinline__ void build_touched(uint32_t *touched, int words, const LaneMove &mv,
                                              int lane) {
    for (int w = lane; w < words; w += 32) touched[w] = 0u;
    __syncwarp();
    if (mv.kind == kMoveFlip) {
        for (int f = 0; f < mv.nflip; f++) {
            const int32_t q = mv.fpos[f];
            atomicOr(&touched[q >> 5], 1u << (q & 31));
        }
    } else if (mv.kind == kMoveWindow && mv.wl > 0) {
        const int32_t a = mv.ws, e = mv.ws + mv.wl;   // [a, e)
        for (int32_t w = a >> 5; w <= (e - 1) >> 5; w++) {
            const int32_t lo = max(a, w * 32) - w * 32, hi = min(e, w * 32 + 32) - w * 32;
            const uint32_t msk = (hi - lo == 32) ? 0xffffffffu : (((1u << (hi - lo)) - 1u) << lo);
            atomicOr(&touched[w], msk);
        }
    }
    __syncwarp();
}

__device__ __forceinline__ LaneMove no_move() {
    LaneMove mv;
    mv.kind = kMoveNone;
    mv.nflip = 0;
    mv.ws = mv.wl = mv.wd = 0;
    for (int q = 0; q < 4; q++) { mv.fpos[q] = -1; mv.fdev[q] = 0; }
    return mv;
}

}  // namespace dev
}  // namespace pesto
