// roofs.cu -- roof microbenchmarks of SURVEY §8(d) ("bench/roofs.cu"): the ceilings K1 is
// measured against, taken on the box that runs the bench.
//
//   * integer issue: independent uint32 chains of the K1 arithmetic -- c = min(max(r, d) + p, sat)
//     (one VIMNMX + one VIADDMNMX per chain step, 3 algorithmic ops: max, add, saturate) --
//     8 chains per thread, every SM full; reported as algorithmic int ops/s and SASS
//     instructions/s of that loop body;
//   * L2 bandwidth: a buffer of a quarter of the L2, swept 100 times with 128-bit loads
//     (read-only) and in K1's cold-slot pattern (32 consecutive 4-byte lanes, read + write);
//   * HBM bandwidth: a 1 GiB read + 1 GiB write copy kernel.
// Each is timed with CUDA events on a private stream, best of `reps`.
#include <cuda_runtime.h>
#include <stdint.h>

#include "host.h"
#include "internal.h"

namespace pesto {
namespace {

constexpr int kChains = 8;

// K1's per-op arithmetic on 8 independent chains: c = min(max(r, d) + p, sat)
__global__ void __launch_bounds__(256) roof_int_kernel(uint32_t *out, uint32_t seed, int iters) {
    uint32_t d[kChains], r[kChains];
#pragma unroll
    for (int k = 0; k < kChains; k++) {
        d[k] = seed * (threadIdx.x + 1) + k;
        r[k] = seed ^ (blockIdx.x * 131u + k);
    }
    const uint32_t p = seed & 0xFFu, sat = 0xF0000000u;
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int k = 0; k < kChains; k++) {
            d[k] = min(max(r[k], d[k]) + p, sat);
            r[k] = min(max(d[k], r[k]) + p + 1u, sat);
        }
    }
    uint32_t acc = 0;
#pragma unroll
    for (int k = 0; k < kChains; k++) acc ^= d[k] ^ r[k];
    if (acc == 0x12345678u) out[0] = acc;          // keeps the chains live
}

// L2-resident sweeps: read-only (128-bit) and K1's cold-slot read-modify-write (4-byte lanes)
__global__ void roof_l2_read_kernel(const uint4 *buf, size_t n16, int sweeps, uint32_t *out) {
    uint32_t acc = 0;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (int s = 0; s < sweeps; s++)
        for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) {
            const uint4 v = __ldcg(buf + i);
            acc ^= v.x ^ v.y ^ v.z ^ v.w;
        }
    if (acc == 0x12345678u) out[0] = acc;
}
__global__ void roof_l2_rmw_kernel(uint32_t *buf, size_t n4, int sweeps) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (int s = 0; s < sweeps; s++)
        for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride)
            __stcg(buf + i, max(__ldcg(buf + i), (uint32_t)s));
}
__global__ void roof_copy_kernel(const uint4 *src, uint4 *dst, size_t n16) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride)
        __stcs(dst + i, __ldcs(src + i));
}

struct Timer {
    cudaEvent_t a = nullptr, b = nullptr;
    Timer() { cudaEventCreate(&a); cudaEventCreate(&b); }
    ~Timer() { cudaEventDestroy(a); cudaEventDestroy(b); }
};

}  // namespace
}  // namespace pesto

using namespace pesto;

extern "C" pesto_status pesto_measure_roofs(int32_t device, int32_t reps, pesto_roofs *out) {
    if (!out || reps < 1) return fail(PESTO_EINVAL, "NULL output or reps < 1");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
        return fail(PESTO_ESTATE, "no such CUDA device");
    DeviceGuard guard(device);
    cudaDeviceProp prop;
    cudaError_t e = cudaGetDeviceProperties(&prop, device);
    if (e != cudaSuccess) return cuda_fail(e, "device properties");
    cudaStream_t st;
    if ((e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking)) != cudaSuccess)
        return cuda_fail(e, "stream");
    Timer tm;
    auto best_ms = [&](auto launch) {
        float best = 1e30f;
        for (int r = 0; r < reps + 1; r++) {          // the first run warms up
            cudaEventRecord(tm.a, st);
            launch();
            cudaEventRecord(tm.b, st);
            cudaEventSynchronize(tm.b);
            float ms = 0.f;
            cudaEventElapsedTime(&ms, tm.a, tm.b);
            if (r > 0 && ms < best) best = ms;
        }
        return (double)best;
    };
    const int sms = prop.multiProcessorCount;
    DevBuf scratch;
    if ((e = scratch.ensure(64)) != cudaSuccess) { cudaStreamDestroy(st); return cuda_fail(e, "allocate"); }
    // integer issue: every SM full (8 CTAs of 256 threads), 8 chains x 2 steps x iters per thread
    {
        const int grid = sms * 8, iters = 4096;
        const double ms = best_ms([&] {
            roof_int_kernel<<<grid, 256, 0, st>>>(scratch.as<uint32_t>(), 0x9E3779B9u, iters);
        });
        const double steps = (double)grid * 256 * iters * kChains * 2;
        out->int_ops_per_s = steps * 3.0 / (ms * 1e-3);          // max, add, saturate
        out->int_chain_steps_per_s = steps / (ms * 1e-3);
    }
    // L2: a quarter of the L2, 100 sweeps
    {
        const size_t bytes = ((size_t)prop.l2CacheSize / 4) & ~size_t(4095);
        DevBuf buf;
        if ((e = buf.ensure(bytes)) != cudaSuccess) { cudaStreamDestroy(st); return cuda_fail(e, "allocate"); }
        cudaMemsetAsync(buf.ptr, 1, bytes, st);
        const int grid = sms * 8, sweeps = 100;
        double ms = best_ms([&] {
            roof_l2_read_kernel<<<grid, 256, 0, st>>>(buf.as<uint4>(), bytes / 16, sweeps,
                                                      scratch.as<uint32_t>());
        });
        out->l2_read_gbs = (double)bytes * sweeps / (ms * 1e-3) / 1e9;
        ms = best_ms([&] { roof_l2_rmw_kernel<<<grid, 256, 0, st>>>(buf.as<uint32_t>(), bytes / 4, sweeps); });
        out->l2_rmw_gbs = 2.0 * (double)bytes * sweeps / (ms * 1e-3) / 1e9;
        out->l2_buffer_bytes = (int64_t)bytes;
    }
    // HBM: 1 GiB copy (read + write bytes)
    {
        const size_t bytes = (size_t)1 << 30;
        DevBuf a, b;
        if ((e = a.ensure(bytes)) != cudaSuccess || (e = b.ensure(bytes)) != cudaSuccess) {
            cudaStreamDestroy(st);
            return cuda_fail(e, "allocate");
        }
        cudaMemsetAsync(a.ptr, 1, bytes, st);
        const double ms = best_ms([&] {
            roof_copy_kernel<<<sms * 8, 256, 0, st>>>(a.as<uint4>(), b.as<uint4>(), bytes / 16);
        });
        out->hbm_copy_gbs = 2.0 * (double)bytes / (ms * 1e-3) / 1e9;
    }
    e = cudaStreamSynchronize(st);
    cudaStreamDestroy(st);
    if (e == cudaSuccess) e = cudaGetLastError();
    return e == cudaSuccess ? PESTO_OK : cuda_fail(e, "roof kernels");
}
