// feasibility.cuh -- row f3: memory footprint and colocation (L175)
// checks of a search candidate, in the prologue of the search kernels (product code).
//
// A candidate differs from its base only at the moved positions of its group's region, and the
// base satisfies the constraints, so the check is local: footprint_d = base footprint_d +
// the moved ops' footprints in minus out; and every colocation group touched by a move must
// end on one device, which means all its members are inside the region and moved together
// (members outside keep the base device, the moved op's old one).
#pragma once
#include "device_common.cuh"
#include "internal.h"

namespace pesto {
namespace dev {

// base: the base's bit planes (position space), order: op at each position, fbase: the base's
// footprint per device ([8]).  Returns false if the candidate violates a constraint.
template <int PL>
__device__ bool move_feasible(const LaneMove &mv, Region rg, int D, const uint32_t *bits, int words,
                              const int32_t *order, const uint8_t *allowed_pos, int all_allowed,
                              const Feasibility &F, const int64_t *fbase) {
    if (mv.kind == kMoveNone) return true;
    int64_t f[8];
#pragma unroll
    for (int d = 0; d < 8; d++) f[d] = d < D && F.has_cap ? __ldg(reinterpret_cast<const long long *>(fbase) + d) : 0;
    for (int32_t dq = 0; dq < rg.len; dq++) {
        const int32_t q = rg.c + dq;
        const int xb = ldg_bits_dev_at<PL>(bits, words, q);
        const unsigned aq = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q);
        const int xn = apply_lane(mv, q, xb, aq);
        if (xn == xb) continue;
        const int32_t op = __ldg(order + q);
        if (F.has_cap) {
            const int64_t m = __ldg(reinterpret_cast<const long long *>(F.mem) + op);
#pragma unroll
            for (int d = 0; d < 8; d++) f[d] += (d == xn ? m : 0) - (d == xb ? m : 0);
        }
        if (F.has_coloc) {
            const int32_t grp = __ldg(F.coloc + op);
            if (grp >= 0) {
                int32_t together = 0;                       // members in the region moved to xn
                for (int32_t dq2 = 0; dq2 < rg.len; dq2++) {
                    const int32_t q2 = rg.c + dq2;
                    if (__ldg(F.coloc + __ldg(order + q2)) != grp) continue;
                    const int xb2 = ldg_bits_dev_at<PL>(bits, words, q2);
                    const unsigned aq2 = all_allowed ? 0xFFu : (unsigned)__ldg(allowed_pos + q2);
                    if (apply_lane(mv, q2, xb2, aq2) == xn) together++;
                }
                if (together != __ldg(F.coloc_size + grp)) return false;
            }
        }
    }
    if (F.has_cap)
        for (int d = 0; d < D; d++)
            if (f[d] > __ldg(reinterpret_cast<const long long *>(F.cap) + d)) return false;
    return true;
}

}  // namespace dev
}  // namespace pesto
