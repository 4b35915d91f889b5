// layout_format.h -- position-space record stream streamed to the eval kernel (product code).
//
// For a schedule order pi (the per-device op order), ops are relabelled by
// position v = pos(op).  The record stream lists, for v = 0..n-1, one 16-byte OpRec followed by
// the op's out-edges (EdgeRec, `edge_stride` bytes each) sorted by successor position, ties by
// edge input index -- this is the FCFS tie order of reading R3, so pushing the
// transfers of a producer in record order advances each directed link's queue exactly as the
// First-Come-First-Served link of L144 / L188-198 does.  Ops whose out-degree exceeds
// kMaxInlineOut keep their edges out of line (OP_HEAVY + ExtRec).  The stream is cut into
// tiles at op boundaries; each tile is moved to shared memory with one cp.async.bulk.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define PESTO_LF_HD __host__ __device__
#else
#define PESTO_LF_HD
#endif

namespace pesto {

constexpr uint32_t kOpHeavy = 1u << 31;        // OpRec.nout: edges out of line, ExtRec follows
constexpr uint32_t kOpNoutMask = (1u << 24) - 1;
constexpr uint32_t kEdgeFirst = 1u << 31;      // EdgeRec.slot: first push into this slot
constexpr uint32_t kEdgeSlotMask = (1u << 31) - 1;
constexpr int kMaxInlineOut = 128;
constexpr int kNoSlot = -1;

struct alignas(16) OpRec {
    int64_t p;          // compute time p_v (ns)
    int32_t in_slot;    // ready-time slot read before the op starts; -1 = no predecessors
    uint32_t nout;      // out-degree | kOpHeavy
};

struct alignas(16) EdgeRec {
    int64_t t0;         // transfer time on link class 0 (further classes follow in 8-byte words)
    int32_t succ_pos;   // successor position
    uint32_t slot;      // successor's ready-time slot | kEdgeFirst
};

struct alignas(16) ExtRec {
    int64_t edge_off;   // byte offset of this op's EdgeRecs in the out-of-line edge array
    int64_t nout;
};

struct alignas(16) TileDesc {
    int64_t byte_off;   // offset of the tile in the record stream
    int32_t bytes;      // multiple of 16
    int32_t pos_begin;  // first position in the tile
    int32_t pos_end;    // one past the last
    int32_t pad[3];
};

// edge record stride for C link classes: 16 bytes + 8 bytes per extra class, 16-aligned
inline int edge_stride_for(int classes) { return 16 * ((classes + 2) / 2); }

// ---------------------------------------------------------------------------------------------
// 32-bit saturating layout (eval32).  Times are uint32 ns saturating at kSat32:
// every duration is < kMaxDur32 (else the graph is not eval32-eligible), so a + b never wraps
// (kSat32 + kMaxDur32 < 2^32) and min(a + b, kSat32) is exact while the true value is below
// kSat32.  Every start, finish and arrival time is <= the makespan, so a candidate whose
// makespan comes out < kSat32 is exact; the others are re-evaluated by the 64-bit path.
//
// A producer within kNearDelta positions of its consumer pushes into the warp's shared-memory
// ring (slot = consumer position mod kRing); farther producers push to a global "cold" slot
// with fire-and-forget stores / atomic max, and the cold value is prefetched to L1
// kPrefetchDist positions before the consumer reads it.
// ---------------------------------------------------------------------------------------------
constexpr uint32_t kSat32 = 0xF0000000u;        // 4,026,531,840 ns
constexpr uint32_t kMaxDur32 = 0x10000000u;     // durations must be < 2^28 ns
constexpr int kNearDelta = 12;
constexpr int kRing = 16;                       // >= kNearDelta + 3 (swap margins)
constexpr int kPrefetchDist = kNearDelta - 1;
constexpr uint32_t kOp32HasNear = 1u << 24;     // OpRec32.nout: read the near ring
constexpr int kOpXShift = 25;                   // OpRec32.nout bits 25-27: base device code
constexpr uint32_t kOpAdj = 1u << 28;           // producer feeds two adjacent positions
constexpr int kSuccXShift = 24;                 // EdgeRec32.succ_pos bits 24-26: base device
constexpr uint32_t kSuccPosMask = (1u << 24) - 1;
// EdgeRec32.succ_pos bits 27-29: the target's class as a dense code (0 far, 1 far first,
// 2 near, 3 near first, 4 next), so that the walk's uniform-device push finds (class, successor
// code) in one word and dispatches on them with a single jump table (eval32.cu push_uni)
constexpr int kSuccTcShift = 27;
constexpr uint32_t kSuccTcMask = 7u << kSuccTcShift;
constexpr uint32_t kSuccClassNone = 5;          // class code of an empty edge slot of a step
PESTO_LF_HD constexpr uint32_t target_class32(uint32_t target) {
    return (target & (1u << 29)) ? 4u : (((target >> 30) & 1u) << 1 | (target >> 31));
}
constexpr uint32_t kPinHeavy = 1u << 31;        // patch reference into the out-of-line array
constexpr uint32_t kPinSlot = 1u << 30;         // eval32 edge record in slot 1 of its step (else 0)
constexpr uint32_t kPinOffMask = kPinSlot - 1;  // byte offset part of a patch reference
constexpr uint32_t kT32First = 1u << 31;        // EdgeRec32.target: first push into its slot
constexpr uint32_t kT32Near = 1u << 30;         // push into the near ring (slot = succ & 15)
constexpr uint32_t kT32Next = 1u << 29;         // consumer is the next position: register
constexpr uint32_t kT32SlotMask = (1u << 29) - 1;   // byte offset (slot x 128) of the target

struct alignas(16) OpRec32 {
    uint32_t p;          // p_v (< kMaxDur32)
    int32_t cold_slot;   // this op's cold slot (far arrivals); -1 = none
    int32_t pf_slot;     // cold slot of the op kPrefetchDist positions ahead (async-copied); -1
    uint32_t nout;       // out-degree | kOp32HasNear | kOpAdj | base code << 25 | kOpHeavy
};

struct alignas(16) EdgeRec32 {
    uint32_t t0;         // transfer time (< kMaxDur32): D = 2 link 0 -> 1, else link class 0
    int32_t succ_pos;    // successor position | its base code << 24
    uint32_t target;     // slot byte offset (ring: (pos & 15) * 128, cold: slot * 128) | kT32Near | kT32First
    uint32_t t1;         // D = 2: link 1 -> 0, else link class 1
};

inline int edge_stride32_for(int classes) {
    return classes <= 2 ? 16 : 16 * (1 + (classes - 2 + 3) / 4);
}

// eval32 step stream: the π-ordered ops as fixed 48-byte steps -- a head and
// two EdgeRec32 slots -- so the walk is a straight-line loop with no per-op edge loop.  An op
// with more than two out-edges continues in CONT steps (head p/cold/pf unused).  Graphs with
// more than two distinct link classes use eval64.
struct alignas(16) StepHead {
    uint32_t p;          // p_v (< kMaxDur32)
    uint32_t kinds;      // D = 2: the fast walk's jump-table entry of each edge slot (byte k for
                         // slot k): yu | class << 1 | xu << 4 (kKind*); 0 for D > 2
    int32_t pf_slot;     // cold slot of the op kPrefetchDist positions ahead; -1 = none
    uint32_t flags;      // base code | kStHasNear | kStCont | edges << 5 | op steps << 8
};
// StepHead.kinds, per slot byte, D = 2: bit 0 the successor's base code yu, bits 1-3 the edge's
// class (kSuccTcShift codes, kSuccClassNone for an empty slot), bit 4 the op's base code xu;
// D = 3..4: bits 0-1 yu, 2-4 class, 5-6 xu.  0 for D > 4.  The layout writes them; K4 keeps the
// yu / xu bits in step with committed placement moves, a committed swap's retarget the class
// bits (each owner touches only its bits)
constexpr uint32_t kKindYu = 1u, kKindClassShift = 1, kKindClassMask = 7u << 1, kKindXu = 1u << 4;
PESTO_LF_HD constexpr int kind_cshift(int D) { return D <= 2 ? 1 : 2; }        // class bits
PESTO_LF_HD constexpr int kind_xshift(int D) { return D <= 2 ? 4 : 5; }        // xu bits
PESTO_LF_HD constexpr uint32_t kind_code_mask(int D) { return D <= 2 ? 1u : 3u; }
PESTO_LF_HD constexpr uint32_t kind_byte(int D, uint32_t yu, uint32_t cls, uint32_t xu) {
    return D > 4 ? 0u : (yu | cls << kind_cshift(D) | xu << kind_xshift(D));
}
constexpr int kStepBytes = 48;
constexpr uint32_t kStXMask = 7u;               // bits 0-2: base device code of the op
constexpr uint32_t kStHasNear = 1u << 3;        // read the near ring
constexpr uint32_t kStCont = 1u << 4;           // continuation step of the previous op
constexpr int kStEdgeShift = 5;                 // bits 5-6: edges in this step (0..2)
constexpr int kStStepsShift = 8;                // bits 8-31 (first step): steps of this op

}  // namespace pesto
