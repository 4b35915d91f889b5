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

}  // namespace pesto
