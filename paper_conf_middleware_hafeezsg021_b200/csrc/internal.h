// internal.h -- product-internal declarations shared by the host code and the CUDA kernels.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "layout_format.h"

namespace pesto {

constexpr int kWarps = 8;            // consumer warps per CTA (each = 32 candidates)
constexpr int kStages = 4;           // TMA tile ring depth
constexpr int kTileTarget32Search = 6144;   // eval32 layouts, D = 2 (five CTAs per SM)
constexpr int kTileTarget = 8192;    // record bytes per tile (a single op may exceed it)
constexpr int kTileHeader = 16;      // {pos_begin, pos_end, bytes, 0} at the head of each tile

// One schedule order's layout on the device (the eval path uses one, the search one per base).
struct BaseLayoutDev {
    const uint8_t *blob;        // tiles, each = 16-byte header + records
    const TileDesc *tiles;
    const uint8_t *heavy;       // out-of-line edge records of high fan-out ops
    const int32_t *pos_of;      // [n] op id -> position
    const uint8_t *allowed_pos; // [n] device mask by position
    const uint8_t *swap_blocked; // [n] 1 if positions (k, k+1) may not be swapped (DESIGN §4 S3)
    const uint32_t *bits;       // search: base placement, [planes][words] bit planes, by position
    int32_t n_tiles;
    int32_t W;                  // live ready-time slots
    // eval32 stream
    const uint8_t *blob32;
    const TileDesc *tiles32;
    const uint8_t *heavy32;
    int32_t n_tiles32;
    int32_t W32;                // cold slots
    const int32_t *order;       // [n] op id at each position
    const uint32_t *op_off32;   // [n] byte offset of the op record at each position (blob32)
    const uint32_t *pin_off;    // [n+1] CSR: edge records whose successor is at each position
    const uint32_t *pin_ref;    // byte offsets (| kPinHeavy for the out-of-line array)
    // row f4(i) non-delay kernel: out-edges by producer op id (graph CSR offsets), each
    // producer's edges in (successor position, edge index) order -- the FCFS tie order R3
    const int32_t *nd_dst;      // [m] consumer op id
    const int64_t *nd_t;        // [m][n_classes] transfer time per link class
    // search spec S9 (row f2 group moves): merged vertex of the op at each position, or null
    const uint8_t *coarse_pos;
    // eval32 search fast walk: special positions per region (Layout::spec_pos), CSR by region
    const uint32_t *spec_off;
    const int32_t *spec_pos;
};

// Row f3 constraints as the kernels see them (PAPER.md L202 memory, L175 colocation).
struct Feasibility {
    int32_t has_cap, has_coloc;
    const int64_t *mem;                 // [n] footprint by op id
    const int64_t *cap;                 // [D]
    const int32_t *coloc;               // [n] group by op id (-1 none)
    const int32_t *coloc_size;          // [n] members per group id
    const int2 *coloc_pairs;            // {op, representative op} for every non-first member
    int32_t n_pairs;
    int64_t *fbase;                     // search: [P][8] footprint of each base per device
};

struct EvalParams {
    int32_t n, D, planes, words;        // planes = bits per device code; words = ceil(n/32)
    int32_t edge_stride, n_classes;
    uint8_t link_class[64];             // class of directed link a*D+b
    int32_t stage_bytes;                // per-stage smem bytes (>= largest tile)
    int32_t all_allowed;
    // ready-time slot state: [cta][warp][W_max][32] int64
    int64_t *state;
    int32_t max_W;
    // explicit-placement mode
    const uint32_t *planes_in;          // [group][pos][planes] bit-sliced codes
    const uint32_t *yplanes;            // [group][slot][planes] codes of each edge slot's successor
    int64_t n_slots;                    // edge slots of the eval32 stream (2 per step)
    const uint32_t *invalid;            // [group] lanes with an infeasible row
    int64_t n_cand;
    int64_t *makespans;
    // search mode
    const BaseLayoutDev *bases;         // [P_local]
    int32_t b_offset, P_total;          // real base id = b_offset + local
    int64_t j_begin, j_end;             // candidate ids this launch covers (per base)
    uint64_t seed, step;
    int32_t mix[4];
    const int32_t *movable;
    int32_t n_movable;
    const uint8_t *allowed_op;          // [n] by op id
    uint64_t *keys;                     // [P_local] atomicMin targets
    uint64_t *keys_dbg;                 // nullable: key of every candidate in [j_begin, j_end)
    // work decomposition
    int64_t group_begin, groups_per_base, tasks_per_base, n_tasks;
    // eval32 (32-bit saturating) state and its explicit-mode fixup list
    uint32_t *state32;                  // [cta][warp][W32_max][32] cold slots
    int32_t max_W32, stage_bytes32, edge_stride32;
    int32_t *flag_list, *flag_count;    // saturated candidates, re-evaluated by eval64
    // search: base b runs on eval32 iff base_mk[b] < kSat32 (gate 1), on eval64 iff not (gate 2)
    const int64_t *base_mk;
    int32_t gate;
    // eval32 candidates per lane (1 or 2): more warps vs. more work per warp instruction
    int32_t cpl32;
    // eval32 search (mode 1): 1 = the wide instance (exact 64-bit times, same records) for the
    // bases at or above saturation (gate 2)
    int32_t wide32;
    // eval32 search, two candidates per lane, 32-bit time, launched alone (no wide launch
    // beside it): 1 = the instance without a producer warp at five CTAs per SM
    int32_t np32;
    // 1: FCFS link queues; 0: congestion-free links (row f4(ii))
    int32_t link_queue;
    // row f3 feasibility (search mode prologue): memory caps and colocation
    Feasibility feas;
    // row f2 exhaustive coarse search (eval32 mode 4): candidate j gives coarse vertex k the
    // device (j >> (coarse_bits * k)) & (D - 1); every op takes its merged vertex's device
    const uint8_t *coarse_pos;          // [n] merged vertex of the op at each position
    int32_t coarse_bits, n_coarse;
    int32_t coarse_pct;                 // search (mode 1): S9 coarse-group percentage (0 = off);
                                        // merged vertices per position in bases[b].coarse_pos
    uint8_t coarse_allowed[32];         // device mask of each merged vertex (AND of members)
    // eval64 list mode (MODE 2): candidates list[0 .. *list_count)
    const int32_t *list;
    const int32_t *list_count;
};

// Row f4(i): non-delay dispatch, one warp per candidate.
struct NdParams {
    int32_t n, D, planes, words;        // words = ceil(n/32)
    int32_t nw1, nw2, rb;               // ready-set bitmap levels: words, nw1, nw2 words; rb = sum
    int32_t n_classes, link_queue, all_allowed, warps_per_cta;
    uint8_t link_class[64];
    const int64_t *p;                   // [n] by op id
    const int32_t *indeg;               // [n] by op id
    const int64_t *out_off;             // [n+1] out-edge CSR offsets by producer op id
    int32_t *rem;                       // scratch per resident warp: [slot][n] inputs missing
    int64_t *rdy;                       // [slot][n] latest arrival so far
    uint64_t *pend;                     // [slot][D][n] per-device heaps of ops whose inputs arrive later
    // explicit rows (mode 0)
    const uint8_t *rows;                // [n_cand][stride], op i's code in bits [b*i, b*i+b)
    int64_t stride, n_cand;
    const uint32_t *invalid;            // [group] K5 (+ f3) infeasible-row masks
    int64_t *makespans;
    const int32_t *nd_dst, *pos_of, *order;
    const int64_t *nd_t;
    // search (mode 1)
    const BaseLayoutDev *bases;
    int32_t n_bases, b_offset, P_total;
    int64_t j_begin, j_end;
    uint64_t seed, step;
    int32_t mix[4];
    const uint8_t *allowed_op;
    uint64_t *keys, *keys_dbg;
    Feasibility feas;
    int32_t n_coarse, coarse_pct;       // S9 coarse groups (0 = off)
};

struct TransposeParams {
    const uint8_t *rows;
    int64_t stride, n_cand, n_groups;
    int32_t n, planes;
    const int32_t *pos_of;
    const uint16_t *fmask;              // [n] forbidden device codes per op (bit c = code c)
    uint32_t *planes_out;
    uint32_t *invalid_out;
    const int32_t *slot_succ;           // [n_slots] successor position of each edge slot, -1 none
    int64_t n_slots;
    uint32_t *yplanes_out;              // [group][n_slots][planes]
};

struct CommitParams {
    const BaseLayoutDev *bases;         // [P]
    uint32_t *bits;                     // [P][planes][words] (writable view of bases[b].bits)
    int32_t n, D, planes, words, P;
    uint64_t seed, step;
    int32_t mix[4];
    const int32_t *movable;
    int32_t n_movable;
    const uint8_t *allowed_op;
    const uint64_t *keys;
    int64_t *base_mk;
    int32_t *swap_out;                  // [P] committed swap position or -1
    Feasibility feas;                   // f3: the committed move updates fbase
    int32_t n_coarse, coarse_pct;       // S9 coarse groups (0 = off)
};

// explicit rows: OR the candidates violating the f3 constraints into the per-group masks
struct FeasParams {
    const uint32_t *planes;             // [group][pos][planes] (K5 output)
    uint32_t *invalid;                  // [group]
    int64_t n_groups;
    int32_t n, D, planes_n;
    const int32_t *order;               // [n] op at each position
    const int32_t *pos_of;              // [n] position of each op
    Feasibility feas;
};

// In-place layout patch (a committed adjacent swap, search.cpp): block rotations first, in list
// order, then masked word / byte stores in list order.
enum PatchKind : uint32_t { kPatchSet32 = 0, kPatchRotate = 1, kPatchSet8 = 2 };
struct PatchOp {
    uint64_t ptr;        // device address (16-aligned for rotations, 4-aligned for Set32)
    uint32_t kind;
    uint32_t a, b;       // rotate: [ptr, ptr+a) and [ptr+a, ptr+a+b) exchange places (16-multiples)
    uint32_t mask, val;  // set: *ptr = (*ptr & ~mask) | (val & mask)
    uint32_t pad;
};
constexpr int kPatchMaxBlock = 48 * 1024;      // rotation bytes a + b (shared-memory staging)
constexpr size_t kStreamPad = 512;              // zeroed bytes after K5's word streams
constexpr int kTransposeSmemMax = 200 * 1024;  // K5 smem variant: a group's n*planes words

// launchers (kernels.cu / eval32.cu); they return the launch error, if any.
cudaError_t launch_patch(const PatchOp *ops_dev, int n_ops, int max_block, cudaStream_t st);
// mode: 0 explicit rows, 1 search, 2 explicit list (eval64 only), 4 exhaustive coarse (eval32)
cudaError_t launch_eval(const EvalParams &p, int search_mode, int grid, cudaStream_t st);
cudaError_t launch_eval32(const EvalParams &p, int search_mode, int grid, cudaStream_t st);
int eval32_smem_bytes(const EvalParams &p, int search_mode);
// candidate ids per eval32 task (one CTA's share) for CPL candidates per lane
int eval32_task_size(int cpl);
int eval32_max_ctas_per_sm(const EvalParams &p, int search_mode);
cudaError_t launch_transpose(const TransposeParams &p, cudaStream_t st);
cudaError_t launch_feasibility(const FeasParams &p, cudaStream_t st);
cudaError_t launch_commit(const CommitParams &p, cudaStream_t st);
int eval_smem_bytes(const EvalParams &p, int search_mode);
// row f4(i): warps per CTA that fit the shared-memory budget (0: the graph does not fit), the
// resident CTAs per SM, and the launch (mode 0 explicit rows, 1 search)
int nondelay_warps_per_cta(const NdParams &p);
int nondelay_max_ctas_per_sm(const NdParams &p);
cudaError_t launch_nondelay(const NdParams &p, int mode, int grid, cudaStream_t st);
int eval_max_ctas_per_sm(const EvalParams &p, int search_mode);
void note_launch();

}  // namespace pesto
