// host.h -- host-side structures of libpesto (product code).
#pragma once
#include <nvtx3/nvToolsExt.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <list>
#include <memory>
#include <string>
#include <vector>

#include "internal.h"
#include "pesto.h"

namespace pesto {

constexpr int kMaxInlineBytes = 2048;   // eval64: an op's edges beyond this go out of line

void set_error(const std::string &msg);
pesto_status fail(pesto_status s, const std::string &msg);
pesto_status cuda_fail(cudaError_t e, const char *what);
int64_t launch_count_value();

// RAII device buffer
// NVTX ranges (SURVEY §5 tracing): header-only NVTX 3, a no-op unless a profiler (nsys, ncu
// --nvtx) injects itself; the C ABI's entry points name their phases
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

struct DevBuf {
    void *ptr = nullptr;
    size_t bytes = 0;
    DevBuf() = default;
    DevBuf(const DevBuf &) = delete;
    DevBuf &operator=(const DevBuf &) = delete;
    ~DevBuf() { release(); }
    void release() {
        if (ptr) cudaFree(ptr);
        ptr = nullptr;
        bytes = 0;
    }
    cudaError_t ensure(size_t want) {          // grow-only, contents not preserved
        if (want <= bytes && ptr) return cudaSuccess;
        release();
        cudaError_t e = cudaMalloc(&ptr, want ? want : 16);
        if (e == cudaSuccess) bytes = want ? want : 16;
        else ptr = nullptr;
        return e;
    }
    template <class T> T *as() const { return static_cast<T *>(ptr); }
};

// Position-space layout of one schedule order.
struct Layout {
    std::vector<int32_t> order, pos;
    int32_t W = 0;                      // live ready-time slots (padded intervals)
    int32_t stage_bytes = 0;            // largest tile (incl. header)
    std::vector<uint8_t> blob, heavy;   // record stream (tiles) and out-of-line edges
    std::vector<TileDesc> tiles;
    std::vector<uint8_t> swap_blocked, allowed_pos;   // swap_blocked[k]: (k, k+1) not swappable
    // 32-bit saturating stream (eval32)
    int32_t W32 = 0, stage_bytes32 = 0;
    std::vector<uint8_t> blob32, heavy32;
    std::vector<TileDesc> tiles32;
    std::vector<uint32_t> op_off32, pin_off, pin_ref;   // K4 patch index into blob32/heavy32
    // in-place swap patching (search.cpp): slot colourings and record locations
    std::vector<int32_t> slot64, first64;           // [op] eval64 slot, first producer position
    std::vector<int32_t> cslot, first_far;          // [op] eval32 cold slot (-1), first far producer
    std::vector<uint32_t> op_off64;                 // [pos] byte offset of the op record in blob
    std::vector<int32_t> tile64_of, tile32_of;      // [pos] tile holding the op's records
    std::vector<uint32_t> eloc64, eloc32;           // [edge] record offset (| kPinHeavy: heavy)
    std::vector<int32_t> slot_succ;                 // [2 * steps] successor position of each
                                                    // eval32 edge slot, -1 = empty (K5 y stream)
    // eval32 search fast walk: per region r (positions [64r, 64r + 64)), the
    // sorted positions where a group of that region is not warp-uniform -- the region itself and
    // every producer before it of an op inside it -- followed by INT32_MAX sentinels (slack, so a
    // committed swap can rewrite a region's list in place); CSR by region
    std::vector<uint32_t> spec_off;
    std::vector<int32_t> spec_pos;
    int64_t comm_gen = -1;
    // device copies
    DevBuf d_blob, d_heavy, d_tiles, d_pos, d_adj, d_allowed_pos, d_view, d_order;
    DevBuf d_blob32, d_heavy32, d_tiles32, d_op_off32, d_pin_off, d_pin_ref, d_slot_succ;
    DevBuf d_spec_off, d_spec_pos;
    // row f4(i): producer-grouped out-edges in this order's FCFS tie order (built on demand)
    DevBuf d_nd_dst, d_nd_t;
    int64_t nd_gen = -1;                // comm tables generation the nd arrays were built for
    bool on_device = false;
};

// Evaluation scratch (device): one set per graph for the synchronous calls and the search, one
// per pesto_workspace for asynchronous host-buffer evaluations that may overlap each other.
struct Scratch {
    DevBuf state;                 // eval64 ready-time slots
    DevBuf state32;               // eval32 cold slots
    DevBuf state32w;              // the search's wide eval32 launch (runs beside the 32-bit one)
    DevBuf planes, invalid;       // K5: bit-sliced rows, per-group infeasible-lane masks
    DevBuf yplanes;               // K5: codes per eval32 edge slot (explicit rows)
    DevBuf flags;                 // [count | list of saturated candidates]
    DevBuf rows, out;             // host-buffer calls: rows copied in, makespans copied out
    DevBuf nd_rem, nd_rdy, nd_pend;   // row f4(i) per-warp scratch
};

}  // namespace pesto

struct pesto_graph {
    int32_t n = 0, D = 1, planes = 1, words = 0;
    int64_t m = 0;
    int32_t device = -1;
    std::vector<int64_t> p, bytes;
    std::vector<int32_t> src, dst;
    std::vector<uint8_t> allowed;         // always filled (full mask when the caller gave NULL)
    bool all_allowed = true;
    std::vector<int64_t> out_off;         // CSR of out-edges by producer (edge ids)
    std::vector<int64_t> out_edges;
    std::vector<int64_t> in_off;          // CSR of in-edges by consumer, ascending edge id
    std::vector<int64_t> in_edges;
    std::vector<int32_t> indeg;
    // comm model per directed link a*D+b
    std::vector<int64_t> beta0, beta1;
    std::vector<uint8_t> link_set;
    int64_t comm_gen = 0;
    // derived from the comm model
    int32_t n_classes = 0;
    uint8_t link_class[64] = {0};
    std::vector<int64_t> t_class;         // [m][n_classes]
    int64_t t_gen = -1;
    bool eligible32 = false;              // every p and t < kMaxDur32: eval32 may run
    int64_t worst_total = 0;              // sum p + sum_e max_L t_e
    // movable ops (>= 2 allowed devices), ascending id; forbidden-code masks
    std::vector<int32_t> movable;
    std::vector<uint16_t> fmask;
    // layout cache (most recent first)
    std::list<std::shared_ptr<pesto::Layout>> cache;
    // device buffers
    pesto::DevBuf d_fmask, d_movable, d_allowed, d_bases;
    pesto::Scratch ws;                    // scratch of the synchronous calls and the search
    int32_t sms = 148;
    int32_t link_model = 0;               // PESTO_LINKS_FCFS / PESTO_LINKS_UNLIMITED
    int32_t dispatch = 0;                 // PESTO_DISPATCH_FIXED / PESTO_DISPATCH_NONDELAY
    pesto::DevBuf d_nd_p, d_nd_indeg, d_nd_off;
    bool nd_graph_ready = false;
    // row f3 constraints (host copies + device arrays); cons_gen counts changes
    bool has_cap = false, has_coloc = false;
    std::vector<int64_t> mem, cap;
    std::vector<int32_t> coloc, coloc_size;
    std::vector<int2> coloc_pairs;
    int64_t cons_gen = 0;
    pesto::DevBuf d_mem, d_cap, d_coloc, d_coloc_size, d_coloc_pairs;
    pesto::DevBuf d_cpos, d_ckey;         // row f2 exhaustive coarse search
};

namespace pesto {
// graph.cpp helpers used by search.cpp
pesto_status ensure_comm_tables(pesto_graph *g);
// x_op (device code per op id, nullable) is embedded in the eval32 records (search bases)
// tile32: the eval32 tile budget in bytes (0 = automatic: 6 KB at D = 2, else 8 KB)
pesto_status build_layout(pesto_graph *g, const int32_t *order, std::shared_ptr<Layout> &out,
                          bool use_cache, const uint8_t *x_op = nullptr, int32_t tile32 = 0);
pesto_status upload_layout(pesto_graph *g, Layout &L);
// v4 swap rule (DESIGN.md §4 S3) for the ops a (first) and c (second) of an adjacent pair
bool pair_blocked(const pesto_graph *g, int32_t a, int32_t c);
// the special positions of region r under L's order (see Layout::spec_pos), sorted, unique
void spec_region(const pesto_graph *g, const Layout &L, int32_t r, std::vector<int32_t> &out);
constexpr int kSpecSlack = 8;       // sentinels after each region's list
// row f4(i): device arrays of the non-delay kernel (graph-level and per order), the domain
// check (positive durations, n <= 2^20) and the scratch for `slots` resident warps
pesto_status nd_check(pesto_graph *g);
pesto_status nd_ensure_layout(pesto_graph *g, Layout &L);
pesto_status nd_fill(pesto_graph *g, Scratch &ws, NdParams &p, int64_t n_tasks, int *grid_out);
// row f2: PAPER.md §3.3 coarsening to at most `target` merged vertices (coarsen.cpp)
pesto_status coarsen_graph(const pesto_graph *g, int32_t target, std::vector<int32_t> &coarse_of,
                           int32_t &n_coarse);
// row f3: the kernels' view of the constraints; a placement (by op id) satisfies them?
Feasibility feasibility_view(const pesto_graph *g);
bool placement_feasible(const pesto_graph *g, const uint8_t *x, int64_t *footprint8);
BaseLayoutDev layout_view(const Layout &L);
void fill_eval_common(const pesto_graph *g, EvalParams &p);
pesto_status ensure_state(pesto_graph *g, Scratch &ws, const EvalParams &p, int search_mode,
                          int64_t n_tasks, int *grid_out);
// eval32 candidates per lane for a launch of n_tasks 256-candidate tasks:
// 1 when every task is resident at once (latency-bound: more warps), else 2
int choose_cpl32(const pesto_graph *g, int64_t n_tasks);
// eval32 launch plan for candidate ids [j0, j1) of n_bases bases: p.cpl32 (from the launch size
// in 256-candidate units), p.tasks_per_base and p.n_tasks in tasks of eval32_task_size(cpl)
void plan_eval32(const pesto_graph *g, EvalParams &p, int64_t j0, int64_t j1, int n_bases);
pesto_status ensure_state32(pesto_graph *g, Scratch &ws, const EvalParams &p, int search_mode,
                            int64_t n_tasks, int *grid_out, bool wide_buf = false);
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (dev >= 0 && dev != prev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};
}  // namespace pesto
