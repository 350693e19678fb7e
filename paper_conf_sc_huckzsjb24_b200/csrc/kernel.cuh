// Shared declarations of the shadow-check kernels and the host code that launches them
// (kernel.cu, check_api.cpp, session.cpp).  Not part of the C ABI.
#pragma once

#include <cuda_runtime.h>

#include <string>

#include "common.h"

namespace cusan {


constexpr int CHUNK = 128;              // granule multiple of a warp range (16-B aligned cell pairs per lane)
#ifndef CUSAN_UL
#define CUSAN_UL 4
#endif
#ifndef CUSAN_MIN_BLOCKS
#define CUSAN_MIN_BLOCKS 3
#endif
#ifndef CUSAN_MIN_BLOCKS_NT
#define CUSAN_MIN_BLOCKS_NT 4     // the compressed (no-TMA) instantiation of K1
#endif
constexpr int UL = CUSAN_UL;            // 16-B loads / stores in flight per lane when streaming
#ifndef CUSAN_DYNAMIC
#define CUSAN_DYNAMIC 1
#endif
#ifndef CUSAN_RANGE_PER_ACCESS
#define CUSAN_RANGE_PER_ACCESS 512
#endif
#ifndef CUSAN_RANGE_MIN
#define CUSAN_RANGE_MIN 16384
#endif
#ifndef CUSAN_RANGE_MAX
#define CUSAN_RANGE_MAX 262144
#endif
#ifndef CUSAN_TMA
#define CUSAN_TMA 1
#endif
#ifndef CUSAN_TMA_CHUNK
#define CUSAN_TMA_CHUNK 4096
#endif
#ifndef CUSAN_TMA_PAT
#define CUSAN_TMA_PAT 2048
#endif
constexpr uint32_t TMA_CHUNK = CUSAN_TMA_CHUNK;   // bytes per bulk load (double-buffered per warp)
constexpr uint32_t TMA_PAT = CUSAN_TMA_PAT;       // bytes of the store tile per warp
constexpr uint32_t TMA_MIN_BYTES = 8192; // ranges smaller than this stream through registers
constexpr uint32_t TMA_WARP_BYTES = 2 * TMA_CHUNK + TMA_PAT + 128;
constexpr size_t DYN_SMEM = CUSAN_TMA ? (size_t)8 * TMA_WARP_BYTES : 0;   // 8 = WARPS (K1 dynamic smem)
#ifndef CUSAN_RANGES_PER_WARP
#define CUSAN_RANGES_PER_WARP 1
#endif
#ifndef CUSAN_RANGE_BAL_MIN
#define CUSAN_RANGE_BAL_MIN 4096
#endif
#ifndef CUSAN_TAIL_PCT
#define CUSAN_TAIL_PCT 67         // guided tail (check_api.cpp build_span_tables): % of a span's ranges
#endif
#ifndef CUSAN_TAIL_DIV
#define CUSAN_TAIL_DIV 3          // ... cut this many times smaller, queued after every head
#endif
#ifndef CUSAN_GRAB
#define CUSAN_GRAB 1
#endif
constexpr int GRAB = CUSAN_GRAB;        // ranges a warp takes per dynamic-scheduler grab
constexpr int WARPS = 8;                // warps per block
constexpr int THREADS = 32 * WARPS;
constexpr int MAXS = 256;               // shared-memory read set per warp (≥ 255 readers)
constexpr unsigned FULL = 0xffffffffu;
static_assert(CHUNK % CELL_ALIGN == 0, "ranges start on aligned shadow slots");

// counters[]: 0 race granules, 1 raw runs, 2 heap top (record units), 3 heap overflow flag,
// 4 ranges whose cells were not all equal (planner invariant violated: the check fails)
enum { C_RACE = 0, C_RUNS = 1, C_HEAP = 2, C_HEAP_OVF = 3, C_INVARIANT = 4, N_COUNTERS = 5 };

// A window's work on one elementary interval, cut into warp ranges of `rsize` granules.
struct DSpan {
    uint64_t abs_begin, dense_begin, len;
    uint64_t tile0, weight0;     // prefix of ranges / of range weights over the window's spans
    uint32_t rsize, rweight;     // granules per range (multiple of CHUNK), weight of one range
    uint32_t list_off, list_cnt, flags, rec, rec_units, pad;
};
static_assert(sizeof(DSpan) == 72, "DSpan layout");

struct Ctx {                     // kernel-wide pointers
    const AccRec* __restrict__ inc;
    const uint32_t* __restrict__ segvc;
    uint32_t F;
    uint2* __restrict__ shadow;
    uint32_t* __restrict__ heap;
    unsigned long long heap_cap;  // record units
    cusan_race_run* __restrict__ runs;
    unsigned long long* __restrict__ counters;
    unsigned long long run_cap;
};


// Cells copied inside a session's shadow (pieces of a split compressed interval, f3).
struct CopySeg {
    uint64_t prefix, src, dst, len;       // cells [prefix, prefix + len) of the copy space
};

// A renumbered cell written over `len` cells from shadow index `dst` (fill space [prefix, prefix+len)).
struct CellFill {
    uint64_t prefix, dst, len;
    uint32_t w, r;
};

inline int cuda_fail(cudaError_t e, const char* what) {
    return fail(CUSAN_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
#define CK(call)                                        \
    do {                                                \
        cudaError_t _e = (call);                        \
        if (_e != cudaSuccess) return cuda_fail(_e, #call); \
    } while (0)

constexpr uint64_t ALIGN = 256;
inline uint64_t align_up(uint64_t x) { return (x + ALIGN - 1) / ALIGN * ALIGN; }

struct Window {
    uint64_t span_off;      // into d_spans (window-local array incl. sentinel)
    uint32_t nspans;
    uint64_t tiles, weight;
    uint32_t grid;
};

// A window as the device planner describes it (plan_dev.cu; downloaded for the launches).
struct WinDesc {
    uint64_t span_off, tiles, weight;
    uint32_t nspans, pad;
};


// ---- launch wrappers (kernel.cu) ----------------------------------------------------------------
// K1: one window of the shadow check
// (compressed: every span of the window is one interval-compressed cell — the instantiation without
// TMA buffers, on a grid of its own occupancy)
cudaError_t launch_shadow_check(uint32_t grid, cudaStream_t stream, const DSpan* spans, uint32_t nspans,
                                uint64_t tiles, uint64_t weight, const Ctx& k, unsigned long long* sched,
                                bool compressed);
// sessions: copy the cell of a split compressed interval to its new piece
cudaError_t launch_copy_cells(uint32_t grid, cudaStream_t stream, const uint2* src, uint2* dst,
                              const CopySeg* segs, uint32_t nseg, uint64_t total);
// sessions: epoch renumbering — one cell per interval out, renumbered cells back in
cudaError_t launch_gather_cells(uint32_t grid, cudaStream_t stream, const uint2* shadow, const uint64_t* at, uint64_t n,
                                uint2* out);
cudaError_t launch_fill_cells(uint32_t grid, cudaStream_t stream, uint2* shadow, const CellFill* f, uint32_t nf,
                              uint64_t total);
// resident blocks of K1 per SM (sets K1's dynamic shared memory limit first)
cudaError_t shadow_check_blocks_per_sm(int* per_sm);        // cached per device
cudaError_t shadow_check_blocks_per_sm_query(int* per_sm);  // sets the smem attribute, asks the occupancy API
cudaError_t shadow_check_max_blocks(bool compressed, int* max_blocks);   // SMs × blocks per SM, cached

// ---- host helpers shared by check_api.cpp and session.cpp -----------------------------------------
// Device-side span tables: per window its spans plus a sentinel, with range / weight prefixes.
struct SpanTables {
    pinned_vector<DSpan> ds;
    std::vector<Window> wins;
    bool need_shadow = false;
    uint64_t cell_bytes = 0;      // algorithmic shadow bytes (8 B per LOAD + 8 B per STORE cell)
};
void build_span_tables(const HostPlan& hp, int max_blocks, SpanTables& out);
int device_info(int device, int* max_blocks);

// ---- a4 on the device (merge.cu): raw runs -> canonical runs, downloaded into `out` -------------
struct RunMerge {                 // scratch: the caller's (plan workspace) or own, grown on demand
    char* buf = nullptr;
    uint64_t cap = 0;
    bool own = false;
    ~RunMerge();
};
int merge_scratch_bytes(uint64_t n, uint64_t* bytes);   // scratch for merging n raw runs
int merge_reserve(RunMerge& m, uint64_t n);               // own scratch for n raw runs
constexpr int MERGE_LAUNCHES = 4; // own kernels per merge (plus CUB's sort / scan kernels)
int merge_runs_device(RunMerge& m, cudaStream_t stream, const cusan_race_run* d_runs, uint64_t n,
                      std::vector<cusan_race_run>& out, uint64_t* d2h_bytes);

}  // namespace cusan
