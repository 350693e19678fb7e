// Device part of the check (steps a3, a4) and the plan / check C ABI.
//
// K1 shadow_check_window — one launch per window of consecutive access events.
//   Shadow cell: 8 B per 8-byte granule {W, R} (FastTrack's representation: the last write as an
//   epoch, the reads as an epoch while one fiber reads, a read vector when several do), each u32 =
//   fiber:8 | (event id + 1):24, 0 = empty.  When two or more fibers have read since the last
//   write, R = SPILL_TAG | r names a read-set record r in the device heap ({header with n,
//   epoch_1..epoch_n}), so the read set stays exact with a fixed 8-B cell.
//   The per-granule rule is the FastTrack-style check of SURVEY.md §8(c) step 3:
//       any access b:      W ≠ ∅ ∧ ¬HB(W, b)            → race (W, b)
//       write b:           ∀ read r ≠ ∅ ∧ ¬HB(r, b)     → race (r, b);   W := b, R := ∅
//       read b on fiber f: R[f] := b
//   with HB(e = (g, i+1), b in segment s of fiber f) ⇔ g = f ∨ i+1 ≤ segvc[s][g].
//   Work unit = a warp range: consecutive granules of one elementary interval, all covered by the
//   same accesses of the window.  Warps own contiguous runs of ranges (coverage-weighted).
//   Per range:
//     pass 1  stream the cells in (coalesced 128-bit loads = 2 cells, 8 in flight per lane) and vote
//             whether they are all equal (skipped in the interval's first window: known empty);
//     pass 2  equal cells evolve identically under the same accesses, so the warp applies the
//             window's accesses once to the common cell (the read set in shared memory); each hit
//             is a run over the whole range;
//     pass 3  stream the final cell out (128-bit stores; skipped when no later window needs it).
//   Ranges whose cells differ take the exact lane-parallel path: 32 lanes × 4 consecutive granules
//   per step, each lane its own cell and private read-set record (shared records are copied before
//   they are modified), hits compacted in the warp (__ballot_sync over hit lanes, __shfl_up_sync
//   comparison with the left neighbour, run heads sized from the continuation mask).  Both paths
//   feed a 32-entry per-warp run cache (one entry per lane) that extends runs across steps and
//   ranges before appending them to global memory.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <new>
#include <string>

#include "common.h"

using namespace cusan;

namespace {

constexpr int U = 4;                    // 32-granule chunks per lane-parallel step
constexpr int CHUNK = 32 * U;           // granules per lane-parallel step
#ifndef CUSAN_UL
#define CUSAN_UL 4
#endif
#ifndef CUSAN_MIN_BLOCKS
#define CUSAN_MIN_BLOCKS 3
#endif
constexpr int UL = CUSAN_UL;            // 16-B loads / stores in flight per lane when streaming
#ifndef CUSAN_DYNAMIC
#define CUSAN_DYNAMIC 0
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
constexpr size_t DYN_SMEM = CUSAN_TMA ? (size_t)8 * TMA_WARP_BYTES : 0;   // 8 = WARPS
#ifndef CUSAN_RANGES_PER_WARP
#define CUSAN_RANGES_PER_WARP 1
#endif
#ifndef CUSAN_RANGE_BAL_MIN
#define CUSAN_RANGE_BAL_MIN 4096
#endif
constexpr int GRAB = 2;                 // ranges a warp takes per dynamic-scheduler grab
constexpr int WARPS = 8;                // warps per block
constexpr int THREADS = 32 * WARPS;
constexpr int MAXS = 256;               // shared-memory read set per warp (≥ 255 readers)
constexpr unsigned FULL = 0xffffffffu;
static_assert(CHUNK % CELL_ALIGN == 0, "ranges start on aligned shadow slots");

// counters[]: 0 race granules, 1 raw runs, 2 heap top (record units), 3 heap overflow flag
enum { C_RACE = 0, C_RUNS = 1, C_HEAP = 2, C_HEAP_OVF = 3, N_COUNTERS = 4 };

// A window's work on one elementary interval, cut into warp ranges of `rsize` granules.
struct DSpan {
    uint64_t abs_begin, dense_begin, len;
    uint64_t tile0, weight0;     // prefix of ranges / of range weights over the window's spans
    uint32_t rsize, rweight;     // granules per range (multiple of CHUNK), weight of one range
    uint32_t list_off, list_cnt, flags, rec, rec_units, pad;
    uint64_t src_begin;          // where LOAD reads the cells: `shadow` (or `shadow_old` with SPAN_SRC_OLD)
};
static_assert(sizeof(DSpan) == 80, "DSpan layout");

struct Ctx {                     // kernel-wide pointers
    const AccRec* __restrict__ inc;
    const uint32_t* __restrict__ segvc;
    uint32_t F;
    uint2* __restrict__ shadow;
    const uint2* __restrict__ shadow_old;   // previous layout (incremental sessions), else null
    uint32_t* __restrict__ heap;
    unsigned long long heap_cap;  // record units
    cusan_race_run* __restrict__ runs;
    unsigned long long* __restrict__ counters;
    unsigned long long run_cap;
    int cow_all;                  // sessions: never modify a record in place (the previous check's
                                  // shadow must stay a consistent snapshot so a check can re-run)
};

struct RunCache {
    uint32_t e, l;       // earlier / later event id
    uint64_t gb, ge;     // [gb, ge), empty when ge == gb
    uint32_t rr;         // round-robin victim lane (warp-uniform)
    unsigned long long nrace;
};

__device__ __forceinline__ bool is_spill(uint32_t v) { return (v >> 24) == 0xFFu; }
__device__ __forceinline__ uint32_t* rec_ptr(const Ctx& k, uint32_t v) {
    return k.heap + (uint64_t)(v & 0xffffffu) * REC_WORDS;
}

__device__ __forceinline__ void flush_entry(const RunCache& c, const Ctx& k) {
    unsigned long long idx = atomicAdd(&k.counters[C_RUNS], 1ull);
    if (idx < k.run_cap) {
        cusan_race_run r;
        r.g_begin = c.gb;
        r.g_end = c.ge;
        r.earlier = c.e;
        r.later = c.l;
        k.runs[idx] = r;
    }
}

// Warp-collective: add run [rgb, rge) of (re, rl) to the per-warp run cache (one entry per lane):
// extend an entry that ends where the run begins, else evict the round-robin victim.
__device__ __forceinline__ void cache_insert(uint32_t re, uint32_t rl, uint64_t rgb, uint64_t rge, int lane,
                                             RunCache& rc, const Ctx& k) {
    const unsigned mm = __ballot_sync(FULL, rc.ge > rc.gb && rc.e == re && rc.l == rl && rc.ge == rgb);
    if (mm) {
        if (lane == __ffs(mm) - 1) rc.ge = rge;
    } else {
        if (lane == (int)rc.rr) {
            if (rc.ge > rc.gb) flush_entry(rc, k);
            rc.e = re;
            rc.l = rl;
            rc.gb = rgb;
            rc.ge = rge;
        }
        rc.rr = (rc.rr + 1) & 31u;
    }
}

// Warp-collective, lane-parallel granules: every lane passes its own hit flag (false for lanes
// without a granule).  Lanes hold consecutive granules g.
__device__ __forceinline__ void emit(bool hit, uint32_t earlier_epoch, uint32_t later_id, uint64_t g,
                                     int lane, RunCache& rc, const Ctx& k) {
    const unsigned m = __ballot_sync(FULL, hit);
    if (!m) return;
    rc.nrace += __popc(m);
    const uint32_t e_id = (earlier_epoch & 0xffffffu) - 1u;
    const uint32_t prev = __shfl_up_sync(FULL, e_id, 1);
    const bool cont = hit && lane > 0 && ((m >> (lane - 1)) & 1u) && prev == e_id;
    const unsigned cm = __ballot_sync(FULL, cont);
    unsigned heads = m & ~cm;
    uint32_t len = 0;
    if (hit && !cont) {
        const unsigned long long rest = (unsigned long long)cm >> (lane + 1);
        len = (uint32_t)__ffsll((long long)~rest);   // 1 + number of continuing lanes
    }
    while (heads) {
        const int h = __ffs(heads) - 1;
        heads &= heads - 1;
        const uint32_t re = __shfl_sync(FULL, e_id, h);
        const uint64_t rgb = __shfl_sync(FULL, g, h);
        const uint32_t rl = __shfl_sync(FULL, len, h);
        cache_insert(re, later_id, rgb, rgb + rl, lane, rc, k);
    }
}

// Warp-uniform: one hit covering every granule of [gb, ge).
__device__ __forceinline__ void emit_range(bool hit, uint32_t earlier_epoch, uint32_t later_id, uint64_t gb,
                                           uint64_t ge, int lane, RunCache& rc, const Ctx& k) {
    if (!hit) return;
    rc.nrace += ge - gb;
    cache_insert((earlier_epoch & 0xffffffu) - 1u, later_id, gb, ge, lane, rc, k);
}

// ¬HB(earlier epoch e, later access of fiber f whose segment row is `row`)
__device__ __forceinline__ bool unordered(uint32_t e, uint32_t f, const uint32_t* __restrict__ row) {
    if (!e) return false;
    const uint32_t g = e >> 24;
    return g != f && (e & 0xffffffu) > __ldg(row + g);
}

// ---- TMA bulk copies (cp.async.bulk, sm_90+; SASS UBLKCP) --------------------------------------
// Used by the streaming passes when CUSAN_TMA: pass 1 pulls the range's cells into a per-warp
// double buffer in shared memory (mbarrier completion), pass 3 pushes a shared-memory tile filled
// with the final cell out in bulk.  Addresses 16-B aligned, sizes multiples of 16.
__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred p;\n"
        "WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}\n"
        ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst_smem, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst_smem)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, const void* src_smem, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                 ::"l"(dst), "r"(smem_u32(src_smem)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// ---- lane path: per-granule read-set records ----------------------------------------------------
// Record header word: n (bits 0..15) | units (bits 16..23) | PRIVATE (bit 31).  Records written by
// the range path are shared by every granule of a range (never modified in place); records the
// lane path allocates belong to one granule's cell and are updated in place while they have room.
constexpr uint32_t REC_PRIVATE = 0x80000000u;
__device__ __forceinline__ uint32_t rec_n(uint32_t hdr) { return hdr & 0xffffu; }

// allocate a private record with room for `cap` entries holding n; returns the tagged slot value,
// or 0 on heap overflow (flagged; the host grows the heap and re-runs)
__device__ __forceinline__ uint32_t rec_alloc(const Ctx& k, uint32_t n, uint32_t cap, uint32_t** out) {
    const uint32_t units = (cap + 1 + REC_WORDS - 1) / REC_WORDS;
    const unsigned long long at = atomicAdd(&k.counters[C_HEAP], (unsigned long long)units);
    if (at + units > k.heap_cap) {
        k.counters[C_HEAP_OVF] = 1ull;
        *out = nullptr;
        return 0;
    }
    *out = k.heap + at * REC_WORDS;
    (*out)[0] = REC_PRIVATE | (units << 16) | n;
    return SPILL_TAG | (uint32_t)at;
}

// R[f] := ep on one lane's cell
__device__ void lane_read_update(uint2& c, uint32_t ep, uint32_t f, const Ctx& k) {
    if (!c.y) { c.y = ep; return; }
    uint32_t* dst;
    if (!is_spill(c.y)) {
        if ((c.y >> 24) == f) { c.y = ep; return; }
        const uint32_t v = rec_alloc(k, 2, 2 * REC_WORDS - 1, &dst);   // second reader: {R, ep}
        if (dst) { dst[1] = c.y; dst[2] = ep; }
        c.y = v;
        return;
    }
    uint32_t* src = rec_ptr(k, c.y);
    const uint32_t hdr = src[0];
    const uint32_t n = rec_n(hdr);
    int pos = -1;
    for (uint32_t j = 0; j < n; j++)
        if ((src[1 + j] >> 24) == f) { pos = (int)j; break; }
    if (pos >= 0 && src[1 + pos] == ep) return;
    if ((hdr & REC_PRIVATE) && !k.cow_all) {   // this granule's own record: update in place
        const uint32_t cap = ((hdr >> 16) & 0xffu) * REC_WORDS - 1;
        if (pos >= 0) { src[1 + pos] = ep; return; }
        if (n < cap) { src[1 + n] = ep; src[0] = hdr + 1; return; }
    }
    const uint32_t v = rec_alloc(k, pos >= 0 ? n : n + 1, 2 * (n + 1), &dst);   // copy, with room
    if (dst) {
        for (uint32_t j = 0; j < n; j++) dst[1 + j] = src[1 + j];
        if (pos >= 0) dst[1 + pos] = ep; else dst[1 + n] = ep;
    }
    c.y = v;
}

// Where a span's LOAD reads its cells (SPAN_SRC_OLD: the previous check's shadow of a session).
__device__ __forceinline__ const uint2* src_cells(const DSpan& sp, const Ctx& k) {
    return ((sp.flags & SPAN_SRC_OLD) ? k.shadow_old : k.shadow) + sp.src_begin;
}

// Lane-parallel exact path for granules [x0, x0 + n) of span sp (each lane its own cells).
__device__ void check_lanes(const DSpan& sp, uint64_t x0, uint64_t n, int lane, RunCache& rc, const Ctx& k) {
    for (uint64_t xc = x0; xc < x0 + n; xc += CHUNK) {
        uint2 cell[U];
        bool valid[U];
#pragma unroll
        for (int c = 0; c < U; c++) {
            const uint64_t x = xc + c * 32 + lane;
            valid[c] = x < x0 + n;
            cell[c] = make_uint2(0, 0);
            if (valid[c] && (sp.flags & SPAN_LOAD)) cell[c] = __ldcs(src_cells(sp, k) + x);
        }
        const uint32_t qe = sp.list_off + sp.list_cnt;
        for (uint32_t q = sp.list_off; q < qe; q++) {
            const AccRec r = k.inc[q];
            const uint32_t f = r.epoch >> 24;
            const uint32_t later = (r.epoch & 0xffffffu) - 1u;
            const uint32_t* row = k.segvc + (uint64_t)(r.segm & 0x7fffffffu) * k.F;
            const bool wr = r.segm >> 31;
#pragma unroll
            for (int c = 0; c < U; c++) {
                const uint64_t g = sp.abs_begin + xc + c * 32 + lane;
                emit(valid[c] && unordered(cell[c].x, f, row), cell[c].x, later, g, lane, rc, k);
                if (wr) {
                    const bool sp_r = valid[c] && is_spill(cell[c].y);
                    emit(valid[c] && !sp_r && unordered(cell[c].y, f, row), cell[c].y, later, g, lane, rc, k);
                    uint32_t* rp = sp_r ? rec_ptr(k, cell[c].y) : nullptr;
                    const uint32_t nr = sp_r ? rec_n(rp[0]) : 0u;
                    const uint32_t nmax = __reduce_max_sync(FULL, nr);
                    for (uint32_t j = 0; j < nmax; j++) {
                        const uint32_t v = j < nr ? rp[1 + j] : 0u;
                        emit(unordered(v, f, row), v, later, g, lane, rc, k);
                    }
                    // R := ∅.  A private record stays attached, emptied, for this granule's next
                    // readers (a record with n = 0 is the empty read set); shared ones detach.
                    uint32_t keep = 0;
                    if (sp_r && (rp[0] & REC_PRIVATE) && !k.cow_all) {
                        rp[0] &= ~0xffffu;
                        keep = cell[c].y;
                    }
                    cell[c] = make_uint2(r.epoch, keep);
                } else if (valid[c]) {
                    lane_read_update(cell[c], r.epoch, f, k);
                }
            }
        }
        if (sp.flags & SPAN_STORE) {
#pragma unroll
            for (int c = 0; c < U; c++) {
                const uint64_t x = xc + c * 32 + lane;
                if (valid[c]) __stcs(k.shadow + sp.dense_begin + x, cell[c]);
            }
        }
    }
}

__device__ __forceinline__ uint32_t find_span_by_tile(const DSpan* __restrict__ sp, uint32_t n, uint64_t t) {
    uint32_t lo = 0, hi = n;        // last span with tile0 <= t
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (sp[mid].tile0 <= t) lo = mid; else hi = mid;
    }
    return lo;
}

// first range whose start weight is >= pos
__device__ __forceinline__ uint64_t tile_at_weight(const DSpan* __restrict__ sp, uint32_t n,
                                                   uint64_t pos, uint64_t total_w, uint64_t total_t) {
    if (pos >= total_w) return total_t;
    uint32_t lo = 0, hi = n;
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (sp[mid].weight0 <= pos) lo = mid; else hi = mid;
    }
    const uint64_t w = sp[lo].rweight;
    return sp[lo].tile0 + (pos - sp[lo].weight0 + w - 1) / w;
}

__global__ void __launch_bounds__(THREADS, CUSAN_MIN_BLOCKS)
shadow_check_window(const DSpan* __restrict__ spans, uint32_t nspans, uint64_t total_tiles,
                    uint64_t total_weight, Ctx k, int force_lanes, unsigned long long* sched) {
    __shared__ uint32_t s_list[WARPS][MAXS];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    uint32_t* lst = s_list[warp];
#if CUSAN_TMA
    extern __shared__ __align__(128) unsigned char dsm[];
    unsigned char* wsm = dsm + (size_t)warp * TMA_WARP_BYTES;
    uint4* s_ld0 = reinterpret_cast<uint4*>(wsm);
    uint4* s_ld1 = reinterpret_cast<uint4*>(wsm + TMA_CHUNK);
    uint4* s_pat = reinterpret_cast<uint4*>(wsm + 2 * TMA_CHUNK);
    uint64_t* s_bar = reinterpret_cast<uint64_t*>(wsm + 2 * TMA_CHUNK + TMA_PAT);
    if (lane == 0) {
        mbar_init(&s_bar[0]);
        mbar_init(&s_bar[1]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t ph0 = 0, ph1 = 0;              // mbarrier phases (warp-uniform)
#endif
    RunCache rc;
    rc.e = rc.l = 0;
    rc.gb = rc.ge = 0;
    rc.rr = 0;
    rc.nrace = 0;
    // Range assignment: with `sched`, warps grab GRAB consecutive ranges at a time from a per-launch
    // counter (dynamic balance); without, each warp owns one coverage-weighted contiguous slice.
    uint64_t tend = 0;
    uint32_t s = 0;
    bool first = true;
    {
        for (uint64_t t = 0;; t++) {
            if (t >= tend) {
                uint64_t b, e;
                if (sched) {
                    unsigned long long base = 0;
                    if (lane == 0) base = atomicAdd(sched, (unsigned long long)GRAB);
                    b = __shfl_sync(FULL, base, 0);
                    e = min(b + (uint64_t)GRAB, total_tiles);
                } else {
                    if (!first) break;
                    const uint64_t nwarps = (uint64_t)gridDim.x * WARPS;
                    const uint64_t wid = (uint64_t)blockIdx.x * WARPS + warp;
                    b = tile_at_weight(spans, nspans, (uint64_t)((unsigned __int128)total_weight * wid / nwarps),
                                       total_weight, total_tiles);
                    e = tile_at_weight(spans, nspans, (uint64_t)((unsigned __int128)total_weight * (wid + 1) / nwarps),
                                       total_weight, total_tiles);
                    first = false;
                }
                if (b >= e) break;
                t = b;
                tend = e;
                s = find_span_by_tile(spans, nspans, t);
            }
            while (t >= spans[s + 1].tile0) s++;   // spans[nspans] is a sentinel
            const DSpan sp = spans[s];
            const uint64_t x0 = (t - sp.tile0) * sp.rsize;
            const uint64_t n = min((uint64_t)sp.rsize, sp.len - x0);   // granules of the range
            const bool comp = sp.flags & SPAN_COMPRESSED;           // f3: one cell per interval
            const uint64_t ncell = comp ? 1 : n;
            uint2* cells = k.shadow + sp.dense_begin + x0;      // 256-B aligned (CELL_ALIGN)
            const uint2* src = src_cells(sp, k) + x0;
            const uint4* cells2 = reinterpret_cast<const uint4*>(src);
            const uint64_t n2 = ncell >> 1;                     // cell pairs
            // ---- pass 1: stream the range's cells in and vote that they are all equal ----------
            uint2 c = make_uint2(0, 0);            // first window of the interval: known empty
            bool uniform = comp || !force_lanes;
            if (uniform && (sp.flags & SPAN_LOAD)) {
                c = src[0];
                bool ok = true;
#if CUSAN_TMA
                if ((reinterpret_cast<uintptr_t>(src) & 15u) == 0 && n2 * 16 >= TMA_MIN_BYTES) {
                    // bulk copies through a double buffer in shared memory (TMA engine)
                    const uint64_t bytes = n2 * 16;
                    const uint64_t nch = (bytes + TMA_CHUNK - 1) / TMA_CHUNK;
                    const unsigned char* gsrc = reinterpret_cast<const unsigned char*>(src);
                    if (lane == 0) {
                        const uint32_t sz = (uint32_t)umin64(TMA_CHUNK, bytes);
                        mbar_arrive_expect_tx(&s_bar[0], sz);
                        bulk_load(s_ld0, gsrc, sz, &s_bar[0]);
                    }
                    const uint4 cc = make_uint4(c.x, c.y, c.x, c.y);
                    for (uint64_t q = 0; q < nch; q++) {
                        const int st = (int)(q & 1);
                        if (q + 1 < nch && lane == 0) {          // prefetch the next chunk
                            const uint64_t off = (q + 1) * TMA_CHUNK;
                            const uint32_t sz = (uint32_t)umin64(TMA_CHUNK, bytes - off);
                            mbar_arrive_expect_tx(&s_bar[st ^ 1], sz);
                            bulk_load(st ? s_ld0 : s_ld1, gsrc + off, sz, &s_bar[st ^ 1]);
                        }
                        if (st == 0) { mbar_wait(&s_bar[0], ph0); ph0 ^= 1u; }
                        else { mbar_wait(&s_bar[1], ph1); ph1 ^= 1u; }
                        const uint4* buf = st ? s_ld1 : s_ld0;
                        const uint32_t nv = (uint32_t)(umin64(TMA_CHUNK, bytes - q * TMA_CHUNK) / 16);
                        for (uint32_t j = lane; j < nv; j += 32) {
                            const uint4 v = buf[j];
                            ok &= ((v.x ^ cc.x) | (v.y ^ cc.y) | (v.z ^ cc.z) | (v.w ^ cc.w)) == 0u;
                        }
                        __syncwarp();
                    }
                    if ((ncell & 1) && lane == 0) {
                        const uint2 tl = __ldcs(src + ncell - 1);
                        ok &= tl.x == c.x && tl.y == c.y;
                    }
                } else
#endif
                if ((reinterpret_cast<uintptr_t>(src) & 15u) == 0) {
                    for (uint64_t i = lane; i < n2; i += 32 * UL) {
                        uint4 v[UL];
#pragma unroll
                        for (int u = 0; u < UL; u++)
                            v[u] = (i + u * 32 < n2) ? __ldcs(cells2 + i + u * 32) : make_uint4(c.x, c.y, c.x, c.y);
#pragma unroll
                        for (int u = 0; u < UL; u++)
                            ok &= ((v[u].x ^ c.x) | (v[u].y ^ c.y) | (v[u].z ^ c.x) | (v[u].w ^ c.y)) == 0u;
                    }
                    if ((ncell & 1) && lane == 0) {
                        const uint2 tl = __ldcs(src + ncell - 1);
                        ok &= tl.x == c.x && tl.y == c.y;
                    }
                } else {                           // a session's old-layout source off a 16-B boundary
                    for (uint64_t i = lane; i < ncell; i += 32) {
                        const uint2 v = __ldcs(src + i);
                        ok &= v.x == c.x && v.y == c.y;
                    }
                }
                uniform = __all_sync(FULL, ok);
            }
            if (!uniform) {
                check_lanes(sp, x0, n, lane, rc, k);
                continue;
            }
            // ---- pass 2: all cells of the range equal `c`: apply the window's accesses once -----
            // the read set is kept in shared memory (ns entries); c.x = W
            uint32_t ns = 0;
            if (c.y) {
                if (is_spill(c.y)) {
                    const uint32_t* rp = rec_ptr(k, c.y);
                    ns = rec_n(rp[0]);
                    for (uint32_t j = lane; j < ns; j += 32) lst[j] = rp[1 + j];
                } else {
                    if (lane == 0) lst[0] = c.y;
                    ns = 1;
                }
                __syncwarp();
            }
            const uint64_t gb = sp.abs_begin + x0, ge = gb + n;
            const uint32_t qe = sp.list_off + sp.list_cnt;
            AccRec nxt = k.inc[sp.list_off];
            for (uint32_t q = sp.list_off; q < qe; q++) {
                const AccRec r = nxt;
                if (q + 1 < qe) nxt = k.inc[q + 1];
                const uint32_t f = r.epoch >> 24;
                const uint32_t later = (r.epoch & 0xffffffu) - 1u;
                const uint32_t* row = k.segvc + (uint64_t)(r.segm & 0x7fffffffu) * k.F;
                emit_range(unordered(c.x, f, row), c.x, later, gb, ge, lane, rc, k);
                if (r.segm >> 31) {
                    for (uint32_t j = 0; j < ns; j++) {
                        const uint32_t v = lst[j];
                        emit_range(unordered(v, f, row), v, later, gb, ge, lane, rc, k);
                    }
                    c.x = r.epoch;
                    ns = 0;
                } else {
                    int pos = -1;
                    for (uint32_t b = 0; b < ns; b += 32) {
                        const uint32_t j = b + lane;
                        const unsigned m = __ballot_sync(FULL, j < ns && (lst[j] >> 24) == f);
                        if (m) { pos = (int)(b + __ffs(m) - 1); break; }
                    }
                    if (lane == 0) lst[pos >= 0 ? pos : ns] = r.epoch;
                    if (pos < 0) ns++;
                    __syncwarp();
                }
            }
            // ---- pass 3: stream the final cell out -----------------------------------------------
            if (sp.flags & SPAN_STORE) {
                if (ns == 0) {
                    c.y = 0;
                } else if (ns == 1) {
                    c.y = lst[0];
                } else {
                    uint32_t* dst = nullptr;
                    uint32_t v = 0;
                    if (ns + 1 <= sp.rec_units * REC_WORDS) {      // the span's pre-assigned record
                        v = SPILL_TAG | sp.rec;
                        dst = k.heap + (uint64_t)sp.rec * REC_WORDS;
                    } else {
                        if (lane == 0) v = rec_alloc(k, ns, ns, &dst);
                        v = __shfl_sync(FULL, v, 0);
                        dst = v ? rec_ptr(k, v) : nullptr;
                    }
                    if (dst) {
                        if (lane == 0) dst[0] = ns;                 // shared: no PRIVATE bit
                        for (uint32_t j = lane; j < ns; j += 32) dst[1 + j] = lst[j];
                    }
                    c.y = v;
                }
                uint4* out2 = reinterpret_cast<uint4*>(cells);
                const uint4 cc = make_uint4(c.x, c.y, c.x, c.y);
#if CUSAN_TMA
                if (n2 * 16 >= TMA_MIN_BYTES) {
                    // a shared-memory tile of the final cell, pushed out by bulk copies
                    if (lane == 0) bulk_wait_read();          // the previous range's stores read the tile
                    __syncwarp();
                    for (uint32_t j = lane; j < TMA_PAT / 16; j += 32) s_pat[j] = cc;
                    fence_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        unsigned char* gdst = reinterpret_cast<unsigned char*>(out2);
                        const uint64_t bytes = n2 * 16;
                        for (uint64_t off = 0; off < bytes; off += TMA_PAT)
                            bulk_store(gdst + off, s_pat, (uint32_t)umin64(TMA_PAT, bytes - off));
                        bulk_commit();
                    }
                } else
#endif
                for (uint64_t i = lane; i < n2; i += 32 * UL) {
#pragma unroll
                    for (int u = 0; u < UL; u++)
                        if (i + u * 32 < n2) __stcs(out2 + i + u * 32, cc);
                }
                if ((ncell & 1) && lane == 0) __stcs(cells + ncell - 1, c);
            }
            __syncwarp();
        }
    }
#if CUSAN_TMA
    if (lane == 0) bulk_wait_all();                 // bulk stores done before the tile goes away
    __syncwarp();
#endif
    if (rc.ge > rc.gb) flush_entry(rc, k);
    if (lane == 0 && rc.nrace) atomicAdd(&k.counters[C_RACE], rc.nrace);
}

int cuda_fail(cudaError_t e, const char* what) {
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

}  // namespace

struct cusan_plan {
    const cusan_trace* trace = nullptr;
    HostPlan hp;
    int device = 0;
    cudaStream_t stream = nullptr;
    int max_blocks = 0;
    // device memory
    char* own = nullptr;          // library-allocated workspace (null when the caller's is used)
    char* ws = nullptr;
    uint64_t ws_bytes = 0;
    AccRec* d_inc = nullptr;
    uint32_t* d_segvc = nullptr;
    DSpan* d_spans = nullptr;
    unsigned long long* d_counters = nullptr;
    uint2* d_shadow = nullptr;
    uint32_t* d_heap = nullptr;
    uint64_t heap_cap = 0;                  // record units
    uint32_t* d_heap_own = nullptr;         // grown heap after an overflow
    cusan_race_run* d_runs = nullptr;
    cusan_race_run* d_runs_own = nullptr;   // grown run buffer after an overflow
    uint64_t run_cap = 0;
    bool need_shadow = false;
    bool bound = false;                     // workspace carved and tables uploaded
    uint64_t o_inc = 0, o_seg = 0, o_spans = 0, o_cnt = 0, o_heap = 0, o_shadow = 0, o_runs = 0;
    std::vector<DSpan> ds;                  // device span tables (host copy, uploaded at bind)
    std::vector<Window> wins;
    uint64_t shadow_cell_bytes = 0;
    uint64_t table_bytes = 0;               // tables uploaded by plan_create
    std::vector<unsigned long long> counter_init;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;

    ~cusan_plan() {
        if (ev0) cudaEventDestroy(ev0);
        if (ev1) cudaEventDestroy(ev1);
        if (own) cudaFree(own);
        if (d_runs_own) cudaFree(d_runs_own);
        if (d_heap_own) cudaFree(d_heap_own);
    }
};

static int plan_bind(cusan_plan* p, char* ws, uint64_t bytes);

// Device-side span tables: per window its spans plus a sentinel, with range / weight prefixes.
struct SpanTables {
    std::vector<DSpan> ds;
    std::vector<Window> wins;
    bool need_shadow = false;
    uint64_t cell_bytes = 0;      // algorithmic shadow bytes (8 B per LOAD + 8 B per STORE cell)
};

static void build_span_tables(const HostPlan& hp, int max_blocks, SpanTables& out) {
    std::vector<DSpan>& ds = out.ds;
    ds.clear();
    ds.reserve(hp.spans.size() + hp.win_span_off.size());
    out.wins.clear();
    out.need_shadow = false;
    out.cell_bytes = 0;
    for (size_t w = 0; w + 1 < hp.win_span_off.size(); w++) {
        Window win{};
        win.span_off = ds.size();
        uint64_t tiles = 0, weight = 0;
        // balance: at least RANGES_PER_WARP ranges per warp of a full grid in this window
        uint64_t moving = 0;
        for (uint64_t i = hp.win_span_off[w]; i < hp.win_span_off[w + 1]; i++)
            if (!(hp.spans[i].flags & SPAN_COMPRESSED) && (hp.spans[i].flags & (SPAN_LOAD | SPAN_STORE)))
                moving += hp.spans[i].len;
        const uint64_t rs_cap = std::max<uint64_t>(
            CUSAN_RANGE_BAL_MIN, moving / ((uint64_t)CUSAN_RANGES_PER_WARP * WARPS * std::max(max_blocks, 1)));
        for (uint64_t i = hp.win_span_off[w]; i < hp.win_span_off[w + 1]; i++) {
            const Span& s = hp.spans[i];
            DSpan d{};
            d.abs_begin = s.abs_begin;
            d.dense_begin = s.dense_begin;
            d.len = s.len;
            d.list_off = s.list_off;
            d.list_cnt = s.list_cnt;
            d.flags = s.flags;
            d.rec = s.rec;
            d.rec_units = s.rec_units;
            d.src_begin = s.src_begin;
            // warp range: long enough that replaying the window's accesses once per range stays
            // small next to streaming its cells, capped for balance; spans that move no cells
            // are one range each
            const bool comp = s.flags & SPAN_COMPRESSED;
            const bool moves = !comp && (s.flags & (SPAN_LOAD | SPAN_STORE));
            uint64_t rs;
            if (moves)
                rs = std::min<uint64_t>(std::min<uint64_t>(std::max<uint64_t>((uint64_t)CUSAN_RANGE_PER_ACCESS * s.list_cnt,
                                                                              (uint64_t)CUSAN_RANGE_MIN),
                                                           (uint64_t)CUSAN_RANGE_MAX),
                                        rs_cap);
            else
                rs = std::max<uint64_t>(s.len, 1);
            rs = std::min<uint64_t>((rs + CHUNK - 1) / CHUNK * CHUNK, 1ull << 31);
            d.rsize = (uint32_t)rs;
            const uint64_t nt = (s.len + rs - 1) / rs;
            const uint64_t mem = moves ? rs / 32 : 0;
            d.rweight = (uint32_t)std::min<uint64_t>(mem + 4ull * s.list_cnt + 8, 0xffffffffull);
            d.tile0 = tiles;
            d.weight0 = weight;
            tiles += nt;
            weight += nt * d.rweight;
            if (s.flags & (SPAN_LOAD | SPAN_STORE)) out.need_shadow = true;
            out.cell_bytes += (comp ? 1 : s.len) * (((s.flags & SPAN_LOAD) ? 8 : 0) + ((s.flags & SPAN_STORE) ? 8 : 0));
            ds.push_back(d);
        }
        win.nspans = (uint32_t)(ds.size() - win.span_off);
        DSpan sent{};
        sent.tile0 = tiles;
        sent.weight0 = weight;
        ds.push_back(sent);
        win.tiles = tiles;
        win.weight = weight;
        win.grid = (uint32_t)std::min<uint64_t>((uint64_t)max_blocks, (tiles + WARPS - 1) / WARPS);
        if (win.grid == 0) win.grid = 1;
        out.wins.push_back(win);
    }
}

static int device_info(int device, int* max_blocks) {
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0)
        return fail(CUSAN_ECUDA, std::string("no CUDA device available: ") + cudaGetErrorString(e));
    if (device < 0 || device >= ndev) return fail(CUSAN_EINVAL, "bad device ordinal");
    CK(cudaSetDevice(device));
    int sms = 0, per_sm = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    if (DYN_SMEM)
        CK(cudaFuncSetAttribute(shadow_check_window, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)DYN_SMEM));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, shadow_check_window, THREADS, DYN_SMEM));
    *max_blocks = sms * std::max(per_sm, 1);
    return CUSAN_OK;
}

static int plan_device_setup(cusan_plan* p) {
    HostPlan& hp = p->hp;
    const cusan_check_opts& o = hp.opts;
    int st0 = device_info(o.device, &p->max_blocks);
    if (st0) return st0;
    p->device = o.device;
    p->stream = (cudaStream_t)o.stream;

    SpanTables st;
    build_span_tables(hp, p->max_blocks, st);
    std::vector<DSpan>& ds = st.ds;
    p->wins = st.wins;
    p->need_shadow = st.need_shadow;
    p->shadow_cell_bytes = st.cell_bytes;

    // workspace layout
    p->heap_cap = hp.rec_units + (1ull << 16);             // pre-assigned records + lane-path room
    uint64_t off = 0;
    const uint64_t o_inc = off;     off = align_up(off + hp.inc.size() * sizeof(AccRec));
    const uint64_t o_seg = off;     off = align_up(off + hp.segvc.size() * sizeof(uint32_t));
    const uint64_t o_spans = off;   off = align_up(off + ds.size() * sizeof(DSpan));
    const uint64_t o_cnt = off;     off = align_up(off + (N_COUNTERS + p->wins.size()) * sizeof(unsigned long long));
    const uint64_t o_heap = off;    off = align_up(off + p->heap_cap * REC_WORDS * sizeof(uint32_t));
    const uint64_t o_shadow = off;  off = align_up(off + (p->need_shadow ? hp.shadow_cells * sizeof(uint2) : 0));
    p->run_cap = std::max<uint64_t>(1ull << 16, 4 * p->wins.size() + 1024);
    const uint64_t o_runs = off;    off = align_up(off + p->run_cap * sizeof(cusan_race_run));
    p->ws_bytes = off;
    p->o_inc = o_inc;
    p->o_seg = o_seg;
    p->o_spans = o_spans;
    p->o_cnt = o_cnt;
    p->o_heap = o_heap;
    p->o_shadow = o_shadow;
    p->o_runs = o_runs;
    p->ds = std::move(ds);
    p->table_bytes = hp.inc.size() * sizeof(AccRec) + hp.segvc.size() * sizeof(uint32_t) +
                     p->ds.size() * sizeof(DSpan);
    hp.ctr.shadow_bytes = p->need_shadow ? hp.shadow_cells * sizeof(uint2) : 0;
    hp.ctr.workspace_bytes = p->ws_bytes;
    CK(cudaEventCreate(&p->ev0));
    CK(cudaEventCreate(&p->ev1));
    if (o.workspace) return plan_bind(p, (char*)o.workspace, o.workspace_bytes);
    if (o.flags & CUSAN_CHECK_DEFER_WORKSPACE) return CUSAN_OK;   // caller binds later
    cudaError_t me = cudaMalloc((void**)&p->own, std::max<uint64_t>(off, ALIGN));
    if (me != cudaSuccess) return fail(CUSAN_ENOMEM, std::string("cudaMalloc workspace: ") + cudaGetErrorString(me));
    return plan_bind(p, p->own, off);
}

// Carve the workspace and upload the tables (a2 -> HBM).
static int plan_bind(cusan_plan* p, char* ws, uint64_t bytes) {
    if (bytes < p->ws_bytes)
        return fail(CUSAN_ENOMEM, "workspace too small: need " + std::to_string(p->ws_bytes) + " bytes");
    const HostPlan& hp = p->hp;
    CK(cudaSetDevice(p->device));
    p->ws = ws;
    p->d_inc = (AccRec*)(p->ws + p->o_inc);
    p->d_segvc = (uint32_t*)(p->ws + p->o_seg);
    p->d_spans = (DSpan*)(p->ws + p->o_spans);
    p->d_counters = (unsigned long long*)(p->ws + p->o_cnt);
    p->d_shadow = p->need_shadow ? (uint2*)(p->ws + p->o_shadow) : nullptr;
    if (!p->d_runs_own) p->d_runs = (cusan_race_run*)(p->ws + p->o_runs);
    if (!p->d_heap_own) p->d_heap = (uint32_t*)(p->ws + p->o_heap);
    else p->d_heap = p->d_heap_own;
    CK(cudaMemcpyAsync(p->d_inc, hp.inc.data(), hp.inc.size() * sizeof(AccRec), cudaMemcpyHostToDevice, p->stream));
    CK(cudaMemcpyAsync(p->d_segvc, hp.segvc.data(), hp.segvc.size() * sizeof(uint32_t), cudaMemcpyHostToDevice, p->stream));
    CK(cudaMemcpyAsync(p->d_spans, p->ds.data(), p->ds.size() * sizeof(DSpan), cudaMemcpyHostToDevice, p->stream));
    CK(cudaStreamSynchronize(p->stream));
    p->bound = true;
    return CUSAN_OK;
}

static int launch_all(cusan_plan* p) {
    // counters: race granules, runs, heap top (after the pre-assigned records), overflow flag
    // + one dynamic-scheduler counter per window
    p->counter_init.assign(N_COUNTERS + p->wins.size(), 0ull);
    p->counter_init[C_HEAP] = p->hp.rec_units;
    CK(cudaMemcpyAsync(p->d_counters, p->counter_init.data(), p->counter_init.size() * sizeof(unsigned long long),
                       cudaMemcpyHostToDevice, p->stream));
    CK(cudaEventRecord(p->ev0, p->stream));
    Ctx k;
    k.inc = p->d_inc;
    k.segvc = p->d_segvc;
    k.F = p->hp.F;
    k.shadow = p->d_shadow;
    k.shadow_old = nullptr;
    k.cow_all = 0;
    k.heap = p->d_heap;
    k.heap_cap = p->heap_cap;
    k.runs = p->d_runs;
    k.counters = p->d_counters;
    k.run_cap = p->run_cap;
    const int force_lanes = (p->hp.opts.flags & CUSAN_CHECK_FORCE_LANES) ? 1 : 0;
    for (size_t i = 0; i < p->wins.size(); i++) {
        const Window& w = p->wins[i];
        unsigned long long* sched = CUSAN_DYNAMIC ? p->d_counters + N_COUNTERS + i : nullptr;
        shadow_check_window<<<w.grid, THREADS, DYN_SMEM, p->stream>>>(p->d_spans + w.span_off, w.nspans, w.tiles,
                                                               w.weight, k, force_lanes, sched);
    }
    CK(cudaGetLastError());
    CK(cudaEventRecord(p->ev1, p->stream));
    return CUSAN_OK;
}

extern "C" {

int cusan_plan_create(const cusan_trace* t, const cusan_check_opts* o, cusan_plan** out) {
    if (!t || !o || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    cusan_plan* p = new (std::nothrow) cusan_plan;
    if (!p) return fail(CUSAN_ENOMEM, "cannot allocate plan");
    p->trace = t;
    int st;
    try {
        st = build_host_plan(t->t, *o, p->hp);
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while planning");
    }
    if (!st) st = plan_device_setup(p);
    if (st) {
        delete p;
        return st;
    }
    *out = p;
    return CUSAN_OK;
}

int cusan_plan_describe(const cusan_trace* t, const cusan_check_opts* o, cusan_counters* out) {
    if (!t || !o || !out) return fail(CUSAN_EINVAL, "null argument");
    HostPlan hp;
    int st;
    try {
        st = build_host_plan(t->t, *o, hp);
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while planning");
    }
    if (!st) *out = hp.ctr;
    return st;
}

int cusan_plan_workspace_bytes(const cusan_plan* p, uint64_t* bytes) {
    if (!p || !bytes) return fail(CUSAN_EINVAL, "null argument");
    *bytes = p->ws_bytes;
    return CUSAN_OK;
}

int cusan_plan_bind_workspace(cusan_plan* p, void* workspace, uint64_t bytes) {
    if (!p || !workspace) return fail(CUSAN_EINVAL, "null argument");
    if (p->own) return fail(CUSAN_ESTATE, "plan already owns a workspace");
    return plan_bind(p, (char*)workspace, bytes);
}

int cusan_plan_run(cusan_plan* p, cusan_report** out) {
    if (!p || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (!p->bound) return fail(CUSAN_ESTATE, "plan has no workspace: call cusan_plan_bind_workspace");
    const auto t_start = std::chrono::steady_clock::now();
    CK(cudaSetDevice(p->device));
    unsigned long long cnt[N_COUNTERS];
    for (int attempt = 0;; attempt++) {
        int st = launch_all(p);
        if (st) return st;
        CK(cudaMemcpyAsync(cnt, p->d_counters, sizeof(cnt), cudaMemcpyDeviceToHost, p->stream));
        CK(cudaStreamSynchronize(p->stream));
        const bool runs_ovf = cnt[C_RUNS] > p->run_cap, heap_ovf = cnt[C_HEAP_OVF] != 0;
        if (!runs_ovf && !heap_ovf) break;
        if (attempt >= 8) return fail(CUSAN_ENOMEM, "run buffer / spill heap keeps overflowing");
        if (runs_ovf) {                        // grow the run buffer and re-run (counts are exact)
            if (p->d_runs_own) cudaFree(p->d_runs_own);
            p->d_runs_own = nullptr;
            const uint64_t cap = cnt[C_RUNS] + cnt[C_RUNS] / 8 + 1024;
            if (cudaMalloc((void**)&p->d_runs_own, cap * sizeof(cusan_race_run)) != cudaSuccess)
                return fail(CUSAN_ENOMEM, "cannot grow the run buffer");
            p->d_runs = p->d_runs_own;
            p->run_cap = cap;
        }
        if (heap_ovf) {                        // grow the spill heap (24-bit record index)
            const uint64_t cap = std::min<uint64_t>(2 * p->heap_cap, (1ull << 24) - 1);
            if (cap <= p->heap_cap) return fail(CUSAN_ENOMEM, "spill heap exceeds the 24-bit record index");
            uint32_t* nh = nullptr;
            if (cudaMalloc((void**)&nh, cap * REC_WORDS * sizeof(uint32_t)) != cudaSuccess)
                return fail(CUSAN_ENOMEM, "cannot grow the spill heap");
            if (p->d_heap_own) cudaFree(p->d_heap_own);
            p->d_heap_own = nh;
            p->d_heap = nh;
            p->heap_cap = cap;
        }
    }
    float kms = 0.f;
    CK(cudaEventElapsedTime(&kms, p->ev0, p->ev1));
    cusan_report* r = new (std::nothrow) cusan_report;
    if (!r) return fail(CUSAN_ENOMEM, "cannot allocate report");
    try {
        r->runs.resize(cnt[C_RUNS]);
    } catch (...) {
        delete r;
        return fail(CUSAN_ENOMEM, "cannot allocate report runs");
    }
    if (cnt[C_RUNS]) {
        cudaError_t ce = cudaMemcpyAsync(r->runs.data(), p->d_runs, cnt[C_RUNS] * sizeof(cusan_race_run),
                                         cudaMemcpyDeviceToHost, p->stream);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(p->stream);
        if (ce != cudaSuccess) {
            delete r;
            return cuda_fail(ce, "run download");
        }
    }
    canonicalize_runs(r->runs);
    r->n_runs = r->runs.size();
    r->n_race_granules = cnt[C_RACE];
    const uint64_t max_runs = p->hp.opts.max_runs;
    if (max_runs && r->runs.size() > max_runs) {
        r->runs.resize(max_runs);
        r->truncated = 1;
    }
    r->ctr = p->hp.ctr;
    r->ctr.raw_runs = cnt[C_RUNS];
    r->ctr.kernel_ms = kms;
    r->ctr.kernel_launches = p->wins.size();
    r->ctr.shadow_cell_bytes = p->shadow_cell_bytes;
    r->ctr.h2d_bytes = p->table_bytes + sizeof(unsigned long long) * N_COUNTERS;
    r->ctr.d2h_bytes = sizeof(cnt) + cnt[C_RUNS] * sizeof(cusan_race_run);
    r->ctr.run_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count();
    *out = r;
    return CUSAN_OK;
}

int cusan_plan_destroy(cusan_plan* p) {
    if (!p) return fail(CUSAN_EINVAL, "plan is null");
    if (p->stream) cudaStreamSynchronize(p->stream);
    delete p;
    return CUSAN_OK;
}

int cusan_check(const cusan_trace* t, const cusan_check_opts* o, cusan_report** out) {
    cusan_plan* p = nullptr;
    int st = cusan_plan_create(t, o, &p);
    if (st) return st;
    st = cusan_plan_run(p, out);
    cusan_plan_destroy(p);
    return st;
}

}  // extern "C"

// ================================================================================================
// Incremental sessions: CuSan checks while the program runs
// (PAPER.md:606-612); a session keeps the shadow on the device between calls and each call checks
// only the accesses appended since the previous one.
//
// New accesses can split elementary intervals or add new ones, so every call re-plans the layout
// (a1, a2 over the whole trace; host cost only).  The previous call's shadow stays untouched as
// the source: intervals the call does not touch are copied to the new layout (copy_cells), the
// first span of a touched interval loads its cells from the old layout (SPAN_SRC_OLD), and read-set
// records are never modified in place (cow_all).  A call therefore only writes the new buffer and
// can be re-run as a whole after a run-buffer or heap overflow.  The buffers then swap.
// ================================================================================================
namespace {

struct CopySeg {
    uint64_t prefix, src, dst, len;       // cells [prefix, prefix + len) of the copy space
};

constexpr uint64_t COPY_CHUNK = 8192;     // cells per warp work item

__global__ void __launch_bounds__(THREADS)
copy_cells(const uint2* __restrict__ src, uint2* __restrict__ dst, const CopySeg* __restrict__ segs,
           uint32_t nseg, uint64_t total) {
    const int lane = threadIdx.x & 31;
    const uint64_t nwarps = (uint64_t)gridDim.x * WARPS;
    const uint64_t nchunks = (total + COPY_CHUNK - 1) / COPY_CHUNK;
    for (uint64_t ch = (uint64_t)blockIdx.x * WARPS + (threadIdx.x >> 5); ch < nchunks; ch += nwarps) {
        const uint64_t c0 = ch * COPY_CHUNK, c1 = min(c0 + COPY_CHUNK, total);
        uint32_t lo = 0, hi = nseg;                       // last segment with prefix <= c0
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (segs[mid].prefix <= c0) lo = mid; else hi = mid;
        }
        for (uint64_t c = c0; c < c1; lo++) {
            const CopySeg sg = segs[lo];
            const uint64_t end = min(c1, sg.prefix + sg.len);
            for (uint64_t i = c + lane; i < end; i += 32)
                __stcs(dst + sg.dst + (i - sg.prefix), __ldcs(src + sg.src + (i - sg.prefix)));
            c = end;
        }
    }
}

}  // namespace

struct cusan_session {
    const cusan_trace* trace = nullptr;
    cusan_check_opts opts{};
    int device = 0, max_blocks = 0;
    cudaStream_t stream = nullptr;
    std::vector<Interval> layout;                   // layout of `shadow`
    uint2* shadow = nullptr;
    uint64_t shadow_cap = 0;                        // cells
    uint2* spare = nullptr;
    uint64_t spare_cap = 0;
    uint32_t* heap = nullptr;
    uint64_t heap_cap = 0, heap_top = 0;            // record units
    char* scratch = nullptr;
    uint64_t scratch_cap = 0;
    cusan_race_run* runs = nullptr;
    uint64_t run_cap = 0;
    uint64_t checked_access = 0, checked_events = 0, n_calls = 0;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;

    ~cusan_session() {
        if (ev0) cudaEventDestroy(ev0);
        if (ev1) cudaEventDestroy(ev1);
        cudaFree(shadow);
        cudaFree(spare);
        cudaFree(heap);
        cudaFree(scratch);
        cudaFree(runs);
    }
};

template <class T>
static int ensure(T** p, uint64_t* cap, uint64_t need, const char* what) {
    if (*cap >= need && *p) return CUSAN_OK;
    cudaFree(*p);
    *p = nullptr;
    *cap = 0;
    const uint64_t n = std::max<uint64_t>(need, 1);
    if (cudaMalloc((void**)p, n * sizeof(T)) != cudaSuccess)
        return fail(CUSAN_ENOMEM, std::string("cannot allocate ") + what);
    *cap = n;
    return CUSAN_OK;
}

// grow the heap keeping records [0, heap_top)
static int grow_heap(cusan_session* s, uint64_t need) {
    if (s->heap_cap >= need && s->heap) return CUSAN_OK;
    if (need >= (1ull << 24)) return fail(CUSAN_ENOMEM, "read-set heap exceeds the 24-bit record index");
    const uint64_t cap = std::min<uint64_t>(std::max<uint64_t>(need, 2 * s->heap_cap), (1ull << 24) - 1);
    uint32_t* nh = nullptr;
    if (cudaMalloc((void**)&nh, cap * REC_WORDS * sizeof(uint32_t)) != cudaSuccess)
        return fail(CUSAN_ENOMEM, "cannot grow the read-set heap");
    if (s->heap && s->heap_top)
        CK(cudaMemcpyAsync(nh, s->heap, s->heap_top * REC_WORDS * sizeof(uint32_t), cudaMemcpyDeviceToDevice,
                           s->stream));
    CK(cudaStreamSynchronize(s->stream));
    cudaFree(s->heap);
    s->heap = nh;
    s->heap_cap = cap;
    return CUSAN_OK;
}

extern "C" {

int cusan_session_create(const cusan_trace* t, const cusan_check_opts* o, cusan_session** out) {
    if (!t || !o || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (o->nshards != 1 || o->shard != 0)
        return fail(CUSAN_EINVAL, "sessions check the whole granule space (nshards = 1)");
    if (o->workspace) return fail(CUSAN_EINVAL, "sessions manage their own device memory");
    cusan_session* s = new (std::nothrow) cusan_session;
    if (!s) return fail(CUSAN_ENOMEM, "cannot allocate session");
    s->trace = t;
    s->opts = *o;
    s->opts.persist_shadow = 1;
    int st = device_info(o->device, &s->max_blocks);
    if (!st) {
        s->device = o->device;
        s->stream = (cudaStream_t)o->stream;
        if (cudaEventCreate(&s->ev0) != cudaSuccess || cudaEventCreate(&s->ev1) != cudaSuccess)
            st = fail(CUSAN_ECUDA, "cannot create events");
    }
    if (st) {
        delete s;
        return st;
    }
    *out = s;
    return CUSAN_OK;
}

int cusan_session_check(cusan_session* s, cusan_report** out) {
    if (!s || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    const auto t_start = std::chrono::steady_clock::now();
    CK(cudaSetDevice(s->device));
    const Trace& tr = s->trace->t;
    if (tr.ev.size() < s->checked_events) return fail(CUSAN_ESTATE, "the trace shrank");

    // ---- a1 + a2 over the whole trace; spans only for the new accesses ------------------------
    HostPlan hp;
    int st;
    try {
        st = build_host_plan(tr, s->opts, hp, s->checked_access, s->heap_top);
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while planning");
    }
    if (st) return st;
    const uint64_t first = s->checked_access, n_acc = hp.acc_g0.size();
    uint64_t new_tracked = 0;
    for (uint64_t k = first; k < n_acc; k++) new_tracked += 8 * (hp.acc_g1[k] - hp.acc_g0[k]);

    // ---- old layout -> new layout ----------------------------------------------------------------
    // intervals are elementary for all accesses so far, so each new interval lies inside one old
    // interval or outside the old coverage
    std::vector<uint64_t> old_src(hp.iv.size(), UINT64_MAX);
    std::vector<CopySeg> segs;
    uint64_t copy_cells_n = 0;
    const bool compressed = (s->opts.flags & CUSAN_CHECK_INTERVAL_SHADOW) != 0;
    {
        size_t j = 0;
        for (size_t i = 0; i < hp.iv.size(); i++) {
            const Interval& v = hp.iv[i];
            while (j < s->layout.size() && s->layout[j].abs_begin + s->layout[j].len <= v.abs_begin) j++;
            if (j < s->layout.size() && s->layout[j].abs_begin <= v.abs_begin) {
                const Interval& u = s->layout[j];
                // compressed layouts (f3) keep one cell per interval: a split piece copies it
                old_src[i] = compressed ? u.dense_begin : u.dense_begin + (v.abs_begin - u.abs_begin);
                const uint64_t ncell = compressed ? 1 : v.len;
                const bool touched = v.list_cnt && hp.inc_acc[v.list_off + v.list_cnt - 1] >= first;
                if (!touched) {
                    segs.push_back({copy_cells_n, old_src[i], v.dense_begin, ncell});
                    copy_cells_n += ncell;
                }
            }
        }
    }
    for (Span& sp : hp.spans) {
        if (!(sp.flags & SPAN_FIRST_IN_CALL) || !(sp.flags & SPAN_LOAD)) continue;
        auto it = std::lower_bound(hp.iv.begin(), hp.iv.end(), sp.dense_begin,
                                   [](const Interval& a, uint64_t d) { return a.dense_begin < d; });
        const size_t i = it - hp.iv.begin();
        if (i >= hp.iv.size() || old_src[i] == UINT64_MAX)
            return fail(CUSAN_ESTATE, "internal: a loaded interval has no previous state");
        sp.flags |= SPAN_SRC_OLD;
        sp.src_begin = old_src[i];
    }
    SpanTables tabs;
    build_span_tables(hp, s->max_blocks, tabs);

    // ---- device memory ---------------------------------------------------------------------------
    if ((st = ensure(&s->spare, &s->spare_cap, hp.shadow_cells, "shadow"))) return st;
    if ((st = grow_heap(s, s->heap_top + hp.rec_units + (1ull << 16)))) return st;
    if ((st = ensure(&s->runs, &s->run_cap, std::max<uint64_t>(s->run_cap, 1ull << 16), "run buffer"))) return st;
    const uint64_t nwin = tabs.wins.size();
    uint64_t off = 0;
    const uint64_t o_inc = off;   off = align_up(off + hp.inc.size() * sizeof(AccRec));
    const uint64_t o_seg = off;   off = align_up(off + hp.segvc.size() * sizeof(uint32_t));
    const uint64_t o_spans = off; off = align_up(off + tabs.ds.size() * sizeof(DSpan));
    const uint64_t o_copy = off;  off = align_up(off + segs.size() * sizeof(CopySeg));
    const uint64_t o_cnt = off;   off = align_up(off + (N_COUNTERS + nwin) * sizeof(unsigned long long));
    if ((st = ensure(&s->scratch, &s->scratch_cap, off, "plan tables"))) return st;
    AccRec* d_inc = (AccRec*)(s->scratch + o_inc);
    uint32_t* d_seg = (uint32_t*)(s->scratch + o_seg);
    DSpan* d_spans = (DSpan*)(s->scratch + o_spans);
    CopySeg* d_copy = (CopySeg*)(s->scratch + o_copy);
    unsigned long long* d_cnt = (unsigned long long*)(s->scratch + o_cnt);
    CK(cudaMemcpyAsync(d_inc, hp.inc.data(), hp.inc.size() * sizeof(AccRec), cudaMemcpyHostToDevice, s->stream));
    CK(cudaMemcpyAsync(d_seg, hp.segvc.data(), hp.segvc.size() * sizeof(uint32_t), cudaMemcpyHostToDevice, s->stream));
    CK(cudaMemcpyAsync(d_spans, tabs.ds.data(), tabs.ds.size() * sizeof(DSpan), cudaMemcpyHostToDevice, s->stream));
    CK(cudaMemcpyAsync(d_copy, segs.data(), segs.size() * sizeof(CopySeg), cudaMemcpyHostToDevice, s->stream));

    // ---- a3 / a4 (re-runnable: only `spare` and fresh heap units are written) ----------------------
    std::vector<unsigned long long> init(N_COUNTERS + nwin, 0ull), cnt(N_COUNTERS, 0ull);
    float kms = 0.f;
    for (int attempt = 0;; attempt++) {
        init[C_HEAP] = s->heap_top + hp.rec_units;
        CK(cudaMemcpyAsync(d_cnt, init.data(), init.size() * sizeof(unsigned long long), cudaMemcpyHostToDevice,
                           s->stream));
        CK(cudaEventRecord(s->ev0, s->stream));
        if (copy_cells_n)
            copy_cells<<<s->max_blocks, THREADS, 0, s->stream>>>(s->shadow, s->spare, d_copy, (uint32_t)segs.size(),
                                                                  copy_cells_n);
        Ctx k;
        k.inc = d_inc;
        k.segvc = d_seg;
        k.F = hp.F;
        k.shadow = s->spare;
        k.shadow_old = s->shadow;
        k.heap = s->heap;
        k.heap_cap = s->heap_cap;
        k.runs = s->runs;
        k.counters = d_cnt;
        k.run_cap = s->run_cap;
        k.cow_all = 1;
        const int force_lanes = (s->opts.flags & CUSAN_CHECK_FORCE_LANES) ? 1 : 0;
        for (size_t i = 0; i < nwin; i++) {
            const Window& w = tabs.wins[i];
            unsigned long long* sched = CUSAN_DYNAMIC ? d_cnt + N_COUNTERS + i : nullptr;
            shadow_check_window<<<w.grid, THREADS, DYN_SMEM, s->stream>>>(d_spans + w.span_off, w.nspans, w.tiles, w.weight,
                                                                   k, force_lanes, sched);
        }
        CK(cudaGetLastError());
        CK(cudaEventRecord(s->ev1, s->stream));
        CK(cudaMemcpyAsync(cnt.data(), d_cnt, N_COUNTERS * sizeof(unsigned long long), cudaMemcpyDeviceToHost,
                           s->stream));
        CK(cudaStreamSynchronize(s->stream));
        const bool runs_ovf = cnt[C_RUNS] > s->run_cap, heap_ovf = cnt[C_HEAP_OVF] != 0;
        if (!runs_ovf && !heap_ovf) break;
        if (attempt >= 8) return fail(CUSAN_ENOMEM, "run buffer / read-set heap keeps overflowing");
        if (runs_ovf && (st = ensure(&s->runs, &s->run_cap, cnt[C_RUNS] + cnt[C_RUNS] / 8 + 1024, "run buffer")))
            return st;
        if (heap_ovf && (st = grow_heap(s, 2 * s->heap_cap))) return st;
    }
    CK(cudaEventElapsedTime(&kms, s->ev0, s->ev1));

    // ---- commit: the new buffer becomes the shadow ------------------------------------------------
    std::swap(s->shadow, s->spare);
    std::swap(s->shadow_cap, s->spare_cap);
    s->layout = hp.iv;
    s->heap_top = cnt[C_HEAP];
    s->checked_access = n_acc;
    s->checked_events = tr.ev.size();
    s->n_calls++;

    cusan_report* r = new (std::nothrow) cusan_report;
    if (!r) return fail(CUSAN_ENOMEM, "cannot allocate report");
    try {
        r->runs.resize(cnt[C_RUNS]);
    } catch (...) {
        delete r;
        return fail(CUSAN_ENOMEM, "cannot allocate report runs");
    }
    if (cnt[C_RUNS]) {
        cudaError_t ce = cudaMemcpy(r->runs.data(), s->runs, cnt[C_RUNS] * sizeof(cusan_race_run),
                                    cudaMemcpyDeviceToHost);
        if (ce != cudaSuccess) {
            delete r;
            return cuda_fail(ce, "run download");
        }
    }
    canonicalize_runs(r->runs);
    r->n_runs = r->runs.size();
    r->n_race_granules = cnt[C_RACE];
    if (s->opts.max_runs && r->runs.size() > s->opts.max_runs) {
        r->runs.resize(s->opts.max_runs);
        r->truncated = 1;
    }
    r->ctr = hp.ctr;
    r->ctr.tracked_bytes_shard = new_tracked;       // checked by this call
    r->ctr.raw_runs = cnt[C_RUNS];
    r->ctr.kernel_ms = kms;
    r->ctr.kernel_launches = nwin + (copy_cells_n ? 1 : 0);
    r->ctr.shadow_cell_bytes = tabs.cell_bytes + 16 * copy_cells_n;
    r->ctr.shadow_bytes = hp.shadow_cells * sizeof(uint2);
    r->ctr.h2d_bytes = hp.inc.size() * sizeof(AccRec) + hp.segvc.size() * sizeof(uint32_t) +
                       tabs.ds.size() * sizeof(DSpan) + segs.size() * sizeof(CopySeg);
    r->ctr.d2h_bytes = N_COUNTERS * sizeof(unsigned long long) + cnt[C_RUNS] * sizeof(cusan_race_run);
    r->ctr.run_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count();
    *out = r;
    return CUSAN_OK;
}

int cusan_session_destroy(cusan_session* s) {
    if (!s) return fail(CUSAN_EINVAL, "session is null");
    if (s->stream) cudaStreamSynchronize(s->stream);
    delete s;
    return CUSAN_OK;
}

}  // extern "C"
