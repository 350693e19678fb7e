// The shadow-check kernels (steps a3, a4) and their launch wrappers.
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
//   same accesses of the window.  Warps take ranges one at a time from a per-launch counter.
//   Per range:
//     pass 1  stream the cells in (coalesced 128-bit loads = 2 cells, 8 in flight per lane) and vote
//             whether they are all equal (skipped in the interval's first window: known empty);
//     pass 2  equal cells evolve identically under the same accesses, so the warp applies the
//             window's accesses once to the common cell (the read set in shared memory); each hit
//             is a run over the whole range;
//     pass 3  stream the final cell out (128-bit stores; skipped when no later window needs it).
//   Every granule of a range is covered by the same accesses (ranges lie inside one elementary
//   interval of the plan), so in the per-granule (dense) shadow all cells of a range are equal by
//   construction; pass 1's vote verifies that invariant (a violation is counted and fails the check
//   with CUSAN_ESTATE: it would be a planner bug).  With the interval-compressed shadow (f3, the
//   default) the range is the whole interval and its one cell is loaded once.  Hits feed a 32-entry
//   per-warp run cache (one entry per lane) that extends runs across ranges before appending them
//   to global memory.
#include <algorithm>
#include <atomic>

#include "kernel.cuh"

using namespace cusan;

namespace {

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

// Warp-uniform: one hit covering every granule of [gb, ge).
__device__ __forceinline__ void emit_range(bool hit, uint32_t earlier_epoch, uint32_t later_id, uint64_t gb,
                                           uint64_t ge, int lane, RunCache& rc, const Ctx& k) {
    if (!hit) return;
    rc.nrace += ge - gb;
    cache_insert((earlier_epoch & 0xffffffu) - 1u, later_id, gb, ge, lane, rc, k);
}

// Warp-collective: every lane with `hit` emits one run over the whole range [gb, ge) for its own
// (earlier epoch, later event), one lane after another.
__device__ __forceinline__ void emit_range_lanes(bool hit, uint32_t earlier_epoch, uint32_t later_id, uint64_t gb,
                                                 uint64_t ge, int lane, RunCache& rc, const Ctx& k) {
    for (unsigned m = __ballot_sync(FULL, hit); m; m &= m - 1) {
        const int h = __ffs(m) - 1;
        emit_range(true, __shfl_sync(FULL, earlier_epoch, h), __shfl_sync(FULL, later_id, h), gb, ge, lane, rc, k);
    }
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

// ---- read-set records ---------------------------------------------------------------------------
// Record = {header n, epoch_1 .. epoch_n} in REC_WORDS-word units, written once by the range that
// ends with that read set (pass 3) and only read afterwards.  The host pre-assigns one per span;
// rec_alloc is the fallback should a pre-assigned record be too small (never with an exact plan).
__device__ __forceinline__ uint32_t rec_n(uint32_t hdr) { return hdr & 0xffffu; }

// allocate a record with room for `cap` entries holding n; returns the tagged slot value, or 0 on
// heap overflow (flagged; a plan grows the heap and re-runs)
__device__ __forceinline__ uint32_t rec_alloc(const Ctx& k, uint32_t n, uint32_t cap, uint32_t** out) {
    const uint32_t units = (cap + 1 + REC_WORDS - 1) / REC_WORDS;
    const unsigned long long at = atomicAdd(&k.counters[C_HEAP], (unsigned long long)units);
    if (at + units > k.heap_cap) {
        k.counters[C_HEAP_OVF] = 1ull;
        *out = nullptr;
        return 0;
    }
    *out = k.heap + at * REC_WORDS;
    (*out)[0] = n;
    return SPILL_TAG | (uint32_t)at;
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

// TMA = false: the instantiation for windows whose spans are all interval-compressed (one cell per
// span, never streamed) — no dynamic shared memory, so more blocks fit on an SM (the compressed
// check is latency-bound: more warps in flight, fewer spans per warp).
template <bool TMA>
__global__ void __launch_bounds__(THREADS, TMA ? CUSAN_MIN_BLOCKS : CUSAN_MIN_BLOCKS_NT)
shadow_check_window(const DSpan* __restrict__ spans, uint32_t nspans, uint64_t total_tiles,
                    uint64_t total_weight, Ctx k, unsigned long long* sched) {
    constexpr bool kTMA = CUSAN_TMA && TMA;
    __shared__ uint32_t s_list[WARPS][MAXS];
    __shared__ uint8_t s_slot[WARPS][256];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    uint32_t* lst = s_list[warp];
    uint8_t* slot = s_slot[warp];
    for (int i = lane; i < 256; i += 32) slot[i] = 0xFFu;
    __syncwarp();
    extern __shared__ __align__(128) unsigned char dsm[];     // TMA buffers (none when !kTMA)
    unsigned char* wsm = dsm + (size_t)warp * TMA_WARP_BYTES;
    uint4* s_ld0 = reinterpret_cast<uint4*>(wsm);
    uint4* s_ld1 = reinterpret_cast<uint4*>(wsm + TMA_CHUNK);
    uint4* s_pat = reinterpret_cast<uint4*>(wsm + 2 * TMA_CHUNK);
    uint64_t* s_bar = reinterpret_cast<uint64_t*>(wsm + 2 * TMA_CHUNK + TMA_PAT);
    if constexpr (kTMA) {
        if (lane == 0) {
            mbar_init(&s_bar[0]);
            mbar_init(&s_bar[1]);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncwarp();
    }
    uint32_t ph0 = 0, ph1 = 0;              // mbarrier phases (warp-uniform)
    RunCache rc;
    rc.e = rc.l = 0;
    rc.gb = rc.ge = 0;
    rc.rr = 0;
    rc.nrace = 0;
    // Range assignment: with `sched`, warps grab GRAB consecutive ranges at a time from a per-launch
    // counter (dynamic balance); without, each warp owns one coverage-weighted contiguous slice.
    // The first grab is static (warp w takes range w: no atomic round trip before the first range of
    // a launch); later grabs continue after the grid's ranges.  When every span is one range (the
    // compressed layout, and short dense spans) range t is span t: no search.
    uint64_t tend = 0;
    uint32_t s = 0;
    bool first = true;
    const bool one_per_span = total_tiles == (uint64_t)nspans;
    const uint64_t nwarps_all = (uint64_t)gridDim.x * WARPS;
    {
        for (uint64_t t = 0;; t++) {
            if (t >= tend) {
                uint64_t b, e;
                if (sched) {
                    if (first) {
                        b = (uint64_t)blockIdx.x * WARPS + warp;
                        first = false;
                    } else {
                        unsigned long long base = 0;
                        if (lane == 0) base = atomicAdd(sched, (unsigned long long)GRAB);
                        b = nwarps_all + __shfl_sync(FULL, base, 0);
                    }
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
                s = one_per_span ? (uint32_t)t : find_span_by_tile(spans, nspans, t);
            }
            if (one_per_span) s = (uint32_t)t;
            else while (t >= spans[s + 1].tile0) s++;   // spans[nspans] is a sentinel
            const DSpan sp = spans[s];
            // f3: one cell per interval, and a compressed span is always a single range (its cell
            // must have exactly one owner, whatever the interval's length)
            const bool comp = sp.flags & SPAN_COMPRESSED;
            const uint64_t x0 = comp ? 0 : (t - sp.tile0) * sp.rsize;
            const uint64_t n = comp ? sp.len : min((uint64_t)sp.rsize, sp.len - x0);   // granules of the range
            const uint64_t ncell = comp ? 1 : n;
            uint2* cells = k.shadow + sp.dense_begin + x0;      // 8-B aligned (256-B for plan layouts)
            const uint2* src = cells;
            // 128-bit / bulk streaming needs 16-B alignment: a cell off it is handled on its own
            const uint64_t shead = (reinterpret_cast<uintptr_t>(src) & 15u) ? 1 : 0;
            const uint4* cells2 = reinterpret_cast<const uint4*>(src + shead);
            const uint64_t n2 = ncell > shead ? (ncell - shead) >> 1 : 0;   // aligned cell pairs
            const bool stail = ncell > shead && ((ncell - shead) & 1);
            // ---- pass 1: stream the range's cells in and vote that they are all equal ----------
            uint2 c = make_uint2(0, 0);            // first window of the interval: known empty
            bool uniform = true;
            if (sp.flags & SPAN_LOAD) {
                c = src[0];
                bool ok = true;
                if (kTMA && n2 * 16 >= TMA_MIN_BYTES) {
                    // bulk copies through a double buffer in shared memory (TMA engine)
                    const uint64_t bytes = n2 * 16;
                    const uint64_t nch = (bytes + TMA_CHUNK - 1) / TMA_CHUNK;
                    const unsigned char* gsrc = reinterpret_cast<const unsigned char*>(cells2);
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
                } else {
                    for (uint64_t i = lane; i < n2; i += 32 * UL) {
                        uint4 v[UL];
#pragma unroll
                        for (int u = 0; u < UL; u++)
                            v[u] = (i + u * 32 < n2) ? __ldcs(cells2 + i + u * 32) : make_uint4(c.x, c.y, c.x, c.y);
#pragma unroll
                        for (int u = 0; u < UL; u++)
                            ok &= ((v[u].x ^ c.x) | (v[u].y ^ c.y) | (v[u].z ^ c.x) | (v[u].w ^ c.y)) == 0u;
                    }
                }
                if (stail && lane == 0) {                  // (the head cell is src[0] = c itself)
                    const uint2 tl = __ldcs(src + ncell - 1);
                    ok &= tl.x == c.x && tl.y == c.y;
                }
                uniform = __all_sync(FULL, ok);
            }
            if (!uniform) {                        // planner invariant broken: fail the check
                if (lane == 0) atomicAdd(&k.counters[C_INVARIANT], 1ull);
                continue;
            }
            // ---- pass 2: all cells of the range equal `c`: apply the window's accesses once -----
            // 32 accesses at a time, lane l taking access q0 + l.  The state each access sees
            // follows from the batch's pattern of writes and reads (ballots, __match_any_sync), so
            // every happens-before test of a batch is one load per lane, issued in parallel.  The
            // read set lives in shared memory (lst, ns entries, one per fiber; slot[fiber] = its
            // index, 0xFF = absent); c.x = W.
            uint32_t ns = 0;
            if (c.y) {
                if (is_spill(c.y)) {
                    const uint32_t* rp = rec_ptr(k, c.y);
                    ns = rec_n(rp[0]);
                    for (uint32_t j = lane; j < ns; j += 32) {
                        const uint32_t v = rp[1 + j];
                        lst[j] = v;
                        slot[v >> 24] = (uint8_t)j;
                    }
                } else {
                    if (lane == 0) {
                        lst[0] = c.y;
                        slot[c.y >> 24] = 0;
                    }
                    ns = 1;
                }
                __syncwarp();
            }
            const uint64_t gb = sp.abs_begin + x0, ge = gb + n;
            const uint32_t qe = sp.list_off + sp.list_cnt;
            const unsigned below = (1u << lane) - 1u;
            for (uint32_t q0 = sp.list_off; q0 < qe; q0 += 32) {
                const bool act = q0 + lane < qe;
                AccRec r{0u, 0u};
                if (act) r = k.inc[q0 + lane];
                const bool isw = act && (r.segm >> 31);
                const bool isr = act && !isw;
                const uint32_t f = r.epoch >> 24;
                const uint32_t later = (r.epoch & 0xffffffu) - 1u;
                const uint32_t* row = k.segvc + (uint64_t)(r.segm & 0x7fffffffu) * k.F;
                const unsigned wm = __ballot_sync(FULL, isw);
                const unsigned rm = __ballot_sync(FULL, isr);
                const unsigned pw = wm & below;
                const int lw = pw ? 31 - __clz(pw) : -1;            // the last write before this access
                const uint32_t w_ep = __shfl_sync(FULL, r.epoch, lw < 0 ? 0 : lw);
                const uint32_t W = lw < 0 ? c.x : w_ep;
                // (1) every access against the last write before it
                emit_range_lanes(act && unordered(W, f, row), W, later, gb, ge, lane, rc, k);
                // the next read by the same fiber in this batch (32 = none)
                const unsigned same = __match_any_sync(FULL, isr ? f : 0x100u + (unsigned)lane);
                const unsigned above = same & ~((2u << lane) - 1u);
                const int nxt = above ? __ffs(above) - 1 : 32;
                if (wm) {
                    // (2) a write against the batch's reads since the last write before it that are
                    //     the last read of their fiber before it
                    if (rm) {
                        const unsigned cand = isw ? (rm & below & ~(lw < 0 ? 0u : ((2u << lw) - 1u))) : 0u;
                        unsigned hm = 0;
                        // groups of 8 candidate reads (8 independent clock loads in flight); a group
                        // no write of the batch must check is skipped (short spans: most of them)
                        const unsigned anyc = __reduce_or_sync(FULL, cand);
                        for (int p0 = 0; p0 < 32; p0 += 8) {
                            if (!((anyc >> p0) & 0xffu)) continue;
#pragma unroll
                            for (int p = p0; p < p0 + 8; p++) {
                                const uint32_t ep = __shfl_sync(FULL, r.epoch, p);
                                const int np = __shfl_sync(FULL, nxt, p);
                                if (((cand >> p) & 1u) && np > lane && unordered(ep, f, row)) hm |= 1u << p;
                            }
                        }
                        for (;;) {                                   // one run per (read, write) hit
                            const unsigned any = __ballot_sync(FULL, hm != 0);
                            if (!any) break;
                            const int h = __ffs(any) - 1;
                            const int pr = __ffs(__shfl_sync(FULL, hm, h)) - 1;
                            const uint32_t e = __shfl_sync(FULL, r.epoch, pr);
                            const uint32_t l = __shfl_sync(FULL, later, h);
                            emit_range(true, e, l, gb, ge, lane, rc, k);
                            if (lane == h) hm &= hm - 1;
                        }
                    }
                    // (3) the first write of the batch against the incoming read set, except the
                    //     fibers that read again in the batch before it
                    if (ns) {
                        const int l0 = __ffs(wm) - 1;
                        const uint32_t f0 = __shfl_sync(FULL, f, l0);
                        const uint32_t seg0 = __shfl_sync(FULL, r.segm & 0x7fffffffu, l0);
                        const uint32_t later0 = __shfl_sync(FULL, later, l0);
                        const uint32_t* row0 = k.segvc + (uint64_t)seg0 * k.F;
                        const unsigned rb = rm & ((1u << l0) - 1u);
                        for (uint32_t j0 = 0; j0 < ns; j0 += 32) {
                            const uint32_t j = j0 + lane;
                            const uint32_t v = j < ns ? lst[j] : 0u;
                            bool shadowed = false;
                            for (unsigned bb = rb; bb; bb &= bb - 1)
                                shadowed |= (v >> 24) == __shfl_sync(FULL, f, __ffs(bb) - 1);
                            emit_range_lanes(j < ns && !shadowed && unordered(v, f0, row0), v, later0, gb, ge,
                                             lane, rc, k);
                        }
                    }
                    // new state: W = the batch's last write, R = the reads after it (last per fiber)
                    const int lwl = 31 - __clz(wm);
                    c.x = __shfl_sync(FULL, r.epoch, lwl);
                    const unsigned live = __ballot_sync(FULL, isr && lane > lwl && nxt == 32);
                    __syncwarp();                          // reads of lst above before its rewrite
                    for (uint32_t j = lane; j < ns; j += 32) slot[lst[j] >> 24] = 0xFFu;
                    __syncwarp();
                    if ((live >> lane) & 1u) {
                        const uint32_t at = __popc(live & below);
                        lst[at] = r.epoch;
                        slot[f] = (uint8_t)at;
                    }
                    ns = __popc(live);
                    __syncwarp();
                } else if (rm) {
                    // reads only: each fiber's last read of the batch replaces its entry or joins
                    const bool last = isr && nxt == 32;
                    const uint32_t pos = last ? slot[f] : 0xFFu;
                    const unsigned app = __ballot_sync(FULL, last && pos == 0xFFu);
                    __syncwarp();
                    if (last) {
                        const uint32_t at = pos != 0xFFu ? pos : ns + __popc(app & below);
                        lst[at] = r.epoch;
                        slot[f] = (uint8_t)at;
                    }
                    ns += __popc(app);
                    __syncwarp();
                }
            }
            for (uint32_t j = lane; j < ns; j += 32) slot[lst[j] >> 24] = 0xFFu;   // index empty again
            __syncwarp();
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
                const uint64_t dhead = (reinterpret_cast<uintptr_t>(cells) & 15u) ? 1 : 0;
                uint4* out2 = reinterpret_cast<uint4*>(cells + dhead);
                const uint64_t m2 = ncell > dhead ? (ncell - dhead) >> 1 : 0;
                const bool dtail = ncell > dhead && ((ncell - dhead) & 1);
                const uint4 cc = make_uint4(c.x, c.y, c.x, c.y);
                if (dhead && lane == 0) __stcs(cells, c);
                if (kTMA && m2 * 16 >= TMA_MIN_BYTES) {
                    // a shared-memory tile of the final cell, pushed out by bulk copies
                    if (lane == 0) bulk_wait_read();          // the previous range's stores read the tile
                    __syncwarp();
                    for (uint32_t j = lane; j < TMA_PAT / 16; j += 32) s_pat[j] = cc;
                    fence_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        unsigned char* gdst = reinterpret_cast<unsigned char*>(out2);
                        const uint64_t bytes = m2 * 16;
                        for (uint64_t off = 0; off < bytes; off += TMA_PAT)
                            bulk_store(gdst + off, s_pat, (uint32_t)umin64(TMA_PAT, bytes - off));
                        bulk_commit();
                    }
                } else
                for (uint64_t i = lane; i < m2; i += 32 * UL) {
#pragma unroll
                    for (int u = 0; u < UL; u++)
                        if (i + u * 32 < m2) __stcs(out2 + i + u * 32, cc);
                }
                if (dtail && lane == 0) __stcs(cells + ncell - 1, c);
            }
            __syncwarp();
        }
    }
    if constexpr (kTMA) {
        if (lane == 0) bulk_wait_all();             // bulk stores done before the tile goes away
        __syncwarp();
    }
    if (rc.ge > rc.gb) flush_entry(rc, k);
    if (lane == 0 && rc.nrace) atomicAdd(&k.counters[C_RACE], rc.nrace);
}

constexpr uint64_t COPY_CHUNK = 8192;     // cells per warp work item

// Copy cells between layouts (a session splitting a compressed interval in place: the copy names the
// same read-set record, which is never modified after it is written).
__global__ void __launch_bounds__(THREADS)
copy_cells(const uint2* src, uint2* dst, const CopySeg* __restrict__ segs, uint32_t nseg, uint64_t total) {
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
            for (uint64_t i = c + lane; i < end; i += 32) {
                const uint2 v = __ldcs(src + sg.src + (i - sg.prefix));
                __stcs(dst + sg.dst + (i - sg.prefix), v);
            }
            c = end;
        }
    }
}


// Session epoch renumbering (session.cpp): read one cell per interval, and write a renumbered cell
// over every cell of an interval (all cells of an interval are equal).
__global__ void __launch_bounds__(THREADS)
gather_cells(const uint2* __restrict__ shadow, const uint64_t* __restrict__ at, uint64_t n, uint2* __restrict__ out) {
    for (uint64_t i = (uint64_t)blockIdx.x * THREADS + threadIdx.x; i < n; i += (uint64_t)gridDim.x * THREADS)
        out[i] = shadow[at[i]];
}

__global__ void __launch_bounds__(THREADS)
fill_cells(uint2* __restrict__ shadow, const CellFill* __restrict__ f, uint32_t nf, uint64_t total) {
    const int lane = threadIdx.x & 31;
    const uint64_t nwarps = (uint64_t)gridDim.x * WARPS;
    const uint64_t nchunks = (total + COPY_CHUNK - 1) / COPY_CHUNK;
    for (uint64_t ch = (uint64_t)blockIdx.x * WARPS + (threadIdx.x >> 5); ch < nchunks; ch += nwarps) {
        const uint64_t c0 = ch * COPY_CHUNK, c1 = min(c0 + COPY_CHUNK, total);
        uint32_t lo = 0, hi = nf;                         // last fill with prefix <= c0
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (f[mid].prefix <= c0) lo = mid; else hi = mid;
        }
        for (uint64_t c = c0; c < c1; lo++) {
            const CellFill x = f[lo];
            const uint64_t end = min(c1, x.prefix + x.len);
            const uint2 v = make_uint2(x.w, x.r);
            for (uint64_t i = c + lane; i < end; i += 32) __stcs(shadow + x.dst + (i - x.prefix), v);
            c = end;
        }
    }
}

}  // namespace

namespace cusan {

cudaError_t launch_gather_cells(uint32_t grid, cudaStream_t stream, const uint2* shadow, const uint64_t* at, uint64_t n,
                                uint2* out) {
    gather_cells<<<grid, THREADS, 0, stream>>>(shadow, at, n, out);
    return cudaGetLastError();
}

cudaError_t launch_fill_cells(uint32_t grid, cudaStream_t stream, uint2* shadow, const CellFill* f, uint32_t nf,
                              uint64_t total) {
    fill_cells<<<grid, THREADS, 0, stream>>>(shadow, f, nf, total);
    return cudaGetLastError();
}

// A compressed window runs the !TMA instantiation on a grid of its own occupancy (more blocks per
// SM); `grid` is the caller's for the TMA one, so only its range count matters there.
cudaError_t launch_shadow_check(uint32_t grid, cudaStream_t stream, const DSpan* spans, uint32_t nspans,
                                uint64_t tiles, uint64_t weight, const Ctx& k, unsigned long long* sched,
                                bool compressed) {
    if (compressed) {
        int max_blocks = 0;
        cudaError_t e = shadow_check_max_blocks(true, &max_blocks);
        if (e != cudaSuccess) return e;
        const uint64_t want = (tiles + WARPS - 1) / WARPS;
        const uint32_t g = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)max_blocks, want));
        shadow_check_window<false><<<g, THREADS, 0, stream>>>(spans, nspans, tiles, weight, k, sched);
    } else {
        shadow_check_window<true><<<grid, THREADS, DYN_SMEM, stream>>>(spans, nspans, tiles, weight, k, sched);
    }
    return cudaGetLastError();
}

cudaError_t launch_copy_cells(uint32_t grid, cudaStream_t stream, const uint2* src, uint2* dst,
                              const CopySeg* segs, uint32_t nseg, uint64_t total) {
    copy_cells<<<grid, THREADS, 0, stream>>>(src, dst, segs, nseg, total);
    return cudaGetLastError();
}

template <bool TMA>
static cudaError_t blocks_per_sm_query(int* per_sm) {
    const size_t dyn = TMA ? DYN_SMEM : 0;
    if (dyn) {
        cudaError_t e = cudaFuncSetAttribute(shadow_check_window<TMA>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)dyn);
        if (e != cudaSuccess) return e;
    }
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, shadow_check_window<TMA>, THREADS, dyn);
}

cudaError_t shadow_check_blocks_per_sm_query(int* per_sm) { return blocks_per_sm_query<true>(per_sm); }

// Once per device: setting a function attribute while that kernel runs waits for it, so a plan
// prepared on another host thread while a check runs (pipelined checks) would stall here.
cudaError_t shadow_check_blocks_per_sm(int* per_sm) {
    static std::atomic<int> known[256];
    int dev = 0;
    cudaError_t e0 = cudaGetDevice(&dev);
    if (e0 != cudaSuccess) return e0;
    if (dev >= 0 && dev < 256) {
        const int k = known[dev].load(std::memory_order_acquire);
        if (k > 0) {
            *per_sm = k;
            return cudaSuccess;
        }
    }
    cudaError_t e1 = shadow_check_blocks_per_sm_query(per_sm);
    if (e1 == cudaSuccess && dev >= 0 && dev < 256 && *per_sm > 0) known[dev].store(*per_sm, std::memory_order_release);
    return e1;
}

// Resident blocks of one K1 instantiation on the whole device (SMs × blocks per SM), cached.
cudaError_t shadow_check_max_blocks(bool compressed, int* max_blocks) {
    static std::atomic<int> known[2][256];
    int dev = 0;
    cudaError_t e0 = cudaGetDevice(&dev);
    if (e0 != cudaSuccess) return e0;
    const int c = compressed ? 1 : 0;
    if (dev >= 0 && dev < 256) {
        const int v = known[c][dev].load(std::memory_order_acquire);
        if (v > 0) {
            *max_blocks = v;
            return cudaSuccess;
        }
    }
    int sms = 0, per_sm = 0;
    cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (e != cudaSuccess) return e;
    e = compressed ? blocks_per_sm_query<false>(&per_sm) : shadow_check_blocks_per_sm(&per_sm);
    if (e != cudaSuccess) return e;
    *max_blocks = std::max(1, sms * per_sm);
    if (dev >= 0 && dev < 256) known[c][dev].store(*max_blocks, std::memory_order_release);
    return cudaSuccess;
}

}  // namespace cusan
