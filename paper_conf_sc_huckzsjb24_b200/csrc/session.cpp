// Incremental (online) sessions — SURVEY.md §8(f) f1.
#include <algorithm>
#include <bitset>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <new>
#include <string>
#include <unordered_map>

#include <cuda.h>

#include "kernel.cuh"

using namespace cusan;

// ================================================================================================
// Incremental sessions: CuSan checks while the program runs
// (PAPER.md:606-612); a session keeps the shadow on the device between calls and each call checks
// only the accesses appended since the previous one.
//
// The host plan is incremental too: the vector clocks, sync clocks and segment rows (a1) carry over
// between calls, and so does the layout (a2) — the elementary intervals seen so far, each with the
// set of fibers that read it since its last write.  A call processes only the new events: its
// accesses' endpoints split old intervals (a split piece inherits the state) or open new ones, the
// new incidences are grouped into windows and spans, and only new segment rows are uploaded.  Host
// cost per call is O(new events × fibers + intervals).
//
// On the device the layout is stable: a piece of a split interval keeps its cells where they are
// (the pieces of an interval are consecutive sub-ranges of it), memory touched for the first time
// gets new cells appended to the shadow, and the check updates the cells in place.  A call costs
// only the cells its accesses touch (the shadow grows in place, see Vmm below).  With the
// interval-compressed shadow (f3) an interval has one cell, so a split piece other than the first
// gets a new cell copied from it (copy_cells).  In-place updates cannot be re-run: if the run buffer
// overflows, the call's run list is marked truncated (race-granule counts stay exact) and the buffer
// grows for later calls.  Read-set records are assigned on the host (RecAlloc below: dead ones are
// reused), and event ids are renumbered when the trace outgrows the 24-bit epoch field
// (session_renumber).
// ================================================================================================
namespace {

constexpr uint32_t NO_SEG = 0xffffffffu;
constexpr uint64_t STAGE_MAX = 256 << 10;            // calls with more table bytes upload them directly

// ---- growable shadow in a reserved virtual range (CUDA virtual memory management) --------------
// The session reserves a virtual range as large as the device's memory once and maps physical
// chunks at its end as the shadow grows, so growth neither copies the cells nor needs room for two
// copies (a 70 GB shadow could not be re-allocated next to itself in 180 GB).  Driver entry points
// come from the runtime (no link against libcuda); if they are unavailable the shadow falls back to
// re-allocation with a copy.
struct Vmm {
    decltype(&cuMemAddressReserve) reserve = nullptr;
    decltype(&cuMemAddressFree) addr_free = nullptr;
    decltype(&cuMemCreate) create = nullptr;
    decltype(&cuMemMap) map = nullptr;
    decltype(&cuMemSetAccess) set_access = nullptr;
    decltype(&cuMemUnmap) unmap = nullptr;
    decltype(&cuMemRelease) release = nullptr;
    decltype(&cuMemGetAllocationGranularity) granularity = nullptr;
    bool ok = false;
};

const Vmm& vmm() {
    static const Vmm v = [] {
        Vmm r;
        auto get = [](const char* name, void** fn) {
            cudaDriverEntryPointQueryResult q;
            return cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q) == cudaSuccess &&
                   q == cudaDriverEntryPointSuccess && *fn;
        };
        r.ok = get("cuMemAddressReserve", (void**)&r.reserve) && get("cuMemAddressFree", (void**)&r.addr_free) &&
               get("cuMemCreate", (void**)&r.create) && get("cuMemMap", (void**)&r.map) &&
               get("cuMemSetAccess", (void**)&r.set_access) && get("cuMemUnmap", (void**)&r.unmap) &&
               get("cuMemRelease", (void**)&r.release) &&
               get("cuMemGetAllocationGranularity", (void**)&r.granularity);
        return r;
    }();
    return v;
}

struct VmRange {
    CUdeviceptr base = 0;
    size_t reserved = 0, mapped = 0, gran = 0;
    std::vector<std::pair<CUmemGenericAllocationHandle, size_t>> chunks;   // mapped back to back

    ~VmRange() {
        const Vmm& v = vmm();
        size_t off = 0;
        for (auto& c : chunks) {
            v.unmap(base + off, c.second);
            v.release(c.first);
            off += c.second;
        }
        if (base) v.addr_free(base, reserved);
    }
};

// A growable device buffer.  With VMM: a virtual range of `reserve` bytes (0 = the device's memory)
// whose end gets physical chunks mapped as it grows — the address and contents stay, nothing is
// copied or freed (cudaMalloc / cudaFree next to a tens-of-GB shadow cost up to 100s of ms).
// Without: cudaMalloc + copy of the kept prefix.  Contents past the kept prefix are undefined.
template <class T>
struct DevBuf {
    VmRange vr;
    T* p = nullptr;
    uint64_t cap = 0;             // elements
    uint64_t reserve = 0;         // bytes of virtual range
    bool vm = false;
    ~DevBuf() {
        if (!vm && p) cudaFree(p);
    }
};

}  // namespace

// make at least `bytes` of the range usable (maps one new chunk with 1/8 headroom); false = not
// possible (no VMM support, or out of memory)
static bool vm_grow(VmRange& r, int device, size_t bytes, size_t reserve = 0) {
    if (bytes <= r.mapped) return true;
    const Vmm& v = vmm();
    if (!v.ok) return false;
    CUmemAllocationProp prop{};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    prop.location.id = device;
    if (!r.base) {
        size_t free_b = 0, total_b = 0;
        if (v.granularity(&r.gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS ||
            cudaMemGetInfo(&free_b, &total_b) != cudaSuccess)
            return false;
        r.reserved = (std::max(reserve ? reserve : total_b, bytes) + r.gran - 1) / r.gran * r.gran;
        if (v.reserve(&r.base, r.reserved, 0, 0, 0) != CUDA_SUCCESS) {
            r.base = 0;
            return false;
        }
    }
    size_t want = bytes + bytes / 8;
    want = std::min(std::max(want, bytes), r.reserved);
    if (bytes > r.reserved) return false;
    const size_t sz = (want - r.mapped + r.gran - 1) / r.gran * r.gran;
    if (r.mapped + sz > r.reserved) return false;
    CUmemGenericAllocationHandle h;
    if (v.create(&h, sz, &prop, 0) != CUDA_SUCCESS) {
        release_parked_workspace(device);      // a one-shot check's parked workspace, then retry
        if (v.create(&h, sz, &prop, 0) != CUDA_SUCCESS) return false;
    }
    if (v.map(r.base + r.mapped, sz, 0, h, 0) != CUDA_SUCCESS) {
        v.release(h);
        return false;
    }
    CUmemAccessDesc acc{};
    acc.location = prop.location;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if (v.set_access(r.base + r.mapped, sz, &acc, 1) != CUDA_SUCCESS) {
        v.unmap(r.base + r.mapped, sz);
        v.release(h);
        return false;
    }
    r.chunks.push_back({h, sz});
    r.mapped += sz;
    return true;
}

namespace {

constexpr uint32_t NO_REC = 0xffffffffu;

// one elementary interval of the session's layout
struct SIv {
    uint64_t abs_begin, len, dense;
    std::bitset<CUSAN_MAX_FIBERS + 1> readers;   // fibers that read it since its last write
    uint32_t rec = NO_REC;                       // read-set record its cells name (>= 2 readers)
};

// Read-set records of a session, allocated on the host.  A record is written once, by the span
// that ends with its read set, and only read afterwards; it stays live while some interval's cells
// name it (pieces of a split interval share their parent's record).  After each call's plan the
// records no interval names any more are dead: they become reusable from the NEXT call's plan on —
// the current call's kernels may still read them, and the next call's kernels run after them on
// the same stream.  So the heap holds the live read sets (bounded by intervals × fibers) however
// long the session runs, instead of growing with every call.
struct RecAlloc {
    uint64_t hwm = 0;                                       // units ever handed out = heap size needed
    std::vector<std::vector<uint32_t>> free_by_units;       // reusable records by size (units)
    std::vector<std::pair<uint32_t, uint32_t>> pending;     // dead in the current call: (rec, units)
    std::vector<std::pair<uint32_t, uint32_t>> live;        // allocated: (rec, units)
    std::vector<uint32_t> stamp;                            // by record unit: last collect naming it
    uint32_t gen = 0;
    uint64_t live_units = 0;

    // a record of `units` units; false if the 24-bit record index is exhausted
    bool alloc(uint32_t units, uint32_t* rec) {
        if (units < free_by_units.size() && !free_by_units[units].empty()) {
            *rec = free_by_units[units].back();
            free_by_units[units].pop_back();
        } else {
            if (hwm + units >= (1ull << 24) - 1) return false;
            *rec = (uint32_t)hwm;
            hwm += units;
        }
        live.emplace_back(*rec, units);
        live_units += units;
        return true;
    }
    // records dead in the previous call become reusable (called when a call is planned)
    void promote() {
        for (const auto& d : pending) {
            if (free_by_units.size() <= d.second) free_by_units.resize(d.second + 1);
            free_by_units[d.second].push_back(d.first);
        }
        pending.clear();
    }
    // after a call's plan: every allocated record the layout no longer names is dead
    // (mark the named records with this collect's stamp, sweep the live list)
    template <class Layout>
    void collect(const Layout& ivs) {
        if (stamp.size() < hwm) stamp.resize(hwm, 0);
        if (++gen == 0) {                                   // stamp wrapped: clear and restart
            std::fill(stamp.begin(), stamp.end(), 0);
            gen = 1;
        }
        for (const auto& v : ivs)
            if (v.rec != NO_REC) stamp[v.rec] = gen;
        for (size_t i = 0; i < live.size();) {
            if (stamp[live[i].first] == gen) { i++; continue; }
            pending.push_back(live[i]);
            live_units -= live[i].second;
            live[i] = live.back();
            live.pop_back();
        }
    }
};

}  // namespace

struct PendingCall;

struct cusan_session {
    const cusan_trace* trace = nullptr;
    cusan_check_opts opts{};
    int device = 0, max_blocks = 0;
    cudaStream_t stream = nullptr;
    // ---- host state carried between calls ----
    uint32_t F = 1;                                 // clock width = the trace's max_fibers
    std::vector<uint32_t> C;                        // F × F fiber clocks
    KeySlots key_slot;
    std::vector<uint32_t> sc;                       // sync clocks, F per key
    std::vector<uint32_t> cur_seg;                  // open segment per fiber
    pinned_vector<uint32_t> segvc;                  // segment rows not uploaded yet: [seg_uploaded, nseg)
    uint32_t F_used = 1;                            // fibers seen so far: clock columns >= it are all 0
    uint64_t nseg = 0;
    std::vector<SIv> ivs;                           // layout of `shadow`
    std::vector<std::pair<uint64_t, uint64_t>> forget;   // granule ranges to drop after the next plan
    pinned_vector<char> stage;                      // a small call's tables, staged for one upload
    uint64_t used = 0;                              // cells of `shadow` in use
    uint64_t checked_access = 0, checked_events = 0, n_calls = 0;
    // epoch renumbering (sessions longer than the 24-bit epoch field, see session_renumber):
    // trace event i >= the last renumbering point has compact id i - delta; compact values
    // (id + 1) 1..orig->size()-1 name older events, orig[v] = their trace value (event id + 1)
    uint64_t delta = 0;
    std::shared_ptr<const std::vector<uint32_t>> orig = std::make_shared<const std::vector<uint32_t>>(1, 0u);
    uint64_t limit = CUSAN_MAX_EVENTS;              // compact ids stay below this (CUSAN_SESSION_EVENT_LIMIT)
    uint64_t renumberings = 0;
    uint32_t blk_log2 = 21;                         // block-cyclic shard map (nshards > 1)
    bool broken = false;                            // a call failed after changing the state
    // ---- device state (every buffer grows in place, see DevBuf) ----
    DevBuf<uint2> shadow;                           // cells
    DevBuf<uint32_t> segvc_d;                       // segment rows, u32 words
    uint64_t seg_uploaded = 0;                      // rows on the device
    DevBuf<uint32_t> heap;                          // read-set records, u32 words
    RecAlloc recs;                                  // which records are live / reusable
    DevBuf<char> scratch;                           // one call's tables and counters
    DevBuf<cusan_race_run> runs;                    // raw runs of one call
    DevBuf<char> merge_buf;                         // a4 scratch
    RunMerge merge;                                 // views merge_buf
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    std::unique_ptr<PendingCall> pending;           // a submitted call not collected yet

    ~cusan_session();
    uint64_t heap_cap() const { return std::min<uint64_t>(heap.cap / REC_WORDS, (1ull << 24) - 1); }

    uint32_t* sync_clock(uint64_t key) {
        bool fresh;
        const uint32_t slot = key_slot.get(key, &fresh);
        if (fresh) sc.resize(sc.size() + F, 0);
        return &sc[(size_t)slot * F];
    }
};

// grow a buffer to at least `need` elements keeping the first `keep` (see DevBuf)
template <class T>
static int grow_buf(cusan_session* s, DevBuf<T>& b, uint64_t need, uint64_t keep, const char* what) {
    if (b.cap >= need && b.p) return CUSAN_OK;
    need = std::max<uint64_t>(need, 1);
    if (b.vm || (!b.p && vmm().ok)) {
        if (vm_grow(b.vr, s->device, need * sizeof(T), b.reserve)) {
            b.vm = true;
            b.p = (T*)b.vr.base;
            b.cap = b.vr.mapped / sizeof(T);
            return CUSAN_OK;
        }
        if (b.vm) return fail(CUSAN_ENOMEM, std::string("cannot map more device memory for ") + what);
    }
    const uint64_t n = std::max<uint64_t>(need + need / 8, 64);
    T* np = nullptr;
    if (cudaMalloc((void**)&np, n * sizeof(T)) != cudaSuccess)
        return fail(CUSAN_ENOMEM, std::string("cannot allocate ") + what);
    cudaError_t e = cudaSuccess;
    if (b.p && keep) e = cudaMemcpyAsync(np, b.p, std::min(keep, b.cap) * sizeof(T), cudaMemcpyDeviceToDevice, s->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s->stream);
    if (e != cudaSuccess) {
        cudaFree(np);
        return cuda_fail(e, what);
    }
    cudaFree(b.p);
    b.p = np;
    b.cap = n;
    return CUSAN_OK;
}

// grow the heap keeping every record handed out so far
static int grow_heap(cusan_session* s, uint64_t need_units) {
    if (s->heap_cap() >= need_units && s->heap.p) return CUSAN_OK;
    need_units = std::min<uint64_t>(need_units, (1ull << 24) - 1);
    return grow_buf(s, s->heap, need_units * REC_WORDS, s->recs.hwm * REC_WORDS, "the read-set heap");
}

// run buffer for `n` raw runs and the a4 scratch to merge them
static int grow_runs(cusan_session* s, uint64_t n) {
    if (int st = grow_buf(s, s->runs, n, 0, "the run buffer")) return st;
    uint64_t mb = 0;
    if (int st = merge_scratch_bytes(s->runs.cap, &mb)) return st;
    if (int st = grow_buf(s, s->merge_buf, mb, 0, "the run merge scratch")) return st;
    if (!s->merge.own) {
        s->merge.buf = s->merge_buf.p;
        s->merge.cap = s->merge_buf.cap;
    }
    return CUSAN_OK;
}

// The incremental host plan of one call (a1 + a2 for the new events).
struct CallPlan {
    std::vector<uint64_t> g0, g1;                   // new accesses (granule ranges)
    std::vector<AccRec> rec;
    std::vector<SIv> ivs;                           // new layout
    std::vector<char> has_state;                    // per new interval: covered before this call
    std::vector<uint32_t> inc_off, inc_cnt;         // per new interval: new incidences (CSR)
    pinned_vector<AccRec> inc;                      // uploaded
    std::vector<uint32_t> inc_acc;                  // call-local access index of each incidence
    HostPlan hp;                                    // spans, windows and counters for the launches
    std::vector<CopySeg> segs;                      // cells to copy (compressed split pieces)
    uint64_t copy_cells = 0, used = 0, tracked = 0; // used: shadow cells in use after the call
};

static int plan_call(cusan_session* s, const Trace& tr, CallPlan& cp) {
    static const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    const auto t0 = std::chrono::steady_clock::now();
    auto tick = [&](const char* what) {
        if (dbg)
            std::fprintf(stderr, "plan_call: %-10s %8.3f ms\n", what,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    };
    const uint32_t F = s->F;
    cusan_counters& c = cp.hp.ctr;
    c = cusan_counters{};
    c.n_fibers = F;
    s->recs.promote();                 // records dead since the previous call's plan are free now
    // ---- a1: clocks and segments for the new events (build_host_plan's pass, resumed) ----------
    if (tr.ev.size() - s->delta > s->limit)
        return fail(CUSAN_ERANGE, "one session call holds more events than the 24-bit epoch field can number");
    for (uint64_t i = s->checked_events; i < tr.ev.size(); i++) {
        const cusan_event& e = tr.ev[i];
        const uint32_t f = e.fiber;
        uint32_t* Cf = &s->C[(size_t)f * F];
        const uint32_t ci = (uint32_t)(i - s->delta);       // compact event id (= i before any renumbering)
        c.n_events++;
        // clock columns of fibers never seen are 0 everywhere: the joins stop at the fibers seen
        s->F_used = std::max(s->F_used, f + 1);
        if (e.kind == CUSAN_EV_FORK) s->F_used = std::max(s->F_used, (uint32_t)e.a + 1);
        const uint32_t FU = s->F_used;
        if (e.kind == CUSAN_EV_FORK) {
            const uint32_t src = (uint32_t)e.a;
            uint32_t* Cs = &s->C[(size_t)src * F];
            Cs[src] = ci + 1;
            for (uint32_t g = 0; g < FU; g++) Cf[g] = std::max(Cf[g], Cs[g]);
            s->cur_seg[f] = NO_SEG;
            c.n_fork++;
            continue;
        }
        Cf[f] = ci + 1;
        switch (e.kind) {
            case CUSAN_EV_ACCESS: {
                if (s->cur_seg[f] == NO_SEG) {
                    if (s->nseg >= 0x7fffffffu) return fail(CUSAN_ERANGE, "too many segments");
                    s->cur_seg[f] = (uint32_t)s->nseg++;
                    s->segvc.insert(s->segvc.end(), Cf, Cf + F);
                }
                const uint64_t g0 = e.a >> 3, g1 = e.b ? (e.a + e.b + 7) >> 3 : g0;
                cp.g0.push_back(g0);
                cp.g1.push_back(g1);
                cp.rec.push_back({pack_epoch(f, ci), s->cur_seg[f] | ((uint32_t)e.mode << 31)});
                const uint64_t bytes = 8 * (g1 - g0);
                c.n_access++;
                cp.tracked += bytes;
                if (e.mode) { c.n_write++; c.bytes_written += bytes; }
                else { c.n_read++; c.bytes_read += bytes; }
                break;
            }
            case CUSAN_EV_RELEASE: {
                uint32_t* S = s->sync_clock(e.a);
                for (uint32_t g = 0; g < FU; g++) S[g] = std::max(S[g], Cf[g]);
                c.n_release++;
                break;
            }
            case CUSAN_EV_RELEASE_STORE: {
                uint32_t* S = s->sync_clock(e.a);
                std::copy(Cf, Cf + FU, S);
                c.n_release_store++;
                break;
            }
            case CUSAN_EV_ACQUIRE: {
                uint32_t* S = s->sync_clock(e.a);
                for (uint32_t g = 0; g < FU; g++) Cf[g] = std::max(Cf[g], S[g]);
                s->cur_seg[f] = NO_SEG;
                c.n_acquire++;
                break;
            }
            default:
                return fail(CUSAN_EINVAL, "bad event kind in trace");
        }
    }
    c.tracked_bytes = cp.tracked;
    c.n_segments = s->nseg;
    tick("a1");

    // ---- a2: refine the layout by the new endpoints -----------------------------------------------
    const uint64_t n_new = cp.g0.size();
    std::vector<uint64_t> E;
    E.reserve(2 * n_new);
    // with shards, every block edge inside a new access is a boundary too, so each new elementary
    // interval lies in one block and belongs to one shard (old intervals are this shard's already)
    const int nsh = s->opts.nshards;
    const uint32_t L = s->blk_log2;
    for (uint64_t k = 0; k < n_new; k++)
        if (cp.g1[k] > cp.g0[k]) {
            E.push_back(cp.g0[k]);
            E.push_back(cp.g1[k]);
            if (nsh > 1)
                for (uint64_t b = ((cp.g0[k] >> L) + 1) << L; b < cp.g1[k]; b += 1ull << L) E.push_back(b);
        }
    std::sort(E.begin(), E.end());
    E.erase(std::unique(E.begin(), E.end()), E.end());
    // P = the old intervals' endpoints (already in order: the layout is sorted and disjoint) merged
    // with the new ones — linear in the layout, so a small call does not re-sort the whole layout
    std::vector<uint64_t> P;
    P.reserve(E.size() + 2 * s->ivs.size());
    {
        size_t e = 0;
        auto put = [&](uint64_t x) {
            for (; e < E.size() && E[e] < x; e++)
                if (P.empty() || P.back() != E[e]) P.push_back(E[e]);
            if (P.empty() || P.back() != x) P.push_back(x);
        };
        for (const SIv& u : s->ivs) {
            put(u.abs_begin);
            put(u.abs_begin + u.len);
        }
        for (; e < E.size(); e++)
            if (P.empty() || P.back() != E[e]) P.push_back(E[e]);
    }
    const uint64_t np = P.size();
    std::vector<int64_t> diff(np + 1, 0);
    std::vector<uint32_t> b0(n_new, 0), b1(n_new, 0);
    for (uint64_t k = 0; k < n_new; k++) {
        if (cp.g1[k] <= cp.g0[k]) continue;
        b0[k] = (uint32_t)(std::lower_bound(P.begin(), P.end(), cp.g0[k]) - P.begin());
        b1[k] = (uint32_t)(std::lower_bound(P.begin(), P.end(), cp.g1[k]) - P.begin());
        diff[b0[k]]++;
        diff[b1[k]]--;
    }
    const bool compressed = compressed_shadow(s->opts);
    std::vector<uint32_t> iv_of(np ? np - 1 : 0, 0xffffffffu);
    uint64_t used = s->used;
    cp.ivs.reserve(np);
    cp.has_state.reserve(np);
    {
        int64_t cov = 0;
        size_t u = 0;
        for (uint64_t j = 0; j + 1 < np; j++) {
            cov += diff[j];
            while (u < s->ivs.size() && s->ivs[u].abs_begin + s->ivs[u].len <= P[j]) u++;
            const bool old = u < s->ivs.size() && s->ivs[u].abs_begin <= P[j];
            if (cov <= 0 && !old) continue;
            if (!old && nsh > 1 && (int)((P[j] >> L) % (uint64_t)nsh) != s->opts.shard) continue;   // another shard's
            SIv v;
            v.abs_begin = P[j];
            v.len = P[j + 1] - P[j];
            if (old) {                 // a piece of an old interval: its state, its cells in place
                const SIv& o = s->ivs[u];
                v.readers = o.readers;
                v.rec = o.rec;
                if (!compressed) {
                    v.dense = o.dense + (P[j] - o.abs_begin);
                } else if (P[j] == o.abs_begin) {
                    v.dense = o.dense;
                } else {               // compressed: a further piece gets a copy of the one cell
                    v.dense = used++;
                    cp.segs.push_back({cp.copy_cells, o.dense, v.dense, 1});
                    cp.copy_cells++;
                }
            } else {                   // memory touched for the first time: new cells at the end
                if (compressed) {
                    v.dense = used++;
                } else {
                    v.dense = (used + CELL_ALIGN - 1) / CELL_ALIGN * CELL_ALIGN;
                    used = v.dense + v.len;
                }
            }
            iv_of[j] = (uint32_t)cp.ivs.size();
            cp.ivs.push_back(v);
            cp.has_state.push_back(old ? 1 : 0);
        }
    }
    cp.used = used;
    tick("layout");
    const size_t niv = cp.ivs.size();
    c.n_intervals = niv;
    // new incidences per interval, in trace order
    cp.inc_cnt.assign(niv, 0);
    for (uint64_t k = 0; k < n_new; k++)
        for (uint32_t j = b0[k]; j < b1[k]; j++)
            if (iv_of[j] != 0xffffffffu) cp.inc_cnt[iv_of[j]]++;
    cp.inc_off.assign(niv, 0);
    uint64_t n_inc = 0;
    for (size_t i = 0; i < niv; i++) {
        cp.inc_off[i] = (uint32_t)n_inc;
        n_inc += cp.inc_cnt[i];
    }
    if (n_inc > 0xffffffffull) return fail(CUSAN_ERANGE, "too many interval incidences");
    c.n_incidences = n_inc;
    tick("incid cnt");
    cp.inc.resize(n_inc);
    cp.inc_acc.resize(n_inc);
    {
        std::vector<uint32_t> at(cp.inc_off);
        for (uint64_t k = 0; k < n_new; k++)
            for (uint32_t j = b0[k]; j < b1[k]; j++) {
                if (iv_of[j] == 0xffffffffu) continue;
                const uint32_t q = at[iv_of[j]]++;
                cp.inc[q] = cp.rec[k];
                cp.inc_acc[q] = (uint32_t)k;
            }
    }
    uint64_t granules = 0, tracked_shard = 0;
    for (size_t i = 0; i < niv; i++) {
        granules += cp.ivs[i].len;
        tracked_shard += 8 * cp.ivs[i].len * cp.inc_cnt[i];
    }
    c.shard_granules = granules;
    c.tracked_bytes_shard = tracked_shard;

    tick("incidences");
    // ---- windows and spans for the new incidences; moves for the untouched intervals ---------------
    const uint64_t W = s->opts.window_events > 0 ? (uint64_t)s->opts.window_events : std::max<uint64_t>(n_new, 1);
    const uint64_t nwin = n_new ? (n_new + W - 1) / W : 0;
    std::vector<std::pair<uint64_t, Span>> out;
    for (size_t i = 0; i < niv; i++) {
        SIv& v = cp.ivs[i];
        const bool has_state = cp.has_state[i];
        const uint32_t qa = cp.inc_off[i], qe = qa + cp.inc_cnt[i];
        if (qa == qe) continue;                      // untouched: its cells stay where they are
        for (uint32_t q = qa; q < qe;) {
            const uint64_t w = cp.inc_acc[q] / W;
            uint32_t q2 = q;
            while (q2 < qe && cp.inc_acc[q2] / W == w) {
                const AccRec& r = cp.inc[q2];
                if (r.segm >> 31) v.readers.reset();
                else v.readers.set(r.epoch >> 24);
                q2++;
            }
            Span sp{};
            sp.abs_begin = v.abs_begin;
            sp.dense_begin = v.dense;
            sp.len = v.len;
            sp.list_off = q;
            sp.list_cnt = q2 - q;
            const bool first_span = q == qa;
            sp.flags = ((!first_span || has_state) ? SPAN_LOAD : 0u) | SPAN_STORE |
                       (first_span ? SPAN_FIRST_IN_CALL : 0u) | (compressed ? SPAN_COMPRESSED : 0u);
            const uint64_t nr = v.readers.count();
            v.rec = NO_REC;                         // the span's store replaces the cells' R
            if (nr >= 2) {
                sp.rec_units = (uint32_t)((nr + 1 + REC_WORDS - 1) / REC_WORDS);
                if (!s->recs.alloc(sp.rec_units, &sp.rec))
                    return fail(CUSAN_ERANGE, "live read-set records exceed the 24-bit record index");
                v.rec = sp.rec;
            }
            out.emplace_back(w, sp);
            q = q2;
        }
    }
    // window-major (stable by interval), records numbered from 0 (the heap top at launch is added)
    std::vector<uint64_t> wstart(nwin + 1, 0);
    for (const auto& ws : out) wstart[ws.first + 1]++;
    for (uint64_t w = 0; w < nwin; w++) wstart[w + 1] += wstart[w];
    HostPlan& hp = cp.hp;
    hp.spans.assign(out.size(), Span{});
    {
        std::vector<uint64_t> at(wstart.begin(), wstart.end() - 1);
        for (const auto& ws : out) hp.spans[at[ws.first]++] = ws.second;
    }
    hp.rec_units = 0;
    hp.spill_spans = 0;
    for (Span& sp : hp.spans)
        if (sp.rec_units) {
            hp.rec_units += sp.rec_units;
            hp.spill_spans++;
        }
    hp.win_span_off.assign(1, 0);
    for (uint64_t w = 0; w < nwin; w++)
        if (wstart[w + 1] > wstart[w]) hp.win_span_off.push_back(wstart[w + 1]);
    hp.F = F;
    hp.window_accesses = W;
    c.n_windows = hp.win_span_off.size() - 1;
    c.n_spans = hp.spans.size();
    c.spill_spans = hp.spill_spans;
    c.spill_heap_bytes = hp.rec_units * REC_WORDS * 4;
    tick("spans");
    if (!s->forget.empty()) {          // cusan_session_forget: released memory leaves the layout
        std::vector<std::pair<uint64_t, uint64_t>>& fg = s->forget;
        std::sort(fg.begin(), fg.end());
        size_t keep = 0, r = 0;
        uint64_t reach = 0;            // furthest end of the ranges starting at or before the interval
        for (size_t i = 0; i < cp.ivs.size(); i++) {
            const SIv& v = cp.ivs[i];
            while (r < fg.size() && fg[r].first <= v.abs_begin) reach = std::max(reach, fg[r++].second);
            if (reach >= v.abs_begin + v.len) continue;          // wholly inside a released range
            if (keep != i) cp.ivs[keep] = cp.ivs[i];
            keep++;
        }
        cp.ivs.resize(keep);
        fg.clear();
        c.n_intervals = keep;
    }
    s->recs.collect(cp.ivs);           // records no interval of the new layout names are dead
    tick("collect");
    c.heap_live_bytes = s->recs.live_units * REC_WORDS * 4;
    c.heap_bytes = s->recs.hwm * REC_WORDS * 4;
    return CUSAN_OK;
}

// A call launched by cusan_session_submit and not collected yet.  Its host tables stay here until
// the call completes: their uploads are asynchronous DMA transfers from page-locked memory.
struct PendingCall {
    CallPlan cp;
    SpanTables tabs;
    pinned_vector<uint32_t> seg_rows;               // segment rows new in this call (staged)
    uint64_t seg_first_word = 0;                    // where they go in segvc_d
    uint64_t used_before = 0;                       // shadow cells in use before the call
    pinned_vector<unsigned long long> init, cnt;    // counter initial values / read-back
    pinned_vector<CopySeg> segs_pinned;             // cell copies, page-locked (large calls)
    uint64_t h2d = 0;
    uint64_t delta = 0;                             // event numbering the call was planned with
    std::shared_ptr<const std::vector<uint32_t>> orig;
    std::chrono::steady_clock::time_point t_start;
};

cusan_session::~cusan_session() {
    if (ev0) cudaEventDestroy(ev0);
    if (ev1) cudaEventDestroy(ev1);
}

static void session_tick(const PendingCall& pc, const char* what) {
    static const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    if (dbg)
        std::fprintf(stderr, "cusan_session: %-10s %8.3f ms\n", what,
                     std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - pc.t_start).count());
}

// Host part of a call: the incremental a1 + a2 of the events appended since the previous call.
// The session's host state (clocks, layout, counts) moves on at once, so the next call can be
// planned while this one runs on the device; only the read-set heap top waits for the device
// (record numbers are relative until launch).
static int session_plan(cusan_session* s, PendingCall& pc) {
    const Trace& tr = s->trace->t;
    if (tr.ev.size() < s->checked_events) return fail(CUSAN_ESTATE, "the trace shrank");
    s->broken = true;                  // cleared once the call is launched
    CallPlan& cp = pc.cp;
    int st;
    try {
        st = plan_call(s, tr, cp);
        if (!st) {
            build_span_tables(cp.hp, s->max_blocks, pc.tabs);
            pc.seg_first_word = s->seg_uploaded * s->F;   // the rows new in this call move to the call
            pc.seg_rows.swap(s->segvc);
            s->segvc.clear();
        }
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while planning");
    }
    if (st) return st;
    session_tick(pc, "plan");
    pc.delta = s->delta;
    pc.orig = s->orig;
    // the new layout becomes the session's
    pc.used_before = s->used;
    s->ivs.swap(cp.ivs);
    s->used = cp.used;
    s->seg_uploaded = s->nseg;
    s->checked_access += cp.g0.size();
    s->checked_events = tr.ev.size();
    s->n_calls++;
    return CUSAN_OK;
}

// Device part, asynchronous: buffers, uploads, the check launches and the counter read-back are
// queued on the session's stream (a4's merge happens in session_finish).
static int session_launch(cusan_session* s, PendingCall& pc) {
    CallPlan& cp = pc.cp;
    SpanTables& tabs = pc.tabs;
    // the shadow grows as new memory is touched: new chunks mapped in place, else re-allocated
    // with its cells moved (1/8 headroom either way)
    int st;
    if ((st = grow_buf(s, s->shadow, cp.used, pc.used_before, "the shadow"))) return st;
    if ((st = grow_heap(s, s->recs.hwm + (s->recs.hwm >> 3) + 1024))) return st;
    uint64_t tiles = 0;                 // raw-run bound heuristic, as in plans (an overflow truncates)
    for (const Window& w : tabs.wins) tiles += w.tiles;
    if ((st = grow_runs(s, 2 * tiles + 1024))) return st;
    const uint64_t seg_words = pc.seg_first_word + pc.seg_rows.size();
    if ((st = grow_buf(s, s->segvc_d, seg_words, pc.seg_first_word, "segment rows"))) return st;
    if (!pc.seg_rows.empty())                        // only the rows new since the last call
        CK(cudaMemcpyAsync(s->segvc_d.p + pc.seg_first_word, pc.seg_rows.data(), pc.seg_rows.size() * sizeof(uint32_t),
                           cudaMemcpyHostToDevice, s->stream));
    const uint64_t nwin = tabs.wins.size();
    uint64_t off = 0;
    const uint64_t o_inc = off;   off = align_up(off + cp.inc.size() * sizeof(AccRec));
    const uint64_t o_spans = off; off = align_up(off + tabs.ds.size() * sizeof(DSpan));
    const uint64_t o_copy = off;  off = align_up(off + cp.segs.size() * sizeof(CopySeg));
    const uint64_t o_cnt = off;   off = align_up(off + (N_COUNTERS + nwin) * sizeof(unsigned long long));
    if ((st = grow_buf(s, s->scratch, off, 0, "plan tables"))) return st;
    AccRec* d_inc = (AccRec*)(s->scratch.p + o_inc);
    DSpan* d_spans = (DSpan*)(s->scratch.p + o_spans);
    CopySeg* d_copy = (CopySeg*)(s->scratch.p + o_copy);
    unsigned long long* d_cnt = (unsigned long long*)(s->scratch.p + o_cnt);
    pc.init.assign(N_COUNTERS + nwin, 0ull);
    pc.cnt.assign(N_COUNTERS, 0ull);
    pc.init[C_HEAP] = s->heap_cap();     // records are host-assigned: no device allocation
    if (off <= STAGE_MAX) {
        // a small call's tables and the counters' initial values go up in ONE transfer, staged in
        // the session's page-locked buffer laid out as the scratch is (its latency is mostly
        // per-copy cost).  The buffer is free again: the previous call finished before this launch.
        if (s->stage.size() < off) s->stage.resize(STAGE_MAX);
        auto put = [&](uint64_t at, const void* src, size_t bytes) {
            if (bytes) std::memcpy(s->stage.data() + at, src, bytes);
        };
        put(o_inc, cp.inc.data(), cp.inc.size() * sizeof(AccRec));
        put(o_spans, tabs.ds.data(), tabs.ds.size() * sizeof(DSpan));
        put(o_copy, cp.segs.data(), cp.segs.size() * sizeof(CopySeg));
        put(o_cnt, pc.init.data(), pc.init.size() * sizeof(unsigned long long));
        CK(cudaMemcpyAsync(s->scratch.p, s->stage.data(), off, cudaMemcpyHostToDevice, s->stream));
    } else {                             // large tables: straight from their page-locked vectors
        pc.segs_pinned.assign(cp.segs.begin(), cp.segs.end());
        CK(cudaMemcpyAsync(d_inc, cp.inc.data(), cp.inc.size() * sizeof(AccRec), cudaMemcpyHostToDevice, s->stream));
        CK(cudaMemcpyAsync(d_spans, tabs.ds.data(), tabs.ds.size() * sizeof(DSpan), cudaMemcpyHostToDevice,
                           s->stream));
        CK(cudaMemcpyAsync(d_copy, pc.segs_pinned.data(), pc.segs_pinned.size() * sizeof(CopySeg),
                           cudaMemcpyHostToDevice, s->stream));
        CK(cudaMemcpyAsync(d_cnt, pc.init.data(), pc.init.size() * sizeof(unsigned long long), cudaMemcpyHostToDevice,
                           s->stream));
    }
    pc.h2d = cp.inc.size() * sizeof(AccRec) + tabs.ds.size() * sizeof(DSpan) + cp.segs.size() * sizeof(CopySeg) +
             pc.seg_rows.size() * sizeof(uint32_t);
    session_tick(pc, "memory");

    // ---- a3, in place ------------------------------------------------------------------------------
    CK(cudaEventRecord(s->ev0, s->stream));
    if (cp.copy_cells)
        CK(launch_copy_cells(s->max_blocks, s->stream, s->shadow.p, s->shadow.p, d_copy, (uint32_t)cp.segs.size(),
                             cp.copy_cells));
    Ctx k;
    k.inc = d_inc;
    k.segvc = s->segvc_d.p;
    k.F = s->F;
    k.shadow = s->shadow.p;
    k.heap = s->heap.p;
    k.heap_cap = s->heap_cap();
    k.runs = s->runs.p;
    k.counters = d_cnt;
    k.run_cap = s->runs.cap;
    for (size_t i = 0; i < nwin; i++) {
        const Window& w = tabs.wins[i];
        unsigned long long* sched = CUSAN_DYNAMIC ? d_cnt + N_COUNTERS + i : nullptr;
        CK(launch_shadow_check(w.grid, s->stream, d_spans + w.span_off, w.nspans, w.tiles, w.weight, k, sched,
                               compressed_shadow(s->opts)));
    }
    CK(cudaEventRecord(s->ev1, s->stream));
    CK(cudaMemcpyAsync(pc.cnt.data(), d_cnt, N_COUNTERS * sizeof(unsigned long long), cudaMemcpyDeviceToHost,
                       s->stream));
    return CUSAN_OK;
}

// Wait for a launched call, merge its runs on the device (a4) and build its report (a5).
static int session_finish(cusan_session* s, PendingCall& pc, cusan_report** out) {
    CK(cudaStreamSynchronize(s->stream));
    session_tick(pc, "check");
    const CallPlan& cp = pc.cp;
    const uint64_t* cnt = (const uint64_t*)pc.cnt.data();
    float kms = 0.f;
    CK(cudaEventElapsedTime(&kms, s->ev0, s->ev1));
    if (cnt[C_HEAP_OVF] || cnt[C_INVARIANT]) {
        s->broken = true;
        return fail(CUSAN_ESTATE, "internal error: a read set outgrew its record or cells of one interval "
                                  "differ; the session's state is lost");
    }
    const bool runs_ovf = cnt[C_RUNS] > s->runs.cap;
    const uint64_t kept_runs = std::min<uint64_t>(cnt[C_RUNS], s->runs.cap);
    cusan_report* r = new (std::nothrow) cusan_report;
    if (!r) return fail(CUSAN_ENOMEM, "cannot allocate report");
    uint64_t d2h = N_COUNTERS * sizeof(unsigned long long);
    const int mst = merge_runs_device(s->merge, s->stream, s->runs.p, kept_runs, r->runs, &d2h);   // a4
    session_tick(pc, "merge");
    if (mst) {
        delete r;
        return mst;
    }
    if (pc.orig->size() > 1) {          // compact ids -> trace positions (monotone: order is kept)
        const std::vector<uint32_t>& orig = *pc.orig;
        auto to_trace = [&](uint32_t id) -> uint32_t {
            const uint64_t v = (uint64_t)id + 1;
            return v < orig.size() ? orig[v] - 1 : (uint32_t)(id + pc.delta);
        };
        for (cusan_race_run& x : r->runs) {
            x.earlier = to_trace(x.earlier);
            x.later = to_trace(x.later);
        }
    }
    r->n_runs = r->runs.size();
    r->n_race_granules = cnt[C_RACE];   // exact even when the run list overflowed
    if (runs_ovf) r->truncated = 1;     // the shadow moved on; the call cannot be re-run
    if (s->opts.max_runs && r->runs.size() > s->opts.max_runs) {
        r->runs.resize(s->opts.max_runs);
        r->truncated = 1;
    }
    r->ctr = cp.hp.ctr;
    r->ctr.raw_runs = cnt[C_RUNS];
    r->ctr.kernel_ms = kms;
    r->ctr.kernel_launches = pc.tabs.wins.size() + (cp.copy_cells ? 1 : 0) + (kept_runs ? MERGE_LAUNCHES : 0);
    r->ctr.shadow_cell_bytes = pc.tabs.cell_bytes + 16 * cp.copy_cells;
    r->ctr.shadow_bytes = cp.used * sizeof(uint2);
    r->ctr.h2d_bytes = pc.h2d + pc.init.size() * sizeof(unsigned long long);
    r->ctr.d2h_bytes = d2h;
    r->ctr.renumberings = s->renumberings;
    r->ctr.run_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - pc.t_start).count();
    *out = r;
    // a run list that overflowed is sized for the next call (best effort: this call succeeded)
    if (runs_ovf) grow_runs(s, cnt[C_RUNS] + cnt[C_RUNS] / 8 + 1024);
    return CUSAN_OK;
}

// Epoch renumbering.  Shadow cells, read-set records and clocks hold event ids + 1 in 24 bits, so a
// session whose trace outgrows 2^24-2 events renumbers, between two calls, every id value still in
// use: the values in live cells and live records, and every entry of the fiber and sync clocks
// (which are all future clock entries derive from).  Sorted and ranked, each value v becomes
// rank(v) in 1..n: injective and monotone on that set, so every later happens-before comparison
// (an earlier epoch's value against a clock entry of its fiber) and every order
// between ids comes out as before.  Later events continue above n (compact id = trace id - delta)
// and reports translate ids back to trace positions (orig[] for the renumbered values).  The
// segment rows of earlier calls are never read again, so segments restart from 0.
static int session_renumber(cusan_session* s) {
    CK(cudaStreamSynchronize(s->stream));
    const size_t niv = s->ivs.size();
    const bool compressed = compressed_shadow(s->opts);
    // one cell per interval (all cells of an interval are equal) and the heap's records
    std::vector<uint2> cells(niv);
    if (niv) {
        if (int st = grow_buf(s, s->scratch, 16 * niv + 512, 0, "plan tables")) return st;
        std::vector<uint64_t> at(niv);
        for (size_t i = 0; i < niv; i++) at[i] = s->ivs[i].dense;
        uint64_t* d_at = (uint64_t*)s->scratch.p;
        uint2* d_out = (uint2*)(s->scratch.p + align_up(8 * niv));
        CK(cudaMemcpyAsync(d_at, at.data(), 8 * niv, cudaMemcpyHostToDevice, s->stream));
        CK(launch_gather_cells(std::max(1, std::min(s->max_blocks, (int)((niv + THREADS - 1) / THREADS))), s->stream,
                               s->shadow.p, d_at, niv, d_out));
        CK(cudaMemcpyAsync(cells.data(), d_out, 8 * niv, cudaMemcpyDeviceToHost, s->stream));
    }
    std::vector<uint32_t> heap(s->recs.hwm * REC_WORDS);
    if (!heap.empty())
        CK(cudaMemcpyAsync(heap.data(), s->heap.p, heap.size() * 4, cudaMemcpyDeviceToHost, s->stream));
    CK(cudaStreamSynchronize(s->stream));
    // the id values in use
    auto is_spill = [](uint32_t e) { return (e >> 24) == 0xFFu; };
    std::vector<uint32_t> vals;
    vals.reserve(2 * niv + s->C.size() + s->sc.size());
    auto add_epoch = [&](uint32_t e) { if (e & 0xffffffu) vals.push_back(e & 0xffffffu); };
    for (const uint2& c : cells) {
        add_epoch(c.x);
        if (!is_spill(c.y)) add_epoch(c.y);
    }
    for (const auto& rec : s->recs.live) {
        const uint32_t* r = &heap[(size_t)rec.first * REC_WORDS];
        for (uint32_t j = 0; j < (r[0] & 0xffffu); j++) add_epoch(r[1 + j]);
    }
    for (uint32_t v : s->C) if (v) vals.push_back(v);
    for (uint32_t v : s->sc) if (v) vals.push_back(v);
    std::sort(vals.begin(), vals.end());
    vals.erase(std::unique(vals.begin(), vals.end()), vals.end());
    if (vals.size() + 1 >= s->limit / 2)
        return fail(CUSAN_ERANGE, "too many live event ids to renumber into the 24-bit epoch field");
    auto rank = [&](uint32_t v) -> uint32_t {
        return v ? 1u + (uint32_t)(std::lower_bound(vals.begin(), vals.end(), v) - vals.begin()) : 0u;
    };
    auto remap = [&](uint32_t e) -> uint32_t { return e ? (e & 0xff000000u) | rank(e & 0xffffffu) : 0u; };
    // rewrite: cells (one fill per interval), live records, clocks
    std::vector<CellFill> fills(niv);
    uint64_t total = 0;
    for (size_t i = 0; i < niv; i++) {
        const uint2 c = cells[i];
        fills[i] = CellFill{total, s->ivs[i].dense, compressed ? 1 : s->ivs[i].len, remap(c.x),
                            is_spill(c.y) ? c.y : remap(c.y)};
        total += fills[i].len;
    }
    for (const auto& rec : s->recs.live) {
        uint32_t* r = &heap[(size_t)rec.first * REC_WORDS];
        for (uint32_t j = 0; j < (r[0] & 0xffffu); j++) r[1 + j] = remap(r[1 + j]);
    }
    for (uint32_t& v : s->C) v = rank(v);
    for (uint32_t& v : s->sc) v = rank(v);
    if (niv) {
        if (int st = grow_buf(s, s->scratch, sizeof(CellFill) * niv + 256, 0, "plan tables")) return st;
        CK(cudaMemcpyAsync(s->scratch.p, fills.data(), sizeof(CellFill) * niv, cudaMemcpyHostToDevice, s->stream));
        CK(launch_fill_cells(s->max_blocks, s->stream, s->shadow.p, (const CellFill*)s->scratch.p, (uint32_t)niv, total));
    }
    if (!heap.empty())
        CK(cudaMemcpyAsync(s->heap.p, heap.data(), heap.size() * 4, cudaMemcpyHostToDevice, s->stream));
    CK(cudaStreamSynchronize(s->stream));
    // numbering: renumbered values -> trace values; later events continue above them
    const std::vector<uint32_t>& old = *s->orig;
    auto no = std::make_shared<std::vector<uint32_t>>(vals.size() + 1, 0u);
    for (size_t r = 0; r < vals.size(); r++) {
        const uint32_t u = vals[r];
        (*no)[r + 1] = u < old.size() ? old[u] : (uint32_t)(u + s->delta);
    }
    s->orig = no;
    s->delta = s->checked_events - vals.size();
    // earlier segment rows are never read again
    s->cur_seg.assign(s->F, NO_SEG);
    s->nseg = 0;
    s->seg_uploaded = 0;
    s->segvc.clear();
    s->renumberings++;
    return CUSAN_OK;
}

extern "C" {

int cusan_session_create(const cusan_trace* t, const cusan_check_opts* o, cusan_session** out) {
    if (!t || !o || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (o->nshards < 1 || o->shard < 0 || o->shard >= o->nshards)
        return fail(CUSAN_EINVAL, "need 0 <= shard < nshards");
    if (o->shard_block & (o->shard_block - 1))
        return fail(CUSAN_EINVAL, "shard_block must be a power of two (or 0)");
    if (o->workspace) return fail(CUSAN_EINVAL, "sessions manage their own device memory");
    if (o->window_events < 0) return fail(CUSAN_EINVAL, "window_events must be >= 0");
    if (int st = check_flags(*o)) return st;
    if (o->flags & CUSAN_CHECK_DEFER_WORKSPACE) return fail(CUSAN_EINVAL, "sessions manage their own device memory");
    cusan_session* s = new (std::nothrow) cusan_session;
    if (!s) return fail(CUSAN_ENOMEM, "cannot allocate session");
    s->trace = t;
    s->opts = *o;
    s->opts.persist_shadow = 1;
    s->blk_log2 = o->shard_block ? (uint32_t)__builtin_ctzll(o->shard_block) : 21u;
    if (const char* e = std::getenv("CUSAN_SESSION_EVENT_LIMIT")) {     // tests: renumber early
        const unsigned long long v = std::strtoull(e, nullptr, 10);
        if (v >= 64) s->limit = std::min<uint64_t>(v, CUSAN_MAX_EVENTS);
    }
    s->F = t->t.max_fibers;
    s->C.assign((size_t)s->F * s->F, 0);
    s->cur_seg.assign(s->F, NO_SEG);
    int st = device_info(o->device, &s->max_blocks);
    if (!st) {
        s->device = o->device;
        s->stream = (cudaStream_t)o->stream;
        if (cudaEventCreate(&s->ev0) != cudaSuccess || cudaEventCreate(&s->ev1) != cudaSuccess)
            st = fail(CUSAN_ECUDA, "cannot create events");
    }
    // run buffer and its merge scratch now, while allocation is cheap (before the shadow is mapped)
    if (!st) {
        size_t free_b = 0, total_b = 0;
        cudaMemGetInfo(&free_b, &total_b);
        s->heap.reserve = (1ull << 24) * REC_WORDS * sizeof(uint32_t);   // the 24-bit record index
        s->segvc_d.reserve = s->scratch.reserve = total_b / 8;
        s->runs.reserve = s->merge_buf.reserve = total_b / 16;
        st = grow_runs(s, 1ull << 20);
    }
    if (!st) st = grow_heap(s, 1ull << 16);
    if (!st) st = grow_buf(s, s->scratch, 16ull << 20, 0, "plan tables");
    if (st) {
        delete s;
        return st;
    }
    *out = s;
    return CUSAN_OK;
}

static int cusan_session_submit_impl(cusan_session* s, cusan_report** prev) {
    if (!s || !prev) return fail(CUSAN_EINVAL, "null argument");
    *prev = nullptr;
    if (s->broken) return fail(CUSAN_ESTATE, "an earlier call failed after changing the session's state");
    CK(cudaSetDevice(s->device));
    std::unique_ptr<PendingCall> next(new (std::nothrow) PendingCall);
    if (!next) return fail(CUSAN_ENOMEM, "cannot allocate a call");
    next->t_start = std::chrono::steady_clock::now();
    int st;
    if (s->trace->t.ev.size() - s->delta > s->limit) {   // ids would outgrow 24 bits: renumber first
        if (s->pending) {                                  // (needs the device state of the call in flight)
            std::unique_ptr<PendingCall> done = std::move(s->pending);
            st = session_finish(s, *done, prev);
            if (st) {
                s->broken = true;
                return st;
            }
        }
        try {
            st = session_renumber(s);
        } catch (const std::bad_alloc&) {
            st = fail(CUSAN_ENOMEM, "host memory exhausted while renumbering the session's event ids");
        }
        if (st) {
            s->broken = true;
            return st;
        }
    }
    st = session_plan(s, *next);                     // host: overlaps the call in flight
    if (st) return st;
    if (s->pending) {                                // collect the call in flight
        std::unique_ptr<PendingCall> done = std::move(s->pending);
        st = session_finish(s, *done, prev);
        if (st) {
            s->broken = true;
            return st;
        }
    }
    st = session_launch(s, *next);
    if (st) return st;
    s->pending = std::move(next);
    s->broken = false;
    return CUSAN_OK;
}

static int cusan_session_finish_impl(cusan_session* s, cusan_report** out) {
    if (!s || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (!s->pending) return CUSAN_OK;
    CK(cudaSetDevice(s->device));
    std::unique_ptr<PendingCall> done = std::move(s->pending);
    return session_finish(s, *done, out);
}

int cusan_session_check(cusan_session* s, cusan_report** out) {
    if (!s || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (s->pending) return fail(CUSAN_ESTATE, "a submitted call is in flight: collect it with cusan_session_finish");
    cusan_report* none = nullptr;
    int st = cusan_session_submit(s, &none);
    if (st) return st;
    return cusan_session_finish(s, out);
}

int cusan_session_forget(cusan_session* s, uint64_t addr, uint64_t nbytes) {
    if (!s) return fail(CUSAN_EINVAL, "session is null");
    if (addr + nbytes < addr) return fail(CUSAN_ERANGE, "addr + nbytes overflows");
    if (!nbytes) return CUSAN_OK;
    try {
        const uint64_t g0 = (addr + 7) >> 3, g1 = (addr + nbytes) >> 3;   // granules wholly inside
        if (g1 > g0) s->forget.push_back({g0, g1});
    } catch (const std::bad_alloc&) {
        return fail(CUSAN_ENOMEM, "host memory exhausted in cusan_session_forget");
    }
    return CUSAN_OK;
}

int cusan_session_destroy(cusan_session* s) {
    if (!s) return fail(CUSAN_EINVAL, "session is null");
    if (s->stream || s->pending) cudaStreamSynchronize(s->stream);
    delete s;
    return CUSAN_OK;
}


int cusan_session_submit(cusan_session* s, cusan_report** prev) {
    try {
        return cusan_session_submit_impl(s, prev);
    } catch (const std::bad_alloc&) {
        return fail(CUSAN_ENOMEM, "host memory exhausted in cusan_session_submit");
    } catch (const std::exception& e) {
        return fail(CUSAN_ESTATE, std::string("internal error in cusan_session_submit: ") + e.what());
    }
}


int cusan_session_finish(cusan_session* s, cusan_report** out) {
    try {
        return cusan_session_finish_impl(s, out);
    } catch (const std::bad_alloc&) {
        return fail(CUSAN_ENOMEM, "host memory exhausted in cusan_session_finish");
    } catch (const std::exception& e) {
        return fail(CUSAN_ESTATE, std::string("internal error in cusan_session_finish: ") + e.what());
    }
}

}  // extern "C"
