// Plan / check C ABI (host side of steps a3-a5): device span tables, workspace layout and binding,
// the window launches, overflow re-runs, run download and the canonical report.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <map>
#include <mutex>
#include <new>
#include <string>
#include <thread>

#include "kernel.cuh"
#include "plan_dev.h"

using namespace cusan;

// ---- library-owned workspaces: one parked block per device ----------------------------------------
// A check without a caller workspace needs up to tens of GB (the shadow); cudaMalloc / cudaFree of
// that much cost tens of ms each and cudaFree waits for the device, so repeated cusan_check calls
// would pay both every time.  A destroyed plan parks its workspace instead (one block per device,
// the largest seen); the next plan on that device takes it when it is large enough.  Released by
// cusan_release_cached_memory() (or set CUSAN_NO_WORKSPACE_CACHE=1 to disable).
namespace {
struct WsCache {
    std::mutex m;
    char* p[256] = {};
    uint64_t bytes[256] = {};
};
WsCache& ws_cache() { static WsCache* c = new WsCache; return *c; }
bool ws_cache_on() {
    static const bool on = std::getenv("CUSAN_NO_WORKSPACE_CACHE") == nullptr;
    return on;
}
// a block of >= bytes on `device` (the current device): the parked one if it fits, else a new one
// (freeing a parked block that is too small first, so both never coexist)
cudaError_t ws_acquire(int device, uint64_t bytes, char** out, uint64_t* got) {
    *out = nullptr;
    *got = 0;
    if (ws_cache_on() && device >= 0 && device < 256) {
        WsCache& c = ws_cache();
        std::lock_guard<std::mutex> lk(c.m);
        if (c.p[device] && c.bytes[device] >= bytes) {
            *out = c.p[device];
            *got = c.bytes[device];
            c.p[device] = nullptr;
            c.bytes[device] = 0;
            return cudaSuccess;
        }
        if (c.p[device]) {
            cudaFree(c.p[device]);
            c.p[device] = nullptr;
            c.bytes[device] = 0;
        }
    }
    cudaError_t e = cudaMalloc((void**)out, bytes);
    if (e == cudaErrorMemoryAllocation) {      // blocks parked on other devices do not matter, but
        (void)cudaGetLastError();              // a racing thread may have parked one here: retry once
        cusan::release_parked_workspace(device);
        e = cudaMalloc((void**)out, bytes);
    }
    if (e == cudaSuccess) *got = bytes;
    return e;
}
// park a block (the plan's work on it is complete); frees whichever of it and the parked one is smaller
void ws_release(int device, char* p, uint64_t bytes) {
    if (!p) return;
    if (ws_cache_on() && device >= 0 && device < 256) {
        WsCache& c = ws_cache();
        std::lock_guard<std::mutex> lk(c.m);
        if (!c.p[device] || c.bytes[device] < bytes) {
            char* old = c.p[device];
            c.p[device] = p;
            c.bytes[device] = bytes;
            if (old) {
                int cur = 0;
                cudaGetDevice(&cur);
                cudaSetDevice(device);
                cudaFree(old);
                cudaSetDevice(cur);
            }
            return;
        }
    }
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(device);
    cudaFree(p);
    cudaSetDevice(cur);
}
}  // namespace

void cusan::release_parked_workspace(int device) {
    if (device < 0 || device >= 256) return;
    WsCache& c = ws_cache();
    std::lock_guard<std::mutex> lk(c.m);
    if (!c.p[device]) return;
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(device);
    cudaFree(c.p[device]);
    cudaSetDevice(cur);
    c.p[device] = nullptr;
    c.bytes[device] = 0;
}

struct cusan_plan {
    const cusan_trace* trace = nullptr;
    HostPlan hp;
    int device = 0;
    cudaStream_t stream = nullptr;
    int max_blocks = 0;
    // device memory
    char* own = nullptr;          // library-allocated workspace (null when the caller's is used)
    uint64_t own_bytes = 0;
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
    uint64_t o_inc = 0, o_seg = 0, o_spans = 0, o_cnt = 0, o_heap = 0, o_shadow = 0, o_runs = 0, o_merge = 0;
    uint64_t merge_bytes = 0;
    pinned_vector<DSpan> ds;                // device span tables (host copy, uploaded at bind)
    std::vector<Window> wins;
    uint64_t shadow_cell_bytes = 0;
    uint64_t table_bytes = 0;               // tables uploaded by plan_create
    std::vector<unsigned long long> counter_init;
    RunMerge merge;                         // a4 scratch (device run merge)
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    bool dev_planned = false;               // a2 ran on the device: tables live in dscr
    const Trace* a1_trace = nullptr;        // a1 still to run (overlapping the device planner)
    DevScratch* dscr = nullptr;
    uint64_t n_ds = 0;                      // span table records (device-planned)

    ~cusan_plan() {
        if (dscr) plan_dev_release(dscr);
        if (ev0) cudaEventDestroy(ev0);
        if (ev1) cudaEventDestroy(ev1);
        if (own) ws_release(device, own, own_bytes);
        if (d_runs_own) cudaFree(d_runs_own);
        if (d_heap_own) cudaFree(d_heap_own);
    }
};

static int plan_bind(cusan_plan* p, char* ws, uint64_t bytes);
static int plan_device_setup(cusan_plan* p);
// plan_device_setup with host allocation failures turned into a status (nothing throws through the C ABI)
static int guarded_setup(cusan_plan* p) {
    try {
        return plan_device_setup(p);
    } catch (const std::bad_alloc&) {
        return fail(CUSAN_ENOMEM, "host memory exhausted while preparing the plan");
    } catch (const std::exception& e) {
        return fail(CUSAN_ESTATE, std::string("internal error while preparing the plan: ") + e.what());
    }
}

// Traces with at least this many accesses build their a2 tables on the device (cusan.h)
static uint64_t device_plan_min_accesses() {
    static const uint64_t v = [] {
        const char* e = std::getenv("CUSAN_DEVICE_PLAN_MIN_ACCESSES");
        return e && *e ? (uint64_t)std::strtoull(e, nullptr, 10) : (uint64_t)32768;
    }();
    return v;
}

// ---- pinned host blocks for uploaded tables (common.h) ------------------------------------------
// Every block carries a 64-byte header {size class, pinned?}.  Freed blocks go back to a cache by
// size class (powers of two from 64 KiB) up to PINNED_CACHE_MAX bytes; a process without a usable
// CUDA device gets heap blocks.
namespace {
constexpr size_t PIN_HDR = 64, PINNED_CACHE_MAX = size_t(1) << 30;
struct PinHdr { size_t cls; int pinned; };
struct PinCache {
    std::mutex m;
    std::map<size_t, std::vector<void*>> free_by_cls;
    size_t cached = 0;
    std::atomic<int> device_ok{-1};   // -1 unknown, 0 no CUDA device, 1 cudaHostAlloc works
};
PinCache& pin_cache() { static PinCache* c = new PinCache; return *c; }
// CUSAN_DEBUG_ALLOC=1: every page-locking allocation / release the cache could not serve, timed
// (and, in plan_dev.cu, every device planning scratch created or grown)
// (cudaHostAlloc pins pages, cudaFreeHost waits for the device: both stall a pipeline)
bool debug_pinned() {
    static const bool on = std::getenv("CUSAN_DEBUG_ALLOC") != nullptr;
    return on;
}
}  // namespace

void* cusan::pinned_alloc(size_t bytes) {
    size_t cls = size_t(1) << 16;
    while (cls < bytes + PIN_HDR) cls <<= 1;
    PinCache& c = pin_cache();
    {
        std::lock_guard<std::mutex> lk(c.m);
        auto it = c.free_by_cls.find(cls);
        if (it != c.free_by_cls.end() && !it->second.empty()) {
            void* b = it->second.back();
            it->second.pop_back();
            c.cached -= cls;
            return (char*)b + PIN_HDR;
        }
    }
    void* b = nullptr;
    int pinned = 0;
    if (c.device_ok != 0) {
        const auto t0 = std::chrono::steady_clock::now();
        const cudaError_t he = cudaHostAlloc(&b, cls, cudaHostAllocPortable);
        if (debug_pinned())
            std::fprintf(stderr, "cusan pinned: cudaHostAlloc %zu B %.3f ms (cached %zu B)\n", cls,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count(),
                         c.cached);
        if (he == cudaSuccess) {
            pinned = 1;
            c.device_ok = 1;
        } else {
            (void)cudaGetLastError();
            b = nullptr;
            int n = 0;
            if (c.device_ok == -1 && (cudaGetDeviceCount(&n) != cudaSuccess || n == 0)) c.device_ok = 0;
            (void)cudaGetLastError();
        }
    }
    if (!b) b = std::malloc(cls);
    if (!b) throw std::bad_alloc();
    *(PinHdr*)b = PinHdr{cls, pinned};
    return (char*)b + PIN_HDR;
}

void cusan::pinned_free(void* p) noexcept {
    if (!p) return;
    void* b = (char*)p - PIN_HDR;
    const PinHdr h = *(const PinHdr*)b;
    PinCache& c = pin_cache();
    {
        std::lock_guard<std::mutex> lk(c.m);
        if (c.cached + h.cls <= PINNED_CACHE_MAX) {
            c.free_by_cls[h.cls].push_back(b);
            c.cached += h.cls;
            return;
        }
    }
    if (h.pinned) {
        const auto t0 = std::chrono::steady_clock::now();
        cudaFreeHost(b);
        if (debug_pinned())
            std::fprintf(stderr, "cusan pinned: cudaFreeHost %zu B %.3f ms\n", h.cls,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    } else {
        std::free(b);
    }
}

// Work-unit (warp range) sizing, granules.  The compiled defaults (kernel.cuh) can be overridden
// at run time by CUSAN_RANGE_MIN / CUSAN_RANGE_MAX / CUSAN_RANGE_PER_ACCESS / CUSAN_RANGE_BAL_MIN /
// CUSAN_RANGES_PER_WARP: tuning sweeps, and the parity tests that check results do not depend on
// the work decomposition.  Ranges are rounded up to whole lane steps (CHUNK granules).
namespace {
uint64_t env_u64(const char* name, uint64_t dflt) {
    const char* e = std::getenv(name);
    if (!e || !*e) return dflt;
    const unsigned long long v = std::strtoull(e, nullptr, 10);
    return v ? (uint64_t)v : dflt;
}
uint64_t env_u64_or_zero(const char* name, uint64_t dflt) {
    const char* e = std::getenv(name);
    if (!e || !*e) return dflt;
    return (uint64_t)std::strtoull(e, nullptr, 10);
}
}  // namespace

// guided tail: the last TAIL_PCT % of each long span's ranges are cut TAIL_DIV times smaller and
// queued after every span's head, so the last work a launch hands out is small and the grid drains
// evenly (warps take ranges in queue order from the dynamic scheduler)
static DevPlanArgs span_args(int max_blocks) {
    DevPlanArgs a;
    a.R_MIN = env_u64("CUSAN_RANGE_MIN", CUSAN_RANGE_MIN);
    a.R_MAX = std::max<uint64_t>(env_u64("CUSAN_RANGE_MAX", CUSAN_RANGE_MAX), 1);
    a.R_PER_ACC = env_u64("CUSAN_RANGE_PER_ACCESS", CUSAN_RANGE_PER_ACCESS);
    a.R_BAL_MIN = env_u64("CUSAN_RANGE_BAL_MIN", CUSAN_RANGE_BAL_MIN);
    a.R_PER_WARP = env_u64("CUSAN_RANGES_PER_WARP", CUSAN_RANGES_PER_WARP);
    a.TAIL_PCT = std::min<uint64_t>(env_u64_or_zero("CUSAN_TAIL_PCT", CUSAN_TAIL_PCT), 99);
    a.TAIL_DIV = std::max<uint64_t>(env_u64("CUSAN_TAIL_DIV", CUSAN_TAIL_DIV), 1);
    a.max_blocks = max_blocks;
    return a;
}

void cusan::build_span_tables(const HostPlan& hp, int max_blocks, SpanTables& out) {
    const DevPlanArgs a = span_args(max_blocks);
    const uint64_t R_MIN = a.R_MIN, R_MAX = a.R_MAX, R_PER_ACC = a.R_PER_ACC, R_BAL_MIN = a.R_BAL_MIN;
    const uint64_t R_PER_WARP = a.R_PER_WARP, TAIL_PCT = a.TAIL_PCT, TAIL_DIV = a.TAIL_DIV;
    pinned_vector<DSpan>& ds = out.ds;
    std::vector<DSpan> tails;
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
            R_BAL_MIN, moving / (R_PER_WARP * WARPS * std::max(max_blocks, 1)));
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
            // warp range: long enough that replaying the window's accesses once per range stays
            // small next to streaming its cells, capped for balance; spans that move no cells
            // are one range each
            const bool comp = s.flags & SPAN_COMPRESSED;
            const bool moves = !comp && (s.flags & (SPAN_LOAD | SPAN_STORE));
            uint64_t rs;
            if (moves)
                rs = std::min<uint64_t>(std::min<uint64_t>(std::max<uint64_t>(R_PER_ACC * s.list_cnt, R_MIN), R_MAX),
                                        rs_cap);
            else
                rs = std::max<uint64_t>(s.len, 1);
            rs = std::min<uint64_t>((rs + CHUNK - 1) / CHUNK * CHUNK, 1ull << 31);
            if (s.flags & (SPAN_LOAD | SPAN_STORE)) out.need_shadow = true;
            out.cell_bytes += (comp ? 1 : s.len) * (((s.flags & SPAN_LOAD) ? 8 : 0) + ((s.flags & SPAN_STORE) ? 8 : 0));
            auto place = [&](DSpan x, uint64_t r) {       // x covers x.len granules in ranges of r
                x.rsize = (uint32_t)r;
                const uint64_t nt = comp ? 1 : (x.len + r - 1) / r;   // a compressed span: one range
                const uint64_t mem = moves ? r / 32 : 0;
                x.rweight = (uint32_t)std::min<uint64_t>(mem + 4ull * x.list_cnt + 8, 0xffffffffull);
                x.tile0 = tiles;
                x.weight0 = weight;
                tiles += nt;
                weight += nt * x.rweight;
                ds.push_back(x);
            };
            const uint64_t nt_all = (s.len + rs - 1) / rs;
            const uint64_t rs_t = std::max<uint64_t>((rs / TAIL_DIV + CHUNK - 1) / CHUNK * CHUNK, CHUNK);
            const uint64_t n_tail = nt_all * TAIL_PCT / 100;
            if (moves && TAIL_PCT && TAIL_DIV > 1 && rs_t < rs && n_tail >= 1 && n_tail < nt_all) {
                const uint64_t head = (nt_all - n_tail) * rs;      // whole head ranges
                DSpan t = d;
                d.len = head;
                t.abs_begin += head;
                t.dense_begin += head;
                t.len = s.len - head;
                t.rsize = (uint32_t)rs_t;
                place(d, rs);
                tails.push_back(t);
            } else {
                place(d, rs);
            }
        }
        for (DSpan t : tails) {                          // the guided tail, after every head
            const uint64_t r = t.rsize;
            const bool mv = !(t.flags & SPAN_COMPRESSED) && (t.flags & (SPAN_LOAD | SPAN_STORE));
            const uint64_t nt = (t.len + r - 1) / r;
            t.rweight = (uint32_t)std::min<uint64_t>((mv ? r / 32 : 0) + 4ull * t.list_cnt + 8, 0xffffffffull);
            t.tile0 = tiles;
            t.weight0 = weight;
            tiles += nt;
            weight += nt * t.rweight;
            ds.push_back(t);
        }
        tails.clear();
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

int cusan::device_info(int device, int* max_blocks) {
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0)
        return fail(CUSAN_ECUDA, std::string("no CUDA device available: ") + cudaGetErrorString(e));
    if (device < 0 || device >= ndev) return fail(CUSAN_EINVAL, "bad device ordinal");
    CK(cudaSetDevice(device));
    int sms = 0, per_sm = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    CK(shadow_check_blocks_per_sm(&per_sm));
    *max_blocks = sms * std::max(per_sm, 1);
    return CUSAN_OK;
}

static int plan_device_setup(cusan_plan* p) {
    HostPlan& hp = p->hp;
    const cusan_check_opts& o = hp.opts;
    const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    auto tick = [t0 = std::chrono::steady_clock::now(), dbg](const char* what) {
        if (dbg)
            std::fprintf(stderr, "plan_device_setup: %-12s %8.3f ms\n", what,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    };
    int st0 = device_info(o.device, &p->max_blocks);
    if (st0) return st0;
    tick("device info");
    p->device = o.device;
    p->stream = (cudaStream_t)o.stream;

    SpanTables st;
    uint64_t dev_h2d = 0;
    if (p->dev_planned) {
        // a2 on the device: the tables stay in the plan's planning scratch
        p->dscr = plan_dev_acquire(p->device);
        if (!p->dscr) return fail(CUSAN_ENOMEM, "cannot create the device planning scratch");
        DevPlanOut dp;
        std::function<int()> host_a1;
        if (p->a1_trace)
            host_a1 = [p, &hp] {
                const std::pair<int, std::string> r =
                    run_a1(*p->a1_trace, hp, a1_threads_for(p->a1_trace->ev.size()), false);
                if (r.first) return fail(r.first, r.second);
                p->a1_trace = nullptr;                   // a1 done
                return CUSAN_OK;
            };
        int e = device_plan_a2(hp, span_args(p->max_blocks), *p->dscr, dp, host_a1);
        if (e == CUSAN_ERANGE && !p->a1_trace) {   // beyond the device planner's 2^31 items: a2 on the host
            plan_dev_release(p->dscr);
            p->dscr = nullptr;
            p->dev_planned = false;
            if ((e = build_host_plan(nullptr, hp.opts, hp))) return e;
            return plan_device_setup(p);
        }
        if (e) return e;
        cusan_counters& c = hp.ctr;
        c.n_intervals = dp.n_intervals;
        c.n_incidences = dp.n_inc;
        c.shard_granules = hp.shard_granules = dp.shard_granules;
        c.tracked_bytes_shard = dp.tracked_bytes_shard;
        c.spill_spans = hp.spill_spans = dp.spill_spans;
        hp.rec_units = dp.rec_units;
        c.spill_heap_bytes = dp.rec_units * REC_WORDS * 4;
        c.n_windows = dp.wins.size();
        c.n_spans = dp.n_spans;
        hp.shadow_cells = dp.shadow_cells;
        for (const WinDesc& d : dp.wins) {
            Window w{};
            w.span_off = d.span_off;
            w.nspans = d.nspans;
            w.tiles = d.tiles;
            w.weight = d.weight;
            w.grid = (uint32_t)std::min<uint64_t>((uint64_t)p->max_blocks, (d.tiles + WARPS - 1) / WARPS);
            if (w.grid == 0) w.grid = 1;
            st.wins.push_back(w);
        }
        st.need_shadow = dp.need_shadow;
        st.cell_bytes = dp.cell_bytes;
        p->d_inc = const_cast<AccRec*>(dp.inc);
        p->d_spans = const_cast<DSpan*>(dp.ds);
        p->n_ds = dp.n_ds;
        dev_h2d = dp.h2d_bytes;
    } else {
        build_span_tables(hp, p->max_blocks, st);
    }
    pinned_vector<DSpan>& ds = st.ds;
    p->wins = st.wins;
    p->need_shadow = st.need_shadow;
    p->shadow_cell_bytes = st.cell_bytes;
    tick("span tables");

    // workspace layout
    p->heap_cap = hp.rec_units + (1ull << 16);             // pre-assigned records + lane-path room
    uint64_t off = 0;
    const uint64_t o_inc = off;     off = align_up(off + hp.inc.size() * sizeof(AccRec));
    const uint64_t o_seg = off;     off = align_up(off + hp.segvc.size() * sizeof(uint32_t));
    const uint64_t o_spans = off;   off = align_up(off + ds.size() * sizeof(DSpan));
    const uint64_t o_cnt = off;     off = align_up(off + (N_COUNTERS + p->wins.size()) * sizeof(unsigned long long));
    const uint64_t o_heap = off;    off = align_up(off + p->heap_cap * REC_WORDS * sizeof(uint32_t));
    const uint64_t o_shadow = off;  off = align_up(off + (p->need_shadow ? hp.shadow_cells * sizeof(uint2) : 0));
    // raw runs: a range with equal cells emits one run per racing pair, and ranges taken by different
    // warps are not joined before the device merge, so the buffer is sized from the ranges (an
    // overflow re-runs the check with a larger buffer)
    uint64_t tiles = 0;
    for (const Window& w : p->wins) tiles += w.tiles;
    p->run_cap = std::min<uint64_t>(std::max<uint64_t>(1ull << 16, 2 * tiles + 4 * p->wins.size() + 1024), 1ull << 24);
    const uint64_t o_runs = off;    off = align_up(off + p->run_cap * sizeof(cusan_race_run));
    // a4 scratch for merging up to run_cap raw runs (no allocation per run)
    const int mst = merge_scratch_bytes(p->run_cap, &p->merge_bytes);
    if (mst) return mst;
    const uint64_t o_merge = off;   off = align_up(off + p->merge_bytes);
    p->ws_bytes = off;
    p->o_inc = o_inc;
    p->o_seg = o_seg;
    p->o_spans = o_spans;
    p->o_cnt = o_cnt;
    p->o_heap = o_heap;
    p->o_shadow = o_shadow;
    p->o_runs = o_runs;
    p->o_merge = o_merge;
    p->ds = std::move(ds);
    p->table_bytes = hp.inc.size() * sizeof(AccRec) + hp.segvc.size() * sizeof(uint32_t) +
                     p->ds.size() * sizeof(DSpan) + dev_h2d;
    hp.ctr.shadow_bytes = p->need_shadow ? hp.shadow_cells * sizeof(uint2) : 0;
    hp.ctr.workspace_bytes = p->ws_bytes;
    tick("layout");
    // (the timing events are created at the first run, on the thread that runs the plan:
    // cudaEventCreate waits while another thread of the process synchronises with the device, so
    // creating them here would stall a plan prepared while the previous check runs)
    if (o.workspace) return plan_bind(p, (char*)o.workspace, o.workspace_bytes);
    if (o.flags & CUSAN_CHECK_DEFER_WORKSPACE) return CUSAN_OK;   // caller binds later
    cudaError_t me = ws_acquire(p->device, std::max<uint64_t>(off, ALIGN), &p->own, &p->own_bytes);
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
    if (!p->dev_planned) {
        p->d_inc = (AccRec*)(p->ws + p->o_inc);
        p->d_spans = (DSpan*)(p->ws + p->o_spans);
    }
    p->d_segvc = (uint32_t*)(p->ws + p->o_seg);
    p->d_counters = (unsigned long long*)(p->ws + p->o_cnt);
    p->d_shadow = p->need_shadow ? (uint2*)(p->ws + p->o_shadow) : nullptr;
    if (!p->d_runs_own) p->d_runs = (cusan_race_run*)(p->ws + p->o_runs);
    if (!p->merge.own) {
        p->merge.buf = p->ws + p->o_merge;
        p->merge.cap = p->merge_bytes;
    }
    if (!p->d_heap_own) p->d_heap = (uint32_t*)(p->ws + p->o_heap);
    else p->d_heap = p->d_heap_own;
    if (!p->dev_planned) {
        CK(cudaMemcpyAsync(p->d_inc, hp.inc.data(), hp.inc.size() * sizeof(AccRec), cudaMemcpyHostToDevice, p->stream));
        CK(cudaMemcpyAsync(p->d_spans, p->ds.data(), p->ds.size() * sizeof(DSpan), cudaMemcpyHostToDevice, p->stream));
    }
    CK(cudaMemcpyAsync(p->d_segvc, hp.segvc.data(), hp.segvc.size() * sizeof(uint32_t), cudaMemcpyHostToDevice, p->stream));
    // no wait: the kernels follow on the same stream, and the page-locked tables live until the
    // plan is destroyed (which synchronises the stream)
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
    if (!p->ev0) CK(cudaEventCreate(&p->ev0));
    if (!p->ev1) CK(cudaEventCreate(&p->ev1));
    CK(cudaEventRecord(p->ev0, p->stream));
    Ctx k;
    k.inc = p->d_inc;
    k.segvc = p->d_segvc;
    k.F = p->hp.F;
    k.shadow = p->d_shadow;
    k.heap = p->d_heap;
    k.heap_cap = p->heap_cap;
    k.runs = p->d_runs;
    k.counters = p->d_counters;
    k.run_cap = p->run_cap;
    for (size_t i = 0; i < p->wins.size(); i++) {
        const Window& w = p->wins[i];
        unsigned long long* sched = CUSAN_DYNAMIC ? p->d_counters + N_COUNTERS + i : nullptr;
        CK(launch_shadow_check(w.grid, p->stream, p->d_spans + w.span_off, w.nspans, w.tiles, w.weight, k, sched,
                               compressed_shadow(p->hp.opts)));
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
    // a2 on the device for large traces (or when asked), on the host for small ones
    const uint64_t dev_min = device_plan_min_accesses();
    uint64_t n_acc = 0;
    for (const cusan_event& e : t->t.ev) n_acc += e.kind == CUSAN_EV_ACCESS;
    p->dev_planned = n_acc > 0 && !(o->flags & CUSAN_CHECK_HOST_PLAN) &&
                     ((o->flags & CUSAN_CHECK_DEVICE_PLAN) || n_acc >= dev_min);
    int st;
    try {
        if (p->dev_planned) {          // a1 runs inside the device planner, overlapping its first phase
            st = prepare_plan_accesses(t->t, *o, p->hp);
            p->a1_trace = &t->t;
        } else {
            st = build_host_plan(&t->t, *o, p->hp);
        }
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while planning");
    }
    if (!st) st = guarded_setup(p);
    if (st) {
        delete p;
        return st;
    }
    *out = p;
    return CUSAN_OK;
}

// ---- a1 products as a transferable object (multi-GPU: one rank computes, all plan their shard) ----
namespace {
constexpr uint32_t CLOCKS_MAGIC = 0x4c435343u;   // "CSCL"
struct ClocksHdr {
    uint32_t magic, version, F, pad;
    uint64_t n_acc, nseg, n_events;
    cusan_counters ctr;
};
}  // namespace

int cusan_clocks_compute(const cusan_trace* t, cusan_clocks** out) {
    if (!t || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    cusan_clocks* c = new (std::nothrow) cusan_clocks;
    if (!c) return fail(CUSAN_ENOMEM, "cannot allocate clocks");
    int st;
    try {
        st = compute_clocks(t->t, c->hp);
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while computing clocks");
    }
    if (st) {
        delete c;
        return st;
    }
    *out = c;
    return CUSAN_OK;
}

int cusan_clocks_bytes(const cusan_clocks* c, uint64_t* bytes) {
    if (!c || !bytes) return fail(CUSAN_EINVAL, "null argument");
    const HostPlan& hp = c->hp;
    *bytes = sizeof(ClocksHdr) + hp.acc_g0.size() * (16 + sizeof(AccRec)) + hp.segvc.size() * 4;
    return CUSAN_OK;
}

int cusan_clocks_export(const cusan_clocks* c, void* buf, uint64_t bytes) {
    uint64_t need = 0;
    if (int st = cusan_clocks_bytes(c, &need)) return st;
    if (!buf || bytes < need) return fail(CUSAN_EINVAL, "buffer smaller than cusan_clocks_bytes");
    const HostPlan& hp = c->hp;
    ClocksHdr h{};
    h.magic = CLOCKS_MAGIC;
    h.version = 1;
    h.F = hp.F;
    h.n_acc = hp.acc_g0.size();
    h.nseg = hp.nseg;
    h.n_events = hp.ctr.n_events;
    h.ctr = hp.ctr;
    char* p = (char*)buf;
    std::memcpy(p, &h, sizeof(h));
    p += sizeof(h);
    std::memcpy(p, hp.acc_g0.data(), h.n_acc * 8);
    p += h.n_acc * 8;
    std::memcpy(p, hp.acc_g1.data(), h.n_acc * 8);
    p += h.n_acc * 8;
    std::memcpy(p, hp.acc_rec.data(), h.n_acc * sizeof(AccRec));
    p += h.n_acc * sizeof(AccRec);
    std::memcpy(p, hp.segvc.data(), hp.segvc.size() * 4);
    return CUSAN_OK;
}

int cusan_clocks_import(const void* buf, uint64_t bytes, cusan_clocks** out) {
    if (!buf || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    ClocksHdr h;
    if (bytes < sizeof(h)) return fail(CUSAN_EINVAL, "clocks image too short");
    std::memcpy(&h, buf, sizeof(h));
    if (h.magic != CLOCKS_MAGIC || h.version != 1) return fail(CUSAN_EINVAL, "not a clocks image");
    if (h.F < 1 || h.F > 256 || h.n_acc > (1ull << 40) || h.nseg > (1ull << 40))
        return fail(CUSAN_EINVAL, "corrupt clocks image");
    const uint64_t need = sizeof(h) + h.n_acc * (16 + sizeof(AccRec)) + h.nseg * h.F * 4;
    if (bytes < need) return fail(CUSAN_EINVAL, "clocks image truncated");
    cusan_clocks* c = new (std::nothrow) cusan_clocks;
    if (!c) return fail(CUSAN_ENOMEM, "cannot allocate clocks");
    try {
        HostPlan& hp = c->hp;
        hp.F = h.F;
        hp.nseg = h.nseg;
        hp.ctr = h.ctr;
        const char* p = (const char*)buf + sizeof(h);
        hp.acc_g0.resize(h.n_acc);
        hp.acc_g1.resize(h.n_acc);
        hp.acc_rec.resize(h.n_acc);
        hp.segvc.resize(h.nseg * h.F);
        std::memcpy(hp.acc_g0.data(), p, h.n_acc * 8);
        p += h.n_acc * 8;
        std::memcpy(hp.acc_g1.data(), p, h.n_acc * 8);
        p += h.n_acc * 8;
        std::memcpy(hp.acc_rec.data(), p, h.n_acc * sizeof(AccRec));
        p += h.n_acc * sizeof(AccRec);
        std::memcpy(hp.segvc.data(), p, hp.segvc.size() * 4);
    } catch (const std::bad_alloc&) {
        delete c;
        return fail(CUSAN_ENOMEM, "host memory exhausted while importing clocks");
    }
    *out = c;
    return CUSAN_OK;
}

int cusan_clocks_destroy(cusan_clocks* c) {
    if (!c) return fail(CUSAN_EINVAL, "clocks is null");
    delete c;
    return CUSAN_OK;
}

int cusan_plan_create_from_clocks(const cusan_clocks* c, const cusan_check_opts* o, cusan_plan** out) {
    if (!c || !o || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (o->nshards < 1 || o->shard < 0 || o->shard >= o->nshards) return fail(CUSAN_EINVAL, "need 0 <= shard < nshards");
    if (o->window_events < 0) return fail(CUSAN_EINVAL, "window_events must be >= 0");
    if (int st = check_flags(*o)) return st;
    cusan_plan* p = new (std::nothrow) cusan_plan;
    if (!p) return fail(CUSAN_ENOMEM, "cannot allocate plan");
    int st = CUSAN_OK;
    try {
        HostPlan& hp = p->hp;
        hp.opts = *o;
        hp.F = c->hp.F;
        hp.nseg = c->hp.nseg;
        hp.ctr = c->hp.ctr;
        hp.acc_g0 = c->hp.acc_g0;
        hp.acc_g1 = c->hp.acc_g1;
        hp.acc_rec = c->hp.acc_rec;
        hp.segvc = c->hp.segvc;
        p->dev_planned = !hp.acc_g0.empty() && !(o->flags & CUSAN_CHECK_HOST_PLAN) &&
                         ((o->flags & CUSAN_CHECK_DEVICE_PLAN) || hp.acc_g0.size() >= device_plan_min_accesses());
        if (!p->dev_planned) st = build_host_plan(nullptr, *o, hp);   // a2 on the host, from the clocks
    } catch (const std::bad_alloc&) {
        st = fail(CUSAN_ENOMEM, "host memory exhausted while planning");
    }
    if (!st) st = guarded_setup(p);
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
        st = build_host_plan(&t->t, *o, hp);
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

static int cusan_plan_run_impl(cusan_plan* p, cusan_report** out) {
    if (!p || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (!p->bound) return fail(CUSAN_ESTATE, "plan has no workspace: call cusan_plan_bind_workspace");
    const auto t_start = std::chrono::steady_clock::now();
    CK(cudaSetDevice(p->device));
    unsigned long long cnt[N_COUNTERS];
    int attempts = 0;
    for (int attempt = 0;; attempt++) {
        attempts = attempt + 1;
        int st = launch_all(p);
        if (st) return st;
        CK(cudaMemcpyAsync(cnt, p->d_counters, sizeof(cnt), cudaMemcpyDeviceToHost, p->stream));
        CK(cudaStreamSynchronize(p->stream));
        if (cnt[C_INVARIANT])
            return fail(CUSAN_ESTATE, "internal error: cells of one elementary interval differ (" +
                                          std::to_string(cnt[C_INVARIANT]) + " ranges)");
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
    uint64_t d2h = sizeof(cnt);
    const auto t_checked = std::chrono::steady_clock::now();
    const int mst = merge_runs_device(p->merge, p->stream, p->d_runs, cnt[C_RUNS], r->runs, &d2h);   // a4
    if (std::getenv("CUSAN_DEBUG_TIMING")) {
        using ms = std::chrono::duration<double, std::milli>;
        std::fprintf(stderr, "cusan_plan_run: %d attempt(s), check %.3f ms (kernels %.3f), merge %.3f ms of %llu raw runs\n",
                     attempts, ms(t_checked - t_start).count(), kms, ms(std::chrono::steady_clock::now() - t_checked).count(),
                     (unsigned long long)cnt[C_RUNS]);
    }
    if (mst) {
        delete r;
        return mst;
    }
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
    r->ctr.kernel_launches = p->wins.size() + (cnt[C_RUNS] ? MERGE_LAUNCHES : 0);
    r->ctr.shadow_cell_bytes = p->shadow_cell_bytes;
    r->ctr.h2d_bytes = p->table_bytes + sizeof(unsigned long long) * N_COUNTERS;
    r->ctr.d2h_bytes = d2h;
    r->ctr.run_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count();
    *out = r;
    return CUSAN_OK;
}

int cusan_plan_tables(const cusan_plan* p, void* inc, uint64_t inc_cap, void* spans, uint64_t spans_cap,
                      uint64_t* n_inc, uint64_t* n_spans) {
    if (!p || !n_inc || !n_spans) return fail(CUSAN_EINVAL, "null argument");
    if (!p->bound) return fail(CUSAN_ESTATE, "plan has no workspace: call cusan_plan_bind_workspace");
    CK(cudaSetDevice(p->device));
    CK(cudaStreamSynchronize(p->stream));
    *n_inc = p->dev_planned ? p->hp.ctr.n_incidences : p->hp.inc.size();
    *n_spans = p->dev_planned ? p->n_ds : p->ds.size();
    if (inc && inc_cap >= *n_inc && *n_inc)
        CK(cudaMemcpy(inc, p->d_inc, *n_inc * sizeof(AccRec), cudaMemcpyDeviceToHost));
    if (spans && spans_cap >= *n_spans && *n_spans)
        CK(cudaMemcpy(spans, p->d_spans, *n_spans * sizeof(DSpan), cudaMemcpyDeviceToHost));
    return CUSAN_OK;
}

int cusan_device_count(int* n) {
    if (!n) return fail(CUSAN_EINVAL, "null argument");
    *n = 0;
    cudaError_t e = cudaGetDeviceCount(n);
    if (e != cudaSuccess) {
        (void)cudaGetLastError();
        *n = 0;
        return fail(CUSAN_ECUDA, std::string("no CUDA device available: ") + cudaGetErrorString(e));
    }
    return CUSAN_OK;
}

int cusan_release_cached_memory(void) {
    WsCache& c = ws_cache();
    std::lock_guard<std::mutex> lk(c.m);
    int cur = 0;
    cudaGetDevice(&cur);
    for (int d = 0; d < 256; d++)
        if (c.p[d]) {
            cudaSetDevice(d);
            cudaFree(c.p[d]);
            c.p[d] = nullptr;
            c.bytes[d] = 0;
        }
    cudaSetDevice(cur);
    plan_dev_release_all();
    return CUSAN_OK;
}

int cusan_plan_destroy(cusan_plan* p) {
    if (!p) return fail(CUSAN_EINVAL, "plan is null");
    if (p->bound || p->stream) {          // pending uploads / work on the plan's stream
        cudaSetDevice(p->device);
        cudaStreamSynchronize(p->stream);
    }
    delete p;
    return CUSAN_OK;
}

// Whole-node check (opts.ngpus > 1): clocks once, one host thread per device planning (a2 on its
// device) and checking its granule-range shard, runs merged on the host.  The shards' canonical
// runs come back to host memory with each plan's report anyway, so the gather needs no collective.
// CUSAN_NODE_SHARE_DEVICES=1 (tests on a one-GPU machine) maps shard d to device (device+d) mod n.
static int check_node(const cusan_trace* t, const cusan_check_opts* o, cusan_report** out) {
    if (o->nshards != 1 || o->shard != 0) return fail(CUSAN_EINVAL, "ngpus > 1 shards by itself: nshards must be 1");
    if (o->workspace || o->stream) return fail(CUSAN_EINVAL, "ngpus > 1 takes no workspace and no stream");
    if (o->flags & (CUSAN_CHECK_HOST_PLAN | CUSAN_CHECK_DEFER_WORKSPACE))
        return fail(CUSAN_EINVAL, "ngpus > 1 plans on the devices with library workspaces");
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0)
        return fail(CUSAN_ECUDA, std::string("no CUDA device available: ") + cudaGetErrorString(e));
    const bool share = std::getenv("CUSAN_NODE_SHARE_DEVICES") != nullptr;
    if (o->device < 0 || (!share && o->device + o->ngpus > ndev))
        return fail(CUSAN_ECUDA, "ngpus = " + std::to_string(o->ngpus) + " from device " + std::to_string(o->device) +
                                     " but the node has " + std::to_string(ndev) + " CUDA devices");
    const auto t0 = std::chrono::steady_clock::now();
    cusan_clocks* clocks = nullptr;
    if (int st = cusan_clocks_compute(t, &clocks)) return st;
    const int n = o->ngpus;
    std::vector<cusan_report*> parts(n, nullptr);
    std::vector<int> status(n, CUSAN_OK);
    std::vector<std::string> errors(n);
    std::vector<std::thread> th;
    for (int d = 0; d < n; d++)
        th.emplace_back([&, d] {
            cusan_check_opts so = *o;
            so.ngpus = 0;
            so.nshards = n;
            so.shard = d;
            so.device = (o->device + d) % ndev;
            cusan_plan* p = nullptr;
            int st;
            try {
                st = cusan_plan_create_from_clocks(clocks, &so, &p);
                if (!st) {
                    st = cusan_plan_run(p, &parts[d]);
                    cusan_plan_destroy(p);
                }
            } catch (const std::exception& e) {            // a thread must not end in an exception
                st = fail(CUSAN_ENOMEM, std::string("shard thread: ") + e.what());
            }
            status[d] = st;
            if (st) errors[d] = cusan_last_error();
        });
    for (auto& x : th) x.join();
    cusan_clocks_destroy(clocks);
    int st = CUSAN_OK;
    for (int d = 0; d < n && !st; d++)
        if (status[d]) st = fail(status[d], "shard " + std::to_string(d) + ": " + errors[d]);
    cusan_report* r = nullptr;
    if (!st) {
        std::vector<cusan_race_run> runs;
        uint64_t nrace = 0;
        for (cusan_report* x : parts) {
            runs.insert(runs.end(), x->runs.begin(), x->runs.end());
            nrace += x->n_race_granules;
        }
        st = cusan_report_merge(runs.data(), runs.size(), nrace, o->max_runs, &r);
    }
    if (!st) {                              // counters: the trace's, summed / maxed over shards
        cusan_counters& c = r->ctr;
        c = parts[0]->ctr;
        for (int d = 1; d < n; d++) {
            const cusan_counters& x = parts[d]->ctr;
            c.tracked_bytes_shard += x.tracked_bytes_shard;
            c.shard_granules += x.shard_granules;
            c.n_incidences += x.n_incidences;
            c.n_spans += x.n_spans;
            c.spill_spans += x.spill_spans;
            c.spill_heap_bytes += x.spill_heap_bytes;
            c.shadow_bytes += x.shadow_bytes;
            c.workspace_bytes += x.workspace_bytes;
            c.raw_runs += x.raw_runs;
            c.kernel_launches += x.kernel_launches;
            c.shadow_cell_bytes += x.shadow_cell_bytes;
            c.h2d_bytes += x.h2d_bytes;
            c.d2h_bytes += x.d2h_bytes;
            c.kernel_ms = std::max(c.kernel_ms, x.kernel_ms);
            c.n_windows = std::max(c.n_windows, x.n_windows);
        }
        c.run_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        *out = r;
    }
    for (cusan_report* x : parts)
        if (x) cusan_report_free(x);
    return st;
}

int cusan_check(const cusan_trace* t, const cusan_check_opts* o, cusan_report** out) {
    if (!t || !o || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    if (o->ngpus < 0) return fail(CUSAN_EINVAL, "ngpus must be >= 0");
    if (o->ngpus > 1) return check_node(t, o, out);
    cusan_plan* p = nullptr;
    int st = cusan_plan_create(t, o, &p);
    if (st) return st;
    st = cusan_plan_run(p, out);
    cusan_plan_destroy(p);
    return st;
}


int cusan_plan_run(cusan_plan* p, cusan_report** out) {
    try {
        return cusan_plan_run_impl(p, out);
    } catch (const std::bad_alloc&) {
        return fail(CUSAN_ENOMEM, "host memory exhausted in cusan_plan_run");
    } catch (const std::exception& e) {
        return fail(CUSAN_ESTATE, std::string("internal error in cusan_plan_run: ") + e.what());
    }
}

}  // extern "C"
