// Incremental (online) sessions — SURVEY.md §8(f) f1.
#include <algorithm>
#include <chrono>
#include <cstring>
#include <new>
#include <string>

#include "kernel.cuh"

using namespace cusan;

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
    // zeroed, so the copy below never moves uninitialised words (unused tails of records)
    cudaError_t e = cudaMemsetAsync(nh, 0, cap * REC_WORDS * sizeof(uint32_t), s->stream);
    if (e == cudaSuccess && s->heap && s->heap_top)
        e = cudaMemcpyAsync(nh, s->heap, s->heap_top * REC_WORDS * sizeof(uint32_t), cudaMemcpyDeviceToDevice,
                            s->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s->stream);
    if (e != cudaSuccess) {
        cudaFree(nh);
        return cuda_fail(e, "grow_heap");
    }
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
            CK(launch_copy_cells(s->max_blocks, s->stream, s->shadow, s->spare, d_copy, (uint32_t)segs.size(),
                                  copy_cells_n));
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
            CK(launch_shadow_check(w.grid, s->stream, d_spans + w.span_off, w.nspans, w.tiles, w.weight, k,
                                   force_lanes, sched));
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

