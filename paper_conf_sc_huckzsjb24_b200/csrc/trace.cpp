// Trace object (step a0), error reporting and the host side of the report (a4 merge, a5).
#include <algorithm>
#include <cstring>
#include <new>

#include "common.h"

namespace cusan {

static thread_local std::string g_last_error;

int fail(int status, const std::string& msg) {
    g_last_error = msg;
    return status;
}

// Canonical order and maximal runs: sort by (later, earlier, g_begin),
// then merge runs with equal (earlier, later) whose granule ranges abut.
void canonicalize_runs(std::vector<cusan_race_run>& runs) {
    std::sort(runs.begin(), runs.end(), [](const cusan_race_run& a, const cusan_race_run& b) {
        if (a.later != b.later) return a.later < b.later;
        if (a.earlier != b.earlier) return a.earlier < b.earlier;
        return a.g_begin < b.g_begin;
    });
    size_t m = 0;
    for (size_t i = 0; i < runs.size(); i++) {
        if (m && runs[m - 1].later == runs[i].later && runs[m - 1].earlier == runs[i].earlier &&
            runs[m - 1].g_end == runs[i].g_begin)
            runs[m - 1].g_end = runs[i].g_end;
        else
            runs[m++] = runs[i];
    }
    runs.resize(m);
}

static int validate(const Trace& t, const cusan_event& e, uint64_t pos) {
    if (pos >= CUSAN_MAX_TRACE_EVENTS) return fail(CUSAN_ERANGE, "trace longer than 2^32-2 events");
    if (e.fiber >= t.max_fibers) return fail(CUSAN_EINVAL, "fiber >= max_fibers");
    switch (e.kind) {
        case CUSAN_EV_ACCESS:
            if (e.mode > 1) return fail(CUSAN_EINVAL, "bad access mode");
            if (e.a + e.b < e.a || e.a + e.b + 7 < e.a + e.b)
                return fail(CUSAN_ERANGE, "addr + nbytes overflows");
            return CUSAN_OK;
        case CUSAN_EV_RELEASE:
        case CUSAN_EV_RELEASE_STORE:
        case CUSAN_EV_ACQUIRE:
            return CUSAN_OK;
        case CUSAN_EV_FORK:
            if (e.a >= t.max_fibers) return fail(CUSAN_EINVAL, "fork source fiber >= max_fibers");
            return CUSAN_OK;
        default:
            return fail(CUSAN_EINVAL, "bad event kind");
    }
}

}  // namespace cusan

using namespace cusan;

extern "C" {

const char* cusan_last_error(void) { return g_last_error.c_str(); }
const char* cusan_version(void) { return "cusan-b200 0.1 (sm_100a)"; }

int cusan_trace_create(uint32_t max_fibers, uint64_t reserve_events, cusan_trace** out) {
    if (!out) return fail(CUSAN_EINVAL, "out is null");
    *out = nullptr;
    if (max_fibers < 1 || max_fibers > CUSAN_MAX_FIBERS)
        return fail(CUSAN_EINVAL, "max_fibers must be in [1, 255]");
    cusan_trace* t = new (std::nothrow) cusan_trace;
    if (!t) return fail(CUSAN_ENOMEM, "cannot allocate trace");
    t->t.max_fibers = max_fibers;
    try {
        t->t.ev.reserve(std::min<uint64_t>(reserve_events, CUSAN_MAX_TRACE_EVENTS));
    } catch (...) {
        delete t;
        return fail(CUSAN_ENOMEM, "cannot reserve trace");
    }
    *out = t;
    return CUSAN_OK;
}

int cusan_trace_destroy(cusan_trace* t) {
    if (!t) return fail(CUSAN_EINVAL, "trace is null");
    delete t;
    return CUSAN_OK;
}

static int push(cusan_trace* t, const cusan_event& e, uint32_t* id) {
    int st = validate(t->t, e, t->t.ev.size());
    if (st) return st;
    try {
        t->t.ev.push_back(e);
    } catch (...) {
        return fail(CUSAN_ENOMEM, "trace append failed");
    }
    if (id) *id = (uint32_t)(t->t.ev.size() - 1);
    return CUSAN_OK;
}

int cusan_trace_append_access(cusan_trace* t, uint32_t fiber, enum cusan_mode mode, uint64_t addr,
                              uint64_t nbytes, uint32_t* event_id) {
    if (!t) return fail(CUSAN_EINVAL, "trace is null");
    cusan_event e{};
    e.kind = CUSAN_EV_ACCESS;
    e.mode = (uint8_t)mode;
    if ((unsigned)mode > 1) return fail(CUSAN_EINVAL, "bad access mode");
    e.fiber = fiber;
    e.a = addr;
    e.b = nbytes;
    return push(t, e, event_id);
}

int cusan_trace_append_sync(cusan_trace* t, enum cusan_sync kind, uint32_t fiber,
                            uint64_t key_or_src_fiber, uint32_t* event_id) {
    if (!t) return fail(CUSAN_EINVAL, "trace is null");
    cusan_event e{};
    switch (kind) {
        case CUSAN_RELEASE: e.kind = CUSAN_EV_RELEASE; break;
        case CUSAN_RELEASE_STORE: e.kind = CUSAN_EV_RELEASE_STORE; break;
        case CUSAN_ACQUIRE: e.kind = CUSAN_EV_ACQUIRE; break;
        case CUSAN_FORK: e.kind = CUSAN_EV_FORK; break;
        default: return fail(CUSAN_EINVAL, "bad sync kind");
    }
    e.fiber = fiber;
    e.a = key_or_src_fiber;
    return push(t, e, event_id);
}

int cusan_trace_append_events(cusan_trace* t, const cusan_event* events, uint64_t n) {
    if (!t || (!events && n)) return fail(CUSAN_EINVAL, "null argument");
    uint64_t base = t->t.ev.size();
    for (uint64_t i = 0; i < n; i++) {
        int st = validate(t->t, events[i], base + i);
        if (st) return st;
    }
    try {
        t->t.ev.insert(t->t.ev.end(), events, events + n);
    } catch (...) {
        return fail(CUSAN_ENOMEM, "trace append failed");
    }
    return CUSAN_OK;
}

int cusan_trace_size(const cusan_trace* t, uint64_t* n_events, uint32_t* max_fibers) {
    if (!t) return fail(CUSAN_EINVAL, "trace is null");
    if (n_events) *n_events = t->t.ev.size();
    if (max_fibers) *max_fibers = t->t.max_fibers;
    return CUSAN_OK;
}

int cusan_trace_read(const cusan_trace* t, uint64_t first, uint64_t n, cusan_event* out) {
    if (!t || (!out && n)) return fail(CUSAN_EINVAL, "null argument");
    if (first > t->t.ev.size() || n > t->t.ev.size() - first) return fail(CUSAN_ERANGE, "range");
    if (n) std::memcpy(out, t->t.ev.data() + first, n * sizeof(cusan_event));
    return CUSAN_OK;
}

void cusan_check_opts_init(cusan_check_opts* o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->nshards = 1;
}

int cusan_report_get(const cusan_report* r, uint64_t* n_race_granules, uint64_t* n_runs,
                     const cusan_race_run** runs, int* truncated) {
    if (!r) return fail(CUSAN_EINVAL, "report is null");
    if (n_race_granules) *n_race_granules = r->n_race_granules;
    if (n_runs) *n_runs = r->n_runs;
    if (runs) *runs = r->runs.empty() ? nullptr : r->runs.data();
    if (truncated) *truncated = r->truncated;
    return CUSAN_OK;
}

int cusan_report_counters(const cusan_report* r, cusan_counters* out) {
    if (!r || !out) return fail(CUSAN_EINVAL, "null argument");
    *out = r->ctr;
    return CUSAN_OK;
}

int cusan_report_merge(const cusan_race_run* runs, uint64_t n_runs, uint64_t n_race_granules,
                       uint64_t max_runs, cusan_report** out) {
    if (!out || (!runs && n_runs)) return fail(CUSAN_EINVAL, "null argument");
    *out = nullptr;
    cusan_report* r = new (std::nothrow) cusan_report;
    if (!r) return fail(CUSAN_ENOMEM, "cannot allocate report");
    try {
        r->runs.assign(runs, runs + n_runs);
    } catch (...) {
        delete r;
        return fail(CUSAN_ENOMEM, "cannot allocate report runs");
    }
    canonicalize_runs(r->runs);
    r->n_runs = r->runs.size();
    r->n_race_granules = n_race_granules;
    if (max_runs && r->runs.size() > max_runs) {
        r->runs.resize(max_runs);
        r->truncated = 1;
    }
    *out = r;
    return CUSAN_OK;
}

int cusan_report_free(cusan_report* r) {
    if (!r) return fail(CUSAN_EINVAL, "report is null");
    delete r;
    return CUSAN_OK;
}

}  // extern "C"
