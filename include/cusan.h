/*
 * cusan.h — C ABI of the B200-native happens-before race check over device memory
 * (CuSan, Hück et al., SC-W 2024; /root/reference/PAPER.md).
 *
 * The library is the data-parallel hot path of CuSan's method: a trace of range accesses and
 * release / acquire / fork edges goes in (the TSan primitives CuSan and MUST emit,
 * PAPER.md:164-186, §II-A), an exact per-8-byte-granule race set comes out.
 *
 *   a0  append primitives (this header) or lower CUDA / MPI calls to them (cusan_lower.h)
 *   a1  vector-clock / segment pass (host)                             — cusan_plan_create
 *   a2  range → granule expansion, interval compaction, shard clip, windows (host) + upload
 *   a3  shadow check, one sm_100a kernel launch per window (device)    — cusan_plan_run
 *   a4  race-hit compaction into runs (in the kernel) + canonical merge (device sort / scan kernels)
 *   a5  report                                                          — cusan_report_*
 *
 * Conventions for every function:
 *   - returns CUSAN_OK (0) or a negative CUSAN_E* status; cusan_last_error() then returns a
 *     thread-local message describing the failure.  No function aborts the process.
 *   - pointers are host pointers unless stated; the library never retains caller pointers beyond
 *     the call except the trace passed to cusan_plan_create (which must outlive the plan).
 *   - objects are not thread-safe: one host thread per trace / plan.
 *   - there is no CPU fallback: without a usable CUDA device the check returns CUSAN_ECUDA.
 */
#ifndef CUSAN_H
#define CUSAN_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CUSAN_OK 0
#define CUSAN_EINVAL (-1)  /* null pointer, fiber >= max_fibers, bad enum, bad option            */
#define CUSAN_ERANGE (-2)  /* one-shot check of > 2^24-2 events, addr + nbytes overflows, ...    */
#define CUSAN_ENOMEM (-3)  /* host or device allocation failed / workspace too small             */
#define CUSAN_ECUDA (-4)   /* CUDA runtime error (includes: no device)                           */
#define CUSAN_ESTATE (-5)  /* object used in the wrong state                                     */

#define CUSAN_MAX_FIBERS 255u          /* fiber id is 8 bits in a shadow slot; 0xFF tags a spill record */
#define CUSAN_MAX_EVENTS ((1u << 24) - 2u) /* one-shot checks: event index + 1 is 24 bits in a shadow slot */
#define CUSAN_MAX_TRACE_EVENTS 0xFFFFFFFEu /* a trace (event ids are u32 in reports); sessions renumber
                                               their live epochs to stay inside 24 bits            */

typedef struct cusan_trace cusan_trace;   /* opaque; caller owns (create / destroy)            */
typedef struct cusan_plan cusan_plan;     /* opaque; caller owns (create / destroy)            */
typedef struct cusan_report cusan_report; /* library-allocated; free with cusan_report_free    */
typedef struct cusan_counters cusan_counters; /* defined below (report section)                */

/* Access mode of a range annotation (tsan_read_range / tsan_write_range).
 * A kernel argument the analysis marks RW is passed as CUSAN_WRITE. */
enum cusan_mode { CUSAN_READ = 0, CUSAN_WRITE = 1 };

/* Synchronisation primitives (TSan annotation API; fibers PAPER.md:178-186). */
enum cusan_sync {
    CUSAN_RELEASE = 0,       /* AnnotateHappensBefore(key): SC_key := SC_key ⊔ C_fiber             */
    CUSAN_RELEASE_STORE = 1, /* SC_key := C_fiber (a re-recorded CUDA event replaces its capture)    */
    CUSAN_ACQUIRE = 2,       /* AnnotateHappensAfter(key): C_fiber := C_fiber ⊔ SC_key             */
    CUSAN_FORK = 3           /* issue edge src -> dst: `fiber` = dst, `key_or_src_fiber` = src;
                                an event of src's program order; C_dst := C_dst ⊔ C_src          */
};

/* Event kinds of the bulk record format (cusan_event.kind). */
enum cusan_event_kind {
    CUSAN_EV_ACCESS = 0, CUSAN_EV_RELEASE = 1, CUSAN_EV_RELEASE_STORE = 2,
    CUSAN_EV_ACQUIRE = 3, CUSAN_EV_FORK = 4
};

/* 24-byte primitive record, little-endian (same layout as tracegen.EVENT_DTYPE).
 * ACCESS: a = address, b = nbytes, mode = cusan_mode.  RELEASE / RELEASE_STORE / ACQUIRE:
 * a = key.  FORK: fiber = dst, a = src fiber.  The event id of a record is its trace position. */
typedef struct cusan_event {
    uint8_t kind, mode;
    uint16_t pad;
    uint32_t fiber;
    uint64_t a, b;
} cusan_event;

/* A maximal run of consecutive granules [g_begin, g_end) (granule = address >> 3) on which the
 * access event `earlier` races with the later access event `later` (event ids = trace positions). */
typedef struct cusan_race_run {
    uint64_t g_begin, g_end;
    uint32_t earlier, later;
} cusan_race_run;

/* ---- trace (step a0) ------------------------------------------------------------------------ */
/* max_fibers in [1, 255]; reserve_events is a capacity hint. */
int cusan_trace_create(uint32_t max_fibers, uint64_t reserve_events, cusan_trace** out);
int cusan_trace_destroy(cusan_trace* t);
/* tsan_{read,write}_range(addr, nbytes) on `fiber`.  nbytes = 0 covers no
 * granule.  event_id (nullable) receives the trace position. */
int cusan_trace_append_access(cusan_trace* t, uint32_t fiber, enum cusan_mode mode, uint64_t addr,
                              uint64_t nbytes, uint32_t* event_id);
int cusan_trace_append_sync(cusan_trace* t, enum cusan_sync kind, uint32_t fiber,
                            uint64_t key_or_src_fiber, uint32_t* event_id);
/* Bulk append of n records; validated as the single-record calls; all-or-nothing. */
int cusan_trace_append_events(cusan_trace* t, const cusan_event* events, uint64_t n);
int cusan_trace_size(const cusan_trace* t, uint64_t* n_events, uint32_t* max_fibers);
/* Copies events [first, first + n) into out (host buffer of n records). */
int cusan_trace_read(const cusan_trace* t, uint64_t first, uint64_t n, cusan_event* out);

/* ---- check (steps a1-a5) ---------------------------------------------------------------------- */
typedef struct cusan_check_opts {
    int nshards;          /* granule-range shards of the shadow space (1 = whole space); one per GPU */
    int shard;            /* shard this call checks, 0 <= shard < nshards                        */
    int device;           /* CUDA device ordinal                                                   */
    int window_events;    /* access events per shadow window; 0 = library default (one window)    */
    int persist_shadow;   /* 1: store every window's final cells (shadow left valid after the run) */
    int flags;            /* CUSAN_CHECK_* flags (0 = interval-compressed shadow, library-allocated) */
    uint64_t max_runs;    /* runs kept in the report (0 = all); counts stay exact when truncated   */
    void* stream;         /* cudaStream_t to run on (NULL = the legacy default stream)             */
    void* workspace;      /* optional caller-owned device memory (e.g. a torch tensor); NULL = the
                             library allocates with cudaMalloc                                     */
    uint64_t workspace_bytes;
    uint64_t shard_block; /* sessions with nshards > 1: granules per block of the block-cyclic shard
                             map, a power of two (0 = 2^21); one-shot checks shard by range instead */
    int ngpus;            /* cusan_check only: a whole-node check on devices device .. device+ngpus-1
                             (0 or 1 = one device): the clocks are computed
                             once, one host thread per device plans and checks one granule-range
                             shard, the shards' canonical runs are merged (cusan_report_merge).
                             Needs nshards == 1, no workspace and no stream (each device's legacy
                             default stream); CUSAN_ECUDA if the node has fewer devices.      */
} cusan_check_opts;

/* cusan_plan_create computes the plan but neither allocates nor uploads: the caller queries
 * cusan_plan_workspace_bytes, allocates device memory (e.g. a torch tensor from PyTorch's caching
 * allocator) and calls cusan_plan_bind_workspace before cusan_plan_run. */
#define CUSAN_CHECK_DEFER_WORKSPACE 2
/* Shadow representation (results are identical):
 *   CUSAN_CHECK_INTERVAL_SHADOW — the DEFAULT: one 8-B shadow cell per elementary interval (a maximal
 *     granule range no access endpoint splits).  Exact, because every granule of an elementary
 *     interval is covered by the same accesses, so all its cells would hold the same state; the
 *     paper's proposed remedy for the cost of tracking whole allocations.
 *   CUSAN_CHECK_DENSE_SHADOW — one 8-B cell per 8-byte granule, TSan's layout:
 *     every covered granule's cell is read and written in every window that touches it (the HBM
 *     roofline line of SURVEY.md §8(d)); the kernel verifies that the cells of each range agree.
 * Passing both is CUSAN_EINVAL.  (Flag value 1, a removed diagnostic, is rejected too.) */
#define CUSAN_CHECK_INTERVAL_SHADOW 4
#define CUSAN_CHECK_DENSE_SHADOW 8
/* Where cusan_plan_create builds the interval, incidence and span tables (step a2): on the GPU
 * (sm_100a kernels + CUB sorts and scans, plan_dev.cu; the plan waits for it) or on the host
 * (build_host_plan).  The tables are byte-identical either way.  Default: the device for traces of
 * at least 32768 accesses (env CUSAN_DEVICE_PLAN_MIN_ACCESSES), the host below — the device
 * planner's fixed cost (three host round trips, ~70 launches, ~0.7 ms) only pays off on large
 * traces (config 5: 2.3 ms vs 7.4 ms per plan; configs 2-4: the host is faster).  These flags force
 * one side; passing both is CUSAN_EINVAL.  cusan_plan_describe always plans on the host. */
#define CUSAN_CHECK_HOST_PLAN 16
#define CUSAN_CHECK_DEVICE_PLAN 32

/* Defaults: nshards 1, shard 0, device 0, window_events 0, persist 0, max_runs 0, all NULL. */
void cusan_check_opts_init(cusan_check_opts* o);

/* Whole check: plan_create + plan_run + plan_destroy (or, with opts.ngpus > 1, one shard per
 * device, checked concurrently and merged).  The trace is not mutated. */
int cusan_check(const cusan_trace* t, const cusan_check_opts* o, cusan_report** out);

/* Host preparation (a1, a2) and upload of the event / clock / interval tables to the device.
 * The trace must stay alive and unmodified while the plan exists. */
int cusan_plan_create(const cusan_trace* t, const cusan_check_opts* o, cusan_plan** out);
/* Device bytes the plan needs (tables + shadow + read-set heap + run buffer). */
int cusan_plan_workspace_bytes(const cusan_plan* p, uint64_t* bytes);
/* Binds caller-owned device memory (>= cusan_plan_workspace_bytes, 256-B aligned, on the plan's
 * device) to a plan created with CUSAN_CHECK_DEFER_WORKSPACE and uploads the tables (queued on the
 * plan's stream, not waited for: the check follows on the same stream).  The memory must stay
 * valid until cusan_plan_destroy.  CUSAN_ESTATE if the plan owns a workspace.
 * cusan_plan_create calls no CUDA function that waits for the device, so a plan can be prepared on
 * one host thread while another thread's check runs (pipelined checks). */
int cusan_plan_bind_workspace(cusan_plan* p, void* workspace, uint64_t bytes);
/* Device part (a3, a4) and the report (a5).  May be called repeatedly (each run starts from an
 * empty shadow); asynchronous work is complete when it returns. */
int cusan_plan_run(cusan_plan* p, cusan_report** out);
/* Waits for the plan's stream (pending uploads / work), then frees the plan.  A library-allocated
 * workspace is parked for the next plan on the device (one block per device, the largest) instead
 * of freed: cudaMalloc / cudaFree of a tens-of-GB shadow cost tens of ms each. */
int cusan_plan_destroy(cusan_plan* p);
/* Diagnostics: copies the plan's device tables to host memory — the incidence table (8-B records
 * {epoch, segment | write << 31}, *n_inc of them) and the span tables of every window (72-B DSpan
 * records incl. one sentinel per window, *n_spans of them) — if the buffers hold them (capacities
 * in records; NULL buffers only report the counts).  Used to check that device-built tables equal
 * host-built ones (CUSAN_CHECK_HOST_PLAN).  Waits for the plan's stream. */
int cusan_plan_tables(const cusan_plan* p, void* inc, uint64_t inc_cap, void* spans, uint64_t spans_cap,
                      uint64_t* n_inc, uint64_t* n_spans);
/* Frees the parked check workspaces and the pooled device-planning scratch (all devices).  Set
 * CUSAN_NO_WORKSPACE_CACHE=1 to never park a check workspace. */
int cusan_release_cached_memory(void);
/* ---- a1's products as a transferable object ("event clocks broadcast") ----------
 * cusan_clocks_compute runs a1 over the whole trace (on all of the node's cores): per access its
 * granule range and record {epoch, segment | write << 31}, the segment clock rows (u32 × fibers) and
 * the trace counters.  On a multi-GPU node the rank that recorded the trace computes them once,
 * exports a flat little-endian image (cusan_clocks_bytes / _export: header, g0[n], g1[n], records[n],
 * rows[nseg × F]), broadcasts it (NCCL over NVLink) and every rank imports it and plans its own
 * shard on its own GPU with cusan_plan_create_from_clocks (a2 on the device) — no rank repeats a1
 * and no rank needs the trace.  The image is validated on import (CUSAN_EINVAL if corrupt). */
typedef struct cusan_clocks cusan_clocks;
int cusan_clocks_compute(const cusan_trace* t, cusan_clocks** out);
int cusan_clocks_bytes(const cusan_clocks* c, uint64_t* bytes);
int cusan_clocks_export(const cusan_clocks* c, void* buf, uint64_t bytes);
int cusan_clocks_import(const void* buf, uint64_t bytes, cusan_clocks** out);
int cusan_clocks_destroy(cusan_clocks* c);
/* As cusan_plan_create, from clocks (the clocks need not outlive the plan; a2 on the device or the
 * host by the same rule).  Tables and results equal cusan_plan_create's on the trace the clocks came
 * from.  Splitting a0 / a1 / a2 this way lets a pipeline run them on separate host threads. */
int cusan_plan_create_from_clocks(const cusan_clocks* c, const cusan_check_opts* o, cusan_plan** out);
/* Host steps a1 and a2 only (no device needed): fills the trace / plan counters the same
 * plan_create would compute (shard clip, intervals, segments, windows, spill records). */
int cusan_plan_describe(const cusan_trace* t, const cusan_check_opts* o, cusan_counters* out);

/* ---- incremental (online) checking: SURVEY.md §8(f) f1 ------------------------------------------
 * CuSan checks while the program runs.  A session keeps the shadow on the device
 * between calls; each cusan_session_check() checks the accesses appended to the trace since the
 * previous call (in windows of opts.window_events, 0 = one window) against it and reports the races
 * whose later access is among them.  The union of all calls' reports equals one cusan_check of the
 * final trace; n_race_granules of the calls add up to its count.  The trace may only grow.
 * The host plan is incremental (clocks, sync clocks and the interval layout carry over; a call
 * processes only its new events) and the shadow layout is stable: cells are updated in place and
 * memory touched for the first time gets cells appended (every device buffer grows inside a
 * reserved virtual range).  Because a call updates the shadow in place it cannot be re-run: a run
 * buffer overflow truncates that call's run list (counts stay exact) and grows the buffer.
 * Read-set records are assigned on the host and reclaimed once no interval names them (reused from
 * the next call on), so the heap holds the live read sets rather than growing per call (counters
 * heap_live_bytes / heap_bytes).  Traces longer than the 24-bit epoch field: before a call that
 * would exceed 2^24-2 event ids the session renumbers every id value still in use (live cells, live
 * records, fiber and sync clocks — ranked, so all later comparisons are unchanged) and reports keep
 * trace positions (u32); CUSAN_ERANGE only if one call alone, or the live ids, need more than half
 * the field (counter renumberings).  A call that fails after changing the session's state leaves
 * it unusable (CUSAN_ESTATE afterwards).
 * Multi-GPU sessions (nshards > 1, one session per rank, each on its own device): the address space
 * is not known in advance, so the granule space is dealt out block-cyclically — granule g belongs
 * to shard (g / shard_block) mod nshards, shard_block a power of two (0 = 2^21 granules = 16 MiB of
 * address).  The shards' reports of one call, merged (cusan_report_merge), are the call's report.
 * No caller workspace.  Report counter tracked_bytes = bytes checked by this call (all shards),
 * tracked_bytes_shard = the part in this session's shard. */
typedef struct cusan_session cusan_session;
int cusan_session_create(const cusan_trace* t, const cusan_check_opts* o, cusan_session** out);
int cusan_session_check(cusan_session* s, cusan_report** out);
/* Pipelined form of cusan_session_check, so the host and the device work at the same time:
 * cusan_session_submit plans the events appended since the previous submit on the host (while the
 * call in flight runs on the device), then collects the call in flight (*prev = its report, NULL if
 * there was none), then queues this call's uploads and check on the session's stream and returns
 * without waiting.  cusan_session_finish waits for the call in flight and returns its report (NULL
 * if none).  Reports are identical to cusan_session_check's; cusan_session_check fails with
 * CUSAN_ESTATE while a submitted call is in flight.  *prev / *out are freed with cusan_report_free. */
int cusan_session_submit(cusan_session* s, cusan_report** prev);
int cusan_session_finish(cusan_session* s, cusan_report** out);
/* Memory reclamation for long-running sessions: the caller promises that no access appended after
 * this call touches [addr, addr + nbytes) — the memory was released and a later allocation at that
 * address is recorded under a new range, as the live capture does (f2; PyTorch's stream sanitizer
 * resets a block's state at deallocation for the same reason).  At the end of the next call's plan
 * (after the accesses appended before this call are checked against the old state) the session
 * drops the elementary intervals lying wholly inside the range from its layout, and read-set
 * records only they named become reusable; reports are unchanged.  Without it the layout grows with
 * every allocation a program ever touched, and so does each call's host cost.  An access that
 * breaks the promise starts from empty state on the dropped part (its races with accesses before
 * the forget are not reported).  Counter n_intervals = the live layout after the call.  Shadow
 * cells are not compacted (8 B per dropped interval with the compressed shadow). */
int cusan_session_forget(cusan_session* s, uint64_t addr, uint64_t nbytes);
int cusan_session_destroy(cusan_session* s);

/* ---- report (a5) ------------------------------------------------------------------------------ */
typedef struct cusan_counters {
    /* trace counters, cf. CuSan's Table I */
    uint64_t n_events, n_access, n_read, n_write, n_release, n_release_store, n_acquire, n_fork;
    uint64_t tracked_bytes;        /* Σ over accesses of 8 × granules covered (the metric)        */
    uint64_t tracked_bytes_shard;  /* the part of it inside this report's shard                    */
    uint64_t bytes_read, bytes_written;
    /* plan */
    /* n_intervals: covered elementary intervals of the whole trace; n_incidences, n_spans: the    */
    /* (interval, access) pairs and (window, interval) pieces of this plan's shard               */
    uint64_t n_fibers, n_segments, n_intervals, n_incidences, n_windows, n_spans;
    uint64_t shard_granules, spill_heap_bytes, spill_spans; /* read-set records: >= 2 reader fibers since the last write */
    uint64_t shadow_bytes, workspace_bytes, raw_runs;
    /* device timings of the last run, CUDA events on the plan's stream, milliseconds */
    double kernel_ms;              /* all shadow-check launches                                  */
    double run_ms;                 /* whole cusan_plan_run incl. run download and merge          */
    uint64_t kernel_launches;
    uint64_t shadow_cell_bytes;    /* algorithmic shadow bytes moved by the check kernels          */
    uint64_t h2d_bytes;            /* host -> device bytes: plan tables (create) + counters (run)  */
    uint64_t d2h_bytes;            /* device -> host bytes of the last run (counters + runs)       */
    /* sessions: read-set heap after this call — records some interval still names, and the heap's
       high-water mark (dead records are reused from the next call on, so it tracks the live set) */
    uint64_t heap_live_bytes, heap_bytes;
    uint64_t renumberings;         /* sessions: epoch renumberings so far (traces past 2^24-2 events) */
} cusan_counters;

int cusan_report_get(const cusan_report* r, uint64_t* n_race_granules, uint64_t* n_runs,
                     const cusan_race_run** runs, int* truncated);
int cusan_report_counters(const cusan_report* r, cusan_counters* out);
/* Report from explicit parts (e.g. runs gathered from the shards of a multi-GPU check):
 * concatenates, sorts canonically by (later, earlier, g_begin) and merges abutting runs. */
int cusan_report_merge(const cusan_race_run* runs, uint64_t n_runs, uint64_t n_race_granules,
                       uint64_t max_runs, cusan_report** out);
int cusan_report_free(cusan_report* r);

/* Number of CUDA devices visible to the process (CUSAN_ECUDA if none / no driver). */
int cusan_device_count(int* n);

const char* cusan_last_error(void);
const char* cusan_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CUSAN_H */
