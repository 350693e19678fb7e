// Lowering of CUDA / CUDA-aware MPI calls to happens-before primitives (step a0).
//
// CuSan runtime semantics (§IV-A, 606-734) plus MUST's MPI modelling,
// in the form of SURVEY.md §8(b)'s table.  Every operation on a stream s is bracketed by
//   prologue:  FORK(H -> s)                         issue order (Fig. 4 rank 1)
//              s blocking stream: ACQUIRE(s, K(S0))            legacy barrier (Fig. 3 (i))
//              s = S0: ACQUIRE(S0, K(u)) ∀ blocking u          legacy barrier (Fig. 3 (ii))
//   epilogue:  RELEASE(s, K(s))                     AnnotateHappensBefore
// H is the calling host thread's fiber.  Host threads and per-thread default streams (SURVEY §8(f)
// f4): thread creation is an issue edge FORK(parent -> child), a join is
// RELEASE(child, K(thread)) + ACQUIRE(parent, K(thread)); a per-thread default stream is a blocking
// stream of its thread ("not a non-blocking stream and will synchronize with the legacy default
// stream").  Stream handle 1 = cudaStreamLegacy, 2 = cudaStreamPerThread,
// 0 = the default stream of the selected mode.
#include <algorithm>
#include <functional>
#include <new>
#include <unordered_map>

#include "../../include/cusan_lower.h"
#include "common.h"

using namespace cusan;

namespace {
constexpr uint32_t S0 = 1;
constexpr uint64_t STREAM_LEGACY = 1, STREAM_PER_THREAD = 2;
inline uint64_t K_stream(uint32_t f) { return (1ull << 56) | f; }
inline uint64_t K_event(uint64_t e) { return (2ull << 56) | e; }
inline uint64_t K_req(uint64_t r) { return (3ull << 56) | r; }
inline uint64_t K_thread(uint64_t t) { return (4ull << 56) | t; }
}  // namespace

struct cusan_lowering {
    cusan_trace* trace;
    FlatMap<uint32_t> stream_fiber;                        // user stream handle -> fiber
    std::vector<uint32_t> streams;                         // S0, then streams (creation order)
    std::vector<uint32_t> blocking;                        // blocking streams (creation order)
    std::vector<char> is_blocking;                         // by fiber
    uint32_t next_fiber = 2;
    std::vector<uint32_t> mpi_free;                        // pool of completed request fibers (min-heap)
    FlatMap<uint32_t> req_fiber;                           // MPI request -> its fiber
    struct Alloc {
        uint64_t base, size;
        int kind;
    };
    std::vector<Alloc> allocs;                             // registered allocations, sorted by base
    FlatMap<Alloc> by_base;                                // the same, by exact base pointer
    FlatMap<uint32_t> thread_fiber;                        // host thread -> fiber (thread 0 -> 0)
    FlatMap<uint32_t> ptds;                                // host thread -> per-thread default stream
    uint64_t thread = 0;                                   // calling host thread
    uint32_t h_fiber = 0;                                  // its fiber (thread_fiber[thread])
    bool per_thread_mode = false;
    std::vector<std::pair<int, uint64_t>> fiber_info;      // by fiber: (cusan_fiber_kind, handle)

    void note(uint32_t f, int kind, uint64_t handle) {
        if (fiber_info.size() <= f) fiber_info.resize(f + 1, {-1, 0});
        fiber_info[f] = {kind, handle};
    }

    uint32_t H() const { return h_fiber; }

    // --- primitives ---------------------------------------------------------------------------
    // Appended straight to the trace: the lowering's fibers, modes and kinds are valid by
    // construction (fibers come from new_fiber, below max_fibers), so only what a caller's values
    // decide is checked — the trace length and addr + n overflowing (cusan_trace_append_* check
    // everything for events a user appends).
    int push(uint8_t kind, uint8_t mode, uint32_t f, uint64_t a, uint64_t b) {
        std::vector<cusan_event>& ev = trace->t.ev;
        if (ev.size() >= CUSAN_MAX_TRACE_EVENTS) return fail(CUSAN_ERANGE, "trace longer than 2^32-2 events");
        cusan_event e{};
        e.kind = kind;
        e.mode = mode;
        e.fiber = f;
        e.a = a;
        e.b = b;
        try {
            ev.push_back(e);
        } catch (...) {
            return fail(CUSAN_ENOMEM, "trace append failed");
        }
        return CUSAN_OK;
    }
    int access(uint32_t f, int mode, uint64_t addr, uint64_t n) {
        if (addr + n < addr || addr + n + 7 < addr + n) return fail(CUSAN_ERANGE, "addr + nbytes overflows");
        return push(CUSAN_EV_ACCESS, (uint8_t)(mode ? 1 : 0), f, addr, n);
    }
    int sync(cusan_sync k, uint32_t f, uint64_t key) {
        static constexpr uint8_t kind_of[4] = {CUSAN_EV_RELEASE, CUSAN_EV_RELEASE_STORE, CUSAN_EV_ACQUIRE,
                                               CUSAN_EV_FORK};
        return push(kind_of[k], 0, f, key, 0);
    }

    // --- helpers -------------------------------------------------------------------------------
    // allocation containing p (TypeART's extent lookup)
    // (the allocation with the greatest base <= p, if it contains p; a flat sorted array: lookups
    // happen for every kernel argument, registrations rarely)
    const Alloc* find(uint64_t p) const {
        // kernel arguments are nearly always allocation bases: an exact hit is the allocation with
        // the greatest base <= p, so it decides alone
        if (const Alloc* hit = by_base.get(p)) return hit->size ? hit : nullptr;
        auto it = std::upper_bound(allocs.begin(), allocs.end(), p,
                                   [](uint64_t x, const Alloc& a) { return x < a.base; });
        if (it == allocs.begin()) return nullptr;
        --it;
        if (p >= it->base && p - it->base < it->size) return &*it;
        return nullptr;
    }
    void add_alloc(uint64_t base, uint64_t size, int kind) {
        auto it = std::lower_bound(allocs.begin(), allocs.end(), base,
                                   [](const Alloc& a, uint64_t x) { return a.base < x; });
        if (it != allocs.end() && it->base == base)
            *it = {base, size, kind};                      // re-registration replaces
        else
            allocs.insert(it, {base, size, kind});
        by_base[base] = {base, size, kind};
    }
    // cudaFree(base): TypeART drops the allocation from its lookup table
    void remove_alloc(uint64_t base) {
        auto it = std::lower_bound(allocs.begin(), allocs.end(), base,
                                   [](const Alloc& a, uint64_t x) { return a.base < x; });
        if (it != allocs.end() && it->base == base) allocs.erase(it);
        by_base.erase(base);
    }
    int new_fiber(uint32_t* f) {
        uint32_t mf = 0;
        cusan_trace_size(trace, nullptr, &mf);
        if (next_fiber >= mf) return fail(CUSAN_EINVAL, "more fibers than the trace's max_fibers");
        *f = next_fiber++;
        if (is_blocking.size() <= *f) is_blocking.resize(*f + 1, 0);
        return CUSAN_OK;
    }
    int add_stream(uint32_t* f, bool blocking_stream) {
        int st = new_fiber(f);
        if (st) return st;
        streams.push_back(*f);
        if (blocking_stream) {
            blocking.push_back(*f);
            is_blocking[*f] = 1;
        }
        return CUSAN_OK;
    }
    // the calling thread's per-thread default stream (a blocking stream), created on first use
    int thread_ptds(uint32_t* f) {
        if (const uint32_t* it = ptds.get(thread)) {
            *f = *it;
            return CUSAN_OK;
        }
        int st = add_stream(f, true);
        if (!st) {
            ptds[thread] = *f;
            note(*f, CUSAN_FIBER_PER_THREAD_STREAM, thread);
        }
        return st;
    }
    int fiber_of(uint64_t stream, uint32_t* f) {
        if (stream == 0) {
            if (per_thread_mode) return thread_ptds(f);
            *f = S0;
            return CUSAN_OK;
        }
        if (stream == STREAM_LEGACY) {
            *f = S0;
            return CUSAN_OK;
        }
        if (stream == STREAM_PER_THREAD) return thread_ptds(f);
        const uint32_t* it = stream_fiber.get(stream);
        if (!it) return fail(CUSAN_EINVAL, "unknown stream handle");
        *f = *it;
        return CUSAN_OK;
    }
    int thread_fiber_of(uint64_t t, uint32_t* f) {
        if (const uint32_t* it = thread_fiber.get(t)) {
            *f = *it;
            return CUSAN_OK;
        }
        int st = new_fiber(f);
        if (!st) {
            thread_fiber[t] = *f;
            note(*f, CUSAN_FIBER_HOST, t);
        }
        return st;
    }
    int prologue(uint32_t f) {
        int st = sync(CUSAN_FORK, f, H());
        if (st) return st;
        if (f != S0 && f < is_blocking.size() && is_blocking[f]) return sync(CUSAN_ACQUIRE, f, K_stream(S0));
        if (f == S0)
            for (uint32_t u : blocking)
                if ((st = sync(CUSAN_ACQUIRE, S0, K_stream(u)))) return st;
        return CUSAN_OK;
    }
    int epilogue(uint32_t f) { return sync(CUSAN_RELEASE, f, K_stream(f)); }
    // cudaStreamSynchronize; on S0 also every blocking stream (724-727)
    int host_sync_stream(uint32_t f) {
        int st = sync(CUSAN_ACQUIRE, H(), K_stream(f));
        if (st || f != S0) return st;
        for (uint32_t u : blocking)
            if ((st = sync(CUSAN_ACQUIRE, H(), K_stream(u)))) return st;
        return CUSAN_OK;
    }
    // cudaDeviceSynchronize: every stream; work other threads submit
    // afterwards comes later in the trace and is not covered
    int host_sync_device() {
        for (uint32_t f : streams) {
            int st = sync(CUSAN_ACQUIRE, H(), K_stream(f));
            if (st) return st;
        }
        return CUSAN_OK;
    }
    bool tracked(uint64_t p, uint64_t n) const { return n > 0 && find(p) != nullptr; }
};

extern "C" {

int cusan_lowering_create(cusan_trace* trace, cusan_lowering** out) {
    if (!trace || !out) return fail(CUSAN_EINVAL, "null argument");
    uint32_t mf = 0;
    cusan_trace_size(trace, nullptr, &mf);
    if (mf < 2) return fail(CUSAN_EINVAL, "a lowering needs max_fibers >= 2 (host + default stream)");
    cusan_lowering* l = new (std::nothrow) cusan_lowering;
    if (!l) return fail(CUSAN_ENOMEM, "cannot allocate lowering");
    l->trace = trace;
    l->streams.push_back(S0);
    l->is_blocking.assign(2, 0);
    l->thread_fiber[0] = 0;
    l->note(0, CUSAN_FIBER_HOST, 0);
    l->note(S0, CUSAN_FIBER_LEGACY_STREAM, 0);
    *out = l;
    return CUSAN_OK;
}

int cusan_lowering_destroy(cusan_lowering* l) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    delete l;
    return CUSAN_OK;
}

int cusan_lowering_fibers(const cusan_lowering* l, uint32_t* n) {
    if (!l || !n) return fail(CUSAN_EINVAL, "null argument");
    *n = l->next_fiber;
    return CUSAN_OK;
}

int cusan_on_malloc(cusan_lowering* l, uint64_t ptr, uint64_t size, enum cusan_mem_kind kind) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    if ((unsigned)kind > 3) return fail(CUSAN_EINVAL, "bad memory kind");
    l->add_alloc(ptr, size, (int)kind);   // allocation is not an access
    return CUSAN_OK;
}

int cusan_on_free(cusan_lowering* l, uint64_t ptr) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    l->remove_alloc(ptr);                 // no longer tracked (★A25)
    return l->host_sync_device();
}

int cusan_on_stream_create(cusan_lowering* l, uint64_t stream, int nonblocking) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    if (stream <= STREAM_PER_THREAD) return fail(CUSAN_EINVAL, "stream handles 0, 1, 2 are reserved");
    uint32_t f = 0;
    int st = l->add_stream(&f, !nonblocking);   // track the non-blocking attribute
    if (st) return st;
    l->stream_fiber[stream] = f;
    l->note(f, CUSAN_FIBER_STREAM, stream);
    return CUSAN_OK;
}

int cusan_lowering_fiber_info(const cusan_lowering* l, uint32_t fiber, int* kind, uint64_t* handle) {
    if (!l || !kind || !handle) return fail(CUSAN_EINVAL, "null argument");
    if (fiber >= l->fiber_info.size() || l->fiber_info[fiber].first < 0)
        return fail(CUSAN_EINVAL, "unknown fiber");
    *kind = l->fiber_info[fiber].first;
    *handle = l->fiber_info[fiber].second;
    return CUSAN_OK;
}

int cusan_on_kernel(cusan_lowering* l, uint64_t stream, uint32_t nargs, const uint64_t* ptrs,
                    const uint32_t* modes) {
    if (!l || (nargs && (!ptrs || !modes))) return fail(CUSAN_EINVAL, "null argument");
    uint32_t f = 0;
    int st = l->fiber_of(stream, &f);
    if (st || (st = l->prologue(f))) return st;
    // (ii) of PAPER.md:650-654: each argument's whole allocation, by its R/W attribute
    for (uint32_t i = 0; i < nargs; i++) {
        auto* a = l->find(ptrs[i]);
        if (!a) continue;
        if (modes[i] > 2) return fail(CUSAN_EINVAL, "bad argument mode");
        int mode = modes[i] == 0 ? CUSAN_READ : CUSAN_WRITE;   // RW -> WRITE
        if ((st = l->access(f, mode, a->base, a->size))) return st;
    }
    return l->epilogue(f);
}

int cusan_on_stream_sync(cusan_lowering* l, uint64_t stream) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t f = 0;
    int st = l->fiber_of(stream, &f);
    return st ? st : l->host_sync_stream(f);
}

int cusan_on_device_sync(cusan_lowering* l) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    return l->host_sync_device();
}

int cusan_on_event_record(cusan_lowering* l, uint64_t event, uint64_t stream) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t f = 0;
    int st = l->fiber_of(stream, &f);
    if (st || (st = l->prologue(f))) return st;
    return l->sync(CUSAN_RELEASE_STORE, f, K_event(event));
}

int cusan_on_event_sync(cusan_lowering* l, uint64_t event) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    return l->sync(CUSAN_ACQUIRE, l->H(), K_event(event));
}

int cusan_on_stream_wait_event(cusan_lowering* l, uint64_t stream, uint64_t event) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t f = 0;
    int st = l->fiber_of(stream, &f);
    if (st || (st = l->prologue(f))) return st;
    return l->sync(CUSAN_ACQUIRE, f, K_event(event));
}

int cusan_on_stream_query(cusan_lowering* l, uint64_t stream, int success) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    if (!success) {            // no synchronisation, so no event and no (lazy) fiber either
        if (stream == 0 || stream == STREAM_LEGACY || stream == STREAM_PER_THREAD || l->stream_fiber.count(stream))
            return CUSAN_OK;
        return fail(CUSAN_EINVAL, "unknown stream handle");
    }
    uint32_t f = 0;
    int st = l->fiber_of(stream, &f);
    if (st) return st;
    return l->host_sync_stream(f);
}

int cusan_on_memcpy(cusan_lowering* l, uint64_t dst, uint64_t src, uint64_t n,
                    enum cusan_copy_kind kind, int async, uint64_t stream) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    if ((unsigned)kind > 3) return fail(CUSAN_EINVAL, "bad copy kind");
    uint32_t f = 0;
    int st = l->fiber_of(async ? stream : 0, &f);              // cudaMemcpy: the default stream
    if (st || (st = l->prologue(f))) return st;
    if (l->tracked(dst, n) && (st = l->access(f, CUSAN_WRITE, dst, n))) return st;
    if (l->tracked(src, n) && (st = l->access(f, CUSAN_READ, src, n))) return st;
    if ((st = l->epilogue(f))) return st;
    if (!async && kind != CUSAN_D2D)
        return l->sync(CUSAN_ACQUIRE, l->H(), K_stream(f));
    return CUSAN_OK;
}

int cusan_on_memset(cusan_lowering* l, uint64_t ptr, uint64_t n, int async, uint64_t stream) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t f = 0;
    int st = l->fiber_of(async ? stream : 0, &f);
    if (st || (st = l->prologue(f))) return st;
    auto* a = l->find(ptr);
    if (l->tracked(ptr, n) && (st = l->access(f, CUSAN_WRITE, ptr, n))) return st;
    if ((st = l->epilogue(f))) return st;
    if (!async && a && a->kind == CUSAN_MEM_PINNED)
        return l->sync(CUSAN_ACQUIRE, l->H(), K_stream(f));
    return CUSAN_OK;
}

int cusan_on_host_access(cusan_lowering* l, uint64_t addr, uint64_t n, enum cusan_mode mode) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    return l->access(l->H(), mode ? CUSAN_WRITE : CUSAN_READ, addr, n);
}

static int mpi_nonblocking(cusan_lowering* l, uint64_t buf, uint64_t n, uint64_t req, int mode) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t m = 0;
    if (!l->mpi_free.empty()) {            // recycled only after completion
        std::pop_heap(l->mpi_free.begin(), l->mpi_free.end(), std::greater<uint32_t>());   // lowest id
        m = l->mpi_free.back();
        l->mpi_free.pop_back();
    } else {
        int st = l->new_fiber(&m);
        if (st) return st;
    }
    l->req_fiber[req] = m;
    l->note(m, CUSAN_FIBER_MPI_REQUEST, req);
    int st = l->sync(CUSAN_FORK, m, l->H());   // fiber per non-blocking request
    if (st || (st = l->access(m, mode, buf, n))) return st;
    return l->sync(CUSAN_RELEASE, m, K_req(req));
}

int cusan_on_mpi_isend(cusan_lowering* l, uint64_t buf, uint64_t n, uint64_t req) {
    return mpi_nonblocking(l, buf, n, req, CUSAN_READ);
}

int cusan_on_mpi_irecv(cusan_lowering* l, uint64_t buf, uint64_t n, uint64_t req) {
    return mpi_nonblocking(l, buf, n, req, CUSAN_WRITE);
}

int cusan_on_mpi_wait(cusan_lowering* l, uint64_t req) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    int st = l->sync(CUSAN_ACQUIRE, l->H(), K_req(req));
    if (st) return st;
    if (const uint32_t* it = l->req_fiber.get(req)) {
        l->mpi_free.push_back(*it);
        std::push_heap(l->mpi_free.begin(), l->mpi_free.end(), std::greater<uint32_t>());
        l->req_fiber.erase(req);
    }
    return CUSAN_OK;
}

int cusan_on_mpi_test(cusan_lowering* l, uint64_t req, int flag) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    return flag ? cusan_on_mpi_wait(l, req) : CUSAN_OK;
}

int cusan_on_mpi_send(cusan_lowering* l, uint64_t buf, uint64_t n) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    return l->access(l->H(), CUSAN_READ, buf, n);
}

int cusan_on_mpi_recv(cusan_lowering* l, uint64_t buf, uint64_t n) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    return l->access(l->H(), CUSAN_WRITE, buf, n);
}

int cusan_on_thread(cusan_lowering* l, uint64_t thread) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t f = 0;
    int st = l->thread_fiber_of(thread, &f);
    if (!st) {
        l->thread = thread;
        l->h_fiber = f;
    }
    return st;
}

int cusan_on_thread_create(cusan_lowering* l, uint64_t child) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    uint32_t f = 0;
    int st = l->thread_fiber_of(child, &f);
    return st ? st : l->sync(CUSAN_FORK, f, l->H());           // creation is an issue edge
}

int cusan_on_thread_join(cusan_lowering* l, uint64_t child) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    const uint32_t* it = l->thread_fiber.get(child);
    if (!it) return CUSAN_OK;
    int st = l->sync(CUSAN_RELEASE, *it, K_thread(child));   // the child's end ...
    return st ? st : l->sync(CUSAN_ACQUIRE, l->H(), K_thread(child));   // ... HB the join
}

int cusan_lowering_set_default_stream(cusan_lowering* l, int per_thread) {
    if (!l) return fail(CUSAN_EINVAL, "lowering is null");
    l->per_thread_mode = per_thread != 0;
    return CUSAN_OK;
}

int cusan_lower_program(cusan_lowering* l, const cusan_api_call* calls, uint64_t n,
                        const cusan_api_arg* args, uint64_t nargs, uint32_t* op_first_event) {
    if (!l || (n && !calls) || (nargs && !args)) return fail(CUSAN_EINVAL, "null argument");
    {   // room for the typical expansion (a launch is ~6 primitives), so the trace grows once
        std::vector<cusan_event>& ev = l->trace->t.ev;
        const uint64_t want = std::min<uint64_t>(ev.size() + 4 * n + nargs, CUSAN_MAX_TRACE_EVENTS);
        if (want > ev.capacity()) {
            try {
                ev.reserve(want);
            } catch (...) {
                return fail(CUSAN_ENOMEM, "cannot reserve the trace");
            }
        }
    }
    std::vector<uint64_t> ptrs;
    std::vector<uint32_t> modes;
    for (uint64_t i = 0; i < n; i++) {
        const cusan_api_call& c = calls[i];
        if (op_first_event) {
            uint64_t ne = 0;
            cusan_trace_size(l->trace, &ne, nullptr);
            op_first_event[i] = (uint32_t)ne;
        }
        int st = CUSAN_OK;
        switch (c.op) {
            case CUSAN_OP_MALLOC: st = cusan_on_malloc(l, c.a, c.b, (cusan_mem_kind)c.x); break;
            case CUSAN_OP_FREE: st = cusan_on_free(l, c.a); break;
            case CUSAN_OP_STREAM_CREATE: st = cusan_on_stream_create(l, c.s, c.x & 1); break;
            case CUSAN_OP_KERNEL: {
                if (c.b + c.x > nargs) return fail(CUSAN_EINVAL, "kernel arguments out of range");
                ptrs.resize(c.x);
                modes.resize(c.x);
                for (uint32_t j = 0; j < c.x; j++) {
                    ptrs[j] = args[c.b + j].ptr;
                    modes[j] = args[c.b + j].mode;
                }
                st = cusan_on_kernel(l, c.s, c.x, ptrs.data(), modes.data());
                break;
            }
            case CUSAN_OP_STREAM_SYNC: st = cusan_on_stream_sync(l, c.s); break;
            case CUSAN_OP_DEVICE_SYNC: st = cusan_on_device_sync(l); break;
            case CUSAN_OP_EVENT_RECORD: st = cusan_on_event_record(l, c.c, c.s); break;
            case CUSAN_OP_EVENT_SYNC: st = cusan_on_event_sync(l, c.c); break;
            case CUSAN_OP_STREAM_WAIT_EVENT: st = cusan_on_stream_wait_event(l, c.s, c.c); break;
            case CUSAN_OP_STREAM_QUERY: st = cusan_on_stream_query(l, c.s, (int)c.x); break;
            case CUSAN_OP_MEMCPY: st = cusan_on_memcpy(l, c.a, c.b, c.c, (cusan_copy_kind)c.x, 0, 0); break;
            case CUSAN_OP_MEMCPY_ASYNC:
                st = cusan_on_memcpy(l, c.a, c.b, c.c, (cusan_copy_kind)c.x, 1, c.s);
                break;
            case CUSAN_OP_MEMSET: st = cusan_on_memset(l, c.a, c.c, 0, 0); break;
            case CUSAN_OP_MEMSET_ASYNC: st = cusan_on_memset(l, c.a, c.c, 1, c.s); break;
            case CUSAN_OP_HOST_ACCESS: st = cusan_on_host_access(l, c.a, c.c, (cusan_mode)(c.x ? 1 : 0)); break;
            case CUSAN_OP_MPI_ISEND: st = cusan_on_mpi_isend(l, c.a, c.c, c.b); break;
            case CUSAN_OP_MPI_IRECV: st = cusan_on_mpi_irecv(l, c.a, c.c, c.b); break;
            case CUSAN_OP_MPI_WAIT: st = cusan_on_mpi_wait(l, c.b); break;
            case CUSAN_OP_MPI_TEST: st = cusan_on_mpi_test(l, c.b, (int)c.x); break;
            case CUSAN_OP_MPI_SEND: st = cusan_on_mpi_send(l, c.a, c.c); break;
            case CUSAN_OP_MPI_RECV: st = cusan_on_mpi_recv(l, c.a, c.c); break;
            case CUSAN_OP_SET_THREAD: st = cusan_on_thread(l, c.a); break;
            case CUSAN_OP_THREAD_CREATE: st = cusan_on_thread_create(l, c.a); break;
            case CUSAN_OP_THREAD_JOIN: st = cusan_on_thread_join(l, c.a); break;
            case CUSAN_OP_DEFAULT_STREAM: st = cusan_lowering_set_default_stream(l, (int)c.x); break;
            default: return fail(CUSAN_EINVAL, "unknown API op");
        }
        if (st) return st;
    }
    return CUSAN_OK;
}

}  // extern "C"
