// Host preparation of a check (steps a1 and a2).
//
// a1  vector-clock / segment pass.  One pass over the trace keeps the current vector clock C_f of
//     every fiber and the sync clock SC_k of every key (TSan annotation semantics, PAPER.md:164-173;
//     fibers PAPER.md:178-186).  A fiber's clock entries for *other* fibers change only at an
//     ACQUIRE or an incoming FORK, so the accesses of a fiber between two such events share one
//     "segment" row segvc[seg][0..F) = C_f.  The shadow kernel's happens-before test for an earlier
//     epoch (g, i+1) against a later access of fiber f in segment s is then
//         g == f  ||  i+1 <= segvc[s][g]
//     Rows are created lazily at the first access after a segment opens (no row for a segment
//     without accesses).
//
// a2  range -> granule expansion and compaction.  Granule = addr >> 3 and an access covers
//     [addr >> 3, (addr + n + 7) >> 3).  All access endpoints split the granule space into
//     elementary intervals; the covered ones are numbered densely (the shadow index space), each with
//     its list of covering accesses in trace order (its "incidences").  The space is cut into
//     `nshards` contiguous dense ranges of equal coverage weight (Σ granules × incidences), and this
//     plan keeps the clip of its shard.  Windows are runs of `window_events` consecutive accesses;
//     a window's spans are its incidences grouped by interval.
#include <sched.h>

#include <algorithm>
#include <bitset>
#include <chrono>
#include <condition_variable>
#include <cstdio>
#include <cstdlib>
#include <functional>
#include <future>
#include <mutex>
#include <thread>
#include <unordered_map>

#include "common.h"

namespace cusan {

// Host threads for the planning loops (1 for small traces).  One core stays free for the thread
// that launches and waits on the device work (pipelined checks plan while a check runs).  The cores
// are those this process may run on (its affinity mask, which follows container cpusets), shared
// among the ranks of the node when torchrun says how many there are (LOCAL_WORLD_SIZE), so 8 ranks
// on one host do not each start a pool the size of the machine.  CUSAN_PLAN_THREADS overrides.
static unsigned max_plan_threads() {
    static const unsigned n = [] {
        if (const char* e = std::getenv("CUSAN_PLAN_THREADS")) {
            const long v = std::strtol(e, nullptr, 10);
            if (v > 0) return (unsigned)std::min<long>(v, 256);
        }
        unsigned hw = std::max(1u, std::thread::hardware_concurrency());
        cpu_set_t set;
        if (sched_getaffinity(0, sizeof(set), &set) == 0) hw = std::max(1, CPU_COUNT(&set));
        if (const char* e = std::getenv("LOCAL_WORLD_SIZE")) {
            const long ranks = std::strtol(e, nullptr, 10);
            if (ranks > 1) hw = std::max<unsigned>(1, hw / (unsigned)ranks);
        }
        return std::max(1u, std::min<unsigned>(hw > 2 ? hw - 1 : hw, 16));
    }();
    return n;
}
static unsigned plan_threads(uint64_t work) {
    if (work < (1u << 15)) return 1;
    return max_plan_threads();
}

// A persistent pool of planning threads (created on first use, never torn down): a parallel loop
// costs a wake-up instead of thread creation.  One loop at a time; a concurrent caller (another host
// thread planning) falls back to its own threads.
class Pool {
  public:
    explicit Pool(unsigned workers) {
        for (unsigned i = 0; i < workers; i++) th_.emplace_back([this] { loop(); });
    }
    unsigned size() const { return (unsigned)th_.size() + 1; }
    std::mutex busy;                                // held by the caller for a whole loop
    void run(unsigned T, const std::function<void(unsigned)>& fn) {
        {
            std::lock_guard<std::mutex> lk(m_);
            job_ = &fn;
            njobs_ = T;
            next_ = 1;
            pending_ = T - 1;
            gen_++;
        }
        cv_.notify_all();
        fn(0u);
        std::unique_lock<std::mutex> lk(m_);
        done_.wait(lk, [&] { return pending_ == 0; });
        job_ = nullptr;
    }

  private:
    void loop() {
        uint64_t seen = 0;
        std::unique_lock<std::mutex> lk(m_);
        for (;;) {
            cv_.wait(lk, [&] { return gen_ != seen; });
            seen = gen_;
            while (job_ && next_ < njobs_) {
                const unsigned t = next_++;
                const std::function<void(unsigned)>* f = job_;
                lk.unlock();
                (*f)(t);
                lk.lock();
                if (--pending_ == 0) done_.notify_one();
            }
        }
    }
    std::vector<std::thread> th_;
    std::mutex m_;
    std::condition_variable cv_, done_;
    const std::function<void(unsigned)>* job_ = nullptr;
    unsigned njobs_ = 0, next_ = 0, pending_ = 0;
    uint64_t gen_ = 0;
};

static Pool& pool() {
    static Pool* p = new Pool(max_plan_threads() - 1);
    return *p;
}

template <class Fn>
static void parallel_for(unsigned T, Fn&& fn) {
    if (T <= 1) {
        fn(0u);
        return;
    }
    Pool& P = pool();
    std::unique_lock<std::mutex> lk(P.busy, std::try_to_lock);
    if (lk && T <= P.size()) {
        P.run(T, std::function<void(unsigned)>(fn));
        return;
    }
    std::vector<std::thread> th;
    th.reserve(T - 1);
    for (unsigned t = 1; t < T; t++) th.emplace_back(fn, t);
    fn(0u);
    for (auto& x : th) x.join();
}

// Stable LSD radix sort of (key, id) pairs by key: 11-bit digits over the bits in which the keys
// differ (granule numbers of one address space: a few passes).
static void radix_sort_pairs(std::vector<uint64_t>& key, std::vector<uint32_t>& id) {
    const size_t n = key.size();
    if (n < 2) return;
    const auto mm = std::minmax_element(key.begin(), key.end());
    const uint64_t mn = *mm.first, span = *mm.second - mn;
    const int bits = span ? 64 - __builtin_clzll(span) : 0;
    std::vector<uint64_t> k2(n);
    std::vector<uint32_t> i2(n);
    for (int sh = 0; sh < bits; sh += 11) {
        std::vector<size_t> cnt(2049, 0);
        for (size_t i = 0; i < n; i++) cnt[((key[i] - mn) >> sh & 2047) + 1]++;
        for (int d = 0; d < 2048; d++) cnt[d + 1] += cnt[d];
        for (size_t i = 0; i < n; i++) {
            const size_t at = cnt[(key[i] - mn) >> sh & 2047]++;
            k2[at] = key[i];
            i2[at] = id[i];
        }
        key.swap(k2);
        id.swap(i2);
    }
}

// a1.  Two passes.
//  (1) Serial, cheap: which events open a segment (the first access of a fiber after an ACQUIRE or
//      an incoming FORK), the segment id and epoch of every access (acc_rec), the sync-clock slot of
//      every sync event, the Table I counters.
//  (2) The vector clocks.  Column g of every clock (C_f[g] for all fibers f, SC_k[g] for all keys k)
//      evolves independently of the other columns — each primitive is an element-wise max, copy or
//      tick — so the columns are split among threads, each replaying the whole trace on its columns
//      and writing them into the segment rows.  Same rows as one pass over whole clocks.
// a1 in ONE pass with whole clock rows, on one thread: the default.  Every primitive is a row
// operation (max, copy, tick), so rows padded to a multiple of 8 u32 make each one a few 256-bit
// vector instructions (the function is compiled for AVX2 as well as the baseline ISA, chosen at load
// time); one pass reads the trace once and leaves the other cores to the stages a pipelined checker
// runs beside it (lowering, device planning).  Same segment rows, records and counters as the
// two-pass column form below (CUSAN_A1_COLUMNS=1 selects that one; tests compare the two).
static inline void row_max(uint32_t* __restrict__ d, const uint32_t* __restrict__ s, uint32_t n) {
    for (uint32_t g = 0; g < n; g++) d[g] = d[g] > s[g] ? d[g] : s[g];
}

__attribute__((target_clones("avx2", "default")))
static std::pair<int, std::string> run_a1_fused(const Trace& t, HostPlan& hp, bool fill_accesses) {
    constexpr uint32_t NO_SEG = 0xffffffffu;
    const uint64_t n = t.ev.size();
    cusan_counters& c = hp.ctr;
    uint32_t F;
    if (fill_accesses) {                   // the accesses, the clock width and the counters too
        c = cusan_counters{};
        c.n_events = n;
        F = 1;
        uint64_t n_acc = 0, nseg = 0;
        std::vector<char> open(CUSAN_MAX_FIBERS + 1, 0);   // segments, counted for the row allocation
        for (const cusan_event& e : t.ev) {
            F = std::max<uint32_t>(F, e.fiber + 1);
            if (e.fiber > CUSAN_MAX_FIBERS) continue;
            if (e.kind == CUSAN_EV_ACCESS) {
                n_acc++;
                nseg += !open[e.fiber];
                open[e.fiber] = 1;
            } else if (e.kind == CUSAN_EV_ACQUIRE || e.kind == CUSAN_EV_FORK) {
                if (e.kind == CUSAN_EV_FORK) F = std::max<uint32_t>(F, (uint32_t)e.a + 1);
                open[e.fiber] = 0;
            }
        }
        hp.nseg_count = nseg;
        if (F > CUSAN_MAX_FIBERS + 1) return {CUSAN_EINVAL, "fiber id beyond the trace's fibers"};
        hp.F = F;
        c.n_fibers = F;
        hp.acc_g0.resize(n_acc);
        hp.acc_g1.resize(n_acc);
        hp.acc_rec.resize(n_acc);
        hp.acc_event.clear();
    } else {
        F = hp.F;
    }
    const uint32_t FP = (F + 7) & ~7u;     // padded row (the padding columns stay 0)
    std::vector<uint32_t> C((size_t)F * FP, 0), S;
    S.reserve((size_t)1024 * FP);
    std::vector<uint32_t> cur_seg(F, NO_SEG);
    KeySlots key_slot;
    hp.nseg = 0;
    hp.segvc.clear();
    hp.segvc.reserve(hp.nseg_count * F);     // counted by the access scan (0: rows grow as they come)
    uint64_t k = 0;
    for (uint64_t i = 0; i < n; i++) {
        const cusan_event& e = t.ev[i];
        const uint32_t f = e.fiber;
        if (f >= F) return {CUSAN_EINVAL, "fiber id beyond the trace's fibers"};
        uint32_t* Cf = &C[(size_t)f * FP];
        const uint32_t tick = (uint32_t)(i + 1);
        switch (e.kind) {
            case CUSAN_EV_FORK: {                  // an event of src: C_src[src] := i+1; C_dst ⊔= C_src
                const uint32_t src = (uint32_t)e.a;
                if (src >= F) return {CUSAN_EINVAL, "fiber id beyond the trace's fibers"};
                uint32_t* Cs = &C[(size_t)src * FP];
                Cs[src] = tick;
                if (src != f) row_max(Cf, Cs, FP);
                cur_seg[f] = NO_SEG;               // opens a segment on dst
                c.n_fork++;
                break;
            }
            case CUSAN_EV_ACCESS: {
                Cf[f] = tick;
                if (cur_seg[f] == NO_SEG) {        // a segment opens: its row is C_f
                    if (hp.nseg >= 0x7fffffffu) return {CUSAN_ERANGE, "too many segments"};
                    cur_seg[f] = (uint32_t)hp.nseg++;
                    hp.segvc.insert(hp.segvc.end(), Cf, Cf + F);
                }
                if (fill_accesses) {
                    hp.acc_g0[k] = e.a >> 3;
                    hp.acc_g1[k] = e.b ? (e.a + e.b + 7) >> 3 : e.a >> 3;
                }
                hp.acc_rec[k] = {pack_epoch(f, (uint32_t)i), cur_seg[f] | ((uint32_t)e.mode << 31)};
                const uint64_t bytes = 8 * (hp.acc_g1[k] - hp.acc_g0[k]);
                k++;
                c.n_access++;
                c.tracked_bytes += bytes;
                if (e.mode) { c.n_write++; c.bytes_written += bytes; }
                else { c.n_read++; c.bytes_read += bytes; }
                break;
            }
            case CUSAN_EV_RELEASE:
            case CUSAN_EV_RELEASE_STORE:
            case CUSAN_EV_ACQUIRE: {
                Cf[f] = tick;
                bool fresh;
                const uint32_t slot = key_slot.get(e.a, &fresh);
                if (fresh) S.resize(S.size() + FP, 0u);
                uint32_t* Sk = &S[(size_t)slot * FP];
                if (e.kind == CUSAN_EV_RELEASE) {              // SC_k := SC_k ⊔ C_f
                    row_max(Sk, Cf, FP);
                    c.n_release++;
                } else if (e.kind == CUSAN_EV_RELEASE_STORE) { // SC_k := C_f
                    std::copy(Cf, Cf + FP, Sk);
                    c.n_release_store++;
                } else {                                       // C_f := C_f ⊔ SC_k
                    row_max(Cf, Sk, FP);
                    cur_seg[f] = NO_SEG;
                    c.n_acquire++;
                }
                break;
            }
            default:
                return {CUSAN_EINVAL, "bad event kind in trace"};
        }
    }
    c.n_segments = hp.nseg;
    return {CUSAN_OK, ""};
}

std::pair<int, std::string> run_a1(const Trace& t, HostPlan& hp, unsigned threads, bool fill_accesses) {
    const auto t_start = std::chrono::steady_clock::now();
    static const bool columns = [] {
        const char* e = std::getenv("CUSAN_A1_COLUMNS");
        return e && *e && *e != '0';
    }();
    if (!columns) {
        std::pair<int, std::string> st = run_a1_fused(t, hp, fill_accesses);
        if (std::getenv("CUSAN_DEBUG_TIMING"))
            std::fprintf(stderr, "run_a1: one pass %.3f ms (%llu events, %llu segments)\n",
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count(),
                         (unsigned long long)t.ev.size(), (unsigned long long)hp.nseg);
        return st;
    }
    const uint64_t n = t.ev.size();
    cusan_counters& c = hp.ctr;
    if (fill_accesses) {                   // one pass: the accesses, the clock width and the counters too
        c = cusan_counters{};
        c.n_events = n;
        hp.acc_g0.clear();
        hp.acc_g1.clear();
        hp.acc_rec.clear();
        hp.acc_event.clear();
        hp.acc_g0.reserve(n);
        hp.acc_g1.reserve(n);
        hp.acc_rec.reserve(n);
        hp.F = 1;
    }
    uint32_t F = fill_accesses ? CUSAN_MAX_FIBERS + 1 : hp.F;   // (cur_seg size; the width is set below)
    uint32_t f_max = 1;
    constexpr uint32_t NO_SEG = 0xffffffffu;
    // The column pass replays only the events that move clock values: forks, syncs and the accesses
    // that open a segment (their row is the fiber's clock).  A fiber's tick at any other access is
    // dead: every later read of C_f[f] — a release, a fork from f, a segment row — follows a tick of
    // its own, so the value is overwritten first.
    struct Op {
        uint8_t kind;
        uint32_t f, aux, tick;             // aux: key slot (sync) / segment (access) / source (fork)
    };
    std::vector<Op> ops;
    ops.reserve(n);
    std::vector<uint32_t> cur_seg(F, NO_SEG);
    KeySlots key_slot;
    hp.nseg = 0;
    uint64_t k = 0;
    for (uint64_t i = 0; i < n; i++) {
        const cusan_event& e = t.ev[i];
        const uint32_t f = e.fiber;
        f_max = std::max(f_max, f + 1);
        switch (e.kind) {
            case CUSAN_EV_FORK:                    // an event of src's program order; opens a segment on dst
                cur_seg[f] = NO_SEG;
                ops.push_back({CUSAN_EV_FORK, f, (uint32_t)e.a, (uint32_t)(i + 1)});
                f_max = std::max(f_max, (uint32_t)e.a + 1);
                c.n_fork++;
                break;
            case CUSAN_EV_ACCESS: {
                if (cur_seg[f] == NO_SEG) {
                    if (hp.nseg >= 0x7fffffffu) return {CUSAN_ERANGE, "too many segments"};
                    cur_seg[f] = (uint32_t)hp.nseg++;
                    ops.push_back({CUSAN_EV_ACCESS, f, cur_seg[f], (uint32_t)(i + 1)});
                }
                if (fill_accesses) {
                    hp.acc_g0.push_back(e.a >> 3);
                    hp.acc_g1.push_back(e.b ? (e.a + e.b + 7) >> 3 : e.a >> 3);
                    hp.acc_rec.push_back({pack_epoch(f, (uint32_t)i), cur_seg[f] | ((uint32_t)e.mode << 31)});
                } else {
                    hp.acc_rec[k] = {pack_epoch(f, (uint32_t)i), cur_seg[f] | ((uint32_t)e.mode << 31)};
                }
                const uint64_t bytes = 8 * (hp.acc_g1[k] - hp.acc_g0[k]);
                k++;
                c.n_access++;
                c.tracked_bytes += bytes;
                if (e.mode) { c.n_write++; c.bytes_written += bytes; }
                else { c.n_read++; c.bytes_read += bytes; }
                break;
            }
            case CUSAN_EV_RELEASE:
            case CUSAN_EV_RELEASE_STORE:
            case CUSAN_EV_ACQUIRE: {
                bool fresh;
                ops.push_back({e.kind, f, key_slot.get(e.a, &fresh), (uint32_t)(i + 1)});
                if (e.kind == CUSAN_EV_ACQUIRE) { cur_seg[f] = NO_SEG; c.n_acquire++; }
                else if (e.kind == CUSAN_EV_RELEASE) c.n_release++;
                else c.n_release_store++;
                break;
            }
            default:
                return {CUSAN_EINVAL, "bad event kind in trace"};
        }
    }
    c.n_segments = hp.nseg;
    if (fill_accesses) {
        hp.F = F = f_max;
        c.n_fibers = F;
    }
    if (std::getenv("CUSAN_DEBUG_TIMING"))
        std::fprintf(stderr, "run_a1: pre-pass %.3f ms (%zu of %llu events replayed)\n",
                     std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count(),
                     ops.size(), (unsigned long long)n);
    static const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    const auto t_pre = std::chrono::steady_clock::now();
    hp.segvc.resize(hp.nseg * F);
    const uint32_t nkeys = key_slot.size();
    const uint64_t nops = ops.size();
    // columns per thread: multiples of 8, at least 8 (one AVX2 vector of u32)
    const unsigned T = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>({threads, (F + 7) / 8, nops / 4096 + 1}));
    parallel_for(T, [&](unsigned th) {
        const uint32_t c0 = (uint32_t)((uint64_t)((F + 7) / 8) * th / T) * 8;
        const uint32_t c1 = std::min<uint32_t>(F, (uint32_t)((uint64_t)((F + 7) / 8) * (th + 1) / T) * 8);
        if (c0 >= c1) return;
        const uint32_t G = c1 - c0;
        std::vector<uint32_t> C((size_t)F * G, 0), S((size_t)nkeys * G, 0);
        uint32_t* segvc = hp.segvc.data();
        for (uint64_t q = 0; q < nops; q++) {
            const Op o = ops[q];
            const uint32_t f = o.f;
            uint32_t* __restrict__ Cf = &C[(size_t)f * G];
            if (o.kind == CUSAN_EV_FORK) {         // C_src[src] := i+1; C_dst := C_dst ⊔ C_src
                const uint32_t src = o.aux;
                uint32_t* __restrict__ Cs = &C[(size_t)src * G];
                if (src >= c0 && src < c1) Cs[src - c0] = o.tick;
                if (src != f)
                    for (uint32_t g = 0; g < G; g++) Cf[g] = std::max(Cf[g], Cs[g]);
                continue;
            }
            if (f >= c0 && f < c1) Cf[f - c0] = o.tick;
            if (o.kind == CUSAN_EV_ACCESS) {       // a segment opens: its row is C_f
                std::copy(Cf, Cf + G, segvc + (size_t)o.aux * F + c0);
                continue;
            }
            uint32_t* __restrict__ Sk = &S[(size_t)o.aux * G];
            if (o.kind == CUSAN_EV_RELEASE)        // SC_k := SC_k ⊔ C_f
                for (uint32_t g = 0; g < G; g++) Sk[g] = std::max(Sk[g], Cf[g]);
            else if (o.kind == CUSAN_EV_RELEASE_STORE)   // SC_k := C_f
                std::copy(Cf, Cf + G, Sk);
            else                                   // C_f := C_f ⊔ SC_k
                for (uint32_t g = 0; g < G; g++) Cf[g] = std::max(Cf[g], Sk[g]);
        }
    });
    if (dbg)
        std::fprintf(stderr, "run_a1: segvc resize + column pass %.3f ms on %u threads (%u keys)\n",
                     std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_pre).count(), T,
                     nkeys);
    return {CUSAN_OK, ""};
}

// The accesses of a trace (granule ranges, event ids) and the clock width; resets the counters.
static void prepare_accesses(const Trace& t, HostPlan& hp) {
    // clock width = fibers the trace actually uses (≤ max_fibers); the accesses' granule ranges
    uint32_t F = 1;
    uint64_t n_acc = 0;
    for (const auto& e : t.ev) {
        F = std::max<uint32_t>(F, e.fiber + 1);
        if (e.kind == CUSAN_EV_FORK) F = std::max<uint32_t>(F, (uint32_t)e.a + 1);
        n_acc += e.kind == CUSAN_EV_ACCESS;
    }
    hp.F = F;
    cusan_counters& c = hp.ctr;
    c = cusan_counters{};
    c.n_events = t.ev.size();
    c.n_fibers = F;
    hp.acc_g0.resize(n_acc);
    hp.acc_g1.resize(n_acc);
    hp.acc_event.resize(n_acc);
    hp.acc_rec.resize(n_acc);
    {
        uint64_t k = 0, nseg = 0;
        std::vector<char> open(F, 0);             // segments, counted for a1's row allocation
        for (uint64_t i = 0; i < t.ev.size(); i++) {
            const cusan_event& e = t.ev[i];
            if (e.kind != CUSAN_EV_ACCESS) {
                if (e.kind == CUSAN_EV_ACQUIRE || e.kind == CUSAN_EV_FORK) open[e.fiber] = 0;
                continue;
            }
            nseg += !open[e.fiber];
            open[e.fiber] = 1;
            hp.acc_g0[k] = e.a >> 3;
            hp.acc_g1[k] = e.b ? (e.a + e.b + 7) >> 3 : e.a >> 3;
            hp.acc_event[k] = (uint32_t)i;
            k++;
        }
        hp.nseg_count = nseg;
    }
}

// The first part of a device-planned plan: options checked, the accesses' granule ranges; a1 follows
// (run_a1) while the device builds the intervals from the ranges.
int prepare_plan_accesses(const Trace& t, const cusan_check_opts& o, HostPlan& hp) {
    if (o.nshards < 1 || o.shard < 0 || o.shard >= o.nshards)
        return fail(CUSAN_EINVAL, "need 0 <= shard < nshards");
    if (o.window_events < 0) return fail(CUSAN_EINVAL, "window_events must be >= 0");
    if (int st = check_flags(o)) return st;
    if (t.ev.size() > CUSAN_MAX_EVENTS)
        return fail(CUSAN_ERANGE, "a one-shot check takes at most 2^24-2 events (sessions renumber longer traces)");
    hp.opts = o;
    prepare_accesses(t, hp);
    return CUSAN_OK;
}

unsigned a1_threads_for(uint64_t n_events) { return plan_threads(n_events); }

// a1 alone for a clocks object (cusan_clocks_compute): every core of the node — on a multi-GPU
// node one rank computes the clocks while the others wait for the broadcast.
int compute_clocks(const Trace& t, HostPlan& hp) {
    if (t.ev.size() > CUSAN_MAX_EVENTS)
        return fail(CUSAN_ERANGE, "a one-shot check takes at most 2^24-2 events (sessions renumber longer traces)");
    unsigned hw = std::max(1u, std::thread::hardware_concurrency());
    cpu_set_t set;
    if (sched_getaffinity(0, sizeof(set), &set) == 0) hw = std::max(1, CPU_COUNT(&set));
    if (const char* e = std::getenv("CUSAN_PLAN_THREADS")) {
        const long v = std::strtol(e, nullptr, 10);
        if (v > 0) hw = (unsigned)std::min<long>(v, 256) + 1;
    }
    const unsigned T = (uint64_t)t.ev.size() < (1u << 15) ? 1 : std::max(1u, std::min(hw > 1 ? hw - 1 : 1, 32u));
    const std::pair<int, std::string> st = run_a1(t, hp, T, true);
    return st.first ? fail(st.first, st.second) : CUSAN_OK;
}

int check_flags(const cusan_check_opts& o) {
    const int known = CUSAN_CHECK_DEFER_WORKSPACE | CUSAN_CHECK_INTERVAL_SHADOW | CUSAN_CHECK_DENSE_SHADOW |
                      CUSAN_CHECK_HOST_PLAN | CUSAN_CHECK_DEVICE_PLAN;
    if (o.flags & ~known) return fail(CUSAN_EINVAL, "unknown cusan_check_opts.flags bits");
    if ((o.flags & CUSAN_CHECK_INTERVAL_SHADOW) && (o.flags & CUSAN_CHECK_DENSE_SHADOW))
        return fail(CUSAN_EINVAL, "CUSAN_CHECK_INTERVAL_SHADOW and CUSAN_CHECK_DENSE_SHADOW exclude each other");
    if ((o.flags & CUSAN_CHECK_HOST_PLAN) && (o.flags & CUSAN_CHECK_DEVICE_PLAN))
        return fail(CUSAN_EINVAL, "CUSAN_CHECK_HOST_PLAN and CUSAN_CHECK_DEVICE_PLAN exclude each other");
    return CUSAN_OK;
}

int build_host_plan(const Trace* tp, const cusan_check_opts& o, HostPlan& hp, uint64_t first_access,
                    uint64_t rec_base, bool a1_only) {
    if (o.nshards < 1 || o.shard < 0 || o.shard >= o.nshards)
        return fail(CUSAN_EINVAL, "need 0 <= shard < nshards");
    if (o.window_events < 0) return fail(CUSAN_EINVAL, "window_events must be >= 0");
    if (int st = check_flags(o)) return st;
    if (tp && tp->ev.size() > CUSAN_MAX_EVENTS)
        return fail(CUSAN_ERANGE, "a one-shot check takes at most 2^24-2 events (sessions renumber longer traces)");
    hp.opts = o;
    const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    auto tick = [t0 = std::chrono::steady_clock::now(), dbg](const char* what) {
        if (dbg)
            std::fprintf(stderr, "build_host_plan: %-12s %8.3f ms\n", what,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    };
    // (no trace: hp holds the accesses and a1's products; a1 only: one fused pass below)
    if (tp && !a1_only) prepare_accesses(*tp, hp);
    const uint64_t n_acc = hp.acc_g0.size();
    cusan_counters& c = hp.ctr;
    // ---------------------------------------------------------------- a1: clocks and segments --
    // Runs on its own thread while a2 builds the intervals (a2 needs a1's records only to fill the
    // incidence table at the end).  Errors come back as (status, message).
    const unsigned a1_threads = plan_threads(tp ? (uint64_t)tp->ev.size() : 0);
    auto a1 = [&]() -> std::pair<int, std::string> {
        if (!tp) return {CUSAN_OK, ""};
        const auto a1_t0 = std::chrono::steady_clock::now();
        std::pair<int, std::string> st = run_a1(*tp, hp, a1_threads, a1_only);
        tick("a1 (thread)");
        if (dbg)
            std::fprintf(stderr, "build_host_plan: a1 alone     %8.3f ms (%llu segments, %u threads)\n",
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - a1_t0).count(),
                         (unsigned long long)hp.nseg, a1_threads);
        return st;
    };
    tick("acc scan");
    if (a1_only) {                     // a2 runs on the device (plan_dev.cu)
        const std::pair<int, std::string> st = a1();
        return st.first ? fail(st.first, st.second) : CUSAN_OK;
    }
    const bool concurrent = n_acc >= (1u << 12);
    std::future<std::pair<int, std::string>> a1_done;
    std::pair<int, std::string> a1_status{CUSAN_OK, ""};
    if (concurrent) a1_done = std::async(std::launch::async, a1);
    else a1_status = a1();
    // joins a1 (at the latest when the plan is left early)
    struct Join {
        std::future<std::pair<int, std::string>>* f;
        std::pair<int, std::string>* out;
        ~Join() { if (f->valid()) *out = f->get(); }
    } a1_join{&a1_done, &a1_status};
    auto a1_finish = [&]() -> int {
        if (a1_done.valid()) a1_status = a1_done.get();
        tick("a1 clocks");
        return a1_status.first ? fail(a1_status.first, a1_status.second) : CUSAN_OK;
    };

    // ---------------------------------------------------------------- a2: elementary intervals --
    // Endpoints of the non-empty accesses, radix-sorted with their access ids: the distinct values
    // are the interval boundaries B, and each endpoint's rank is its boundary index (b0, b1).
    std::vector<uint32_t> b0(n_acc, 0), b1(n_acc, 0);
    std::vector<uint64_t> B;
    {
        std::vector<uint64_t> ek;
        std::vector<uint32_t> eid;
        ek.reserve(2 * n_acc);
        eid.reserve(2 * n_acc);
        for (uint64_t k = 0; k < n_acc; k++)
            if (hp.acc_g1[k] > hp.acc_g0[k]) {
                ek.push_back(hp.acc_g0[k]);
                eid.push_back((uint32_t)(2 * k));
                ek.push_back(hp.acc_g1[k]);
                eid.push_back((uint32_t)(2 * k + 1));
            }
        tick("a2 endpoints");
        radix_sort_pairs(ek, eid);
        tick("a2 sort");
        B.reserve(ek.size());
        for (size_t i = 0; i < ek.size(); i++) {
            if (i == 0 || ek[i] != ek[i - 1]) B.push_back(ek[i]);
            ((eid[i] & 1) ? b1 : b0)[eid[i] >> 1] = (uint32_t)(B.size() - 1);
        }
    }
    tick("a2 bounds");
    const uint64_t nb = B.size();
    // coverage of elementary interval j = [B[j], B[j+1]) = the accesses covering it (difference
    // array); covered ones get ids in ascending address order.  An interval's incidence count is
    // its coverage.
    struct GIv { uint64_t abs_begin, dense_begin, len; uint32_t cnt, j; };
    std::vector<GIv> giv;
    {
        std::vector<int64_t> diff(nb + 1, 0);
        for (uint64_t k = 0; k < n_acc; k++)
            if (b1[k] > b0[k]) { diff[b0[k]]++; diff[b1[k]]--; }
        int64_t cov = 0;
        uint64_t dense = 0;
        for (uint64_t j = 0; j + 1 < nb; j++) {
            cov += diff[j];
            if (cov > 0) {
                if (cov > 0xffffffffll) return fail(CUSAN_ERANGE, "too many interval incidences");
                giv.push_back({B[j], dense, B[j + 1] - B[j], (uint32_t)cov, (uint32_t)j});
                dense += B[j + 1] - B[j];
            }
        }
    }
    c.n_intervals = giv.size();
    tick("a2 intervals");
    // ---------------------------------------------------------------- a2: shard clip ------------
    const uint64_t total_dense = giv.empty() ? 0 : giv.back().dense_begin + giv.back().len;
    uint64_t d_lo = 0, d_hi = total_dense;
    if (o.nshards > 1 && !giv.empty()) {
        // Boundaries at equal cumulative cost.  Per granule: with several windows
        // the kernel moves the cell 2(k−1) times for an interval touched in k windows (memory-bound);
        // with one window (or one cell per interval, f3) the work is the accesses replayed, so the
        // weight is the coverage (accesses covering the granule).
        const uint64_t Ws = o.window_events > 0 ? (uint64_t)o.window_events : std::max<uint64_t>(n_acc, 1);
        const bool windowed = Ws < n_acc && !compressed_shadow(o);
        std::vector<uint64_t> wpg(giv.size());
        if (!windowed) {
            for (size_t i = 0; i < giv.size(); i++) wpg[i] = std::max<uint64_t>(giv[i].cnt, 1);
        } else {
            // k per interval = windows whose accesses cover it: each window's covered boundary
            // ranges (its accesses' [b0, b1) merged) add one on a difference array
            const uint64_t nw = (n_acc + Ws - 1) / Ws;
            std::vector<std::vector<std::pair<uint32_t, uint32_t>>> wr(nw);
            const unsigned TW = (unsigned)std::min<uint64_t>(plan_threads(n_acc * 4), nw);
            parallel_for(TW, [&](unsigned t) {
                for (uint64_t w = t; w < nw; w += TW) {
                    std::vector<std::pair<uint32_t, uint32_t>> r;
                    for (uint64_t k = w * Ws; k < std::min(n_acc, (w + 1) * Ws); k++)
                        if (b1[k] > b0[k]) r.emplace_back(b0[k], b1[k]);
                    std::sort(r.begin(), r.end());
                    auto& out = wr[w];
                    for (const auto& x : r) {
                        if (!out.empty() && x.first <= out.back().second) out.back().second = std::max(out.back().second, x.second);
                        else out.push_back(x);
                    }
                }
            });
            std::vector<int64_t> kd(nb + 1, 0);
            for (const auto& out : wr)
                for (const auto& x : out) { kd[x.first]++; kd[x.second]--; }
            for (uint64_t j = 1; j <= nb; j++) kd[j] += kd[j - 1];
            for (size_t i = 0; i < giv.size(); i++) {
                const uint64_t k = (uint64_t)kd[giv[i].j];
                wpg[i] = 2 * (k ? k - 1 : 0) + 1;
            }
        }
        unsigned __int128 wtot = 0;
        for (size_t i = 0; i < giv.size(); i++) wtot += (unsigned __int128)giv[i].len * wpg[i];
        auto boundary = [&](int k) -> uint64_t {
            if (k <= 0) return 0;
            if (k >= o.nshards) return total_dense;
            unsigned __int128 target = wtot * (unsigned)k / (unsigned)o.nshards, acc = 0;
            for (size_t i = 0; i < giv.size(); i++) {
                const GIv& g = giv[i];
                unsigned __int128 w = (unsigned __int128)g.len * wpg[i];
                if (acc + w >= target) {
                    uint64_t x = (uint64_t)((target - acc + wpg[i] - 1) / wpg[i]);
                    return g.dense_begin + std::min<uint64_t>(x, g.len);
                }
                acc += w;
            }
            return total_dense;
        };
        d_lo = boundary(o.shard);
        d_hi = boundary(o.shard + 1);
    }
    // shard-local shadow slots: each clipped interval starts on a CELL_ALIGN boundary so warp
    // ranges can move their cells with aligned 128-bit accesses (≤ CELL_ALIGN−1 unused cells each)
    // (interval-compressed tracking, f3: one slot per interval).  The incidence table holds only
    // the shard's intervals, so a rank of a multi-GPU check builds and uploads only its part.
    hp.iv.clear();
    std::vector<uint32_t> iv_j;                      // elementary interval of each shard interval
    uint64_t slot = 0, n_inc = 0;
    const bool compressed = compressed_shadow(o);
    for (auto& g : giv) {
        uint64_t lo = std::max(g.dense_begin, d_lo), hi = std::min(g.dense_begin + g.len, d_hi);
        if (lo >= hi) continue;
        Interval v{};
        v.abs_begin = g.abs_begin + (lo - g.dense_begin);
        v.dense_begin = slot;
        v.len = hi - lo;
        v.list_off = (uint32_t)n_inc;
        v.list_cnt = g.cnt;
        n_inc += g.cnt;
        if (n_inc > 0xffffffffull) return fail(CUSAN_ERANGE, "too many interval incidences");
        slot = compressed ? slot + 1 : (slot + v.len + CELL_ALIGN - 1) / CELL_ALIGN * CELL_ALIGN;
        hp.iv.push_back(v);
        iv_j.push_back(g.j);
        c.tracked_bytes_shard += 8 * v.len * g.cnt;
    }
    hp.shard_granules = d_hi - d_lo;
    hp.shadow_cells = slot;
    c.shard_granules = hp.shard_granules;
    c.n_incidences = n_inc;
    tick("a2 clip");
    // incidences: per shard interval, its covering accesses in trace order (CSR).  Threads own
    // contiguous chunks of the shard's intervals (equal numbers of incidences) and each scans the
    // accesses in trace order, so every list comes out in the serial order.
    hp.inc.resize(n_inc);
    hp.inc_acc.resize(n_inc);
    {
        const size_t niv = hp.iv.size();
        const unsigned T = niv ? std::min<unsigned>(plan_threads(std::max<uint64_t>(n_acc, n_inc)), (unsigned)niv) : 1;
        std::vector<size_t> icut(T + 1, niv);
        icut[0] = 0;
        for (unsigned t = 1; t < T; t++) {
            const uint64_t want = n_inc * t / T;
            size_t lo = 0, hi = niv;                 // first interval whose list starts at >= want
            while (lo < hi) {
                const size_t m = (lo + hi) / 2;
                if (hp.iv[m].list_off < want) lo = m + 1;
                else hi = m;
            }
            icut[t] = std::max(lo, icut[t - 1]);
        }
        parallel_for(T, [&](unsigned t) {
            const size_t ia = icut[t], ib = icut[t + 1];
            if (ia >= ib) return;
            const uint32_t ja = iv_j[ia], jb = iv_j[ib - 1] + 1;
            // elementary j -> shard interval (the clip keeps at most one piece per j)
            std::vector<uint32_t> at(jb - ja, 0xffffffffu);
            for (size_t i = ia; i < ib; i++) at[iv_j[i] - ja] = hp.iv[i].list_off;
            for (uint64_t k = 0; k < n_acc; k++) {
                const uint32_t lo = std::max(b0[k], ja), hi = std::min(b1[k], jb);
                for (uint32_t j = lo; j < hi; j++) {
                    uint32_t& s = at[j - ja];
                    if (s != 0xffffffffu) hp.inc_acc[s++] = (uint32_t)k;
                }
            }
        });
    }
    tick("a2 incidence");
    if (int st = a1_finish()) return st;                 // a1's records fill the incidence table
    {
        const unsigned TI = plan_threads(n_inc);
        parallel_for(TI, [&](unsigned t) {
            const uint64_t qa = n_inc * t / TI, qb = n_inc * (t + 1) / TI;
            for (uint64_t q = qa; q < qb; q++) hp.inc[q] = hp.acc_rec[hp.inc_acc[q]];
        });
    }
    // ---------------------------------------------------------------- windows and spans ---------
    // A span that stores its final cells and ends with two or more reader fibers since the
    // interval's last write gets a pre-assigned read-set record: the cell keeps W inline and its R
    // slot points at the record holding the readers (the reader *set* depends only on the fibers
    // and modes covering the interval, never on happens-before, so its size is known here exactly).
    // Incremental checks (f1) plan only the accesses from `first_access` on; earlier incidences
    // still count for the LOAD flag and the reader sets, and records are numbered from `rec_base`.
    const uint64_t first = std::min<uint64_t>(first_access, n_acc);
    const uint64_t n_new = n_acc - first;
    const uint64_t W = o.window_events > 0 ? (uint64_t)o.window_events : std::max<uint64_t>(n_new, 1);
    hp.window_accesses = W;
    const uint64_t nwin = n_new ? (n_new + W - 1) / W : 0;
    // Two passes over contiguous chunks of intervals (equal numbers of incidences): the first counts
    // each chunk's spans per window; a prefix over (window, chunk) gives every chunk its slots in the
    // window-major order of the serial loop; the second writes the spans straight into them.
    std::vector<uint64_t> wi(hp.iv.size() + 1, 0);
    for (size_t i = 0; i < hp.iv.size(); i++) wi[i + 1] = wi[i] + hp.iv[i].list_cnt + 1;
    unsigned TS = plan_threads(wi.back() * 2);
    TS = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(TS, (1ull << 24) / std::max<uint64_t>(nwin, 1)));
    std::vector<size_t> icut(TS + 1, hp.iv.size());
    for (unsigned t = 0; t < TS; t++)
        icut[t] = (size_t)(std::lower_bound(wi.begin(), wi.end(), wi.back() * t / TS) - wi.begin());
    std::vector<std::vector<uint64_t>> at(TS, std::vector<uint64_t>(nwin, 0));
    auto window_of = [&](uint32_t q) { return (hp.inc_acc[q] - first) / W; };
    parallel_for(TS, [&](unsigned t) {
        const size_t ia = std::min(icut[t], hp.iv.size()), ib = std::min(icut[t + 1], hp.iv.size());
        std::vector<uint64_t>& n = at[t];
        for (size_t i = ia; i < ib; i++) {
            const Interval& v = hp.iv[i];
            uint32_t q = v.list_off;
            const uint32_t qe = v.list_off + v.list_cnt;
            while (q < qe && hp.inc_acc[q] < first) q++;
            uint64_t last = UINT64_MAX;
            for (; q < qe; q++) {
                const uint64_t w = window_of(q);
                if (w != last) { n[w]++; last = w; }
            }
        }
    });
    std::vector<uint64_t> wstart(nwin + 1, 0);
    {
        uint64_t pos = 0;
        for (uint64_t w = 0; w < nwin; w++) {
            wstart[w] = pos;
            for (unsigned t = 0; t < TS; t++) {
                const uint64_t n = at[t][w];
                at[t][w] = pos;
                pos += n;
            }
        }
        wstart[nwin] = pos;
    }
    hp.spans.resize(wstart[nwin]);
    parallel_for(TS, [&](unsigned t) {
        const size_t ia = std::min(icut[t], hp.iv.size()), ib = std::min(icut[t + 1], hp.iv.size());
        std::vector<uint64_t>& slot = at[t];
        for (size_t i = ia; i < ib; i++) {
            const Interval& v = hp.iv[i];
            std::bitset<CUSAN_MAX_FIBERS + 1> readers;
            uint32_t q = v.list_off, qe = v.list_off + v.list_cnt;
            for (; q < qe && hp.inc_acc[q] < first; q++) {
                const AccRec& r = hp.inc[q];
                if (r.segm >> 31) readers.reset();
                else readers.set(r.epoch >> 24);
            }
            const uint32_t first_new = q;
            while (q < qe) {
                const uint64_t w = window_of(q);
                uint32_t q2 = q;
                while (q2 < qe && window_of(q2) == w) {
                    const AccRec& r = hp.inc[q2];
                    if (r.segm >> 31) readers.reset();
                    else readers.set(r.epoch >> 24);
                    q2++;
                }
                Span& s = hp.spans[slot[w]++];
                s = Span{};
                s.abs_begin = v.abs_begin;
                s.dense_begin = v.dense_begin;
                s.len = v.len;
                s.list_off = q;
                s.list_cnt = q2 - q;
                s.flags = (q > v.list_off ? SPAN_LOAD : 0u) | ((q2 < qe || o.persist_shadow) ? SPAN_STORE : 0u) |
                          (q == first_new ? SPAN_FIRST_IN_CALL : 0u) | (compressed ? SPAN_COMPRESSED : 0u);
                const uint64_t nr = readers.count();
                if ((s.flags & SPAN_STORE) && nr >= 2)         // record index assigned below
                    s.rec_units = (uint32_t)((nr + 1 + REC_WORDS - 1) / REC_WORDS);
                q = q2;
            }
        }
    });
    hp.rec_units = 0;
    hp.spill_spans = 0;
    for (Span& s : hp.spans)
        if (s.rec_units) {
            s.rec = (uint32_t)(rec_base + hp.rec_units);
            hp.rec_units += s.rec_units;
            hp.spill_spans++;
        }
    if (rec_base + hp.rec_units >= (1u << 24) - 1)
        return fail(CUSAN_ERANGE, "too many read-set records for the 24-bit record index");
    c.spill_spans = hp.spill_spans;
    c.spill_heap_bytes = hp.rec_units * REC_WORDS * 4;
    hp.win_span_off.assign(1, 0);
    for (uint64_t w = 0; w < nwin; w++)
        if (wstart[w + 1] > wstart[w]) hp.win_span_off.push_back(wstart[w + 1]);   // skip empty windows
    c.n_windows = hp.win_span_off.size() - 1;
    c.n_spans = hp.spans.size();
    tick("spans");
    return CUSAN_OK;
}

}  // namespace cusan
