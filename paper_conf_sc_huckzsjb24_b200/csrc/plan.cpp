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

// Host threads for the planning loops (1 for small traces).
static unsigned plan_threads(uint64_t work) {
    if (work < (1u << 15)) return 1;
    const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
    return std::min<unsigned>(hw, 16);
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
    static Pool* p = new Pool(std::min<unsigned>(std::max(1u, std::thread::hardware_concurrency()), 16) - 1);
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

int build_host_plan(const Trace& t, const cusan_check_opts& o, HostPlan& hp, uint64_t first_access,
                    uint64_t rec_base) {
    if (o.nshards < 1 || o.shard < 0 || o.shard >= o.nshards)
        return fail(CUSAN_EINVAL, "need 0 <= shard < nshards");
    if (o.window_events < 0) return fail(CUSAN_EINVAL, "window_events must be >= 0");
    hp.opts = o;
    const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    auto tick = [t0 = std::chrono::steady_clock::now(), dbg](const char* what) {
        if (dbg)
            std::fprintf(stderr, "build_host_plan: %-12s %8.3f ms\n", what,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    };
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
        uint64_t k = 0;
        for (uint64_t i = 0; i < t.ev.size(); i++) {
            const cusan_event& e = t.ev[i];
            if (e.kind != CUSAN_EV_ACCESS) continue;
            hp.acc_g0[k] = e.a >> 3;
            hp.acc_g1[k] = e.b ? (e.a + e.b + 7) >> 3 : e.a >> 3;
            hp.acc_event[k] = (uint32_t)i;
            k++;
        }
    }

    // ---------------------------------------------------------------- a1: clocks and segments --
    // Runs on its own thread while a2 builds the intervals (a2 needs a1's records only to fill the
    // incidence table at the end).  Errors come back as (status, message).
    auto a1 = [&]() -> std::pair<int, std::string> {
        std::vector<uint32_t> C((size_t)F * F, 0);
        std::unordered_map<uint64_t, uint32_t> key_slot;
        std::vector<uint32_t> sc;                   // sync clocks, F entries per key
        const uint32_t NO_SEG = 0xffffffffu;
        std::vector<uint32_t> cur_seg(F, NO_SEG);
        auto sync_clock = [&](uint64_t key) -> uint32_t* {
            auto it = key_slot.find(key);
            if (it == key_slot.end()) {
                it = key_slot.emplace(key, (uint32_t)(sc.size() / F)).first;
                sc.resize(sc.size() + F, 0);
            }
            return &sc[(size_t)it->second * F];
        };
        uint64_t k = 0;
        for (uint64_t i = 0; i < t.ev.size(); i++) {
            const cusan_event& e = t.ev[i];
            const uint32_t f = e.fiber;
            uint32_t* Cf = &C[(size_t)f * F];
            if (e.kind == CUSAN_EV_FORK) {          // an event of the source fiber's program order
                const uint32_t s = (uint32_t)e.a;
                uint32_t* Cs = &C[(size_t)s * F];
                Cs[s] = (uint32_t)(i + 1);
                for (uint32_t g = 0; g < F; g++) Cf[g] = std::max(Cf[g], Cs[g]);
                cur_seg[f] = NO_SEG;                // incoming edge opens a segment on dst
                c.n_fork++;
                continue;
            }
            Cf[f] = (uint32_t)(i + 1);
            switch (e.kind) {
                case CUSAN_EV_ACCESS: {
                    if (cur_seg[f] == NO_SEG) {
                        if (hp.nseg >= 0x7fffffffu) return {CUSAN_ERANGE, "too many segments"};
                        cur_seg[f] = (uint32_t)hp.nseg++;
                        hp.segvc.insert(hp.segvc.end(), Cf, Cf + F);
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
                case CUSAN_EV_RELEASE: {            // SC_k := SC_k ⊔ C_f
                    uint32_t* S = sync_clock(e.a);
                    for (uint32_t g = 0; g < F; g++) S[g] = std::max(S[g], Cf[g]);
                    c.n_release++;
                    break;
                }
                case CUSAN_EV_RELEASE_STORE: {      // SC_k := C_f
                    uint32_t* S = sync_clock(e.a);
                    std::copy(Cf, Cf + F, S);
                    c.n_release_store++;
                    break;
                }
                case CUSAN_EV_ACQUIRE: {            // C_f := C_f ⊔ SC_k
                    uint32_t* S = sync_clock(e.a);
                    for (uint32_t g = 0; g < F; g++) Cf[g] = std::max(Cf[g], S[g]);
                    cur_seg[f] = NO_SEG;
                    c.n_acquire++;
                    break;
                }
                default:
                    return {CUSAN_EINVAL, "bad event kind in trace"};
            }
        }
        c.n_segments = hp.nseg;
        return {CUSAN_OK, ""};
    };
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
    std::vector<uint64_t> B;
    B.reserve(2 * n_acc);
    for (uint64_t k = 0; k < n_acc; k++)
        if (hp.acc_g1[k] > hp.acc_g0[k]) { B.push_back(hp.acc_g0[k]); B.push_back(hp.acc_g1[k]); }
    std::sort(B.begin(), B.end());
    B.erase(std::unique(B.begin(), B.end()), B.end());
    tick("a2 sort");
    const uint64_t nb = B.size();
    std::vector<int64_t> diff(nb + 1, 0);
    std::vector<uint32_t> b0(n_acc), b1(n_acc);
    {
        const unsigned TB = plan_threads(n_acc * 8);
        parallel_for(TB, [&](unsigned t) {
            const uint64_t ka = n_acc * t / TB, kb = n_acc * (t + 1) / TB;
            for (uint64_t k = ka; k < kb; k++) {
                if (hp.acc_g1[k] <= hp.acc_g0[k]) { b0[k] = b1[k] = 0; continue; }
                b0[k] = (uint32_t)(std::lower_bound(B.begin(), B.end(), hp.acc_g0[k]) - B.begin());
                b1[k] = (uint32_t)(std::lower_bound(B.begin(), B.end(), hp.acc_g1[k]) - B.begin());
            }
        });
        for (uint64_t k = 0; k < n_acc; k++)
            if (b1[k] > b0[k]) { diff[b0[k]]++; diff[b1[k]]--; }
    }
    tick("a2 bounds");
    // elementary interval j = [B[j], B[j+1]); covered ones get ids in ascending address order
    std::vector<uint32_t> iv_of(nb ? nb - 1 : 0, 0xffffffffu);
    struct GIv { uint64_t abs_begin, dense_begin, len; uint32_t cnt, off; };
    std::vector<GIv> giv;
    {
        int64_t cov = 0;
        uint64_t dense = 0;
        for (uint64_t j = 0; j + 1 < nb; j++) {
            cov += diff[j];
            if (cov > 0) {
                iv_of[j] = (uint32_t)giv.size();
                giv.push_back({B[j], dense, B[j + 1] - B[j], 0, 0});
                dense += B[j + 1] - B[j];
            }
        }
    }
    c.n_intervals = giv.size();
    tick("a2 intervals");
    // incidences: per interval, covering accesses in trace order (CSR).  Threads take contiguous
    // chunks of accesses; per-chunk counts give every chunk its slots, so the order is the serial one.
    // Chunks hold equal numbers of incidences (an access covering many intervals is more work).
    std::vector<uint64_t> wk(n_acc + 1, 0);
    for (uint64_t k = 0; k < n_acc; k++) wk[k + 1] = wk[k] + (b1[k] - b0[k]);
    const unsigned T = plan_threads(std::max<uint64_t>(n_acc, wk[n_acc]));
    std::vector<std::vector<uint32_t>> cnt_t(T, std::vector<uint32_t>(giv.size(), 0));
    std::vector<uint64_t> cut(T + 1, n_acc);
    for (unsigned t = 0; t < T; t++)
        cut[t] = (uint64_t)(std::lower_bound(wk.begin(), wk.end(), wk[n_acc] * t / T) - wk.begin());
    auto chunk = [&](unsigned t, uint64_t) { return std::make_pair(std::min(cut[t], n_acc), std::min(cut[t + 1], n_acc)); };
    parallel_for(T, [&](unsigned t) {
        auto [ka, kb] = chunk(t, n_acc);
        for (uint64_t k = ka; k < kb; k++)
            for (uint32_t j = b0[k]; j < b1[k]; j++) cnt_t[t][iv_of[j]]++;
    });
    uint64_t n_inc = 0;
    for (size_t i = 0; i < giv.size(); i++) {
        GIv& g = giv[i];
        g.off = (uint32_t)n_inc;
        uint64_t at = n_inc;
        for (unsigned t = 0; t < T; t++) {           // counts -> each chunk's first slot
            const uint32_t n = cnt_t[t][i];
            cnt_t[t][i] = (uint32_t)at;
            at += n;
        }
        if (at > 0xffffffffull) return fail(CUSAN_ERANGE, "too many interval incidences");
        g.cnt = (uint32_t)(at - n_inc);
        n_inc = at;
    }
    c.n_incidences = n_inc;
    hp.inc.resize(n_inc);
    hp.inc_acc.resize(n_inc);
    parallel_for(T, [&](unsigned t) {
        auto [ka, kb] = chunk(t, n_acc);
        std::vector<uint32_t>& slot = cnt_t[t];
        for (uint64_t k = ka; k < kb; k++)
            for (uint32_t j = b0[k]; j < b1[k]; j++) hp.inc_acc[slot[iv_of[j]]++] = (uint32_t)k;
    });
    tick("a2 incidence");
    if (int st = a1_finish()) return st;                 // a1's records fill the incidence table
    {
        const unsigned TI = plan_threads(n_inc);
        parallel_for(TI, [&](unsigned t) {
            const uint64_t qa = n_inc * t / TI, qb = n_inc * (t + 1) / TI;
            for (uint64_t q = qa; q < qb; q++) hp.inc[q] = hp.acc_rec[hp.inc_acc[q]];
        });
    }
    // ---------------------------------------------------------------- a2: shard clip ------------
    const uint64_t total_dense = giv.empty() ? 0 : giv.back().dense_begin + giv.back().len;
    uint64_t d_lo = 0, d_hi = total_dense;
    if (o.nshards > 1 && !giv.empty()) {
        // Boundaries at equal cumulative cost.  Per granule: with several windows
        // the kernel moves the cell 2(k−1) times for an interval touched in k windows (memory-bound);
        // with one window (or one cell per interval, f3) the work is the accesses replayed, so the
        // weight is the coverage (accesses covering the granule).
        const uint64_t Ws = o.window_events > 0 ? (uint64_t)o.window_events : std::max<uint64_t>(n_acc, 1);
        const bool windowed = Ws < n_acc && !(o.flags & CUSAN_CHECK_INTERVAL_SHADOW);
        std::vector<uint64_t> wpg(giv.size());
        for (size_t i = 0; i < giv.size(); i++) {
            const GIv& g = giv[i];
            if (!windowed) {
                wpg[i] = std::max<uint64_t>(g.cnt, 1);
                continue;
            }
            uint64_t k = 0, last = UINT64_MAX;
            for (uint32_t q = g.off; q < g.off + g.cnt; q++) {
                const uint64_t w = hp.inc_acc[q] / Ws;
                if (w != last) { k++; last = w; }
            }
            wpg[i] = 2 * (k ? k - 1 : 0) + 1;
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
    // (interval-compressed tracking, f3: one slot per interval)
    hp.iv.clear();
    uint64_t slot = 0;
    const bool compressed = (o.flags & CUSAN_CHECK_INTERVAL_SHADOW) != 0;
    for (auto& g : giv) {
        uint64_t lo = std::max(g.dense_begin, d_lo), hi = std::min(g.dense_begin + g.len, d_hi);
        if (lo >= hi) continue;
        Interval v{};
        v.abs_begin = g.abs_begin + (lo - g.dense_begin);
        v.dense_begin = slot;
        v.len = hi - lo;
        v.list_off = g.off;
        v.list_cnt = g.cnt;
        slot = compressed ? slot + 1 : (slot + v.len + CELL_ALIGN - 1) / CELL_ALIGN * CELL_ALIGN;
        hp.iv.push_back(v);
        c.tracked_bytes_shard += 8 * v.len * g.cnt;
    }
    hp.shard_granules = d_hi - d_lo;
    hp.shadow_cells = slot;
    c.shard_granules = hp.shard_granules;

    tick("a2 clip");
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
    // Threads take contiguous chunks of intervals and emit (window, span) in interval order; a
    // stable counting sort by window then gives the window-major order of the serial loop.
    // Chunks hold equal numbers of incidences.
    std::vector<uint64_t> wi(hp.iv.size() + 1, 0);
    for (size_t i = 0; i < hp.iv.size(); i++) wi[i + 1] = wi[i] + hp.iv[i].list_cnt + 1;
    const unsigned TS = plan_threads(wi.back() * 2);
    std::vector<size_t> icut(TS + 1, hp.iv.size());
    for (unsigned t = 0; t < TS; t++)
        icut[t] = (size_t)(std::lower_bound(wi.begin(), wi.end(), wi.back() * t / TS) - wi.begin());
    std::vector<std::vector<std::pair<uint64_t, Span>>> part(TS);
    parallel_for(TS, [&](unsigned t) {
        const size_t ia = std::min(icut[t], hp.iv.size()), ib = std::min(icut[t + 1], hp.iv.size());
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
                uint64_t w = (hp.inc_acc[q] - first) / W;
                uint32_t q2 = q;
                while (q2 < qe && (hp.inc_acc[q2] - first) / W == w) {
                    const AccRec& r = hp.inc[q2];
                    if (r.segm >> 31) readers.reset();
                    else readers.set(r.epoch >> 24);
                    q2++;
                }
                Span s{};
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
                part[t].emplace_back(w, s);
                q = q2;
            }
        }
    });
    std::vector<uint64_t> wstart(nwin + 1, 0);
    for (const auto& pt : part)
        for (const auto& ws : pt) wstart[ws.first + 1]++;
    for (uint64_t w = 0; w < nwin; w++) wstart[w + 1] += wstart[w];
    hp.spans.assign(wstart[nwin], Span{});
    {
        std::vector<uint64_t> at(wstart.begin(), wstart.end() - 1);
        for (const auto& pt : part)
            for (const auto& ws : pt) hp.spans[at[ws.first]++] = ws.second;
    }
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
