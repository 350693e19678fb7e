// Internal declarations shared by the library's translation units (not part of the C ABI).
#pragma once

#include <cstdint>
#include <string>
#include <utility>
#include <vector>

#include "../../include/cusan.h"

namespace cusan {

// thread-local last error (cusan_last_error)
int fail(int status, const std::string& msg);

// Host memory for the tables a plan or session uploads to the device: page-locked
// (cudaHostAlloc) so every upload is a DMA transfer, taken from a process-wide cache of blocks
// (pinning costs milliseconds per call); plain heap memory in a process without a CUDA device
// (host planning only: cusan_plan_describe).
void* pinned_alloc(size_t bytes);
// Frees the check workspace parked on `device` (check_api.cpp), e.g. before a session's shadow
// growth fails for want of device memory.
void release_parked_workspace(int device);
void pinned_free(void* p) noexcept;
template <class T>
struct PinnedAllocator {
    using value_type = T;
    PinnedAllocator() = default;
    template <class U> PinnedAllocator(const PinnedAllocator<U>&) noexcept {}
    T* allocate(size_t n) { return static_cast<T*>(pinned_alloc(n * sizeof(T))); }
    void deallocate(T* p, size_t) noexcept { pinned_free(p); }
    template <class U> bool operator==(const PinnedAllocator<U>&) const noexcept { return true; }
    template <class U> bool operator!=(const PinnedAllocator<U>&) const noexcept { return false; }
};
template <class T>
using pinned_vector = std::vector<T, PinnedAllocator<T>>;

// Sync-clock slot of each key (open addressing, linear probing): keys are arbitrary u64 values,
// slots are numbered 0, 1, 2 ... in order of first use.
class KeySlots {
  public:
    uint32_t size() const { return n_; }
    // slot of `key`; a new key gets the next slot and *fresh = true
    uint32_t get(uint64_t key, bool* fresh) {
        if (2 * (n_ + 1) > cap_) grow();
        for (size_t i = hash(key) & (cap_ - 1);; i = (i + 1) & (cap_ - 1)) {
            if (val_[i] == EMPTY) {
                key_[i] = key;
                val_[i] = n_;
                *fresh = true;
                return n_++;
            }
            if (key_[i] == key) {
                *fresh = false;
                return val_[i];
            }
        }
    }

  private:
    static constexpr uint32_t EMPTY = 0xffffffffu;
    static size_t hash(uint64_t k) {           // splitmix64 finalizer: every key bit reaches every slot bit
        k ^= k >> 30; k *= 0xBF58476D1CE4E5B9ull; k ^= k >> 27; k *= 0x94D049BB133111EBull; k ^= k >> 31;
        return (size_t)k;
    }
    void grow() {
        std::vector<uint64_t> k = std::move(key_);
        std::vector<uint32_t> v = std::move(val_);
        cap_ = cap_ ? 2 * cap_ : 1024;
        key_.assign(cap_, 0);
        val_.assign(cap_, EMPTY);
        for (size_t j = 0; j < v.size(); j++) {
            if (v[j] == EMPTY) continue;
            size_t i = hash(k[j]) & (cap_ - 1);
            while (val_[i] != EMPTY) i = (i + 1) & (cap_ - 1);
            key_[i] = k[j];
            val_[i] = v[j];
        }
    }
    std::vector<uint64_t> key_;
    std::vector<uint32_t> val_;
    size_t cap_ = 0;
    uint32_t n_ = 0;
};

// A u64 -> V hash map with open addressing (linear probing, backward-shift erase): the lowering
// looks up stream, request and allocation handles for every recorded call.
template <class V>
class FlatMap {
  public:
    V* get(uint64_t key) {
        if (!n_) return nullptr;
        for (size_t i = slot(key);; i = (i + 1) & (cap_ - 1)) {
            if (!used_[i]) return nullptr;
            if (keys_[i] == key) return &vals_[i];
        }
    }
    const V* get(uint64_t key) const { return const_cast<FlatMap*>(this)->get(key); }
    size_t count(uint64_t key) const { return get(key) ? 1 : 0; }
    V& operator[](uint64_t key) {
        if (V* v = get(key)) return *v;
        if (2 * (n_ + 1) > cap_) grow();
        size_t i = slot(key);
        while (used_[i]) i = (i + 1) & (cap_ - 1);
        used_[i] = 1;
        keys_[i] = key;
        vals_[i] = V{};
        n_++;
        return vals_[i];
    }
    bool erase(uint64_t key) {
        if (!n_) return false;
        size_t i = slot(key);
        for (;; i = (i + 1) & (cap_ - 1)) {
            if (!used_[i]) return false;
            if (keys_[i] == key) break;
        }
        used_[i] = 0;                                 // backward shift: keep every probe chain intact
        for (size_t j = (i + 1) & (cap_ - 1); used_[j]; j = (j + 1) & (cap_ - 1)) {
            const size_t h = slot(keys_[j]);
            if (((j - h) & (cap_ - 1)) >= ((j - i) & (cap_ - 1))) {
                keys_[i] = keys_[j];
                vals_[i] = vals_[j];
                used_[i] = 1;
                used_[j] = 0;
                i = j;
            }
        }
        n_--;
        return true;
    }

  private:
    size_t slot(uint64_t k) const {
        k ^= k >> 30; k *= 0xBF58476D1CE4E5B9ull; k ^= k >> 27; k *= 0x94D049BB133111EBull; k ^= k >> 31;
        return (size_t)k & (cap_ - 1);
    }
    void grow() {
        std::vector<uint64_t> k = std::move(keys_);
        std::vector<V> v = std::move(vals_);
        std::vector<char> u = std::move(used_);
        cap_ = cap_ ? 2 * cap_ : 64;
        keys_.assign(cap_, 0);
        vals_.assign(cap_, V{});
        used_.assign(cap_, 0);
        n_ = 0;
        for (size_t j = 0; j < u.size(); j++)
            if (u[j]) (*this)[k[j]] = v[j];
    }
    std::vector<uint64_t> keys_;
    std::vector<V> vals_;
    std::vector<char> used_;
    size_t cap_ = 0, n_ = 0;
};

// Interval-compressed shadow (f3) unless the caller asks for the per-granule dense shadow.
inline bool compressed_shadow(const cusan_check_opts& o) { return !(o.flags & CUSAN_CHECK_DENSE_SHADOW); }
// CUSAN_EINVAL for unknown or contradictory flags
int check_flags(const cusan_check_opts& o);

struct Trace {
    uint32_t max_fibers = 1;
    std::vector<cusan_event> ev;
};

// ----------------------------------------------------------------------------------------------
// Shadow cell (FastTrack's epoch / read-VC representation): 8 B per granule
// {W, R}, each u32 = fiber:8 | (event id + 1):24, 0 = empty.  R is the single reader's epoch, or —
// when two or more fibers have read since the last write — 0xFF:24-bit index of a read-set record
// (fiber 0xFF is reserved for this tag).
// ----------------------------------------------------------------------------------------------
inline uint32_t pack_epoch(uint32_t fiber, uint32_t event_id) { return (fiber << 24) | (event_id + 1); }
constexpr uint32_t SPILL_TAG = 0xFF000000u;
constexpr uint32_t REC_WORDS = 8;        // read-set record allocation unit (u32 words)
constexpr uint64_t CELL_ALIGN = 32;      // interval shadow slots start on 32-cell (256-B) boundaries

// Per access event, what the shadow kernel needs (8 B, one per interval incidence):
//   epoch  = pack_epoch(fiber, event id)
//   segm   = segment id (bits 0..30) | is_write << 31
struct AccRec {
    uint32_t epoch;
    uint32_t segm;
};

// One elementary interval of the granule space (a maximal granule range no access endpoint splits),
// clipped to the plan's shard.
struct Interval {
    uint64_t abs_begin;   // absolute granule (address >> 3) of the first granule in the shard clip
    uint64_t dense_begin; // index of that granule in the shard's shadow array
    uint64_t len;         // granules in the shard clip
    uint32_t list_off;    // first incidence (into the AccRec table) — all windows
    uint32_t list_cnt;
};

// A window's piece of work on one interval: the interval's incidences inside the window.
struct Span {
    uint64_t abs_begin, dense_begin, len;
    uint32_t list_off;    // into the AccRec table
    uint32_t list_cnt;
    uint32_t flags;       // SPAN_LOAD: cells hold state from an earlier window; SPAN_STORE: write back
    uint32_t rec;         // pre-assigned read-set record (REC_WORDS-word units) for the final state
    uint32_t rec_units;   // its size; 0 = the final state needs no record (≤ 1 reader)
};
// SPAN_LOAD: cells hold state from an earlier window; SPAN_STORE: a later window needs the result;
// SPAN_FIRST_IN_CALL: the interval's first span of this check (incremental sessions);
// SPAN_COMPRESSED: the interval keeps one shadow cell for all its granules (f3).
enum : uint32_t { SPAN_LOAD = 1u, SPAN_STORE = 2u, SPAN_FIRST_IN_CALL = 8u,
                  SPAN_COMPRESSED = 16u };

struct HostPlan {
    // options
    cusan_check_opts opts{};
    // a1
    uint32_t F = 1;                       // fibers (row length of segvc)
    pinned_vector<uint32_t> segvc;        // nseg × F (uploaded)
    uint64_t nseg = 0;
    uint64_t nseg_count = 0;              // segments of the trace, counted ahead of a1 (0 = unknown)
    // accesses in trace order
    std::vector<uint64_t> acc_g0, acc_g1; // granule ranges
    std::vector<uint32_t> acc_event;      // trace position
    std::vector<AccRec> acc_rec;
    // a2
    std::vector<Interval> iv;             // shard-clipped intervals (len > 0)
    pinned_vector<AccRec> inc;            // incidence table: per interval, its accesses in trace order (uploaded)
    std::vector<uint32_t> inc_acc;        // access index of each incidence
    uint64_t shard_granules = 0;          // covered granules in this shard
    uint64_t shadow_cells = 0;            // shadow slots incl. alignment padding
    uint64_t rec_units = 0;               // pre-assigned read-set record units
    uint64_t spill_spans = 0;
    // windows
    std::vector<Span> spans;              // all windows, window-major
    std::vector<uint64_t> win_span_off;   // nwin + 1
    uint64_t window_accesses = 0;
    // counters
    cusan_counters ctr{};
};

// a1 + a2.  Spans (windows) are planned for the accesses from `first_access` on (0 = all);
// pre-assigned read-set records are numbered from `rec_base`.  a1_only: the accesses and a1 only
// (a2 runs on the device, plan_dev.cu).  t = nullptr: a2 only, hp already holds the accesses and
// a1's products (a plan from clocks).
int build_host_plan(const Trace* t, const cusan_check_opts& o, HostPlan& hp, uint64_t first_access = 0,
                    uint64_t rec_base = 0, bool a1_only = false);

// a1 of a whole trace for a clocks object (cusan_clocks_compute), with the node's cores
int compute_clocks(const Trace& t, HostPlan& hp);
// a1 itself (plan.cpp): with fill_accesses the accesses' ranges and the counters too (one pass),
// else hp holds the ranges already (prepare_plan_accesses)
std::pair<int, std::string> run_a1(const Trace& t, HostPlan& hp, unsigned threads, bool fill_accesses);
int prepare_plan_accesses(const Trace& t, const cusan_check_opts& o, HostPlan& hp);
unsigned a1_threads_for(uint64_t n_events);

// canonical merge of runs (sort by (later, earlier, g_begin), merge abutting) — a4 host part
void canonicalize_runs(std::vector<cusan_race_run>& runs);

}  // namespace cusan

struct cusan_trace {
    cusan::Trace t;
};

// a1's products for a whole trace (cusan_clocks_*): accesses, records, segment rows, counters
struct cusan_clocks {
    cusan::HostPlan hp;
};

struct cusan_report {
    uint64_t n_race_granules = 0;
    uint64_t n_runs = 0;
    int truncated = 0;
    std::vector<cusan_race_run> runs;
    cusan_counters ctr{};
};
