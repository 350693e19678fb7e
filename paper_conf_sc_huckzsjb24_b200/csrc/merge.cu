// Step a4 on the device: raw race runs → canonical runs.
//
// K1's warps append runs as they find them: a run ends where a warp's range ends or its run cache
// evicts, so one canonical run arrives as many raw pieces (dynamic range scheduling interleaves
// the ranges of different warps).  Canonical order is (later, earlier, g_begin) with maximal runs
// of consecutive granules per (earlier, later) pair.  Here:
//   1. LSD radix sort of run indices: by g_begin (64 bits), then stably by later:24 | earlier:24;
//   2. head flags: a run starts a canonical run unless the previous one has the same pair and ends
//      where it begins (the pieces of one pair never overlap: each race triple is emitted once);
//   3. inclusive scan of the flags = canonical run index of every piece;
//   4. scatter: a head writes g_begin / earlier / later, the last piece of a run its g_end.
// Only the canonical runs cross PCIe.  Sorting and scanning are CUB library primitives.
#include <cub/cub.cuh>

#include "kernel.cuh"

namespace {

constexpr int MT = 256;

__global__ void keys_by_begin(const cusan_race_run* __restrict__ runs, uint32_t n, uint64_t* __restrict__ key,
                              uint32_t* __restrict__ idx) {
    const uint32_t i = blockIdx.x * MT + threadIdx.x;
    if (i < n) {
        key[i] = runs[i].g_begin;
        idx[i] = i;
    }
}

__global__ void keys_by_pair(const cusan_race_run* __restrict__ runs, const uint32_t* __restrict__ idx, uint32_t n,
                             uint64_t* __restrict__ key) {
    const uint32_t i = blockIdx.x * MT + threadIdx.x;
    if (i < n) {
        const cusan_race_run r = runs[idx[i]];
        key[i] = ((uint64_t)r.later << 24) | r.earlier;
    }
}

__global__ void run_heads(const cusan_race_run* __restrict__ runs, const uint32_t* __restrict__ idx,
                          const uint64_t* __restrict__ key, uint32_t n, uint32_t* __restrict__ head) {
    const uint32_t i = blockIdx.x * MT + threadIdx.x;
    if (i < n)
        head[i] = (i == 0 || key[i] != key[i - 1] || runs[idx[i - 1]].g_end != runs[idx[i]].g_begin) ? 1u : 0u;
}

__global__ void run_scatter(const cusan_race_run* __restrict__ runs, const uint32_t* __restrict__ idx,
                            const uint32_t* __restrict__ head, const uint32_t* __restrict__ seg, uint32_t n,
                            cusan_race_run* __restrict__ out, unsigned long long* __restrict__ count) {
    const uint32_t i = blockIdx.x * MT + threadIdx.x;
    if (i >= n) return;
    const cusan_race_run r = runs[idx[i]];
    const uint32_t s = seg[i] - 1;
    if (head[i]) {
        out[s].g_begin = r.g_begin;
        out[s].earlier = r.earlier;
        out[s].later = r.later;
    }
    if (i == n - 1 || head[i + 1]) out[s].g_end = r.g_end;
    if (i == n - 1) *count = seg[i];
}

inline uint64_t up(uint64_t x) { return (x + 255) & ~255ull; }

struct Layout {
    uint64_t o_ka, o_kb, o_ia, o_ib, o_hd, o_sg, o_out, o_cnt, o_tmp, total;
    size_t temp;
};

int layout(uint32_t n, cudaStream_t stream, Layout& L) {
    using cusan::cuda_fail;
    // temp storage of the three CUB calls (sizes depend only on n)
    size_t t1 = 0, t2 = 0, t3 = 0;
    CK(cub::DeviceRadixSort::SortPairs(nullptr, t1, (const uint64_t*)nullptr, (uint64_t*)nullptr,
                                       (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)n, 0, 64, stream));
    CK(cub::DeviceRadixSort::SortPairs(nullptr, t2, (const uint64_t*)nullptr, (uint64_t*)nullptr,
                                       (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)n, 0, 48, stream));
    CK(cub::DeviceScan::InclusiveSum(nullptr, t3, (const uint32_t*)nullptr, (uint32_t*)nullptr, (int)n, stream));
    L.temp = std::max(t1, std::max(t2, t3));
    L.o_ka = 0;
    L.o_kb = L.o_ka + up(8ull * n);
    L.o_ia = L.o_kb + up(8ull * n);
    L.o_ib = L.o_ia + up(4ull * n);
    L.o_hd = L.o_ib + up(4ull * n);
    L.o_sg = L.o_hd + up(4ull * n);
    L.o_out = L.o_sg + up(4ull * n);
    L.o_cnt = L.o_out + up(sizeof(cusan_race_run) * n);
    L.o_tmp = L.o_cnt + 256;
    L.total = L.o_tmp + up(L.temp);
    return CUSAN_OK;
}

}  // namespace

namespace cusan {

RunMerge::~RunMerge() {
    if (own && buf) cudaFree(buf);
}

int merge_scratch_bytes(uint64_t n, uint64_t* bytes) {
    if (n >= (1ull << 31)) return fail(CUSAN_ENOMEM, "more than 2^31 raw race runs");
    Layout L;
    const int st = layout((uint32_t)std::max<uint64_t>(n, 1), nullptr, L);
    if (!st) *bytes = L.total;
    return st;
}

int merge_reserve(RunMerge& m, uint64_t n) {
    uint64_t need = 0;
    if (int st = merge_scratch_bytes(n, &need)) return st;
    if (m.cap >= need) return CUSAN_OK;
    if (m.own && m.buf) cudaFree(m.buf);
    m.buf = nullptr;
    m.cap = 0;
    m.own = true;
    if (cudaMalloc((void**)&m.buf, need) != cudaSuccess) return fail(CUSAN_ENOMEM, "cannot allocate run merge buffers");
    m.cap = need;
    return CUSAN_OK;
}

int merge_runs_device(RunMerge& m, cudaStream_t stream, const cusan_race_run* d_runs, uint64_t n64,
                      std::vector<cusan_race_run>& out, uint64_t* d2h_bytes) {
    out.clear();
    if (n64 == 0) return CUSAN_OK;
    if (n64 >= (1ull << 31)) return fail(CUSAN_ENOMEM, "more than 2^31 raw race runs");
    const uint32_t n = (uint32_t)n64;
    Layout L;
    int st = layout(n, stream, L);
    if (st) return st;
    if (m.cap < L.total) {              // the caller's scratch is too small: own, grown buffer
        if (m.own && m.buf) cudaFree(m.buf);
        m.buf = nullptr;
        m.cap = 0;
        m.own = true;
        const uint64_t want = L.total + L.total / 4;
        if (cudaMalloc((void**)&m.buf, want) != cudaSuccess) return fail(CUSAN_ENOMEM, "cannot allocate run merge buffers");
        m.cap = want;
    }
    char* b = m.buf;
    uint64_t* ka = (uint64_t*)(b + L.o_ka);
    uint64_t* kb = (uint64_t*)(b + L.o_kb);
    uint32_t* ia = (uint32_t*)(b + L.o_ia);
    uint32_t* ib = (uint32_t*)(b + L.o_ib);
    uint32_t* hd = (uint32_t*)(b + L.o_hd);
    uint32_t* sg = (uint32_t*)(b + L.o_sg);
    cusan_race_run* d_out = (cusan_race_run*)(b + L.o_out);
    unsigned long long* d_cnt = (unsigned long long*)(b + L.o_cnt);
    void* tmp = b + L.o_tmp;
    const size_t temp = L.temp;
    size_t tb = temp;
    const uint32_t grid = (n + MT - 1) / MT;
    keys_by_begin<<<grid, MT, 0, stream>>>(d_runs, n, ka, ia);
    CK(cub::DeviceRadixSort::SortPairs(tmp, tb, ka, kb, ia, ib, (int)n, 0, 64, stream));
    keys_by_pair<<<grid, MT, 0, stream>>>(d_runs, ib, n, ka);
    tb = temp;
    CK(cub::DeviceRadixSort::SortPairs(tmp, tb, ka, kb, ib, ia, (int)n, 0, 48, stream));
    run_heads<<<grid, MT, 0, stream>>>(d_runs, ia, kb, n, hd);
    tb = temp;
    CK(cub::DeviceScan::InclusiveSum(tmp, tb, hd, sg, (int)n, stream));
    run_scatter<<<grid, MT, 0, stream>>>(d_runs, ia, hd, sg, n, d_out, d_cnt);
    CK(cudaGetLastError());
    unsigned long long cnt = 0;
    CK(cudaMemcpyAsync(&cnt, d_cnt, sizeof(cnt), cudaMemcpyDeviceToHost, stream));
    CK(cudaStreamSynchronize(stream));
    try {
        out.resize(cnt);
    } catch (...) {
        return fail(CUSAN_ENOMEM, "cannot allocate report runs");
    }
    CK(cudaMemcpyAsync(out.data(), d_out, cnt * sizeof(cusan_race_run), cudaMemcpyDeviceToHost, stream));
    CK(cudaStreamSynchronize(stream));
    if (d2h_bytes) *d2h_bytes += sizeof(cnt) + cnt * sizeof(cusan_race_run);
    return CUSAN_OK;
}

}  // namespace cusan
