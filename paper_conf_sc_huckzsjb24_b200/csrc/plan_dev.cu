// Step a2 on the device (§8(e) "host-side window/tile building ... moved to the
// GPU"): range -> granule expansion, elementary-interval compaction, shard clip, incidence lists,
// windows, spans and the kernel's span tables — the same tables build_host_plan + build_span_tables
// make on the host, byte for byte (tests/test_gpu_plan.py), from the accesses' granule ranges and
// a1's records (event epoch, segment) uploaded once.
//
//   endpoints   (g0, g1) of every non-empty access, CUB radix sort        -> boundaries B, ranks b0/b1
//   coverage    difference array + scan                                   -> covered elementary intervals,
//                                                                            dense offsets, incidence counts
//   incidences  one (interval, access) pair per covered interval of every access, CUB stable sort by
//               interval                                                  -> per interval its accesses in
//                                                                            trace order
//   shard clip  cost weights + scan, boundary search (nshards > 1)        -> this shard's intervals, their
//                                                                            shadow slots and list offsets
//   spans       per interval a walk over its incidences: one span per window touching it, the
//               LOAD / STORE flags and the reader-set size for the pre-assigned read-set record;
//               CUB sort into window-major order, record numbers by scan
//   tables      warp ranges, guided tail, range / weight prefixes per window (build_span_tables' rules)
//
// Two synchronisations with the host: after the coverage (to size the pair / span buffers) and at
// the end (window descriptors and counters: the launches need each window's range count).  All
// other work stays on the plan's stream.  Sorting and scanning are CUB library primitives; every
// other step is a kernel here.
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <mutex>
#include <new>

#include "kernel.cuh"
#include "plan_dev.h"

using namespace cusan;

namespace {

constexpr int MT = 256;
inline uint32_t nblk(uint64_t n) { return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>((n + MT - 1) / MT, 148ull * 16)); }
#define GRID_STRIDE(i, n) for (uint64_t i = (uint64_t)blockIdx.x * MT + threadIdx.x; i < (n); i += (uint64_t)gridDim.x * MT)

inline int bitlen(uint64_t x) { return x ? 64 - __builtin_clzll(x) : 1; }

// header fields written by the kernels (device) and downloaded (pinned host)
enum : int {
    H_NB = 0, H_NIV, H_DENSE, H_NPAIRS, H_NKEPT, H_NINC, H_CELLS, H_TRACKED, H_NSPANS, H_RECUNITS, H_SPILL,
    H_NWIN, H_NDS, H_CELLBYTES, H_NEEDSHADOW, H_DLO, H_DHI, H_COUNT
};

// ---- phase 1: boundaries, coverage --------------------------------------------------------------
__global__ void k_endpoints(uint64_t n, const uint64_t* __restrict__ g0, const uint64_t* __restrict__ g1,
                            uint64_t gmin, uint64_t sent, uint64_t* __restrict__ key, uint32_t* __restrict__ val) {
    GRID_STRIDE(k, n) {
        const bool ne = g1[k] > g0[k];
        key[2 * k] = ne ? g0[k] - gmin : sent;
        key[2 * k + 1] = ne ? g1[k] - gmin : sent;
        val[2 * k] = (uint32_t)(2 * k);
        val[2 * k + 1] = (uint32_t)(2 * k + 1);
    }
}

__global__ void k_bound_flags(uint64_t n2, const uint64_t* __restrict__ key, uint64_t sent, uint32_t* __restrict__ flag) {
    GRID_STRIDE(i, n2) flag[i] = key[i] != sent && (i == 0 || key[i] != key[i - 1]) ? 1u : 0u;
}

// B[r] = boundary r (absolute granule), b[2k] / b[2k+1] = boundary index of access k's ends
__global__ void k_bound_scatter(uint64_t n2, const uint64_t* __restrict__ key, const uint32_t* __restrict__ val,
                                const uint32_t* __restrict__ flag, const uint32_t* __restrict__ rank, uint64_t sent,
                                uint64_t gmin, uint64_t* __restrict__ B, uint32_t* __restrict__ b,
                                unsigned long long* __restrict__ hdr) {
    GRID_STRIDE(i, n2) {
        if (key[i] == sent) {
            b[val[i]] = 0;
        } else {
            const uint32_t r = rank[i] + flag[i] - 1;
            if (flag[i]) B[r] = key[i] + gmin;
            b[val[i]] = r;
        }
        if (i == n2 - 1) hdr[H_NB] = rank[i] + flag[i];
    }
}

__global__ void k_cov_diff(uint64_t n, const uint32_t* __restrict__ b, int* __restrict__ diff) {
    GRID_STRIDE(k, n) {
        const uint32_t b0 = b[2 * k], b1 = b[2 * k + 1];
        if (b1 > b0) {
            atomicAdd(diff + b0, 1);
            atomicAdd(diff + b1, -1);
        }
    }
}

// per elementary interval j < nb-1: granules if covered, covered flag
__global__ void k_iv_len(uint64_t n2, const unsigned long long* __restrict__ hdr, const int* __restrict__ cov,
                         const uint64_t* __restrict__ B, uint64_t* __restrict__ ilen, uint32_t* __restrict__ icov) {
    const uint64_t nb = hdr[H_NB];
    GRID_STRIDE(j, n2) {
        const bool c = j + 1 < nb && cov[j] > 0;
        ilen[j] = c ? B[j + 1] - B[j] : 0;
        icov[j] = c ? 1u : 0u;
    }
}

__global__ void k_npair(uint64_t n, const uint32_t* __restrict__ b, uint64_t* __restrict__ np) {
    GRID_STRIDE(k, n) np[k] = b[2 * k + 1] - b[2 * k];
}

__global__ void k_hdr1(uint64_t n, uint64_t n2, const uint64_t* __restrict__ ilen, const uint64_t* __restrict__ idense,
                       const uint32_t* __restrict__ icov, const uint32_t* __restrict__ ivid,
                       const uint64_t* __restrict__ np, const uint64_t* __restrict__ poff,
                       unsigned long long* __restrict__ hdr) {
    hdr[H_NIV] = ivid[n2 - 1] + icov[n2 - 1];
    hdr[H_DENSE] = idense[n2 - 1] + ilen[n2 - 1];
    hdr[H_NPAIRS] = poff[n - 1] + np[n - 1];
}

// ---- phase 2: intervals, incidences, clip ---------------------------------------------------------
struct GIv {                         // a covered elementary interval (global, before the clip)
    uint64_t abs, dense, len;
    uint32_t cnt, goff;
};

__global__ void k_ivs(uint64_t n2, const unsigned long long* __restrict__ hdr, const uint32_t* __restrict__ icov,
                      const uint32_t* __restrict__ ivid, const uint64_t* __restrict__ B,
                      const uint64_t* __restrict__ idense, const uint64_t* __restrict__ ilen,
                      const int* __restrict__ cov, GIv* __restrict__ iv, uint32_t* __restrict__ cnt) {
    GRID_STRIDE(j, n2) {
        if (!icov[j]) continue;
        GIv g;
        g.abs = B[j];
        g.dense = idense[j];
        g.len = ilen[j];
        g.cnt = (uint32_t)cov[j];
        g.goff = 0;
        iv[ivid[j]] = g;
        cnt[ivid[j]] = g.cnt;
    }
}

// one (interval, access) pair per covered elementary interval of every access, in access order
__global__ void k_pairs(uint64_t n, const uint32_t* __restrict__ b, const uint64_t* __restrict__ poff,
                        const uint32_t* __restrict__ ivid, uint32_t* __restrict__ pkey, uint32_t* __restrict__ pval) {
    GRID_STRIDE(k, n) {
        const uint32_t b0 = b[2 * k], b1 = b[2 * k + 1];
        uint64_t o = poff[k];
        for (uint32_t j = b0; j < b1; j++, o++) {
            pkey[o] = ivid[j];
            pval[o] = (uint32_t)k;
        }
    }
}

// windowed shard weights: the number of windows whose accesses cover the interval
__global__ void k_weights(uint64_t niv, const GIv* __restrict__ iv, const uint32_t* __restrict__ goff,
                          const uint32_t* __restrict__ pval, uint64_t W, int windowed, uint64_t* __restrict__ wt) {
    GRID_STRIDE(i, niv) {
        const GIv g = iv[i];
        uint64_t wpg;
        if (windowed) {
            uint64_t k = 0, last = ~0ull;
            for (uint32_t q = goff[i]; q < goff[i] + g.cnt; q++) {
                const uint64_t w = pval[q] / W;
                if (w != last) { k++; last = w; }
            }
            wpg = 2 * (k ? k - 1 : 0) + 1;
        } else {
            wpg = g.cnt ? g.cnt : 1;
        }
        wt[i] = g.len * wpg;
    }
}

// shard boundaries at equal cumulative cost (build_host_plan's rule, exact integer arithmetic)
__device__ uint64_t shard_boundary(int k, int nshards, uint64_t niv, const GIv* iv, const uint64_t* wt,
                                   const uint64_t* wpre, uint64_t total_dense) {
    if (k <= 0) return 0;
    if (k >= nshards) return total_dense;
    const unsigned __int128 wtot = (unsigned __int128)wpre[niv - 1] + wt[niv - 1];
    const unsigned __int128 target = wtot * (unsigned)k / (unsigned)nshards;
    uint64_t lo = 0, hi = niv;                 // first interval whose inclusive prefix reaches target
    while (lo < hi) {
        const uint64_t m = (lo + hi) / 2;
        if ((unsigned __int128)wpre[m] + wt[m] >= target) hi = m;
        else lo = m + 1;
    }
    if (lo >= niv) return total_dense;
    const uint64_t wpg = wt[lo] / iv[lo].len;
    const uint64_t x = (uint64_t)((target - wpre[lo] + wpg - 1) / wpg);
    return iv[lo].dense + (x < iv[lo].len ? x : iv[lo].len);
}

__global__ void k_bounds(int shard, int nshards, uint64_t niv, const GIv* __restrict__ iv, const uint64_t* __restrict__ wt,
                         const uint64_t* __restrict__ wpre, unsigned long long* __restrict__ hdr) {
    const uint64_t total = hdr[H_DENSE];
    hdr[H_DLO] = shard_boundary(shard, nshards, niv, iv, wt, wpre, total);
    hdr[H_DHI] = shard_boundary(shard + 1, nshards, niv, iv, wt, wpre, total);
}

__global__ void k_keep(uint64_t niv, const GIv* __restrict__ iv, const unsigned long long* __restrict__ hdr,
                       int compressed, uint32_t* __restrict__ kflag, uint64_t* __restrict__ kslots,
                       uint64_t* __restrict__ kcnt) {
    const uint64_t dlo = hdr[H_DLO], dhi = hdr[H_DHI];
    GRID_STRIDE(i, niv) {
        const GIv g = iv[i];
        const uint64_t lo = g.dense > dlo ? g.dense : dlo;
        const uint64_t hi = g.dense + g.len < dhi ? g.dense + g.len : dhi;
        const bool keep = lo < hi;
        kflag[i] = keep;
        kslots[i] = !keep ? 0 : compressed ? 1 : (hi - lo + CELL_ALIGN - 1) / CELL_ALIGN * CELL_ALIGN;
        kcnt[i] = keep ? g.cnt : 0;
    }
}

struct KIv {                         // an interval of this shard (host Interval + its pair offset)
    uint64_t abs, dense, len;
    uint32_t list_off, cnt, goff, pad;
};

__global__ void k_kept(uint64_t niv, const GIv* __restrict__ iv, const uint32_t* __restrict__ goff,
                       const uint32_t* __restrict__ kflag, const uint32_t* __restrict__ kidx,
                       const uint64_t* __restrict__ kslot, const uint64_t* __restrict__ klist,
                       unsigned long long* __restrict__ hdr, KIv* __restrict__ kiv) {
    const uint64_t dlo = hdr[H_DLO], dhi = hdr[H_DHI];
    GRID_STRIDE(i, niv) {
        if (!kflag[i]) continue;
        const GIv g = iv[i];
        const uint64_t lo = g.dense > dlo ? g.dense : dlo;
        const uint64_t hi = g.dense + g.len < dhi ? g.dense + g.len : dhi;
        KIv v;
        v.abs = g.abs + (lo - g.dense);
        v.dense = kslot[i];
        v.len = hi - lo;
        v.list_off = (uint32_t)klist[i];
        v.cnt = g.cnt;
        v.goff = goff[i];
        v.pad = 0;
        kiv[kidx[i]] = v;
        atomicAdd(&hdr[H_TRACKED], (unsigned long long)(8 * v.len * g.cnt));
    }
}

__global__ void k_hdr2(uint64_t niv, const uint32_t* __restrict__ kflag, const uint32_t* __restrict__ kidx,
                       const uint64_t* __restrict__ kslots, const uint64_t* __restrict__ kslot,
                       const uint64_t* __restrict__ kcnt, const uint64_t* __restrict__ klist,
                       unsigned long long* __restrict__ hdr) {
    hdr[H_NKEPT] = kidx[niv - 1] + kflag[niv - 1];
    hdr[H_CELLS] = kslot[niv - 1] + kslots[niv - 1];
    hdr[H_NINC] = klist[niv - 1] + kcnt[niv - 1];
}

// incidence table: per kept interval its accesses' records in trace order (a warp per interval)
__global__ void k_inc(const unsigned long long* __restrict__ hdr, const KIv* __restrict__ kiv,
                      const uint32_t* __restrict__ pval, const AccRec* __restrict__ rec, AccRec* __restrict__ inc,
                      uint32_t* __restrict__ inck) {
    const uint64_t nk = hdr[H_NKEPT];
    const uint64_t warps = (uint64_t)gridDim.x * (MT / 32);
    for (uint64_t m = ((uint64_t)blockIdx.x * MT + threadIdx.x) / 32; m < nk; m += warps) {
        const KIv v = kiv[m];
        for (uint32_t t = threadIdx.x & 31; t < v.cnt; t += 32) {
            const uint32_t k = pval[v.goff + t];
            inc[v.list_off + t] = rec[k];
            inck[v.list_off + t] = k;
        }
    }
}

// ---- spans ----------------------------------------------------------------------------------------
struct SRec {                        // a span before the window-major sort
    uint64_t abs, dense, len;
    uint32_t list_off, cnt, flags, rec_units;
    uint32_t w, pad;
};

__global__ void k_span_count(const unsigned long long* __restrict__ hdr, const KIv* __restrict__ kiv,
                             const uint32_t* __restrict__ inck, uint64_t W, uint32_t* __restrict__ nsp) {
    const uint64_t nk = hdr[H_NKEPT];
    GRID_STRIDE(m, nk) {
        const KIv v = kiv[m];
        uint32_t c = 0;
        uint64_t last = ~0ull;
        for (uint32_t q = v.list_off; q < v.list_off + v.cnt; q++) {
            const uint64_t w = inck[q] / W;
            if (w != last) { c++; last = w; }
        }
        nsp[m] = c;
    }
}

// one thread per interval walks its incidences in trace order: a span per window, with the number of
// reader fibers since the last write at its end (the size of the read-set record its store needs)
__global__ void k_spans(const unsigned long long* __restrict__ hdr, const KIv* __restrict__ kiv,
                        const AccRec* __restrict__ inc, const uint32_t* __restrict__ inck,
                        const uint32_t* __restrict__ spoff, uint64_t W, int persist, int compressed,
                        SRec* __restrict__ sp, uint64_t* __restrict__ skey) {
    const uint64_t nk = hdr[H_NKEPT];
    GRID_STRIDE(m, nk) {
        const KIv v = kiv[m];
        uint32_t rd[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        uint32_t o = spoff[m];
        const uint32_t qe = v.list_off + v.cnt;
        for (uint32_t q = v.list_off; q < qe;) {
            const uint64_t w = inck[q] / W;
            uint32_t q2 = q;
            while (q2 < qe && inck[q2] / W == w) {
                const AccRec r = inc[q2];
                if (r.segm >> 31) {
#pragma unroll
                    for (int x = 0; x < 8; x++) rd[x] = 0;
                } else {
                    const uint32_t f = r.epoch >> 24;
#pragma unroll
                    for (int x = 0; x < 8; x++)
                        if ((f >> 5) == (uint32_t)x) rd[x] |= 1u << (f & 31);
                }
                q2++;
            }
            SRec s;
            s.abs = v.abs;
            s.dense = v.dense;
            s.len = v.len;
            s.list_off = q;
            s.cnt = q2 - q;
            s.flags = (q > v.list_off ? SPAN_LOAD : 0u) | ((q2 < qe || persist) ? SPAN_STORE : 0u) |
                      (q == v.list_off ? SPAN_FIRST_IN_CALL : 0u) | (compressed ? SPAN_COMPRESSED : 0u);
            uint32_t nr = 0;
#pragma unroll
            for (int x = 0; x < 8; x++) nr += __popc(rd[x]);
            s.rec_units = ((s.flags & SPAN_STORE) && nr >= 2) ? (nr + 1 + REC_WORDS - 1) / REC_WORDS : 0u;
            s.w = (uint32_t)w;
            s.pad = 0;
            sp[o] = s;
            skey[o] = w * nk + m;                 // window-major, intervals in order within a window
            o++;
            q = q2;
        }
    }
}

struct Params {                      // build_span_tables' range sizing rules
    uint64_t R_MIN, R_MAX, R_PER_ACC, R_BAL_MIN, R_PER_WARP, TAIL_PCT, TAIL_DIV;
    int max_blocks;
};

// sorted span r: its record units (for the record scan), window bookkeeping, moving cells
__global__ void k_span_sorted(uint64_t ns, const SRec* __restrict__ sp, const uint32_t* __restrict__ sidx,
                              SRec* __restrict__ ss, uint32_t* __restrict__ runits, uint32_t* __restrict__ wcount,
                              unsigned long long* __restrict__ wmoving, unsigned long long* __restrict__ hdr) {
    GRID_STRIDE(r, ns) {
        const SRec s = sp[sidx[r]];
        ss[r] = s;
        runits[r] = s.rec_units;
        atomicAdd(&wcount[s.w], 1u);
        const bool comp = s.flags & SPAN_COMPRESSED;
        if (!comp && (s.flags & (SPAN_LOAD | SPAN_STORE))) atomicAdd(&wmoving[s.w], (unsigned long long)s.len);
        if (s.rec_units) atomicAdd(&hdr[H_SPILL], 1ull);
        const uint64_t mv = (comp ? 1 : s.len) * (((s.flags & SPAN_LOAD) ? 8 : 0) + ((s.flags & SPAN_STORE) ? 8 : 0));
        if (mv) atomicAdd(&hdr[H_CELLBYTES], (unsigned long long)mv);
        if (s.flags & (SPAN_LOAD | SPAN_STORE)) hdr[H_NEEDSHADOW] = 1;
    }
}

__device__ __forceinline__ uint64_t ceil128(uint64_t x) { return (x + CHUNK - 1) / CHUNK * CHUNK; }

// per sorted span: warp-range size, head / tail split (the guided tail)
struct Cut { uint64_t rs, rs_t, head; uint32_t has_tail, moves; };
__device__ Cut span_cut(const SRec& s, uint64_t moving, const Params& P) {
    Cut c;
    const bool comp = s.flags & SPAN_COMPRESSED;
    c.moves = !comp && (s.flags & (SPAN_LOAD | SPAN_STORE));
    const uint64_t rs_cap = max(P.R_BAL_MIN, moving / (P.R_PER_WARP * WARPS * (uint64_t)max(P.max_blocks, 1)));
    uint64_t rs;
    if (c.moves) rs = min(min(max(P.R_PER_ACC * s.cnt, P.R_MIN), P.R_MAX), rs_cap);
    else rs = max(s.len, (uint64_t)1);
    rs = min(ceil128(rs), (uint64_t)1 << 31);
    c.rs = rs;
    const uint64_t nt_all = (s.len + rs - 1) / rs;
    c.rs_t = max(ceil128(rs / P.TAIL_DIV), (uint64_t)CHUNK);
    const uint64_t n_tail = nt_all * P.TAIL_PCT / 100;
    c.has_tail = c.moves && P.TAIL_PCT && P.TAIL_DIV > 1 && c.rs_t < rs && n_tail >= 1 && n_tail < nt_all;
    c.head = c.has_tail ? (nt_all - n_tail) * rs : s.len;
    return c;
}

__global__ void k_tail_flags(uint64_t ns, const SRec* __restrict__ ss, const unsigned long long* __restrict__ wmoving,
                             Params P, uint32_t* __restrict__ tflag) {
    GRID_STRIDE(r, ns) tflag[r] = span_cut(ss[r], wmoving[ss[r].w], P).has_tail;
}

// window layout: first sorted span of every window, compacted (non-empty) window index, DSpan counts
__global__ void k_win_first(uint64_t ns, const SRec* __restrict__ ss, uint32_t* __restrict__ wfirst) {
    GRID_STRIDE(r, ns) if (r == 0 || ss[r].w != ss[r - 1].w) wfirst[ss[r].w] = (uint32_t)r;
}

__global__ void k_win_sizes(uint64_t nwin, const uint32_t* __restrict__ wcount, const uint32_t* __restrict__ wfirst,
                            const uint32_t* __restrict__ trank, const uint32_t* __restrict__ tflag, uint64_t ns,
                            uint32_t* __restrict__ wne, uint64_t* __restrict__ wds) {
    GRID_STRIDE(w, nwin) {
        const uint32_t c = wcount[w];
        wne[w] = c ? 1u : 0u;
        if (!c) { wds[w] = 0; continue; }
        const uint32_t a = wfirst[w], e = a + c;      // tails of the window: trank difference
        const uint32_t tails = (e < ns ? trank[e] : trank[ns - 1] + tflag[ns - 1]) - trank[a];
        wds[w] = (uint64_t)c + tails + 1;              // heads, tails, sentinel
    }
}

// DSpans: heads in span order, then the tails, then a sentinel, per window; tiles / weight per slot
__global__ void k_place(uint64_t ns, const SRec* __restrict__ ss, const unsigned long long* __restrict__ wmoving, Params P, const uint32_t* __restrict__ wfirst,
                        const uint32_t* __restrict__ wcount, const uint32_t* __restrict__ trank,
                        const uint32_t* __restrict__ recoff, const uint64_t* __restrict__ woff,
                        DSpan* __restrict__ ds, uint64_t* __restrict__ dtiles, uint64_t* __restrict__ dweight,
                        uint32_t* __restrict__ dwin, const uint32_t* __restrict__ wrank) {
    GRID_STRIDE(r, ns) {
        const SRec s = ss[r];
        const uint32_t w = s.w;
        const Cut c = span_cut(s, wmoving[w], P);
        const uint64_t base = woff[w];
        DSpan d;
        d.abs_begin = s.abs;
        d.dense_begin = s.dense;
        d.len = c.head;
        d.tile0 = d.weight0 = 0;
        d.list_off = s.list_off;
        d.list_cnt = s.cnt;
        d.flags = s.flags;
        d.rec = s.rec_units ? recoff[r] : 0u;
        d.rec_units = s.rec_units;
        d.pad = 0;
        d.rsize = (uint32_t)c.rs;
        const bool comp = s.flags & SPAN_COMPRESSED;
        const uint64_t nt = comp ? 1 : (d.len + c.rs - 1) / c.rs;
        d.rweight = (uint32_t)min((uint64_t)((c.moves ? c.rs / 32 : 0) + 4ull * s.cnt + 8), (uint64_t)0xffffffffull);
        const uint64_t hp = base + (r - wfirst[w]);
        ds[hp] = d;
        dtiles[hp] = nt;
        dweight[hp] = nt * d.rweight;
        dwin[hp] = wrank[w];
        if (c.has_tail) {
            DSpan t = d;
            t.abs_begin += c.head;
            t.dense_begin += c.head;
            t.len = s.len - c.head;
            t.rsize = (uint32_t)c.rs_t;
            const uint64_t tnt = (t.len + c.rs_t - 1) / c.rs_t;
            t.rweight = (uint32_t)min((uint64_t)((c.moves ? c.rs_t / 32 : 0) + 4ull * s.cnt + 8), (uint64_t)0xffffffffull);
            const uint64_t tp = base + wcount[w] + (trank[r] - trank[wfirst[w]]);
            ds[tp] = t;
            dtiles[tp] = tnt;
            dweight[tp] = tnt * t.rweight;
            dwin[tp] = wrank[w];
        }
    }
}

__global__ void k_sentinels(uint64_t nwin, const uint32_t* __restrict__ wne, const uint64_t* __restrict__ woff,
                            const uint64_t* __restrict__ wds, const uint32_t* __restrict__ wrank, DSpan* __restrict__ ds,
                            uint64_t* __restrict__ dtiles, uint64_t* __restrict__ dweight, uint32_t* __restrict__ dwin) {
    GRID_STRIDE(w, nwin) {
        if (!wne[w]) continue;
        const uint64_t p = woff[w] + wds[w] - 1;
        DSpan z;
        memset(&z, 0, sizeof(z));
        ds[p] = z;
        dtiles[p] = 0;
        dweight[p] = 0;
        dwin[p] = wrank[w];
    }
}

// range / weight prefixes within each window (sentinel = window totals) and the window descriptors
__global__ void k_prefix_fix(const unsigned long long* __restrict__ hdr, const uint32_t* __restrict__ dwin,
                             const uint64_t* __restrict__ woffc, const uint64_t* __restrict__ dt0,
                             const uint64_t* __restrict__ dw0, DSpan* __restrict__ ds, WinDesc* __restrict__ wd,
                             const uint64_t* __restrict__ wdsc) {
    const uint64_t nds = hdr[H_NDS];
    GRID_STRIDE(p, nds) {
        const uint32_t w = dwin[p];
        const uint64_t a = woffc[w];
        ds[p].tile0 = dt0[p] - dt0[a];
        ds[p].weight0 = dw0[p] - dw0[a];
        if (p == a + wdsc[w] - 1) {               // the sentinel: totals of the window
            WinDesc d;
            d.span_off = a;
            d.tiles = dt0[p] - dt0[a];
            d.weight = dw0[p] - dw0[a];
            d.nspans = (uint32_t)(wdsc[w] - 1);
            d.pad = 0;
            wd[w] = d;
        }
    }
}

// compacted (non-empty) window arrays
__global__ void k_win_compact(uint64_t nwin, const uint32_t* __restrict__ wne, const uint32_t* __restrict__ wrank,
                              const uint64_t* __restrict__ woff, const uint64_t* __restrict__ wds,
                              uint64_t* __restrict__ woffc, uint64_t* __restrict__ wdsc, unsigned long long* __restrict__ hdr) {
    GRID_STRIDE(w, nwin) {
        if (wne[w]) {
            woffc[wrank[w]] = woff[w];
            wdsc[wrank[w]] = wds[w];
        }
        if (w == nwin - 1) {
            hdr[H_NWIN] = wrank[w] + wne[w];
            hdr[H_NDS] = woff[w] + wds[w];
        }
    }
}

__global__ void k_span_iota(uint64_t ns, uint32_t* __restrict__ idx) {
    GRID_STRIDE(r, ns) idx[r] = (uint32_t)r;
}

__global__ void k_hdr_nspans(uint64_t niv, const uint32_t* __restrict__ nsp, const uint32_t* __restrict__ spoff,
                             unsigned long long* __restrict__ hdr) {
    hdr[H_NSPANS] = (uint64_t)spoff[niv - 1] + nsp[niv - 1];
}

__global__ void k_hdr_spans(uint64_t ns, const uint32_t* __restrict__ runits, const uint32_t* __restrict__ recoff,
                            unsigned long long* __restrict__ hdr) {
    hdr[H_RECUNITS] = ns ? (uint64_t)recoff[ns - 1] + runits[ns - 1] : 0;
}

// ---- scratch --------------------------------------------------------------------------------------
struct ScratchPool {
    std::mutex m;
    std::vector<DevScratch*> free;
};
ScratchPool& scratch_pool() { static ScratchPool* p = new ScratchPool; return *p; }

// The planning buffers (DevScratch::a per access, ::b per incidence and span: hundreds of MB for a
// large trace) are needed only while a plan is being built; the plan keeps its output tables in
// ::o.  So a and b go back to this pool when the planning is done: plans waiting to run (a pipeline
// keeps several in flight) hold only their tables, and a pipeline needs as many planning buffers
// as plans are built at once — no cudaMalloc / cudaFree (which waits for the device) per plan.
struct BufPool {
    std::mutex m;
    struct Buf { int device, kind; char* p; uint64_t cap; };
    std::vector<Buf> free;
};
BufPool& buf_pool() { static BufPool* p = new BufPool; return *p; }

void buf_take(int device, int kind, char** p, uint64_t* cap) {
    if (*p) return;
    BufPool& P = buf_pool();
    std::lock_guard<std::mutex> lk(P.m);
    int best = -1;
    for (size_t i = 0; i < P.free.size(); i++)
        if (P.free[i].device == device && P.free[i].kind == kind &&
            (best < 0 || P.free[i].cap > P.free[(size_t)best].cap))
            best = (int)i;
    if (best < 0) return;
    *p = P.free[(size_t)best].p;
    *cap = P.free[(size_t)best].cap;
    P.free.erase(P.free.begin() + best);
}

// (only once no work on the stream uses the buffer)
void buf_give(int device, int kind, char** p, uint64_t* cap) {
    if (!*p) return;
    BufPool& P = buf_pool();
    {
        std::lock_guard<std::mutex> lk(P.m);
        if (P.free.size() < 32) {
            P.free.push_back({device, kind, *p, *cap});
            *p = nullptr;
            *cap = 0;
            return;
        }
    }
    cudaFree(*p);
    *p = nullptr;
    *cap = 0;
}

// planning is over (its stream idle): the planning buffers go back to the pool
void planning_done(DevScratch& S) {
    buf_give(S.device, 0, &S.a, &S.a_cap);
    buf_give(S.device, 1, &S.b, &S.b_cap);
}

struct Carver {
    char* base;
    uint64_t off = 0;
    bool measure;
    template <class T>
    T* take(uint64_t n) {
        const uint64_t o = off;
        off = align_up(off + std::max<uint64_t>(n, 1) * sizeof(T));
        return measure ? nullptr : reinterpret_cast<T*>(base + o);
    }
};

}  // namespace

namespace cusan {

DevScratch::~DevScratch() {
    if (a) cudaFree(a);
    if (b) cudaFree(b);
    if (o) cudaFree(o);
    if (hdr_host) cudaFreeHost(hdr_host);
    if (stream) cudaStreamDestroy(stream);
}


DevScratch* plan_dev_acquire(int device) {
    ScratchPool& P = scratch_pool();
    {
        std::lock_guard<std::mutex> lk(P.m);
        for (size_t i = 0; i < P.free.size(); i++)
            if (P.free[i]->device == device) {
                DevScratch* s = P.free[i];
                P.free.erase(P.free.begin() + (long)i);
                return s;
            }
    }
    DevScratch* s = new (std::nothrow) DevScratch;
    if (!s) return nullptr;
    if (std::getenv("CUSAN_DEBUG_ALLOC")) std::fprintf(stderr, "cusan plan_dev: new scratch (device %d)\n", device);
    s->device = device;
    if (cudaStreamCreateWithFlags(&s->stream, cudaStreamNonBlocking) != cudaSuccess) {
        (void)cudaGetLastError();
        s->stream = nullptr;
        delete s;
        return nullptr;
    }
    return s;
}

void plan_dev_release(DevScratch* s) {
    if (!s) return;
    ScratchPool& P = scratch_pool();
    std::lock_guard<std::mutex> lk(P.m);
    if (P.free.size() < 32) P.free.push_back(s);     // (a plan waiting to run holds only its tables)
    else {
        if (std::getenv("CUSAN_DEBUG_ALLOC")) std::fprintf(stderr, "cusan plan_dev: scratch destroyed\n");
        delete s;
    }
}

// cusan_release_cached_memory: the pooled planning scratches and buffers (all devices)
void plan_dev_release_all() {
    std::vector<DevScratch*> scr;
    {
        ScratchPool& P = scratch_pool();
        std::lock_guard<std::mutex> lk(P.m);
        scr.swap(P.free);
    }
    int cur = 0;
    cudaGetDevice(&cur);
    for (DevScratch* s : scr) {
        cudaSetDevice(s->device);
        delete s;
    }
    std::vector<BufPool::Buf> bufs;
    {
        BufPool& P = buf_pool();
        std::lock_guard<std::mutex> lk(P.m);
        bufs.swap(P.free);
    }
    for (const BufPool::Buf& b : bufs) {
        cudaSetDevice(b.device);
        cudaFree(b.p);
    }
    cudaSetDevice(cur);
}

static int grow(char** p, uint64_t* cap, uint64_t need) {
    if (*cap >= need && *p) return CUSAN_OK;
    if (*p) cudaFree(*p);
    *p = nullptr;
    *cap = 0;
    const uint64_t n = std::max<uint64_t>(need + need / 4, 1 << 20);
    if (std::getenv("CUSAN_DEBUG_ALLOC")) std::fprintf(stderr, "cusan plan_dev: scratch grows to %llu B\n", (unsigned long long)n);
    if (cudaMalloc((void**)p, n) != cudaSuccess) {
        (void)cudaGetLastError();
        return fail(CUSAN_ENOMEM, "cannot allocate device planning scratch");
    }
    *cap = n;
    return CUSAN_OK;
}

int device_plan_a2(HostPlan& hp, const DevPlanArgs& A, DevScratch& S, DevPlanOut& out,
                   const std::function<int()>& host_a1) {
    cudaStream_t st = S.stream;
    const uint64_t n = hp.acc_g0.size();
    static const bool dbg = std::getenv("CUSAN_DEBUG_TIMING") != nullptr;
    const auto t0 = std::chrono::steady_clock::now();
    auto tick = [&](const char* what) {
        if (dbg)
            std::fprintf(stderr, "device_plan_a2: %-14s %8.3f ms\n", what,
                         std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    };
    out = DevPlanOut{};
    const cusan_check_opts& o = hp.opts;
    const bool compressed = compressed_shadow(o);
    const uint64_t W = o.window_events > 0 ? (uint64_t)o.window_events : std::max<uint64_t>(n, 1);
    const uint64_t nwin_all = n ? (n + W - 1) / W : 0;
    // key range of the endpoints (granules relative to the smallest; sentinel above the largest)
    uint64_t gmin = ~0ull, gmax = 0, nonempty = 0;
    for (uint64_t k = 0; k < n; k++)
        if (hp.acc_g1[k] > hp.acc_g0[k]) {
            gmin = std::min(gmin, hp.acc_g0[k]);
            gmax = std::max(gmax, hp.acc_g1[k]);
            nonempty++;
        }
    if (!nonempty) return host_a1 ? host_a1() : CUSAN_OK;   // nothing covered: no intervals, no windows
    const uint64_t sent = gmax - gmin + 1;
    const int kbits = bitlen(sent);
    const uint64_t n2 = 2 * n;

    // ---- phase 1 buffers --------------------------------------------------------------------------
    size_t t_sort = 0, t_s32 = 0, t_s64 = 0, t_si = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, t_sort, (uint64_t*)nullptr, (uint64_t*)nullptr, (uint32_t*)nullptr,
                                    (uint32_t*)nullptr, (int)n2, 0, kbits, st);
    cub::DeviceScan::ExclusiveSum(nullptr, t_s32, (uint32_t*)nullptr, (uint32_t*)nullptr, (int)n2, st);
    cub::DeviceScan::ExclusiveSum(nullptr, t_s64, (uint64_t*)nullptr, (uint64_t*)nullptr, (int)n2, st);
    cub::DeviceScan::InclusiveSum(nullptr, t_si, (int*)nullptr, (int*)nullptr, (int)n2 + 1, st);
    const size_t tmp1 = std::max({t_sort, t_s32, t_s64, t_si});
    auto carve1 = [&](Carver& c) {
        struct P1 {
            uint64_t *g0, *g1, *key, *key2, *B, *ilen, *idense, *np, *poff;
            uint32_t *val, *val2, *flag, *rank, *b, *icov, *ivid;
            AccRec* rec;
            int *diff, *cov;
            unsigned long long* hdr;
            void* tmp;
        } p;
        p.g0 = c.take<uint64_t>(n);
        p.g1 = c.take<uint64_t>(n);
        p.rec = c.take<AccRec>(n);
        p.key = c.take<uint64_t>(n2);
        p.key2 = c.take<uint64_t>(n2);
        p.val = c.take<uint32_t>(n2);
        p.val2 = c.take<uint32_t>(n2);
        p.flag = c.take<uint32_t>(n2);
        p.rank = c.take<uint32_t>(n2);
        p.B = c.take<uint64_t>(n2);
        p.b = c.take<uint32_t>(n2);
        p.diff = c.take<int>(n2 + 1);
        p.cov = c.take<int>(n2 + 1);
        p.ilen = c.take<uint64_t>(n2);
        p.idense = c.take<uint64_t>(n2);
        p.icov = c.take<uint32_t>(n2);
        p.ivid = c.take<uint32_t>(n2);
        p.np = c.take<uint64_t>(n);
        p.poff = c.take<uint64_t>(n);
        p.hdr = c.take<unsigned long long>(H_COUNT);
        p.tmp = c.take<char>(tmp1);
        return p;
    };
    Carver m1{nullptr, 0, true};
    carve1(m1);
    buf_take(S.device, 0, &S.a, &S.a_cap);
    if (int e = grow(&S.a, &S.a_cap, m1.off)) return e;
    Carver c1{S.a, 0, false};
    auto P1 = carve1(c1);
    if (!S.hdr_host) CK(cudaHostAlloc((void**)&S.hdr_host, H_COUNT * sizeof(unsigned long long), cudaHostAllocPortable));
    unsigned long long* hh = S.hdr_host;

    CK(cudaMemcpyAsync(P1.g0, hp.acc_g0.data(), n * 8, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(P1.g1, hp.acc_g1.data(), n * 8, cudaMemcpyHostToDevice, st));
    CK(cudaMemsetAsync(P1.hdr, 0, H_COUNT * sizeof(unsigned long long), st));
    CK(cudaMemsetAsync(P1.diff, 0, (n2 + 1) * sizeof(int), st));
    out.h2d_bytes = n * (16 + sizeof(AccRec));
    size_t tb = tmp1;
    k_endpoints<<<nblk(n), MT, 0, st>>>(n, P1.g0, P1.g1, gmin, sent, P1.key, P1.val);
    CK(cub::DeviceRadixSort::SortPairs(P1.tmp, tb, P1.key, P1.key2, P1.val, P1.val2, (int)n2, 0, kbits, st));
    k_bound_flags<<<nblk(n2), MT, 0, st>>>(n2, P1.key2, sent, P1.flag);
    tb = tmp1;
    CK(cub::DeviceScan::ExclusiveSum(P1.tmp, tb, P1.flag, P1.rank, (int)n2, st));
    k_bound_scatter<<<nblk(n2), MT, 0, st>>>(n2, P1.key2, P1.val2, P1.flag, P1.rank, sent, gmin, P1.B, P1.b, P1.hdr);
    k_cov_diff<<<nblk(n), MT, 0, st>>>(n, P1.b, P1.diff);
    tb = tmp1;
    CK(cub::DeviceScan::InclusiveSum(P1.tmp, tb, P1.diff, P1.cov, (int)n2 + 1, st));
    k_iv_len<<<nblk(n2), MT, 0, st>>>(n2, P1.hdr, P1.cov, P1.B, P1.ilen, P1.icov);
    tb = tmp1;
    CK(cub::DeviceScan::ExclusiveSum(P1.tmp, tb, P1.ilen, P1.idense, (int)n2, st));
    tb = tmp1;
    CK(cub::DeviceScan::ExclusiveSum(P1.tmp, tb, P1.icov, P1.ivid, (int)n2, st));
    k_npair<<<nblk(n), MT, 0, st>>>(n, P1.b, P1.np);
    tb = tmp1;
    CK(cub::DeviceScan::ExclusiveSum(P1.tmp, tb, P1.np, P1.poff, (int)n, st));
    k_hdr1<<<1, 1, 0, st>>>(n, n2, P1.ilen, P1.idense, P1.icov, P1.ivid, P1.np, P1.poff, P1.hdr);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(hh, P1.hdr, H_COUNT * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    if (host_a1) {                     // a1 on the host while the device builds the intervals (phase 1
        const int e = host_a1();       // needs only the access ranges; the records go up afterwards)
        if (e) {
            cudaStreamSynchronize(st);
            return e;
        }
        tick("host a1");
    }
    CK(cudaMemcpyAsync(P1.rec, hp.acc_rec.data(), n * sizeof(AccRec), cudaMemcpyHostToDevice, st));
    CK(cudaStreamSynchronize(st));                             // sync 1: sizes of the pair / span buffers
    tick("sync 1");
    out.launches += 8;
    const uint64_t niv = hh[H_NIV], npairs = hh[H_NPAIRS], total_dense = hh[H_DENSE];
    out.n_intervals = niv;
    if (npairs > 0x7fffffffull)      // CUB's item counts are int; the host planner takes up to 2^32
        return fail(CUSAN_ERANGE, "more than 2^31 interval incidences: plan on the host (CUSAN_CHECK_HOST_PLAN)");
    if (!niv) return CUSAN_OK;
    // the weights of the shard search must fit 64 bits (the host planner uses 128-bit sums)
    const bool windowed = W < n && !compressed;
    if (o.nshards > 1) {
        const unsigned __int128 bound = (unsigned __int128)total_dense * (windowed ? 2 * nwin_all + 1 : n);
        if (bound >> 63) return fail(CUSAN_ERANGE, "shard weights exceed 64 bits (use the host planner)");
    }

    // ---- phase 2 buffers ---------------------------------------------------------------------------
    const uint64_t np2 = npairs, nsp_max = npairs;
    size_t u_sort = 0, u_sort64 = 0, u_s32 = 0, u_s64 = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, u_sort, (uint32_t*)nullptr, (uint32_t*)nullptr, (uint32_t*)nullptr,
                                    (uint32_t*)nullptr, (int)np2, 0, bitlen(niv), st);
    cub::DeviceRadixSort::SortPairs(nullptr, u_sort64, (uint64_t*)nullptr, (uint64_t*)nullptr, (uint32_t*)nullptr,
                                    (uint32_t*)nullptr, (int)nsp_max, 0, 64, st);
    const uint64_t nscan = std::max<uint64_t>({niv, nsp_max, 2 * nsp_max + nwin_all, nwin_all});
    cub::DeviceScan::ExclusiveSum(nullptr, u_s32, (uint32_t*)nullptr, (uint32_t*)nullptr, (int)nscan, st);
    cub::DeviceScan::ExclusiveSum(nullptr, u_s64, (uint64_t*)nullptr, (uint64_t*)nullptr, (int)nscan, st);
    const size_t tmp2 = std::max({u_sort, u_sort64, u_s32, u_s64});
    const uint64_t nds_max = 2 * nsp_max + nwin_all;
    auto carve2 = [&](Carver& c) {
        struct P2 {
            GIv* iv;
            uint32_t *cnt, *goff, *pkey, *pkey2, *pval, *pval2, *kflag, *kidx, *inck, *nsp, *spoff, *sidx, *sidx2;
            uint32_t *runits, *recoff, *wcount, *wfirst, *tflag, *trank, *wne, *wrank, *dwin;
            uint64_t *wt, *wpre, *kslots, *kslot, *kcnt, *klist, *skey, *skey2, *wds, *woff, *woffc, *wdsc;
            uint64_t *dtiles, *dweight, *dt0, *dw0;
            unsigned long long* wmoving;
            KIv* kiv;
            SRec *sp, *ss;
            void* tmp;
        } p;
        p.iv = c.take<GIv>(niv);
        p.cnt = c.take<uint32_t>(niv);
        p.goff = c.take<uint32_t>(niv);
        p.pkey = c.take<uint32_t>(np2);
        p.pkey2 = c.take<uint32_t>(np2);
        p.pval = c.take<uint32_t>(np2);
        p.pval2 = c.take<uint32_t>(np2);
        p.wt = c.take<uint64_t>(niv);
        p.wpre = c.take<uint64_t>(niv);
        p.kflag = c.take<uint32_t>(niv);
        p.kidx = c.take<uint32_t>(niv);
        p.kslots = c.take<uint64_t>(niv);
        p.kslot = c.take<uint64_t>(niv);
        p.kcnt = c.take<uint64_t>(niv);
        p.klist = c.take<uint64_t>(niv);
        p.kiv = c.take<KIv>(niv);
        p.inck = c.take<uint32_t>(np2);
        p.nsp = c.take<uint32_t>(niv);
        p.spoff = c.take<uint32_t>(niv);
        p.sp = c.take<SRec>(nsp_max);
        p.ss = c.take<SRec>(nsp_max);
        p.skey = c.take<uint64_t>(nsp_max);
        p.skey2 = c.take<uint64_t>(nsp_max);
        p.sidx = c.take<uint32_t>(nsp_max);
        p.sidx2 = c.take<uint32_t>(nsp_max);
        p.runits = c.take<uint32_t>(nsp_max);
        p.recoff = c.take<uint32_t>(nsp_max);
        p.tflag = c.take<uint32_t>(nsp_max);
        p.trank = c.take<uint32_t>(nsp_max);
        p.wcount = c.take<uint32_t>(nwin_all);
        p.wfirst = c.take<uint32_t>(nwin_all);
        p.wmoving = c.take<unsigned long long>(nwin_all);
        p.wne = c.take<uint32_t>(nwin_all);
        p.wrank = c.take<uint32_t>(nwin_all);
        p.wds = c.take<uint64_t>(nwin_all);
        p.woff = c.take<uint64_t>(nwin_all);
        p.woffc = c.take<uint64_t>(nwin_all);
        p.wdsc = c.take<uint64_t>(nwin_all);
        p.dtiles = c.take<uint64_t>(nds_max);
        p.dweight = c.take<uint64_t>(nds_max);
        p.dt0 = c.take<uint64_t>(nds_max);
        p.dw0 = c.take<uint64_t>(nds_max);
        p.dwin = c.take<uint32_t>(nds_max);
        p.tmp = c.take<char>(tmp2);
        return p;
    };
    // outputs the check reads (kept by the plan): inc, span tables, window descriptors
    auto carve_out = [&](Carver& c) {
        struct PO { AccRec* inc; DSpan* ds; WinDesc* wd; } p;
        p.inc = c.take<AccRec>(np2);
        p.ds = c.take<DSpan>(nds_max);
        p.wd = c.take<WinDesc>(nwin_all);
        return p;
    };
    Carver m2{nullptr, 0, true}, mo{nullptr, 0, true};
    carve2(m2);
    carve_out(mo);
    buf_take(S.device, 1, &S.b, &S.b_cap);
    if (int e = grow(&S.b, &S.b_cap, m2.off)) return e;
    if (int e = grow(&S.o, &S.o_cap, mo.off)) return e;
    Carver c2{S.b, 0, false}, co{S.o, 0, false};
    auto P2 = carve2(c2);
    auto PO = carve_out(co);

    k_ivs<<<nblk(n2), MT, 0, st>>>(n2, P1.hdr, P1.icov, P1.ivid, P1.B, P1.idense, P1.ilen, P1.cov, P2.iv, P2.cnt);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.cnt, P2.goff, (int)niv, st));
    k_pairs<<<nblk(n), MT, 0, st>>>(n, P1.b, P1.poff, P1.ivid, P2.pkey, P2.pval);
    tb = tmp2;
    CK(cub::DeviceRadixSort::SortPairs(P2.tmp, tb, P2.pkey, P2.pkey2, P2.pval, P2.pval2, (int)np2, 0, bitlen(niv), st));
    // shard clip
    if (o.nshards > 1) {
        k_weights<<<nblk(niv), MT, 0, st>>>(niv, P2.iv, P2.goff, P2.pval2, W, windowed ? 1 : 0, P2.wt);
        tb = tmp2;
        CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.wt, P2.wpre, (int)niv, st));
        k_bounds<<<1, 1, 0, st>>>(o.shard, o.nshards, niv, P2.iv, P2.wt, P2.wpre, P1.hdr);
    } else {
        hh[H_DLO] = 0;
        hh[H_DHI] = total_dense;
        CK(cudaMemcpyAsync(P1.hdr + H_DLO, hh + H_DLO, 2 * sizeof(unsigned long long), cudaMemcpyHostToDevice, st));
    }
    k_keep<<<nblk(niv), MT, 0, st>>>(niv, P2.iv, P1.hdr, compressed ? 1 : 0, P2.kflag, P2.kslots, P2.kcnt);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.kflag, P2.kidx, (int)niv, st));
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.kslots, P2.kslot, (int)niv, st));
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.kcnt, P2.klist, (int)niv, st));
    k_kept<<<nblk(niv), MT, 0, st>>>(niv, P2.iv, P2.goff, P2.kflag, P2.kidx, P2.kslot, P2.klist, P1.hdr, P2.kiv);
    k_hdr2<<<1, 1, 0, st>>>(niv, P2.kflag, P2.kidx, P2.kslots, P2.kslot, P2.kcnt, P2.klist, P1.hdr);
    k_inc<<<nblk(32 * niv), MT, 0, st>>>(P1.hdr, P2.kiv, P2.pval2, P1.rec, PO.inc, P2.inck);
    // spans (entries of nsp past the kept count stay 0, so the scan may run over all intervals)
    CK(cudaMemsetAsync(P2.nsp, 0, niv * sizeof(uint32_t), st));
    k_span_count<<<nblk(niv), MT, 0, st>>>(P1.hdr, P2.kiv, P2.inck, W, P2.nsp);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.nsp, P2.spoff, (int)niv, st));
    k_spans<<<nblk(niv), MT, 0, st>>>(P1.hdr, P2.kiv, PO.inc, P2.inck, P2.spoff, W, o.persist_shadow ? 1 : 0,
                                      compressed ? 1 : 0, P2.sp, P2.skey);
    k_hdr_nspans<<<1, 1, 0, st>>>(niv, P2.nsp, P2.spoff, P1.hdr);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(hh, P1.hdr, H_COUNT * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));                             // sync 2: kept intervals and spans
    tick("sync 2");
    out.launches += 14;
    const uint64_t nk = hh[H_NKEPT], ns = hh[H_NSPANS];
    out.n_inc = hh[H_NINC];
    out.inc = PO.inc;
    out.shadow_cells = hh[H_CELLS];
    out.shard_granules = hh[H_DHI] - hh[H_DLO];
    out.d_lo = hh[H_DLO];
    out.tracked_bytes_shard = hh[H_TRACKED];
    if (!nk || !ns) {
        planning_done(S);                                      // (the stream is idle: sync 2)
        return CUSAN_OK;
    }
    k_span_iota<<<nblk(ns), MT, 0, st>>>(ns, P2.sidx);
    tb = tmp2;
    CK(cub::DeviceRadixSort::SortPairs(P2.tmp, tb, P2.skey, P2.skey2, P2.sidx, P2.sidx2, (int)ns, 0,
                                       bitlen(nwin_all * nk), st));
    CK(cudaMemsetAsync(P2.wcount, 0, nwin_all * sizeof(uint32_t), st));
    CK(cudaMemsetAsync(P2.wmoving, 0, nwin_all * sizeof(unsigned long long), st));
    k_span_sorted<<<nblk(ns), MT, 0, st>>>(ns, P2.sp, P2.sidx2, P2.ss, P2.runits, P2.wcount, P2.wmoving, P1.hdr);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.runits, P2.recoff, (int)ns, st));
    k_hdr_spans<<<1, 1, 0, st>>>(ns, P2.runits, P2.recoff, P1.hdr);
    Params prm{A.R_MIN, A.R_MAX, A.R_PER_ACC, A.R_BAL_MIN, A.R_PER_WARP, A.TAIL_PCT, A.TAIL_DIV, A.max_blocks};
    k_tail_flags<<<nblk(ns), MT, 0, st>>>(ns, P2.ss, P2.wmoving, prm, P2.tflag);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.tflag, P2.trank, (int)ns, st));
    k_win_first<<<nblk(ns), MT, 0, st>>>(ns, P2.ss, P2.wfirst);
    k_win_sizes<<<nblk(nwin_all), MT, 0, st>>>(nwin_all, P2.wcount, P2.wfirst, P2.trank, P2.tflag, ns, P2.wne, P2.wds);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.wne, P2.wrank, (int)nwin_all, st));
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.wds, P2.woff, (int)nwin_all, st));
    k_win_compact<<<nblk(nwin_all), MT, 0, st>>>(nwin_all, P2.wne, P2.wrank, P2.woff, P2.wds, P2.woffc, P2.wdsc, P1.hdr);
    // DSpan slots past the last window stay 0 in the range / weight arrays: scans over the bound
    CK(cudaMemsetAsync(P2.dtiles, 0, nds_max * sizeof(uint64_t), st));
    CK(cudaMemsetAsync(P2.dweight, 0, nds_max * sizeof(uint64_t), st));
    k_place<<<nblk(ns), MT, 0, st>>>(ns, P2.ss, P2.wmoving, prm, P2.wfirst, P2.wcount, P2.trank, P2.recoff,
                                     P2.woff, PO.ds, P2.dtiles, P2.dweight, P2.dwin, P2.wrank);
    k_sentinels<<<nblk(nwin_all), MT, 0, st>>>(nwin_all, P2.wne, P2.woff, P2.wds, P2.wrank, PO.ds, P2.dtiles,
                                                P2.dweight, P2.dwin);
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.dtiles, P2.dt0, (int)nds_max, st));
    tb = tmp2;
    CK(cub::DeviceScan::ExclusiveSum(P2.tmp, tb, P2.dweight, P2.dw0, (int)nds_max, st));
    k_prefix_fix<<<nblk(nds_max), MT, 0, st>>>(P1.hdr, P2.dwin, P2.woffc, P2.dt0, P2.dw0, PO.ds, PO.wd, P2.wdsc);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(hh, P1.hdr, H_COUNT * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    S.wins_host.resize(nwin_all);
    CK(cudaMemcpyAsync(S.wins_host.data(), PO.wd, nwin_all * sizeof(WinDesc), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));                             // sync 3: window descriptors for the launches
    tick("sync 3");
    out.launches += 20;
    const uint64_t nw = hh[H_NWIN];
    out.wins.assign(S.wins_host.begin(), S.wins_host.begin() + nw);
    out.ds = PO.ds;
    out.n_ds = hh[H_NDS];
    out.n_spans = ns;
    out.rec_units = hh[H_RECUNITS];
    out.spill_spans = hh[H_SPILL];
    out.cell_bytes = hh[H_CELLBYTES];
    out.need_shadow = hh[H_NEEDSHADOW] != 0;
    planning_done(S);                                          // (the stream is idle: sync 3)
    return CUSAN_OK;
}

}  // namespace cusan
