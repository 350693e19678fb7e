/*
 * ORACLE — test infrastructure only.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline leg may build, link or execute this program.  It shares no code with the product
 * library (paper_conf_sc_huckzsjb24_b200/csrc): its own trace reader, its own vector clocks, its own
 * per-granule race loop and its own run canonicalisation.
 *
 * A plain, slow, obviously correct CPU implementation of the happens-before race set over a
 * primitive trace:
 *
 *   1. read the trace                         — events e_0..e_{n-1}, event id = trace position
 *   2. naive vector clocks, one full VC per access event
 *        C_f[f] := i+1 for event e_i on fiber f, then
 *        ACCESS: VC(e_i) := C_f          RELEASE:  SC_k := SC_k ⊔ C_f   (AnnotateHappensBefore)
 *        RELEASE_STORE: SC_k := C_f      ACQUIRE:  C_f := C_f ⊔ SC_k    (AnnotateHappensAfter)
 *        FORK(src s -> dst d): event of s: C_s[s] := i+1; C_d := C_d ⊔ C_s
 *      ("comparing the logical time of the memory access with the logical time
 *       recorded for the last synchronization"; PAPER.md:164-173 release/acquire keyed by address;
 *       PAPER.md:178-186 fibers; DJIT+/TSan logical-clock test)
 *      HB(a = e_i on fiber g, b = e_j on fiber f, i < j)  <=>  g == f  ||  i+1 <= VC(b)[g]
 *   3. per 8-byte granule g (range [addr>>3, (addr+n+7)>>3)), accesses in trace order,
 *      state W (last write) and R: fiber -> last read since W.  For access b:
 *        if W exists and !HB(W, b): emit (g, W, b)
 *        if b is a write: for every t with R[t]: if !HB(R[t], b) emit (g, R[t], b);
 *                         W := b; R := {}
 *        else R[fiber(b)] := b
 *   4. canonical output: count triples; merge into maximal runs [g_begin, g_end) of consecutive
 *      granules with equal (earlier, later); sort by (later, earlier, g_begin).
 *
 * Usage: oracle TRACE REPORT [--threads T] [--sample GRANULES]
 *   TRACE   : 'CSTR' u32 version u32 max_fibers u32 pad u64 n, then n × 24-B records
 *             {u8 kind, u8 mode, u16 pad, u32 fiber, u64 a, u64 b}
 *   REPORT  : 'CSRP' u32 version u32 pad u64 n_events u64 n_access u64 tracked_bytes
 *             u64 n_race_granules u64 n_runs, then n_runs × {u64 g_begin, u64 g_end, u32 earlier,
 *             u32 later}
 *   GRANULES: optional file of sorted u64 absolute granule numbers; only those granules are checked
 *             (sampled parity at full sizes).
 *   --range LO HI: only granules in [LO, HI) are checked (a bounded contiguous sample).
 */
#define _GNU_SOURCE
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

enum { EV_ACCESS = 0, EV_RELEASE = 1, EV_RELEASE_STORE = 2, EV_ACQUIRE = 3, EV_FORK = 4 };

typedef struct {
    uint8_t kind, mode;
    uint16_t pad;
    uint32_t fiber;
    uint64_t a, b;
} event_t;

typedef struct {
    uint64_t g;
    uint32_t earlier, later;
} triple_t;

typedef struct {
    uint64_t g_begin, g_end;
    uint32_t earlier, later;
} run_t;

static void die(const char* msg) {
    fprintf(stderr, "oracle: %s\n", msg);
    exit(2);
}

static void* xmalloc(size_t n) {
    void* p = malloc(n ? n : 1);
    if (!p) die("out of memory");
    return p;
}

static void* xcalloc(size_t n, size_t s) {
    void* p = calloc(n ? n : 1, s ? s : 1);
    if (!p) die("out of memory");
    return p;
}

/* ------------------------------------------------------------------------------------------ */
/* global inputs                                                                              */
/* ------------------------------------------------------------------------------------------ */
static uint32_t F;            /* number of fibers */
static uint64_t n_events;
static event_t* events;
/* access table */
static uint64_t n_acc;
static uint32_t* acc_event;   /* trace position of access k */
static uint32_t* acc_fiber;
static uint8_t* acc_write;
static uint64_t* acc_g0;
static uint64_t* acc_g1;
static uint32_t* acc_vc;      /* n_acc × F: VC(e) snapshot (step 2) */

/* ------------------------------------------------------------------------------------------ */
/* step 2: naive vector clocks                                                                */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
    uint64_t key;
    uint32_t* vc;
    int used;
} slot_t;
static slot_t* sc_tab;
static uint64_t sc_cap, sc_n;

static uint32_t* sync_clock(uint64_t key) {  /* SC_k, created as all-zero on first use */
    if (2 * (sc_n + 1) > sc_cap) {
        uint64_t old = sc_cap;
        slot_t* o = sc_tab;
        sc_cap = sc_cap ? 2 * sc_cap : 1024;
        sc_tab = xcalloc(sc_cap, sizeof(slot_t));
        for (uint64_t i = 0; i < old; i++)
            if (o[i].used) {
                uint64_t h = (o[i].key * 0x9E3779B97F4A7C15ull) & (sc_cap - 1);
                while (sc_tab[h].used) h = (h + 1) & (sc_cap - 1);
                sc_tab[h] = o[i];
            }
        free(o);
    }
    uint64_t h = (key * 0x9E3779B97F4A7C15ull) & (sc_cap - 1);
    while (sc_tab[h].used && sc_tab[h].key != key) h = (h + 1) & (sc_cap - 1);
    if (!sc_tab[h].used) {
        sc_tab[h].used = 1;
        sc_tab[h].key = key;
        sc_tab[h].vc = xcalloc(F, sizeof(uint32_t));
        sc_n++;
    }
    return sc_tab[h].vc;
}

static void vector_clocks(void) {
    uint32_t* C = xcalloc((size_t)F * F, sizeof(uint32_t));   /* C[f*F + t] */
    uint64_t k = 0;
    for (uint64_t i = 0; i < n_events; i++) {
        const event_t* e = &events[i];
        uint32_t f = e->fiber;
        uint32_t* Cf = &C[(size_t)f * F];
        if (e->kind == EV_FORK) {
            uint32_t s = (uint32_t)e->a;          /* FORK is an event of the source fiber */
            uint32_t* Cs = &C[(size_t)s * F];
            Cs[s] = (uint32_t)(i + 1);
            for (uint32_t t = 0; t < F; t++)
                if (Cs[t] > Cf[t]) Cf[t] = Cs[t];
            continue;
        }
        Cf[f] = (uint32_t)(i + 1);
        if (e->kind == EV_ACCESS) {
            uint64_t g0 = e->a >> 3, g1 = (e->a + e->b + 7) >> 3;
            if (e->b == 0) g1 = g0;
            acc_event[k] = (uint32_t)i;
            acc_fiber[k] = f;
            acc_write[k] = e->mode ? 1 : 0;
            acc_g0[k] = g0;
            acc_g1[k] = g1;
            memcpy(&acc_vc[k * F], Cf, F * sizeof(uint32_t));
            k++;
        } else if (e->kind == EV_RELEASE) {
            uint32_t* S = sync_clock(e->a);
            for (uint32_t t = 0; t < F; t++)
                if (Cf[t] > S[t]) S[t] = Cf[t];
        } else if (e->kind == EV_RELEASE_STORE) {
            uint32_t* S = sync_clock(e->a);
            memcpy(S, Cf, F * sizeof(uint32_t));
        } else if (e->kind == EV_ACQUIRE) {
            uint32_t* S = sync_clock(e->a);
            for (uint32_t t = 0; t < F; t++)
                if (S[t] > Cf[t]) Cf[t] = S[t];
        }
    }
    free(C);
}

/* HB(earlier access a, later access b) — the logical-clock test of step 2 */
static int hb(uint64_t a, uint64_t b) {
    uint32_t g = acc_fiber[a];
    if (g == acc_fiber[b]) return 1;
    return acc_event[a] + 1 <= acc_vc[b * F + g];
}

/* ------------------------------------------------------------------------------------------ */
/* tiles: chop the union of covered granules into tiles of <= G granules; per tile the list    */
/* of access indices that overlap it, in trace order                                          */
/* ------------------------------------------------------------------------------------------ */
static uint64_t G;
static uint64_t n_tiles;
static uint64_t* tile_b;      /* tile [tile_b, tile_e) */
static uint64_t* tile_e;
static uint64_t* tile_off;    /* CSR into tile_acc */
static uint32_t* tile_acc;

static int cmp_u64pair(const void* x, const void* y) {
    const uint64_t* a = x;
    const uint64_t* b = y;
    return (a[0] > b[0]) - (a[0] < b[0]);
}

static uint64_t find_tile(uint64_t g) {    /* first tile with tile_e > g */
    uint64_t lo = 0, hi = n_tiles;
    while (lo < hi) {
        uint64_t m = (lo + hi) / 2;
        if (tile_e[m] <= g) lo = m + 1; else hi = m;
    }
    return lo;
}

static void build_tiles(void) {
    /* union of [g0, g1) over accesses */
    uint64_t* iv = xmalloc(2 * n_acc * sizeof(uint64_t));
    uint64_t m = 0;
    for (uint64_t k = 0; k < n_acc; k++)
        if (acc_g1[k] > acc_g0[k]) { iv[2 * m] = acc_g0[k]; iv[2 * m + 1] = acc_g1[k]; m++; }
    qsort(iv, m, 2 * sizeof(uint64_t), cmp_u64pair);
    uint64_t cap = 1024;
    tile_b = xmalloc(cap * sizeof(uint64_t));
    tile_e = xmalloc(cap * sizeof(uint64_t));
    n_tiles = 0;
    uint64_t i = 0;
    while (i < m) {
        uint64_t b = iv[2 * i], e = iv[2 * i + 1];
        i++;
        while (i < m && iv[2 * i] <= e) { if (iv[2 * i + 1] > e) e = iv[2 * i + 1]; i++; }
        for (uint64_t t = b; t < e; t += G) {
            if (n_tiles == cap) {
                cap *= 2;
                tile_b = realloc(tile_b, cap * sizeof(uint64_t));
                tile_e = realloc(tile_e, cap * sizeof(uint64_t));
                if (!tile_b || !tile_e) die("out of memory");
            }
            tile_b[n_tiles] = t;
            tile_e[n_tiles] = (t + G < e) ? t + G : e;
            n_tiles++;
        }
    }
    free(iv);
    tile_off = xcalloc(n_tiles + 1, sizeof(uint64_t));
    for (uint64_t k = 0; k < n_acc; k++) {
        if (acc_g1[k] <= acc_g0[k]) continue;
        for (uint64_t t = find_tile(acc_g0[k]); t < n_tiles && tile_b[t] < acc_g1[k]; t++)
            tile_off[t + 1]++;
    }
    for (uint64_t t = 0; t < n_tiles; t++) tile_off[t + 1] += tile_off[t];
    tile_acc = xmalloc(tile_off[n_tiles] * sizeof(uint32_t) + 4);
    uint64_t* fill = xmalloc((n_tiles + 1) * sizeof(uint64_t));
    memcpy(fill, tile_off, (n_tiles + 1) * sizeof(uint64_t));
    for (uint64_t k = 0; k < n_acc; k++) {   /* trace order is preserved inside each tile list */
        if (acc_g1[k] <= acc_g0[k]) continue;
        for (uint64_t t = find_tile(acc_g0[k]); t < n_tiles && tile_b[t] < acc_g1[k]; t++)
            tile_acc[fill[t]++] = (uint32_t)k;
    }
    free(fill);
}

/* ------------------------------------------------------------------------------------------ */
/* step 3 + 4 per tile                                                                        */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
    triple_t* t;
    uint64_t n, cap;
} tvec_t;
typedef struct {
    run_t* r;
    uint64_t n, cap;
} rvec_t;

static void tpush(tvec_t* v, uint64_t g, uint32_t e, uint32_t l) {
    if (v->n == v->cap) {
        v->cap = v->cap ? 2 * v->cap : 4096;
        v->t = realloc(v->t, v->cap * sizeof(triple_t));
        if (!v->t) die("out of memory");
    }
    v->t[v->n].g = g;
    v->t[v->n].earlier = e;
    v->t[v->n].later = l;
    v->n++;
}

static void rpush(rvec_t* v, run_t r) {
    if (v->n == v->cap) {
        v->cap = v->cap ? 2 * v->cap : 1024;
        v->r = realloc(v->r, v->cap * sizeof(run_t));
        if (!v->r) die("out of memory");
    }
    v->r[v->n++] = r;
}

static int cmp_triple(const void* x, const void* y) {   /* (later, earlier, g) */
    const triple_t* a = x;
    const triple_t* b = y;
    if (a->later != b->later) return a->later < b->later ? -1 : 1;
    if (a->earlier != b->earlier) return a->earlier < b->earlier ? -1 : 1;
    return (a->g > b->g) - (a->g < b->g);
}

static int cmp_run(const void* x, const void* y) {      /* (later, earlier, g_begin) */
    const run_t* a = x;
    const run_t* b = y;
    if (a->later != b->later) return a->later < b->later ? -1 : 1;
    if (a->earlier != b->earlier) return a->earlier < b->earlier ? -1 : 1;
    return (a->g_begin > b->g_begin) - (a->g_begin < b->g_begin);
}

/* triples sorted by (later, earlier, g) -> maximal runs of consecutive g */
static void merge_triples(tvec_t* tv, rvec_t* out) {
    qsort(tv->t, tv->n, sizeof(triple_t), cmp_triple);
    for (uint64_t i = 0; i < tv->n;) {
        run_t r = {tv->t[i].g, tv->t[i].g + 1, tv->t[i].earlier, tv->t[i].later};
        uint64_t j = i + 1;
        while (j < tv->n && tv->t[j].later == r.later && tv->t[j].earlier == r.earlier &&
               tv->t[j].g == r.g_end) { r.g_end++; j++; }
        rpush(out, r);
        i = j;
    }
    tv->n = 0;
}

typedef struct {
    /* per-thread granule state for one tile (G granules × F fibers) */
    uint32_t* W;      /* access index + 1 of the last write, 0 = none */
    uint32_t* R;      /* R[g*F + t] = access index + 1 of fiber t's last read since W, 0 = none */
    uint8_t* rl;      /* rl[g*F + k] = k-th fiber with a read since W (iteration list for R) */
    uint16_t* rc;
    tvec_t trip;
    rvec_t runs;
    uint64_t n_triples;
} worker_t;

/* process granules [gb, ge) of tile t with all accesses of that tile, in trace order */
static void check_range(worker_t* w, uint64_t t, uint64_t gb, uint64_t ge) {
    uint64_t n = ge - gb;
    memset(w->W, 0, n * sizeof(uint32_t));
    memset(w->rc, 0, n * sizeof(uint16_t));
    memset(w->R, 0, n * F * sizeof(uint32_t));
    for (uint64_t q = tile_off[t]; q < tile_off[t + 1]; q++) {
        uint64_t b = tile_acc[q];
        uint64_t lo = acc_g0[b] > gb ? acc_g0[b] : gb;
        uint64_t hi = acc_g1[b] < ge ? acc_g1[b] : ge;
        for (uint64_t g = lo; g < hi; g++) {
            uint64_t x = g - gb;
            uint32_t wv = w->W[x];
            if (wv && !hb(wv - 1, b)) { tpush(&w->trip, g, acc_event[wv - 1], acc_event[b]); w->n_triples++; }
            uint32_t* Rg = &w->R[x * F];
            uint8_t* rlg = &w->rl[x * F];
            if (acc_write[b]) {
                for (uint32_t k = 0; k < w->rc[x]; k++) {
                    uint32_t tf = rlg[k];
                    uint32_t rv = Rg[tf];
                    if (!hb(rv - 1, b)) { tpush(&w->trip, g, acc_event[rv - 1], acc_event[b]); w->n_triples++; }
                    Rg[tf] = 0;
                }
                w->rc[x] = 0;
                w->W[x] = (uint32_t)(b + 1);
            } else {
                uint32_t f = acc_fiber[b];
                if (Rg[f] == 0) rlg[w->rc[x]++] = (uint8_t)f;
                Rg[f] = (uint32_t)(b + 1);
            }
        }
    }
    if (w->trip.n > (1u << 20)) merge_triples(&w->trip, &w->runs);
}

/* work distribution */
static uint64_t* sample;
static uint64_t n_sample;
static uint64_t next_item;
static uint64_t range_lo = 0, range_hi = UINT64_MAX;   /* --range: bounded sample of granules */
static pthread_mutex_t mu = PTHREAD_MUTEX_INITIALIZER;

static void* worker_main(void* arg) {
    worker_t* w = arg;
    for (;;) {
        pthread_mutex_lock(&mu);
        uint64_t it = next_item++;
        pthread_mutex_unlock(&mu);
        if (sample) {
            if (it >= n_sample) break;
            uint64_t g = sample[it];
            uint64_t t = find_tile(g);
            if (t < n_tiles && tile_b[t] <= g) check_range(w, t, g, g + 1);
        } else {
            if (it >= n_tiles) break;
            uint64_t gb = tile_b[it] > range_lo ? tile_b[it] : range_lo;
            uint64_t ge = tile_e[it] < range_hi ? tile_e[it] : range_hi;
            if (gb < ge) check_range(w, it, gb, ge);
        }
    }
    merge_triples(&w->trip, &w->runs);
    return NULL;
}

int main(int argc, char** argv) {
    if (argc < 3) die("usage: oracle TRACE REPORT [--threads T] [--sample GRANULES]");
    int threads = 1;
    const char* sample_path = NULL;
    for (int i = 3; i < argc; i++) {
        if (!strcmp(argv[i], "--threads") && i + 1 < argc) threads = atoi(argv[++i]);
        else if (!strcmp(argv[i], "--sample") && i + 1 < argc) sample_path = argv[++i];
        else if (!strcmp(argv[i], "--range") && i + 2 < argc) {
            range_lo = strtoull(argv[++i], NULL, 0);
            range_hi = strtoull(argv[++i], NULL, 0);
        }
        else die("bad argument");
    }
    if (threads < 1) threads = 1;

    /* step 1: read the trace */
    FILE* fp = fopen(argv[1], "rb");
    if (!fp) die("cannot open trace");
    char magic[4];
    uint32_t hdr[3];
    if (fread(magic, 1, 4, fp) != 4 || memcmp(magic, "CSTR", 4)) die("bad trace magic");
    if (fread(hdr, 4, 3, fp) != 3 || fread(&n_events, 8, 1, fp) != 1) die("bad trace header");
    F = hdr[1];
    events = xmalloc(n_events * sizeof(event_t));
    if (fread(events, sizeof(event_t), n_events, fp) != n_events) die("short trace");
    fclose(fp);
    if (n_events >= 0xFFFFFFFFull) die("trace too long (event ids are u32)");
    for (uint64_t i = 0; i < n_events; i++) {
        if (events[i].fiber + 1 > F) F = events[i].fiber + 1;
        if (events[i].kind == EV_FORK && events[i].a + 1 > F) F = (uint32_t)events[i].a + 1;
        if (events[i].kind == EV_ACCESS) n_acc++;
    }
    if (F == 0) F = 1;
    acc_event = xmalloc(n_acc * sizeof(uint32_t) + 4);
    acc_fiber = xmalloc(n_acc * sizeof(uint32_t) + 4);
    acc_write = xmalloc(n_acc + 1);
    acc_g0 = xmalloc(n_acc * sizeof(uint64_t) + 8);
    acc_g1 = xmalloc(n_acc * sizeof(uint64_t) + 8);
    acc_vc = xmalloc(n_acc * F * sizeof(uint32_t) + 4);

    /* step 2 */
    vector_clocks();
    uint64_t tracked = 0;
    for (uint64_t k = 0; k < n_acc; k++) tracked += 8 * (acc_g1[k] - acc_g0[k]);

    /* step 3 */
    G = (4u << 20) / F;
    if (G < 4096) G = 4096;
    if (G > 65536) G = 65536;
    build_tiles();
    if (sample_path) {
        FILE* sp = fopen(sample_path, "rb");
        if (!sp) die("cannot open sample");
        fseek(sp, 0, SEEK_END);
        n_sample = (uint64_t)ftell(sp) / 8;
        fseek(sp, 0, SEEK_SET);
        sample = xmalloc(n_sample * 8 + 8);
        if (fread(sample, 8, n_sample, sp) != n_sample) die("short sample");
        fclose(sp);
    }
    uint64_t gmax = sample ? 1 : G;
    worker_t* ws = xcalloc(threads, sizeof(worker_t));
    pthread_t* th = xmalloc(threads * sizeof(pthread_t));
    for (int i = 0; i < threads; i++) {
        ws[i].W = xmalloc(gmax * sizeof(uint32_t));
        ws[i].R = xmalloc(gmax * F * sizeof(uint32_t));
        ws[i].rl = xmalloc(gmax * F);
        ws[i].rc = xmalloc(gmax * sizeof(uint16_t));
        pthread_create(&th[i], NULL, worker_main, &ws[i]);
    }
    for (int i = 0; i < threads; i++) pthread_join(th[i], NULL);

    /* step 4: canonical runs over all tiles */
    rvec_t all = {0};
    uint64_t n_race = 0;
    for (int i = 0; i < threads; i++) {
        for (uint64_t j = 0; j < ws[i].runs.n; j++) rpush(&all, ws[i].runs.r[j]);
        n_race += ws[i].n_triples;
    }
    qsort(all.r, all.n, sizeof(run_t), cmp_run);
    uint64_t m = 0;
    for (uint64_t i = 0; i < all.n; i++) {
        if (m && all.r[m - 1].later == all.r[i].later && all.r[m - 1].earlier == all.r[i].earlier &&
            all.r[m - 1].g_end == all.r[i].g_begin)
            all.r[m - 1].g_end = all.r[i].g_end;
        else
            all.r[m++] = all.r[i];
    }

    FILE* op = fopen(argv[2], "wb");
    if (!op) die("cannot open report");
    uint32_t rh[2] = {1, 0};
    uint64_t counts[5] = {n_events, n_acc, tracked, n_race, m};
    fwrite("CSRP", 1, 4, op);
    fwrite(rh, 4, 2, op);
    fwrite(counts, 8, 5, op);
    fwrite(all.r, sizeof(run_t), m, op);
    fclose(op);
    return 0;
}
