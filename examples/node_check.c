/*
 * A whole-node check from C (include/cusan.h, cusan_check_opts.ngpus):
 * reads a primitive trace file (tracegen format: 'CSTR' u32 version, u32 max_fibers, u32 pad,
 * u64 n, then n 24-byte cusan_event records), checks it on `ngpus` devices — the event clocks
 * computed once, one host thread per device checking one granule-range shard, the shards' runs
 * merged — and prints the race-granule count, the run count and every run.
 *
 *   cc -I include examples/node_check.c -L paper_conf_sc_huckzsjb24_b200 -lcusan -o node_check
 *   ./node_check TRACE [NGPUS] [WINDOW_EVENTS] [dense]
 *
 * NGPUS 0 = every device of the node.  Exit status 0 on success, 2 on an error.
 */
#include <inttypes.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "cusan.h"

#define CK(x)                                                                   \
    do {                                                                        \
        int st_ = (x);                                                          \
        if (st_ != CUSAN_OK) {                                                  \
            fprintf(stderr, "%s failed (%d): %s\n", #x, st_, cusan_last_error()); \
            return 2;                                                           \
        }                                                                       \
    } while (0)

int main(int argc, char** argv) {
    if (argc < 2) {
        fprintf(stderr, "usage: %s TRACE [NGPUS] [WINDOW_EVENTS] [dense]\n", argv[0]);
        return 2;
    }
    FILE* f = fopen(argv[1], "rb");
    if (!f) { perror(argv[1]); return 2; }
    char magic[4];
    uint32_t version, max_fibers, pad;
    uint64_t n;
    if (fread(magic, 1, 4, f) != 4 || memcmp(magic, "CSTR", 4) || fread(&version, 4, 1, f) != 1 ||
        fread(&max_fibers, 4, 1, f) != 1 || fread(&pad, 4, 1, f) != 1 || fread(&n, 8, 1, f) != 1) {
        fprintf(stderr, "%s: not a trace file\n", argv[1]);
        return 2;
    }
    cusan_event* ev = malloc(n ? n * sizeof(cusan_event) : 1);
    if (!ev || fread(ev, sizeof(cusan_event), n, f) != n) { fprintf(stderr, "short trace\n"); return 2; }
    fclose(f);
    int ngpus = argc > 2 ? atoi(argv[2]) : 0;
    if (ngpus == 0) CK(cusan_device_count(&ngpus));
    cusan_trace* t = NULL;
    CK(cusan_trace_create(max_fibers ? max_fibers : 255, n, &t));
    CK(cusan_trace_append_events(t, ev, n));
    free(ev);
    cusan_check_opts o;
    cusan_check_opts_init(&o);
    o.ngpus = ngpus;
    o.window_events = argc > 3 ? atoi(argv[3]) : 0;
    if (argc > 4 && !strcmp(argv[4], "dense")) o.flags |= CUSAN_CHECK_DENSE_SHADOW;
    cusan_report* r = NULL;
    CK(cusan_check(t, &o, &r));
    uint64_t nrace = 0, nruns = 0;
    const cusan_race_run* runs = NULL;
    int trunc = 0;
    CK(cusan_report_get(r, &nrace, &nruns, &runs, &trunc));
    printf("ngpus %d: %" PRIu64 " race granules, %" PRIu64 " runs\n", ngpus, nrace, nruns);
    for (uint64_t i = 0; i < nruns; i++)
        printf("run %" PRIu64 " %" PRIu64 " %u %u\n", runs[i].g_begin, runs[i].g_end, runs[i].earlier, runs[i].later);
    CK(cusan_report_free(r));
    CK(cusan_trace_destroy(t));
    return 0;
}
