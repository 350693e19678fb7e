/*
 * Online checking through the C ABI (CuSan checks while the
 * program runs): a Jacobi iteration on two streams — a halo stream packs the boundary rows of A
 * through a temporary buffer allocated per iteration, a compute stream updates B from A and
 * unpacks the received halo into B after waiting for the halo stream — recorded with the lowering
 * callbacks and checked by a session after every iteration.  Each temporary is released after its
 * last use and forgotten by the session (cusan_session_forget), so the session's layout stays at
 * the live buffers however many iterations run.  With --racy the halo stream does not wait for
 * the compute stream, so each pack reads A while the previous iteration's compute kernel may still
 * write it.  At the end, the sum of the calls' race granules is compared with one cusan_check of
 * the whole trace.
 *
 *   ./online_jacobi [--racy] [--iters N]
 *
 * Exit status: 0 when the online total equals the one-shot check, the classification is the
 * expected one (racy: races, clean: none) and the layout stayed bounded; 1 otherwise; 2 on an error.
 */
#include <inttypes.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "cusan.h"
#include "cusan_lower.h"

#define CK(x)                                                                   \
    do {                                                                        \
        if ((x) != CUSAN_OK) {                                                  \
            fprintf(stderr, "%s failed: %s\n", #x, cusan_last_error());         \
            return 2;                                                           \
        }                                                                       \
    } while (0)

static int kernel(cusan_lowering* l, uint64_t stream, uint64_t r, uint64_t w) {
    const uint64_t ptrs[2] = {r, w};
    const uint32_t modes[2] = {0, 1};                         /* reads r, writes w */
    return cusan_on_kernel(l, stream, 2, ptrs, modes);
}

int main(int argc, char** argv) {
    int racy = 0, iters = 200;
    for (int i = 1; i < argc; i++) {
        if (!strcmp(argv[i], "--racy")) racy = 1;
        else if (!strcmp(argv[i], "--iters") && i + 1 < argc) iters = atoi(argv[++i]);
    }
    const uint64_t MB = 1 << 20, base = 0x7f0000000000ull;
    uint64_t A = base, B = base + MB, send = base + 2 * MB, recv = send + 4096;
    const uint64_t comp = 16, halo = 17, ev_comp = 100, ev_halo = 101;
    cusan_trace* t = NULL;
    cusan_lowering* l = NULL;
    cusan_session* s = NULL;
    CK(cusan_trace_create(8, 0, &t));
    CK(cusan_lowering_create(t, &l));
    CK(cusan_on_malloc(l, A, MB, CUSAN_MEM_DEVICE));
    CK(cusan_on_malloc(l, B, MB, CUSAN_MEM_DEVICE));
    CK(cusan_on_malloc(l, send, 4096, CUSAN_MEM_DEVICE));
    CK(cusan_on_malloc(l, recv, 4096, CUSAN_MEM_DEVICE));
    CK(cusan_on_stream_create(l, comp, 1));                   /* non-blocking streams */
    CK(cusan_on_stream_create(l, halo, 1));
    cusan_check_opts o;
    cusan_check_opts_init(&o);
    CK(cusan_session_create(t, &o, &s));
    uint64_t online = 0, max_intervals = 0, last_intervals = 0;
    uint64_t tmp = base + 16 * MB;                            /* temporaries: a fresh range each */
    for (int it = 0; it < iters; it++) {
        CK(cusan_on_malloc(l, tmp, 4096, CUSAN_MEM_DEVICE));          /* the pack's temporary */
        if (!racy) CK(cusan_on_stream_wait_event(l, halo, ev_comp));  /* A is the last B */
        CK(kernel(l, halo, A, tmp));                                   /* pack */
        CK(kernel(l, halo, tmp, send));
        CK(kernel(l, halo, send, recv));                               /* the "exchange" */
        CK(cusan_on_event_record(l, ev_halo, halo));
        CK(kernel(l, comp, A, B));                                     /* interior */
        CK(cusan_on_stream_wait_event(l, comp, ev_halo));
        CK(kernel(l, comp, recv, B));                                  /* unpack */
        CK(cusan_on_event_record(l, ev_comp, comp));
        cusan_report* r = NULL;
        CK(cusan_session_check(s, &r));                                /* this iteration's accesses */
        uint64_t ng = 0, nr = 0;
        const cusan_race_run* runs = NULL;
        int trunc = 0;
        cusan_counters c;
        CK(cusan_report_get(r, &ng, &nr, &runs, &trunc));
        CK(cusan_report_counters(r, &c));
        CK(cusan_report_free(r));
        online += ng;
        last_intervals = c.n_intervals;
        if (c.n_intervals > max_intervals) max_intervals = c.n_intervals;
        CK(cusan_session_forget(s, tmp, 4096));                        /* the temporary is released */
        tmp += 4096;
        const uint64_t x = A;                                          /* swap */
        A = B;
        B = x;
    }
    CK(cusan_on_device_sync(l));
    cusan_report* all = NULL;
    CK(cusan_check(t, &o, &all));
    uint64_t ng = 0, nr = 0;
    const cusan_race_run* runs = NULL;
    int trunc = 0;
    CK(cusan_report_get(all, &ng, &nr, &runs, &trunc));
    printf("%s: %d iterations, online %" PRIu64 " race granules, one-shot %" PRIu64 " (%" PRIu64
           " runs); session layout %" PRIu64 " intervals at the end (max %" PRIu64 ")\n",
           racy ? "racy" : "clean", iters, online, ng, nr, last_intervals, max_intervals);
    CK(cusan_report_free(all));
    CK(cusan_session_destroy(s));
    CK(cusan_lowering_destroy(l));
    CK(cusan_trace_destroy(t));
    const int ok = online == ng && (racy ? ng > 0 : ng == 0) && max_intervals < 64;
    return ok ? 0 : 1;
}
