/*
 * The C ABI from C: the paper's Fig. 6A listing (§IV) — a CUDA-aware
 * MPI_Isend of a device buffer, then a kernel writing the buffer before MPI_Wait — recorded with
 * the lowering callbacks (include/cusan_lower.h) and checked with cusan_check (include/cusan.h).
 * With --fixed the MPI_Wait comes before the kernel (race-free).  With --describe only the host
 * steps run (cusan_plan_describe: no GPU needed).
 *
 *   cc -I include examples/fig6a.c -L paper_conf_sc_huckzsjb24_b200 -lcusan -o fig6a
 *   ./fig6a [--fixed] [--describe]
 *
 * Exit status: 0 when the result is the paper's classification (racy: one run over the buffer,
 * earlier = the Isend's read, later = the kernel's write; fixed: none), 1 otherwise, 2 on an error.
 */
#include <inttypes.h>
#include <stdio.h>
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

int main(int argc, char** argv) {
    int fixed = 0, describe = 0;
    for (int i = 1; i < argc; i++) {
        if (!strcmp(argv[i], "--fixed")) fixed = 1;
        else if (!strcmp(argv[i], "--describe")) describe = 1;
    }
    const uint64_t buf = 0x7f0000000000ull, n = 4096, stream = 16, req = 1;
    cusan_trace* t = NULL;
    cusan_lowering* l = NULL;
    CK(cusan_trace_create(8, 0, &t));
    CK(cusan_lowering_create(t, &l));
    CK(cusan_on_malloc(l, buf, n, CUSAN_MEM_DEVICE));        /* cudaMalloc(&buf, 4096)          */
    CK(cusan_on_stream_create(l, stream, 0));                /* cudaStreamCreate(&s)            */
    uint32_t isend_event = 0, kernel_event = 0;
    CK(cusan_on_mpi_isend(l, buf, n, req));                  /* MPI_Isend(buf, ..., &r)         */
    uint64_t pos = 0;
    uint32_t nf = 0;
    if (fixed) CK(cusan_on_mpi_wait(l, req));                /* MPI_Wait(&r) before the kernel  */
    CK(cusan_trace_size(t, &pos, &nf));
    const uint64_t ptrs[1] = {buf};
    const uint32_t modes[1] = {1};                           /* the kernel writes buf           */
    CK(cusan_on_kernel(l, stream, 1, ptrs, modes));          /* kernel<<<..., s>>>(buf)         */
    if (!fixed) CK(cusan_on_mpi_wait(l, req));
    CK(cusan_on_stream_sync(l, stream));                     /* cudaStreamSynchronize(s)        */

    /* event ids: the Isend's read is the access of the request fiber, the kernel's write the
     * first access at or after `pos` */
    uint64_t total = 0;
    CK(cusan_trace_size(t, &total, &nf));
    cusan_event ev[64];
    if (total > 64) return 2;
    CK(cusan_trace_read(t, 0, total, ev));
    int seen_isend = 0;
    for (uint64_t i = 0; i < total; i++) {
        if (ev[i].kind != CUSAN_EV_ACCESS) continue;
        if (!seen_isend) {
            isend_event = (uint32_t)i;
            seen_isend = 1;
        } else if (i >= pos) {
            kernel_event = (uint32_t)i;
            break;
        }
    }

    cusan_check_opts o;
    cusan_check_opts_init(&o);
    if (describe) {
        cusan_counters c;
        CK(cusan_plan_describe(t, &o, &c));
        printf("events %" PRIu64 " accesses %" PRIu64 " fibers %" PRIu64 " tracked %" PRIu64 " B intervals %" PRIu64 "\n",
               c.n_events, c.n_access, c.n_fibers, c.tracked_bytes, c.n_intervals);
        CK(cusan_lowering_destroy(l));
        CK(cusan_trace_destroy(t));
        return (c.n_access == 2 && c.tracked_bytes == 2 * n) ? 0 : 1;
    }
    cusan_report* r = NULL;
    CK(cusan_check(t, &o, &r));
    uint64_t n_race = 0, n_runs = 0;
    const cusan_race_run* runs = NULL;
    int truncated = 0;
    CK(cusan_report_get(r, &n_race, &n_runs, &runs, &truncated));
    printf("%s: %" PRIu64 " race granules, %" PRIu64 " runs\n", fixed ? "fixed" : "racy", n_race, n_runs);
    for (uint64_t i = 0; i < n_runs; i++)
        printf("  granules [%#" PRIx64 ", %#" PRIx64 ") earlier event %u later event %u\n", runs[i].g_begin,
               runs[i].g_end, runs[i].earlier, runs[i].later);
    int ok;
    if (fixed) ok = n_race == 0 && n_runs == 0;
    else ok = n_runs == 1 && n_race == n / 8 && runs[0].g_begin == buf >> 3 && runs[0].g_end == (buf + n) >> 3 &&
              runs[0].earlier == isend_event && runs[0].later == kernel_event;
    CK(cusan_report_free(r));
    CK(cusan_lowering_destroy(l));
    CK(cusan_trace_destroy(t));
    return ok ? 0 : 1;
}
