/*
 * cusan_lower.h — lowering of CUDA and CUDA-aware MPI calls to the primitives of cusan.h
 * (method step a0; CuSan runtime §IV-A; MUST §II-B).
 *
 * A cusan_lowering is CuSan's per-device context: stream -> fiber table with a
 * non-blocking flag, event handles, the memory-attribute table (allocation registry with the
 * whole-allocation extents TypeART provides), the host fiber and MUST's
 * request -> fiber map.  Each cusan_on_* call appends the primitive sequence of
 * SURVEY.md §8(b) to the bound trace.
 *
 * Fibers: 0 = host thread H, 1 = legacy default stream S0 (always tracked), user
 * streams in creation order, MPI-request fibers from a pool (lowest free id first; a fiber returns
 * to the pool at the request's completion).  Keys: K(stream fiber f) = 1<<56 | f,
 * K(event e) = 2<<56 | e, K(request r) = 3<<56 | r (handles < 2^56).
 * Stream handle 0 is the legacy default stream.  Handles are opaque u64 values chosen by the caller.
 *
 * Errors: CUSAN_EINVAL for an unknown stream / kind, more fibers than the trace's max_fibers;
 * otherwise the status of the underlying cusan_trace_append_* call.
 */
#ifndef CUSAN_LOWER_H
#define CUSAN_LOWER_H

#include "cusan.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct cusan_lowering cusan_lowering;

enum cusan_mem_kind { CUSAN_MEM_DEVICE = 0, CUSAN_MEM_MANAGED = 1, CUSAN_MEM_PINNED = 2,
                      CUSAN_MEM_PAGEABLE = 3 };
enum cusan_copy_kind { CUSAN_H2H = 0, CUSAN_H2D = 1, CUSAN_D2H = 2, CUSAN_D2D = 3 };
enum cusan_arg_mode { CUSAN_ARG_R = 0, CUSAN_ARG_W = 1, CUSAN_ARG_RW = 2 };

/* The lowering appends to `trace`, which must outlive it. */
int cusan_lowering_create(cusan_trace* trace, cusan_lowering** out);
int cusan_lowering_destroy(cusan_lowering* l);
/* Fibers used so far (H, S0, user streams, MPI pool). */
int cusan_lowering_fibers(const cusan_lowering* l, uint32_t* n_fibers);

/* cudaMalloc / cudaMallocManaged / cudaHostAlloc / host malloc: registers [ptr, ptr+size). */
int cusan_on_malloc(cusan_lowering* l, uint64_t ptr, uint64_t size, enum cusan_mem_kind kind);
/* cudaFree: host sync with every stream. */
int cusan_on_free(cusan_lowering* l, uint64_t ptr);
int cusan_on_stream_create(cusan_lowering* l, uint64_t stream, int nonblocking);
/* kernel<<<..., stream>>>(args): one whole-allocation access per registered pointer argument
 * (Fig. 6); modes[i] is a cusan_arg_mode; RW is lowered as a write. */
int cusan_on_kernel(cusan_lowering* l, uint64_t stream, uint32_t nargs, const uint64_t* ptrs,
                    const uint32_t* modes);
int cusan_on_stream_sync(cusan_lowering* l, uint64_t stream);
int cusan_on_device_sync(cusan_lowering* l);
int cusan_on_event_record(cusan_lowering* l, uint64_t event, uint64_t stream);
int cusan_on_event_sync(cusan_lowering* l, uint64_t event);
int cusan_on_stream_wait_event(cusan_lowering* l, uint64_t stream, uint64_t event);
/* cudaStreamQuery: synchronises only when it returned cudaSuccess. */
int cusan_on_stream_query(cusan_lowering* l, uint64_t stream, int success);
/* cudaMemcpy (async = 0, legacy stream, host-synchronous for H2H/H2D/D2H) or cudaMemcpyAsync. */
int cusan_on_memcpy(cusan_lowering* l, uint64_t dst, uint64_t src, uint64_t nbytes,
                    enum cusan_copy_kind kind, int async, uint64_t stream);
/* cudaMemset (async = 0; host-synchronous only on pinned memory) / Async. */
int cusan_on_memset(cusan_lowering* l, uint64_t ptr, uint64_t nbytes, int async, uint64_t stream);
/* host load / store on device-accessible memory. */
int cusan_on_host_access(cusan_lowering* l, uint64_t addr, uint64_t nbytes, enum cusan_mode mode);
int cusan_on_mpi_isend(cusan_lowering* l, uint64_t buf, uint64_t nbytes, uint64_t request);
int cusan_on_mpi_irecv(cusan_lowering* l, uint64_t buf, uint64_t nbytes, uint64_t request);
int cusan_on_mpi_wait(cusan_lowering* l, uint64_t request);
int cusan_on_mpi_test(cusan_lowering* l, uint64_t request, int flag);
int cusan_on_mpi_send(cusan_lowering* l, uint64_t buf, uint64_t nbytes);
int cusan_on_mpi_recv(cusan_lowering* l, uint64_t buf, uint64_t nbytes);

/* ---- host threads and the per-thread default stream ----
 * Every host thread is a fiber (thread 0 = fiber 0, the others get fibers when first seen).  The
 * calls after cusan_on_thread(t) are made by thread t: their host-side edges (issue FORKs, host
 * syncs, MPI requests, host accesses) use t's fiber.  cudaDeviceSynchronize covers the work
 * submitted so far; work other threads submit after it is not covered.
 * Stream handles: 1 = cudaStreamLegacy (S0), 2 = cudaStreamPerThread (the calling thread's
 * per-thread default stream, a blocking stream: "not a non-blocking stream and will synchronize
 * with the legacy default stream"), 0 = the default stream of the mode set by
 * cusan_lowering_set_default_stream (legacy unless per_thread != 0).  User stream handles must be
 * > 2.  K(thread t) = 4<<56 | t. */
int cusan_on_thread(cusan_lowering* l, uint64_t thread);
/* pthread_create by the calling thread: issue edge FORK(parent -> child) */
int cusan_on_thread_create(cusan_lowering* l, uint64_t child);
/* pthread_join by the calling thread: RELEASE(child, K(child)) + ACQUIRE(caller, K(child)) */
int cusan_on_thread_join(cusan_lowering* l, uint64_t child);
int cusan_lowering_set_default_stream(cusan_lowering* l, int per_thread);

/* What a fiber stands for, for race reports: kind = CUSAN_FIBER_*, handle = the thread id, stream
 * handle or (latest) MPI request of the fiber.  CUSAN_EINVAL for a fiber the lowering never made. */
enum cusan_fiber_kind { CUSAN_FIBER_HOST = 0, CUSAN_FIBER_LEGACY_STREAM = 1, CUSAN_FIBER_STREAM = 2,
                        CUSAN_FIBER_PER_THREAD_STREAM = 3, CUSAN_FIBER_MPI_REQUEST = 4 };
int cusan_lowering_fiber_info(const cusan_lowering* l, uint32_t fiber, int* kind, uint64_t* handle);

/* ---- bulk form: a recorded API program (same layout as tracegen.OP_DTYPE / ARG_DTYPE) -------- */
enum cusan_api_op {
    CUSAN_OP_MALLOC = 1, CUSAN_OP_FREE = 2, CUSAN_OP_STREAM_CREATE = 3, CUSAN_OP_KERNEL = 4,
    CUSAN_OP_STREAM_SYNC = 5, CUSAN_OP_DEVICE_SYNC = 6, CUSAN_OP_EVENT_RECORD = 7,
    CUSAN_OP_EVENT_SYNC = 8, CUSAN_OP_STREAM_WAIT_EVENT = 9, CUSAN_OP_STREAM_QUERY = 10,
    CUSAN_OP_MEMCPY = 11, CUSAN_OP_MEMCPY_ASYNC = 12, CUSAN_OP_MEMSET = 13,
    CUSAN_OP_MEMSET_ASYNC = 14, CUSAN_OP_HOST_ACCESS = 15, CUSAN_OP_MPI_ISEND = 16,
    CUSAN_OP_MPI_IRECV = 17, CUSAN_OP_MPI_WAIT = 18, CUSAN_OP_MPI_SEND = 19,
    CUSAN_OP_MPI_RECV = 20, CUSAN_OP_MPI_TEST = 21, CUSAN_OP_SET_THREAD = 22,
    CUSAN_OP_THREAD_CREATE = 23, CUSAN_OP_THREAD_JOIN = 24, CUSAN_OP_DEFAULT_STREAM = 25
};
/* 40-byte call record; field use per op is listed in DESIGN.md §"Input formats":
 *   MALLOC a=ptr b=size x=kind | FREE a=ptr | STREAM_CREATE s=stream x=nonblocking
 *   KERNEL s=stream b=first arg x=nargs | STREAM_SYNC s | DEVICE_SYNC | EVENT_RECORD c=event s
 *   EVENT_SYNC c | STREAM_WAIT_EVENT s c | STREAM_QUERY s x=success | MEMCPY a=dst b=src c=n x=kind
 *   MEMCPY_ASYNC + s | MEMSET a=ptr c=n | MEMSET_ASYNC + s | HOST_ACCESS a c x=mode
 *   MPI_ISEND / MPI_IRECV a=buf c=n b=request | MPI_WAIT b | MPI_TEST b x=flag | MPI_SEND/RECV a c
 *   SET_THREAD a=thread | THREAD_CREATE a=child | THREAD_JOIN a=child | DEFAULT_STREAM x=per_thread */
typedef struct cusan_api_call {
    uint32_t op, x;
    uint64_t a, b, c, s;
} cusan_api_call;
typedef struct cusan_api_arg {
    uint64_t ptr;
    uint32_t mode, pad;
} cusan_api_arg;

/* Lowers calls[0..n) in order.  op_first_event (nullable, n entries) receives the trace position of
 * the first primitive each call appended (= the next call's value when it appended none). */
int cusan_lower_program(cusan_lowering* l, const cusan_api_call* calls, uint64_t n,
                        const cusan_api_arg* args, uint64_t nargs, uint32_t* op_first_event);

#ifdef __cplusplus
}
#endif
#endif /* CUSAN_LOWER_H */
