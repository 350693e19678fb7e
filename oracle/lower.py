"""ORACLE — test infrastructure only (tests/, __graft_entry__.smoke(), bench.py cpu_baseline).

Plain-Python lowering of CUDA / CUDA-aware-MPI calls to happens-before primitives (method step a0),
written directly from the paper's CuSan runtime description and SURVEY.md §8(b)'s table.  It shares no
code with the product library (``paper_conf_sc_huckzsjb24_b200/csrc/lower.cpp``).

Fibers (§IV-A(a)): 0 = host thread H of thread 0, 1 = legacy default stream S0
(always tracked), then — in the order they are first needed — user streams (at creation), MPI-request
fibers from a pool, further host threads and per-thread default streams.
Sync keys: K(stream fiber f) = 1<<56 | f, K(event e) = 2<<56 | e, K(request r) = 3<<56 | r,
K(thread t) = 4<<56 | t.

Host threads and the per-thread default stream: every host
thread is a fiber; the calls after OP_SET_THREAD t are made by thread t; thread creation is an issue
edge FORK(parent → child); a join is RELEASE(child, K(t)) then ACQUIRE(parent, K(t)).  Stream handle 1
(cudaStreamLegacy) is S0, handle 2 (cudaStreamPerThread) the calling thread's per-thread default
stream, handle 0 S0 in legacy mode or the per-thread default stream in per-thread mode.  A per-thread
default stream "is not a non-blocking stream and will synchronize with the legacy default stream"
(PAPER.md:1210-1213): it is a blocking stream.
"""
from __future__ import annotations

import bisect

import numpy as np

from tracegen.program import (ARG_DTYPE, CPY_D2H, CPY_H2D, CPY_H2H, EVENT_DTYPE, EV_ACCESS, EV_ACQUIRE,
                              EV_FORK, EV_RELEASE, EV_RELEASE_STORE, MEM_PINNED, MODE_R, OP_DEFAULT_STREAM,
                              OP_DEVICE_SYNC, OP_DTYPE, OP_EVENT_RECORD, OP_EVENT_SYNC, OP_FREE,
                              OP_HOST_ACCESS, OP_KERNEL, OP_MALLOC, OP_MEMCPY, OP_MEMCPY_ASYNC, OP_MEMSET,
                              OP_MEMSET_ASYNC, OP_MPI_IRECV, OP_MPI_ISEND, OP_MPI_RECV, OP_MPI_SEND,
                              OP_MPI_TEST, OP_MPI_WAIT, OP_SET_THREAD, OP_STREAM_CREATE, OP_STREAM_QUERY,
                              OP_STREAM_SYNC, OP_STREAM_WAIT_EVENT, OP_THREAD_CREATE, OP_THREAD_JOIN, READ,
                              STREAM_NONBLOCKING, WRITE)

S0 = 1


def K_stream(f):
    return (1 << 56) | f


def K_event(e):
    return (2 << 56) | e


def K_req(r):
    return (3 << 56) | r


def K_thread(t):
    return (4 << 56) | t


class Lowering:
    """CuSan per-device context: stream → fiber table with a non-blocking flag,
    event handles, memory-attribute table (allocation registry), host
    fiber(s), plus MUST's request → fiber map."""

    def __init__(self):
        self.ev: list[tuple] = []            # (kind, fiber, a, b, mode)
        self.stream_fiber = {}               # user stream handle -> fiber
        self.blocking_user: list[int] = []   # fibers of blocking streams (user + per-thread), creation order
        self.all_streams: list[int] = [S0]   # S0 then streams, creation order
        self.next_fiber = 2
        self.free_mpi: list[int] = []        # pool of returned MPI fibers
        self.req_fiber: dict[int, int] = {}
        self.alloc_base: list[int] = []      # sorted bases
        self.alloc: dict[int, tuple[int, int]] = {}   # base -> (size, kind)
        self.thread_fiber = {0: 0}           # host thread -> fiber
        self.thread = 0                      # calling thread
        self.ptds: dict[int, int] = {}       # host thread -> its per-thread default stream fiber
        self.per_thread_mode = False

    @property
    def H(self):
        """The calling host thread's fiber."""
        return self.thread_fiber[self.thread]

    def new_fiber(self):
        f = self.next_fiber
        self.next_fiber += 1
        return f

    # -- primitives (TSan API) ---------------------------------------------
    def access(self, f, mode, addr, n):
        self.ev.append((EV_ACCESS, f, addr, n, mode))

    def release(self, f, key):
        self.ev.append((EV_RELEASE, f, key, 0, 0))

    def release_store(self, f, key):
        self.ev.append((EV_RELEASE_STORE, f, key, 0, 0))

    def acquire(self, f, key):
        self.ev.append((EV_ACQUIRE, f, key, 0, 0))

    def fork(self, src, dst):
        self.ev.append((EV_FORK, dst, src, 0, 0))

    # -- helpers -------------------------------------------------------------------------------
    def find_alloc(self, p):
        """Allocation containing pointer p (TypeART extent lookup)."""
        i = bisect.bisect_right(self.alloc_base, p) - 1
        if i < 0:
            return None
        base = self.alloc_base[i]
        size, kind = self.alloc[base]
        if base <= p < base + size:
            return base, size, kind
        return None

    def thread_ptds(self):
        """The calling thread's per-thread default stream, a blocking stream."""
        t = self.thread
        if t not in self.ptds:
            f = self.new_fiber()
            self.ptds[t] = f
            self.all_streams.append(f)
            self.blocking_user.append(f)
        return self.ptds[t]

    def stream(self, handle):
        """Stream handle -> fiber: 0 the default stream of the mode, 1 legacy, 2 per-thread."""
        if handle == 0:
            return self.thread_ptds() if self.per_thread_mode else S0
        if handle == 1:
            return S0
        if handle == 2:
            return self.thread_ptds()
        return self.stream_fiber[handle]

    def prologue(self, f):
        """Issue edge host → stream and the legacy default-stream barriers (Fig. 3,
        PAPER.md:356-364)."""
        self.fork(self.H, f)
        if f in self.blocking_user:
            self.acquire(f, K_stream(S0))
        if f == S0:
            for u in self.blocking_user:
                self.acquire(S0, K_stream(u))

    def epilogue(self, f):
        """AnnotateHappensBefore on the stream after each operation."""
        self.release(f, K_stream(f))

    def sync_stream_host(self, f):
        """cudaStreamSynchronize; on S0 it also covers every blocking
        stream."""
        self.acquire(self.H, K_stream(f))
        if f == S0:
            for u in self.blocking_user:
                self.acquire(self.H, K_stream(u))

    def sync_device_host(self):
        """cudaDeviceSynchronize: acquire on every stream; work other
        threads submit later is not covered — it is later in the trace."""
        for f in self.all_streams:
            self.acquire(self.H, K_stream(f))

    def tracked_range(self, p, n):
        return n > 0 and self.find_alloc(p) is not None

    # -- one API call --------------------------------------------------------------------------
    def call(self, op, args):
        kind = int(op["op"])
        x, a, b, c, s = int(op["x"]), int(op["a"]), int(op["b"]), int(op["c"]), int(op["s"])
        if kind == OP_MALLOC:
            bisect.insort(self.alloc_base, a)
            self.alloc[a] = (b, x)
        elif kind == OP_FREE:
            if a in self.alloc:                          # TypeART's table drops it (★A25,
                del self.alloc[a]                        # PAPER.md:306-308, 835-855)
                self.alloc_base.remove(a)
            self.sync_device_host()
        elif kind == OP_STREAM_CREATE:
            f = self.new_fiber()
            self.stream_fiber[s] = f
            self.all_streams.append(f)
            if not (x & STREAM_NONBLOCKING):
                self.blocking_user.append(f)
        elif kind == OP_KERNEL:
            f = self.stream(s)
            self.prologue(f)
            for j in range(b, b + x):
                al = self.find_alloc(int(args[j]["ptr"]))
                if al is None:
                    continue
                mode = READ if int(args[j]["mode"]) == MODE_R else WRITE   # RW → WRITE (A10)
                self.access(f, mode, al[0], al[1])         # whole allocation
            self.epilogue(f)
        elif kind in (OP_STREAM_SYNC,):
            self.sync_stream_host(self.stream(s))
        elif kind == OP_STREAM_QUERY:
            if x:                                          # only a successful query syncs (A9)
                self.sync_stream_host(self.stream(s))
        elif kind == OP_DEVICE_SYNC:
            self.sync_device_host()
        elif kind == OP_EVENT_RECORD:
            f = self.stream(s)
            self.prologue(f)
            self.release_store(f, K_event(c))             # re-record replaces the capture (A4)
        elif kind == OP_EVENT_SYNC:
            self.acquire(self.H, K_event(c))
        elif kind == OP_STREAM_WAIT_EVENT:
            f = self.stream(s)
            self.prologue(f)
            self.acquire(f, K_event(c))
        elif kind in (OP_MEMCPY, OP_MEMCPY_ASYNC):
            f = self.stream(0) if kind == OP_MEMCPY else self.stream(s)
            self.prologue(f)
            if self.tracked_range(a, c):
                self.access(f, WRITE, a, c)
            if self.tracked_range(b, c):
                self.access(f, READ, b, c)
            self.epilogue(f)
            if kind == OP_MEMCPY and x in (CPY_H2H, CPY_H2D, CPY_D2H):   # PAPER.md:433-436 (A6)
                self.acquire(self.H, K_stream(f))
        elif kind in (OP_MEMSET, OP_MEMSET_ASYNC):
            f = self.stream(0) if kind == OP_MEMSET else self.stream(s)
            self.prologue(f)
            al = self.find_alloc(a)
            if self.tracked_range(a, c):
                self.access(f, WRITE, a, c)
            self.epilogue(f)
            if kind == OP_MEMSET and al is not None and al[2] == MEM_PINNED:  # PAPER.md:463-466 (A7)
                self.acquire(self.H, K_stream(f))
        elif kind == OP_HOST_ACCESS:
            self.access(self.H, WRITE if x else READ, a, c)
        elif kind in (OP_MPI_ISEND, OP_MPI_IRECV):
            if self.free_mpi:
                m = min(self.free_mpi)
                self.free_mpi.remove(m)
            else:
                m = self.new_fiber()
            self.req_fiber[b] = m
            self.fork(self.H, m)
            self.access(m, READ if kind == OP_MPI_ISEND else WRITE, a, c)
            self.release(m, K_req(b))
        elif kind in (OP_MPI_WAIT, OP_MPI_TEST):
            if kind == OP_MPI_WAIT or x:
                self.acquire(self.H, K_req(b))
                m = self.req_fiber.pop(b, None)
                if m is not None:
                    self.free_mpi.append(m)
        elif kind == OP_MPI_SEND:
            self.access(self.H, READ, a, c)
        elif kind == OP_MPI_RECV:
            self.access(self.H, WRITE, a, c)
        elif kind == OP_SET_THREAD:
            if a not in self.thread_fiber:                 # a thread the trace never saw created
                self.thread_fiber[a] = self.new_fiber()
            self.thread = a
        elif kind == OP_THREAD_CREATE:
            if a not in self.thread_fiber:
                self.thread_fiber[a] = self.new_fiber()
            self.fork(self.H, self.thread_fiber[a])        # pthread_create: issue edge
        elif kind == OP_THREAD_JOIN:
            if a in self.thread_fiber:
                self.release(self.thread_fiber[a], K_thread(a))   # child's end ...
                self.acquire(self.H, K_thread(a))                  # ... HB the join's return
        elif kind == OP_DEFAULT_STREAM:
            self.per_thread_mode = bool(x)
        else:
            raise ValueError(f"unknown op {kind}")

    def events(self) -> np.ndarray:
        out = np.zeros(len(self.ev), EVENT_DTYPE)
        if self.ev:
            arr = np.array(self.ev, dtype=object)
            out["kind"] = arr[:, 0].astype(np.uint8)
            out["fiber"] = arr[:, 1].astype(np.uint32)
            out["a"] = np.array([int(v) for v in arr[:, 2]], dtype=np.uint64)
            out["b"] = np.array([int(v) for v in arr[:, 3]], dtype=np.uint64)
            out["mode"] = arr[:, 4].astype(np.uint8)
        return out


def lower(ops: np.ndarray, args: np.ndarray) -> tuple[np.ndarray, int]:
    """API program → (primitive events, number of fibers used)."""
    L = Lowering()
    ops = np.asarray(ops, OP_DTYPE)
    args = np.asarray(args, ARG_DTYPE)
    for op in ops:
        L.call(op, args)
    return L.events(), L.next_fiber
