"""Input formats shared by the product path and the oracle (inputs only — no race-check arithmetic).

Two record formats are defined here, both little-endian and fixed-size so that the C library
(``include/cusan.h``) and the oracle's own reader can consume the same bytes independently:

* **API program** (``OP_DTYPE`` + ``ARG_DTYPE``): the sequence of CUDA / MPI calls a CUDA-aware MPI
  program issues, i.e. what CuSan's compiler pass forwards to its runtime (Fig. 9)
  and what MUST intercepts.  Lowering these calls to happens-before primitives is
  the method's step a0 and is *not* done here.
* **Primitive trace** (``EVENT_DTYPE``): TSan-level events — range accesses and release/acquire/fork
  edges.  Only the fuzz generators emit these directly.

Field meanings per opcode are listed in ``OPS`` and in DESIGN.md §"Input formats".
"""
from __future__ import annotations

import numpy as np

# ---------------------------------------------------------------------------------------------
# API program records (40 B): op u32, x u32, a u64, b u64, c u64, s u64
# ---------------------------------------------------------------------------------------------
OP_DTYPE = np.dtype([("op", "<u4"), ("x", "<u4"), ("a", "<u8"), ("b", "<u8"), ("c", "<u8"), ("s", "<u8")])
ARG_DTYPE = np.dtype([("ptr", "<u8"), ("mode", "<u4"), ("pad", "<u4")])
assert OP_DTYPE.itemsize == 40 and ARG_DTYPE.itemsize == 16

OP_MALLOC = 1            # a=ptr b=size x=mem kind
OP_FREE = 2              # a=ptr
OP_STREAM_CREATE = 3     # s=stream handle x=flags (1 = cudaStreamNonBlocking)
OP_KERNEL = 4            # s=stream b=first arg index x=nargs
OP_STREAM_SYNC = 5       # s=stream
OP_DEVICE_SYNC = 6       # —
OP_EVENT_RECORD = 7      # c=event s=stream
OP_EVENT_SYNC = 8        # c=event
OP_STREAM_WAIT_EVENT = 9  # s=stream c=event
OP_STREAM_QUERY = 10     # s=stream x=1 if it returned cudaSuccess
OP_MEMCPY = 11           # a=dst b=src c=nbytes x=copy kind
OP_MEMCPY_ASYNC = 12     # a=dst b=src c=nbytes x=copy kind s=stream
OP_MEMSET = 13           # a=ptr c=nbytes
OP_MEMSET_ASYNC = 14     # a=ptr c=nbytes s=stream
OP_HOST_ACCESS = 15      # a=addr c=nbytes x=mode   (host load/store, e.g. on managed memory)
OP_MPI_ISEND = 16        # a=buf c=nbytes b=request
OP_MPI_IRECV = 17        # a=buf c=nbytes b=request
OP_MPI_WAIT = 18         # b=request
OP_MPI_SEND = 19         # a=buf c=nbytes
OP_MPI_RECV = 20         # a=buf c=nbytes
OP_MPI_TEST = 21         # b=request x=1 if flag returned true
OP_SET_THREAD = 22       # a=host thread id: the calls that follow are made by this thread
OP_THREAD_CREATE = 23    # a=child thread id (created by the current thread)
OP_THREAD_JOIN = 24      # a=child thread id (joined by the current thread)
OP_DEFAULT_STREAM = 25   # x=1: per-thread default stream mode (handle 0), x=0: legacy (default)

OPS = {v: k for k, v in dict(globals()).items() if k.startswith("OP_") and isinstance(v, int)}

# memory kinds
MEM_DEVICE, MEM_MANAGED, MEM_PINNED, MEM_PAGEABLE = 0, 1, 2, 3
# cudaMemcpyKind
CPY_H2H, CPY_H2D, CPY_D2H, CPY_D2D = 0, 1, 2, 3
# access modes of kernel arguments (R, W or RW)
MODE_R, MODE_W, MODE_RW = 0, 1, 2
STREAM_NONBLOCKING = 1
DEFAULT_STREAM = 0       # stream handle 0 = the default stream (legacy, or per-thread in that mode)
STREAM_LEGACY = 1        # cudaStreamLegacy
STREAM_PER_THREAD = 2    # cudaStreamPerThread
FIRST_USER_STREAM = 16   # generated user-stream handles start here (clear of CUDA's special handles)

# ---------------------------------------------------------------------------------------------
# Primitive trace records (24 B): kind u8, mode u8, pad u16, fiber u32, a u64, b u64
# ---------------------------------------------------------------------------------------------
EVENT_DTYPE = np.dtype([("kind", "u1"), ("mode", "u1"), ("pad", "<u2"), ("fiber", "<u4"),
                        ("a", "<u8"), ("b", "<u8")])
assert EVENT_DTYPE.itemsize == 24
EV_ACCESS, EV_RELEASE, EV_RELEASE_STORE, EV_ACQUIRE, EV_FORK = 0, 1, 2, 3, 4
READ, WRITE = 0, 1

SYNTH_BASE = 0x7F00_0000_0000   # synthetic device address base; allocations are 256-B aligned


class Program:
    """Builder for an API program.  Handles (streams, events, requests) are small integers."""

    def __init__(self, base: int = SYNTH_BASE):
        self.ops: list[tuple] = []
        self.args: list[tuple] = []
        self._next_addr = base
        self._next_stream = FIRST_USER_STREAM
        self._next_event = 1
        self._next_req = 1
        self.allocs: list[tuple[int, int, int]] = []   # (ptr, size, kind)

    # -- allocation ---------------------------------------------------------------------------
    def malloc(self, size: int, kind: int = MEM_DEVICE, align: int = 256) -> int:
        ptr = (self._next_addr + align - 1) // align * align
        self._next_addr = ptr + size
        self.ops.append((OP_MALLOC, kind, ptr, size, 0, 0))
        self.allocs.append((ptr, size, kind))
        return ptr

    def free(self, ptr: int):
        self.ops.append((OP_FREE, 0, ptr, 0, 0, 0))

    # -- streams / events ---------------------------------------------------------------------
    def stream_create(self, nonblocking: bool = False) -> int:
        h = self._next_stream
        self._next_stream += 1
        self.ops.append((OP_STREAM_CREATE, STREAM_NONBLOCKING if nonblocking else 0, 0, 0, 0, h))
        return h

    def new_event(self) -> int:
        h = self._next_event
        self._next_event += 1
        return h

    def kernel(self, stream: int, args: list[tuple[int, int]]):
        first = len(self.args)
        for ptr, mode in args:
            self.args.append((ptr, mode, 0))
        self.ops.append((OP_KERNEL, len(args), 0, first, 0, stream))

    def stream_sync(self, stream: int):
        self.ops.append((OP_STREAM_SYNC, 0, 0, 0, 0, stream))

    def device_sync(self):
        self.ops.append((OP_DEVICE_SYNC, 0, 0, 0, 0, 0))

    def event_record(self, event: int, stream: int):
        self.ops.append((OP_EVENT_RECORD, 0, 0, 0, event, stream))

    def event_sync(self, event: int):
        self.ops.append((OP_EVENT_SYNC, 0, 0, 0, event, 0))

    def stream_wait_event(self, stream: int, event: int):
        self.ops.append((OP_STREAM_WAIT_EVENT, 0, 0, 0, event, stream))

    def stream_query(self, stream: int, success: bool):
        self.ops.append((OP_STREAM_QUERY, 1 if success else 0, 0, 0, 0, stream))

    # -- memory operations --------------------------------------------------------------------
    def memcpy(self, dst: int, src: int, n: int, kind: int):
        self.ops.append((OP_MEMCPY, kind, dst, src, n, 0))

    def memcpy_async(self, dst: int, src: int, n: int, kind: int, stream: int):
        self.ops.append((OP_MEMCPY_ASYNC, kind, dst, src, n, stream))

    def memset(self, ptr: int, n: int):
        self.ops.append((OP_MEMSET, 0, ptr, 0, n, 0))

    def memset_async(self, ptr: int, n: int, stream: int):
        self.ops.append((OP_MEMSET_ASYNC, 0, ptr, 0, n, stream))

    def host_access(self, addr: int, n: int, mode: int):
        self.ops.append((OP_HOST_ACCESS, mode, addr, 0, n, 0))

    # -- MPI ----------------------------------------------------------------------------------
    def isend(self, buf: int, n: int) -> int:
        r = self._next_req
        self._next_req += 1
        self.ops.append((OP_MPI_ISEND, 0, buf, r, n, 0))
        return r

    def irecv(self, buf: int, n: int) -> int:
        r = self._next_req
        self._next_req += 1
        self.ops.append((OP_MPI_IRECV, 0, buf, r, n, 0))
        return r

    def wait(self, req: int):
        self.ops.append((OP_MPI_WAIT, 0, 0, req, 0, 0))

    def test(self, req: int, success: bool):
        self.ops.append((OP_MPI_TEST, 1 if success else 0, 0, req, 0, 0))

    def send(self, buf: int, n: int):
        self.ops.append((OP_MPI_SEND, 0, buf, 0, n, 0))

    def recv(self, buf: int, n: int):
        self.ops.append((OP_MPI_RECV, 0, buf, 0, n, 0))

    # -- host threads and the per-thread default stream --------------------
    def set_thread(self, thread: int):
        self.ops.append((OP_SET_THREAD, 0, thread, 0, 0, 0))

    def thread_create(self, child: int):
        self.ops.append((OP_THREAD_CREATE, 0, child, 0, 0, 0))

    def thread_join(self, child: int):
        self.ops.append((OP_THREAD_JOIN, 0, child, 0, 0, 0))

    def default_stream_mode(self, per_thread: bool):
        self.ops.append((OP_DEFAULT_STREAM, 1 if per_thread else 0, 0, 0, 0, 0))

    # -- output -------------------------------------------------------------------------------
    def arrays(self) -> tuple[np.ndarray, np.ndarray]:
        ops = np.array(self.ops, dtype=OP_DTYPE) if self.ops else np.zeros(0, OP_DTYPE)
        args = np.array(self.args, dtype=ARG_DTYPE) if self.args else np.zeros(0, ARG_DTYPE)
        return ops, args


def events_from_list(evs: list[tuple]) -> np.ndarray:
    """Primitive events given as (kind, fiber, a, b, mode) tuples → EVENT_DTYPE array."""
    out = np.zeros(len(evs), EVENT_DTYPE)
    for i, (kind, fiber, a, b, mode) in enumerate(evs):
        out[i] = (kind, mode, 0, fiber, a, b)
    return out


def save_events(path: str, ev: np.ndarray, max_fibers: int):
    """Trace file: 16-B header ('CSTR', version 1, max_fibers u32, pad) + n u64 + records."""
    with open(path, "wb") as f:
        f.write(b"CSTR")
        f.write(np.array([1, max_fibers], "<u4").tobytes())
        f.write(np.array([0], "<u4").tobytes())
        f.write(np.array([len(ev)], "<u8").tobytes())
        f.write(np.ascontiguousarray(ev, EVENT_DTYPE).tobytes())
