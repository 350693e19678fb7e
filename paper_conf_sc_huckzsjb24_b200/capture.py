"""Live capture of a PyTorch program's CUDA semantics into a cusan trace.

The paper's CuSan gets CUDA calls from a compiler pass (Fig. 9).  For PyTorch
programs the same information is available at run time — the hook points PyTorch's own CUDA Stream
Sanitizer uses (the comparison the paper draws):

* every ATen operator dispatch (TorchDispatchMode): the current stream, and per CUDA tensor argument
  whether the operator schema marks it written (`alias_info.is_write`, outputs) or read — CuSan's
  per-argument R/W attributes; the extent is the tensor's whole storage, the
  allocation TypeART would report;
* the CUDA trace callbacks (`torch.cuda._gpu_trace`): stream creation, event record / wait /
  synchronize, stream and device synchronize.

Each is forwarded to the lowering C ABI (`cusan_on_*`, include/cusan_lower.h), which appends the
happens-before primitives; the check itself is `Capture.check()` on the GPU.  PyTorch creates its
side streams with cudaStreamNonBlocking, so they are registered as non-blocking streams; stream 0 is
the legacy default stream.  A host-blocking device->host copy (`.cpu()`, `.item()`) is a kernel on
the current stream followed by a stream synchronisation, which is what PyTorch does.

Point-to-point communication through `torch.distributed` (`isend`, `irecv`, `send`, `recv`,
`batch_isend_irecv`) is recorded automatically inside a capture: the functions are wrapped for its
duration and the `Work` handles they return record the completion when waited on (or when
`is_completed()` first returns True, MPI_Test).  Two semantics, by the process group's backend:
MPI's for host-driven backends (a request fiber, completed by the wait) and
NCCL's for `nccl` (the transfer runs on a communication stream that waits on the current stream,
and `wait()` makes the current stream wait on it) — so a kernel that touches the buffer before
the wait races with the transfer, as in Fig. 6A.  The same records can be made
by hand with `Capture.isend` / `irecv` / `send` / `recv` / `wait` (e.g. for another communication
library).  Collectives (`c10d::allreduce_` …) are recorded as an operation on the current stream
(NCCL's stream-ordered semantics for synchronous collectives).

Host threads: every Python thread that issues CUDA work
inside a capture is its own host fiber (`cusan_on_thread`); `threading.Thread.start` is recorded as
an issue edge from the starting thread and a completed `join` as the joined thread's release
acquired by the joiner, and threads started inside the capture get the operator-dispatch hook too
(dispatch modes are thread-local).  Records are serialised by a lock, so the trace order is the
order in which the threads issued their calls.
"""
from __future__ import annotations

import functools
import itertools
import threading
import weakref
from typing import Any

import torch
from torch.utils._python_dispatch import TorchDispatchMode

from . import Report, Session, Trace, Lowering, check

_aten = torch.ops.aten
_COPY_OPS = ("aten::copy_", "aten::_to_copy", "aten::_local_scalar_dense", "aten::_copy_from",
             "aten::_copy_from_and_resize")
_P2P_OPS = ("c10d::send", "c10d::recv_", "c10d::recv_any_source_")
_ACTIVE: "Capture | None" = None
_HOOKS_INSTALLED = False


def _install_hooks():
    """Register the CUDA trace callbacks once per process; they forward to the active capture."""
    global _HOOKS_INSTALLED
    if _HOOKS_INSTALLED:
        return
    from torch.cuda import _gpu_trace as gt
    torch._C._activate_gpu_trace()

    def fwd(name):
        def cb(*a):
            cap = _ACTIVE
            if cap is not None:
                getattr(cap, name)(*a)
        return cb

    gt.register_callback_for_stream_creation(fwd("_on_stream_creation"))
    gt.register_callback_for_event_record(fwd("_on_event_record"))
    gt.register_callback_for_event_wait(fwd("_on_event_wait"))
    gt.register_callback_for_event_synchronization(fwd("_on_event_sync"))
    gt.register_callback_for_stream_synchronization(fwd("_on_stream_sync"))
    gt.register_callback_for_device_synchronization(fwd("_on_device_sync"))
    gt.register_callback_for_memory_deallocation(fwd("_on_memory_deallocation"))
    _HOOKS_INSTALLED = True


def _recording(fn):
    """A recording entry point: serialised, and attributed to the calling host thread."""
    @functools.wraps(fn)
    def wrapped(self, *a, **k):
        with self._lock:
            self._as_current_thread()
            return fn(self, *a, **k)
    return wrapped


class _Dispatch(TorchDispatchMode):
    def __init__(self, cap: "Capture"):
        super().__init__()
        self.cap = cap

    def __torch_dispatch__(self, func, types, args=(), kwargs=None):
        kwargs = kwargs or {}
        out = func(*args, **kwargs)
        if func not in self.cap._silent and func is not _aten.record_stream.default and _ACTIVE is self.cap:
            self.cap._on_op(func, args, kwargs, out)          # (threads may outlive the capture)
        return out


class Capture:
    """Context manager recording the CUDA work of the enclosed PyTorch code.

        with Capture() as cap:
            ...                      # PyTorch code on CUDA tensors
        rep = cap.check()            # GPU happens-before race check of what ran
    """

    def __init__(self, max_fibers: int = 255, intercept_distributed: bool = True):
        self.intercept_distributed = intercept_distributed
        self._patched: list[tuple[Any, str, Any]] = []
        self._in_p2p = False
        self._lock = threading.RLock()
        self._tids: dict[threading.Thread, int] = {}   # host thread -> thread id in the trace
        self._cur_tid = 0
        self.trace = Trace(max_fibers)
        self.low = Lowering(self.trace)
        self.streams: set[int] = {0}
        # Every allocation instance gets its own synthetic address range in the trace: the caching
        # allocator hands a freed block to the next tensor (after the stream / event ordering it
        # enforces itself), and that tensor's accesses must start from fresh shadow state, as
        # PyTorch's stream sanitizer resets a tensor's state at deallocation.  `allocs` maps a live
        # storage pointer to (synthetic base, size); `real` maps synthetic bases back.
        self.allocs: dict[int, tuple[int, int]] = {}
        self.real: dict[int, tuple[int, int]] = {}
        self._next_base = 1 << 44
        self.ops = 0
        self.op_names: dict[int, str] = {}           # first event id of an op -> op name
        self._plans: dict[Any, tuple] = {}           # operator -> its schema's recording plan
        self._silent: set = set()                    # operators that never touch tensor memory (views)
        self._sessions: list = []                    # weak references to sessions from session()
        self._req = itertools.count(1)
        self._ev = itertools.count(1 << 40)          # synthetic event handles for NCCL modelling
        self._mode = None

    # ---- context ---------------------------------------------------------------------------------
    def __enter__(self):
        global _ACTIVE
        if _ACTIVE is not None:
            raise RuntimeError("a Capture is already active")
        _install_hooks()
        if torch.cuda.is_available():
            torch.cuda.synchronize()                 # work issued before the capture is complete
        _ACTIVE = self
        self._tids = {threading.current_thread(): 0}    # the capturing thread is thread 0 (fiber 0)
        self._cur_tid = 0
        if self.intercept_distributed:
            self._patch_distributed()
        self._patch_threads()
        self._mode = _Dispatch(self)
        self._mode.__enter__()
        return self

    def __exit__(self, *exc):
        global _ACTIVE
        self._mode.__exit__(*exc)
        self._mode = None
        for mod, name, fn in reversed(self._patched):
            setattr(mod, name, fn)
        self._patched.clear()
        _ACTIVE = None
        return False

    def check(self, **kw) -> Report:
        """Run the race check on the captured trace (kw: cusan_check options)."""
        return check(self.trace, **kw)

    def session(self, **kw) -> Session:
        """An online check of the captured trace (f1): `session().check()` checks what the program
        did since the previous call.  Allocation instances the caching allocator releases are
        forgotten by the session (cusan_session_forget: their ranges are never touched again — the
        next tensor at that address gets a new range), so its layout and per-call cost stay
        bounded however long the program runs.  kw: Session options."""
        ses = Session(self.trace, **kw)
        self._sessions.append(weakref.ref(ses))
        return ses

    # ---- helpers ----------------------------------------------------------------------------------
    def _stream(self, handle: int) -> int:
        if handle not in self.streams:
            self.streams.add(handle)
            self.low.cusan_on_stream_create(handle, 1)   # PyTorch streams are non-blocking
        return handle

    def _storage(self, t: torch.Tensor) -> int:
        """The trace address of a tensor's storage: its allocation instance's synthetic base."""
        st = t.untyped_storage()
        ptr, size = st.data_ptr(), st.nbytes()
        if not ptr:
            return 0
        cur = self.allocs.get(ptr)
        if cur is None or cur[1] != size:
            base = self._next_base
            self._next_base += (max(size, 1) + 255) // 256 * 256 + 256
            self.allocs[ptr] = (base, size)
            self.real[base] = (ptr, size)
            self.low.cusan_on_malloc(base, size, 0)
        return self.allocs[ptr][0]

    def real_address(self, addr: int) -> int:
        """Device address of a trace (synthetic) address, e.g. ``8 * run["g_begin"]``."""
        import bisect
        bases = sorted(self.real)
        i = bisect.bisect_right(bases, addr) - 1
        if i < 0:
            raise KeyError(addr)
        ptr, size = self.real[bases[i]]
        if addr - bases[i] > size:
            raise KeyError(addr)
        return ptr + (addr - bases[i])

    # ---- CUDA trace callbacks -----------------------------------------------------------------------
    @_recording
    def _on_stream_creation(self, stream: int):
        self._stream(stream)

    @_recording
    def _on_event_record(self, event: int, stream: int):
        self.low.cusan_on_event_record(event, self._stream(stream))

    @_recording
    def _on_event_wait(self, event: int, stream: int):
        self.low.cusan_on_stream_wait_event(self._stream(stream), event)

    @_recording
    def _on_event_sync(self, event: int):
        self.low.cusan_on_event_sync(event)

    @_recording
    def _on_stream_sync(self, stream: int):
        self.low.cusan_on_stream_sync(self._stream(stream))

    @_recording
    def _on_device_sync(self):
        self.low.cusan_on_device_sync()

    @_recording
    def _on_memory_deallocation(self, ptr: int):
        # the block goes back to the caching allocator (no cudaFree, no device sync): forget this
        # instance, so the next tensor at the same address gets a fresh range
        inst = self.allocs.pop(ptr, None)
        if inst is not None and self._sessions:
            live = []
            for ref in self._sessions:
                ses = ref()
                if ses is not None and getattr(ses, "h", None):
                    ses.forget(inst[0], inst[1])
                    live.append(ref)
            self._sessions = live

    # ---- operator dispatch ---------------------------------------------------------------------------
    def _op_plan(self, func):
        """What the operator schema says about each argument, computed once per operator: (name,
        alloc_only, is the blocking-copy candidate, per argument (name, write, metadata only), per
        return metadata only)."""
        plan = self._plans.get(func)
        if plan is None:
            schema = func._schema
            name = schema.name
            # allocation only (no kernel touches the memory) / tensors passed only for their shape
            alloc_only = name in ("aten::empty", "aten::empty_like", "aten::empty_strided", "aten::new_empty",
                                  "aten::new_empty_strided")
            shape_only_inputs = alloc_only or name.endswith("_like")
            argv = tuple((a.name, a.alias_info is not None and a.alias_info.is_write,
                          shape_only_inputs or (a.alias_info is not None and not a.alias_info.is_write))
                         for a in schema.arguments)
            rets = tuple(alloc_only or (r.alias_info is not None and not r.alias_info.is_write) for r in schema.returns)
            plan = (name, name in _COPY_OPS, argv, rets)
            self._plans[func] = plan
            if all(meta and not write for _, write, meta in argv) and all(rets) and name not in _P2P_OPS \
                    and name != "aten::_local_scalar_dense":
                self._silent.add(func)                # views: no tensor is read or written
        return plan

    @_recording
    def _on_op(self, func, args, kwargs, out):
        name, copy_op, argv, rets = self._op_plan(func)
        if self._in_p2p and name in _P2P_OPS:
            return                                    # recorded by the torch.distributed wrapper
        acc: dict[int, int] = {}                      # storage -> mode (0 R, 1 W)
        host_copy = name == "aten::_local_scalar_dense"   # .item(): blocking device->host read
        Tensor = torch.Tensor

        def add(v, write, meta):                      # a tensor, or lists / tuples of them
            nonlocal host_copy
            if isinstance(v, Tensor):
                if not v.is_cuda:
                    host_copy = True
                    return
                ptr = self._storage(v)
                if not ptr:
                    return
                if write:
                    acc[ptr] = 1
                elif not meta:
                    acc.setdefault(ptr, 0)
            elif isinstance(v, (list, tuple)):
                for x in v:
                    add(x, write, meta)

        na = len(args)
        for i, (aname, write, meta) in enumerate(argv):
            v = args[i] if i < na else kwargs.get(aname)
            if v is not None:
                add(v, write, meta)
        outs = out if isinstance(out, (tuple, list)) else (out,)
        for meta, v in zip(rets, outs):
            add(v, not meta, meta)
        if not acc:
            return
        stream = self._stream(torch._C._cuda_getCurrentRawStream(torch.cuda.current_device()))
        first = len(self.trace)
        self.low.cusan_on_kernel(stream, list(acc.keys()), list(acc.values()))
        self.op_names[first] = name
        self.ops += 1
        if host_copy and copy_op:
            non_blocking = bool(kwargs.get("non_blocking", False)) or (
                func is _aten.copy_.default and len(args) > 2 and bool(args[2]))
            if not non_blocking:
                self.low.cusan_on_stream_sync(stream)     # blocking host<->device copy

    # ---- point-to-point communication ----------------------------------------------------------------
    @_recording
    def isend(self, tensor: torch.Tensor, stream_ordered: bool = False):
        return self._p2p(tensor, 0, stream_ordered)

    @_recording
    def irecv(self, tensor: torch.Tensor, stream_ordered: bool = False):
        return self._p2p(tensor, 1, stream_ordered)

    def _p2p(self, tensor, write, stream_ordered):
        ptr = self._storage(tensor)
        n = tensor.untyped_storage().nbytes()
        if not stream_ordered:                         # MPI: a request fiber
            req = next(self._req)
            (self.low.cusan_on_mpi_irecv if write else self.low.cusan_on_mpi_isend)(ptr, n, req)
            return ("mpi", req)
        # NCCL: the communication stream waits on the current stream, runs the transfer, and
        # records an event the waiter's stream later waits on
        cur = self._stream(torch.cuda.current_stream().cuda_stream)
        comm = self._stream((1 << 41) + 1)
        e1, e2 = next(self._ev), next(self._ev)
        self.low.cusan_on_event_record(e1, cur)
        self.low.cusan_on_stream_wait_event(comm, e1)
        self.low.cusan_on_kernel(comm, [ptr], [write])
        self.low.cusan_on_event_record(e2, comm)
        return ("nccl", e2)

    @_recording
    def wait(self, handle: Any):
        kind, v = handle
        if kind == "mpi":
            self.low.cusan_on_mpi_wait(v)
        else:
            self.low.cusan_on_stream_wait_event(self._stream(torch.cuda.current_stream().cuda_stream), v)

    @_recording
    def send(self, tensor: torch.Tensor):
        self.low.cusan_on_mpi_send(self._storage(tensor), tensor.untyped_storage().nbytes())

    @_recording
    def recv(self, tensor: torch.Tensor):
        self.low.cusan_on_mpi_recv(self._storage(tensor), tensor.untyped_storage().nbytes())

    # ---- host threads ---------------------------------------------------------------------------------
    def _thread_id(self, th: threading.Thread) -> int:
        if th not in self._tids:
            self._tids[th] = len(self._tids)
        return self._tids[th]

    def _as_current_thread(self):
        tid = self._thread_id(threading.current_thread())
        if tid != self._cur_tid:
            self.low.cusan_on_thread(tid)
            self._cur_tid = tid

    def _patch_threads(self):
        cap = self
        orig_start, orig_join = threading.Thread.start, threading.Thread.join

        def start(th):
            with cap._lock:
                cap._as_current_thread()
                cap.low.cusan_on_thread_create(cap._thread_id(th))   # issue edge parent -> child
            body = th.run

            def run():
                with _Dispatch(cap):               # dispatch modes are per thread
                    body()
            th.run = run
            return orig_start(th)

        def join(th, timeout=None):
            out = orig_join(th, timeout)
            if not th.is_alive() and th in cap._tids and _ACTIVE is cap:
                with cap._lock:
                    cap._as_current_thread()
                    cap.low.cusan_on_thread_join(cap._tids[th])       # child release, caller acquire
            return out

        for name, fn, orig in (("start", start, orig_start), ("join", join, orig_join)):
            self._patched.append((threading.Thread, name, orig))
            setattr(threading.Thread, name, fn)

    # ---- torch.distributed interception --------------------------------------------------------------
    def _patch_distributed(self):
        import torch.distributed as dist
        if not dist.is_available():
            return
        import torch.distributed.distributed_c10d as c10d
        cap = self

        def nccl(group) -> bool:
            try:
                return dist.get_backend(group) == "nccl"
            except Exception:                          # no default group yet
                return False

        def start(tensor, write, group):
            if not isinstance(tensor, torch.Tensor) or not tensor.is_cuda:
                return None                            # host tensors are not tracked
            return (cap.irecv if write else cap.isend)(tensor, nccl(group))   # serialised, this thread

        def call(fn, *a, **k):
            prev, cap._in_p2p = cap._in_p2p, True
            try:
                return fn(*a, **k)
            finally:
                cap._in_p2p = prev

        orig = {n: getattr(c10d, n) for n in ("isend", "irecv", "send", "recv", "batch_isend_irecv")}

        def nonblocking(name, write):
            def wrapped(tensor, *a, **k):
                if cap._in_p2p:                        # inside batch_isend_irecv: recorded there
                    return orig[name](tensor, *a, **k)
                h = start(tensor, write, k.get("group", a[1] if len(a) > 1 else None))
                work = call(orig[name], tensor, *a, **k)
                return _Work(work, cap, [h] if h else [])
            wrapped.__name__ = name
            return wrapped

        def blocking(name, write):
            def wrapped(tensor, *a, **k):
                group = k.get("group", a[1] if len(a) > 1 else None)
                out = call(orig[name], tensor, *a, **k)
                if isinstance(tensor, torch.Tensor) and tensor.is_cuda:
                    if nccl(group):                    # stream-ordered transfer, waited on
                        cap.wait((cap.irecv if write else cap.isend)(tensor, True))
                    else:                              # host-blocking (MPI_Send / MPI_Recv)
                        (cap.recv if write else cap.send)(tensor)
                return out
            wrapped.__name__ = name
            return wrapped

        def batch(p2p_op_list):
            handles = []
            for op in p2p_op_list:
                write = getattr(op.op, "__name__", "") == "irecv"
                h = start(op.tensor, write, op.group)
                if h:
                    handles.append(h)
            works = call(orig["batch_isend_irecv"], p2p_op_list)
            return [_Work(w, cap, handles) for w in works]

        repl = {"isend": nonblocking("isend", 0), "irecv": nonblocking("irecv", 1),
                "send": blocking("send", 0), "recv": blocking("recv", 1), "batch_isend_irecv": batch}
        for mod in (c10d, dist):
            for name, fn in repl.items():
                if getattr(mod, name, None) is orig[name]:
                    self._patched.append((mod, name, orig[name]))
                    setattr(mod, name, fn)


class _Work:
    """A torch.distributed Work whose completion (wait, or is_completed() returning True) is
    recorded in the capture: MPI_Wait / MPI_Test(success) for request fibers, the current stream
    waiting on the transfer for NCCL.  Everything else is the wrapped Work's."""

    def __init__(self, work, cap: Capture, handles: list):
        self._work = work
        self._cap = cap
        self._handles = handles

    def _complete(self):
        for h in self._handles:
            if not h[0].endswith("done"):
                self._cap.wait(h)
        self._handles[:] = [(k + "-done", v) for k, v in self._handles]

    def wait(self, *a, **k):
        out = self._work.wait(*a, **k) if self._work is not None else True
        if _ACTIVE is self._cap:
            self._complete()
        return out

    def is_completed(self):
        done = self._work.is_completed() if self._work is not None else True
        if done and _ACTIVE is self._cap:
            self._complete()
        return done

    def __getattr__(self, name):
        return getattr(self._work, name)
