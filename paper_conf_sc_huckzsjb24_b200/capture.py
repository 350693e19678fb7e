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

Point-to-point communication (`isend`, `irecv`, `send`, `recv`) can be recorded with
`Capture.isend` / `irecv` / `send` / `recv` / `wait`: MPI semantics (a fiber per request, completed
by the wait) — or, for NCCL (`stream_ordered=True`), NCCL's: the communication
runs on a communication stream that waits on the current stream and the wait makes the current
stream wait.
"""
from __future__ import annotations

import itertools
from typing import Any

import torch
from torch.utils._python_dispatch import TorchDispatchMode
from torch.utils import _pytree as pytree

from . import Report, Trace, Lowering, check

_aten = torch.ops.aten
_COPY_OPS = ("aten::copy_", "aten::_to_copy", "aten::_local_scalar_dense", "aten::_copy_from",
             "aten::_copy_from_and_resize")
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
    _HOOKS_INSTALLED = True


class _Dispatch(TorchDispatchMode):
    def __init__(self, cap: "Capture"):
        super().__init__()
        self.cap = cap

    def __torch_dispatch__(self, func, types, args=(), kwargs=None):
        kwargs = kwargs or {}
        out = func(*args, **kwargs)
        if func is not _aten.record_stream.default:
            self.cap._on_op(func, args, kwargs, out)
        return out


class Capture:
    """Context manager recording the CUDA work of the enclosed PyTorch code.

        with Capture() as cap:
            ...                      # PyTorch code on CUDA tensors
        rep = cap.check()            # GPU happens-before race check of what ran
    """

    def __init__(self, max_fibers: int = 255):
        self.trace = Trace(max_fibers)
        self.low = Lowering(self.trace)
        self.streams: set[int] = {0}
        self.allocs: dict[int, int] = {}
        self.ops = 0
        self.op_names: dict[int, str] = {}           # first event id of an op -> op name
        self._req = itertools.count(1)
        self._ev = itertools.count(1 << 40)          # synthetic event handles for NCCL modelling
        self._mode = None

    # ---- context ---------------------------------------------------------------------------------
    def __enter__(self):
        global _ACTIVE
        if _ACTIVE is not None:
            raise RuntimeError("a Capture is already active")
        _install_hooks()
        torch.cuda.synchronize()                     # work issued before the capture is complete
        _ACTIVE = self
        self._mode = _Dispatch(self)
        self._mode.__enter__()
        return self

    def __exit__(self, *exc):
        global _ACTIVE
        self._mode.__exit__(*exc)
        self._mode = None
        _ACTIVE = None
        return False

    def check(self, **kw) -> Report:
        """Run the race check on the captured trace (kw: cusan_check options)."""
        return check(self.trace, **kw)

    # ---- helpers ----------------------------------------------------------------------------------
    def _stream(self, handle: int) -> int:
        if handle not in self.streams:
            self.streams.add(handle)
            self.low.cusan_on_stream_create(handle, 1)   # PyTorch streams are non-blocking
        return handle

    def _storage(self, t: torch.Tensor) -> int:
        st = t.untyped_storage()
        ptr, size = st.data_ptr(), st.nbytes()
        if ptr and self.allocs.get(ptr) != size:
            self.allocs[ptr] = size
            self.low.cusan_on_malloc(ptr, size, 0)
        return ptr

    # ---- CUDA trace callbacks -----------------------------------------------------------------------
    def _on_stream_creation(self, stream: int):
        self._stream(stream)

    def _on_event_record(self, event: int, stream: int):
        self.low.cusan_on_event_record(event, self._stream(stream))

    def _on_event_wait(self, event: int, stream: int):
        self.low.cusan_on_stream_wait_event(self._stream(stream), event)

    def _on_event_sync(self, event: int):
        self.low.cusan_on_event_sync(event)

    def _on_stream_sync(self, stream: int):
        self.low.cusan_on_stream_sync(self._stream(stream))

    def _on_device_sync(self):
        self.low.cusan_on_device_sync()

    # ---- operator dispatch ---------------------------------------------------------------------------
    def _on_op(self, func, args, kwargs, out):
        schema = func._schema
        name = schema.name
        # allocation only (no kernel touches the memory) / tensors passed only for their shape
        alloc_only = name in ("aten::empty", "aten::empty_like", "aten::empty_strided", "aten::new_empty",
                              "aten::new_empty_strided")
        shape_only_inputs = alloc_only or name.endswith("_like")
        acc: dict[int, int] = {}                      # storage -> mode (0 R, 1 W)
        host_copy = name == "aten::_local_scalar_dense"   # .item(): blocking device->host read

        def add(v, write, metadata_only):
            nonlocal host_copy
            if not isinstance(v, torch.Tensor):
                return
            if not v.is_cuda:
                host_copy = True
                return
            ptr = self._storage(v)
            if not ptr:
                return
            if write:
                acc[ptr] = 1
            elif not metadata_only:
                acc.setdefault(ptr, 0)

        values = list(args) + [kwargs.get(a.name) for a in schema.arguments[len(args):]]
        for a, v in zip(schema.arguments, values):
            write = a.alias_info is not None and a.alias_info.is_write
            meta = shape_only_inputs or (a.alias_info is not None and not a.alias_info.is_write)
            pytree.tree_map_(lambda x: add(x, write, meta), v)
        outs = out if isinstance(out, (tuple, list)) else (out,)
        for r, v in zip(schema.returns, outs):
            meta = alloc_only or (r.alias_info is not None and not r.alias_info.is_write)
            pytree.tree_map_(lambda x: add(x, not meta, meta), v)
        if not acc:
            return
        stream = self._stream(torch.cuda.current_stream().cuda_stream)
        first = len(self.trace)
        self.low.cusan_on_kernel(stream, list(acc.keys()), list(acc.values()))
        self.op_names[first] = schema.name
        self.ops += 1
        non_blocking = bool(kwargs.get("non_blocking", False)) or (
            func in (_aten.copy_.default,) and len(args) > 2 and bool(args[2]))
        if host_copy and not non_blocking and name in _COPY_OPS:
            self.low.cusan_on_stream_sync(stream)     # blocking host<->device copy

    # ---- point-to-point communication ----------------------------------------------------------------
    def isend(self, tensor: torch.Tensor, stream_ordered: bool = False):
        return self._p2p(tensor, 0, stream_ordered)

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

    def wait(self, handle: Any):
        kind, v = handle
        if kind == "mpi":
            self.low.cusan_on_mpi_wait(v)
        else:
            self.low.cusan_on_stream_wait_event(self._stream(torch.cuda.current_stream().cuda_stream), v)

    def send(self, tensor: torch.Tensor):
        self.low.cusan_on_mpi_send(self._storage(tensor), tensor.untyped_storage().nbytes())

    def recv(self, tensor: torch.Tensor):
        self.low.cusan_on_mpi_recv(self._storage(tensor), tensor.untyped_storage().nbytes())
