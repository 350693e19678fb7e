"""paper_conf_sc_huckzsjb24_b200 — B200-native happens-before race check over device memory.

Thin Python binding of ``libcusan.so`` (C ABI in ``include/cusan.h`` and ``include/cusan_lower.h``).
Function and method names follow the C names; everything here is argument marshalling — every step
of the check runs in the library (host C++ for a0-a2, sm_100a kernels for a3/a4).  Importing this
module fails if the library is missing; there is no CPU fallback.

    tr = Trace(max_fibers=8)
    low = Lowering(tr); low.cusan_lower_program(ops, args)    # or tr.cusan_trace_append_*
    rep = check(tr)                                            # K1 on cuda:0
    rep.n_race_granules, rep.runs                              # canonical race runs
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from ._lib import (CusanError, check as _ck, cusan_check_opts, cusan_counters, cusan_race_run, lib)

RUN_DTYPE = np.dtype([("g_begin", "<u8"), ("g_end", "<u8"), ("earlier", "<u4"), ("later", "<u4")])
EVENT_DTYPE = np.dtype([("kind", "u1"), ("mode", "u1"), ("pad", "<u2"), ("fiber", "<u4"),
                        ("a", "<u8"), ("b", "<u8")])
OP_DTYPE = np.dtype([("op", "<u4"), ("x", "<u4"), ("a", "<u8"), ("b", "<u8"), ("c", "<u8"), ("s", "<u8")])
ARG_DTYPE = np.dtype([("ptr", "<u8"), ("mode", "<u4"), ("pad", "<u4")])

CUSAN_READ, CUSAN_WRITE = 0, 1
CUSAN_RELEASE, CUSAN_RELEASE_STORE, CUSAN_ACQUIRE, CUSAN_FORK = 0, 1, 2, 3
__all__ = ["Trace", "Lowering", "Clocks", "Plan", "Report", "check", "pipelined_checks", "report_merge", "CusanError", "version",
           "RUN_DTYPE", "EVENT_DTYPE", "release_cached_memory"]


def version() -> str:
    return lib.cusan_version().decode()


def _ptr(a: np.ndarray) -> C.c_void_p:
    return C.c_void_p(a.ctypes.data) if a.size else C.c_void_p(0)


class Trace:
    """cusan_trace: the primitive event trace (step a0)."""

    def __init__(self, max_fibers: int = 255, reserve_events: int = 0):
        h = C.c_void_p()
        _ck(lib.cusan_trace_create(max_fibers, reserve_events, C.byref(h)))
        self.h = h

    def __del__(self, _destroy=lib.cusan_trace_destroy):   # bound now: safe at interpreter exit
        if getattr(self, "h", None):
            _destroy(self.h)
            self.h = None

    def cusan_trace_append_access(self, fiber: int, mode: int, addr: int, nbytes: int) -> int:
        ev = C.c_uint32()
        _ck(lib.cusan_trace_append_access(self.h, fiber, mode, addr, nbytes, C.byref(ev)))
        return ev.value

    def cusan_trace_append_sync(self, kind: int, fiber: int, key_or_src: int) -> int:
        ev = C.c_uint32()
        _ck(lib.cusan_trace_append_sync(self.h, kind, fiber, key_or_src, C.byref(ev)))
        return ev.value

    def cusan_trace_append_events(self, events: np.ndarray):
        ev = np.ascontiguousarray(events, EVENT_DTYPE)
        _ck(lib.cusan_trace_append_events(self.h, _ptr(ev), len(ev)))

    def cusan_trace_size(self) -> tuple[int, int]:
        n, f = C.c_uint64(), C.c_uint32()
        _ck(lib.cusan_trace_size(self.h, C.byref(n), C.byref(f)))
        return n.value, f.value

    def cusan_trace_read(self, first: int = 0, n: int | None = None) -> np.ndarray:
        total, _ = self.cusan_trace_size()
        n = total - first if n is None else n
        out = np.zeros(n, EVENT_DTYPE)
        _ck(lib.cusan_trace_read(self.h, first, n, _ptr(out)))
        return out

    def __len__(self):
        return self.cusan_trace_size()[0]


_LOWERING_FNS: dict = {}                     # cusan_on_* name -> its ctypes function


class Lowering:
    """cusan_lowering: CUDA / MPI call -> primitive lowering (CuSan's per-device context)."""

    def __init__(self, trace: Trace):
        h = C.c_void_p()
        _ck(lib.cusan_lowering_create(trace.h, C.byref(h)))
        self.h = h
        self.trace = trace

    def __del__(self, _destroy=lib.cusan_lowering_destroy):
        if getattr(self, "h", None):
            _destroy(self.h)
            self.h = None

    def cusan_lowering_fiber_info(self, fiber: int) -> tuple[int, int]:
        """(cusan_fiber_kind, handle) of a fiber: thread id, stream handle or MPI request."""
        kind, handle = C.c_int(), C.c_uint64()
        _ck(lib.cusan_lowering_fiber_info(self.h, fiber, C.byref(kind), C.byref(handle)))
        return kind.value, handle.value

    def cusan_lowering_set_default_stream(self, per_thread: bool):
        _ck(lib.cusan_lowering_set_default_stream(self.h, int(per_thread)))

    def cusan_lowering_fibers(self) -> int:
        n = C.c_uint32()
        _ck(lib.cusan_lowering_fibers(self.h, C.byref(n)))
        return n.value

    def cusan_lower_program(self, ops: np.ndarray, args: np.ndarray) -> np.ndarray:
        """Lower a recorded API program; returns the first event id of every call."""
        ops = np.ascontiguousarray(ops, OP_DTYPE)
        args = np.ascontiguousarray(args, ARG_DTYPE)
        first = np.zeros(len(ops), np.uint32)
        _ck(lib.cusan_lower_program(self.h, _ptr(ops), len(ops), _ptr(args), len(args),
                                    first.ctypes.data_as(C.POINTER(C.c_uint32))))
        return first

    def __getattr__(self, name):
        """cusan_on_*(...) → the C call with this lowering as first argument."""
        if name.startswith("cusan_on_"):
            fn = _LOWERING_FNS.get(name)
            if fn is None:
                fn = _LOWERING_FNS[name] = getattr(lib, name)
            if name == "cusan_on_kernel":
                def call(stream, ptrs, modes):
                    n = len(ptrs)
                    _ck(fn(self.h, stream, n, (C.c_uint64 * n)(*ptrs), (C.c_uint32 * n)(*modes)))
            else:
                def call(*a):
                    _ck(fn(self.h, *a))
            return call
        raise AttributeError(name)


class Report:
    """cusan_report: race count, canonical runs, counters."""

    def __init__(self, h: C.c_void_p, max_runs: int = 0):
        self.h = h
        ng, nr, tr = C.c_uint64(), C.c_uint64(), C.c_int()
        rp = C.POINTER(cusan_race_run)()
        _ck(lib.cusan_report_get(h, C.byref(ng), C.byref(nr), C.byref(rp), C.byref(tr)))
        self.n_race_granules = ng.value
        self.n_runs = nr.value
        self.truncated = bool(tr.value)
        kept = nr.value if not tr.value else min(nr.value, max_runs)
        self._counters = None
        if kept:
            buf = (C.c_char * (kept * RUN_DTYPE.itemsize)).from_address(C.addressof(rp.contents))
            self.runs = np.frombuffer(bytes(buf), RUN_DTYPE).copy()
        else:
            self.runs = np.zeros(0, RUN_DTYPE)

    @property
    def counters(self) -> dict:
        """cusan_report_counters as a dict (read on first use: an online checker's per-call report
        need not pay for it)."""
        if self._counters is None:
            ctr = cusan_counters()
            _ck(lib.cusan_report_counters(self.h, C.byref(ctr)))
            self._counters = {n: getattr(ctr, n) for n, _ in cusan_counters._fields_}
        return self._counters

    def __del__(self, _free=lib.cusan_report_free):
        if getattr(self, "h", None):
            _free(self.h)
            self.h = None


def _opts(nshards=1, shard=0, device=0, window_events=0, persist_shadow=False, max_runs=0, stream=None,
          flags=0, shard_block=0, ngpus=0):
    o = cusan_check_opts()
    lib.cusan_check_opts_init(C.byref(o))
    o.nshards, o.shard, o.device, o.flags = nshards, shard, device, flags
    o.window_events, o.persist_shadow, o.max_runs = window_events, int(persist_shadow), max_runs
    o.stream = stream
    o.shard_block = shard_block
    o.ngpus = ngpus
    return o


def _report(h, max_runs):
    return Report(h, max_runs)


CUSAN_CHECK_DEFER_WORKSPACE = 2
CUSAN_CHECK_INTERVAL_SHADOW = 4    # the default shadow: one cell per elementary interval (f3)
CUSAN_CHECK_DENSE_SHADOW = 8       # one cell per 8-byte granule (TSan's layout, §8(d) roofline line)
CUSAN_CHECK_HOST_PLAN = 16         # build the a2 tables on the host (default: device for >= 32768 accesses)
CUSAN_CHECK_DEVICE_PLAN = 32       # build them on the device whatever the trace size
DSPAN_DTYPE = np.dtype([("abs_begin", "<u8"), ("dense_begin", "<u8"), ("len", "<u8"), ("tile0", "<u8"),
                        ("weight0", "<u8"), ("rsize", "<u4"), ("rweight", "<u4"), ("list_off", "<u4"),
                        ("list_cnt", "<u4"), ("flags", "<u4"), ("rec", "<u4"), ("rec_units", "<u4"),
                        ("pad", "<u4")])
INC_DTYPE = np.dtype([("epoch", "<u4"), ("segm", "<u4")])


def _torch_workspace(nbytes: int, device: int, stream):
    """A uint8 CUDA tensor of nbytes from PyTorch's caching allocator, allocated on the stream the
    plan runs on (`stream`, a cudaStream_t as int), so the allocator orders its reuse after the plan."""
    import torch
    dev = torch.device("cuda", device)
    with torch.cuda.stream(torch.cuda.ExternalStream(stream, device=dev)):
        return torch.empty(max(nbytes, 256), dtype=torch.uint8, device=dev)


def _default_torch_stream(kw: dict) -> None:
    """A plan on torch memory runs on torch's current stream unless a stream is given."""
    if kw.get("stream") is None:
        import torch
        kw["stream"] = torch.cuda.current_stream(kw.get("device", 0)).cuda_stream


class Clocks:
    """cusan_clocks: a1's products for a whole trace (accesses, records, segment clock rows), as a
    flat image one rank computes and broadcasts so every rank plans its shard without the trace."""

    def __init__(self, h: C.c_void_p):
        self.h = h

    @classmethod
    def compute(cls, trace: Trace) -> "Clocks":
        h = C.c_void_p()
        _ck(lib.cusan_clocks_compute(trace.h, C.byref(h)))
        return cls(h)

    def to_bytes(self) -> np.ndarray:
        n = C.c_uint64()
        _ck(lib.cusan_clocks_bytes(self.h, C.byref(n)))
        buf = np.zeros(n.value, np.uint8)
        _ck(lib.cusan_clocks_export(self.h, _ptr(buf), n.value))
        return buf

    @classmethod
    def from_bytes(cls, buf: np.ndarray) -> "Clocks":
        buf = np.ascontiguousarray(buf, np.uint8)
        h = C.c_void_p()
        _ck(lib.cusan_clocks_import(_ptr(buf), len(buf), C.byref(h)))
        return cls(h)

    def __del__(self, _destroy=lib.cusan_clocks_destroy):
        if getattr(self, "h", None):
            _destroy(self.h)
            self.h = None


class Plan:
    """cusan_plan: host preparation (a1, a2) + device tables; run() does a3-a5 on the GPU.

    workspace="torch" takes the plan's device memory from PyTorch's caching allocator (a uint8
    tensor held by the plan) instead of the library's own cudaMalloc.  `trace` may be a Clocks
    object (cusan_plan_create_from_clocks)."""

    def __init__(self, trace, workspace: str | None = None, **kw):
        self.trace = trace            # must outlive the plan
        self.max_runs = kw.get("max_runs", 0)
        self.workspace = None
        if workspace == "torch":
            kw["flags"] = kw.get("flags", 0) | CUSAN_CHECK_DEFER_WORKSPACE
            _default_torch_stream(kw)
        self.device, self.stream = kw.get("device", 0), kw.get("stream")
        o = _opts(**kw)
        h = C.c_void_p()
        create = lib.cusan_plan_create_from_clocks if isinstance(trace, Clocks) else lib.cusan_plan_create
        _ck(create(trace.h, C.byref(o), C.byref(h)))
        self.h = h
        if workspace == "torch":
            nbytes = self.workspace_bytes()
            self.workspace = _torch_workspace(nbytes, self.device, self.stream)
            _ck(lib.cusan_plan_bind_workspace(self.h, C.c_void_p(self.workspace.data_ptr()), nbytes))

    def workspace_bytes(self) -> int:
        b = C.c_uint64()
        _ck(lib.cusan_plan_workspace_bytes(self.h, C.byref(b)))
        return b.value

    def cusan_plan_bind_workspace(self, workspace) -> None:
        """Bind device memory (a CUDA uint8 tensor of at least workspace_bytes(), held by the plan)
        to a plan created with CUSAN_CHECK_DEFER_WORKSPACE and upload its tables."""
        nbytes = self.workspace_bytes()
        if workspace.numel() * workspace.element_size() < nbytes:
            raise ValueError("workspace smaller than workspace_bytes()")
        self.workspace = workspace
        _ck(lib.cusan_plan_bind_workspace(self.h, C.c_void_p(workspace.data_ptr()), nbytes))

    def run(self) -> Report:
        h = C.c_void_p()
        _ck(lib.cusan_plan_run(self.h, C.byref(h)))
        return _report(h, self.max_runs)

    def cusan_plan_tables(self) -> tuple[np.ndarray, np.ndarray]:
        """The plan's device tables (diagnostics): incidence records and span-table records."""
        ni, ns = C.c_uint64(), C.c_uint64()
        _ck(lib.cusan_plan_tables(self.h, None, 0, None, 0, C.byref(ni), C.byref(ns)))
        inc, spans = np.zeros(ni.value, INC_DTYPE), np.zeros(ns.value, DSPAN_DTYPE)
        _ck(lib.cusan_plan_tables(self.h, _ptr(inc), ni.value, _ptr(spans), ns.value, C.byref(ni), C.byref(ns)))
        return inc, spans

    def close(self, _destroy=lib.cusan_plan_destroy):
        if getattr(self, "h", None):
            _destroy(self.h)
            self.h = None
        self.workspace = None

    __del__ = close


class Session:
    """cusan_session: incremental (online) checking with the shadow kept on the device between
    calls; check() checks the accesses appended to the trace since the previous call."""

    def __init__(self, trace: Trace, **kw):
        self.trace = trace            # must outlive the session; may only grow
        self.max_runs = kw.get("max_runs", 0)
        o = _opts(**kw)
        h = C.c_void_p()
        _ck(lib.cusan_session_create(trace.h, C.byref(o), C.byref(h)))
        self.h = h

    def check(self) -> Report:
        h = C.c_void_p()
        _ck(lib.cusan_session_check(self.h, C.byref(h)))
        return _report(h, self.max_runs)

    def submit(self) -> Report | None:
        """cusan_session_submit: plan the new events (overlapping the call in flight), collect the
        call in flight and launch this one; returns the previous call's report (None if none)."""
        h = C.c_void_p()
        _ck(lib.cusan_session_submit(self.h, C.byref(h)))
        return _report(h, self.max_runs) if h.value else None

    def finish(self) -> Report | None:
        """cusan_session_finish: wait for the call in flight and return its report (None if none)."""
        h = C.c_void_p()
        _ck(lib.cusan_session_finish(self.h, C.byref(h)))
        return _report(h, self.max_runs) if h.value else None

    def forget(self, addr: int, nbytes: int) -> None:
        """cusan_session_forget: no access appended from now on touches [addr, addr + nbytes) (the
        memory was released); the session drops that range's intervals after the next call."""
        _ck(lib.cusan_session_forget(self.h, addr, nbytes))

    def close(self, _destroy=lib.cusan_session_destroy):
        if getattr(self, "h", None):
            _destroy(self.h)
            self.h = None

    __del__ = close


def describe(trace: Trace, **kw) -> dict:
    """cusan_plan_describe: the host steps a1/a2 only (no GPU) — plan counters of a shard."""
    o = _opts(**kw)
    ctr = cusan_counters()
    _ck(lib.cusan_plan_describe(trace.h, C.byref(o), C.byref(ctr)))
    return {n: getattr(ctr, n) for n, _ in cusan_counters._fields_}


def check(trace: Trace, workspace: str | None = None, **kw) -> Report:
    """cusan_check: plan + run + destroy.  kw: nshards, shard, device, window_events,
    persist_shadow, max_runs, stream (a cudaStream_t as int, e.g. torch's current stream), flags,
    ngpus (a whole-node check: one shard per device, merged); workspace="torch" allocates the
    device memory through PyTorch."""
    if workspace is not None:
        p = Plan(trace, workspace=workspace, **kw)
        try:
            return p.run()
        finally:
            p.close()
    o = _opts(**kw)
    h = C.c_void_p()
    _ck(lib.cusan_check(trace.h, C.byref(o), C.byref(h)))
    return _report(h, kw.get("max_runs", 0))


def pipelined_checks(make_trace, steps: int, device: int = 0, host_workers: int = 2, lower_workers: int = 1,
                     **kw):
    """Check `steps` traces one after another with the host and the GPU overlapped, as a four-stage
    pipeline on separate threads: while the GPU checks trace i (a3-a5), host threads build the plans
    of the next traces (a2, on the device planner's own stream or on the host), compute their clocks
    (a1, cusan_clocks_compute) and build the traces after them (`make_trace(j)`, e.g. lowering the
    next batch of recorded calls, a0) — a step costs the slowest stage rather than their sum.  Each
    host stage has `host_workers` threads, so consecutive (independent) traces go through a stage at
    the same time; reports still come back in order, one GPU check after another.  This is how an
    online checker keeps host and GPU busy.  Every plan's tables are
    uploaded (host -> device) when it is bound, after the previous plan's run completed, and every
    run downloads its report, so each step still pays its own transfers.  All plans share one
    workspace from PyTorch's caching allocator (a plan's shadow and records are scratch for its own
    run).  Yields (trace, report) per step; kw as for Plan (window_events, nshards, shard, stream,
    flags, ...).  Steps take well under a millisecond, so a full pass of Python's cyclic garbage
    collector over a large process (tens of ms with torch imported) shows up as a stall of every
    stage; a caller that wants flat latency can `gc.freeze()` its long-lived objects first (bench.py
    does)."""
    from concurrent.futures import ThreadPoolExecutor

    kw = dict(kw)
    kw["flags"] = kw.get("flags", 0) | CUSAN_CHECK_DEFER_WORKSPACE
    kw["device"] = device
    _default_torch_stream(kw)
    kw.pop("device")
    hw, lw = max(1, int(host_workers)), max(1, int(lower_workers))
    depth = 3 * max(hw, lw)                     # steps in flight ahead of the GPU

    ws = None
    with ThreadPoolExecutor(lw) as lower_ex, ThreadPoolExecutor(hw) as clock_ex, ThreadPoolExecutor(hw) as plan_ex:
        futures = {}

        def schedule(j):
            lf = lower_ex.submit(make_trace, j)

            def clocks(f=lf):
                tr = f.result()
                return tr, Clocks.compute(tr)

            cf = clock_ex.submit(clocks)

            def plan(f=cf):
                tr, ck = f.result()
                return tr, Plan(ck, device=device, **kw)

            futures[j] = plan_ex.submit(plan)

        for j in range(min(depth + 1, steps)):
            schedule(j)
        for i in range(steps):
            tr, p = futures.pop(i).result()
            if i + depth + 1 < steps:
                schedule(i + depth + 1)
            need = max(p.workspace_bytes(), 256)
            if ws is None or ws.numel() < need:
                ws = None
                ws = _torch_workspace(need, device, kw["stream"])
            try:
                p.cusan_plan_bind_workspace(ws)
                rep = p.run()
            finally:
                p.close()
            yield tr, rep


def release_cached_memory() -> None:
    """cusan_release_cached_memory: free the library's parked check workspaces (all devices)."""
    _ck(lib.cusan_release_cached_memory())


def report_merge(runs: np.ndarray, n_race_granules: int, max_runs: int = 0) -> Report:
    """cusan_report_merge: canonical report from runs gathered from several shards."""
    runs = np.ascontiguousarray(runs, RUN_DTYPE)
    h = C.c_void_p()
    _ck(lib.cusan_report_merge(_ptr(runs), len(runs), n_race_granules, max_runs, C.byref(h)))
    return _report(h, max_runs)
