"""Human-readable race reports in the style of ThreadSanitizer / CuSan warnings.

    text = format_report(rep, trace, lowering=low, calls=ops, first_event=first)

`lowering` (a Lowering) names each fiber by what it stands for (host thread, CUDA stream, MPI
request); `calls` + `first_event` (the recorded API program and cusan_lower_program's per-call
first event ids) name the call an access came from.  Formatting only — the report is the library's.
"""
from __future__ import annotations

import bisect

import numpy as np

_FIBER_KIND = {0: "host thread", 1: "legacy default stream", 2: "stream", 3: "per-thread default stream",
               4: "MPI request"}
_OP_NAME = {1: "cudaMalloc", 2: "cudaFree", 3: "cudaStreamCreate", 4: "kernel launch", 5: "cudaStreamSynchronize",
            6: "cudaDeviceSynchronize", 7: "cudaEventRecord", 8: "cudaEventSynchronize", 9: "cudaStreamWaitEvent",
            10: "cudaStreamQuery", 11: "cudaMemcpy", 12: "cudaMemcpyAsync", 13: "cudaMemset", 14: "cudaMemsetAsync",
            15: "host access", 16: "MPI_Isend", 17: "MPI_Irecv", 18: "MPI_Wait", 19: "MPI_Send", 20: "MPI_Recv",
            21: "MPI_Test", 22: "thread switch", 23: "pthread_create", 24: "pthread_join", 25: "default-stream mode"}


def _who(fiber: int, lowering) -> str:
    if lowering is not None:
        try:
            kind, handle = lowering.cusan_lowering_fiber_info(fiber)
            name = _FIBER_KIND.get(kind, "fiber")
            if kind in (0, 3):
                return f"{name} of thread {handle} (fiber {fiber})"
            if kind == 2:
                return f"{name} {handle:#x} (fiber {fiber})"
            if kind == 4:
                return f"MPI request fiber (fiber {fiber}, latest request {handle})"
            return f"{name} (fiber {fiber})"
        except Exception:
            pass
    return f"fiber {fiber}"


def _call(eid: int, calls, first_event) -> str:
    if calls is None or first_event is None or len(first_event) == 0:
        return ""
    i = bisect.bisect_right(np.asarray(first_event).tolist(), eid) - 1
    if i < 0:
        return ""
    op = calls[i]
    name = _OP_NAME.get(int(op["op"]), f"op {int(op['op'])}")
    extra = ""
    if int(op["op"]) in (4, 7, 9, 12, 14):
        extra = f" on stream {int(op['s']):#x}"
    elif int(op["op"]) in (16, 17):
        extra = f" request {int(op['b'])}"
    return f", in call #{i} {name}{extra}"


def format_report(rep, trace, lowering=None, calls=None, first_event=None, max_runs: int = 20) -> str:
    ev = trace.cusan_trace_read()
    out = [f"cusan: {rep.n_race_granules} racing granules ({8 * rep.n_race_granules} bytes) "
           f"in {rep.n_runs} race runs" + (" (list truncated)" if rep.truncated else "")]
    for r in rep.runs[:max_runs]:
        gb, ge, e, l = int(r["g_begin"]), int(r["g_end"]), int(r["earlier"]), int(r["later"])
        le, ee = ev[l], ev[e]
        mode = lambda x: "write" if int(x["mode"]) else "read"  # noqa: E731
        out.append(f"WARNING: data race on [{8 * gb:#x}, {8 * ge:#x}) ({8 * (ge - gb)} bytes)")
        out.append(f"  {mode(le)} (event {l}) by {_who(int(le['fiber']), lowering)}{_call(l, calls, first_event)}")
        out.append(f"  previous {mode(ee)} (event {e}) by {_who(int(ee['fiber']), lowering)}"
                   f"{_call(e, calls, first_event)}")
    if rep.n_runs > max_runs:
        out.append(f"... {rep.n_runs - max_runs} more race runs")
    return "\n".join(out)
