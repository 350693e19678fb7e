"""ctypes loader and prototypes for libcusan.so (include/cusan.h, include/cusan_lower.h).

Argument marshalling only.  There is no fallback: if the shared library is missing or cannot be
loaded, import fails loudly with the reason.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("CUSAN_LIBRARY", os.path.join(HERE, "libcusan.so"))


class CusanError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"cusan error {status}: {msg}")
        self.status = status


class cusan_event(C.Structure):
    _fields_ = [("kind", C.c_uint8), ("mode", C.c_uint8), ("pad", C.c_uint16), ("fiber", C.c_uint32),
                ("a", C.c_uint64), ("b", C.c_uint64)]


class cusan_race_run(C.Structure):
    _fields_ = [("g_begin", C.c_uint64), ("g_end", C.c_uint64), ("earlier", C.c_uint32),
                ("later", C.c_uint32)]


class cusan_check_opts(C.Structure):
    _fields_ = [("nshards", C.c_int), ("shard", C.c_int), ("device", C.c_int),
                ("window_events", C.c_int), ("persist_shadow", C.c_int), ("flags", C.c_int),
                ("max_runs", C.c_uint64),
                ("stream", C.c_void_p), ("workspace", C.c_void_p), ("workspace_bytes", C.c_uint64),
                ("shard_block", C.c_uint64), ("ngpus", C.c_int)]


_COUNTER_U64 = ["n_events", "n_access", "n_read", "n_write", "n_release", "n_release_store",
                "n_acquire", "n_fork", "tracked_bytes", "tracked_bytes_shard", "bytes_read",
                "bytes_written", "n_fibers", "n_segments", "n_intervals", "n_incidences", "n_windows",
                "n_spans", "shard_granules", "spill_heap_bytes", "spill_spans", "shadow_bytes",
                "workspace_bytes", "raw_runs"]


class cusan_counters(C.Structure):
    _fields_ = ([(n, C.c_uint64) for n in _COUNTER_U64] +
                [("kernel_ms", C.c_double), ("run_ms", C.c_double), ("kernel_launches", C.c_uint64),
                 ("shadow_cell_bytes", C.c_uint64), ("h2d_bytes", C.c_uint64),
                 ("d2h_bytes", C.c_uint64), ("heap_live_bytes", C.c_uint64), ("heap_bytes", C.c_uint64),
                 ("renumberings", C.c_uint64)])


class cusan_api_call(C.Structure):
    _fields_ = [("op", C.c_uint32), ("x", C.c_uint32), ("a", C.c_uint64), ("b", C.c_uint64),
                ("c", C.c_uint64), ("s", C.c_uint64)]


class cusan_api_arg(C.Structure):
    _fields_ = [("ptr", C.c_uint64), ("mode", C.c_uint32), ("pad", C.c_uint32)]


assert C.sizeof(cusan_event) == 24 and C.sizeof(cusan_race_run) == 24
assert C.sizeof(cusan_api_call) == 40 and C.sizeof(cusan_api_arg) == 16

P = C.c_void_p
PP = C.POINTER(C.c_void_p)
u32, u64, i32 = C.c_uint32, C.c_uint64, C.c_int
pu32, pu64, pi32 = C.POINTER(C.c_uint32), C.POINTER(C.c_uint64), C.POINTER(C.c_int)

# name -> argtypes (restype int unless noted)
PROTOS = {
    "cusan_trace_create": [u32, u64, PP],
    "cusan_trace_destroy": [P],
    "cusan_trace_append_access": [P, u32, i32, u64, u64, pu32],
    "cusan_trace_append_sync": [P, i32, u32, u64, pu32],
    "cusan_trace_append_events": [P, P, u64],
    "cusan_trace_size": [P, pu64, pu32],
    "cusan_trace_read": [P, u64, u64, P],
    "cusan_check_opts_init": [C.POINTER(cusan_check_opts)],
    "cusan_check": [P, C.POINTER(cusan_check_opts), PP],
    "cusan_plan_create": [P, C.POINTER(cusan_check_opts), PP],
    "cusan_plan_workspace_bytes": [P, pu64],
    "cusan_plan_bind_workspace": [P, P, u64],
    "cusan_plan_run": [P, PP],
    "cusan_plan_destroy": [P],
    "cusan_release_cached_memory": [],
    "cusan_device_count": [pi32],
    "cusan_plan_tables": [P, P, u64, P, u64, pu64, pu64],
    "cusan_clocks_compute": [P, PP],
    "cusan_clocks_bytes": [P, pu64],
    "cusan_clocks_export": [P, P, u64],
    "cusan_clocks_import": [P, u64, PP],
    "cusan_clocks_destroy": [P],
    "cusan_plan_create_from_clocks": [P, C.POINTER(cusan_check_opts), PP],
    "cusan_plan_describe": [P, C.POINTER(cusan_check_opts), C.POINTER(cusan_counters)],
    "cusan_session_create": [P, C.POINTER(cusan_check_opts), PP],
    "cusan_session_check": [P, PP],
    "cusan_session_submit": [P, PP],
    "cusan_session_finish": [P, PP],
    "cusan_session_forget": [P, u64, u64],
    "cusan_session_destroy": [P],
    "cusan_report_get": [P, pu64, pu64, C.POINTER(C.POINTER(cusan_race_run)), pi32],
    "cusan_report_counters": [P, C.POINTER(cusan_counters)],
    "cusan_report_merge": [P, u64, u64, u64, PP],
    "cusan_report_free": [P],
    "cusan_last_error": [],
    "cusan_version": [],
    "cusan_lowering_create": [P, PP],
    "cusan_lowering_destroy": [P],
    "cusan_lowering_fibers": [P, pu32],
    "cusan_on_malloc": [P, u64, u64, i32],
    "cusan_on_free": [P, u64],
    "cusan_on_stream_create": [P, u64, i32],
    "cusan_on_kernel": [P, u64, u32, pu64, pu32],
    "cusan_on_stream_sync": [P, u64],
    "cusan_on_device_sync": [P],
    "cusan_on_event_record": [P, u64, u64],
    "cusan_on_event_sync": [P, u64],
    "cusan_on_stream_wait_event": [P, u64, u64],
    "cusan_on_stream_query": [P, u64, i32],
    "cusan_on_memcpy": [P, u64, u64, u64, i32, i32, u64],
    "cusan_on_memset": [P, u64, u64, i32, u64],
    "cusan_on_host_access": [P, u64, u64, i32],
    "cusan_on_mpi_isend": [P, u64, u64, u64],
    "cusan_on_mpi_irecv": [P, u64, u64, u64],
    "cusan_on_mpi_wait": [P, u64],
    "cusan_on_mpi_test": [P, u64, i32],
    "cusan_on_mpi_send": [P, u64, u64],
    "cusan_on_mpi_recv": [P, u64, u64],
    "cusan_on_thread": [P, u64],
    "cusan_on_thread_create": [P, u64],
    "cusan_on_thread_join": [P, u64],
    "cusan_lowering_set_default_stream": [P, i32],
    "cusan_lowering_fiber_info": [P, u32, pi32, pu64],
    "cusan_lower_program": [P, P, u64, P, u64, pu32],
}
VOID = {"cusan_check_opts_init"}
STRING = {"cusan_last_error", "cusan_version"}


def load(path: str = LIB_PATH) -> C.CDLL:
    if not os.path.exists(path):
        raise ImportError(f"libcusan.so not built at {path}: run __graft_entry__.build() "
                          f"(there is no CPU fallback)")
    lib = C.CDLL(path)
    for name, argt in PROTOS.items():
        fn = getattr(lib, name)   # AttributeError = a declared symbol is missing
        fn.argtypes = argt
        fn.restype = None if name in VOID else (C.c_char_p if name in STRING else C.c_int)
    return lib


lib = load()


def check(status: int):
    if status != 0:
        raise CusanError(status, lib.cusan_last_error().decode())
