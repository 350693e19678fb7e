"""ORACLE — test infrastructure only.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` leg (and
``bench.py --impl reference``) may import, call, link or execute anything under ``oracle/``.
The product path (``paper_conf_sc_huckzsjb24_b200``) never touches it.

* ``oracle.lower``  — plain-Python lowering of CUDA / MPI calls to primitives (step a0).
* ``oracle.c``      — plain C race checker: naive vector clocks, per-granule race set, canonical runs
                      (steps a1-a5).  Built with gcc by ``build()``.

Parity status: every function here is pinned by ``tests/test_oracle_*.py`` against the paper's
racy / fixed listings, a brute-force graph-HB checker, invariants and closed forms (DESIGN.md
§"Oracle pins").
"""
from __future__ import annotations

import os
import subprocess
import tempfile

import numpy as np

from tracegen.program import EVENT_DTYPE, save_events

HERE = os.path.dirname(os.path.abspath(__file__))
BIN = os.path.join(HERE, "oracle_bin")
RUN_DTYPE = np.dtype([("g_begin", "<u8"), ("g_end", "<u8"), ("earlier", "<u4"), ("later", "<u4")])


def build(force: bool = False) -> str:
    src = os.path.join(HERE, "oracle.c")
    if force or not os.path.exists(BIN) or os.path.getmtime(BIN) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-pthread", "-o", BIN, src])
    return BIN


def read_report(path: str) -> dict:
    with open(path, "rb") as f:
        raw = f.read()
    assert raw[:4] == b"CSRP", "bad report"
    n_events, n_access, tracked, n_race, n_runs = np.frombuffer(raw, "<u8", 5, 12)
    runs = np.frombuffer(raw, RUN_DTYPE, int(n_runs), 52).copy()
    return dict(n_events=int(n_events), n_access=int(n_access), tracked_bytes=int(tracked),
                n_race_granules=int(n_race), n_runs=int(n_runs), runs=runs)


def check_events(events: np.ndarray, max_fibers: int = 0, threads: int | None = None,
                 sample: np.ndarray | None = None, granule_range: tuple[int, int] | None = None) -> dict:
    """Run the C oracle on a primitive trace; returns the canonical report (plus the wall time of
    the oracle process in ``seconds``)."""
    import time
    build()
    threads = threads or os.cpu_count() or 1
    with tempfile.TemporaryDirectory() as d:
        tp, rp = os.path.join(d, "t.bin"), os.path.join(d, "r.bin")
        save_events(tp, np.asarray(events, EVENT_DTYPE), max_fibers)
        cmd = [BIN, tp, rp, "--threads", str(threads)]
        if sample is not None:
            sp = os.path.join(d, "s.bin")
            np.ascontiguousarray(np.unique(np.asarray(sample, np.uint64))).tofile(sp)
            cmd += ["--sample", sp]
        if granule_range is not None:
            cmd += ["--range", str(int(granule_range[0])), str(int(granule_range[1]))]
        t0 = time.perf_counter()
        subprocess.check_call(cmd)
        secs = time.perf_counter() - t0
        rep = read_report(rp)
    rep["threads"] = threads
    rep["seconds"] = secs
    return rep


def check_program(ops, args, threads: int | None = None, sample=None) -> dict:
    """Lower an API program (oracle.lower) and check it (oracle.c)."""
    from .lower import lower
    ev, nf = lower(ops, args)
    rep = check_events(ev, nf, threads=threads, sample=sample)
    rep["events"] = ev
    return rep
