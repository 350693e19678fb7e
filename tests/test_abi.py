"""C-ABI boundary checks that need no GPU: the library loads, exports every declared symbol,
validates its arguments, and its lowering reproduces the oracle's primitive traces."""
from __future__ import annotations

import ctypes as C
import os
import re

import numpy as np
import pytest

import paper_conf_sc_huckzsjb24_b200 as cs
from paper_conf_sc_huckzsjb24_b200 import _lib
from oracle.lower import Lowering as OracleLowering, lower as oracle_lower
from tracegen import configs, fuzz
from tracegen.program import EVENT_DTYPE, OP_DTYPE

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in ("cusan.h", "cusan_lower.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        names |= set(re.findall(r"^\s*(?:const\s+)?(?:int|void|char\s*\*|const char\s*\*)\s*\*?\s*(cusan_\w+)\s*\(",
                                src, re.M))
    return names


def test_every_declared_symbol_is_exported():
    names = declared_functions()
    assert len(names) >= 40
    lib = C.CDLL(_lib.LIB_PATH)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing
    assert set(names) <= set(_lib.PROTOS)


def test_library_is_sm100a_native():
    """The shadow-check kernel is compiled for sm_100a (no PTX JIT, no other arch)."""
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "shadow_check_window" in sass


def test_argument_validation():
    t = cs.Trace(4)
    with pytest.raises(cs.CusanError) as e:
        t.cusan_trace_append_access(4, 0, 0, 8)          # fiber >= max_fibers
    assert e.value.status == -1
    with pytest.raises(cs.CusanError):
        t.cusan_trace_append_access(0, 2, 0, 8)          # bad mode
    with pytest.raises(cs.CusanError) as e:
        t.cusan_trace_append_access(0, 0, 2**64 - 4, 8)  # overflow
    assert e.value.status == -2
    with pytest.raises(cs.CusanError):
        t.cusan_trace_append_sync(9, 0, 0)              # bad sync kind
    with pytest.raises(cs.CusanError):
        t.cusan_trace_append_sync(cs.CUSAN_FORK, 0, 7)   # fork source out of range
    with pytest.raises(cs.CusanError):
        cs.Trace(0)
    with pytest.raises(cs.CusanError):
        cs.Trace(256)                                    # fiber 0xFF is the spill tag
    assert len(t) == 0                                   # failed appends leave no trace
    bad = np.zeros(2, EVENT_DTYPE)
    bad[1]["kind"] = 7
    with pytest.raises(cs.CusanError):
        t.cusan_trace_append_events(bad)
    assert len(t) == 0                                   # bulk append is all-or-nothing
    # session shard arguments are validated before any device work
    for kw in (dict(nshards=2, shard=2), dict(nshards=0), dict(nshards=2, shard=1, shard_block=48)):
        with pytest.raises(cs.CusanError) as e:
            cs.Session(t, **kw)
        assert e.value.status == -1


def test_check_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    t = cs.Trace(4)
    t.cusan_trace_append_access(0, 1, 0x1000, 64)
    with pytest.raises(cs.CusanError) as e:
        cs.check(t)
    assert e.value.status == -4


def test_fiber_info_and_text_report():
    """Fibers are named by what they stand for; the text report names the racing calls."""
    from paper_conf_sc_huckzsjb24_b200.report import format_report
    import oracle
    w = configs.make(1)
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    low = cs.Lowering(tr)
    first = low.cusan_lower_program(ops, args)
    assert low.cusan_lowering_fiber_info(0) == (0, 0)        # host thread 0
    assert low.cusan_lowering_fiber_info(1) == (1, 0)        # legacy default stream
    assert low.cusan_lowering_fiber_info(2)[0] == 2           # the user stream
    assert low.cusan_lowering_fiber_info(3) == (4, 1)        # MPI request 1
    with pytest.raises(cs.CusanError):
        low.cusan_lowering_fiber_info(9)
    ref = oracle.check_events(tr.cusan_trace_read(), 255)

    class Rep:
        n_race_granules, n_runs, truncated, runs = ref["n_race_granules"], ref["n_runs"], False, ref["runs"]
    text = format_report(Rep, tr, lowering=low, calls=ops, first_event=first)
    assert "4096 bytes" in text and "MPI_Isend" in text and "kernel launch" in text


def test_event_index_limit():
    """One-shot checks number events in the 24-bit epoch field: a trace of 2^24 - 2
    events plans, one more event is CUSAN_ERANGE for the one-shot planner (and the clocks) — the
    trace itself grows on (u32 event ids; sessions renumber, tests/test_gpu_session.py)."""
    n = (1 << 24) - 2
    ev = np.zeros(n, EVENT_DTYPE)
    ev["kind"] = 1                                       # RELEASE on key 0 by fiber 0
    t = cs.Trace(2)
    t.cusan_trace_append_events(ev)
    assert len(t) == n
    d = cs.describe(t)                                   # the planner takes the longest trace
    assert d["n_events"] == n and d["n_release"] == n
    t.cusan_trace_append_sync(cs.CUSAN_RELEASE, 0, 1)
    assert len(t) == n + 1
    with pytest.raises(cs.CusanError) as e:
        cs.describe(t)
    assert e.value.status == -2
    with pytest.raises(cs.CusanError) as e:
        cs.Clocks.compute(t)
    assert e.value.status == -2
    del ev, t


def test_trace_roundtrip_and_event_ids():
    t = cs.Trace(8)
    assert t.cusan_trace_append_access(1, 1, 0x100, 24) == 0
    assert t.cusan_trace_append_sync(cs.CUSAN_RELEASE, 1, 77) == 1
    assert t.cusan_trace_append_sync(cs.CUSAN_FORK, 2, 0) == 2
    ev = t.cusan_trace_read()
    assert list(ev["kind"]) == [0, 1, 4] and int(ev[2]["a"]) == 0 and int(ev[2]["fiber"]) == 2


def _product_lower(ops, args, max_fibers=255):
    tr = cs.Trace(max_fibers)
    low = cs.Lowering(tr)
    first = low.cusan_lower_program(ops, args)
    return tr.cusan_trace_read(), low.cusan_lowering_fibers(), first


def _oracle_lower_first(ops, args):
    L = OracleLowering()
    first = []
    for op in np.asarray(ops, OP_DTYPE):
        first.append(len(L.ev))
        L.call(op, args)
    return L.events(), L.next_fiber, first


@pytest.mark.parametrize("c", [1, 2, 3, 4, 5])
def test_lowering_matches_oracle_lowering_configs(c):
    w = configs.make(c, "small")
    for racy in (False, True):
        ops, args = w.arrays(racy)
        ev_p, nf_p, first_p = _product_lower(ops, args)
        ev_o, nf_o, first_o = _oracle_lower_first(ops, args)
        assert nf_p == nf_o
        assert np.array_equal(ev_p, ev_o)
        assert list(first_p) == first_o


def test_failed_stream_query_uses_no_fiber():
    """An unsuccessful cudaStreamQuery appends nothing (A9) and must not open the lazily created
    per-thread default stream fiber either: the next fiber (an MPI request's) gets the same id in
    the product and the oracle lowering (found by tools/fuzz_campaign.py)."""
    from tracegen.program import Program, STREAM_PER_THREAD
    for per_thread in (False, True):
        p = Program()
        p.default_stream_mode(per_thread)
        a = p.malloc(512)
        s = p.stream_create()
        p.kernel(s, [(a, 1)])
        p.stream_query(STREAM_PER_THREAD, False)
        p.stream_query(0, False)
        r = p.isend(a, 256)
        p.wait(r)
        ops, args = p.arrays()
        ev_p, nf_p, first_p = _product_lower(ops, args)
        ev_o, nf_o, first_o = _oracle_lower_first(ops, args)
        assert nf_p == nf_o and np.array_equal(ev_p, ev_o) and list(first_p) == first_o
    t = cs.Trace(8)
    with pytest.raises(cs.CusanError):
        cs.Lowering(t).cusan_on_stream_query(12345, 0)    # unknown handle, even when unsuccessful


def test_lowering_matches_oracle_lowering_fuzz_and_listings():
    import listing_dsl
    progs = [l.program for l in listing_dsl.parse()]
    rng = np.random.default_rng(3)
    progs += [fuzz.random_program(rng, int(rng.integers(1, 60))) for _ in range(200)]
    for p in progs:
        ops, args = p.arrays()
        ev_p, nf_p, first_p = _product_lower(ops, args)
        ev_o, nf_o, first_o = _oracle_lower_first(ops, args)
        assert nf_p == nf_o and np.array_equal(ev_p, ev_o) and list(first_p) == first_o


def test_lowering_single_call_api():
    """cusan_on_* calls append the same primitives as the bulk program form."""
    tr = cs.Trace(16)
    low = cs.Lowering(tr)
    low.cusan_on_malloc(0x1000, 4096, 0)
    low.cusan_on_stream_create(5, 0)
    low.cusan_on_kernel(5, [0x1000], [1])
    low.cusan_on_mpi_isend(0x1000, 4096, 9)
    low.cusan_on_mpi_wait(9)
    ev = tr.cusan_trace_read()
    # FORK(H→s), ACQUIRE(s, K(S0)), ACCESS W, RELEASE(s), FORK(H→m), ACCESS R, RELEASE(m, K(r)), ACQUIRE(H)
    assert list(ev["kind"]) == [4, 3, 0, 1, 4, 0, 1, 3]
    assert list(ev["fiber"]) == [2, 2, 2, 2, 3, 3, 3, 0]
    with pytest.raises(cs.CusanError):
        low.cusan_on_kernel(77, [0x1000], [1])          # unknown stream
    with pytest.raises(cs.CusanError):
        low.cusan_on_memcpy(0, 0, 8, 9, 0, 0)             # bad copy kind


def test_concurrent_planning_threads():
    """Host planning from several threads at once (ctypes releases the GIL): the shared pool of
    planning threads serves one caller, the others run their own threads; results are identical."""
    import threading
    w = configs.make(3, "full")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    want = cs.describe(tr, window_events=512)
    out, errs = [], []

    def work():
        try:
            for _ in range(3):
                out.append(cs.describe(tr, window_events=512))
        except Exception as e:               # pragma: no cover - reported below
            errs.append(e)
    th = [threading.Thread(target=work) for _ in range(4)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=120)
    assert not errs and len(out) == 12
    assert all(d == want for d in out)


def test_planning_with_the_clock_thread():
    """From 4096 accesses on, a1 runs on its own thread next to a2; the plan is the same as the
    serial one would give (one interval and one segment row per disjoint write)."""
    n = 1 << 13
    ev = np.zeros(n, EVENT_DTYPE)
    ev["kind"] = 0
    ev["mode"] = 1
    ev["a"] = np.arange(n, dtype=np.uint64) * 64
    ev["b"] = 64
    t = cs.Trace(4)
    t.cusan_trace_append_events(ev)
    d = cs.describe(t, window_events=100)
    assert d["n_access"] == n and d["n_intervals"] == n and d["n_windows"] == (n + 99) // 100
    assert d["n_segments"] == 1 and d["n_incidences"] == n and d["tracked_bytes"] == 64 * n


def test_c_example_host_steps():
    """examples/fig6a.c drives the C ABI from C (lowering callbacks + cusan_plan_describe, no GPU)."""
    import subprocess
    import __graft_entry__ as g
    exe = [e for e in g.build_examples() if e.endswith("fig6a")][0]
    for extra in ([], ["--fixed"]):
        r = subprocess.run([exe, "--describe", *extra], capture_output=True, text=True, timeout=60)
        assert r.returncode == 0, (r.stdout, r.stderr)
        assert "accesses 2" in r.stdout and "tracked 8192 B" in r.stdout
