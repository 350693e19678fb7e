"""GPU parity: the sm_100a path (through the C ABI) against the oracle, bit-exact.

Integer work, so the bar is equality of the canonical run list and of the race-granule count
(SURVEY.md §8(c) step 4).  Inputs come only from tracegen; expected values only from oracle/.
"""
from __future__ import annotations

import hashlib
import os

import numpy as np
import pytest

import oracle
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs, fuzz
from tracegen.program import EV_ACCESS

import brute
import listing_dsl

pytestmark = pytest.mark.gpu


def gpu_report(events, max_fibers=255, **kw):
    tr = cs.Trace(max_fibers)
    tr.cusan_trace_append_events(events)
    return cs.check(tr, **kw)


def assert_equal(rep, ref):
    assert rep.n_race_granules == ref["n_race_granules"]
    assert rep.n_runs == ref["n_runs"]
    assert np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))


def lower_product(ops, args):
    tr = cs.Trace(255)
    first = cs.Lowering(tr).cusan_lower_program(ops, args)
    return tr, first


# ---------------------------------------------------------------------------------------------
LISTINGS = listing_dsl.parse()


@pytest.mark.parametrize("lst", LISTINGS, ids=[l.name for l in LISTINGS])
def test_listing_on_gpu(lst):
    ops, args = lst.program.arrays()
    tr, first = lower_product(ops, args)
    ev = tr.cusan_trace_read()
    rep = cs.check(tr)
    got = listing_dsl.observed_pairs(rep.runs, listing_dsl.label_events(lst, ev, list(first)))
    assert set(got) == {(a, b) for a, b, _ in lst.expect}
    assert_equal(rep, oracle.check_events(ev, 256, threads=1))


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
@pytest.mark.parametrize("window", [0, 1, 2, 7])
def test_fuzz_primitive_traces(window, flags):
    """Random traces spanning several warp ranges with ragged tails; both shadow layouts (one cell
    per elementary interval, the default, and one cell per granule)."""
    rng = np.random.default_rng(40 + window)
    for i in range(60):
        nf = int(rng.integers(2, 9))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(1, 80)), nf, n_keys=3,
                                         n_granules=int(rng.integers(1, 1500)), unaligned=bool(i % 3 == 0))
        rep = gpu_report(ev, nf, window_events=window, flags=flags)
        assert_equal(rep, oracle.check_events(ev, nf, threads=2))


def test_spill_path_many_readers():
    """More than three reader fibers between writes exercises the exact spill slots."""
    rng = np.random.default_rng(77)
    hit_spill = 0
    for i in range(40):
        nf = int(rng.integers(5, 40))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(20, 200)), nf, n_keys=4,
                                         n_granules=int(rng.integers(50, 700)), p_access=0.8)
        # mostly reads: flip 75% of writes to reads
        acc = ev["kind"] == EV_ACCESS
        flip = acc & (rng.random(len(ev)) < 0.75)
        ev["mode"][flip] = 0
        ref = oracle.check_events(ev, nf, threads=2)
        for window in (0, 3):
            for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
                rep = gpu_report(ev, nf, window_events=window, flags=flags)
                assert_equal(rep, ref)
                hit_spill += rep.counters["spill_spans"] > 0
    assert hit_spill > 0


@pytest.mark.parametrize("nshards", [2, 3, 5])
@pytest.mark.parametrize("window,flags", [(0, cs.CUSAN_CHECK_DENSE_SHADOW), (3, cs.CUSAN_CHECK_DENSE_SHADOW), (3, 0)],
                         ids=["one-window-dense", "windowed-dense", "windowed-compressed"])
def test_shards_merge_to_the_whole(nshards, window, flags):
    """Shard boundaries come from the coverage (one window) or from the windows touching each
    interval (windowed); either way the shards' merged runs are the whole trace's."""
    rng = np.random.default_rng(5 + nshards)
    for _ in range(20):
        nf = int(rng.integers(2, 7))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(5, 80)), nf, n_keys=3,
                                         n_granules=int(rng.integers(100, 2000)))
        kw = dict(window_events=window, flags=flags)
        parts = [gpu_report(ev, nf, nshards=nshards, shard=s, **kw) for s in range(nshards)]
        runs = np.concatenate([p.runs for p in parts])
        merged = cs.report_merge(runs, sum(p.n_race_granules for p in parts))
        assert_equal(merged, oracle.check_events(ev, nf, threads=2))
        whole = gpu_report(ev, nf, **kw)
        assert sum(p.counters["shard_granules"] for p in parts) == whole.counters["shard_granules"]
        assert sum(p.counters["tracked_bytes_shard"] for p in parts) == parts[0].counters["tracked_bytes"]
        assert sum(p.counters["n_incidences"] for p in parts) >= whole.counters["n_incidences"]


@pytest.mark.parametrize("c", [3, 5])
def test_small_configs_sharded_windowed(c):
    w = configs.make(c, "small")
    ops, args = w.arrays(True)
    tr, _ = lower_product(ops, args)
    ref = oracle.check_events(tr.cusan_trace_read(), 256)
    for nshards in (2, 8):
        parts = [cs.check(tr, window_events=97, nshards=nshards, shard=s) for s in range(nshards)]
        merged = cs.report_merge(np.concatenate([p.runs for p in parts]), sum(p.n_race_granules for p in parts))
        assert_equal(merged, ref)


@pytest.mark.parametrize("c", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("racy", [False, True])
def test_small_configs(c, racy):
    w = configs.make(c, "small")
    ops, args = w.arrays(racy)
    tr, _ = lower_product(ops, args)
    ev = tr.cusan_trace_read()
    ref = oracle.check_events(ev, 256)
    for window in (0, 97):
        for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
            assert_equal(cs.check(tr, window_events=window, flags=flags), ref)
    assert (ref["n_race_granules"] > 0) == racy


def test_edge_cases():
    # empty trace, trace without accesses, zero-length access
    assert cs.check(cs.Trace(4)).n_race_granules == 0
    t = cs.Trace(4)
    t.cusan_trace_append_sync(cs.CUSAN_RELEASE, 0, 5)
    assert cs.check(t).n_runs == 0
    t = cs.Trace(4)
    t.cusan_trace_append_access(0, 1, 0x1000, 0)
    t.cusan_trace_append_access(1, 1, 0x1000, 0)
    assert cs.check(t).n_race_granules == 0
    # 255 fibers (the maximum), all reading one granule, then one write: 254 races, exact spill
    t = cs.Trace(255)
    for f in range(255):
        t.cusan_trace_append_access(f, 0, 0x2000, 8)
    t.cusan_trace_append_access(0, 1, 0x2000, 8)
    ref = oracle.check_events(t.cusan_trace_read(), 255)
    for window in (0, 1, 100):
        for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
            rep = cs.check(t, window_events=window, flags=flags)
            assert rep.n_race_granules == 254
            assert_equal(rep, ref)
    # truncation keeps counts exact
    rep = cs.check(t, max_runs=10)
    assert rep.truncated and len(rep.runs) == 10 and rep.n_runs == 254 and rep.n_race_granules == 254


def test_repeated_runs_of_a_plan_are_identical():
    w = configs.make(3, "small")
    ops, args = w.arrays(True)
    tr, _ = lower_product(ops, args)
    plan = cs.Plan(tr, window_events=50)
    a, b = plan.run(), plan.run()
    assert np.array_equal(a.runs, b.runs) and a.n_race_granules == b.n_race_granules
    plan.close()


def _sample_granules(rep_runs, ev, rng, n_random=1500):
    acc = ev[ev["kind"] == EV_ACCESS]
    g0 = (acc["a"] >> np.uint64(3)).astype(np.uint64)
    g1 = ((acc["a"] + acc["b"] + np.uint64(7)) >> np.uint64(3)).astype(np.uint64)
    pick = rng.integers(0, len(acc), n_random)
    inner = g0[pick] + (rng.random(n_random) * (g1[pick] - g0[pick]).astype(np.float64)).astype(np.uint64)
    s = [inner, g0[pick], g1[pick] - np.uint64(1)]
    if len(rep_runs):
        k = rng.integers(0, len(rep_runs), min(300, len(rep_runs)))
        s += [rep_runs["g_begin"][k], rep_runs["g_end"][k] - np.uint64(1), rep_runs["g_end"][k]]
    return np.unique(np.concatenate(s).astype(np.uint64))


@pytest.mark.parametrize("c", [2, 3, 4, 5])
def test_full_size_configs_sampled(c):
    """BASELINE.json sizes, bench launch configuration; oracle on sampled granules (run edges,
    access edges and random interior granules)."""
    w = configs.make(c, "full")
    ops, args = w.arrays(True)
    tr, _ = lower_product(ops, args)
    ev = tr.cusan_trace_read()
    import torch
    s = torch.cuda.Stream()
    rep = cs.check(tr, window_events=4096, workspace="torch", stream=s.cuda_stream,
                   flags=cs.CUSAN_CHECK_DENSE_SHADOW)                                # as bench.py runs it
    one = cs.check(tr)                                                 # compressed, post-mortem: one window
    assert one.n_race_granules == rep.n_race_granules and np.array_equal(one.runs, rep.runs)
    assert rep.n_race_granules > 0
    assert rep.n_race_granules == int(np.sum(rep.runs["g_end"] - rep.runs["g_begin"]))
    sample = _sample_granules(rep.runs, ev, np.random.default_rng(c))
    ref = oracle.check_events(ev, 256, sample=sample)
    sset = set(int(x) for x in sample)
    got = {t for t in brute.runs_to_triples_in(rep.runs, sset)}
    want = brute.runs_to_triples(ref["runs"])
    assert got == want


FULL_GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "full")


@pytest.mark.parametrize("twin", ["racy", "clean"])
@pytest.mark.parametrize("c", [1, 2, 3, 4, 5])
def test_full_size_configs_exact(c, twin):
    """Every BASELINE config at its full size, whole trace, bit-exact against the oracle's complete
    report (every granule checked by oracle.c; written by tools/oracle_full_reports.py, which calls
    only oracle/ and tracegen/).  The GPU runs in the bench launch configuration (4096-access
    windows, torch workspace, a side stream) and, for the two largest traces, also as 8 granule-range
    shards merged (result invariance under the GPU count)."""
    g = np.load(os.path.join(FULL_GOLDEN, f"config{c}_{twin}.npz"))
    w = configs.make(c, "full")
    ops, args = w.arrays(twin == "racy")
    tr, _ = lower_product(ops, args)
    ev = tr.cusan_trace_read()
    # the product lowering produced exactly the trace the oracle checked (oracle.lower)
    assert hashlib.sha256(np.ascontiguousarray(ev).tobytes()).hexdigest() == str(g["events_sha256"])
    ref = dict(n_race_granules=int(g["n_race_granules"]), n_runs=int(g["n_runs"]), runs=g["runs"])
    assert (ref["n_race_granules"] > 0) == (twin == "racy")
    import torch
    s = torch.cuda.Stream()
    for flags in (cs.CUSAN_CHECK_DENSE_SHADOW, 0,       # both bench lines: dense, compressed
                  cs.CUSAN_CHECK_DEVICE_PLAN | cs.CUSAN_CHECK_DENSE_SHADOW, cs.CUSAN_CHECK_HOST_PLAN):
        rep = cs.check(tr, window_events=4096, workspace="torch", stream=s.cuda_stream, flags=flags)
        assert rep.counters["tracked_bytes"] == int(g["tracked_bytes"])
        assert_equal(rep, ref)
    if c in (4, 5):
        for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
            parts = [cs.check(tr, window_events=4096, nshards=8, shard=k, flags=flags) for k in range(8)]
            merged = cs.report_merge(np.concatenate([p.runs for p in parts]), sum(p.n_race_granules for p in parts))
            assert_equal(merged, ref)


def test_torch_workspace_and_stream():
    """Device memory from PyTorch's caching allocator, work on torch's current stream."""
    import torch
    w = configs.make(5, "small")
    ops, args = w.arrays(True)
    tr, _ = lower_product(ops, args)
    ref = oracle.check_events(tr.cusan_trace_read(), 255)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for window in (0, 50):
            rep = cs.check(tr, workspace="torch", window_events=window, stream=s.cuda_stream)
            assert_equal(rep, ref)
    plan = cs.Plan(tr, workspace="torch", window_events=50)
    assert plan.workspace is not None and plan.workspace.numel() >= plan.workspace_bytes()
    assert_equal(plan.run(), ref)
    plan.close()


@pytest.mark.parametrize("window", [0, 1, 5])
def test_interval_compressed_shadow_matches(window):
    """f3: one shadow cell per elementary interval gives exactly the per-granule result."""
    rng = np.random.default_rng(900 + window)
    for i in range(40):
        nf = int(rng.integers(2, 12))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(1, 90)), nf, n_keys=3,
                                         n_granules=int(rng.integers(1, 1500)), unaligned=bool(i % 2),
                                         p_access=0.7)
        rep = gpu_report(ev, nf, window_events=window, flags=cs.CUSAN_CHECK_INTERVAL_SHADOW)
        assert_equal(rep, oracle.check_events(ev, nf, threads=2))
        assert rep.counters["shadow_bytes"] <= 8 * rep.counters["n_intervals"] or window == 0
    for c in (2, 3, 4, 5):
        w = configs.make(c, "small")
        ops, args = w.arrays(True)
        tr, _ = lower_product(ops, args)
        ref = oracle.check_events(tr.cusan_trace_read(), 255)
        assert_equal(cs.check(tr, window_events=max(window, 1) * 40, flags=cs.CUSAN_CHECK_INTERVAL_SHADOW), ref)


def _events(rows):
    from tracegen.program import EVENT_DTYPE
    ev = np.zeros(len(rows), EVENT_DTYPE)
    for i, (k, m, f, a, b) in enumerate(rows):
        ev[i]["kind"], ev[i]["mode"], ev[i]["fiber"], ev[i]["a"], ev[i]["b"] = k, m, f, a, b
    return ev


def test_run_buffer_overflow_reruns_exactly():
    """More raw runs than the first run buffer holds (65536 here): the plan grows it and re-runs;
    the report is exact.  Closed form: 200 unsynchronised whole-range writes on 200 fibers race pairwise with
    their predecessor only (each write resets the state), 199 runs of the whole range."""
    n_gran, n_fib, base = 1 << 21, 200, 1 << 36
    ev = _events([(EV_ACCESS, 1, f, base, 8 * n_gran) for f in range(n_fib)])
    tr = cs.Trace(255)
    tr.cusan_trace_append_events(ev)
    p = cs.Plan(tr, window_events=50, flags=cs.CUSAN_CHECK_DENSE_SHADOW)   # 4 windows, 512 ranges each,
    #                                                                      50 racing pairs per range
    rep = p.run()
    assert rep.counters["raw_runs"] > (1 << 16)                 # beyond the initial buffer
    assert rep.n_race_granules == (n_fib - 1) * n_gran
    assert rep.n_runs == n_fib - 1
    want = [(base >> 3, (base >> 3) + n_gran, e, e + 1) for e in range(n_fib - 1)]
    assert [tuple(int(x) for x in r) for r in rep.runs] == want
    rep2 = p.run()                                              # the grown buffer is kept
    assert np.array_equal(rep2.runs, rep.runs)
    p.close()


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
def test_interval_longer_than_2_31_granules(flags):
    """An elementary interval of more than 2^31 granules (17 GB of address): a compressed span is
    one range owning its single cell, a dense span is cut into ranges at the right offsets.
    Closed form: W f0, W f1, R f2 over the whole range, unsynchronised, each access in its own
    window: runs (0 -> 1) and (1 -> 2) over all N granules.  The oracle checks sampled granules at
    the 2^31 boundary and both ends."""
    n_gran, base = (1 << 31) + 4096 + 40, 1 << 40
    g0 = base >> 3
    rows = [(EV_ACCESS, 1, 0, base, 8 * n_gran), (EV_ACCESS, 1, 1, base, 8 * n_gran),
            (EV_ACCESS, 0, 2, base, 8 * n_gran)]
    ev = _events(rows)
    want = [(g0, g0 + n_gran, 0, 1), (g0, g0 + n_gran, 1, 2)]
    sample = np.array([g0, g0 + 1, g0 + (1 << 31) - 1, g0 + (1 << 31), g0 + n_gran - 1], np.uint64)
    ref = oracle.check_events(ev, 3, sample=sample)
    assert brute.runs_to_triples(ref["runs"]) == {(int(g), e, l) for g in sample for _, _, e, l in want}
    tr = cs.Trace(3)
    tr.cusan_trace_append_events(ev)
    rep = cs.check(tr, window_events=1, flags=flags)
    assert [tuple(int(x) for x in r) for r in rep.runs] == want
    assert rep.n_race_granules == 2 * n_gran
    if flags == 0:
        assert rep.counters["shadow_bytes"] <= 64
        ses = cs.Session(cs.Trace(3), window_events=1)        # the in-place session path
        got = []
        for k in range(3):
            ses.trace.cusan_trace_append_events(ev[k:k + 1])
            got += [tuple(int(x) for x in r) for r in ses.check().runs]
        assert got == want
        ses.close()


def test_largest_event_id_on_the_gpu():
    """Maximum trace length: the last event id 2^24 - 3 packs as epoch 2^24 - 2 in the
    24-bit field; it must race with event 0.  Closed form: one run of the range, (0, last)."""
    from tracegen.program import EV_RELEASE
    n = (1 << 24) - 2
    base, n_gran = 1 << 33, 4096
    ev = np.zeros(n, dtype=_events([]).dtype)
    ev["kind"] = EV_RELEASE                                   # fiber 0 releases key 0, n-2 times
    ev[0]["kind"], ev[0]["mode"], ev[0]["a"], ev[0]["b"] = EV_ACCESS, 1, base, 8 * n_gran
    ev[n - 1]["kind"], ev[n - 1]["mode"], ev[n - 1]["fiber"] = EV_ACCESS, 1, 1
    ev[n - 1]["a"], ev[n - 1]["b"] = base, 8 * n_gran
    tr = cs.Trace(2)
    tr.cusan_trace_append_events(ev)
    for kw in ({}, {"flags": cs.CUSAN_CHECK_DENSE_SHADOW}, {"flags": cs.CUSAN_CHECK_INTERVAL_SHADOW}):
        rep = cs.check(tr, **kw)
        assert [tuple(int(x) for x in r) for r in rep.runs] == [(base >> 3, (base >> 3) + n_gran, 0, n - 1)]


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
def test_maximum_fibers_read_set(flags):
    """255 fibers (the most an epoch encodes) read a range, then fiber 0 writes it: the full read
    set (254 other readers) lives in a record and every unordered reader races."""
    base, n_gran = 1 << 34, 1000
    rows = [(EV_ACCESS, 0, f, base + 8 * (f % 3), 8 * n_gran) for f in range(255)]
    rows.append((EV_ACCESS, 1, 0, base, 8 * (n_gran + 2)))
    ev = _events(rows)
    ref = oracle.check_events(ev, 255)
    assert ref["n_runs"] >= 254
    for window in (0, 7):
        assert_equal(gpu_report(ev, 255, window_events=window, flags=flags), ref)


def test_pipelined_checks_match_the_oracle_per_step():
    """pipelined_checks: plans prepared on a host thread while the previous one runs, one shared
    workspace — every step's report is that trace's oracle report (different sizes and windows per
    step, so the shared workspace is re-carved and grown)."""
    rng = np.random.default_rng(77)
    traces = []
    for i in range(6):
        nf = int(rng.integers(2, 8))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(5, 120)), nf, n_keys=3,
                                         n_granules=int(rng.integers(50, 5000) * (i + 1)))
        traces.append((ev, nf))

    def make(i):
        tr = cs.Trace(traces[i][1])
        tr.cusan_trace_append_events(traces[i][0])
        return tr

    for workers in (1, 2, 4):                  # host stages with several threads: reports still in order
        n = 0
        for i, (tr, rep) in enumerate(cs.pipelined_checks(make, len(traces), window_events=3,
                                                          host_workers=workers, lower_workers=workers)):
            assert_equal(rep, oracle.check_events(traces[i][0], traces[i][1], threads=2))
            n += 1
        assert n == len(traces)


def test_c_example_fig6a():
    """The paper's Fig. 6A through the C ABI from a C program (examples/fig6a.c): racy = one run
    over the 4 KiB buffer, (Isend read, kernel write); fixed (MPI_Wait first) = none."""
    import subprocess
    import __graft_entry__ as g
    exe = [e for e in g.build_examples() if e.endswith("fig6a")][0]
    racy = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert racy.returncode == 0 and "racy: 512 race granules, 1 runs" in racy.stdout, (racy.stdout, racy.stderr)
    fixed = subprocess.run([exe, "--fixed"], capture_output=True, text=True, timeout=120)
    assert fixed.returncode == 0 and "fixed: 0 race granules, 0 runs" in fixed.stdout, (fixed.stdout, fixed.stderr)


def test_library_workspace_is_reused_and_released():
    """Checks without a caller workspace park theirs for the next check (cusan_plan_destroy);
    results are unchanged whether the block is reused, replaced by a larger one or released."""
    small = configs.make(3, "small")
    big = configs.make(5, "small")
    reps = []
    for w in (small, small, big, small, big):
        ops, args = w.arrays(True)
        tr, _ = lower_product(ops, args)
        reps.append((cs.check(tr, window_events=50), oracle.check_events(tr.cusan_trace_read(), 256)))
        if len(reps) == 4:
            cs.release_cached_memory()
    for rep, ref in reps:
        assert_equal(rep, ref)
    cs.release_cached_memory()


@pytest.mark.parametrize("ranges", [
    dict(CUSAN_RANGE_MAX="128", CUSAN_RANGE_BAL_MIN="128"),                  # one lane step per range
    dict(CUSAN_RANGE_MIN="1024", CUSAN_RANGE_MAX="1024", CUSAN_RANGE_BAL_MIN="1024"),
    dict(CUSAN_RANGE_PER_ACCESS="1", CUSAN_RANGE_MIN="128", CUSAN_RANGES_PER_WARP="64",
         CUSAN_RANGE_BAL_MIN="128"),
    dict(CUSAN_RANGE_MIN="2147483648", CUSAN_RANGE_MAX="2147483648",
         CUSAN_RANGE_BAL_MIN="2147483648"),                                   # one range per span
    dict(CUSAN_TAIL_PCT="0"),                                                  # no guided tail
    dict(CUSAN_TAIL_PCT="95", CUSAN_TAIL_DIV="16", CUSAN_RANGE_BAL_MIN="1024"),  # nearly all tail
], ids=["lane-step", "1Ki", "balance", "whole-span", "no-tail", "all-tail"])
def test_results_do_not_depend_on_the_work_decomposition(ranges, monkeypatch):
    """SURVEY §8(c) pin "invariance under tile size": the warp range length (the kernel's work unit,
    sized on the host) from one lane step to a whole span gives the oracle's report, in both shadow
    layouts and with shards."""
    for k, v in ranges.items():
        monkeypatch.setenv(k, v)
    for c in (3, 5):
        w = configs.make(c, "small")
        ops, args = w.arrays(True)
        tr, _ = lower_product(ops, args)
        ref = oracle.check_events(tr.cusan_trace_read(), 256)
        for window in (0, 97):
            for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
                assert_equal(cs.check(tr, window_events=window, flags=flags), ref)
        parts = [cs.check(tr, window_events=97, nshards=3, shard=s) for s in range(3)]
        assert_equal(cs.report_merge(np.concatenate([p.runs for p in parts]),
                                     sum(p.n_race_granules for p in parts)), ref)
