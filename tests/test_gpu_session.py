"""Incremental (online) checking: a session checks the accesses appended since its
previous call against the shadow it keeps on the device.  Each call's report must equal the oracle's
report of the final trace restricted to races whose later access belongs to that call."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs, fuzz
from tracegen.program import EV_ACCESS

pytestmark = pytest.mark.gpu


def _by_later(runs, lo, hi):
    m = (runs["later"] >= lo) & (runs["later"] < hi)
    return runs[m]


def _run_session(ev, nf, cuts, **kw):
    """Append ev in pieces ending at `cuts`, check after each; compare with the oracle."""
    ref = oracle.check_events(ev, nf, threads=2)
    tr = cs.Trace(nf)
    ses = cs.Session(tr, **kw)
    start, total = 0, 0
    for end in list(cuts) + [len(ev)]:
        if end <= start:
            continue
        tr.cusan_trace_append_events(ev[start:end])
        rep = ses.check()
        want = _by_later(ref["runs"], start, end)
        assert np.array_equal(rep.runs, want.astype(rep.runs.dtype)), (start, end)
        assert rep.n_race_granules == int(np.sum(want["g_end"] - want["g_begin"]))
        total += rep.n_race_granules
        start = end
    ses.close()
    assert total == ref["n_race_granules"]
    return ref


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
@pytest.mark.parametrize("window", [0, 3])
def test_session_fuzz(window, flags):
    rng = np.random.default_rng(600 + window)
    for _ in range(25):
        nf = int(rng.integers(2, 9))
        n = int(rng.integers(2, 90))
        ev = fuzz.random_primitive_trace(rng, n, nf, n_keys=3, n_granules=int(rng.integers(1, 900)),
                                         unaligned=bool(rng.integers(2)))
        k = int(rng.integers(1, 6))
        cuts = sorted(int(x) for x in rng.integers(1, n, size=k))
        _run_session(ev, nf, cuts, window_events=window, flags=flags)


def test_session_many_readers_across_calls():
    """Read sets that spill into records survive from one call to the next."""
    rng = np.random.default_rng(77)
    for _ in range(15):
        nf = int(rng.integers(6, 40))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(30, 200)), nf, n_keys=4,
                                         n_granules=int(rng.integers(50, 700)), p_access=0.85)
        acc = ev["kind"] == EV_ACCESS
        ev["mode"][acc & (rng.random(len(ev)) < 0.8)] = 0
        cuts = sorted(int(x) for x in rng.integers(1, len(ev), size=4))
        for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
            _run_session(ev, nf, cuts, flags=flags)


@pytest.mark.parametrize("c", [2, 3, 5])
def test_session_small_configs(c):
    w = configs.make(c, "small")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    ev = tr.cusan_trace_read()
    cuts = list(np.linspace(0, len(ev), 7).astype(int)[1:-1])
    ref = _run_session(ev, 255, cuts, window_events=64)
    assert ref["n_race_granules"] > 0


def test_session_rejects_bad_shards_and_shrinking():
    tr = cs.Trace(4)
    with pytest.raises(cs.CusanError):
        cs.Session(tr, nshards=2, shard=2)
    with pytest.raises(cs.CusanError):
        cs.Session(tr, nshards=2, shard=0, shard_block=48)      # not a power of two
    ses = cs.Session(tr)
    tr.cusan_trace_append_access(0, 1, 0x1000, 64)
    tr.cusan_trace_append_access(1, 1, 0x1000, 64)
    assert ses.check().n_race_granules == 8
    assert ses.check().n_race_granules == 0          # nothing new
    ses.close()


def test_session_interval_compressed():
    rng = np.random.default_rng(31)
    for _ in range(20):
        nf = int(rng.integers(2, 9))
        n = int(rng.integers(2, 90))
        ev = fuzz.random_primitive_trace(rng, n, nf, n_keys=3, n_granules=int(rng.integers(1, 900)))
        cuts = sorted(int(x) for x in rng.integers(1, n, size=int(rng.integers(1, 6))))
        _run_session(ev, nf, cuts, window_events=int(rng.integers(0, 4)), flags=cs.CUSAN_CHECK_INTERVAL_SHADOW)


def test_session_compressed_shared_records_across_splits():
    """f3 sessions: a split compressed interval copies its cell; a read-set record it names becomes
    shared by both cells (records are written once and never updated in place)."""
    rng = np.random.default_rng(91)
    for _ in range(15):
        nf = int(rng.integers(6, 30))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(40, 200)), nf, n_keys=3,
                                         n_granules=int(rng.integers(20, 400)), p_access=0.85)
        acc = ev["kind"] == EV_ACCESS
        ev["mode"][acc & (rng.random(len(ev)) < 0.8)] = 0
        cuts = sorted(set(int(x) for x in rng.integers(1, len(ev), size=10)))
        _run_session(ev, nf, cuts, flags=cs.CUSAN_CHECK_INTERVAL_SHADOW)


def test_session_shadow_growth_many_calls():
    """Every call touches new memory, so the shadow grows (new mapped chunks) call after call;
    the cells of the first call survive every growth."""
    from tracegen.program import EVENT_DTYPE, EV_RELEASE, EV_ACQUIRE
    rows = []
    base, size = 1 << 32, 1 << 20                      # 1 MiB = 131072 granules per call
    n_calls = 40
    order = [c for c in range(n_calls) if c % 2 == 0] + [c for c in range(n_calls) if c % 2]
    for i, c in enumerate(order):                      # fiber 0 writes region c; the even ones
        if i == n_calls // 2:                          # before its release
            rows.append((EV_RELEASE, 0, 0, 7, 0))
        rows.append((EV_ACCESS, 1, 0, base + c * 3 * size, size))
    rows.append((EV_ACQUIRE, 0, 1, 7, 0))
    for c in range(n_calls):                           # fiber 1 reads part of every region: the
        rows.append((EV_ACCESS, 0, 1, base + c * 3 * size + 8 * c, size // 2))   # odd ones race
    ev = np.zeros(len(rows), EVENT_DTYPE)
    for i, (k, m, f, a, b) in enumerate(rows):
        ev[i]["kind"], ev[i]["mode"], ev[i]["fiber"], ev[i]["a"], ev[i]["b"] = k, m, f, a, b
    cuts = list(range(1, n_calls)) + [n_calls + 2 + 5 * i for i in range(8)]
    ref = _run_session(ev, 2, cuts)
    assert ref["n_race_granules"] == (n_calls // 2) * (size // 2) // 8


@pytest.mark.parametrize("nshards,block", [(2, 64), (3, 32), (4, 1 << 12)])
@pytest.mark.parametrize("flags", [cs.CUSAN_CHECK_DENSE_SHADOW, 0], ids=["per-granule", "compressed"])
def test_session_block_cyclic_shards_merge_per_call(nshards, block, flags):
    """Multi-GPU sessions: per call, the merged reports of the block-cyclic shards equal the
    one-shard session's report of that call (which the other session tests pin to the oracle);
    shard granules and checked bytes add up."""
    rng = np.random.default_rng(100 + nshards)
    for _ in range(6):
        nf = int(rng.integers(2, 7))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(20, 150)), nf, n_keys=3,
                                         n_granules=int(rng.integers(200, 6000)))
        cuts = sorted({0, len(ev), *rng.integers(1, len(ev), 3).tolist()})
        trs = [cs.Trace(nf) for _ in range(nshards + 1)]
        whole = cs.Session(trs[0], window_events=3, flags=flags)
        parts = [cs.Session(trs[1 + s], window_events=3, flags=flags, nshards=nshards, shard=s,
                            shard_block=block) for s in range(nshards)]
        for a, b in zip(cuts[:-1], cuts[1:]):
            for t in trs:
                t.cusan_trace_append_events(ev[a:b])
            ref = whole.check()
            reps = [p.check() for p in parts]
            merged = cs.report_merge(np.concatenate([r.runs for r in reps]), sum(r.n_race_granules for r in reps))
            assert merged.n_race_granules == ref.n_race_granules
            assert np.array_equal(merged.runs, ref.runs)
            assert sum(r.counters["tracked_bytes_shard"] for r in reps) == ref.counters["tracked_bytes"]
            assert sum(r.counters["shard_granules"] for r in reps) == ref.counters["shard_granules"]
        whole.close()
        for p in parts:
            p.close()


def test_session_shards_small_config():
    w = configs.make(5, "small")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    ev = tr.cusan_trace_read()
    ref = oracle.check_events(ev, 256)
    trs = [cs.Trace(255) for _ in range(3)]
    ses = [cs.Session(trs[s], window_events=97, nshards=3, shard=s, shard_block=1 << 10) for s in range(3)]
    runs, n = [], 0
    for a in range(0, len(ev), len(ev) // 4 + 1):
        for t in trs:
            t.cusan_trace_append_events(ev[a:a + len(ev) // 4 + 1])
        for s in ses:
            r = s.check()
            runs.append(r.runs)
            n += r.n_race_granules
    merged = cs.report_merge(np.concatenate(runs), n)
    assert merged.n_race_granules == ref["n_race_granules"] > 0
    assert np.array_equal(merged.runs, ref["runs"].astype(merged.runs.dtype))
    for s in ses:
        s.close()


@pytest.mark.parametrize("flags,nshards", [(cs.CUSAN_CHECK_DENSE_SHADOW, 1), (0, 1),
                                           (cs.CUSAN_CHECK_DENSE_SHADOW, 2), (0, 2)],
                         ids=["dense", "compressed", "dense-shards", "compressed-shards"])
def test_session_submit_pipelines_and_matches_check(flags, nshards):
    """submit/finish (host planning of call i+1 overlapping the device work of call i, records
    numbered at launch) return, call by call, exactly what check() returns."""
    rng = np.random.default_rng(300 + flags + nshards)
    for _ in range(6):
        nf = int(rng.integers(2, 9))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(20, 160)), nf, n_keys=3,
                                         n_granules=int(rng.integers(100, 4000)))
        cuts = sorted({0, len(ev), *rng.integers(1, len(ev), 4).tolist()})
        for shard in range(nshards):
            kw = dict(window_events=2, flags=flags, nshards=nshards, shard=shard, shard_block=64)
            ta, tb = cs.Trace(nf), cs.Trace(nf)
            sa, sb = cs.Session(ta, **kw), cs.Session(tb, **kw)
            want, got = [], []
            for a, b in zip(cuts[:-1], cuts[1:]):
                ta.cusan_trace_append_events(ev[a:b])
                tb.cusan_trace_append_events(ev[a:b])
                want.append(sa.check())
                prev = sb.submit()
                if prev is not None:
                    got.append(prev)
                with pytest.raises(cs.CusanError):
                    sb.check()                   # a call is in flight
            got.append(sb.finish())
            assert sb.finish() is None
            assert len(got) == len(want)
            for x, y in zip(got, want):
                assert x.n_race_granules == y.n_race_granules
                assert np.array_equal(x.runs, y.runs)
            sa.close()
            sb.close()


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
def test_session_read_set_records_are_reclaimed(flags):
    """Intervals read by several fibers in every call (weights read by forward and backward
    streams) get a new read-set record per call; the records the layout no longer names are reused
    from the next call on, so the heap stays at its high-water mark of the first calls instead of
    growing call after call.  Every call still equals the oracle's report restricted to it."""
    from tracegen.program import EVENT_DTYPE, EV_ACQUIRE, EV_RELEASE
    rows = []
    base, size, n_calls, per_call = 1 << 33, 1 << 16, 60, []
    for c in range(n_calls):
        start = len(rows)
        for f in (1, 2, 3):                                   # three readers of both buffers
            rows.append((EV_ACCESS, 0, f, base, size))
            rows.append((EV_ACCESS, 0, f, base + 2 * size, size))
        if c % 7 == 3:                                        # an unordered write now and then
            rows.append((EV_ACCESS, 1, 4, base + 2 * size + 64, 256))
        for f in (1, 2, 3):
            rows.append((EV_RELEASE, 0, f, 100 + f, 0))
            rows.append((EV_ACQUIRE, 0, 0, 100 + f, 0))
        rows.append((EV_ACCESS, 1, 0, base + size // 2, size // 4))   # host writes part of buffer 0
        rows.append((EV_RELEASE, 0, 0, 99, 0))
        for f in (1, 2, 3, 4):
            rows.append((EV_ACQUIRE, 0, f, 99, 0))
        per_call.append((start, len(rows)))
    ev = np.zeros(len(rows), EVENT_DTYPE)
    for i, (k, m, f, a, b) in enumerate(rows):
        ev[i]["kind"], ev[i]["mode"], ev[i]["fiber"], ev[i]["a"], ev[i]["b"] = k, m, f, a, b
    ref = oracle.check_events(ev, 5, threads=2)
    assert ref["n_race_granules"] > 0
    tr = cs.Trace(5)
    ses = cs.Session(tr, window_events=2, flags=flags)
    heap = []
    for a, b in per_call:
        tr.cusan_trace_append_events(ev[a:b])
        rep = ses.check()
        want = _by_later(ref["runs"], a, b)
        assert np.array_equal(rep.runs, want.astype(rep.runs.dtype)), (a, b)
        heap.append(rep.counters["heap_bytes"])
        assert rep.counters["heap_live_bytes"] <= rep.counters["heap_bytes"]
    ses.close()
    assert heap[-1] == heap[10] > 0, heap         # bounded: no growth once the layout is stable


FULL_GOLDEN = __import__("os").path.join(__import__("os").path.dirname(__import__("os").path.abspath(__file__)),
                                         "golden", "full")


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
@pytest.mark.parametrize("per_call", [4096, 512])
def test_session_full_size_config5(per_call, flags):
    """The config-5 racy trace at its full size (64 GiB tracked, 64 fibers) fed to an online
    session in calls of `per_call` accesses (9 calls of 4096, 71 of 512): every call's report equals
    the oracle's complete report (tests/golden/full/config5_racy.npz, every granule checked by
    oracle.c) restricted to the races whose later access is in that call (CuSan
    checks on the fly); the counts add up to the whole."""
    import hashlib
    import os

    import torch
    torch.cuda.empty_cache()
    cs.release_cached_memory()
    g = np.load(os.path.join(FULL_GOLDEN, "config5_racy.npz"))
    w = configs.make(5, "full")
    ops, args = w.arrays(True)
    full = cs.Trace(255)
    cs.Lowering(full).cusan_lower_program(ops, args)
    ev = full.cusan_trace_read()
    assert hashlib.sha256(np.ascontiguousarray(ev).tobytes()).hexdigest() == str(g["events_sha256"])
    golden = g["runs"]
    acc_pos = np.flatnonzero(ev["kind"] == EV_ACCESS)
    cuts = [int(acc_pos[k]) for k in range(per_call, len(acc_pos), per_call)] + [len(ev)]
    tr = cs.Trace(255)
    ses = cs.Session(tr, window_events=per_call, flags=flags)
    start, total, calls = 0, 0, 0
    for end in cuts:
        tr.cusan_trace_append_events(ev[start:end])
        rep = ses.check()
        want = _by_later(golden, start, end)
        assert np.array_equal(rep.runs, want.astype(rep.runs.dtype)), (start, end)
        assert rep.n_race_granules == int(np.sum(want["g_end"] - want["g_begin"]))
        total += rep.n_race_granules
        start, calls = end, calls + 1
    ses.close()
    assert calls == -(-len(acc_pos) // per_call)
    assert total == int(g["n_race_granules"]) > 0


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
@pytest.mark.parametrize("window", [0, 3])
def test_session_epoch_renumbering_fuzz(window, flags, monkeypatch):
    """Sessions renumber their live event ids when the trace outgrows the epoch field; with the
    field's limit lowered to a few hundred events (CUSAN_SESSION_EVENT_LIMIT) renumbering happens
    every few calls, and every call still equals the oracle's report restricted to it (ids are
    trace positions in the reports), for many readers (records), splits and windows."""
    monkeypatch.setenv("CUSAN_SESSION_EVENT_LIMIT", "400")
    rng = np.random.default_rng(4400 + window + flags)
    renumbered = 0
    for _ in range(12):
        nf = int(rng.integers(2, 10))
        n = int(rng.integers(300, 900))
        ev = fuzz.random_primitive_trace(rng, n, nf, n_keys=4, n_granules=int(rng.integers(50, 1500)),
                                         unaligned=bool(rng.integers(2)), p_access=0.5)
        acc = ev["kind"] == EV_ACCESS
        ev["mode"][acc & (rng.random(len(ev)) < 0.5)] = 0
        cuts = list(range(int(rng.integers(20, 60)), n, int(rng.integers(20, 60))))
        ref = oracle.check_events(ev, nf, threads=2)
        tr = cs.Trace(nf)
        ses = cs.Session(tr, window_events=window, flags=flags)
        start = 0
        for end in cuts + [n]:
            tr.cusan_trace_append_events(ev[start:end])
            rep = ses.check()
            want = _by_later(ref["runs"], start, end)
            assert np.array_equal(rep.runs, want.astype(rep.runs.dtype)), (start, end)
            start = end
        renumbered += rep.counters["renumberings"]
        ses.close()
    assert renumbered > 10


def test_session_epoch_renumbering_pipelined_and_sharded(monkeypatch):
    """Renumbering with a call in flight (submit / finish) and in block-cyclic shard sessions: the
    merged shard reports of every call equal the oracle's."""
    monkeypatch.setenv("CUSAN_SESSION_EVENT_LIMIT", "300")
    rng = np.random.default_rng(4500)
    for _ in range(6):
        nf = int(rng.integers(2, 8))
        n = 900
        ev = fuzz.random_primitive_trace(rng, n, nf, n_keys=3, n_granules=int(rng.integers(200, 3000)))
        ref = oracle.check_events(ev, nf, threads=2)
        cuts = list(range(40, n, 40)) + [n]
        trs = [cs.Trace(nf) for _ in range(3)]
        ses = [cs.Session(trs[s], window_events=2, nshards=3, shard=s, shard_block=64) for s in range(3)]
        got = {s: [] for s in range(3)}
        start = 0
        for end in cuts:
            for t in trs:
                t.cusan_trace_append_events(ev[start:end])
            for k, x in enumerate(ses):
                prev = x.submit()
                if prev is not None:
                    got[k].append(prev)
            start = end
        for k, x in enumerate(ses):
            got[k].append(x.finish())
            x.close()
        start = 0
        for c, end in enumerate(cuts):
            reps = [got[k][c] for k in range(3)]
            merged = cs.report_merge(np.concatenate([r.runs for r in reps]), sum(r.n_race_granules for r in reps))
            want = _by_later(ref["runs"], start, end)
            assert np.array_equal(merged.runs, want.astype(merged.runs.dtype)), (start, end)
            start = end
        assert got[0][-1].counters["renumberings"] > 0


def test_session_beyond_2_24_events():
    """A session past 2^24 events (the real epoch field): 2^24 + 2^21 events in 12 calls — writes,
    reads and syncs among 4 fibers on a few buffers between long runs of releases; every call equals
    the oracle's report restricted to it, with trace positions past 2^24 in the runs."""
    from tracegen.program import EVENT_DTYPE, EV_ACQUIRE, EV_RELEASE
    rng = np.random.default_rng(2424)
    n = (1 << 24) + (1 << 21)
    ev = np.zeros(n, EVENT_DTYPE)
    ev["kind"] = EV_RELEASE
    ev["fiber"] = 3
    ev["a"] = 99
    pos = np.sort(rng.choice(np.arange(10, n), 3000, replace=False))
    for p in pos:
        r = rng.random()
        f = int(rng.integers(0, 4))
        if r < 0.6:
            ev[p]["kind"], ev[p]["mode"], ev[p]["fiber"] = EV_ACCESS, int(rng.random() < 0.4), f
            ev[p]["a"], ev[p]["b"] = (1 << 32) + 4096 * int(rng.integers(0, 6)), 8 * int(rng.integers(1, 700))
        else:
            ev[p]["kind"], ev[p]["fiber"], ev[p]["a"] = (EV_RELEASE if r < 0.8 else EV_ACQUIRE), f, int(rng.integers(0, 3))
    ref = oracle.check_events(ev, 4, threads=8)
    assert ref["n_race_granules"] > 0 and int(ref["runs"]["later"].max()) > (1 << 24)
    tr = cs.Trace(4)
    ses = cs.Session(tr, window_events=64)
    cuts = [int(x) for x in np.linspace(0, n, 13)[1:]]
    start, total = 0, 0
    for end in cuts:
        tr.cusan_trace_append_events(ev[start:end])
        rep = ses.check()
        want = _by_later(ref["runs"], start, end)
        assert np.array_equal(rep.runs, want.astype(rep.runs.dtype)), (start, end)
        total += rep.n_race_granules
        start = end
    assert rep.counters["renumberings"] >= 1
    assert total == ref["n_race_granules"]
    ses.close()


def _instances_trace(rng, n, nf, n_keys=3):
    """Events over short-lived allocation instances (disjoint 64-granule ranges, a sliding set of
    three live ones), as the live capture records a program's temporaries; returns the events and
    each instance's (range, last access position)."""
    from tracegen.program import EVENT_DTYPE, EV_ACQUIRE, EV_FORK, EV_RELEASE
    base = 1 << 36
    ev = np.zeros(n, EVENT_DTYPE)
    last = {}
    for i in range(n):
        f = int(rng.integers(nf))
        if rng.random() < 0.6:
            inst = i // 12 + int(rng.integers(3))
            g0 = int(rng.integers(64))
            g1 = int(rng.integers(g0 + 1, 65))
            ev[i] = (EV_ACCESS, int(rng.random() < 0.45), 0, f, base + 512 * inst + 8 * g0, 8 * (g1 - g0))
            last[inst] = i
        else:
            u = rng.random()
            if u < 0.4:
                ev[i] = (EV_RELEASE, 0, 0, f, 1000 + int(rng.integers(n_keys)), 0)
            elif u < 0.8:
                ev[i] = (EV_ACQUIRE, 0, 0, f, 1000 + int(rng.integers(n_keys)), 0)
            else:
                src = (f + 1 + int(rng.integers(nf - 1))) % nf
                ev[i] = (EV_FORK, 0, 0, f, src, 0)
    return ev, {k: ((base + 512 * k, 512), p) for k, p in last.items()}


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
def test_session_forget_released_ranges(flags):
    """cusan_session_forget of ranges no later access touches leaves every call's report equal to
    the oracle's, and keeps the layout to the live ranges (it grows without)."""
    rng = np.random.default_rng(4242)
    for _ in range(12):
        nf = int(rng.integers(2, 7))
        n = int(rng.integers(200, 600))
        ev, inst = _instances_trace(rng, n, nf)
        ref = oracle.check_events(ev, nf, threads=2)
        cuts = sorted(set(int(x) for x in rng.integers(1, n, size=12))) + [n]
        tr, tr2 = cs.Trace(nf), cs.Trace(nf)
        ses, ses2 = cs.Session(tr, flags=flags), cs.Session(tr2, flags=flags)
        start, forgotten = 0, set()
        ivs, ivs2 = [], []
        for end in cuts:
            if end <= start:
                continue
            for t in (tr, tr2):
                t.cusan_trace_append_events(ev[start:end])
            rep, rep2 = ses.check(), ses2.check()
            want = _by_later(ref["runs"], start, end)
            for r in (rep, rep2):
                assert np.array_equal(r.runs, want.astype(r.runs.dtype)), (start, end)
                assert r.n_race_granules == int(np.sum(want["g_end"] - want["g_begin"]))
            ivs.append(rep.counters["n_intervals"])
            ivs2.append(rep2.counters["n_intervals"])
            # instances whose last access is already appended are released: never touched again
            for k, ((addr, size), p) in inst.items():
                if p < end and k not in forgotten:
                    ses.forget(addr, size)
                    forgotten.add(k)
            start = end
        ses.close()
        ses2.close()
        assert ivs[-1] < ivs2[-1], (ivs, ivs2)


def test_c_example_online_jacobi():
    """examples/online_jacobi.c: a session through the C ABI checks a two-stream Jacobi after every
    iteration and forgets each released temporary; the calls add up to one cusan_check of the whole
    trace, the racy variant (no halo-stream wait) races and the clean one does not, and the layout
    stays bounded."""
    import subprocess
    import __graft_entry__ as g
    exe = [e for e in g.build_examples() if e.endswith("online_jacobi")][0]
    for racy in (False, True):
        r = subprocess.run([exe] + (["--racy"] if racy else []), capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, (r.stdout, r.stderr)
        assert ("racy:" if racy else "clean:") in r.stdout
