"""Step a2 on the device (plan_dev.cu): the interval, incidence and span tables the GPU builds are
byte-identical to the host planner's (CUSAN_CHECK_HOST_PLAN, build_host_plan + build_span_tables),
for one and many windows, both shadow layouts, granule-range shards and persisted shadows; the
reports agree with each other and with the oracle."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs, fuzz

pytestmark = pytest.mark.gpu

HOST, DEVICE = cs.CUSAN_CHECK_HOST_PLAN, cs.CUSAN_CHECK_DEVICE_PLAN
COUNTERS = ["n_intervals", "n_incidences", "n_spans", "n_windows", "shard_granules", "tracked_bytes",
            "tracked_bytes_shard", "spill_spans", "spill_heap_bytes", "shadow_bytes", "n_segments", "n_access",
            "shadow_cell_bytes"]


def _tables(tr, **kw):
    p = cs.Plan(tr, **kw)
    inc, spans = p.cusan_plan_tables()
    rep = p.run()
    p.close()
    return inc, spans, rep


def assert_same_plan(tr, **kw):
    di, ds, dr = _tables(tr, **dict(kw, flags=kw.get("flags", 0) | DEVICE))
    hi, hs, hr = _tables(tr, **dict(kw, flags=kw.get("flags", 0) | HOST))
    assert di.tobytes() == hi.tobytes(), "incidence tables differ"
    assert len(ds) == len(hs) and ds.tobytes() == hs.tobytes(), "span tables differ"
    for k in COUNTERS:
        assert dr.counters[k] == hr.counters[k], k
    assert dr.n_race_granules == hr.n_race_granules and np.array_equal(dr.runs, hr.runs)
    return dr


@pytest.mark.parametrize("flags", [0, cs.CUSAN_CHECK_DENSE_SHADOW], ids=["compressed", "dense"])
@pytest.mark.parametrize("window", [0, 1, 3, 17])
def test_device_tables_equal_host_tables_fuzz(window, flags):
    rng = np.random.default_rng(1200 + window + flags)
    for i in range(30):
        nf = int(rng.integers(2, 12))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(1, 150)), nf, n_keys=3,
                                         n_granules=int(rng.integers(1, 3000)), unaligned=bool(i % 3 == 0),
                                         p_access=float(rng.uniform(0.3, 0.9)))
        acc = ev["kind"] == 0
        ev["mode"][acc & (rng.random(len(ev)) < 0.5)] = 0          # many readers: read-set records
        tr = cs.Trace(nf)
        tr.cusan_trace_append_events(ev)
        kw = dict(window_events=window, flags=flags, persist_shadow=bool(i % 4 == 1))
        rep = assert_same_plan(tr, **kw)
        ref = oracle.check_events(ev, nf, threads=2)
        assert rep.n_race_granules == ref["n_race_granules"]
        assert np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))
        for nshards in (2, 5):
            for s in range(nshards):
                assert_same_plan(tr, nshards=nshards, shard=s, **kw)


@pytest.mark.parametrize("c", [1, 2, 3, 4, 5])
def test_device_tables_equal_host_tables_configs(c):
    w = configs.make(c, "small")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
        for window in (0, 97):
            assert_same_plan(tr, window_events=window, flags=flags)
        for s in range(3):
            assert_same_plan(tr, window_events=97, flags=flags, nshards=3, shard=s)


@pytest.mark.parametrize("c", [3, 5])
def test_device_tables_equal_host_tables_full_size(c):
    """BASELINE.json sizes in the bench launch configuration (4096-access windows), both layouts,
    and one of 8 shards."""
    import torch
    torch.cuda.empty_cache()                 # earlier tests' 64 GiB torch workspaces
    cs.release_cached_memory()
    w = configs.make(c, "full")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW):
        assert_same_plan(tr, window_events=4096, flags=flags)
    assert_same_plan(tr, window_events=4096, nshards=8, shard=5, flags=cs.CUSAN_CHECK_DENSE_SHADOW)


def test_device_plan_edge_cases():
    # no accesses / only empty accesses / one access
    t = cs.Trace(4)
    t.cusan_trace_append_sync(cs.CUSAN_RELEASE, 0, 5)
    assert_same_plan(t)
    t = cs.Trace(4)
    t.cusan_trace_append_access(0, 1, 0x1000, 0)
    t.cusan_trace_append_access(1, 1, 0x1000, 0)
    assert_same_plan(t, window_events=1)
    t = cs.Trace(4)
    t.cusan_trace_append_access(0, 1, 0x1000, 64)
    assert_same_plan(t, window_events=1)
    # more shards than intervals: empty shards
    t = cs.Trace(4)
    t.cusan_trace_append_access(0, 1, 0x1000, 64)
    t.cusan_trace_append_access(1, 0, 0x1000, 64)
    for s in range(6):
        assert_same_plan(t, nshards=6, shard=s, window_events=1)


@pytest.mark.parametrize("c", [3, 5])
def test_plan_from_clocks_equals_plan_from_trace(c):
    """cusan_plan_create_from_clocks (the multi-GPU path: one rank computes a1, every rank plans its
    shard from the broadcast image) builds the same tables and report as cusan_plan_create, also
    from an exported / imported image and per shard; reports equal the oracle's."""
    w = configs.make(c, "small")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    ref = oracle.check_events(tr.cusan_trace_read(), 256)
    clocks = cs.Clocks.from_bytes(cs.Clocks.compute(tr).to_bytes())
    for kw in (dict(window_events=97), dict(window_events=97, flags=cs.CUSAN_CHECK_DENSE_SHADOW),
               dict(window_events=0)):
        a_inc, a_sp, a_rep = _tables(tr, **kw)
        b_inc, b_sp, b_rep = _tables(clocks, **kw)
        assert a_inc.tobytes() == b_inc.tobytes() and a_sp.tobytes() == b_sp.tobytes()
        for k in COUNTERS:
            assert a_rep.counters[k] == b_rep.counters[k], k
        assert b_rep.n_race_granules == ref["n_race_granules"]
        assert np.array_equal(b_rep.runs, ref["runs"].astype(b_rep.runs.dtype))
        parts = [cs.Plan(clocks, nshards=4, shard=s, **kw) for s in range(4)]
        reps = [p.run() for p in parts]
        for p in parts:
            p.close()
        merged = cs.report_merge(np.concatenate([r.runs for r in reps]), sum(r.n_race_granules for r in reps))
        assert np.array_equal(merged.runs, ref["runs"].astype(merged.runs.dtype))
    h_inc, h_sp, h_rep = _tables(clocks, window_events=97, flags=cs.CUSAN_CHECK_HOST_PLAN)   # host a2
    d_inc, d_sp, _ = _tables(tr, window_events=97, flags=cs.CUSAN_CHECK_DEVICE_PLAN)
    assert h_inc.tobytes() == d_inc.tobytes() and h_sp.tobytes() == d_sp.tobytes()
    with pytest.raises(cs.CusanError):
        cs.Plan(tr, flags=cs.CUSAN_CHECK_HOST_PLAN | cs.CUSAN_CHECK_DEVICE_PLAN)


def test_device_planner_large_random_trace():
    """A 2.5 M-event trace of ~1.5 M small random accesses (hundreds of thousands of elementary
    intervals, grid-stride loops and multi-pass sorts in the device planner): device tables =
    host tables byte for byte, windowed and sharded; the report matches the oracle on sampled
    granules (every run edge and random interior granules)."""
    import brute
    from tracegen.program import EVENT_DTYPE
    rng = np.random.default_rng(2500)
    n = 2_500_000
    ev = np.zeros(n, EVENT_DTYPE)
    kind = rng.choice([0, 1, 2, 3, 4], size=n, p=[0.6, 0.12, 0.04, 0.16, 0.08])
    ev["kind"] = kind
    ev["fiber"] = rng.integers(0, 8, n)
    acc = kind == 0
    ev["mode"][acc] = rng.random(int(acc.sum())) < 0.3
    ev["a"][acc] = (1 << 32) + 8 * rng.integers(0, 1 << 24, int(acc.sum()))          # 128 MiB region
    ev["b"][acc] = 8 * rng.integers(1, 512, int(acc.sum()))
    syn = (kind >= 1) & (kind <= 3)
    ev["a"][syn] = rng.integers(0, 16, int(syn.sum()))
    fk = kind == 4
    ev["a"][fk] = rng.integers(0, 8, int(fk.sum()))
    tr = cs.Trace(8)
    tr.cusan_trace_append_events(ev)
    rep = assert_same_plan(tr, window_events=200_000)
    assert rep.counters["n_intervals"] > 100_000
    assert_same_plan(tr, window_events=200_000, nshards=3, shard=1, flags=cs.CUSAN_CHECK_DENSE_SHADOW)
    g = (ev["a"][acc] >> np.uint64(3)).astype(np.uint64)
    sample = np.unique(np.concatenate([g[rng.integers(0, len(g), 3000)],
                                       rep.runs["g_begin"][:2000], rep.runs["g_end"][:2000] - np.uint64(1)]))
    ref = oracle.check_events(ev, 8, sample=sample)
    sset = set(int(x) for x in sample)
    assert set(brute.runs_to_triples_in(rep.runs, sset)) == brute.runs_to_triples(ref["runs"])


def test_plans_from_clocks_edge_cases():
    """Clocks of an empty trace, of a trace without accesses and of one with only empty accesses
    plan and check to an empty report (host and device planners); a corrupt image is rejected."""
    for rows in ([], [(cs.CUSAN_RELEASE, 0, 5)], None):
        t = cs.Trace(4)
        if rows is None:
            t.cusan_trace_append_access(0, 1, 0x1000, 0)
            t.cusan_trace_append_access(1, 1, 0x1000, 0)
        else:
            for k, f, key in rows:
                t.cusan_trace_append_sync(k, f, key)
        ck = cs.Clocks.from_bytes(cs.Clocks.compute(t).to_bytes())
        for flags in (0, HOST, DEVICE):
            p = cs.Plan(ck, window_events=1, flags=flags)
            r = p.run()
            p.close()
            assert r.n_race_granules == 0 and r.n_runs == 0
