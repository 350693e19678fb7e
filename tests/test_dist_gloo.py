"""Multi-GPU host logic on CPU: world_size-2 gloo process group.

The kernels need a GPU, so here the two ranks exercise everything around them: the host shard
partition (cusan_plan_describe), the run gather (dist.gather_runs over gloo) and rank 0's stitch
and canonical sort (cusan_report_merge).  Each rank's shard runs are the oracle's runs clipped to
that rank's granule range, so a stitch that failed to re-join runs cut at the shard boundary, or
lost a rank's runs, would not reproduce the oracle's whole report.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _clip(runs, lo, hi):
    out = runs.copy()
    out["g_begin"] = np.maximum(out["g_begin"], np.uint64(lo))
    out["g_end"] = np.minimum(out["g_end"], np.uint64(hi))
    return out[out["g_begin"] < out["g_end"]]


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_sc_huckzsjb24_b200 as cs
        from paper_conf_sc_huckzsjb24_b200.dist import gather_runs
        from tracegen import configs
        w = configs.make(4, "small")
        ops, args = w.arrays(True)
        tr = cs.Trace(255)
        cs.Lowering(tr).cusan_lower_program(ops, args)
        ev = tr.cusan_trace_read()
        ref = oracle.check_events(ev, 255, threads=2)
        # shard boundary at the middle of the covered granule space (absolute granules)
        acc = ev[ev["kind"] == 0]
        g_lo = int(acc["a"].min()) >> 3
        g_hi = int((acc["a"] + acc["b"]).max() + 7) >> 3
        cut = (g_lo + g_hi) // 2 + 3
        lo, hi = (g_lo, cut) if rank == 0 else (cut, g_hi)
        mine = _clip(ref["runs"], lo, hi)
        n_mine = int(np.sum(mine["g_end"] - mine["g_begin"]))
        out = gather_runs(mine, n_mine)
        # host shard partition of the product: the two shards tile the granule space and the
        # coverage weight
        parts = [cs.describe(tr, nshards=world, shard=s) for s in range(world)]
        whole = cs.describe(tr)
        part_ok = (sum(p["shard_granules"] for p in parts) == whole["shard_granules"] and
                   sum(p["tracked_bytes_shard"] for p in parts) == whole["tracked_bytes"])
        if rank == 0:
            runs, n = out
            merged = cs.report_merge(runs, n)
            q.put(dict(ok=bool(np.array_equal(merged.runs, ref["runs"].astype(merged.runs.dtype))
                               and merged.n_race_granules == ref["n_race_granules"]
                               and merged.n_runs == ref["n_runs"] and ref["n_runs"] > 0),
                       part_ok=part_ok, split_runs=len(runs)))
        else:
            q.put(dict(ok=out is None, part_ok=part_ok))
    finally:
        dist.destroy_process_group()


def test_two_rank_gather_and_stitch():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(r["ok"] for r in res), res
    assert all(r["part_ok"] for r in res), res


@pytest.mark.parametrize("nshards", [2, 3, 8])
def test_shard_partition_balances_coverage(nshards):
    import paper_conf_sc_huckzsjb24_b200 as cs
    from tracegen import configs
    w = configs.make(5, "small")
    ops, args = w.arrays(False)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    whole = cs.describe(tr)
    parts = [cs.describe(tr, nshards=nshards, shard=s) for s in range(nshards)]
    assert sum(p["shard_granules"] for p in parts) == whole["shard_granules"]
    assert sum(p["tracked_bytes_shard"] for p in parts) == whole["tracked_bytes"]
    ideal = whole["tracked_bytes"] / nshards
    # equal coverage weight up to one interval's granule boundary rounding
    assert max(abs(p["tracked_bytes_shard"] - ideal) for p in parts) <= 0.01 * ideal + 8 * 1000


@pytest.mark.parametrize("nshards", [2, 8])
def test_windowed_shards_balance_moved_cells(nshards):
    """Windowed checks are bound by the cells moved, so shards balance granules × windows."""
    import paper_conf_sc_huckzsjb24_b200 as cs
    from tracegen import configs
    w = configs.make(5, "small")
    ops, args = w.arrays(False)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    parts = [cs.describe(tr, nshards=nshards, shard=s, window_events=64) for s in range(nshards)]
    whole = cs.describe(tr, window_events=64)
    assert sum(p["shard_granules"] for p in parts) == whole["shard_granules"]
    assert sum(p["tracked_bytes_shard"] for p in parts) == whole["tracked_bytes"]
    g = [p["shard_granules"] for p in parts]
    assert min(g) > 0.5 * max(g)


def _bcast_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sc_huckzsjb24_b200 as cs
        from paper_conf_sc_huckzsjb24_b200.dist import broadcast_trace
        from tracegen import configs
        w = configs.make(5, "small")
        ops, args = w.arrays(True)
        half = len(ops) // 2
        mine = cs.Trace(255)                          # what every rank would have lowered itself
        cs.Lowering(mine).cusan_lower_program(ops, args)
        if rank == 0:                                 # only rank 0 records the program
            tr = cs.Trace(255)
            low = cs.Lowering(tr)
            low.cusan_lower_program(ops[:half], args)
            got = broadcast_trace(tr)
            n0 = len(tr)
            low.cusan_lower_program(ops[half:], args)
            got = broadcast_trace(tr, first=n0)       # incremental: only the new events
        else:
            got = broadcast_trace(None)
            got = broadcast_trace(got)
        same = bool(np.array_equal(got.cusan_trace_read(), mine.cusan_trace_read()))
        d_got = cs.describe(got, nshards=world, shard=rank, window_events=64)
        d_mine = cs.describe(mine, nshards=world, shard=rank, window_events=64)
        q.put(dict(rank=rank, same=same, plan_same=d_got == d_mine,
                   fibers=got.cusan_trace_size()[1]))
    finally:
        dist.destroy_process_group()


def test_two_rank_trace_broadcast():
    """Rank 0 records the program and broadcasts its events (whole, then incrementally); rank 1's
    trace, and the shard plan it builds from it, equal what lowering the program itself gives."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bcast_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(r["same"] and r["plan_same"] and r["fibers"] == 255 for r in res), res


def _clocks_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sc_huckzsjb24_b200 as cs
        from paper_conf_sc_huckzsjb24_b200.dist import broadcast_clocks
        from tracegen import configs
        w = configs.make(5, "small")
        ops, args = w.arrays(True)
        mine = cs.Trace(255)                          # what every rank would have lowered itself
        cs.Lowering(mine).cusan_lower_program(ops, args)
        want = cs.Clocks.compute(mine).to_bytes()
        got = broadcast_clocks(cs.Clocks.compute(mine) if rank == 0 else None)   # rank 0 computes
        q.put(dict(rank=rank, same=bool(np.array_equal(got.to_bytes(), want)), n=len(want)))
    finally:
        dist.destroy_process_group()


def test_two_rank_clocks_broadcast():
    """SURVEY §8(e) "event clocks broadcast": rank 0 computes a1 once and broadcasts the clocks
    image; rank 1's clocks equal the ones it would have computed itself."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_clocks_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(r["same"] and r["n"] > 1000 for r in res), res


def test_clocks_image_round_trip_and_validation():
    """Export → import → export is the identity; the image carries a1's counters; a corrupt or
    truncated image is rejected (CUSAN_EINVAL), never read past its end."""
    import paper_conf_sc_huckzsjb24_b200 as cs
    from tracegen import configs
    w = configs.make(3, "small")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    img = cs.Clocks.compute(tr).to_bytes()
    assert np.array_equal(cs.Clocks.from_bytes(img).to_bytes(), img)
    d = cs.describe(tr)
    hdr = img[:40].view(np.uint64)                    # magic/version/F/pad, n_acc, nseg, n_events
    assert int(hdr[2]) == d["n_access"] and int(hdr[3]) == d["n_segments"] and int(hdr[4]) == d["n_events"]
    bad = img.copy()
    bad[0] ^= 1
    with pytest.raises(cs.CusanError):
        cs.Clocks.from_bytes(bad)
    with pytest.raises(cs.CusanError):
        cs.Clocks.from_bytes(img[:-4])


def _a1_reference(ev, F):
    """a1 written out per event (DESIGN §2 / SURVEY §8(c) step 2, with PAPER.md:156-173's clock rules):
    per access its (fiber, id+1) epoch and segment, and one clock row per segment (the accessing
    fiber's clock at the segment's first access; a segment opens at a fiber's first access after an
    ACQUIRE or an incoming FORK)."""
    C = np.zeros((F, F), np.uint32)
    SC = {}
    cur = [None] * F
    rows, recs, g0s, g1s = [], [], [], []
    for i, e in enumerate(ev):
        k, f = int(e["kind"]), int(e["fiber"])
        if k == 4:                                   # FORK(src -> f): an event of src
            s = int(e["a"])
            C[s, s] = i + 1
            C[f] = np.maximum(C[f], C[s])
            cur[f] = None
            continue
        C[f, f] = i + 1
        if k == 0:
            if cur[f] is None:
                cur[f] = len(rows)
                rows.append(C[f].copy())
            recs.append(((f << 24) | (i + 1), cur[f] | (int(e["mode"]) << 31)))
            a, b = int(e["a"]), int(e["b"])
            g0s.append(a >> 3)
            g1s.append((a + b + 7) >> 3 if b else a >> 3)
        elif k == 1:
            SC[int(e["a"])] = np.maximum(SC.get(int(e["a"]), np.zeros(F, np.uint32)), C[f])
        elif k == 2:
            SC[int(e["a"])] = C[f].copy()
        elif k == 3:
            C[f] = np.maximum(C[f], SC.get(int(e["a"]), np.zeros(F, np.uint32)))
            cur[f] = None
    return rows, recs, g0s, g1s


@pytest.mark.parametrize("seed", range(4))
def test_clocks_equal_a1_written_out(seed):
    """The product's a1 (column-parallel, cusan_clocks_compute) against a1 written out per event:
    access ranges, epochs, segments and every segment row of the clocks image."""
    import paper_conf_sc_huckzsjb24_b200 as cs
    from tracegen import fuzz
    rng = np.random.default_rng(90 + seed)
    for t in range(12):
        nf = int(rng.integers(2, 40))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(1, 400)), nf, n_keys=int(rng.integers(1, 6)),
                                         n_granules=int(rng.integers(1, 300)), unaligned=bool(t % 2))
        if seed == 3:                                # large enough for the threaded column pass
            ev = np.concatenate([ev] * 60)
        tr = cs.Trace(nf)
        tr.cusan_trace_append_events(ev)
        img = cs.Clocks.compute(tr).to_bytes()
        F = int(img[8:12].view(np.uint32)[0])
        n_acc, nseg = (int(x) for x in img[16:32].view(np.uint64))
        ctr_bytes = len(img) - (n_acc * 24 + nseg * F * 4) - 40      # the counters struct follows the header
        p = 40 + ctr_bytes
        g0 = img[p:p + 8 * n_acc].view(np.uint64); p += 8 * n_acc
        g1 = img[p:p + 8 * n_acc].view(np.uint64); p += 8 * n_acc
        rec = img[p:p + 8 * n_acc].view(np.uint32).reshape(-1, 2); p += 8 * n_acc
        rows = img[p:p + 4 * nseg * F].view(np.uint32).reshape(nseg, F) if nseg else np.zeros((0, F), np.uint32)
        w_rows, w_recs, w_g0, w_g1 = _a1_reference(ev, F)
        assert len(w_rows) == nseg and n_acc == len(w_recs)
        assert [tuple(int(x) for x in r) for r in rec] == w_recs
        assert list(g0) == w_g0 and list(g1) == w_g1
        for r, wr in zip(rows, w_rows):
            assert np.array_equal(r, wr)


def test_clocks_one_pass_equals_column_form(tmp_path):
    """a1's default one-pass form (whole rows, one thread) and its two-pass column form
    (CUSAN_A1_COLUMNS=1: serial pre-pass, then column blocks on threads) give the same clocks
    image byte for byte — ranges, epochs, segment rows and counters."""
    import subprocess
    import sys

    import paper_conf_sc_huckzsjb24_b200 as cs
    from tracegen import fuzz
    rng = np.random.default_rng(123)
    traces = []
    for t in range(10):
        nf = int(rng.integers(2, 70))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(1, 500)), nf, n_keys=int(rng.integers(1, 9)),
                                         n_granules=int(rng.integers(1, 300)), unaligned=bool(t % 2))
        if t >= 7:                                   # large enough for the threaded column pass
            ev = np.concatenate([ev] * 80)
        traces.append((nf, ev))
    np.savez(tmp_path / "tr.npz", **{f"ev{i}": ev for i, (_, ev) in enumerate(traces)},
             nf=np.array([nf for nf, _ in traces]))
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = (f"import sys; sys.path.insert(0, {root!r}); import numpy as np; "
            "import paper_conf_sc_huckzsjb24_b200 as cs; "
            f"d = np.load({str(tmp_path / 'tr.npz')!r}); out = {{}}\n"
            "for i, nf in enumerate(d['nf']):\n"
            "    tr = cs.Trace(int(nf)); tr.cusan_trace_append_events(d[f'ev{i}'])\n"
            "    out[f'img{i}'] = cs.Clocks.compute(tr).to_bytes()\n"
            f"np.savez({str(tmp_path / 'img.npz')!r}, **out)\n")
    env = dict(os.environ, CUSAN_A1_COLUMNS="1", CUSAN_PLAN_THREADS="4")
    subprocess.run([sys.executable, "-c", code], check=True, env=env)
    col = np.load(tmp_path / "img.npz")
    for i, (nf, ev) in enumerate(traces):
        tr = cs.Trace(nf)
        tr.cusan_trace_append_events(ev)
        assert np.array_equal(cs.Clocks.compute(tr).to_bytes(), col[f"img{i}"]), i
