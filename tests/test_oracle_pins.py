"""Pins for the oracle (oracle/): paper listings, brute-force graph HB, invariants, closed forms.

None of these compare the oracle with itself: expected values come from the paper's stated
classifications (tests/golden/listings.txt), from an explicit-graph transitive closure (tests/brute.py)
or from the mathematics of the definitions (subset / emptiness / relabelling / sync insertion).
"""
from __future__ import annotations

import hashlib
import os

import numpy as np
import pytest

import oracle
from oracle.lower import Lowering, lower
from tracegen import configs, fuzz
from tracegen.program import (EVENT_DTYPE, EV_ACCESS, EV_ACQUIRE, EV_FORK, EV_RELEASE, OP_DTYPE,
                              OP_KERNEL, OP_MEMCPY, OP_MEMCPY_ASYNC, OP_MEMSET, OP_MEMSET_ASYNC)

import brute
import listing_dsl


def oracle_lower_with_offsets(ops, args):
    L = Lowering()
    first = []
    for op in np.asarray(ops, OP_DTYPE):
        first.append(len(L.ev))
        L.call(op, args)
    return L.events(), L.next_fiber, first


# ------------------------------------------------------------------------------------------------
# paper listings (racy / fixed pairs with the paper's classification)
# ------------------------------------------------------------------------------------------------
LISTINGS = listing_dsl.parse()


@pytest.mark.parametrize("lst", LISTINGS, ids=[l.name for l in LISTINGS])
def test_listing_classification(lst):
    ops, args = lst.program.arrays()
    ev, nf, first = oracle_lower_with_offsets(ops, args)
    rep = oracle.check_events(ev, nf, threads=1)
    labels = listing_dsl.label_events(lst, ev, first)
    got = listing_dsl.observed_pairs(rep["runs"], labels)
    want = {(a, b): n for a, b, n in lst.expect}
    assert set(got) == set(want), (lst.name, got, want)
    for k, n in want.items():
        if n is not None:
            assert got[k] == n, (lst.name, k, got[k], n)
    # and the brute-force graph checker agrees on the full triple set
    assert brute.runs_to_triples(rep["runs"]) == brute.per_fiber_race_set(ev)


def test_listing_pairs_are_paired():
    names = {l.name for l in LISTINGS}
    for n in names:
        if n.endswith("_racy"):
            assert n[:-5] + "_fixed" in names


# ------------------------------------------------------------------------------------------------
# brute force on tiny random traces
# ------------------------------------------------------------------------------------------------
def _fuzz_cases(n, seed, **kw):
    rng = np.random.default_rng(seed)
    for _ in range(n):
        ne = int(rng.integers(2, 64))
        nf = int(rng.integers(2, 6))
        yield fuzz.random_primitive_trace(rng, ne, nf, n_keys=int(rng.integers(1, 4)),
                                          n_granules=int(rng.integers(1, 17)), **kw), nf


@pytest.mark.parametrize("seed", range(6))
def test_oracle_equals_graph_hb_bruteforce(seed):
    """RS(oracle, vector clocks) == RS(per-fiber definition over explicit-graph HB)."""
    for ev, nf in _fuzz_cases(60, 100 + seed, unaligned=bool(seed % 2)):
        rep = oracle.check_events(ev, nf, threads=1 + seed % 3)
        got = brute.runs_to_triples(rep["runs"])
        reach = brute.hb_closure(ev)
        want = brute.per_fiber_race_set(ev, reach)
        assert got == want
        assert rep["n_race_granules"] == len(want)
        allp = brute.all_pairs_race_set(ev, reach)
        assert got <= allp                                    # RS ⊆ all racy pairs
        for g in {t[0] for t in allp} | {t[0] for t in got}:  # per-granule emptiness equivalence
            assert any(t[0] == g for t in got) == any(t[0] == g for t in allp)
            first_later = min(t[2] for t in allp if t[0] == g)  # first racy access is reported
            assert any(t[0] == g and t[2] == first_later for t in got)


def test_runs_are_canonical_and_roundtrip():
    for ev, nf in _fuzz_cases(80, 7):
        rep = oracle.check_events(ev, nf, threads=2)
        runs = rep["runs"]
        keys = [(int(r["later"]), int(r["earlier"]), int(r["g_begin"])) for r in runs]
        assert keys == sorted(keys) and len(set(keys)) == len(keys)
        assert rep["n_race_granules"] == int(np.sum(runs["g_end"] - runs["g_begin"]))
        # maximality: no two runs with equal (earlier, later) abut
        for a, b in zip(runs[:-1], runs[1:]):
            if a["later"] == b["later"] and a["earlier"] == b["earlier"]:
                assert a["g_end"] < b["g_begin"]
        # round trip: expand → re-merge gives the same runs
        trip = sorted(brute.runs_to_triples(runs), key=lambda t: (t[2], t[1], t[0]))
        merged = []
        for g, e, l in trip:
            if merged and merged[-1][2] == e and merged[-1][3] == l and merged[-1][1] == g:
                merged[-1][1] += 1
            else:
                merged.append([g, g + 1, e, l])
        assert merged == [[int(r["g_begin"]), int(r["g_end"]), int(r["earlier"]), int(r["later"])]
                          for r in runs]


# ------------------------------------------------------------------------------------------------
# invariants
# ------------------------------------------------------------------------------------------------
def test_fully_synchronised_programs_are_race_free():
    """DeviceSynchronize + completion of every request after each call orders everything."""
    rng = np.random.default_rng(11)
    for _ in range(40):
        # single host thread: concurrent host threads would need joins, not device syncs
        p = fuzz.random_program(rng, int(rng.integers(5, 40)), threads=False)
        ops, args = p.arrays()
        from tracegen.program import Program, OP_MPI_ISEND, OP_MPI_IRECV, OP_MPI_WAIT, OP_MPI_TEST
        q = Program()
        q.args = p.args
        waited = set()
        for op in ops:
            if int(op["op"]) in (OP_MPI_WAIT, OP_MPI_TEST) and int(op["b"]) in waited:
                continue
            q.ops.append(tuple(int(v) for v in op))
            if int(op["op"]) in (OP_MPI_ISEND, OP_MPI_IRECV):
                q.wait(int(op["b"]))
                waited.add(int(op["b"]))
            q.device_sync()
        o2, a2 = q.arrays()
        rep = oracle.check_program(o2, a2, threads=1)
        assert rep["n_race_granules"] == 0 and rep["n_runs"] == 0


def _insert(ev, pos, rows):
    rows = np.array(rows, EVENT_DTYPE)
    return np.concatenate([ev[:pos], rows, ev[pos:]])


def test_sync_insertion_removes_exactly_newly_ordered_candidates():
    rng = np.random.default_rng(5)
    checked = 0
    for ev, nf in _fuzz_cases(150, 23):
        n = len(ev)
        p = int(rng.integers(0, n + 1))
        q = int(rng.integers(p, n + 1))
        f1, f2 = int(rng.integers(nf)), int(rng.integers(nf))
        key = 999_999
        # RELEASE at p, ACQUIRE at q (after the shift): ids ≥ p shift by 1, ids ≥ q (orig) by 2
        ev2 = _insert(ev, q, [(EV_ACQUIRE, 0, 0, f2, key, 0)])
        ev2 = _insert(ev2, p, [(EV_RELEASE, 0, 0, f1, key, 0)])

        def remap(i):
            return i + (1 if i >= p else 0) + (1 if i >= q else 0)

        r1 = brute.runs_to_triples(oracle.check_events(ev, nf, threads=1)["runs"])
        r2 = brute.runs_to_triples(oracle.check_events(ev2, nf, threads=1)["runs"])
        r1m = {(g, remap(a), remap(b)) for g, a, b in r1}
        assert r2 <= r1m
        reach2 = brute.hb_closure(ev2)
        for g, a, b in r1m - r2:
            assert (reach2[a] >> b) & 1          # removed ⇒ newly ordered
        for g, a, b in r2:
            assert not (reach2[a] >> b) & 1      # kept ⇒ still unordered
        checked += len(r1m - r2)
    assert checked > 0


def test_fiber_relabelling_invariance():
    rng = np.random.default_rng(9)
    for ev, nf in _fuzz_cases(40, 31):
        perm = rng.permutation(nf)
        ev2 = ev.copy()
        ev2["fiber"] = perm[ev["fiber"]]
        fork = ev["kind"] == EV_FORK
        ev2["a"][fork] = perm[ev["a"][fork].astype(np.int64)]
        r1 = oracle.check_events(ev, nf, threads=1)
        r2 = oracle.check_events(ev2, nf, threads=1)
        assert np.array_equal(r1["runs"], r2["runs"])


def test_thread_count_invariance_and_sampling():
    w = configs.make(5, "small")
    ops, args = w.arrays(True)
    ev, nf = lower(ops, args)
    r1 = oracle.check_events(ev, nf, threads=1)
    r8 = oracle.check_events(ev, nf, threads=8)
    assert np.array_equal(r1["runs"], r8["runs"]) and r1["n_race_granules"] == r8["n_race_granules"]
    # sampled granules give exactly the full result restricted to the sample
    full = brute.runs_to_triples(r1["runs"])
    gs = sorted({g for g, _, _ in full})
    rng = np.random.default_rng(0)
    acc = ev[ev["kind"] == EV_ACCESS]
    lo, hi = int(acc["a"].min()) >> 3, (int((acc["a"] + acc["b"]).max()) + 7) >> 3
    sample = np.unique(np.concatenate([rng.choice(gs, 200), rng.integers(lo, hi, 200)]).astype(np.uint64))
    rs = oracle.check_events(ev, nf, threads=3, sample=sample)
    sset = set(int(x) for x in sample)
    assert brute.runs_to_triples(rs["runs"]) == {t for t in full if t[0] in sset}


# ------------------------------------------------------------------------------------------------
# closed forms and the paper's counters
# ------------------------------------------------------------------------------------------------
def test_config1_closed_form():
    """Racy listing: exactly one run over the 4 KiB buffer (512 granules), earlier = the compute
    kernel's RW access, later = the MPI_Isend read; the fixed twin is race-free."""
    w = configs.make(1)
    ops, args = w.arrays(True)
    ev, nf, first = oracle_lower_with_offsets(ops, args)
    rep = oracle.check_events(ev, nf)
    assert len(ev) == 14
    assert rep["n_runs"] == 1 and rep["n_race_granules"] == 512
    r = rep["runs"][0]
    d = w.meta["buffer"]
    assert int(r["g_begin"]) == d >> 3 and int(r["g_end"]) == (d + 4096) >> 3
    e, l = ev[int(r["earlier"])], ev[int(r["later"])]
    assert (int(e["kind"]), int(e["mode"]), int(e["fiber"])) == (EV_ACCESS, 1, 2)   # kernel on s
    assert (int(l["kind"]), int(l["mode"]), int(l["fiber"])) == (EV_ACCESS, 0, 3)   # MPI fiber
    ops, args = w.arrays(False)
    ev, nf = lower(ops, args)
    assert len(ev) == 15
    assert oracle.check_events(ev, nf)["n_race_granules"] == 0


def test_table1_release_identity():
    """Table I: HappensBefore = kernels + memcpys + memsets (1200+602+2=1804);
    our lowering emits exactly one stream-key release per kernel / memcpy / memset."""
    for c in (2, 3):
        w = configs.make(c, "small")
        ops, args = w.arrays(False)
        ev, _ = lower(ops, args)
        n_ops = int(np.isin(ops["op"], [OP_KERNEL, OP_MEMCPY, OP_MEMCPY_ASYNC, OP_MEMSET,
                                        OP_MEMSET_ASYNC]).sum())
        stream_rel = int(((ev["kind"] == EV_RELEASE) & ((ev["a"] >> np.uint64(56)) == 1)).sum())
        assert stream_rel == n_ops


@pytest.mark.parametrize("c", [2, 3, 4, 5])
def test_small_configs_clean_and_racy(c):
    w = configs.make(c, "small")
    ops, args = w.arrays(False)
    rep = oracle.check_program(ops, args)
    assert rep["n_race_granules"] == 0
    acc = rep["events"][rep["events"]["kind"] == EV_ACCESS]
    assert rep["tracked_bytes"] == int(np.sum(((acc["a"] + acc["b"] + np.uint64(7)) >> np.uint64(3))
                                              - (acc["a"] >> np.uint64(3)))) * 8
    ops, args = w.arrays(True)
    rep = oracle.check_program(ops, args)
    assert rep["n_race_granules"] > 0


def _listing_failures(mutate):
    """Number of listings whose paper classification a mutated lowering gets wrong."""
    bad = 0
    for lst in LISTINGS:
        ops, args = lst.program.arrays()
        L = Lowering()
        mutate(L)
        first = []
        for op in np.asarray(ops, OP_DTYPE):
            first.append(len(L.ev))
            L.call(op, args)
        ev = L.events()
        rep = oracle.check_events(ev, L.next_fiber, threads=1)
        got = set(listing_dsl.observed_pairs(rep["runs"], listing_dsl.label_events(lst, ev, first)))
        bad += got != {(a, b) for a, b, _ in lst.expect}
    return bad


def test_listings_reject_counterfactual_readings():
    """without the issue edge (FORK H→stream), or with a stream→host edge on return,
    or without the legacy default-stream barriers, some paper listing is misclassified."""
    def no_fork(L):
        L.fork = lambda src, dst: None

    def back_edge(L):
        orig = L.epilogue

        def epi(f):
            orig(f)
            L.acquire(0, (1 << 56) | f)
        L.epilogue = epi

    def no_legacy(L):
        L.prologue = lambda f: L.fork(0, f)

    assert _listing_failures(no_fork) > 0
    assert _listing_failures(back_edge) > 0
    assert _listing_failures(no_legacy) > 0


# ------------------------------------------------------------------------------------------------
# full-size goldens (tests/golden/full, written by tools/oracle_full_reports.py from oracle/ only)
# ------------------------------------------------------------------------------------------------
def test_hb_graph_equals_closure():
    """brute.HBGraph (pairwise search, any trace length) == brute.hb_closure on tiny traces."""
    rng = np.random.default_rng(9)
    for _ in range(200):
        nf = int(rng.integers(2, 6))
        ev = fuzz.random_primitive_trace(rng, int(rng.integers(2, 50)), nf, n_keys=3, n_granules=16)
        reach = brute.hb_closure(ev)
        g = brute.HBGraph(ev)
        for a in range(len(ev)):
            for b in range(a + 1, len(ev)):
                assert g.hb(a, b) == bool((reach[a] >> b) & 1)


FULL_GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "full")


@pytest.mark.parametrize("twin", ["racy", "clean"])
@pytest.mark.parametrize("c", [1, 2, 3, 4, 5])
def test_full_size_golden_reports(c, twin):
    """The stored full-size oracle reports belong to today's generators (hash of the oracle's own
    lowering of the full-size program) and every reported race is one by the paper's definition,
    checked without vector clocks: earlier < later are accesses of different fibers, at least one a
    write, both covering the whole run, and not ordered in the explicit HB graph.
    Runs are canonical and maximal; the race-granule count is their total length; clean twins ∅."""
    g = np.load(os.path.join(FULL_GOLDEN, f"config{c}_{twin}.npz"))
    w = configs.make(c, "full")
    ops, args = w.arrays(twin == "racy")
    ev, nf = lower(ops, args)
    assert hashlib.sha256(np.ascontiguousarray(ev).tobytes()).hexdigest() == str(g["events_sha256"])
    assert int(g["n_events"]) == len(ev) and int(g["max_fibers"]) == nf
    acc = ev[ev["kind"] == EV_ACCESS]
    assert int(g["tracked_bytes"]) == 8 * int(np.sum(((acc["a"] + acc["b"] + np.uint64(7)) >> np.uint64(3))
                                                     - (acc["a"] >> np.uint64(3))))
    runs = g["runs"]
    assert len(runs) == int(g["n_runs"])
    assert int(np.sum(runs["g_end"] - runs["g_begin"])) == int(g["n_race_granules"])
    if twin == "clean":
        assert len(runs) == 0
        return
    assert len(runs) > 0
    if c == 1:
        assert len(runs) == 1 and int(g["n_race_granules"]) == 512     # closed form
    keys = [(int(r["later"]), int(r["earlier"]), int(r["g_begin"])) for r in runs]
    assert keys == sorted(keys) and len(set(keys)) == len(keys)
    for r0, r1 in zip(runs[:-1], runs[1:]):                         # maximal: no two runs abut
        assert not (r0["later"] == r1["later"] and r0["earlier"] == r1["earlier"] and r0["g_end"] == r1["g_begin"])
    graph = brute.HBGraph(ev)
    for e, l in sorted({(int(r["earlier"]), int(r["later"])) for r in runs}):
        a, b = ev[e], ev[l]
        assert e < l and int(a["kind"]) == int(b["kind"]) == EV_ACCESS
        assert int(a["fiber"]) != int(b["fiber"]) and (int(a["mode"]) == 1 or int(b["mode"]) == 1)
        assert not graph.hb(e, l)
    for r in runs:
        for x in (ev[int(r["earlier"])], ev[int(r["later"])]):
            assert int(x["a"]) >> 3 <= int(r["g_begin"]) and int(r["g_end"]) <= (int(x["a"]) + int(x["b"]) + 7) >> 3


# ------------------------------------------------------------------------------------------------
# lowering mutants: each plausible misreading of a sync rule in oracle/lower.py must turn some
# paper listing red (the listings pin the oracle's lowering, not only its equality with the product)
# ------------------------------------------------------------------------------------------------
_LOWER_MUTANTS = {
    # M1: cudaMemcpyAsync H2D/D2H made host-synchronous
    "memcpy_async_host_sync": ("if kind == OP_MEMCPY and x in (CPY_H2H, CPY_H2D, CPY_D2H):",
                               "if x in (CPY_H2H, CPY_H2D, CPY_D2H):"),
    # M2: a failed MPI_Test treated as completion (Fig. 1)
    "mpi_test_fail_completes": ("if kind == OP_MPI_WAIT or x:", "if True:"),
    # M3: cudaMemsetAsync on pinned memory made host-synchronous (PAPER.md:438-440 vs 463-466)
    "memset_async_pinned_sync": ("if kind == OP_MEMSET and al is not None and al[2] == MEM_PINNED:",
                                 "if al is not None and al[2] == MEM_PINNED:"),
    # reading ★A6: H2H cudaMemcpy left asynchronous
    "memcpy_h2h_async": ("x in (CPY_H2H, CPY_H2D, CPY_D2H)", "x in (CPY_H2D, CPY_D2H)"),
    # D2D made host-synchronous (only H2D / D2H / H2H block the host)
    "memcpy_d2d_sync": ("x in (CPY_H2H, CPY_H2D, CPY_D2H)", "True"),
    # synchronous cudaMemset on pinned memory left asynchronous
    "memset_pinned_async": ("if kind == OP_MEMSET and al is not None and al[2] == MEM_PINNED:", "if False:"),
    # a failed cudaStreamQuery treated as a sync (A9)
    "stream_query_fail_syncs": ("if x:                                          # only a successful",
                                "if True:                                       # only a successful"),
    # event re-record joins instead of replacing (A4)
    "event_record_joins": ("self.release_store(f, K_event(c))", "self.release(f, K_event(c))"),
    # cudaFree keeping the freed allocation registered (★A25)
    "free_keeps_allocation": ("if a in self.alloc:", "if False:"),
    # cudaFree without its device-wide sync (A8)
    "free_no_sync": ("self.sync_device_host()                      # PAPER.md:448-450", "pass  #"),
    # cudaStreamSynchronize(S0) not covering the blocking streams (A5)
    "s0_sync_skips_blocking": ("""        self.acquire(self.H, K_stream(f))
        if f == S0:
            for u in self.blocking_user:
                self.acquire(self.H, K_stream(u))""", """        self.acquire(self.H, K_stream(f))"""),
    # an operation on S0 not waiting for the blocking streams (Fig. 3, A5)
    "s0_op_skips_blocking": ("""        if f == S0:
            for u in self.blocking_user:
                self.acquire(S0, K_stream(u))""", ""),
    # an operation on a blocking stream not waiting for S0 (Fig. 3, A5)
    "blocking_op_skips_s0": ("""        if f in self.blocking_user:
            self.acquire(f, K_stream(S0))""", ""),
    # cudaDeviceSynchronize covering only the default stream
    "device_sync_only_s0": ("        for f in self.all_streams:\n            self.acquire(self.H, K_stream(f))",
                            "        for f in [S0]:\n            self.acquire(self.H, K_stream(f))"),
    # a kernel without its release on the stream (AnnotateHappensBefore)
    "kernel_no_release": ("""                self.access(f, mode, al[0], al[1])         # whole allocation (PAPER.md:652-654)
            self.epilogue(f)""", """                self.access(f, mode, al[0], al[1])         # whole allocation (PAPER.md:652-654)"""),
    # a read-write kernel argument annotated as a read (A10)
    "rw_arg_as_read": ("mode = READ if int(args[j][\"mode\"]) == MODE_R else WRITE",
                       "mode = WRITE if int(args[j][\"mode\"]) == 1 else READ"),
    # cudaMemcpy's destination annotated as read
    "memcpy_dst_read": ("                self.access(f, WRITE, a, c)\n            if self.tracked_range(b, c):",
                        "                self.access(f, READ, a, c)\n            if self.tracked_range(b, c):"),
    # MPI_Isend's buffer annotated as written (MPI_Isend reads it)
    "isend_writes": ("READ if kind == OP_MPI_ISEND else WRITE", "WRITE"),
    # a non-blocking MPI call without its issue edge from the host (A3)
    "mpi_no_issue_edge": ("self.fork(self.H, m)                            # PAPER.md:211-218,615-619", "pass"),
    # a joined thread's work not ordered before the join's return
    "join_no_acquire": ("self.acquire(self.H, K_thread(a))                  # ... HB the join's return", "pass"),
    # the per-thread default stream treated as non-blocking
    "ptds_nonblocking": ("            self.all_streams.append(f)\n            self.blocking_user.append(f)\n        return self.ptds[t]",
                         "            self.all_streams.append(f)\n        return self.ptds[t]"),
}


def _mutant_lowering(name):
    import importlib.util
    import oracle.lower as ol
    old, new = _LOWER_MUTANTS[name]
    src = open(ol.__file__).read()
    assert src.count(old) == 1, (name, "mutation site not found exactly once")
    spec = importlib.util.spec_from_loader(f"oracle_lower_{name}", loader=None)
    mod = importlib.util.module_from_spec(spec)
    exec(compile(src.replace(old, new), ol.__file__, "exec"), mod.__dict__)
    return mod.Lowering


@pytest.mark.parametrize("name", sorted(_LOWER_MUTANTS))
def test_listings_kill_lowering_mutants(name):
    """A lowering with one sync rule misread misclassifies at least one paper listing."""
    MutLowering = _mutant_lowering(name)
    bad = []
    for lst in LISTINGS:
        ops, args = lst.program.arrays()
        L = MutLowering()
        first = []
        for op in np.asarray(ops, OP_DTYPE):
            first.append(len(L.ev))
            L.call(op, args)
        ev = L.events()
        rep = oracle.check_events(ev, L.next_fiber, threads=1)
        got = set(listing_dsl.observed_pairs(rep["runs"], listing_dsl.label_events(lst, ev, first)))
        if got != {(a, b) for a, b, _ in lst.expect}:
            bad.append(lst.name)
    assert bad, f"mutant {name} passes every paper listing"


# ------------------------------------------------------------------------------------------------
# traces longer than 2^24 events (sessions renumber their epochs; the oracle numbers events by
# trace position in 32 bits): closed forms
# ------------------------------------------------------------------------------------------------
def test_oracle_beyond_2_24_events():
    """Event ids past 2^24 keep their trace positions.  Fiber 0 writes X (event 0); 2^24 + 5
    releases by fiber 2 follow; fiber 1 writes X unsynchronised (w1), fiber 0 writes Y (wy, an id
    past 2^24) and releases key 3, fiber 1 reads Y (ry).  Closed form: runs
    (0 -> w1) over X and (wy -> ry) over Y; when fiber 1 acquires key 3 before reading Y, only
    (0 -> w1)."""
    from tracegen.program import EV_ACQUIRE, EV_RELEASE
    n_fill = (1 << 24) + 5
    X, Y, nx, ny = 1 << 30, 1 << 31, 64, 40
    head = [(EV_ACCESS, 1, 0, X, 8 * nx), (EV_RELEASE, 0, 0, 1, 0)]
    for racy in (True, False):
        tail = [(EV_ACCESS, 1, 1, X, 8 * nx), (EV_ACCESS, 1, 0, Y, 8 * ny), (EV_RELEASE, 0, 0, 3, 0)]
        if not racy:
            tail.append((EV_ACQUIRE, 0, 1, 3, 0))
        tail.append((EV_ACCESS, 0, 1, Y, 8 * ny))
        ev = np.zeros(len(head) + n_fill + len(tail), EVENT_DTYPE)
        ev["kind"][len(head):len(head) + n_fill] = EV_RELEASE
        ev["fiber"][len(head):len(head) + n_fill] = 2
        ev["a"][len(head):len(head) + n_fill] = 7
        for i, (k, m, f, a, b) in enumerate(head):
            ev[i]["kind"], ev[i]["mode"], ev[i]["fiber"], ev[i]["a"], ev[i]["b"] = k, m, f, a, b
        base = len(head) + n_fill
        for i, (k, m, f, a, b) in enumerate(tail):
            ev[base + i]["kind"], ev[base + i]["mode"], ev[base + i]["fiber"], ev[base + i]["a"], ev[base + i]["b"] = \
                k, m, f, a, b
        rep = oracle.check_events(ev, 3, threads=2)
        w1, wy, ry = base, base + 1, len(ev) - 1
        want = [(X >> 3, (X >> 3) + nx, 0, w1)] + ([(Y >> 3, (Y >> 3) + ny, wy, ry)] if racy else [])
        got = [tuple(int(x) for x in r) for r in rep["runs"]]
        assert got == want, (racy, got, want)
        assert ry > (1 << 24)


# ------------------------------------------------------------------------------------------------
# checker mutants: each plausible mistake in oracle/oracle.c (vector clocks, the HB test, the
# per-granule race rule, granule rounding, run canonicalisation) must fail a pin — the brute-force
# graph-HB race set, the paper listings or a closed form — so the checker is pinned by more than
# its agreement with the product
# ------------------------------------------------------------------------------------------------
# (Two edits that look like mistakes are equivalent for the race set and so cannot be pinned:
#  `i+1 < VC(b)[g]` for `<=` — every event that hands a fiber's clock on (a release, a fork) ticks
#  past the accesses before it, so VC(b)[g] never equals an earlier access's i+1 — and a FORK
#  ticking its destination instead of its source, for the same reason.)
_CHECKER_MUTANTS = {
    # HB test reads the later access's own column (a →hb b ⇔ i+1 <= VC(b)[g(a)])
    "hb_wrong_column": ("return acc_event[a] + 1 <= acc_vc[b * F + g];",
                        "return acc_event[a] + 1 <= acc_vc[b * F + acc_fiber[b]];"),
    # FORK hands over only the source's own entry (no transitivity)
    "fork_not_transitive": ("if (Cs[t] > Cf[t]) Cf[t] = Cs[t];", "if (t == s && Cs[t] > Cf[t]) Cf[t] = Cs[t];"),
    # FORK joins dst into src
    "fork_joins_backwards": ("if (Cs[t] > Cf[t]) Cf[t] = Cs[t];", "if (Cf[t] > Cs[t]) Cs[t] = Cf[t];"),
    # RELEASE overwrites the key clock (AnnotateHappensBefore joins)
    "release_stores": ("                if (Cf[t] > S[t]) S[t] = Cf[t];", "                S[t] = Cf[t];"),
    # RELEASE_STORE joins (event re-record, A4)
    "release_store_joins": ("memcpy(S, Cf, F * sizeof(uint32_t));",
                            "for (uint32_t t = 0; t < F; t++) if (Cf[t] > S[t]) S[t] = Cf[t];"),
    # ACQUIRE overwrites the fiber clock instead of joining
    "acquire_overwrites": ("if (S[t] > Cf[t]) Cf[t] = S[t];", "Cf[t] = S[t];"),
    # reads are not checked against the last write (every access is)
    "reads_skip_w_check": ("if (wv && !hb(wv - 1, b))", "if (wv && acc_write[b] && !hb(wv - 1, b))"),
    # a write is not checked against the reads since the last write
    "write_skips_reads": ("if (!hb(rv - 1, b)) {", "if (0 && !hb(rv - 1, b)) {"),
    # the read set is not emptied by a write
    "reads_survive_write": ("                    Rg[tf] = 0;\n", ""),
    # a write does not become the last write
    "w_not_updated": ("w->W[x] = (uint32_t)(b + 1);", "(void)0;"),
    # a fiber's first read since the write kept instead of its last
    "first_read_kept": ("Rg[f] = (uint32_t)(b + 1);", "if (!Rg[f]) Rg[f] = (uint32_t)(b + 1);"),
    # partial last granule dropped ([addr>>3, (addr+n+7)>>3))
    "granule_end_truncated": ("g1 = (e->a + e->b + 7) >> 3;", "g1 = (e->a + e->b) >> 3;"),
    # partial first granule dropped
    "granule_begin_rounded_up": ("uint64_t g0 = e->a >> 3,", "uint64_t g0 = (e->a + 7) >> 3,"),
    # sync keys share one clock (the key lookup ignores the key)
    "sync_keys_collide": ("while (sc_tab[h].used && sc_tab[h].key != key)", "while (0)"),
    # run merge ignores the earlier access
    "run_merge_ignores_earlier": ("tv->t[j].later == r.later && tv->t[j].earlier == r.earlier &&",
                                  "tv->t[j].later == r.later &&"),
    # canonical order (later, earlier, g_begin) swapped to (earlier, later, ...)
    "run_order_swapped": ("    if (a->later != b->later) return a->later < b->later ? -1 : 1;\n"
                          "    if (a->earlier != b->earlier) return a->earlier < b->earlier ? -1 : 1;\n"
                          "    return (a->g_begin",
                          "    if (a->earlier != b->earlier) return a->earlier < b->earlier ? -1 : 1;\n"
                          "    if (a->later != b->later) return a->later < b->later ? -1 : 1;\n"
                          "    return (a->g_begin"),
    # runs cut at tile boundaries are not stitched
    "tiles_not_stitched": ("all.r[m - 1].g_end == all.r[i].g_begin)", "all.r[m - 1].g_end == all.r[i].g_begin && 0)"),
    # runs stitched across a gap
    "runs_stitched_across_gaps": ("all.r[m - 1].g_end == all.r[i].g_begin)", "1)"),
}


def _pin_battery():
    """The pins a checker must pass (first failure raised): brute-force graph HB on tiny random
    traces (aligned and unaligned), canonical runs, every paper listing, and a closed form across
    tiles (two unordered writes over 150,000 granules: one run)."""
    for seed in (100, 101):
        for ev, nf in _fuzz_cases(40, seed, unaligned=bool(seed % 2)):
            rep = oracle.check_events(ev, nf, threads=1)
            got = brute.runs_to_triples(rep["runs"])
            assert got == brute.per_fiber_race_set(ev, brute.hb_closure(ev))
            assert rep["n_race_granules"] == len(got)
            keys = [(int(r["later"]), int(r["earlier"]), int(r["g_begin"])) for r in rep["runs"]]
            assert keys == sorted(keys)
            for a, b in zip(rep["runs"][:-1], rep["runs"][1:]):
                if a["later"] == b["later"] and a["earlier"] == b["earlier"]:
                    assert a["g_end"] < b["g_begin"]
    for lst in LISTINGS:
        ops, args = lst.program.arrays()
        ev, nf, first = oracle_lower_with_offsets(ops, args)
        rep = oracle.check_events(ev, nf, threads=1)
        got = set(listing_dsl.observed_pairs(rep["runs"], listing_dsl.label_events(lst, ev, first)))
        assert got == {(a, b) for a, b, _ in lst.expect}, lst.name
    n = 150_000                                       # > 2 tiles of 65,536 granules, two workers
    ev = np.zeros(2, EVENT_DTYPE)
    ev[0] = (EV_ACCESS, 1, 0, 0, 1 << 30, 8 * n)
    ev[1] = (EV_ACCESS, 1, 0, 1, 1 << 30, 8 * n)
    rep = oracle.check_events(ev, 2, threads=2)
    assert [tuple(int(x) for x in r) for r in rep["runs"]] == [((1 << 30) >> 3, ((1 << 30) >> 3) + n, 0, 1)]


def test_pin_battery_passes_on_the_oracle():
    _pin_battery()


@pytest.mark.parametrize("name", sorted(_CHECKER_MUTANTS))
def test_pins_kill_checker_mutants(name, tmp_path, monkeypatch):
    """oracle.c with one plausible mistake fails the pin battery (or crashes)."""
    import subprocess
    old, new = _CHECKER_MUTANTS[name]
    src = open(os.path.join(os.path.dirname(oracle.__file__), "oracle.c")).read()
    assert src.count(old) == 1, (name, "mutation site not found exactly once")
    (tmp_path / "oracle.c").write_text(src.replace(old, new))
    binary = str(tmp_path / "oracle_bin")
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-pthread", "-w", "-o", binary, str(tmp_path / "oracle.c")])
    monkeypatch.setattr(oracle, "BIN", binary)
    monkeypatch.setattr(oracle, "build", lambda force=False: binary)
    with pytest.raises((AssertionError, subprocess.CalledProcessError)):
        _pin_battery()
