"""Long randomized parity campaign on the GPU (development aid; results in profiles/).

Every case is a seeded random trace (primitive TSan-level events, or a random CUDA-aware MPI call
program lowered by the product's C lowering and checked against the oracle's own Python lowering)
checked through every mode — one window and small windows, both shadow layouts (interval-compressed,
the default, and dense), host and device planning, plans from (exported / imported) clocks,
whole-node checks (ngpus, shards mapped onto this GPU), granule-range shards (one-shot),
sequential, pipelined and block-cyclic shard sessions, sessions renumbering their event ids every
few calls, sessions forgetting the memory no later access touches — and compared with the oracle bit for bit.

    python tools/fuzz_campaign.py --minutes 20 --seed 1 > profiles/fuzz_campaign_r02.json
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from oracle.lower import lower as oracle_lower  # noqa: E402
from tracegen import fuzz  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--minutes", type=float, default=10.0)
ap.add_argument("--seed", type=int, default=1)
a = ap.parse_args()

rng = np.random.default_rng(a.seed)
stats = {"cases": 0, "checks": 0, "mismatches": 0, "racy_cases": 0, "by_mode": {}, "first_failures": []}
FL, IV = cs.CUSAN_CHECK_DENSE_SHADOW, cs.CUSAN_CHECK_INTERVAL_SHADOW
HP, DP = cs.CUSAN_CHECK_HOST_PLAN, cs.CUSAN_CHECK_DEVICE_PLAN
os.environ["CUSAN_NODE_SHARE_DEVICES"] = "1"          # ngpus > 1 on this one GPU


def same(rep_runs, rep_n, ref):
    return rep_n == ref["n_race_granules"] and np.array_equal(rep_runs, ref["runs"].astype(rep_runs.dtype))


def record(mode, ok, case):
    stats["checks"] += 1
    m = stats["by_mode"].setdefault(mode, [0, 0])
    m[0] += 1
    if not ok:
        m[1] += 1
        stats["mismatches"] += 1
        if len(stats["first_failures"]) < 10:
            stats["first_failures"].append(dict(mode=mode, **case))


def one_case(ev, nf, case):
    ref = oracle.check_events(ev, nf, threads=2)
    stats["racy_cases"] += ref["n_race_granules"] > 0
    tr = cs.Trace(nf)
    tr.cusan_trace_append_events(ev)
    n_acc = int(np.sum(ev["kind"] == 0))
    windows = [0, int(rng.integers(1, 6)), max(1, n_acc // 3)]
    for w in windows:
        for flags in (0, FL, IV):
            plan = int(rng.choice([HP, DP]))
            r = cs.check(tr, window_events=w, flags=flags | plan)
            record(f"oneshot w={'all' if w == 0 else 'small'} flags={flags} {'device' if plan == DP else 'host'} plan",
                   same(r.runs, r.n_race_granules, ref), case)
    ck = cs.Clocks.from_bytes(cs.Clocks.compute(tr).to_bytes())
    flags = int(rng.choice([0, FL])) | int(rng.choice([HP, DP]))
    p = cs.Plan(ck, window_events=int(rng.integers(0, 5)), flags=flags)
    r = p.run()
    p.close()
    record("plan from clocks", same(r.runs, r.n_race_granules, ref), case)
    r = cs.check(tr, ngpus=int(rng.integers(2, 5)), window_events=int(rng.integers(0, 5)), flags=int(rng.choice([0, FL])))
    record("ngpus", same(r.runs, r.n_race_granules, ref), case)
    ns = int(rng.integers(2, 6))
    w = int(rng.integers(0, 5))
    flags = int(rng.choice([0, FL, IV]))          # shards of one check share its options
    parts = [cs.check(tr, window_events=w, nshards=ns, shard=s, flags=flags) for s in range(ns)]
    m = cs.report_merge(np.concatenate([p.runs for p in parts]), sum(p.n_race_granules for p in parts))
    record("oneshot shards", same(m.runs, m.n_race_granules, ref), case)
    # sessions: random cut points, sequential / pipelined / block-cyclic shards
    cuts = sorted({0, len(ev), *rng.integers(1, max(2, len(ev)), int(rng.integers(1, 5))).tolist()})
    # granules no access after position y touches: what "session forget" may release after a call
    acc_i = np.flatnonzero(ev["kind"] == 0)
    g0s = (ev["a"][acc_i] >> 3).astype(np.int64)
    g1s = np.where(ev["b"][acc_i] > 0, (ev["a"][acc_i] + ev["b"][acc_i] + 7) >> 3, ev["a"][acc_i] >> 3).astype(np.int64)
    gbase = int(g0s.min()) if len(acc_i) else 0
    last = np.full(int(g1s.max()) - gbase if len(acc_i) else 0, -1, np.int64)
    for i, a0, a1 in zip(acc_i, g0s, g1s):
        last[a0 - gbase:a1 - gbase] = i
    for mode in ("session", "pipelined", "session shards", "session renumbering", "session forget"):
        flags = int(rng.choice([0, FL, IV]))
        nsh = int(rng.integers(2, 5)) if mode == "session shards" else 1
        blk = int(2 ** rng.integers(3, 9))
        trs = [cs.Trace(nf) for _ in range(nsh)]
        if mode == "session renumbering":          # event-id limit low enough to renumber every few calls
            cuts = sorted({0, len(ev), *range(int(rng.integers(8, 40)), len(ev), int(rng.integers(8, 40)))})
            os.environ["CUSAN_SESSION_EVENT_LIMIT"] = str(max(64, len(ev) // 2))
        ses = [cs.Session(trs[s], window_events=int(rng.integers(0, 4)), flags=flags, nshards=nsh, shard=s,
                          shard_block=blk) for s in range(nsh)]
        os.environ.pop("CUSAN_SESSION_EVENT_LIMIT", None)
        runs, n = [], 0
        try:
            for x, y in zip(cuts[:-1], cuts[1:]):
                for t, se in zip(trs, ses):
                    t.cusan_trace_append_events(ev[x:y])
                    r = se.submit() if mode == "pipelined" else se.check()
                    if r is not None:
                        runs.append(r.runs)
                        n += r.n_race_granules
                    if mode == "session forget":      # released: granules no later access touches
                        dead = (last >= 0) & (last < y)
                        if x > 0:
                            dead &= last >= x          # (earlier ones were forgotten already)
                        edges = np.flatnonzero(np.diff(np.concatenate([[0], dead.astype(np.int8), [0]])))
                        for b, e in zip(edges[::2], edges[1::2]):
                            se.forget(8 * (gbase + int(b)), 8 * int(e - b))
        except cs.CusanError as e:                 # a call or the live ids too large for the lowered limit
            if mode != "session renumbering" or e.status != -2:
                raise
            stats["renumber_limit_too_low"] = stats.get("renumber_limit_too_low", 0) + 1
            for se in ses:
                se.close()
            continue
        for se in ses:
            if mode == "pipelined":
                r = se.finish()
                runs.append(r.runs)
                n += r.n_race_granules
            se.close()
        m = cs.report_merge(np.concatenate(runs) if runs else np.zeros(0, cs.RUN_DTYPE), n)
        record(f"{mode} flags={flags}", same(m.runs, m.n_race_granules, ref), case)


t_end = time.time() + 60 * a.minutes
while time.time() < t_end:
    seed = int(rng.integers(1 << 31))
    r2 = np.random.default_rng(seed)
    if r2.random() < 0.6:
        nf = int(r2.integers(2, 40))
        ev = fuzz.random_primitive_trace(r2, int(r2.integers(5, 300)), nf, n_keys=int(r2.integers(1, 6)),
                                         n_granules=int(r2.integers(10, 20000)), p_access=float(r2.uniform(0.3, 0.9)),
                                         unaligned=bool(r2.random() < 0.3))
        if r2.random() < 0.5:                      # mostly reads: many reader fibers, read-set records
            ev["mode"][(ev["kind"] == 0) & (r2.random(len(ev)) < 0.7)] = 0
        case = dict(kind="primitive", seed=seed)
        one_case(ev, nf, case)
    else:
        prog = fuzz.random_program(r2, int(r2.integers(5, 80)))
        ops, args = prog.arrays()
        tr = cs.Trace(255)
        cs.Lowering(tr).cusan_lower_program(ops, args)
        ev = tr.cusan_trace_read()
        ev_o, nf_o = oracle_lower(ops, args)
        case = dict(kind="program", seed=seed)
        record("lowering", bool(np.array_equal(ev, ev_o)), case)
        one_case(ev, 255, case)
    stats["cases"] += 1
stats["minutes"] = a.minutes
stats["seed"] = a.seed
print(json.dumps(stats))
