"""Small workloads for compute-sanitizer runs over the library's kernels (both shadow layouts,
windows, the device planner, plans from clocks, whole-node checks, sessions incl. epoch
renumbering, spill records).  Asserts parity with the oracle too."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs, fuzz  # noqa: E402

rng = np.random.default_rng(5)
n = 0
for c in (1, 3, 5):
    w = configs.make(c, "small" if c > 1 else "full")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    ref = oracle.check_events(tr.cusan_trace_read(), 255)
    DP = cs.CUSAN_CHECK_DEVICE_PLAN
    os.environ["CUSAN_NODE_SHARE_DEVICES"] = "1"
    for kw in (dict(), dict(window_events=40), dict(window_events=40, flags=cs.CUSAN_CHECK_DENSE_SHADOW),
               dict(window_events=40, flags=cs.CUSAN_CHECK_INTERVAL_SHADOW), dict(nshards=3, shard=1),
               dict(flags=DP), dict(window_events=40, flags=DP | cs.CUSAN_CHECK_DENSE_SHADOW),
               dict(window_events=40, flags=DP, nshards=3, shard=2), dict(window_events=40, ngpus=3)):
        rep = cs.check(tr, **kw)
        if "nshards" not in kw:
            assert rep.n_race_granules == ref["n_race_granules"], (c, kw)
        n += 1
for _ in range(10):
    nf = int(rng.integers(5, 30))
    ev = fuzz.random_primitive_trace(rng, 120, nf, n_keys=3, n_granules=600, p_access=0.8)
    ev["mode"][(ev["kind"] == 0) & (rng.random(len(ev)) < 0.7)] = 0
    ref = oracle.check_events(ev, nf)
    for flags in (0, cs.CUSAN_CHECK_DENSE_SHADOW, cs.CUSAN_CHECK_INTERVAL_SHADOW):
        tr = cs.Trace(nf)
        ses = cs.Session(tr, window_events=7, flags=flags)
        total = 0
        for a, b in ((0, 40), (40, 90), (90, 120)):
            tr.cusan_trace_append_events(ev[a:b])
            total += ses.check().n_race_granules
            n += 1
        ses.close()
        assert total == ref["n_race_granules"], flags
        os.environ["CUSAN_SESSION_EVENT_LIMIT"] = "80"       # renumber the epochs every call
        tr = cs.Trace(nf)
        ses = cs.Session(tr, window_events=7, flags=flags)
        os.environ.pop("CUSAN_SESSION_EVENT_LIMIT")
        renum = 0
        for a, b in ((0, 30), (30, 60), (60, 90), (90, 120)):
            tr.cusan_trace_append_events(ev[a:b])
            try:
                r = ses.check()
            except cs.CusanError:                           # live ids beyond the lowered limit
                break
            renum = r.counters["renumberings"]
            n += 1
        ses.close()
        # pipelined calls (submit / finish) and a 2-shard block-cyclic session
        for kw in (dict(), dict(nshards=2, shard=0, shard_block=64), dict(nshards=2, shard=1, shard_block=64)):
            tr = cs.Trace(nf)
            ses = cs.Session(tr, window_events=7, flags=flags, **kw)
            for a, b in ((0, 40), (40, 90), (90, 120)):
                tr.cusan_trace_append_events(ev[a:b])
                r = ses.submit()
                total -= r.n_race_granules if r is not None else 0
            total -= ses.finish().n_race_granules
            n += 1
            ses.close()
        assert total == -ref["n_race_granules"], flags       # 1 whole + 1 pipelined + 2 shard halves
print("sanitize workloads ok:", n)
