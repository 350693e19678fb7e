"""Predicted multi-GPU scaling from one GPU: run every shard of an N-way split one after another,
each on the full device, and compare the slowest shard with the whole check.  Shards share no
state and the only exchange is the run gather, so max over shards (+ gather) is the N-GPU step.

    python tools/shard_scaling.py --config 5 --window 4096
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--window", type=int, default=4096)
ap.add_argument("--ns", default="1,2,4,8")
a = ap.parse_args()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)
tr = cs.Trace(255)
cs.Lowering(tr).cusan_lower_program(ops, args)
out = {"config": a.config, "window": a.window, "n": {}}
t1 = None
ref = None
for n in [int(x) for x in a.ns.split(",")]:
    times, plan_ms, runs, races = [], [], [], 0
    for s in range(n):
        t0 = time.perf_counter()
        p = cs.Plan(tr, nshards=n, shard=s, window_events=a.window, workspace="torch")
        plan_ms.append(1e3 * (time.perf_counter() - t0))
        p.run()
        r = min((p.run() for _ in range(3)), key=lambda r: r.counters["run_ms"])
        times.append(r.counters["run_ms"])
        runs.append(r.runs)
        races += r.n_race_granules
        p.close()
    merged = cs.report_merge(np.concatenate(runs), races)
    if ref is None:
        ref = merged
    assert np.array_equal(merged.runs, ref.runs) and merged.n_race_granules == ref.n_race_granules
    step = max(times)
    if n == 1:
        t1 = step
    out["n"][n] = {"max_shard_ms": step, "min_shard_ms": min(times), "max_plan_create_ms": max(plan_ms), "speedup": t1 / step if t1 else None,
                   "efficiency": t1 / step / n if t1 else None}
    print(n, out["n"][n], flush=True)
print(json.dumps(out))
