"""Per-stage times inside pipelined_checks (development aid): lowering (a0), clocks (a1), plan from
clocks (a2) and the GPU check + report, each measured where it runs (the stages overlap, so the
step time is bounded by the slowest).

    python tools/pipeline_stages.py --config 5 [--dense]
"""
import argparse
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--steps", type=int, default=60)
ap.add_argument("--dense", action="store_true")
ap.add_argument("--host-workers", type=int, default=2)
ap.add_argument("--no-gc", action="store_true", help="Python's cyclic garbage collector off during the run")
a = ap.parse_args()
if a.no_gc:
    import gc
    gc.disable()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)
T = {"lower": [], "clocks": [], "plan": [], "check": []}
LONG = []          # (stage, start, ms) of stage executions over 10 ms


def make_trace(_i):
    t0 = time.perf_counter()
    t = cs.Trace(255)
    cs.Lowering(t).cusan_lower_program(ops, args)
    T["lower"].append(1e3 * (time.perf_counter() - t0))
    if T["lower"][-1] > 10:
        LONG.append(("lower", t0, T["lower"][-1]))
    return t


orig_compute = cs.Clocks.compute.__func__
orig_plan = cs.Plan


def timed_compute(cls, tr):
    t0 = time.perf_counter()
    r = orig_compute(cls, tr)
    T["clocks"].append(1e3 * (time.perf_counter() - t0))
    if T["clocks"][-1] > 10:
        LONG.append(("clocks", t0, T["clocks"][-1]))
    return r


class TimedPlan(orig_plan):
    def __init__(self, *x, **k):
        t0 = time.perf_counter()
        super().__init__(*x, **k)
        T["plan"].append(1e3 * (time.perf_counter() - t0))
        if T["plan"][-1] > 10:
            LONG.append(("plan", t0, T["plan"][-1]))


cs.Clocks.compute = classmethod(timed_compute)
cs.Plan = TimedPlan
flags = cs.CUSAN_CHECK_DENSE_SHADOW if a.dense else 0
t_prev = None
steps = []
for i, (_t, rep) in enumerate(cs.pipelined_checks(make_trace, a.steps, window_events=4096, flags=flags,
                                                          host_workers=a.host_workers, lower_workers=a.host_workers)):
    now = time.perf_counter()
    if t_prev is not None and i >= 5:
        steps.append(1e3 * (now - t_prev))
        if steps[-1] > 10:
            print(f"pipeline_stages: slow step {i}: {steps[-1]:.1f} ms", file=sys.stderr, flush=True)
        T["check"].append(rep.counters["run_ms"])
    t_prev = now
med = {k: round(statistics.median(v[5:] if len(v) > 10 else v), 3) for k, v in T.items()}
q = sorted(steps)
pct = {p: round(q[min(len(q) - 1, int(p / 100 * len(q)))], 3) for p in (50, 90, 99)}
slow = sorted(((x, i) for i, x in enumerate(steps) if x > 5 * pct[50]), reverse=True)[:8]
t_first = LONG[0][1] if LONG else 0.0
if LONG:
    print("pipeline_stages: stage executions over 10 ms (stage, ms):", [(x[0], round(x[2], 1)) for x in LONG],
          file=sys.stderr)
print(f"config {a.config} {'dense' if a.dense else 'compressed'} ({a.host_workers} host workers per stage): step "
      f"{sum(steps) / len(steps):.3f} ms (mean over {len(steps)} steps; p50/p90/p99 {pct[50]}/{pct[90]}/{pct[99]}, "
      f"max {q[-1]:.2f} ms, {sum(1 for x in steps if x > 5 * pct[50])} steps > 5 x p50, slowest (ms, step) "
      f"{[(round(x, 1), i) for x, i in slow]}); stage medians {med}")
