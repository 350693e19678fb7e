"""Timeline of pipelined_checks (dev aid): when each step's lowering, planning and GPU run start and
end, to see whether the host stages overlap the GPU stage.

    python tools/e2e_timeline.py [--config 5] [--steps 8] [--reps 3]
"""
import argparse
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--steps", type=int, default=8)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--window", type=int, default=4096)
ap.add_argument("--summary", action="store_true", help="only the mean steady-state step (steps 2..)")
a = ap.parse_args()

w = configs.make(a.config, "full")
ops, args = w.arrays(True)
log = []
lock = threading.Lock()
T0 = [0.0]


def rec(what, i, t0, t1):
    with lock:
        log.append((what, i, 1e3 * (t0 - T0[0]), 1e3 * (t1 - T0[0])))


def make(i):
    t0 = time.perf_counter()
    t = cs.Trace(255)
    cs.Lowering(t).cusan_lower_program(ops, args)
    rec("lower", i, t0, time.perf_counter())
    return t


Orig = cs.Plan
counter = {"plan": 0, "run": 0}


class Timed(Orig):
    def __init__(self, *p, **k):
        t0 = time.perf_counter()
        super().__init__(*p, **k)
        rec("plan", counter["plan"], t0, time.perf_counter())
        counter["plan"] += 1

    def run(self):
        t0 = time.perf_counter()
        r = super().run()
        rec("run", counter["run"], t0, time.perf_counter())
        counter["run"] += 1
        return r


cs.Plan = Timed
stream = torch.cuda.current_stream()
for rep in range(a.reps):
    log.clear()
    counter.update(plan=0, run=0)
    torch.cuda.synchronize()
    T0[0] = time.perf_counter()
    ends = []
    for tr, r in cs.pipelined_checks(make, a.steps, window_events=a.window, stream=stream.cuda_stream):
        ends.append(1e3 * (time.perf_counter() - T0[0]))
    steps = [round(b - x, 2) for x, b in zip([0.0] + ends[:-1], ends)]
    if a.summary:
        st = steps[2:]
        print(f"config {a.config} rep {rep}: mean step {sum(st) / len(st):.2f} ms (min {min(st):.2f}, max "
              f"{max(st):.2f}), kernel {r.counters['kernel_ms']:.2f} ms")
        continue
    print(f"rep {rep}: step ms {steps}  kernel {r.counters['kernel_ms']:.1f} ms")
    for what, i, s, e in sorted(log, key=lambda x: x[2]):
        print(f"   {what:5s} {i:2d}  {s:8.1f} -> {e:8.1f}  ({e - s:6.1f} ms)")
