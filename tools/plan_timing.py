"""Host / device planning time of one cusan_plan_create (development aid): per-phase times from
CUSAN_DEBUG_TIMING for a full config, device (default) and host a2.

    CUSAN_DEBUG_TIMING=1 python tools/plan_timing.py --config 5
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--window", type=int, default=4096)
a = ap.parse_args()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)
tr = cs.Trace(255)
cs.Lowering(tr).cusan_lower_program(ops, args)
for name, flags in (("device a2", 0), ("host a2", cs.CUSAN_CHECK_HOST_PLAN)):
    for r in range(a.reps):
        t0 = time.perf_counter()
        p = cs.Plan(tr, window_events=a.window, flags=flags | cs.CUSAN_CHECK_DEFER_WORKSPACE)
        t1 = time.perf_counter()
        p.close()
        print(f"{name} rep {r}: plan_create {1e3 * (t1 - t0):.3f} ms", file=sys.stderr, flush=True)
