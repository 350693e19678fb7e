"""A/B timing of cusan_clocks_compute (a1) for a full config (development aid): median of N runs;
run with CUSAN_LIBRARY=<variant> to compare builds."""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

c = int(sys.argv[1]) if len(sys.argv) > 1 else 5
w = configs.make(c, "full")
ops, args = w.arrays(True)
tr = cs.Trace(255)
cs.Lowering(tr).cusan_lower_program(ops, args)
ts, ps = [], []
for i in range(25):
    t0 = time.perf_counter()
    ck = cs.Clocks.compute(tr)
    t1 = time.perf_counter()
    p = cs.Plan(ck, window_events=4096, flags=cs.CUSAN_CHECK_DEFER_WORKSPACE | cs.CUSAN_CHECK_DEVICE_PLAN)
    t2 = time.perf_counter()
    p.close()
    if i >= 5:
        ts.append(1e3 * (t1 - t0))
        ps.append(1e3 * (t2 - t1))
print(f"{os.environ.get('CUSAN_LIBRARY', 'current')}: clocks median {statistics.median(ts):.3f} ms "
      f"(min {min(ts):.3f}), plan from clocks median {statistics.median(ps):.3f} ms")
