"""Host-only timing of lowering (a0) and clocks (a1, cusan_clocks_compute) of a full config
(development aid; no GPU needed), 5 repetitions:

    CUSAN_DEBUG_TIMING=1 python tools/a1_timing.py [config]
    CUSAN_A1_COLUMNS=1 python tools/a1_timing.py      # a1's two-pass column form instead
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

c = int(sys.argv[1]) if len(sys.argv) > 1 else 5
w = configs.make(c, "full")
ops, args = w.arrays(True)
for _ in range(5):
    t0 = time.perf_counter()
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    t1 = time.perf_counter()
    cs.Clocks.compute(tr)
    t2 = time.perf_counter()
    print(f"config {c}: lower {1e3 * (t1 - t0):.2f} ms, clocks {1e3 * (t2 - t1):.2f} ms", flush=True)
