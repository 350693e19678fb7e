"""Median kernel / run time of the default (interval-compressed) one-shot check of full configs, the
racy twins, 4096-access windows (development aid for K1 A/B runs via CUSAN_LIBRARY).

    python tools/compressed_timing.py 3,5
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

for c in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "5").split(",")]:
    w = configs.make(c, "full")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    plan = cs.Plan(tr, window_events=4096)
    ks, rs = [], []
    for i in range(40):
        r = plan.run()
        if i >= 5:
            ks.append(r.counters["kernel_ms"])
            rs.append(r.counters["run_ms"])
    plan.close()
    print(f"{os.path.basename(os.environ.get('CUSAN_LIBRARY', 'current'))} config {c}: kernel median "
          f"{statistics.median(ks):.4f} ms (min {min(ks):.4f}), run median {statistics.median(rs):.4f} ms, "
          f"{r.n_race_granules} race granules", flush=True)
