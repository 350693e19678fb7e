"""One end-to-end check of a full config through the public API (device planning a2 + the check),
for an ncu launch list of every kernel the step launches (planning kernels of plan_dev.cu, CUB
sorts / scans, K1, the run merge).  Run under ncu; the first check warms up (module loading), the
second is the profiled step.

    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file launches.csv \
        python tools/profile_plan.py --config 5 [--dense]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--window", type=int, default=4096)
ap.add_argument("--dense", action="store_true")
a = ap.parse_args()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)
tr = cs.Trace(255)
cs.Lowering(tr).cusan_lower_program(ops, args)
flags = cs.CUSAN_CHECK_DENSE_SHADOW if a.dense else 0
for i in range(2):
    rep = cs.check(tr, window_events=a.window, flags=flags)
    print(f"check {i}: {rep.n_race_granules} race granules, {rep.n_runs} runs, kernel {rep.counters['kernel_ms']:.3f} ms",
          flush=True)
