"""Short driver for ncu captures of the shadow-check kernel (profiling aid, not a bench).

Runs the bench workload's plan on one shard (default 1 of 8, so ncu's replay save/restore of the
shadow fits next to it) for `--runs` plan runs after one warm-up run.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--nshards", type=int, default=8)
ap.add_argument("--shard", type=int, default=0)
ap.add_argument("--window", type=int, default=4096)
ap.add_argument("--runs", type=int, default=1)
ap.add_argument("--compressed", action="store_true", help="the interval-compressed shadow (default: dense)")
a = ap.parse_args()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)
tr = cs.Trace(255)
cs.Lowering(tr).cusan_lower_program(ops, args)
plan = cs.Plan(tr, window_events=a.window, nshards=a.nshards, shard=a.shard,
               flags=0 if a.compressed else cs.CUSAN_CHECK_DENSE_SHADOW)
for i in range(1 + a.runs):
    r = plan.run()
    c = r.counters
    print(f"run {i}: kernel {c['kernel_ms']:.2f} ms, {c['kernel_launches']} launches, "
          f"cell bytes {c['shadow_cell_bytes'] / 1e9:.2f} GB -> {c['shadow_cell_bytes'] / c['kernel_ms'] / 1e6:.0f} GB/s, "
          f"races {r.n_race_granules}", flush=True)
plan.close()
