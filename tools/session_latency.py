"""Per-call latency of an online session (f1), split into the library's phases.

    CUSAN_DEBUG_TIMING=1 python tools/session_latency.py --config 5 --chunk 8 --calls 300 2> ticks.log

Feeds the full-size racy trace to one session, `--chunk` accesses per call, and prints one JSON
line: per-call medians of the Python-level call time, the library's own time from plan start to
report (`run_ms`), the kernel time, and — when CUSAN_DEBUG_TIMING is set — the medians of the
library's phase ticks read back from stderr (`--ticks FILE`).
"""
import argparse
import json
import os
import re
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--size", default="full")
ap.add_argument("--chunk", type=int, default=8)
ap.add_argument("--calls", type=int, default=300)
ap.add_argument("--skip", type=int, default=20, help="calls not counted (warm-up)")
ap.add_argument("--dense", action="store_true")
ap.add_argument("--ticks", default="", help="parse CUSAN_DEBUG_TIMING lines from this file afterwards")
a = ap.parse_args()

w = configs.make(a.config, a.size)
ops, args = w.arrays(True)
full = cs.Trace(255)
cs.Lowering(full).cusan_lower_program(ops, args)
ev = full.cusan_trace_read()
acc_pos = np.flatnonzero(ev["kind"] == 0)
cuts = [int(acc_pos[i]) for i in range(a.chunk, len(acc_pos), a.chunk)] + [len(ev)]
cuts = cuts[: a.calls]
# import-time objects out of the cyclic collector's way (a full pass is a ~35 ms pause with torch
# imported: it would dominate runs of a few hundred sub-millisecond calls)
import gc  # noqa: E402
gc.collect()
gc.freeze()

tr = cs.Trace(255)
ses = cs.Session(tr, flags=cs.CUSAN_CHECK_DENSE_SHADOW if a.dense else 0)
py, run, ker, niv = [], [], [], []
start = 0
for i, end in enumerate(cuts):
    tr.cusan_trace_append_events(ev[start:end])
    t0 = time.perf_counter()
    r = ses.check()
    dt = time.perf_counter() - t0
    start = end
    if i < a.skip:
        continue
    c = r.counters
    py.append(1e3 * dt)
    run.append(c["run_ms"])
    ker.append(c["kernel_ms"])
    niv.append(c["n_intervals"])
ses.close()
out = dict(config=a.config, chunk=a.chunk, calls=len(py), dense=a.dense,
           python_call_ms=statistics.median(py), library_run_ms=statistics.median(run),
           kernel_ms=statistics.median(ker), intervals_median=statistics.median(niv), intervals_max=max(niv))
if a.ticks and os.path.exists(a.ticks):
    ph = {}
    for line in open(a.ticks):
        m = re.match(r"(plan_call|cusan_session): (.+?)\s+([0-9.]+) ms", line)
        if m:
            ph.setdefault(f"{m.group(1)}.{m.group(2).strip()}", []).append(float(m.group(3)))
    out["ticks_median_ms"] = {k: statistics.median(v[a.skip:] or v) for k, v in ph.items()}
print(json.dumps(out))
