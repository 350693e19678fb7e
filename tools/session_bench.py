"""Online-checking throughput (f1): feed a config's trace to a cusan_session in chunks of
`--chunk` accesses and time every session call (host re-planning + layout move + check).

    python tools/session_bench.py --config 5 --chunk 4096
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
ap.add_argument("--size", default="full")
ap.add_argument("--chunk", type=int, default=4096, help="accesses per session call")
ap.add_argument("--window", type=int, default=0)
a = ap.parse_args()

w = configs.make(a.config, a.size)
ops, args = w.arrays(True)
full = cs.Trace(255)
cs.Lowering(full).cusan_lower_program(ops, args)
ev = full.cusan_trace_read()
acc_pos = np.flatnonzero(ev["kind"] == 0)
cuts = [int(acc_pos[i]) for i in range(a.chunk, len(acc_pos), a.chunk)] + [len(ev)]

tr = cs.Trace(255)
ses = cs.Session(tr, window_events=a.window)
start, calls = 0, []
for end in cuts:
    tr.cusan_trace_append_events(ev[start:end])
    t0 = time.perf_counter()
    rep = ses.check()
    dt = time.perf_counter() - t0
    c = rep.counters
    calls.append(dict(events=end - start, seconds=dt, kernel_ms=c["kernel_ms"], tracked=c["tracked_bytes_shard"],
                      cell_bytes=c["shadow_cell_bytes"], races=rep.n_race_granules, launches=c["kernel_launches"]))
    start = end
ses.close()
tot = sum(x["tracked"] for x in calls)
secs = sum(x["seconds"] for x in calls)
kms = sum(x["kernel_ms"] for x in calls)
cell = sum(x["cell_bytes"] for x in calls)
out = dict(config=a.config, chunk_accesses=a.chunk, calls=len(calls), tracked_bytes=tot,
           checked_gbs=tot / secs / 1e9, kernel_checked_gbs=tot / (kms / 1e3) / 1e9,
           kernel_dram_gbs=cell / (kms / 1e3) / 1e9, seconds=secs, kernel_ms=kms,
           race_granules=sum(x["races"] for x in calls), per_call=calls)
print(json.dumps(out))
