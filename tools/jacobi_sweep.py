"""Fig. 12-style Jacobi domain sweep: how the check
scales with the tracked domain, per-granule shadow vs interval-compressed shadow (f3).

For each domain nx × ny (config 2's Jacobi halo-exchange program, 100 iterations, racy twin) it
times the same plan three ways on one GPU — per-granule cells in windows of `--window` accesses
(online), per-granule in one window (post-mortem), and interval-compressed cells in the same windows
— and checks that all three report the same races.  Writes JSON lines to stdout.

    python tools/jacobi_sweep.py [--window 512] [--iters 100]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

DOMAINS = [(512, 256), (1024, 512), (2048, 1024), (4096, 2048), (8192, 4096), (16384, 8192)]

ap = argparse.ArgumentParser()
ap.add_argument("--window", type=int, default=512)
ap.add_argument("--iters", type=int, default=100)
ap.add_argument("--reps", type=int, default=5)
a = ap.parse_args()
stream = torch.cuda.Stream()


def timed(tr, **kw):
    p = cs.Plan(tr, workspace="torch", stream=stream.cuda_stream, **kw)
    rep = p.run()                                    # warm-up
    ts, ks = [], []
    for _ in range(a.reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rep = p.run()
        ts.append(time.perf_counter() - t0)
        ks.append(rep.counters["kernel_ms"])
    p.close()
    return rep, min(ts), min(ks)


for nx, ny in DOMAINS:
    w = configs.config2(nx=nx, ny=ny, iters=a.iters)
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    modes = {"per_granule_windowed": dict(window_events=a.window),
             "per_granule_postmortem": dict(window_events=0),
             "interval_compressed_windowed": dict(window_events=a.window, flags=cs.CUSAN_CHECK_INTERVAL_SHADOW)}
    out = {"nx": nx, "ny": ny, "iters": a.iters, "window_events": a.window}
    ref = None
    for name, kw in modes.items():
        rep, secs, kms = timed(tr, **kw)
        c = rep.counters
        if ref is None:
            ref = rep
            out.update(events=int(c["n_events"]), accesses=int(c["n_access"]), tracked_bytes=int(c["tracked_bytes"]),
                       race_granules=int(rep.n_race_granules), race_runs=int(rep.n_runs))
        assert rep.n_race_granules == ref.n_race_granules and np.array_equal(rep.runs, ref.runs), name
        out[name] = {"step_ms": secs * 1e3, "kernel_ms": kms, "checked_gbs": c["tracked_bytes"] / secs / 1e9,
                     "shadow_bytes": int(c["shadow_bytes"]), "windows": int(c["n_windows"]),
                     "cell_bytes": int(c["shadow_cell_bytes"])}
    print(json.dumps(out), flush=True)
