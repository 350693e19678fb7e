"""Online-checking throughput (f1): feed a config's trace to a cusan_session in chunks of
`--chunk` accesses and time every session call (incremental host plan + check).

    python tools/session_bench.py --config 5 --chunk 4096 [--nshards N]

With --nshards N, N block-cyclic shard sessions (one per GPU in a multi-GPU run) are run one after
another on this GPU; a call of the N-GPU session takes the slowest shard's time (the gather of a
call's runs is a few KB), so Σ over calls of that max predicts the N-GPU online time.  Reports of
the shards are merged per call and must add up to the one-shard race count.
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
ap.add_argument("--nshards", type=int, default=1)
ap.add_argument("--shard-block", type=int, default=0)
ap.add_argument("--summary", action="store_true", help="omit the per-call list")
ap.add_argument("--max-calls", type=int, default=0, help="stop after this many calls (0 = whole trace)")
ap.add_argument("--dense", action="store_true", help="per-granule shadow (default: interval-compressed)")
ap.add_argument("--pipelined", action="store_true",
                help="submit/finish: plan call i+1 on the host while the GPU checks call i (one shard)")
a = ap.parse_args()
if a.pipelined and a.nshards != 1:
    raise SystemExit("--pipelined times one session (on N GPUs every shard pipelines on its own)")

FLAGS = cs.CUSAN_CHECK_DENSE_SHADOW if a.dense else 0
w = configs.make(a.config, a.size)
ops, args = w.arrays(True)
full = cs.Trace(255)
cs.Lowering(full).cusan_lower_program(ops, args)
ev = full.cusan_trace_read()
acc_pos = np.flatnonzero(ev["kind"] == 0)
cuts = [int(acc_pos[i]) for i in range(a.chunk, len(acc_pos), a.chunk)] + [len(ev)]
if a.max_calls:
    cuts = cuts[:a.max_calls]
# import-time objects out of the cyclic collector's way (a full pass is a ~35 ms pause with torch
# imported: it would dominate runs of a few hundred sub-millisecond calls)
import gc  # noqa: E402
gc.collect()
gc.freeze()

if a.pipelined:
    tr = cs.Trace(255)
    ses = cs.Session(tr, window_events=a.window, flags=FLAGS)
    reps, start = [], 0
    t0 = time.perf_counter()
    for end in cuts:
        tr.cusan_trace_append_events(ev[start:end])
        r = ses.submit()
        if r is not None:
            reps.append(r)
        start = end
    reps.append(ses.finish())
    secs = time.perf_counter() - t0
    ses.close()
    tot = sum(r.counters["tracked_bytes"] for r in reps)
    kms = sum(r.counters["kernel_ms"] for r in reps)
    print(json.dumps(dict(config=a.config, chunk_accesses=a.chunk, pipelined=True, dense=a.dense, calls=len(reps),
                          tracked_bytes=tot, checked_gbs=tot / secs / 1e9, kernel_checked_gbs=tot / (kms / 1e3) / 1e9,
                          seconds=secs, kernel_ms=kms, race_granules=sum(r.n_race_granules for r in reps))))
    raise SystemExit(0)

trs = [cs.Trace(255) for _ in range(a.nshards)]
sess = [cs.Session(trs[s], window_events=a.window, nshards=a.nshards, shard=s, shard_block=a.shard_block,
                   flags=FLAGS)
        for s in range(a.nshards)]
start, calls = 0, []
for end in cuts:
    per = []
    for t, ses in zip(trs, sess):
        t.cusan_trace_append_events(ev[start:end])
        t0 = time.perf_counter()
        rep = ses.check()
        dt = time.perf_counter() - t0
        c = rep.counters
        per.append(dict(seconds=dt, kernel_ms=c["kernel_ms"], tracked=c["tracked_bytes"],
                        cell_bytes=c["shadow_cell_bytes"], races=rep.n_race_granules, launches=c["kernel_launches"]))
    calls.append(dict(events=end - start, seconds=max(x["seconds"] for x in per),
                      kernel_ms=max(x["kernel_ms"] for x in per), tracked=per[0]["tracked"],
                      cell_bytes=sum(x["cell_bytes"] for x in per), races=sum(x["races"] for x in per),
                      launches=max(x["launches"] for x in per),
                      shard_seconds=[x["seconds"] for x in per] if a.nshards > 1 else None))
    start = end
for ses in sess:
    ses.close()
tot = sum(x["tracked"] for x in calls)
secs = sum(x["seconds"] for x in calls)
kms = sum(x["kernel_ms"] for x in calls)
cell = sum(x["cell_bytes"] for x in calls)
out = dict(config=a.config, chunk_accesses=a.chunk, dense=a.dense, nshards=a.nshards, calls=len(calls), tracked_bytes=tot,
           checked_gbs=tot / secs / 1e9, kernel_checked_gbs=tot / (kms / 1e3) / 1e9,
           kernel_dram_gbs_per_shard=cell / a.nshards / (kms / 1e3) / 1e9, seconds=secs, kernel_ms=kms,
           race_granules=sum(x["races"] for x in calls), per_call=calls)
cs_ = sorted(x["seconds"] for x in calls)
ks_ = sorted(x["kernel_ms"] for x in calls)
out.update(call_ms_median=1e3 * cs_[len(cs_) // 2], call_ms_p90=1e3 * cs_[int(0.9 * (len(cs_) - 1))],
           kernel_ms_median=ks_[len(ks_) // 2])
if a.summary:
    out.pop("per_call")
print(json.dumps(out))
