"""Per-rank fixed costs of an N-GPU check on one GPU (development aid for DESIGN §6's budget):
the recording rank's lowering (a0) and clocks (a1), the clocks image size, and every shard's plan
(a2 on the device, from the clocks) and kernel time, each shard measured alone on an idle GPU —
what one rank of an N-GPU node pays — against §8(e)'s f <= T1/20.

    python tools/shard_budget.py --config 5 --nshards 8 [--flags dense|compressed]
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--nshards", type=int, default=8)
ap.add_argument("--window", type=int, default=4096)
ap.add_argument("--reps", type=int, default=5)
a = ap.parse_args()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)


def med(f, reps=a.reps):
    ts = []
    out = None
    for _ in range(reps):
        t0 = time.perf_counter()
        out = f()
        ts.append(1e3 * (time.perf_counter() - t0))
    return statistics.median(ts), out


def lower():
    t = cs.Trace(255)
    cs.Lowering(t).cusan_lower_program(ops, args)
    return t


lower_ms, tr = med(lower)
clocks_ms, vc = med(lambda: cs.Clocks.compute(tr))
img = vc.to_bytes()
res = {"config": a.config, "nshards": a.nshards, "window_events": a.window, "cpu_count": os.cpu_count(),
       "lower_ms": lower_ms, "clocks_ms": clocks_ms, "clocks_image_bytes": int(len(img)), "modes": {}}
s = torch.cuda.Stream()
for name, flags in (("compressed", 0), ("dense", cs.CUSAN_CHECK_DENSE_SHADOW)):
    one = cs.Plan(vc, window_events=a.window, flags=flags, workspace="torch", stream=s.cuda_stream)
    one.run()
    t1 = statistics.median(one.run().counters["kernel_ms"] for _ in range(3))
    one.close()
    del one
    torch.cuda.empty_cache()
    shards = []
    for k in range(a.nshards):
        kw = dict(window_events=a.window, flags=flags, nshards=a.nshards, shard=k)
        plan_ms, _ = med(lambda: cs.Plan(vc, flags=flags | cs.CUSAN_CHECK_DEFER_WORKSPACE,
                                         **{x: y for x, y in kw.items() if x != "flags"}).close())
        p = cs.Plan(vc, workspace="torch", stream=s.cuda_stream, **kw)
        p.run()
        r = p.run()
        shards.append({"shard": k, "plan_ms": plan_ms, "kernel_ms": r.counters["kernel_ms"],
                       "run_ms": r.counters["run_ms"], "shard_granules": int(r.counters["shard_granules"])})
        p.close()
        del p
        torch.cuda.empty_cache()
    res["modes"][name] = {"T1_kernel_ms": t1, "shards": shards,
                          "max_plan_ms": max(x["plan_ms"] for x in shards),
                          "max_kernel_ms": max(x["kernel_ms"] for x in shards)}
print(json.dumps(res, indent=1))
