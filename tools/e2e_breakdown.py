"""Where the end-to-end time of one check goes (development aid): lowering, plan creation (host a1/a2
+ table upload), workspace, run (kernels + merge + report), close — per step, for a full config.

    python tools/e2e_breakdown.py --config 4 --steps 4
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=4)
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--window", type=int, default=4096)
a = ap.parse_args()
w = configs.make(a.config, "full")
ops, args = w.arrays(True)
stream = torch.cuda.Stream()
kw = dict(window_events=a.window, device=0, stream=stream.cuda_stream)
for ws in ("torch", None):
    for s in range(a.steps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        tr = cs.Trace(255)
        cs.Lowering(tr).cusan_lower_program(ops, args)
        t1 = time.perf_counter()
        p = cs.Plan(tr, workspace=ws, **kw)
        t2 = time.perf_counter()
        r = p.run()
        t3 = time.perf_counter()
        p.close()
        torch.cuda.synchronize()
        t4 = time.perf_counter()
        c = r.counters
        print(f"workspace={ws} step {s}: lower {1e3*(t1-t0):.2f} plan {1e3*(t2-t1):.2f} run {1e3*(t3-t2):.2f} "
              f"(kernel {c['kernel_ms']:.2f}, run_ms {c['run_ms']:.2f}) close {1e3*(t4-t3):.2f} "
              f"total {1e3*(t4-t0):.2f} ms; runs {r.n_runs} raw {c['raw_runs']}", flush=True)
