"""What the live capture (f2) and online checking (f1) cost a running PyTorch program — the paper's
measure of a tool (runtime overhead over the uninstrumented "vanilla" run, PAPER.md:888-902,
Fig. 10), here for a Jacobi halo-exchange solver written in PyTorch on two streams (the shape of
BASELINE config 2: compute stream, halo stream, pack / exchange / unpack, a residual read back
every few iterations).

    python tools/capture_overhead.py [--n 4096] [--iters 200] [--racy]

Per iteration (two timed runs of --iters iterations after --warmup, each timed as a whole; the
program synchronises only to read the residual back), the same program four ways:
  vanilla      — no instrumentation;
  dispatch_only — a Python operator-dispatch mode that records nothing (the floor of a capture
                 built on TorchDispatchMode);
  capture      — inside `Capture()`: every ATen operator and CUDA stream / event call recorded;
  online       — the same, plus `Session.check()` on the trace every iteration (the GPU checks
                 the iteration's accesses while the program runs);
and the post-mortem `Capture.check()` of the whole run.  --racy drops the halo stream's wait for
the compute stream, so the pack kernels race with the previous iteration's writes.
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402
import torch.utils._python_dispatch  # noqa: E402

import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from paper_conf_sc_huckzsjb24_b200.capture import Capture  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=4096)
ap.add_argument("--iters", type=int, default=200)
ap.add_argument("--warmup", type=int, default=20)
ap.add_argument("--norm-every", type=int, default=10)
ap.add_argument("--racy", action="store_true")
a = ap.parse_args()

dev = torch.device("cuda", 0)
N = a.n


class Jacobi:
    def __init__(self):
        g = torch.Generator(device=dev).manual_seed(1)
        self.A = torch.rand(N, N, device=dev, generator=g)
        self.B = torch.zeros(N, N, device=dev)
        self.send = [torch.zeros(N, device=dev) for _ in range(4)]
        self.recv = [torch.zeros(N, device=dev) for _ in range(4)]
        self.s_comp = torch.cuda.Stream()
        self.s_halo = torch.cuda.Stream()
        self.norm = 0.0

    def step(self, it: int):
        A, B = self.A, self.B
        with torch.cuda.stream(self.s_halo):
            if not a.racy:
                self.s_halo.wait_stream(self.s_comp)          # the previous iteration's writes
            self.send[0].copy_(A[1, :])                       # pack
            self.send[1].copy_(A[-2, :])
            self.send[2].copy_(A[:, 1])
            self.send[3].copy_(A[:, -2])
            for k in range(4):                                # exchange (a neighbour's copy)
                self.recv[k].copy_(self.send[k])
        with torch.cuda.stream(self.s_comp):
            B[1:-1, 1:-1] = 0.25 * (A[:-2, 1:-1] + A[2:, 1:-1] + A[1:-1, :-2] + A[1:-1, 2:])
            self.s_comp.wait_stream(self.s_halo)
            B[0, :].copy_(self.recv[0])                       # unpack into the boundary
            B[-1, :].copy_(self.recv[1])
            B[:, 0].copy_(self.recv[2])
            B[:, -1].copy_(self.recv[3])
            if it % a.norm_every == 0:
                self.norm = (B - A).abs().sum().item()        # residual, read back on the host
        self.A, self.B = B, A


class _PassThrough(torch.utils._python_dispatch.TorchDispatchMode):
    """The floor of any capture built on Python operator dispatch: a mode that records nothing."""

    def __torch_dispatch__(self, func, types, args=(), kwargs=None):
        return func(*args, **(kwargs or {}))


def run(mode: str):
    torch.cuda.synchronize()
    app = Jacobi()
    times = []
    cap = Capture() if mode in ("capture", "online") else (_PassThrough() if mode == "dispatch_only" else None)
    ses = None
    if cap is not None:
        cap.__enter__()
        ses = cap.session() if mode == "online" else None   # forgets released temporaries
    n_race = [0]

    def iterate(k, start):
        for it in range(start, start + k):
            app.step(it)
            if ses is not None:
                n_race[0] += ses.check().n_race_granules

    try:
        # the program synchronises only where it reads the residual back (no per-iteration
        # device sync, which would order every stream and hide a missing wait); timed as a whole
        iterate(a.warmup, 0)
        torch.cuda.synchronize()
        for r in range(2):
            t0 = time.perf_counter()
            iterate(a.iters, a.warmup + r * a.iters)
            torch.cuda.synchronize()
            times.append(1e3 * (time.perf_counter() - t0) / a.iters)
    finally:
        if cap is not None:
            cap.__exit__(None, None, None)
    out = {"ms_per_iter": statistics.median(times), "ms_per_iter_runs": times}
    if isinstance(cap, Capture):
        out["events"] = len(cap.trace)
        out["ops"] = cap.ops
    if ses is not None:
        out["online_race_granules"] = n_race[0]
        ses.close()
    if mode == "capture":
        t0 = time.perf_counter()
        rep = cap.check()
        out["postmortem_check_ms"] = 1e3 * (time.perf_counter() - t0)
        out["postmortem_race_granules"] = rep.n_race_granules
    return out


res = {m: run(m) for m in ("vanilla", "dispatch_only", "capture", "online")}
v = res["vanilla"]["ms_per_iter"]
line = {"workload": f"PyTorch Jacobi {N}x{N} fp32, two streams, {a.iters} timed iterations"
                    f"{' (racy: no halo-stream wait)' if a.racy else ''}",
        "vanilla_ms_per_iter": v,
        "dispatch_only_ms_per_iter": res["dispatch_only"]["ms_per_iter"],
        "capture_ms_per_iter": res["capture"]["ms_per_iter"],
        "online_ms_per_iter": res["online"]["ms_per_iter"],
        "capture_overhead": res["capture"]["ms_per_iter"] / v,
        "online_overhead": res["online"]["ms_per_iter"] / v,
        "details": res}
print(json.dumps(line))
