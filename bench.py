#!/usr/bin/env python
"""bench.py — race-checked GB/s of the B200 happens-before race check (DESIGN.md §"Measurement").

One step = one pass of the whole hot path over the workload: the shadow-check kernels (a3) with
in-warp run compaction, the device merge into canonical runs (a4), their download and the report
(a5), with the event / clock / interval tables (a1, a2) already resident in HBM.

Two shadow layouts give the identical report; the line carries both:
  * `value`, `roofline`, `e2e`: the DENSE shadow (CUSAN_CHECK_DENSE_SHADOW, one 8-B cell per
    granule, TSan's layout) — every covered granule's cell is read and written in every window
    that touches it, the HBM-bound kernel SURVEY.md §8(d)'s roofline describes;
  * `modes.interval_compressed`: the library DEFAULT (one cell per elementary interval, f3) — the
    fastest exact path; its end-to-end time is host work (lowering, planning), not HBM.
`e2e` repeats the metric through the public API from host buffers: lowering of the recorded
CUDA/MPI call program (a0), planning (a1, a2), table upload from pinned host memory, check and
report download, every step — pipelined (`pipelined_checks`: lowering, clocks and plan of the next
steps on host threads overlap the GPU side of step i), with the unpipelined per-call number under `e2e.serial` and a per-phase
cost breakdown (lower / plan / upload / kernels / merge + download) under `breakdown`.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...      (one rank per GPU, shards by granule range)

Workload: BASELINE.json config 5 (scaling sweep: 64 GiB of log-uniform allocations, 64 fibers,
~100k primitive events; the largest trace, the one the metric is quoted on at 1/2/4/8 GPUs), racy
twin, online (windowed) mode: the shadow lives in HBM between windows of 4096 accesses.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "tracked bytes checked/sec (race-checked GB/s) at 1/2/4/8 B200 vs HBM peak"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--size", default="full", choices=["full", "small"])
    ap.add_argument("--window", type=int, default=4096, help="access events per shadow window")
    ap.add_argument("--clean", action="store_true", help="race-free twin instead of the racy twin")
    ap.add_argument("--e2e-steps", type=int, default=8)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target oracle sample time")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"])
    return ap.parse_args()


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_traffic():
    """dram read+write bytes per launch of the shadow-check kernel from the committed ncu capture."""
    p = os.path.join(ROOT, "profiles", "ncu_k1_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_launch"), d
    except Exception:
        return None, None


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-lms", "200", "-i", str(index)], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.seek(0)
        sm, smax, reasons = [], [], set()
        for line in self.f:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                smax.append(float(parts[2]))
            except ValueError:
                continue
            for name, v in zip(self.NAMES, parts[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        os.unlink(self.f.name)
        loaded = [s for s in sm if s > 500] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(smax) if smax else None, "reasons": sorted(reasons),
                "samples": len(sm)}


def workload(args):
    from tracegen import configs
    w = configs.make(args.config, args.size)
    ops, args_ = w.arrays(not args.clean)
    name = {1: "config1 racy listing", 2: "config2 Jacobi halo exchange 4096x4096 fp32, 100 iterations",
            3: "config3 multi-stream event DAG, 8 streams, 1 GiB, 10k launches",
            4: "config4 large tracked memory, 16 x 1 GiB annotated per launch, 1k launches",
            5: "config5 scaling sweep, 64 GiB log-uniform allocations, 64 fibers, ~100k events"}[args.config]
    return w, ops, args_, f"{name} ({'clean' if args.clean else 'racy'} twin, {args.size} size)"


def bench_config(wname, window, events, accesses, tracked):
    """`config` of the JSON line: the workload only, identical in both arms (--impl ours|reference);
    run-dependent figures go under `workload_stats`."""
    return {"workload": wname, "window_events": window, "events": int(events), "accesses": int(accesses),
            "fibers": 64, "tracked_bytes": int(tracked),
            "l2": "inputs larger than L2 (dense shadow 64 GiB, streamed every window)"}


# ------------------------------------------------------------------------------------------------
# CPU baseline: the oracle (as it stands) on a bounded contiguous granule sample of the same trace
# ------------------------------------------------------------------------------------------------
def oracle_sample(events, max_fibers, target_s, threads):
    import numpy as np
    import oracle
    acc = events[events["kind"] == 0]
    g0 = (acc["a"] >> np.uint64(3)).astype(np.int64)
    g1 = ((acc["a"] + acc["b"] + np.uint64(7)) >> np.uint64(3)).astype(np.int64)
    lo, hi = int(g0.min()), int(g1.max())

    def checked(a, b):
        return int(8 * np.sum(np.clip(np.minimum(g1, b) - np.maximum(g0, a), 0, None)))

    span = max(1, (hi - lo) // 4096)         # calibration slice
    r = oracle.check_events(events, max_fibers, threads=threads, granule_range=(lo, lo + span))
    rate = checked(lo, lo + span) / max(r["seconds"], 1e-3)
    for _ in range(4):                       # grow the slice until the oracle takes ~target_s
        want = target_s * rate
        b = lo + span
        # extend the range until it holds `want` checked bytes (binary search over the end)
        l2, h2 = lo + 1, hi
        while l2 < h2:
            m = (l2 + h2) // 2
            if checked(lo, m) < want:
                l2 = m + 1
            else:
                h2 = m
        b = max(l2, lo + 1)
        r = oracle.check_events(events, max_fibers, threads=threads, granule_range=(lo, b))
        cb = checked(lo, b)
        rate = cb / max(r["seconds"], 1e-3)
        if r["seconds"] >= 0.5 * target_s or b >= hi:
            break
        span = b - lo
    return dict(checked_bytes=cb, seconds=r["seconds"], granules=b - lo, range=(lo, b),
                race_granules=r["n_race_granules"], rate_gbs=cb / r["seconds"] / 1e9)


def run_reference(args):
    """--impl reference: the oracle timed on the host cores, K bounded-sample steps (rank 0)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle.lower import lower
    w, ops, args_, wname = workload(args)
    ev, nf = lower(ops, args_)
    threads = os.cpu_count() or 1
    per_step = max(1.0, min(20.0, 150.0 / max(1, args.steps + args.warmup)))
    s = oracle_sample(ev, nf, per_step, threads)
    for _ in range(args.warmup):
        oracle_sample_step(ev, nf, s, threads)
    tot_b, tot_s = 0, 0.0
    for _ in range(args.steps):
        b, secs = oracle_sample_step(ev, nf, s, threads)
        tot_b += b
        tot_s += secs
    value = tot_b / tot_s / 1e9
    import numpy as np
    acc = ev[ev["kind"] == 0]
    tracked = int(8 * np.sum(((acc["a"] + acc["b"] + np.uint64(7)) >> np.uint64(3)) - (acc["a"] >> np.uint64(3))))
    ref_config = bench_config(wname, args.window, len(ev), len(acc), tracked)
    sample = (f"granules [{s['range'][0]}, {s['range'][1]}) = {s['granules']} granules, "
              f"{s['checked_bytes'] / 1e9:.1f} GB checked per step")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot_s / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": ref_config, "parallelism": f"{threads} host threads",
        "note": "the oracle checks the whole trace at once; the race set does not depend on windows",
        "cpu_baseline": {"value": value, "unit": "GB/s", "cores": threads, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": sample},
        "e2e": {"value": value, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_sample_step(ev, nf, s, threads):
    import oracle
    r = oracle.check_events(ev, nf, threads=threads, granule_range=s["range"])
    return s["checked_bytes"], r["seconds"]


# ------------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------------
def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_sc_huckzsjb24_b200 as cs
    from paper_conf_sc_huckzsjb24_b200.dist import ShardedPlan, broadcast_clocks, gather_runs

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # one rank per GPU; --dist-backend gloo lets several ranks share GPUs (testing the sharded
    # path on a 1-GPU box: shards checked concurrently, runs gathered over gloo)
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    comm_dev = dev
    if world > 1:
        if args.dist_backend == "nccl":
            # communicator lines (rank r of N) for the logs, on stderr so stdout stays one JSON line
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
            comm_dev = torch.device("cpu")
    stream = torch.cuda.current_stream(dev)

    w, ops, args_, wname = workload(args)
    # The interpreter's objects so far (torch and its imports: ~10^6) move to the permanent
    # generation, so Python's cyclic collector does not rescan them during the timed steps (a full
    # collection of them is a ~35 ms pause every ~0.5 s of a pipelined run, all host stages held).
    # Objects created from here on are collected as usual.
    import gc
    gc.collect()
    gc.freeze()
    tr = vc = None
    if world == 1 or rank == 0:
        tr = cs.Trace(255)
        cs.Lowering(tr).cusan_lower_program(ops, args_)
    if world > 1:      # rank 0 recorded the program: it computes the event clocks once (a1) and
        #                broadcasts them; every rank plans its own shard from them on its GPU
        vc = broadcast_clocks(cs.Clocks.compute(tr) if rank == 0 else None, device=comm_dev)
        print(f"cusan bench: rank {rank} of {world} ({args.dist_backend}), device {local}", file=sys.stderr)

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=comm_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # device memory for every plan comes from PyTorch's caching allocator
    DENSE = cs.CUSAN_CHECK_DENSE_SHADOW
    kw = dict(window_events=args.window, device=local, stream=stream.cuda_stream, workspace="torch", flags=DENSE)
    if world > 1:
        plan = ShardedPlan(clocks=vc, comm_device=comm_dev, **kw)
        run = plan.run
    else:
        plan = cs.Plan(tr, **kw)
        run = plan.run
    for _ in range(args.warmup):
        rep = run()
    # ---- timed region: K steps, CUDA events on the plan's stream, max over ranks ------------------
    clocks = Clocks(local)
    barrier()
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    kernel_ms, reps = [], []
    for _ in range(args.steps):
        rep = run()
        shard = plan.last_shard_report if world > 1 else rep
        kernel_ms.append(shard.counters["kernel_ms"])
        reps.append(rep)
    e1.record(stream)
    torch.cuda.synchronize(dev)
    barrier()
    clk = clocks.stop()
    elapsed_s = max_over_ranks(e0.elapsed_time(e1) / 1e3)
    shard = plan.last_shard_report if world > 1 else rep
    ctr = shard.counters
    launches = int(ctr["kernel_launches"]) * args.steps
    final = reps[-1]
    plan.close()
    del plan

    tracked = ctr["tracked_bytes"]                       # whole trace (every rank's shard together)
    value = tracked * args.steps / elapsed_s / 1e9
    k_ms = statistics.mean(kernel_ms)
    cell_bytes = ctr["shadow_cell_bytes"]
    peak, peak_src = measured_peaks()
    achieved = cell_bytes / (k_ms / 1e3) / 1e9 if k_ms > 0 else 0.0
    nl = max(1, int(ctr["n_windows"]))                  # K1 launches per step (one per window)
    traffic, _ = ncu_traffic()
    if not (args.config == 5 and args.size == "full" and args.window == 4096 and world == 1):
        traffic = None                                   # the committed capture is of the bench workload

    # ---- e2e: public API from host buffers, every step: lower + plan + upload + check + report ----
    # (a) pipelined (the value reported): pipelined_checks lowers step i+2 and plans step i+1 on
    #     host threads while the GPU checks step i; every step still uploads its own tables and
    #     downloads its own report.  Two untimed warm-up steps fill the pipeline.
    # (b) serial, for context: one cusan_check after another, nothing overlapped.
    def make_trace(_i):
        t = cs.Trace(255)
        cs.Lowering(t).cusan_lower_program(ops, args_)
        return t

    def e2e_pipelined(flags, step_s_hint, workers):
        """Pipelined end-to-end steps: (GB/s, s/step, h2d, d2h, mean kernel ms).  `workers` host threads
        per stage: 3 where the host stages bound the step (compressed), 1 where the GPU check does
        (dense: more planners in flight only queue behind the persistent check kernel)."""
        pkw = dict(window_events=args.window, stream=stream.cuda_stream, flags=flags)
        if world > 1:
            pkw.update(nshards=world, shard=rank)
        # at least --e2e-steps timed steps and ~2 s of them (short steps are noisy), eight warm-up steps
        n = max(1, args.e2e_steps, min(3000, int(2.0 / max(1e-5, step_s_hint))))
        h2d = d2h = 0
        barrier()
        torch.cuda.synchronize(dev)
        t0 = None
        kms = []
        # make_trace lowers a fresh copy of the recorded program per step: safe on two threads
        for i, (_tr, r2) in enumerate(cs.pipelined_checks(make_trace, n + 8, device=local, host_workers=workers,
                                                          lower_workers=workers, **pkw)):
            if i < 8:                                # warm-up steps: fill the pipeline
                if i == 7:
                    barrier()
                    t0 = time.perf_counter()
                continue
            c2 = r2.counters
            h2d, d2h = int(c2["h2d_bytes"]), int(c2["d2h_bytes"])
            kms.append(float(c2["kernel_ms"]))
            if world > 1:
                out = gather_runs(r2.runs, r2.n_race_granules, comm_dev)
                r2 = cs.report_merge(*out) if out is not None else None
            if rank == 0:
                assert r2.n_race_granules == final.n_race_granules and np.array_equal(r2.runs, final.runs)
        torch.cuda.synchronize(dev)
        step_s = max_over_ranks(time.perf_counter() - t0) / n
        return tracked / step_s / 1e9, step_s, n, h2d, d2h, (statistics.mean(kms) if kms else None)

    def e2e_serial_and_breakdown(flags, reps=3):
        """One check after another (nothing overlapped), timed per phase; medians.  The device
        workspace is allocated once and reused by every step (as pipelined_checks and the library's
        own parked workspaces do), so no step pays a cudaMalloc."""
        ph = {"lower_ms": [], "plan_ms": [], "upload_ms": [], "kernel_ms": [], "merge_download_ms": [],
              "total_ms": []}
        ws = None
        for i in range(reps + 1):                                # one untimed step sizes the workspace
            barrier()
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            t2 = make_trace(0)                                   # a0: lowering of the API program
            t1 = time.perf_counter()
            p2 = cs.Plan(t2, **dict(kw, flags=flags, workspace=None)
                         | {"flags": flags | cs.CUSAN_CHECK_DEFER_WORKSPACE})
            t2b = time.perf_counter()                            # a1 (host) + a2 (device planner)
            need = max(p2.workspace_bytes(), 256)
            if ws is None or ws.numel() < need:
                ws = None
                ws = torch.empty(need, dtype=torch.uint8, device=dev)
                t2b = time.perf_counter()                        # (allocation not part of a step)
            p2.cusan_plan_bind_workspace(ws)                     # table upload (pinned -> HBM)
            torch.cuda.synchronize(dev)
            t3 = time.perf_counter()
            r2 = p2.run()                                        # a3 + a4 + a5
            rc = r2.counters
            p2.close()
            torch.cuda.synchronize(dev)
            t4 = time.perf_counter()
            if rank == 0:
                assert r2.n_race_granules == final.n_race_granules and np.array_equal(r2.runs, final.runs)
            if i == 0:
                continue
            ph["lower_ms"].append(1e3 * (t1 - t0))
            ph["plan_ms"].append(1e3 * (t2b - t1))
            ph["upload_ms"].append(1e3 * (t3 - t2b))
            ph["kernel_ms"].append(float(rc["kernel_ms"]))
            ph["merge_download_ms"].append(max(0.0, 1e3 * (t4 - t3) - float(rc["kernel_ms"])))
            ph["total_ms"].append(1e3 * (t4 - t0))
        med = {k: statistics.median(v) for k, v in ph.items()}
        return tracked / (med["total_ms"] / 1e3) / 1e9, med

    def e2e_sharded(flags, reps):
        """N ranks, every step: rank 0 lowers the program (a0) and computes the clocks (a1), broadcasts
        them; every rank plans its shard on its GPU (a2), checks it (a3, a4), the runs are gathered
        and stitched on rank 0 (a5).  Per-phase times are the max over ranks (medians of steps)."""
        ph = {"lower_ms": [], "clocks_ms": [], "broadcast_ms": [], "plan_ms": [], "check_ms": [],
              "gather_merge_ms": [], "total_ms": []}
        h2d = d2h = 0
        for _ in range(reps):
            barrier()
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            t2 = make_trace(0) if rank == 0 else None
            t1 = time.perf_counter()
            p2 = ShardedPlan(t2, clocks_src=0, comm_device=comm_dev, **dict(kw, flags=flags))
            t3 = time.perf_counter()
            shard = p2.plan.run()
            torch.cuda.synchronize(dev)
            t4 = time.perf_counter()
            out = gather_runs(shard.runs, shard.n_race_granules, comm_dev)
            r2 = cs.report_merge(*out) if out is not None else None
            t5 = time.perf_counter()
            p2.close()
            for k, v in (("lower_ms", t1 - t0), ("clocks_ms", p2.timings["clocks_ms"] / 1e3),
                         ("broadcast_ms", p2.timings["broadcast_ms"] / 1e3), ("plan_ms", p2.timings["plan_ms"] / 1e3),
                         ("check_ms", t4 - t3), ("gather_merge_ms", t5 - t4), ("total_ms", t5 - t0)):
                ph[k].append(max_over_ranks(v) * 1e3)
            h2d, d2h = int(shard.counters["h2d_bytes"]), int(shard.counters["d2h_bytes"])
            if rank == 0:
                assert r2.n_race_granules == final.n_race_granules and np.array_equal(r2.runs, final.runs)
        med = {k: statistics.median(v) for k, v in ph.items()}
        return tracked / (med["total_ms"] / 1e3) / 1e9, med, h2d, d2h

    if world == 1:
        e2e_value, e2e_step_s, n_e2e, h2d, d2h, e2e_kms = e2e_pipelined(DENSE, elapsed_s / args.steps, 1)
        e2e_serial, dense_breakdown = e2e_serial_and_breakdown(DENSE)
    else:
        e2e_value, dense_breakdown, h2d, d2h = e2e_sharded(DENSE, 3)
        e2e_serial, e2e_step_s, n_e2e, e2e_kms = e2e_value, dense_breakdown["total_ms"] / 1e3, 3, None

    # ---- post-mortem variant (extra, for context): one window, no shadow traffic --------------------
    pm = None
    if world == 1:
        p3 = cs.Plan(tr, window_events=0, device=local, stream=stream.cuda_stream, workspace="torch", flags=DENSE)
        p3.run()
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        r3 = p3.run()
        pm_s = time.perf_counter() - t0
        assert r3.n_race_granules == final.n_race_granules and np.array_equal(r3.runs, final.runs)
        pm = {"value": tracked / pm_s / 1e9, "unit": "GB/s", "ms_per_step": pm_s * 1e3,
              "kernel_ms": r3.counters["kernel_ms"], "window_events": "all (one window)"}
        p3.close()

    # ---- interval-compressed shadow (f3, the library default): same windows, one cell per interval --
    # device-timed steps (tables resident, CUDA events on the plan's stream), pipelined and serial
    # end to end through the public API, and its cost breakdown
    ckw = dict(kw, flags=cs.CUSAN_CHECK_INTERVAL_SHADOW)
    p4 = ShardedPlan(clocks=vc, comm_device=comm_dev, **ckw) if world > 1 else cs.Plan(tr, **ckw)
    for _ in range(max(3, args.warmup)):
        p4.run()
    n_ic = max(args.steps, 50)
    barrier()
    torch.cuda.synchronize(dev)
    e0.record(stream)
    ic_kms = []
    for _ in range(n_ic):
        r4 = p4.run()
        ic_kms.append((p4.last_shard_report if world > 1 else r4).counters["kernel_ms"])
    e1.record(stream)
    torch.cuda.synchronize(dev)
    ic_s = max_over_ranks(e0.elapsed_time(e1) / 1e3) / n_ic
    ic_ctr = (p4.last_shard_report if world > 1 else r4).counters
    if rank == 0:
        assert r4.n_race_granules == final.n_race_granules and np.array_equal(r4.runs, final.runs)
    p4.close()
    del p4
    if world == 1:
        ic_e2e, ic_e2e_s, ic_n, ic_h2d, ic_d2h, ic_e2e_kms = e2e_pipelined(cs.CUSAN_CHECK_INTERVAL_SHADOW, 0.0007, 3)
        ic_serial, ic_breakdown = e2e_serial_and_breakdown(cs.CUSAN_CHECK_INTERVAL_SHADOW, reps=5)
    else:
        ic_e2e, ic_breakdown, ic_h2d, ic_d2h = e2e_sharded(cs.CUSAN_CHECK_INTERVAL_SHADOW, 5)
        ic_serial, ic_e2e_s, ic_n, ic_e2e_kms = ic_e2e, ic_breakdown["total_ms"] / 1e3, 5, None
    ic = {"value": tracked / ic_s / 1e9, "unit": "GB/s", "ms_per_step": ic_s * 1e3, "steps": n_ic,
          "kernel_ms_per_step": statistics.mean(ic_kms), "kernel_launches_per_step": int(ic_ctr["kernel_launches"]),
          "shadow_bytes_per_gpu": int(ic_ctr["shadow_bytes"]), "window_events": args.window,
          "flags": "CUSAN_CHECK_INTERVAL_SHADOW (library default)",
          "e2e": {"value": ic_e2e, "unit": "GB/s", "h2d_bytes_per_step": ic_h2d, "d2h_bytes_per_step": ic_d2h,
                  "ms_per_step": 1e3 * ic_e2e_s, "steps": ic_n, "kernel_ms_per_step": ic_e2e_kms,
                  "mode": "pipelined_checks as the dense e2e, three host threads per stage (each step lowers its own copy of "
                          "the program)",
                  "serial": {"value": ic_serial, "unit": "GB/s", "ms_per_step": ic_breakdown["total_ms"]}},
          "breakdown": ic_breakdown}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        ev = tr.cusan_trace_read()
        s = oracle_sample(ev, 255, args.cpu_seconds, os.cpu_count() or 1)
        s1 = oracle_sample(ev, 255, 2.0, 1)          # single-thread rate on a smaller slice
        cpu = {"value": s["rate_gbs"], "unit": "GB/s", "cores": os.cpu_count() or 1, "kind": "oracle",
               "cpu_model": cpu_model(), "single_thread_value": s1["rate_gbs"],
               "sample": (f"contiguous granule range [{s['range'][0]}, {s['range'][1]}) of the same trace: "
                          f"{s['granules']} granules, {s['checked_bytes'] / 1e9:.1f} GB checked in "
                          f"{s['seconds']:.1f} s")}
    d_cov = tracked / 8 / max(1, ctr["n_windows"]) / max(1, ctr["shard_granules"]) if world == 1 else None
    line = {
        "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * elapsed_s / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": bench_config(wname, args.window, ctr["n_events"], ctr["n_access"], tracked),
        "parallelism": f"granule-range shards x{world}",
        "workload_stats": {"windows": int(ctr["n_windows"]), "shadow_bytes_per_gpu": int(ctr["shadow_bytes"]),
                           "granules_per_gpu": int(ctr["shard_granules"]), "coverage_per_window": d_cov,
                           "race_granules": int(final.n_race_granules), "race_runs": int(final.n_runs),
                           "shadow": "dense: one 8-B cell per 8-byte granule (modes.interval_compressed: "
                                     "the library default)"},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                     "kernel": "shadow_check_window", "kernel_ms_per_step": k_ms, "launches_per_step": nl,
                     "algorithmic_bytes_per_launch": cell_bytes / nl},
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_value, "unit": "GB/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "ms_per_step": 1e3 * e2e_step_s, "steps": n_e2e,
                "kernel_ms_per_step": e2e_kms,
                "mode": ("pipelined_checks: lowering (a0), clocks (a1) and plans (a2) of the next steps on host threads "
                         "(one per stage: the GPU check bounds the step) overlap the GPU check of step i; pinned host tables uploaded and the report "
                         "downloaded every step; 8 warm-up steps") if world == 1 else
                        ("sharded, serial: rank 0 lowers + computes clocks, broadcast, every rank plans its shard on its GPU, "
                         "checks, runs gathered to rank 0 (median of 3 steps, phases max over ranks)"),
                "serial": {"value": e2e_serial, "unit": "GB/s", "ms_per_step": dense_breakdown["total_ms"],
                           "mode": "lower + plan + upload + check per step, nothing overlapped (median of 3)"},
                "breakdown": dense_breakdown},
        "gpu_launches": launches,
        "clocks": clk,
        "postmortem": pm,
        "modes": {"dense": {"value": value, "e2e": e2e_value, "flags": "CUSAN_CHECK_DENSE_SHADOW (value, roofline, e2e)"},
                  "interval_compressed": ic},
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
