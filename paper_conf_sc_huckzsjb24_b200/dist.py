"""Multi-GPU check: the shadow space is sharded by granule range, one shard per rank.

Granules are independent.  The rank that recorded the trace computes the event clocks once (a1,
cusan_clocks_compute, on all of the node's cores) and broadcasts them (broadcast_clocks: one flat
image — access ranges, records, segment clock rows — NCCL over NVLink); every rank then builds the
tables of its own shard on its own GPU (a2 on the device, cusan_plan_create_from_clocks), checks
it with no communication inside the check, and the race runs are gathered to rank 0 — the one real
exchange step — with torch.distributed (NCCL on GPUs, gloo in CPU tests).  Rank 0 stitches runs
that abut across shard boundaries and sorts them canonically (cusan_report_merge).  Sessions (f1)
broadcast the raw events instead (broadcast_trace): their planning is incremental per call.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import RUN_DTYPE, Clocks, Plan, Report, Session, Trace, report_merge

_RUN_U64 = RUN_DTYPE.itemsize // 8          # a run record as three u64 words


def gather_runs(runs: np.ndarray, n_race: int, device: torch.device | None = None,
                group=None) -> tuple[np.ndarray, int] | None:
    """All-gather every rank's runs and race-granule count; returns (runs, count) on rank 0."""
    dev = device if device is not None else torch.device("cpu")
    words = torch.from_numpy(np.ascontiguousarray(runs, RUN_DTYPE).view(np.uint64).astype(np.int64)).to(dev)
    world = dist.get_world_size(group)
    meta = torch.tensor([len(runs), n_race], dtype=torch.int64, device=dev)
    metas = [torch.zeros_like(meta) for _ in range(world)]
    dist.all_gather(metas, meta, group=group)
    counts = [int(m[0]) for m in metas]
    cap = max(max(counts), 1)
    buf = torch.zeros(cap * _RUN_U64, dtype=torch.int64, device=dev)
    buf[: words.numel()] = words
    parts = [torch.zeros_like(buf) for _ in range(world)]
    dist.all_gather(parts, buf, group=group)
    if dist.get_rank(group) != 0:
        return None
    allw = [p[: c * _RUN_U64].cpu().numpy().astype(np.uint64) for p, c in zip(parts, counts)]
    merged = np.concatenate(allw).view(RUN_DTYPE) if allw else np.zeros(0, RUN_DTYPE)
    return merged, int(sum(int(m[1]) for m in metas))


def broadcast_trace(trace: Trace | None, src: int = 0, device: torch.device | None = None, group=None,
                    first: int = 0) -> Trace:
    """The recorded trace lives on rank ``src`` (the process that intercepted the application's
    calls); every rank gets the same primitive events (24 B each, SURVEY §8(e) "broadcast the event
    table") and returns a Trace holding them — ``src`` its own trace, the others a new Trace (or
    ``trace`` extended, when given) with events ``first..`` of src's trace appended (same
    max_fibers as src's).  One broadcast of (count, max_fibers), one of the raw event bytes (NCCL
    over NVLink on GPUs)."""
    from . import EVENT_DTYPE
    dev = device if device is not None else torch.device("cpu")
    me = dist.get_rank(group)
    if me == src:
        ev = trace.cusan_trace_read(first)
        meta = torch.tensor([len(ev), trace.cusan_trace_size()[1]], dtype=torch.int64, device=dev)
    else:
        meta = torch.zeros(2, dtype=torch.int64, device=dev)
    dist.broadcast(meta, dist.get_global_rank(group, src) if group is not None else src, group=group)
    n, nf = int(meta[0]), int(meta[1])
    if me == src:
        buf = torch.from_numpy(np.ascontiguousarray(ev).view(np.uint8)).to(dev)
    else:
        buf = torch.empty(n * EVENT_DTYPE.itemsize, dtype=torch.uint8, device=dev)
    if n:
        dist.broadcast(buf, dist.get_global_rank(group, src) if group is not None else src, group=group)
    if me == src:
        return trace
    out = trace if trace is not None else Trace(nf)
    if n:
        out.cusan_trace_append_events(buf.cpu().numpy().view(EVENT_DTYPE))
    return out


def broadcast_clocks(clocks: Clocks | None, src: int = 0, device: torch.device | None = None,
                     group=None) -> Clocks:
    """Rank ``src`` holds the clocks (a1 of the whole trace); every rank returns them: one broadcast
    of the image size, one of the image (NCCL over NVLink on GPUs)."""
    dev = device if device is not None else torch.device("cpu")
    me = dist.get_rank(group)
    root = dist.get_global_rank(group, src) if group is not None else src
    img = clocks.to_bytes() if me == src else None
    meta = torch.tensor([len(img) if me == src else 0], dtype=torch.int64, device=dev)
    dist.broadcast(meta, root, group=group)
    n = int(meta[0])
    buf = torch.from_numpy(img).to(dev) if me == src else torch.empty(n, dtype=torch.uint8, device=dev)
    dist.broadcast(buf, root, group=group)
    return clocks if me == src else Clocks.from_bytes(buf.cpu().numpy())


class ShardedPlan:
    """One rank's shard of a multi-GPU check.  run() checks the shard on this rank's GPU, gathers
    the runs and returns the canonical whole-trace Report on rank 0 (None elsewhere).

    ``trace``: a Trace every rank holds (each rank computes the clocks itself), or — with
    ``clocks_src`` set — the recording rank's Trace (None elsewhere): that rank computes the clocks
    and broadcasts them, the others need no trace.  ``clocks``: clocks every rank already holds."""

    def __init__(self, trace: Trace | None = None, device: int = 0, group=None,
                 comm_device: torch.device | None = None, clocks: Clocks | None = None,
                 clocks_src: int | None = None, **kw):
        import time
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.comm_device = comm_device
        self.max_runs = kw.pop("max_runs", 0)
        self.timings = {}
        t0 = time.perf_counter()
        if clocks is None and clocks_src is not None:
            mine = Clocks.compute(trace) if self.rank == clocks_src else None
            t1 = time.perf_counter()
            clocks = broadcast_clocks(mine, clocks_src, comm_device, group)
            self.timings["clocks_ms"] = 1e3 * (t1 - t0)
            self.timings["broadcast_ms"] = 1e3 * (time.perf_counter() - t1)
        t2 = time.perf_counter()
        self.plan = Plan(clocks if clocks is not None else trace, nshards=self.world, shard=self.rank,
                         device=device, **kw)
        self.timings["plan_ms"] = 1e3 * (time.perf_counter() - t2)
        self.last_shard_report: Report | None = None

    def run(self) -> Report | None:
        import time
        rep = self.plan.run()
        self.last_shard_report = rep
        t0 = time.perf_counter()
        out = gather_runs(rep.runs, rep.n_race_granules, self.comm_device, self.group)
        self.timings["gather_ms"] = 1e3 * (time.perf_counter() - t0)
        if out is None:
            return None
        runs, n_race = out
        return report_merge(runs, n_race, self.max_runs)

    def close(self):
        self.plan.close()


class ShardedSession:
    """One rank's shard of a multi-GPU online check (f1 on N GPUs).  Every rank appends the same
    events to its trace (itself, or from the recording rank with pull()); its session keeps the shadow of its block-cyclic share of the granule
    space (granule g -> shard (g / shard_block) mod N: the address space is not known in advance,
    so a contiguous split cannot be balanced up front).  check() checks this rank's share of the
    new accesses, gathers the runs and returns the call's canonical report on rank 0 (None
    elsewhere)."""

    def __init__(self, trace: Trace, device: int = 0, group=None, comm_device: torch.device | None = None,
                 **kw):
        self.group = group
        self.comm_device = comm_device
        self.max_runs = kw.pop("max_runs", 0)
        self.session = Session(trace, nshards=dist.get_world_size(group), shard=dist.get_rank(group),
                               device=device, **kw)
        self.trace = trace
        self._sent = 0
        self.last_shard_report: Report | None = None

    def pull(self, src: int = 0) -> int:
        """Bring every rank's trace up to date with rank ``src``'s, the one recording the
        application: src broadcasts the events appended since its last pull (broadcast_trace with
        ``first``), the others append them.  Call on every rank before check()/submit(); returns the
        number of events moved."""
        me = dist.get_rank(self.group)
        n0 = len(self.trace)
        broadcast_trace(self.trace, src=src, device=self.comm_device, group=self.group,
                        first=self._sent if me == src else 0)
        if me == src:
            moved = n0 - self._sent
            self._sent = n0
            return moved
        return len(self.trace) - n0

    def _gather(self, rep: Report) -> Report | None:
        self.last_shard_report = rep
        out = gather_runs(rep.runs, rep.n_race_granules, self.comm_device, self.group)
        if out is None:
            return None
        return report_merge(out[0], out[1], self.max_runs)

    def check(self) -> Report | None:
        return self._gather(self.session.check())

    def submit(self) -> Report | None:
        """Pipelined check (cusan_session_submit on every rank): returns the previous call's merged
        report on rank 0 (None elsewhere, and on the first call)."""
        prev = self.session.submit()
        has_prev = prev is not None          # the same on every rank: all ranks submit together
        return self._gather(prev) if has_prev else None

    def finish(self) -> Report | None:
        rep = self.session.finish()
        return self._gather(rep) if rep is not None else None

    def forget(self, addr: int, nbytes: int) -> None:
        """cusan_session_forget on this rank's shard (call it on every rank, like check())."""
        self.session.forget(addr, nbytes)

    def close(self):
        self.session.close()


def merge_shard_reports(parts: list[Report], max_runs: int = 0) -> Report:
    """Single-process form of the gather + stitch (used when shards run one after another)."""
    runs = np.concatenate([p.runs for p in parts]) if parts else np.zeros(0, RUN_DTYPE)
    return report_merge(runs, sum(p.n_race_granules for p in parts), max_runs)
