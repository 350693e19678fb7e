"""Seeded synthetic workloads shaped like the paper's (BASELINE.json ``configs``).

Every generator returns an API program (``Program``) — CUDA / MPI calls, not happens-before
primitives.  The race-free program carries correct synchronisation by construction (dependency
tracking at allocation granularity, over-synchronising where in doubt).  Its *racy twin* is the same
program with a seeded subset of sync calls removed (``droppable`` op indices), so both twins share
every other call and handle.

Workload shapes (DESIGN.md §"Input recipe"):
  1  racy listing  — Fig. 4 / Fig. 6A shape
  2  Jacobi halo exchange — Table I shape, 4096² fp32, 2 streams, 100 iterations
  3  multi-stream event DAG — 8 streams, EventRecord/StreamWaitEvent, 1 GiB, 10k launches
  4  large tracked memory — 16 GiB annotated by every launch, 1k launches
  5  scaling sweep — 64 GiB log-uniform allocations, 64 fibers, ~100k primitive events
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

from .program import (CPY_D2H, CPY_H2D, MEM_DEVICE, MEM_PINNED, MODE_R, MODE_RW, MODE_W,
                      DEFAULT_STREAM, OP_EVENT_SYNC, OP_STREAM_SYNC, OP_STREAM_WAIT_EVENT, Program)

KiB, MiB, GiB = 1 << 10, 1 << 20, 1 << 30


@dataclass
class Workload:
    name: str
    program: Program
    droppable: list[int] = field(default_factory=list)   # op indices a racy twin may remove
    n_drop: int = 0
    racy_seed: int = 0
    meta: dict = field(default_factory=dict)

    def arrays(self, racy: bool):
        ops, args = self.program.arrays()
        if racy and self.n_drop:
            rng = np.random.default_rng(self.racy_seed)
            k = min(self.n_drop, len(self.droppable))
            drop = rng.choice(np.array(self.droppable, np.int64), size=k, replace=False)
            keep = np.ones(len(ops), bool)
            keep[drop] = False
            ops = ops[keep]
        return ops, args


# ---------------------------------------------------------------------------------------------
# config 1: the paper's racy listing (Fig. 4 rank 0 / Fig. 6A shape)
# ---------------------------------------------------------------------------------------------
def config1(nbytes: int = 4 * KiB) -> Workload:
    """init_kernel<<<s>>>(d) W; StreamSync(s); compute_kernel<<<s>>>(d) RW; [StreamSync(s) — dropped
    in the racy twin]; MPI_Isend(d) R; MPI_Wait; StreamSync(s)."""
    p = Program()
    d = p.malloc(nbytes)
    s = p.stream_create()
    p.kernel(s, [(d, MODE_W)])
    p.stream_sync(s)
    p.kernel(s, [(d, MODE_RW)])
    drop_at = len(p.ops)
    p.stream_sync(s)                  # the synchronisation the racy listing forgets
    r = p.isend(d, nbytes)
    p.wait(r)
    p.stream_sync(s)
    w = Workload("config1", p, droppable=[drop_at], n_drop=1, racy_seed=2001)
    w.meta = dict(buffer=d, nbytes=nbytes)
    return w


# ---------------------------------------------------------------------------------------------
# config 2: Jacobi halo exchange, one rank's view
# ---------------------------------------------------------------------------------------------
def config2(nx: int = 4096, ny: int = 4096, iters: int = 100, seed: int = 1002) -> Workload:
    """Per iteration: 4 pack kernels on S2 (R A, W send_k); interior on S1
    (R A, W B); StreamSync(S2); 4 Irecv (W recv_k) + 4 Isend (R send_k); Waitall; 4 unpack on S1
    (R recv_k, W B); boundary on S1 (W B); residual on S1 (R A, R B, W partial); reduce on S1
    (R partial, W d_norm); cudaMemcpy D2H of d_norm (legacy stream, synchronous); swap A, B.
    12 kernels per iteration as in Table I.  The racy twin drops the StreamSync(S2)
    of 5 seeded iterations (pack → Isend race on the send buffers)."""
    p = Program()
    grid = nx * ny * 4
    halo = max(nx, ny) * 4
    A = p.malloc(grid)
    B = p.malloc(grid)
    send = [p.malloc(halo) for _ in range(4)]
    recv = [p.malloc(halo) for _ in range(4)]
    partial = p.malloc(max(nx, 256) * 4)
    d_norm = p.malloc(256)
    h_norm = p.malloc(256, kind=MEM_PINNED)
    s1 = p.stream_create()
    s2 = p.stream_create()
    drops = []
    for _ in range(iters):
        for k in range(4):
            p.kernel(s2, [(A, MODE_R), (send[k], MODE_W)])
        p.kernel(s1, [(A, MODE_R), (B, MODE_W)])
        drops.append(len(p.ops))
        p.stream_sync(s2)
        reqs = [p.irecv(recv[k], halo) for k in range(4)] + [p.isend(send[k], halo) for k in range(4)]
        for r in reqs:
            p.wait(r)
        for k in range(4):
            p.kernel(s1, [(recv[k], MODE_R), (B, MODE_W)])
        p.kernel(s1, [(B, MODE_W)])
        p.kernel(s1, [(A, MODE_R), (B, MODE_R), (partial, MODE_W)])
        p.kernel(s1, [(partial, MODE_R), (d_norm, MODE_W)])
        p.memcpy(h_norm, d_norm, 4, CPY_D2H)
        A, B = B, A
    return Workload("config2", p, droppable=drops, n_drop=5, racy_seed=2002,
                    meta=dict(nx=nx, ny=ny, iters=iters))


# ---------------------------------------------------------------------------------------------
# dependency-tracking helper for the DAG workloads (configs 3 and 5)
# ---------------------------------------------------------------------------------------------
class _DagSync:
    """Tracks, per allocation, the last writer and the readers since, and emits the waits a
    correctly synchronised program needs before an operation (kernels: StreamWaitEvent on the
    producer's event; MPI: host EventSynchronize before the call, MPI_Wait before a later use).
    Knowledge is tracked conservatively (host-known and per-stream-known launch indices); any
    over-synchronisation only adds sync calls."""

    def __init__(self, p: Program, streams: list[int], ring: int, rng: np.random.Generator):
        self.p = p
        self.streams = streams
        self.ring = ring
        self.rng = rng
        self.launch_stream: list[int] = []
        self.launch_count = {s: 0 for s in streams}
        self.slot_owner: dict[int, int] = {}          # event handle -> launch index it captures
        self.launch_event: list[int] = []
        self.events = {s: [p.new_event() for _ in range(ring)] for s in streams}
        self.last_on_stream = {s: -1 for s in streams}
        self.host_known = {s: -1 for s in streams}    # max launch index per stream known to host
        self.stream_known = {s: {t: -1 for t in streams} for s in streams}
        self.writer: dict[int, tuple] = {}            # alloc -> ('k', launch) | ('r', req)
        self.readers: dict[int, list] = {}
        self.open_reqs: list[int] = []
        self.droppable: list[int] = []

    # a stream s must be ordered after launch L
    def _need_launch(self, s: int | None, L: int):
        t = self.launch_stream[L]
        if s is not None and t == s:
            return
        if self.host_known[t] >= L:
            return
        if s is not None and self.stream_known[s][t] >= L:
            return
        ev = self.launch_event[L]
        if self.slot_owner.get(ev) != L:
            ev = self.launch_event[self.last_on_stream[t]]
            L = self.last_on_stream[t]
        self.droppable.append(len(self.p.ops))
        if s is None:
            self.p.event_sync(ev)
            self.host_known[t] = max(self.host_known[t], L)
        else:
            self.p.stream_wait_event(s, ev)
            self.stream_known[s][t] = max(self.stream_known[s][t], L)

    def _need_req(self, r: int):
        if r in self.open_reqs:
            self.p.wait(r)
            self.open_reqs.remove(r)

    def _need(self, s, dep):
        kind, v = dep
        if kind == "k":
            self._need_launch(s, v)
        else:
            self._need_req(v)

    def deps(self, alloc: int, write: bool) -> list:
        out = []
        if alloc in self.writer:
            out.append(self.writer[alloc])
        if write:
            out.extend(self.readers.get(alloc, []))
        return out

    def launch(self, s: int, reads: list[int], writes: list[int], sizes: dict | None = None):
        for a in reads:
            for d in self.deps(a, False):
                self._need(s, d)
        for a in writes:
            for d in self.deps(a, True):
                self._need(s, d)
        self.p.kernel(s, [(a, MODE_R) for a in reads] + [(a, MODE_W) for a in writes])
        L = len(self.launch_stream)
        self.launch_stream.append(s)
        k = self.launch_count[s]
        self.launch_count[s] += 1
        ev = self.events[s][k % self.ring]
        self.p.event_record(ev, s)
        self.slot_owner[ev] = L
        self.launch_event.append(ev)
        self.last_on_stream[s] = L
        for a in reads:
            self.readers.setdefault(a, []).append(("k", L))
        for a in writes:
            self.writer[a] = ("k", L)
            self.readers[a] = []
        return L

    def mpi(self, alloc: int, off: int, n: int, send: bool, max_open: int):
        if len(self.open_reqs) >= max_open:
            self._need_req(self.open_reqs[0])
        for d in self.deps(alloc, not send):
            self._need(None, d)
        r = self.p.isend(alloc + off, n) if send else self.p.irecv(alloc + off, n)
        self.open_reqs.append(r)
        if send:
            self.readers.setdefault(alloc, []).append(("r", r))
        else:
            self.writer[alloc] = ("r", r)
            self.readers[alloc] = []
        return r

    def device_sync(self):
        self.p.device_sync()
        for s in self.streams:
            self.host_known[s] = self.last_on_stream[s]


# ---------------------------------------------------------------------------------------------
# config 3: multi-stream event DAG
# ---------------------------------------------------------------------------------------------
def config3(nbuf: int = 64, buf_size: int = 16 * MiB, launches: int = 10_000, nstreams: int = 8,
            sync_every: int = 1000, seed: int = 1003) -> Workload:
    """64 × 16 MiB buffers; launches round-robin over 8 user streams, each reading 2 and writing 1
    random buffer (whole allocations); StreamWaitEvent on the producers' events before, EventRecord
    after (events recycled from a per-stream ring of 4, so re-recording is exercised);
    DeviceSynchronize every 1k launches.  Racy twin: drop 10 seeded StreamWaitEvents."""
    rng = np.random.default_rng(seed)
    p = Program()
    bufs = [p.malloc(buf_size) for _ in range(nbuf)]
    streams = [p.stream_create() for _ in range(nstreams)]
    dag = _DagSync(p, streams, ring=4, rng=rng)
    for i in range(launches):
        s = streams[i % nstreams]
        pick = rng.choice(nbuf, size=3, replace=False)
        dag.launch(s, [bufs[pick[0]], bufs[pick[1]]], [bufs[pick[2]]])
        if (i + 1) % sync_every == 0:
            dag.device_sync()
    dag.device_sync()
    return Workload("config3", p, droppable=dag.droppable, n_drop=10, racy_seed=2003,
                    meta=dict(nbuf=nbuf, buf_size=buf_size, launches=launches))


# ---------------------------------------------------------------------------------------------
# config 4: large tracked memory (the paper's high-overhead regime)
# ---------------------------------------------------------------------------------------------
def config4(nalloc: int = 16, alloc_size: int = 1 * GiB, launches: int = 1000, nstreams: int = 3,
            seed: int = 1004) -> Workload:
    """16 × 1 GiB allocations; launch i on user stream i mod 3 annotates all 16 allocations, W on
    the 4 selected by i mod 4 and R on the other 12; launch i waits on launch i−1's event (chain).
    Racy twin: drop 3 chain waits.  Cost ∝ tracked bytes as in Fig. 12."""
    p = Program()
    bufs = [p.malloc(alloc_size) for _ in range(nalloc)]
    streams = [p.stream_create() for _ in range(nstreams)]
    ev_prev = None
    drops = []
    per = max(1, nalloc // 4)
    for i in range(launches):
        s = streams[i % nstreams]
        if ev_prev is not None:
            drops.append(len(p.ops))
            p.stream_wait_event(s, ev_prev)
        wsel = set(range((i % 4) * per, (i % 4) * per + per))
        p.kernel(s, [(b, MODE_W if j in wsel else MODE_R) for j, b in enumerate(bufs)])
        ev = p.new_event()
        p.event_record(ev, s)
        ev_prev = ev
    p.device_sync()
    return Workload("config4", p, droppable=drops, n_drop=3, racy_seed=2004,
                    meta=dict(nalloc=nalloc, alloc_size=alloc_size, launches=launches))


# ---------------------------------------------------------------------------------------------
# config 5: scaling sweep
# ---------------------------------------------------------------------------------------------
def config5(total: int = 64 * GiB, lo: int = 1 * MiB, hi: int = 1 * GiB, launches: int = 4000,
            nstreams: int = 30, n_nonblocking: int = 6, mpi_lo: int = 64 * KiB, mpi_hi: int = 1 * MiB,
            max_open: int = 32, seed: int = 1005) -> Workload:
    """64 GiB of allocations with log-uniform sizes in [1 MiB, 1 GiB]; 30 user streams (6 of them
    non-blocking) + up to 32 MPI-request fibers + host + legacy stream = 64 fibers; 4k launches each
    reading 6 and writing 2 whole allocations; one CUDA-aware MPI_Isend/Irecv on a 64 KiB–1 MiB
    sub-range per launch (≤ 32 outstanding); DAG synchronisation as in config 3 plus MPI_Wait and
    host EventSynchronize; a synchronous D2H cudaMemcpy of a scalar every 500 launches (legacy
    default-stream barrier).  Racy twin: drop 20 seeded sync calls."""
    rng = np.random.default_rng(seed)
    p = Program()
    sizes = []
    acc = 0
    while True:
        sz = int(math.exp(rng.uniform(math.log(lo), math.log(hi)))) // 256 * 256
        if acc + sz > total:
            break
        sizes.append(sz)
        acc += sz
    bufs = [p.malloc(sz) for sz in sizes]
    size_of = dict(zip(bufs, sizes))
    h_scalar = p.malloc(256, kind=MEM_PINNED)
    streams = [p.stream_create(nonblocking=(i < n_nonblocking)) for i in range(nstreams)]
    dag = _DagSync(p, streams, ring=4, rng=rng)
    nb = len(bufs)
    for i in range(launches):
        s = streams[int(rng.integers(nstreams))]
        pick = rng.choice(nb, size=8, replace=False)
        dag.launch(s, [bufs[j] for j in pick[:6]], [bufs[j] for j in pick[6:]])
        # one CUDA-aware MPI op on a sub-range of a random allocation
        a = bufs[int(rng.integers(nb))]
        n = int(math.exp(rng.uniform(math.log(mpi_lo), math.log(mpi_hi)))) // 256 * 256
        n = min(n, size_of[a])
        off = int(rng.integers(0, (size_of[a] - n) // 256 + 1)) * 256
        dag.mpi(a, off, n, send=bool(rng.integers(2)), max_open=max_open)
        if (i + 1) % 500 == 0:
            src = bufs[int(rng.integers(nb))]
            for d in dag.deps(src, False):
                dag._need(None, d)
            p.memcpy(h_scalar, src, 8, CPY_D2H)
    for r in list(dag.open_reqs):
        dag._need_req(r)
    dag.device_sync()
    return Workload("config5", p, droppable=dag.droppable, n_drop=20, racy_seed=2005,
                    meta=dict(total=acc, nalloc=nb, launches=launches))


# ---------------------------------------------------------------------------------------------
# presets: "full" = BASELINE.json sizes; "small" = same structure, sizes the oracle finishes in
# seconds (several kernel tiles and a ragged tail per allocation)
# ---------------------------------------------------------------------------------------------
def make(config: int, size: str = "full") -> Workload:
    full = size == "full"
    if config == 1:
        return config1()
    if config == 2:
        return config2() if full else config2(nx=200, ny=136, iters=12)
    if config == 3:
        return config3() if full else config3(buf_size=24 * KiB + 1016, launches=600, sync_every=100)
    if config == 4:
        return config4() if full else config4(alloc_size=40 * KiB + 264, launches=60)
    if config == 5:
        return (config5() if full else
                config5(total=24 * MiB, lo=16 * KiB, hi=3 * MiB, launches=300, mpi_lo=1 * KiB,
                        mpi_hi=16 * KiB))
    raise ValueError(f"unknown config {config}")
