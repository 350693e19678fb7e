"""Seeded random inputs for fuzz / brute-force tests (inputs only — no race-check arithmetic)."""
from __future__ import annotations

import numpy as np

from .program import (EV_ACCESS, EV_ACQUIRE, EV_FORK, EV_RELEASE, EV_RELEASE_STORE, EVENT_DTYPE,
                      MEM_DEVICE, MEM_MANAGED, MEM_PINNED, MODE_R, MODE_RW, MODE_W, CPY_D2D, CPY_D2H,
                      CPY_H2D, SYNTH_BASE, Program)


def random_primitive_trace(rng: np.random.Generator, n_events: int, n_fibers: int, n_keys: int,
                           n_granules: int, p_access: float = 0.55, unaligned: bool = False,
                           base: int = SYNTH_BASE) -> np.ndarray:
    """Random TSan-level trace: ACCESS ranges over [0, n_granules) granules, RELEASE / RELEASE_STORE /
    ACQUIRE on n_keys keys and FORK edges between distinct fibers."""
    ev = np.zeros(n_events, EVENT_DTYPE)
    for i in range(n_events):
        f = int(rng.integers(n_fibers))
        u = rng.random()
        if u < p_access:
            g0 = int(rng.integers(n_granules))
            g1 = int(rng.integers(g0 + 1, min(n_granules, g0 + 1 + max(1, n_granules // 2)) + 1))
            addr = base + 8 * g0
            nbytes = 8 * (g1 - g0)
            if unaligned:
                addr += int(rng.integers(8))
                nbytes = max(0, nbytes - int(rng.integers(8)))
            ev[i] = (EV_ACCESS, int(rng.random() < 0.45), 0, f, addr, nbytes)
        else:
            u = rng.random()
            if u < 0.3:
                ev[i] = (EV_RELEASE, 0, 0, f, 1000 + int(rng.integers(n_keys)), 0)
            elif u < 0.45:
                ev[i] = (EV_RELEASE_STORE, 0, 0, f, 1000 + int(rng.integers(n_keys)), 0)
            elif u < 0.8:
                ev[i] = (EV_ACQUIRE, 0, 0, f, 1000 + int(rng.integers(n_keys)), 0)
            else:
                src = int(rng.integers(n_fibers - 1))
                if src >= f:
                    src += 1
                ev[i] = (EV_FORK, 0, 0, f, src, 0)
    return ev


def random_program(rng: np.random.Generator, n_ops: int, n_allocs: int = 3, n_streams: int = 3,
                   alloc_bytes: int = 512, threads: bool | None = None) -> Program:
    """Random CUDA-aware MPI call sequence over a few allocations, blocking and non-blocking
    streams, events and requests (no attempt at correctness: most traces are racy)."""
    p = Program()
    threads_on = rng.random() < 0.4 if threads is None else threads   # host threads / PTDS
    if threads_on and rng.random() < 0.5:
        p.default_stream_mode(True)
    kinds = [MEM_DEVICE, MEM_DEVICE, MEM_MANAGED, MEM_PINNED]
    allocs = [p.malloc(alloc_bytes + 8 * int(rng.integers(0, 16)), kind=kinds[i % len(kinds)])
              for i in range(n_allocs)]
    sizes = dict((a, s) for a, s, _ in p.allocs)
    streams = [0, 1, 2] + [p.stream_create(nonblocking=bool(i % 2)) for i in range(n_streams)]
    if not threads_on:
        streams = [0] + streams[3:]
    live_threads = [0]
    events = [p.new_event() for _ in range(3)]
    open_reqs: list[int] = []

    def sub(a):
        n = sizes[a]
        off = 8 * int(rng.integers(0, n // 8))
        ln = 8 * int(rng.integers(1, (n - off) // 8 + 1))
        return a + off, ln

    for _ in range(n_ops):
        if threads_on and rng.random() < 0.15:       # thread create / switch / join
            u = rng.random()
            if u < 0.4 and len(live_threads) < 4:
                child = max(live_threads) + 1
                p.thread_create(child)
                live_threads.append(child)
            elif u < 0.8:
                p.set_thread(int(rng.choice(live_threads)))
            elif len(live_threads) > 1:
                p.thread_join(int(rng.choice(live_threads[1:])))
            continue
        op = int(rng.integers(16))
        s = streams[int(rng.integers(len(streams)))]
        a = allocs[int(rng.integers(n_allocs))]
        if op <= 3:
            k = int(rng.integers(1, 3))
            pick = rng.choice(n_allocs, size=k, replace=False)
            p.kernel(s, [(allocs[j] + 8 * int(rng.integers(0, 4)), int(rng.integers(3))) for j in pick])
        elif op == 4:
            p.stream_sync(s)
        elif op == 5:
            p.device_sync() if rng.random() < 0.5 else p.stream_query(s, bool(rng.integers(2)))
        elif op == 6:
            p.event_record(events[int(rng.integers(3))], s)
        elif op == 7:
            p.event_sync(events[int(rng.integers(3))])
        elif op == 8:
            p.stream_wait_event(s, events[int(rng.integers(3))])
        elif op == 9:
            b = allocs[int(rng.integers(n_allocs))]
            x, n = sub(a)
            kind = [CPY_H2D, CPY_D2H, CPY_D2D][int(rng.integers(3))]
            if rng.random() < 0.5:
                p.memcpy(x, b, min(n, sizes[b]), kind)
            else:
                p.memcpy_async(x, b, min(n, sizes[b]), kind, s)
        elif op == 10:
            x, n = sub(a)
            p.memset(x, n) if rng.random() < 0.5 else p.memset_async(x, n, s)
        elif op == 11:
            x, n = sub(a)
            p.host_access(x, n, int(rng.integers(2)))
        elif op in (12, 13):
            if len(open_reqs) < 4:
                x, n = sub(a)
                open_reqs.append(p.isend(x, n) if op == 12 else p.irecv(x, n))
        elif op == 14:
            if open_reqs:
                r = open_reqs.pop(int(rng.integers(len(open_reqs))))
                p.wait(r) if rng.random() < 0.7 else p.test(r, True)
        else:
            x, n = sub(a)
            p.send(x, n) if rng.random() < 0.5 else p.recv(x, n)
    for r in open_reqs:
        p.wait(r)
    return p
