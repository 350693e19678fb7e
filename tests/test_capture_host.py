"""Host-side logic of the live capture (f2) without a GPU: thread fibers, torch.distributed
wrapping and restoring.  The recording is the lowering C ABI (host code); only Capture.check()
needs the device, so these tests read the captured primitive trace instead."""
from __future__ import annotations

import threading

import numpy as np
import torch
import torch.distributed as dist

from paper_conf_sc_huckzsjb24_b200.capture import Capture, _Work
from tracegen.program import EV_ACCESS, EV_ACQUIRE, EV_FORK, EV_RELEASE


def test_threads_become_host_fibers_with_create_and_join_edges():
    x = torch.ones(1024)                               # host buffers: MPI-style blocking send/recv
    orig_start, orig_join = threading.Thread.start, threading.Thread.join
    with Capture() as cap:
        cap.send(x)                                     # thread 0 (fiber 0)
        t = threading.Thread(target=lambda: cap.recv(x))
        t.start()
        t.join()
        cap.send(x)
    assert threading.Thread.start is orig_start and threading.Thread.join is orig_join
    ev = cap.trace.cusan_trace_read()
    acc = ev[ev["kind"] == EV_ACCESS]
    fibers = [int(f) for f in acc["fiber"]]
    assert fibers[0] == 0 and fibers[2] == 0 and fibers[1] not in (0, 1)   # the child's own host fiber
    child = fibers[1]
    i_recv = int(np.flatnonzero(ev["kind"] == EV_ACCESS)[1])
    # thread creation: FORK(0 -> child) before the child's access
    forks = np.flatnonzero((ev["kind"] == EV_FORK) & (ev["fiber"] == child) & (ev["a"] == 0))
    assert len(forks) == 1 and forks[0] < i_recv
    # join: the child releases its thread key, thread 0 acquires it, both after the child's access
    rel = np.flatnonzero((ev["kind"] == EV_RELEASE) & (ev["fiber"] == child))
    acq = np.flatnonzero((ev["kind"] == EV_ACQUIRE) & (ev["fiber"] == 0) & (ev["a"] == ev["a"][rel[-1]]))
    assert len(rel) and len(acq) and i_recv < rel[-1] < acq[-1]


def test_distributed_functions_are_wrapped_only_inside():
    import torch.distributed.distributed_c10d as c10d
    names = ("isend", "irecv", "send", "recv", "batch_isend_irecv")
    before = {n: getattr(dist, n) for n in names}
    with Capture():
        for n in names:
            assert getattr(dist, n) is not before[n] and getattr(c10d, n) is getattr(dist, n)
            assert getattr(dist, n).__module__ == "paper_conf_sc_huckzsjb24_b200.capture"
    assert all(getattr(dist, n) is before[n] and getattr(c10d, n) is before[n] for n in names)
    with Capture(intercept_distributed=False):
        assert all(getattr(dist, n) is before[n] for n in names)


class _FakeWork:
    def __init__(self):
        self.waited = 0

    def wait(self, timeout=None):
        self.waited += 1
        return True

    def is_completed(self):
        return True

    def result(self):
        return ["r"]


def test_work_wrapper_records_completion_once():
    with Capture() as cap:
        calls = []
        cap.wait = lambda h: calls.append(h)           # observe the completions
        handles = [("mpi", 1), ("mpi", 2)]
        w1, w2 = _Work(_FakeWork(), cap, handles), _Work(_FakeWork(), cap, handles)   # one batch
        assert w1.is_completed()                       # MPI_Test(success) completes the batch
        w2.wait()
        w1.wait()
        assert calls == [("mpi", 1), ("mpi", 2)]       # each request completed exactly once
        assert w1.result() == ["r"] and w2._work.waited == 1
