"""Live capture of PyTorch programs: the captured trace is checked on the GPU,
compared with the oracle on the same trace, and classified like the paper's racy/fixed pairs —
here the PyTorch forms of Fig. 3 (streams without synchronisation) and Fig. 6A (a non-blocking send
before its wait)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_huckzsjb24_b200.capture import Capture

pytestmark = pytest.mark.gpu


def _parity(cap):
    rep = cap.check()
    ref = oracle.check_events(cap.trace.cusan_trace_read(), 255, threads=2)
    assert rep.n_race_granules == ref["n_race_granules"]
    assert np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))
    return rep


def test_side_stream_without_sync_races():
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with Capture() as cap:
        x = torch.ones(1 << 16, device="cuda")       # written on the default stream
        with torch.cuda.stream(s):
            y = x * 2                                # side stream reads x with no ordering
        torch.cuda.synchronize()
    rep = _parity(cap)
    assert rep.n_race_granules == (1 << 16) * 4 // 8  # the whole storage of x
    assert cap.ops >= 2 and y.shape == x.shape


def test_side_stream_with_wait_stream_is_clean():
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with Capture() as cap:
        x = torch.ones(1 << 16, device="cuda")
        s.wait_stream(torch.cuda.current_stream())   # event record + stream wait
        with torch.cuda.stream(s):
            y = x * 2
        torch.cuda.current_stream().wait_stream(s)
        z = y + x                                    # back on the default stream, ordered
        torch.cuda.synchronize()
    assert _parity(cap).n_race_granules == 0
    assert float(z[0]) == 3.0


def test_write_after_read_across_streams():
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with Capture() as cap:
        x = torch.ones(4096, device="cuda")
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            y = x.sum()                              # side stream reads x
        x.mul_(3)                                    # default stream writes x: unordered
        torch.cuda.synchronize()
    rep = _parity(cap)
    assert rep.n_race_granules == 4096 * 4 // 8
    del y


def test_blocking_copy_orders_host():
    """.cpu() synchronises the stream: a later MPI-style send of the tensor is safe (Fig. 4 rank 0
    with its cudaDeviceSynchronize), a non-blocking send before the wait is not (Fig. 6A)."""
    torch.cuda.synchronize()
    with Capture() as cap:
        x = torch.ones(4096, device="cuda")
        _ = x.cpu()                                  # stream sync
        cap.send(x)                                  # blocking send after the sync: ordered
        h = cap.isend(x)                             # non-blocking send reads x ...
        x.add_(1)                                    # ... while a kernel writes it: Fig. 6A race
        cap.wait(h)
        torch.cuda.synchronize()
    rep = _parity(cap)
    assert rep.n_race_granules == 4096 * 4 // 8 and rep.n_runs == 1


def test_nccl_style_p2p_is_stream_ordered():
    torch.cuda.synchronize()
    with Capture() as cap:
        x = torch.ones(4096, device="cuda")
        h = cap.irecv(x, stream_ordered=True)        # comm stream waits on the current stream
        cap.wait(h)                                  # current stream waits on the comm stream
        x.add_(1)
        torch.cuda.synchronize()
    assert _parity(cap).n_race_granules == 0


def _dist_worker(port, q):
    import os
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    res = {}
    try:
        from paper_conf_sc_huckzsjb24_b200.capture import Capture as Cap
        n = 1 << 14
        for name, fixed in (("racy", False), ("fixed", True)):
            torch.cuda.synchronize()
            with Cap() as cap:
                x = torch.ones(n, device="cuda")
                y = torch.zeros(n, device="cuda")
                ops = [dist.P2POp(dist.isend, x, 0), dist.P2POp(dist.irecv, y, 0)]
                works = dist.batch_isend_irecv(ops)   # recorded by the capture, no manual calls
                if fixed:
                    for w in works:
                        w.wait()                      # current stream waits on the transfer
                x.add_(1)                             # writes the buffer being sent
                s = y.sum()                           # reads the buffer being received
                for w in works:
                    w.wait()
                torch.cuda.synchronize()
            rep = cap.check()
            ref = oracle.check_events(cap.trace.cusan_trace_read(), 255, threads=2)
            res[name] = dict(races=rep.n_race_granules, runs=rep.n_runs,
                             parity=rep.n_race_granules == ref["n_race_granules"]
                             and bool(np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))),
                             value=float(s), patched_back=dist.isend.__module__ == "torch.distributed.distributed_c10d")
        q.put(res)
    except Exception as e:                          # pragma: no cover - reported to the parent
        q.put({"error": repr(e)})
    finally:
        dist.destroy_process_group()


def test_torch_distributed_p2p_is_captured():
    """torch.distributed P2P inside a capture is recorded without manual calls (NCCL semantics in
    a one-rank NCCL group, exchange with itself): a kernel writing the send buffer and one reading
    the receive buffer before the works are waited on race with the transfer (Fig. 6A in
    PyTorch/NCCL form); waiting first orders them."""
    import socket

    import torch.multiprocessing as mp
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_dist_worker, args=(port, q))
    p.start()
    res = q.get(timeout=300)
    p.join(timeout=60)
    assert p.exitcode == 0 and "error" not in res, res
    n = 1 << 14
    assert res["racy"]["parity"] and res["fixed"]["parity"], res
    # racy: (isend read, add_ write) over x and (irecv write, sum read) over y
    assert res["racy"]["races"] == 2 * n * 4 // 8 and res["racy"]["runs"] == 2, res
    assert res["fixed"]["races"] == 0 and res["fixed"]["value"] == n, res
    assert res["racy"]["patched_back"] and res["fixed"]["patched_back"], res


@pytest.mark.parametrize("fixed", [False, True])
def test_host_threads_are_fibers(fixed):
    """A second Python thread issues work on a side stream (f4 in a captured PyTorch program,
    PAPER.md:1202-1218).  Racy: the main thread, told by a host-level event (invisible to the
    device), writes the tensor on the default stream while the side stream's write is unordered
    with it.  Fixed: the default stream waits on the side stream first."""
    import threading
    torch.cuda.synchronize()
    n = 1 << 14
    s = torch.cuda.Stream()
    done = threading.Event()
    with Capture() as cap:
        x = torch.ones(n, device="cuda")

        def work():
            with torch.cuda.stream(s):
                s.wait_stream(torch.cuda.default_stream())   # after x's initialisation
                x.mul_(2)
            done.set()

        t = threading.Thread(target=work)
        t.start()
        done.wait()
        if fixed:
            t.join()
            torch.cuda.current_stream().wait_stream(s)
        x.add_(1)
        t.join()
        torch.cuda.synchronize()
    assert len(cap._tids) == 2                     # two host fibers
    rep = _parity(cap)
    if fixed:
        assert rep.n_race_granules == 0
    else:
        assert rep.n_race_granules == n * 4 // 8 and rep.n_runs == 1
    assert threading.Thread.start.__module__ == "threading"   # patches removed on exit


def test_caching_allocator_reuse_after_record_stream_is_clean():
    """A tensor read on a side stream, handed back with record_stream + del: PyTorch's caching
    allocator reuses its block only after the side stream's work (an event it queries itself, not
    a traced sync), and the next tensor at the same address must start from fresh state — as in
    PyTorch's stream sanitizer, which resets a tensor at deallocation.  Without the per-instance
    ranges the new tensor's default-stream write would race with the old read (a false positive)."""
    import time
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    ptrs = []
    with Capture() as cap:
        for i in range(6):
            x = torch.empty(1 << 16, device="cuda")
            x.fill_(float(i))                                  # default stream writes the block
            s.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(s):
                y = x * 2                                      # side stream reads it
            x.record_stream(s)
            ptrs.append(x.data_ptr())
            del x, y
            time.sleep(0.05)                                   # side stream done (untraced)
        torch.cuda.synchronize()
    assert len(set(ptrs)) < len(ptrs)                          # the allocator did reuse a block
    rep = _parity(cap)
    assert rep.n_race_granules == 0


def test_reused_block_race_is_still_reported_within_an_instance():
    """Per-instance ranges only separate allocation instances: a race inside one instance (the side
    stream reads a tensor the default stream writes, unordered) is reported, and its addresses map
    back to the tensor's device memory (Capture.real_address)."""
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with Capture() as cap:
        x = torch.zeros(1 << 12, device="cuda")
        with torch.cuda.stream(s):
            y = x + 1                                          # unordered with zeros' write
        torch.cuda.synchronize()
    rep = _parity(cap)
    assert rep.n_race_granules == (1 << 12) * 4 // 8
    g0 = int(rep.runs["g_begin"][0])
    assert cap.real_address(8 * g0) == x.untyped_storage().data_ptr()
    del y


@pytest.mark.parametrize("racy", [False, True], ids=["clean", "racy"])
def test_capture_online_session_forgets_released_temporaries(racy):
    """Capture.session(): checked every iteration while the program runs, the calls' reports add up
    to the post-mortem check of the same trace (which equals the oracle's), and the session forgets
    each temporary the caching allocator releases, so its layout stays at the live tensors."""
    torch.cuda.synchronize()
    comp, halo = torch.cuda.Stream(), torch.cuda.Stream()
    n = 256
    with Capture() as cap:
        a = torch.rand(n, n, device="cuda")
        b = torch.zeros(n, n, device="cuda")
        send = torch.zeros(n, device="cuda")
        torch.cuda.synchronize()                     # (the side streams do not wait for stream 0)
        ses = cap.session()
        total, ivs = 0, []
        for it in range(40):
            with torch.cuda.stream(halo):
                if not racy:
                    halo.wait_stream(comp)
                send.copy_(a[1, :] * 1.0)            # a temporary per iteration
            with torch.cuda.stream(comp):
                b[1:-1, 1:-1] = 0.25 * (a[:-2, 1:-1] + a[2:, 1:-1] + a[1:-1, :-2] + a[1:-1, 2:])
                comp.wait_stream(halo)
                b[0, :].copy_(send)
            a, b = b, a
            rep = ses.check()
            total += rep.n_race_granules
            ivs.append(rep.counters["n_intervals"])
        torch.cuda.synchronize()
        ses.close()
    post = _parity(cap)
    assert total == post.n_race_granules
    assert (post.n_race_granules > 0) == racy
    assert len(cap.real) > 100                       # allocation instances the program went through
    assert ivs[-1] < len(cap.real) // 4, ivs         # the layout holds about the live ones
