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
