"""Multi-rank paths on the GPU: two processes (torch.distributed over gloo, both ranks on cuda:0 —
the round's boxes have one GPU) run the sharded one-shot check (ShardedPlan) and the sharded
online session (ShardedSession, check and submit/finish; events recorded on rank 0 and pulled by
rank 1 for check), gather the runs and compare rank 0's
merged reports with the oracle.  The NCCL launch differs only in the process group backend and
the device of the gathered tensors."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_sc_huckzsjb24_b200 as cs
        from paper_conf_sc_huckzsjb24_b200.dist import ShardedPlan, ShardedSession
        from tracegen import configs
        w = configs.make(5, "small")
        ops, args = w.arrays(True)
        full = cs.Trace(255)
        cs.Lowering(full).cusan_lower_program(ops, args)
        ev = full.cusan_trace_read()
        res = {}
        # one-shot, windowed
        rep = ShardedPlan(full, window_events=97).run()
        # online: four calls, check() and submit()/finish()
        cuts = np.linspace(0, len(ev), 5).astype(int)
        ta, tb = cs.Trace(255), cs.Trace(255)
        sa = ShardedSession(ta, window_events=64, shard_block=1 << 10)
        sb = ShardedSession(tb, window_events=64, shard_block=1 << 10)
        calls_a, calls_b = [], []
        for a, b in zip(cuts[:-1], cuts[1:]):
            if rank == 0:                          # rank 0 records; rank 1 receives (pull)
                ta.cusan_trace_append_events(ev[a:b])
            assert sa.pull() == b - a
            tb.cusan_trace_append_events(ev[a:b])
            calls_a.append(sa.check())
            r = sb.submit()
            if r is not None or rank != 0:
                calls_b.append(r)
        calls_b.append(sb.finish())
        sa.close()
        sb.close()
        if rank == 0:
            ref = oracle.check_events(ev, 256)
            want = ref["runs"].astype(rep.runs.dtype)
            res["plan"] = rep.n_race_granules == ref["n_race_granules"] > 0 and np.array_equal(rep.runs, want)
            for name, calls in (("session", calls_a), ("submit", calls_b)):
                merged = cs.report_merge(np.concatenate([c.runs for c in calls]),
                                         sum(c.n_race_granules for c in calls))
                res[name] = (len(calls) == 4 and merged.n_race_granules == ref["n_race_granules"]
                             and np.array_equal(merged.runs, want))
        else:
            res["others_none"] = rep is None and all(c is None for c in calls_a + calls_b)
        q.put((rank, res))
    except Exception as e:                         # pragma: no cover - reported to the parent
        q.put((rank, {"error": repr(e)}))
    finally:
        dist.destroy_process_group()


def test_two_ranks_sharded_plan_and_sessions_on_gpu():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0] == {"plan": True, "session": True, "submit": True}, res
    assert res[1] == {"others_none": True}, res


def _nccl_worker(port, q):
    import sys
    sys.path.insert(0, ROOT)
    import torch
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        import oracle
        import paper_conf_sc_huckzsjb24_b200 as cs
        from paper_conf_sc_huckzsjb24_b200.dist import ShardedPlan, ShardedSession, broadcast_trace
        from tracegen import configs
        w = configs.make(5, "small")
        ops, args = w.arrays(True)
        tr = cs.Trace(255)
        cs.Lowering(tr).cusan_lower_program(ops, args)
        ev = tr.cusan_trace_read()
        ref = oracle.check_events(ev, 256)
        got = broadcast_trace(tr, device=dev)
        rep = ShardedPlan(got, comm_device=dev, window_events=97).run()
        res = {"plan": rep.n_race_granules == ref["n_race_granules"] > 0
               and np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))}
        t2 = cs.Trace(255)
        ses = ShardedSession(t2, comm_device=dev, window_events=64)
        t2.cusan_trace_append_events(ev)
        res["pull"] = ses.pull() == len(ev)
        r2 = ses.check()
        ses.close()
        res["session"] = r2.n_race_granules == ref["n_race_granules"] and np.array_equal(r2.runs, rep.runs)
        q.put(res)
    except Exception as e:                         # pragma: no cover - reported to the parent
        q.put({"error": repr(e)})
    finally:
        dist.destroy_process_group()


def test_nccl_collectives_on_one_gpu():
    """The NCCL code path of the multi-GPU check (CUDA tensors in broadcast_trace, gather_runs,
    ShardedPlan, ShardedSession.pull) in a one-rank NCCL group — the only NCCL group a one-GPU box
    can form; the multi-rank logic itself is covered over gloo above."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_worker, args=(_free_port(), q))
    p.start()
    res = q.get(timeout=300)
    p.join(timeout=60)
    assert p.exitcode == 0
    assert res == {"plan": True, "pull": True, "session": True}, res
