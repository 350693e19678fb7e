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

import oracle

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


def test_whole_node_check_ngpus(monkeypatch):
    """cusan_check_opts.ngpus: clocks once, one host thread per device checking one
    granule-range shard, runs merged — equal to the oracle for ngpus = 1, and for 2-5 shards mapped
    onto this machine's device(s) (CUSAN_NODE_SHARE_DEVICES, the test hook for a one-GPU box);
    asking for more devices than the node has is CUSAN_ECUDA."""
    import paper_conf_sc_huckzsjb24_b200 as cs
    import torch
    from tracegen import configs
    for c in (3, 5):
        w = configs.make(c, "small")
        ops, args = w.arrays(True)
        tr = cs.Trace(255)
        cs.Lowering(tr).cusan_lower_program(ops, args)
        ref = oracle.check_events(tr.cusan_trace_read(), 256)
        rep = cs.check(tr, ngpus=1, window_events=97)
        assert rep.n_race_granules == ref["n_race_granules"] > 0
        assert np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))
        ndev = torch.cuda.device_count()
        with pytest.raises(cs.CusanError) as e:
            cs.check(tr, ngpus=ndev + 1)
        assert e.value.status == -4
        monkeypatch.setenv("CUSAN_NODE_SHARE_DEVICES", "1")
        for ngpus, flags in ((2, 0), (3, cs.CUSAN_CHECK_DENSE_SHADOW), (5, 0)):
            rep = cs.check(tr, ngpus=ngpus, window_events=97, flags=flags)
            assert rep.n_race_granules == ref["n_race_granules"]
            assert np.array_equal(rep.runs, ref["runs"].astype(rep.runs.dtype))
            assert rep.counters["tracked_bytes_shard"] == rep.counters["tracked_bytes"]
        monkeypatch.delenv("CUSAN_NODE_SHARE_DEVICES")
        with pytest.raises(cs.CusanError):
            cs.check(tr, ngpus=2, nshards=2)                       # ngpus shards by itself


def test_c_example_node_check(tmp_path):
    """examples/node_check.c: a C program checks a trace file on every device of the node through
    cusan_check_opts.ngpus; its runs equal the oracle's."""
    import subprocess
    import __graft_entry__ as g
    import paper_conf_sc_huckzsjb24_b200 as cs
    from tracegen import configs
    from tracegen.program import save_events
    exe = [e for e in g.build_examples() if e.endswith("node_check")][0]
    w = configs.make(5, "small")
    ops, args = w.arrays(True)
    tr = cs.Trace(255)
    cs.Lowering(tr).cusan_lower_program(ops, args)
    ev = tr.cusan_trace_read()
    path = str(tmp_path / "c5.trace")
    save_events(path, ev, 255)
    ref = oracle.check_events(ev, 256)
    want = [f"run {int(r['g_begin'])} {int(r['g_end'])} {int(r['earlier'])} {int(r['later'])}" for r in ref["runs"]]
    for argv, env in (([path], {}), ([path, "3", "64", "dense"], {"CUSAN_NODE_SHARE_DEVICES": "1"})):
        out = subprocess.run([exe, *argv], capture_output=True, text=True, timeout=300,
                             env={**__import__("os").environ, **env})
        assert out.returncode == 0, out.stderr
        lines = out.stdout.splitlines()
        assert f"{ref['n_race_granules']} race granules, {ref['n_runs']} runs" in lines[0]
        assert lines[1:] == want
