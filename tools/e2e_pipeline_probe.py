import sys, time, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs
racy = sys.argv[1] == "racy"
w = configs.make(5, "full"); ops, args = w.arrays(racy)
def make(i):
    t = cs.Trace(255); cs.Lowering(t).cusan_lower_program(ops, args); return t
stream = torch.cuda.current_stream()
for rep in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter(); ts = []
    for tr, r in cs.pipelined_checks(make, 8, window_events=4096, stream=stream.cuda_stream):
        ts.append(time.perf_counter() - t0)
    print("pipelined", [round(1e3*(b-a),1) for a, b in zip([0]+ts[:-1], ts)], "kernel", round(r.counters["kernel_ms"],1), "run_ms", round(r.counters["run_ms"],1), flush=True)
    t0 = time.perf_counter(); ts = []
    for i in range(4):
        r = cs.check(make(0), window_events=4096, stream=stream.cuda_stream, workspace="torch")
        ts.append(time.perf_counter() - t0)
    print("serial", [round(1e3*(b-a),1) for a, b in zip([0]+ts[:-1], ts)], flush=True)
