"""Lowering (a0) and clocks (a1, cusan_clocks_compute) of the full-size config-5 trace, 5 repetitions:
    CUSAN_DEBUG_TIMING=1 python tools/a1_timing.py   (CUSAN_A1_COLUMNS=1: the two-pass column form)"""
import time, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs
w = configs.make(5, 'full')
ops, args = w.arrays(True)
for i in range(5):
    t0=time.perf_counter(); tr = cs.Trace(255); cs.Lowering(tr).cusan_lower_program(ops, args); t1=time.perf_counter()
    c = cs.Clocks.compute(tr); t2=time.perf_counter()
    print(f"lower {1e3*(t1-t0):.2f} ms clocks {1e3*(t2-t1):.2f} ms")
