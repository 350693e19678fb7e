"""Ad-hoc timing of the check on each full config (development aid, not the bench)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs

def main(cfgs, windows):
    for c in cfgs:
        w = configs.make(c, "full")
        ops, args = w.arrays(False)
        t0 = time.time(); tr = cs.Trace(255); cs.Lowering(tr).cusan_lower_program(ops, args); t1 = time.time()
        for win in windows:
            t2 = time.time(); plan = cs.Plan(tr, window_events=win); t3 = time.time()
            ks = []
            for _ in range(3):
                r = plan.run(); ks.append((r.counters['kernel_ms'], r.counters['run_ms']))
            ctr = r.counters
            tb = ctr['tracked_bytes']
            k = min(x[0] for x in ks)
            print(f"config{c} win={win} lower {t1-t0:.2f}s plan {t3-t2:.2f}s kernel {k:.2f} ms run {min(x[1] for x in ks):.2f} ms "
                  f"launches {ctr['kernel_launches']} tracked {tb/2**30:.1f} GiB -> {tb/k/1e6:.1f} GB/s checked; "
                  f"cell bytes {ctr['shadow_cell_bytes']/2**30:.2f} GiB -> {ctr['shadow_cell_bytes']/k/1e6:.1f} GB/s; "
                  f"races {r.n_race_granules} intervals {ctr['n_intervals']} inc {ctr['n_incidences']} spans {ctr['n_spans']} segs {ctr['n_segments']}", flush=True)
            plan.close()

if __name__ == "__main__":
    cfgs = [int(x) for x in sys.argv[1].split(",")]
    windows = [int(x) for x in sys.argv[2].split(",")]
    main(cfgs, windows)
