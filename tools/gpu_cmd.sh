timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -8
for f in 0 4; do for c in 5 4; do timeout 300 python -c "
import sys,time; sys.path.insert(0,'.')
import paper_conf_sc_huckzsjb24_b200 as cs
from tracegen import configs
w=configs.make($c,'full'); ops,args=w.arrays(True); tr=cs.Trace(255); cs.Lowering(tr).cusan_lower_program(ops,args)
p=cs.Plan(tr, window_events=4096, flags=$f, workspace='torch'); p.run(); r=p.run(); c=r.counters
print('config$c flags=$f kernel %.3f ms run %.3f ms checked %.1f TB/s shadow %.3f GB races %d' % (c['kernel_ms'], c['run_ms'], c['tracked_bytes']/c['kernel_ms']/1e9, c['shadow_bytes']/1e9, r.n_race_granules))
"; done; done
timeout 600 python tools/session_bench.py --config 5 --chunk 4096 | cut -c1-600
