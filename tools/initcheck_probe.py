"""compute-sanitizer initcheck probe (development aid): config 3 small, 40-access windows, dense and
compressed shadow, one check each — run once with the shipped library and once with a build
without the TMA bulk-copy paths (CUSAN_LIBRARY=<variant>) to see whether initcheck's reports come
from reads of cells written by cp.async.bulk stores, which it does not track."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import oracle  # noqa: E402
import paper_conf_sc_huckzsjb24_b200 as cs  # noqa: E402
from tracegen import configs  # noqa: E402

w = configs.make(3, "small")
ops, args = w.arrays(True)
tr = cs.Trace(255)
cs.Lowering(tr).cusan_lower_program(ops, args)
ref = oracle.check_events(tr.cusan_trace_read(), 255)
for flags in (cs.CUSAN_CHECK_DENSE_SHADOW, 0):
    rep = cs.check(tr, window_events=40, flags=flags)
    assert rep.n_race_granules == ref["n_race_granules"]
print("probe ok", os.environ.get("CUSAN_LIBRARY", "shipped library"))
