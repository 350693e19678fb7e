import sys, time, torch
sys.path.insert(0, '.')
from paper_conf_sc_huckzsjb24_b200.capture import Capture
Capture._on_memory_deallocation = lambda self, ptr: None      # counterfactual: no reset at dealloc
torch.cuda.synchronize()
s = torch.cuda.Stream()
ptrs = []
with Capture() as cap:
    for i in range(6):
        x = torch.empty(1 << 16, device="cuda"); x.fill_(float(i))
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            y = x * 2
        x.record_stream(s); ptrs.append(x.data_ptr()); del x, y
        time.sleep(0.05)
    torch.cuda.synchronize()
print("counterfactual (no reset at deallocation): reuse", len(set(ptrs)) < len(ptrs), "race granules", cap.check().n_race_granules)
