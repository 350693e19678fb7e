python __graft_entry__.py build > /dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -5 gpurun_out/pytest_gpu.log
timeout 600 python tools/quick_timing.py 2,3,4,5 1024,4096,16384 > gpurun_out/quick2.txt 2>&1; cat gpurun_out/quick2.txt | cut -c1-200
timeout 600 python tools/fuzz_campaign.py --minutes 4 --seed 21 > gpurun_out/fuzz_quick.json 2>gpurun_out/fuzz_quick.err; python -c "
import json; d=json.load(open('gpurun_out/fuzz_quick.json')); print({k: d[k] for k in ('cases','checks','mismatches','racy_cases')}); print(d['first_failures'][:3])"
