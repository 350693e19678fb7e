python __graft_entry__.py build > /dev/null
timeout 1800 python tools/fuzz_campaign.py --minutes 25 --seed 11 > gpurun_out/fuzz_campaign.json 2>gpurun_out/fuzz_campaign.err; echo rc=$?; tail -3 gpurun_out/fuzz_campaign.err; python -c "
import json; d=json.load(open('gpurun_out/fuzz_campaign.json')); print({k: d[k] for k in ('cases','checks','mismatches','racy_cases')}); print(d['first_failures'])"
