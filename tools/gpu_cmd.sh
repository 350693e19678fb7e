python __graft_entry__.py build > /dev/null
timeout 300 python tools/fuzz_campaign.py --minutes 1 --seed 7 > gpurun_out/fuzz_quick.json 2>gpurun_out/fuzz_quick.err; echo rc=$?; tail -3 gpurun_out/fuzz_quick.err; cat gpurun_out/fuzz_quick.json
