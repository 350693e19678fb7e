python __graft_entry__.py build > /dev/null
timeout 900 python -m pytest tests/test_gpu_session.py -x -q > gpurun_out/pytest_ses.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_ses.log
for n in 1 2 4 8; do timeout 300 python tools/session_bench.py --config 5 --chunk 4096 --nshards $n > gpurun_out/ses_c5_n$n.json 2>gpurun_out/ses_err_$n.txt; echo n=$n rc=$?; tail -2 gpurun_out/ses_err_$n.txt; python -c "
import json; d=json.load(open('gpurun_out/ses_c5_n$n.json')); d.pop('per_call'); print(d)"; done
