timeout 900 python -m pytest tests/test_gpu_session.py -x -q 2>&1 | tail -3
timeout 600 python tools/session_bench.py --config 5 --chunk 4096 > gpurun_out/session_c5_4096.json; cut -c1-300 gpurun_out/session_c5_4096.json
timeout 600 python tools/session_bench.py --config 5 --chunk 512 > gpurun_out/session_c5_512.json; cut -c1-300 gpurun_out/session_c5_512.json
python - <<'P'
import json
d=json.load(open('gpurun_out/session_c5_4096.json'))
for c in d['per_call']: print(round(c['seconds']*1e3,1), round(c['kernel_ms'],1), c['launches'])
P
