python __graft_entry__.py build > /dev/null
for i in 1 2; do
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench_rc=$?; python -c "
import json; d=json.load(open('gpurun_out/bench.json')); print(d['value'], d['e2e']['value'], d['e2e']['serial']['value'])"
done
timeout 600 python tools/e2e_pipeline_probe.py racy 2>&1 | tail -4
