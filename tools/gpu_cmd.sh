python __graft_entry__.py build > /dev/null
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench_rc=$?
mkdir -p gpurun_out/r01_configs
for c in 2 3 4 5; do
  timeout 600 python bench.py --config $c > gpurun_out/r01_configs/bench_config${c}_racy.json 2>gpurun_out/r01_configs/err_${c}_racy.txt; echo c=$c racy rc=$?
  timeout 600 python bench.py --config $c --clean --no-cpu-baseline > gpurun_out/r01_configs/bench_config${c}_clean.json 2>gpurun_out/r01_configs/err_${c}_clean.txt; echo c=$c clean rc=$?
done
