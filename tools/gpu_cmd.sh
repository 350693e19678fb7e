mkdir -p gpurun_out/r01_configs
for c in 5 4 3 2; do
  for t in racy clean; do
    fl=""; [ $t = clean ] && fl="--clean"
    cb=""; [ $t = clean ] && cb="--no-cpu-baseline"
    timeout 600 python bench.py --config $c $fl $cb --steps 10 --warmup 3 > gpurun_out/r01_configs/bench_config${c}_$t.json 2> gpurun_out/r01_configs/bench_config${c}_$t.err
    echo "config $c $t rc=$?"
  done
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; cut -c1-300 gpurun_out/bench_reference.json
