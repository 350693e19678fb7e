mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -2 gpurun_out/bench.err; cat gpurun_out/bench.json
timeout 300 python tools/profile_k1.py --nshards 1 --runs 1 > gpurun_out/profile_plain.log 2>&1; cat gpurun_out/profile_plain.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:shadow_check -s 9 -c 9 -o gpurun_out/k1_full_r01c python tools/profile_k1.py --nshards 1 --runs 1 > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
