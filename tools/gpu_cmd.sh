python __graft_entry__.py build > /dev/null
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 1 > gpurun_out/b_ncu.log 2>&1; echo launches rc=$?
timeout 2700 ncu --set full --clock-control none --import-source on -k regex:shadow_check_window --launch-skip 9 -c 9 -o gpurun_out/k1_c5 python tools/profile_k1.py --config 5 --nshards 1 --runs 1 > gpurun_out/ncu_c5.log 2>&1; echo full rc=$?; tail -4 gpurun_out/ncu_c5.log
ls -la gpurun_out/*.ncu-rep
