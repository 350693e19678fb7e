mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -8
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:shadow_check -s 9 -c 9 -o gpurun_out/k1_full_r1 python tools/profile_k1.py --nshards 1 --runs 1 > gpurun_out/ncu_full1.log 2>&1; tail -4 gpurun_out/ncu_full1.log
