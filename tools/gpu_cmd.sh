python __graft_entry__.py build > /dev/null
timeout 600 python -m pytest tests/test_gpu_dist.py -x -q > gpurun_out/pytest_dist.log 2>&1; echo rc=$?; tail -30 gpurun_out/pytest_dist.log
