timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "largest or maximum_fibers or full_size" --durations=6 2>&1 | tail -12
