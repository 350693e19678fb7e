timeout 900 python -m pytest tests/test_gpu_session.py -x -q 2>&1 | tail -25
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
