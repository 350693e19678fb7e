timeout 900 python -m pytest tests/test_gpu_session.py tests/test_gpu_capture.py -x -q 2>&1 | tail -2
CUSAN_DEBUG_TIMING=1 timeout 600 python tools/session_bench.py --config 5 --chunk 4096 2>gpurun_out/sess_dbg.txt > gpurun_out/session_c5_4096.json; cut -c1-330 gpurun_out/session_c5_4096.json
timeout 600 python tools/session_bench.py --config 5 --chunk 512 > gpurun_out/session_c5_512.json; cut -c1-330 gpurun_out/session_c5_512.json
