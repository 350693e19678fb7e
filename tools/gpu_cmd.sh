timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
CUSAN_DEBUG_TIMING=1 timeout 600 python tools/e2e_breakdown.py --config 5 --steps 3 2>&1 | grep "workspace=torch\|build_host_plan" | head -24 | tail -8
