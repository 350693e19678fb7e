CUSAN_DEBUG_TIMING=1 timeout 600 python tools/e2e_breakdown.py --config 4 --steps 3 2>&1 | grep "workspace=torch\|cusan_plan_run" | head -8
