mkdir -p gpurun_out
echo "== racecheck"; timeout 1500 compute-sanitizer --tool racecheck --racecheck-report hazard --error-exitcode 9 --print-limit 10 python tools/sanitize_small.py > gpurun_out/sanitizer_racecheck.log 2>&1; echo "exit $?"; tail -3 gpurun_out/sanitizer_racecheck.log
echo "== initcheck (no TMA build)"; CUSAN_LIBRARY=tools/var_notma.so timeout 1500 compute-sanitizer --tool initcheck --error-exitcode 9 --print-limit 10 python tools/sanitize_small.py > gpurun_out/sanitizer_initcheck_notma.log 2>&1; echo "exit $?"; tail -3 gpurun_out/sanitizer_initcheck_notma.log
