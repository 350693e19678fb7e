set -x
for spec in "2 2 600" "3 3 600" "5 8 600" "5 64 300" "5 512 71"; do
  set -- $spec
  CUSAN_DEBUG_TIMING=1 python tools/session_latency.py --config $1 --chunk $2 --calls $3 --ticks gpurun_out/ticks_$1_$2.log 2> gpurun_out/ticks_$1_$2.log >> gpurun_out/lat.jsonl
  python tools/session_latency.py --config $1 --chunk $2 --calls $3 >> gpurun_out/lat.jsonl
done
