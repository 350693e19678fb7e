set -e
for mode in "" "--dense"; do
  for spec in "3 3 2000" "3 30 1000" "3 300 100" "5 8 1000" "5 64 500" "5 512 71" "5 4096 9"; do
    set -- $spec
    python tools/session_bench.py --config $1 --chunk $2 --max-calls $3 --summary $mode >> gpurun_out/sessions_r02.jsonl
    python tools/session_bench.py --config $1 --chunk $2 --max-calls $3 --pipelined $mode >> gpurun_out/sessions_r02.jsonl
  done
done
