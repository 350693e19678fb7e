# Round-end check on one B200: smoke, the GPU suite, the default bench line, online-session sweeps
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/fc_smoke.log 2>&1; echo "smoke rc $?"
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/fc_gputests.log 2>&1; echo "tests rc $?"; tail -1 gpurun_out/fc_gputests.log
python bench.py > gpurun_out/fc_bench.json 2> gpurun_out/fc_bench.err; echo "bench rc $?"
python bench.py --impl reference > gpurun_out/fc_bench_ref.json 2> gpurun_out/fc_bench_ref.err; echo "ref rc $?"
rm -f gpurun_out/sessions_r02.jsonl gpurun_out/lat.jsonl
bash tools/session_sweep.sh; bash tools/session_latency.sh > /dev/null 2>&1; echo sessions done
