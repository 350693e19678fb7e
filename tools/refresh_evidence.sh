# Round-end evidence on one B200 (outputs in gpurun_out/, copied to profiles/ by hand):
# the bench line (N=1), configs 2-4, session sweeps and per-call latency, the ncu launch list of the
# bench command and the ncu --set full capture of the dense K1.
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/ev_smoke.log 2>&1
python bench.py --steps 20 --warmup 5 > gpurun_out/ev_bench.json 2> gpurun_out/ev_bench.err
for c in 2 3 4; do python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ev_config$c.json 2>/dev/null; done
rm -f gpurun_out/sessions_r02.jsonl gpurun_out/lat.jsonl
bash tools/session_sweep.sh
bash tools/session_latency.sh > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/ev_launches.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ev_ncu_launches.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_plan.csv \
    python tools/profile_plan.py --config 5 > gpurun_out/ev_ncu_plan.log 2>&1
python tools/profile_k1.py --nshards 1 --runs 1 > gpurun_out/ev_k1_plain.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:shadow_check_window --launch-skip 9 --launch-count 9 \
    -o gpurun_out/ev_k1_dense -f python tools/profile_k1.py --nshards 1 --runs 1 > gpurun_out/ev_ncu_k1.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:shadow_check_window --launch-skip 9 --launch-count 9 \
    -o gpurun_out/ev_k1_compressed -f python tools/profile_k1.py --nshards 1 --runs 1 --compressed > gpurun_out/ev_ncu_k1c.log 2>&1
echo done
