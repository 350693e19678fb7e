python __graft_entry__.py build > /dev/null
timeout 900 python tools/jacobi_sweep.py > gpurun_out/jacobi_sweep.jsonl 2> gpurun_out/jacobi_sweep.err; echo jac rc=$?
for ch in 4096 512; do
timeout 300 python tools/session_bench.py --config 5 --chunk $ch > gpurun_out/ses_seq_$ch.json 2>&1
timeout 300 python tools/session_bench.py --config 5 --chunk $ch --pipelined > gpurun_out/ses_pipe_$ch.json 2>&1
done
for n in 1 2 4 8; do timeout 300 python tools/session_bench.py --config 5 --chunk 4096 --nshards $n > gpurun_out/ses_c5_n$n.json 2>gpurun_out/ses_err_$n.txt; echo n=$n rc=$?; done
