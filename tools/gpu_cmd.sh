timeout 900 python tools/jacobi_sweep.py > gpurun_out/jacobi_sweep.jsonl 2> gpurun_out/jacobi_sweep.err; echo rc=$?; tail -3 gpurun_out/jacobi_sweep.err; wc -l gpurun_out/jacobi_sweep.jsonl
