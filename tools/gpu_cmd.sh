python __graft_entry__.py build > /dev/null
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --dist-backend gloo > gpurun_out/bench2.json 2> gpurun_out/bench2.err; echo rc=$?; tail -5 gpurun_out/bench2.err; cat gpurun_out/bench2.json
