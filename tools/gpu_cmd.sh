timeout 900 python tools/shard_scaling.py --config 5 --window 4096 2>&1 | tail -6
timeout 900 python tools/shard_scaling.py --config 4 --window 4096 2>&1 | tail -1
