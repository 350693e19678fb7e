# A/B of K1 builds on one B200: build/libcusan_head.so (the committed kernel) against the working tree
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2; do
  CUSAN_LIBRARY=$PWD/build/libcusan_head.so python tools/compressed_timing.py 3,5
  python tools/compressed_timing.py 3,5
done
CUSAN_LIBRARY=$PWD/build/libcusan_head.so python tools/session_latency.py --config 5 --chunk 8 --calls 600
python tools/session_latency.py --config 5 --chunk 8 --calls 600
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
