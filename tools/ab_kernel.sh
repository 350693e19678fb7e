# A/B of K1 builds on one B200: build/libcusan_head.so (the committed kernel) against the working tree.
# Make the baseline first (here, no GPU needed):
#   git show HEAD:paper_conf_sc_huckzsjb24_b200/csrc/kernel.cu > /tmp/k/kernel.cu && cd paper_conf_sc_huckzsjb24_b200/csrc &&
#   nvcc <__graft_entry__.NVCC_FLAGS> -I. -o ../../build/libcusan_head.so trace.cpp lower.cpp plan.cpp plan_dev.cu /tmp/k/kernel.cu merge.cu check_api.cpp session.cpp
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2; do
  CUSAN_LIBRARY=$PWD/build/libcusan_head.so python tools/compressed_timing.py 3,5
  python tools/compressed_timing.py 3,5
done
CUSAN_LIBRARY=$PWD/build/libcusan_head.so python tools/session_latency.py --config 5 --chunk 8 --calls 600
python tools/session_latency.py --config 5 --chunk 8 --calls 600
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
