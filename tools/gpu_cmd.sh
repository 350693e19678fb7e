python __graft_entry__.py build > /dev/null
timeout 300 python tools/sanitize_small.py 2>&1 | tail -2
for t in memcheck synccheck racecheck; do
timeout 1200 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_small.py > gpurun_out/san_$t.txt 2>&1; echo $t rc=$?; tail -4 gpurun_out/san_$t.txt
done
