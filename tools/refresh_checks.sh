# Round-end correctness evidence on one B200: a GPU fuzz campaign against the oracle and
# compute-sanitizer memcheck / racecheck / synccheck over the small workloads (outputs in gpurun_out/).
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python tools/fuzz_campaign.py --minutes 12 --seed 41 > gpurun_out/fuzz_final.json 2> gpurun_out/fuzz_final.err
# (compute-sanitizer was closed on the pool at the end of round 2: the loop below reports that and exits)
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --error-exitcode 9 python tools/sanitize_small.py > gpurun_out/san_$t.log 2>&1
  echo "$t rc $?"
done
