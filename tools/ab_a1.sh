# A/B of a1 forms on one B200: clocks timing and the bench e2e with the one-pass (default) and column (CUSAN_A1_COLUMNS=1) forms
python -c "import __graft_entry__ as g; g.build()" > /dev/null
nproc
echo "== a1 default"; CUSAN_DEBUG_TIMING=1 python tools/a1_timing.py 2>&1 | tail -4
echo "== a1 columns"; CUSAN_A1_COLUMNS=1 CUSAN_DEBUG_TIMING=1 python tools/a1_timing.py 2>&1 | tail -4
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b_fused.json 2>/dev/null
CUSAN_A1_COLUMNS=1 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b_cols.json 2>/dev/null
python - <<'PY'
import json
for n in ("fused","cols"):
    d=json.load(open(f"gpurun_out/b_{n}.json")); ic=d["modes"]["interval_compressed"]
    print(n, "dense e2e", round(d["e2e"]["value"]), "ic e2e ms", round(ic["e2e"]["ms_per_step"],3), "ic breakdown", {k: round(v,3) for k,v in ic["breakdown"].items()})
PY
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
