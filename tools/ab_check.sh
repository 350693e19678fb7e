# GPU suite + the bench's device-timed and e2e lines (no CPU baseline): one A/B point for a kernel change
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/b_ab.json 2>/dev/null
python - <<'PY'
import json
d=json.load(open("gpurun_out/b_ab.json")); ic=d["modes"]["interval_compressed"]
print("dense", round(d["value"]), "frac", round(d["roofline"]["frac"],4), "e2e", round(d["e2e"]["value"]))
print("ic device ms", round(ic["ms_per_step"],4), "kernel ms", round(ic["kernel_ms_per_step"],4), "e2e ms", round(ic["e2e"]["ms_per_step"],3), {k: round(v,3) for k,v in ic["breakdown"].items()})
PY
