"""Rewrite BASELINE.md's per-config measurement table from profiles/r01_configs/*.json (dev aid)."""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
p = os.path.join(ROOT, "BASELINE.md")
s = open(p).read()
a = s.index("| config | twin | windows | checked (value) |")
b = s.index('"frac" is of the measured copy bandwidth')
rows = ["| config | twin | windows | checked (value) | kernel DRAM | frac | e2e pipelined (serial) | race granules / runs | oracle | f3 (context) |",
        "|---|---|---|---|---|---|---|---|---|---|"]


def tb(x):
    return f"{x / 1e3:.1f} TB/s"


for c in (2, 3, 4, 5):
    for tw in ("racy", "clean"):
        d = json.load(open(os.path.join(ROOT, f"profiles/r01_configs/bench_config{c}_{tw}.json")))
        r, e, cpu = d["roofline"], d["e2e"], d.get("cpu_baseline")
        one = d["config"]["windows"] == 1
        kd = ("— (one window: no shadow traffic)" if tw == "racy" else "—") if one else f"{r['achieved']:,.0f} GB/s"
        fr = "—" if one else f"{r['frac']:.2f}"
        oc = f"{cpu['value']:.2f} GB/s ({cpu['cores']} cores)" if cpu else "—"
        row = [str(c), tw, str(d["config"]["windows"]), tb(d["value"]), kd, fr,
               f"{tb(e['value'])} ({tb(e['serial']['value'])})",
               f"{d['config']['race_granules']:,} / {d['config']['race_runs']}", oc,
               f"{d['interval_compressed']['value'] / 1e6:.2f} PB/s"]
        if c == 5 and tw == "racy":
            row = [f"**{x}**" if i in (0, 1, 3, 4, 5, 6) else x for i, x in enumerate(row)]
        rows.append("| " + " | ".join(row) + " |")
s = s[:a] + "\n".join(rows) + "\n\n" + s[b:]
open(p, "w").write(s)
