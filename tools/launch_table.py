"""Markdown table of an ncu launch list (`ncu --metrics gpu__time_duration.sum --csv --log-file F`):
launches, total time and share per kernel, optionally only the second half of the launches (the
warm step of a two-step run).

    python tools/launch_table.py gpurun_out/launches.csv [--second-half] [--title T] [--cmd C]
"""
import argparse
import csv
from collections import defaultdict

ap = argparse.ArgumentParser()
ap.add_argument("csv")
ap.add_argument("--second-half", action="store_true", help="summarise the second half of the launches only")
ap.add_argument("--title", default="ncu launch list")
ap.add_argument("--cmd", default="")
a = ap.parse_args()

rows = []
hdr = None
for r in csv.reader(open(a.csv)):
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(d["Metric Unit"], 1.0)
        name = d["Kernel Name"].split("(")[0].replace("<unnamed>::", "").replace("void ", "")
        if name.startswith("cub::"):
            name = name.split("<")[0]                # CUB's policy templates: the kernel's name only
        name = name.replace("shadow_check_window<1>", "shadow_check_window<TMA>").replace(
            "shadow_check_window<0>", "shadow_check_window<compressed>")
        rows.append((name, float(d["Metric Value"].replace(",", "")) * scale))
if a.second_half:
    rows = rows[len(rows) // 2:]
agg = defaultdict(lambda: [0, 0.0])
for n, us in rows:
    agg[n][0] += 1
    agg[n][1] += us
total = sum(v[1] for v in agg.values())
print(f"# {a.title}\n")
if a.cmd:
    print(f"`{a.cmd}`\n")
print(f"{len(rows)} launches, {total / 1e3:.3f} ms of kernel time (cold-cache, serialised by ncu: the share is what "
      f"matters).\n")
print("| kernel | launches | total ms | share |\n|---|---|---|---|")
for n, (k, us) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"| {n} | {k} | {us / 1e3:.3f} | {100 * us / total:.2f} % |")
