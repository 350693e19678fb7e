"""Summarise an ncu capture of the shadow-check kernel into profiles/ (JSON + markdown).

    python tools/ncu_summary.py REPORT.ncu-rep --algorithmic-bytes B --launches N --tag r01 \
        [--launch-list gpurun_out/launches.csv]

`--algorithmic-bytes` is the total shadow-cell bytes of the captured launches (from the report
counters of the same run, `shadow_cell_bytes`), so traffic / algorithmic can be checked.
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__bytes.sum.per_second", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "smsp__inst_executed.sum", "lts__t_sector_hit_rate.pct", "launch__occupancy_limit_registers"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-6, "us": 1e-3,
         "ms": 1.0, "s": 1e3, "byte/s": 1, "Kbyte/s": 1e3, "Mbyte/s": 1e6, "Gbyte/s": 1e9, "Tbyte/s": 1e12}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, data = rows[0], rows[1], rows[2:]
    res = []
    for d in data:
        m = {}
        for w in WANT:
            if w in h:
                i = h.index(w)
                try:
                    v = float(d[i].replace(",", ""))
                except ValueError:
                    continue
                m[w] = v * SCALE.get(units[i], 1)
        res.append(m)
    return res


def launch_list(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if len(r) > vi:
            agg[r[ki]][0] += 1
            agg[r[ki]][1] += float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1)
    total = sum(v[1] for v in agg.values())
    return {k.split("(")[0]: {"launches": v[0], "ms": v[1], "share": v[1] / total if total else 0}
            for k, v in agg.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("--algorithmic-bytes", type=float, required=True)
    ap.add_argument("--launches", type=int, required=True)
    ap.add_argument("--tag", default="r01")
    ap.add_argument("--launch-list")
    ap.add_argument("--workload", default="")
    a = ap.parse_args()
    ms = raw(a.report)
    n = len(ms)
    dram = [m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"] for m in ms]
    t = [m["gpu__time_duration.sum"] for m in ms]
    summary = {
        "kernel": "shadow_check_window", "workload": a.workload, "captured_launches": n,
        "dram_bytes_per_launch": sum(dram) / n,
        "algorithmic_bytes_per_launch": a.algorithmic_bytes / a.launches,
        "traffic_over_algorithmic": (sum(dram) / n) / (a.algorithmic_bytes / a.launches),
        "duration_ms_per_launch": sum(t) / n,
        "dram_gbs_mean": sum(dram) / (sum(t) / 1e3) / 1e9,
        "per_launch": [{"ms": m["gpu__time_duration.sum"], "dram_read_gb": m["dram__bytes_read.sum"] / 1e9,
                        "dram_write_gb": m["dram__bytes_write.sum"] / 1e9,
                        "dram_tbs": m.get("dram__bytes.sum.per_second", 0) / 1e12,
                        "sm_throughput_pct": m.get("sm__throughput.avg.pct_of_peak_sustained_elapsed"),
                        "warps_active_pct": m.get("sm__warps_active.avg.pct_of_peak_sustained_active")}
                       for m in ms],
        "registers_per_thread": ms[0].get("launch__registers_per_thread"),
        "grid_size": ms[0].get("launch__grid_size"),
    }
    if a.launch_list:
        summary["launch_list"] = launch_list(a.launch_list)
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", "ncu_k1_summary.json"), "w") as f:
        json.dump(summary, f, indent=1)
    with open(os.path.join(ROOT, "profiles", f"ncu_k1_{a.tag}.json"), "w") as f:
        json.dump(summary, f, indent=1)
    print(json.dumps({k: v for k, v in summary.items() if k != "per_launch"}, indent=1))


if __name__ == "__main__":
    main()
