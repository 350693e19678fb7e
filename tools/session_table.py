"""Markdown tables of the online-session sweeps (development aid): tools/session_sweep.sh lines
(per-call latency, sequential and pipelined throughput, compressed vs dense) and, optionally,
tools/session_latency.py lines (the library's own per-call time and its phases).

    python tools/session_table.py gpurun_out/sessions_r02.jsonl [--latency gpurun_out/lat.jsonl]
"""
import argparse
import json

ap = argparse.ArgumentParser()
ap.add_argument("sweep")
ap.add_argument("--latency", default="")
a = ap.parse_args()

seq, pip = {}, {}
for line in open(a.sweep):
    d = json.loads(line)
    key = (d["config"], d["chunk_accesses"], d["dense"])
    (pip if d.get("pipelined") else seq)[key] = d
print("| config | accesses/call | calls | shadow | per call median / p90 | kernel/call median | checked, sequential "
      "| checked, pipelined |\n|---|---|---|---|---|---|---|---|")
for key in sorted(seq, key=lambda k: (k[0], k[1], k[2])):
    s, p = seq[key], pip.get(key)
    print(f"| {key[0]} | {key[1]} | {s['calls']} | {'dense' if key[2] else 'compressed'} | "
          f"{s['call_ms_median']:.3f} / {s['call_ms_p90']:.3f} ms | {s['kernel_ms_median']:.3f} ms | "
          f"{s['checked_gbs'] / 1e3:.2f} TB/s | {(p['checked_gbs'] / 1e3) if p else float('nan'):.2f} TB/s |")
if a.latency:
    print("\nPer-call phases (`tools/session_latency.py`, compressed; medians, ms; `CUSAN_DEBUG_TIMING` ticks are "
          "cumulative from the call's start):\n")
    print("| config | accesses/call | intervals | Python call | library call | kernel | plan done | uploads queued "
          "| GPU done | report |\n|---|---|---|---|---|---|---|---|---|---|")
    rows = {}
    for line in open(a.latency):
        d = json.loads(line)
        k = (d["config"], d["chunk"])
        r = rows.setdefault(k, {})
        if "ticks_median_ms" in d:
            r["ticks"] = d["ticks_median_ms"]
        else:
            r["plain"] = d
    for k in sorted(rows):
        p, t = rows[k].get("plain"), rows[k].get("ticks", {})
        if not p:
            continue
        print(f"| {k[0]} | {k[1]} | {p['intervals_median']:.0f} | {p['python_call_ms']:.3f} | {p['library_run_ms']:.3f} | "
              f"{p['kernel_ms']:.3f} | {t.get('cusan_session.plan', float('nan')):.3f} | "
              f"{t.get('cusan_session.memory', float('nan')):.3f} | {t.get('cusan_session.check', float('nan')):.3f} | "
              f"{t.get('cusan_session.merge', float('nan')):.3f} |")
