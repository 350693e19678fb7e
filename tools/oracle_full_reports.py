"""Full-size oracle reports for the BASELINE configs (test infrastructure: calls only oracle/ and
the seeded generators in tracegen/).

For every config 1-5 at the full BASELINE.json size and each twin, lower the API program with the
oracle's own lowering (``oracle.lower``), run the C oracle over the WHOLE trace (every granule, all
host threads) and store its canonical report under ``tests/golden/full/``:

    config{C}_{racy,clean}.npz   runs (the oracle's RUN_DTYPE), n_race_granules, n_runs,
                                 n_events, n_access, tracked_bytes, events_sha256 (of the oracle's
                                 primitive trace, so a test can check it checks the same trace)

``tests/test_gpu_parity.py::test_full_size_configs_exact`` compares the GPU report of the same
configs with these files bit-exactly.  No value here comes from the CUDA path.

    python tools/oracle_full_reports.py [--configs 2,3,4,5] [--twins racy,clean] [--threads T]
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from oracle.lower import lower  # noqa: E402
from tracegen import configs  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "full")


def events_sha256(ev: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(ev).tobytes()).hexdigest()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="1,2,3,4,5")
    ap.add_argument("--twins", default="racy,clean")
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--out", default=OUT)
    a = ap.parse_args()
    os.makedirs(a.out, exist_ok=True)
    for c in [int(x) for x in a.configs.split(",")]:
        w = configs.make(c, "full")
        for twin in a.twins.split(","):
            ops, args = w.arrays(twin == "racy")
            ev, nf = lower(ops, args)
            t0 = time.perf_counter()
            rep = oracle.check_events(ev, nf, threads=a.threads)
            secs = time.perf_counter() - t0
            path = os.path.join(a.out, f"config{c}_{twin}.npz")
            np.savez_compressed(path, runs=rep["runs"], n_race_granules=rep["n_race_granules"],
                                n_runs=rep["n_runs"], n_events=rep["n_events"], n_access=rep["n_access"],
                                tracked_bytes=rep["tracked_bytes"], max_fibers=nf,
                                events_sha256=events_sha256(ev))
            print(json.dumps({"config": c, "twin": twin, "events": int(len(ev)), "fibers": int(nf),
                              "tracked_bytes": rep["tracked_bytes"], "n_race_granules": rep["n_race_granules"],
                              "n_runs": rep["n_runs"], "oracle_seconds": round(secs, 1),
                              "threads": a.threads, "file": os.path.relpath(path, ROOT)}), flush=True)


if __name__ == "__main__":
    main()
