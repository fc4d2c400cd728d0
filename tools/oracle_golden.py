#!/usr/bin/env python
"""Write tests/golden/hashes.json: the CPU oracle's verification hash and pair count for
every BASELINE.json configuration at full size, split into eighths.

Calls only ``oracle/`` (test infrastructure) -- no value here comes from the
CUDA path.  Each workload's lookup range [0, T) is cut at the strong-scaling boundaries
floor(r T / 8), r = 0..8 (driver.shard), so the hash of any rank's shard at
N in {1, 2, 4, 8} is a sum of consecutive eighths (floor(r T / 4) = floor(2 r T / 8)).
The hash is an integer sum over lookups, so sums of eighths are exact.

T per workload: tiny 100k, small 17M, large 17M, large-U 100M (BASELINE.json configs[0..3]),
XL 1e9 (configs[4]: 1B lookups; bench.py runs it as 125M per rank, i.e. eighth r is rank r's
range at N = 8).

    python tools/oracle_golden.py [--only XL] [--threads 0]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from xs_workloads import GRID_SEED, GRID_NAMES, LOOKUP_SEED, WORKLOADS  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "hashes.json")
TOTALS = {"tiny": 100_000, "small": 17_000_000, "large": 17_000_000,
          "large-U": 100_000_000, "XL": 1_000_000_000}
PARTS = 8


def eighths(total):
    return [total * r // PARTS for r in range(PARTS + 1)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="")
    ap.add_argument("--threads", type=int, default=0)
    a = ap.parse_args()
    doc = {}
    if os.path.exists(OUT):
        with open(OUT) as f:
            doc = json.load(f)
    doc.setdefault("_about", (
        "CPU-oracle verification hashes (sum of 1 + argmax over the 5 macroscopic channels) and "
        "pair counts, lookup seed %d, grid seed %d, written by tools/oracle_golden.py calling only "
        "oracle/; 'bounds' are floor(r T / 8), hash/pairs[r] cover [bounds[r], bounds[r+1])"
        % (LOOKUP_SEED, GRID_SEED)))
    names = a.only.split(",") if a.only else list(TOTALS)
    for name in names:
        w = WORKLOADS[name]
        T = TOTALS[name]
        t0 = time.time()
        P = oracle.Problem(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED, build_idx=False)
        tb = time.time() - t0
        b = eighths(T)
        hashes, pairs = [], []
        t0 = time.time()
        for r in range(PARTS):
            res = P.run_range(LOOKUP_SEED, b[r], b[r + 1] - b[r], macro=False, threads=a.threads)
            hashes.append(int(res["hash"]))
            pairs.append(int(res["pairs"]))
            print(f"{name} part {r}: [{b[r]}, {b[r + 1]}) hash {hashes[-1]} pairs {pairs[-1]} "
                  f"({time.time() - t0:.0f} s)", flush=True)
        doc[name] = {"n_nuclides": w.n_nuclides, "n_gridpoints": w.n_gridpoints,
                     "grid": GRID_NAMES[w.grid_type], "total": T, "bounds": b,
                     "hash": hashes, "pairs": pairs, "hash_total": sum(hashes),
                     "pairs_total": sum(pairs), "oracle_threads": oracle.max_threads() if not a.threads else a.threads,
                     "oracle_seconds": round(time.time() - t0, 1), "grid_build_seconds": round(tb, 1)}
        del P
        with open(OUT + ".tmp", "w") as f:
            json.dump(doc, f, indent=1)
        os.replace(OUT + ".tmp", OUT)


if __name__ == "__main__":
    main()
