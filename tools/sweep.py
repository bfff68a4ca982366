"""Runs bench.py over the configs[1] sweep points (SuiteSparse-shaped: power-law and banded,
n = 65k..1M, avg degree 8..64, F = 128, 1:2:4 / 64:2:8 / 128:2:16) and writes one JSON line
per point plus a summary table.  The headline bench line is a single point of this sweep.

    python tools/sweep.py [out.jsonl]
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

POINTS = [
    "c2-banded-n65k-d8-f128-1:2:4",
    "c2-banded-n262k-d8-f128-1:2:4",
    "c2-banded-n1m-d16-f128-1:2:4",
    "c2-banded-n1m-d32-f128-1:2:4",
    "c2-banded-n262k-d64-f128-1:2:4",
    "c2-banded-n262k-d16-f128-64:2:8",
    "c2-banded-n262k-d16-f128-128:2:16",
    "c2-powerlaw-n65k-d8-f128-1:2:4",
    "c2-powerlaw-n262k-d16-f128-1:2:4",
    "c2-powerlaw-n262k-d16-f128-128:2:16",
    "c2-powerlaw-n262k-d64-f128-64:2:8",
    "c2-powerlaw-n1m-d16-f128-1:2:4",
]


def main():
    out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "sweep_c2.jsonl")
    rows = []
    with open(out, "w") as f:
        for wl in POINTS:
            r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--workload", wl, "--steps", "30",
                                "--warmup", "3", "--no-cpu"], capture_output=True, text=True, timeout=1200)
            line = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
            if not line:
                print(wl, "FAILED", r.stderr[-500:], flush=True)
                continue
            d = json.loads(line[-1])
            f.write(json.dumps(d) + "\n")
            f.flush()
            pre = d["preprocess"]
            cus = d.get("cusparse") or {}
            row = (wl, d["value"], d["roofline"]["frac"], cus.get("gflops"), d.get("speedup_vs_cusparse"),
                   pre["slots_per_nnz"], pre["residual_nnz"], pre["violation_removal"])
            rows.append(row)
            print("%-38s %9.0f GF/s  roof %.2f  cuSPARSE %s  x%s  slots/nnz %.1f  resid %d  removal %s" %
                  (row[0], row[1], row[2], "%.0f" % row[3] if row[3] else "-",
                   "%.2f" % row[4] if row[4] else "-", row[5], row[6], row[7]), flush=True)


if __name__ == "__main__":
    main()
