"""Runs bench.py over configs[1] sweep points (SuiteSparse-shaped: power-law and banded,
n = 65k..1M, avg degree 8..64, F = 128, 1:2:4 / 64:2:8 / 128:2:16) and writes one JSON line
per point plus a summary table.  The headline bench line is a single point of this sweep.

    python tools/sweep.py [out.jsonl] [point ...]
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# each point: a bench workload, optionally followed by bench flags (e.g. "--gain-rule 1")
POINTS = [
    "c2-banded-n65k-d8-f128-1:2:4",
    "c2-banded-n262k-d8-f128-1:2:4",
    "c2-banded-n1m-d16-f128-1:2:4",
    "c2-banded-n1m-d16-f128-1:2:4-tau0",
    "c2-banded-n1m-d32-f128-1:2:4",
    "c2-banded-n262k-d64-f128-1:2:4",
    "c2-banded-n262k-d16-f128-64:2:8",
    "c2-banded-n262k-d16-f128-128:2:16",
    "c2-powerlaw-n65k-d8-f128-1:2:4",
    "c2-powerlaw-n262k-d16-f128-1:2:4",
    "c2-powerlaw-n262k-d16-f128-1:2:4-tau0",
    "c2-powerlaw-n262k-d16-f128-128:2:16",
    "c2-powerlaw-n262k-d64-f128-64:2:8",
    "c2-powerlaw-n1m-d16-f128-1:2:4",
    # violation removal under the positive-only gain rule (SURVEY §8(c) decision: both rules)
    "c2-banded-n65k-d16-f128-64:2:8",
    "c2-banded-n65k-d16-f128-64:2:8 --gain-rule 1",
    "c2-powerlaw-n65k-d8-f128-1:2:4 --gain-rule 1",
]


def main():
    out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "sweep_c2.jsonl")
    points = sys.argv[2:] or POINTS
    with open(out, "w") as f:
        for spec in points:
            wl, *extra = spec.split(" ")
            r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--workload", wl, "--steps", "30",
                                "--warmup", "3", "--no-cpu"] + extra, capture_output=True, text=True, timeout=1800)
            line = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
            if not line:
                print(wl, "FAILED", r.stderr[-800:], flush=True)
                continue
            d = json.loads(line[-1])
            d["sweep_args"] = extra
            f.write(json.dumps(d) + "\n")
            f.flush()
            pre = d["preprocess"]
            cus = d.get("cusparse") or {}
            rf = d["roofline"]
            ks = " ".join("%s %.3fms/%s %.2f" % (k.replace("k_", ""), v["ms"], v["bound"], v["frac"])
                          for k, v in rf["kernels"].items())
            print("%-40s %-16s %8.0f GF/s  cuSPARSE %6s  x%5s  tau %-4d slots/nnz %6.1f  sptc-share %.2f  removal %s  "
                  "layout %s  [%s]" %
                  (wl, " ".join(extra), d["value"], "%.0f" % cus["gflops"] if cus.get("gflops") else "-",
                   "%.2f" % d["speedup_vs_cusparse"] if d.get("speedup_vs_cusparse") else "-",
                   d["config"]["tau"], pre["slots_per_nnz"], pre["sptc_share_of_nnz"],
                   "%.3f" % pre["violation_removal"] if pre["violation_removal"] is not None else "n/a",
                   d["config"].get("layout"), ks), flush=True)


if __name__ == "__main__":
    main()
