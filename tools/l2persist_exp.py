"""Experiment: does keeping X persisting in L2 (nm_l2_persist) speed up nm_spmm on the GNN
shapes?  Times nm_spmm with the L2 flushed between reps, without and with the persisting
window (the flush cannot evict persisting lines, so the 'with' numbers also keep X across reps).
usage: python tools/l2persist_exp.py [workload ...]"""
import json
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_ppopp_chensz0s25_b200 import api, graphs  # noqa: E402


def timed(fn, flush, reps=20):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        ts.append((a, b))
    torch.cuda.synchronize()
    return statistics.median(x.elapsed_time(y) for x, y in ts)


def main():
    wls = sys.argv[1:] or ["c3-reddit-f128-1:2:4", "c4-proteins-f256-128:2:16"]
    dev = torch.device("cuda:0")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    for wl in wls:
        w = bench.parse_workload(wl)
        ip, ic = graphs.gnn_graph(w["graph"])
        n, F = len(ip) - 1, w["F"]
        vals = graphs.gcn_norm_values(ip, ic)
        P = api.pack(ip, ic, np.arange(n, dtype=np.int32), w["V"], 2, w["M"], dtype="bf16", val=vals, tau="auto",
                     F=F, order="original")
        ldx = (F + 31) // 32 * 32
        X = torch.empty((n, ldx), dtype=torch.bfloat16, device=dev).normal_()[:, :F]
        Y = torch.empty((n, F), dtype=torch.float32, device=dev)
        res = {"workload": wl}
        res["base_ms"] = timed(lambda: api.spmm(P, X, Y), flush)
        res["base_sptc_ms"] = timed(lambda: api.spmm(P, X, Y, part="sptc"), flush)
        api.l2_persist(X)
        res["persist_ms"] = timed(lambda: api.spmm(P, X, Y), flush)
        res["persist_sptc_ms"] = timed(lambda: api.spmm(P, X, Y, part="sptc"), flush)
        api.l2_persist(None)
        res["reset_ms"] = timed(lambda: api.spmm(P, X, Y), flush)
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
