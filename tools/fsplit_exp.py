"""Experiment: does splitting the feature dimension into column slabs (each nm_spmm call sees an
X slab of F/s columns, so the L2 working set of the gathered rows shrinks s-fold) speed up the
gather-bound SpMM on the GNN shapes?  Times, L2 flushed between reps (CUDA events):
  full      : nm_spmm at F
  split-s   : s calls of nm_spmm_sptc on column slabs, then s calls of nm_spmm_residual
  slabwise-s: per slab nm_spmm_sptc + nm_spmm_residual
plus each kernel alone.  usage: python tools/fsplit_exp.py [workload ...]"""
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
        perm = np.arange(n, dtype=np.int32)
        tau = api.hybrid_tau(F)
        P = api.pack(ip, ic, perm, w["V"], 2, w["M"], dtype="bf16", val=vals, tau=tau, order="original")
        ldx = (F + 7) // 8 * 8
        X = torch.empty((n, ldx), dtype=torch.bfloat16, device=dev).normal_()
        Y = torch.empty((n, F), dtype=torch.float32, device=dev)
        Y2 = torch.empty_like(Y)
        res = {"workload": wl, "tau": tau, "F": F}
        res["full_ms"] = timed(lambda: api.spmm(P, X, Y, F=F), flush)
        res["full_sptc_ms"] = timed(lambda: api.spmm(P, X, Y, F=F, part="sptc"), flush)
        res["full_res_ms"] = timed(lambda: api.spmm(P, X, Y, F=F, part="residual"), flush)
        api.spmm(P, X, Y, F=F)
        for s in ((2, 4) if os.environ.get("FSPLIT", "1") == "1" else ()):
            if F % (8 * s):
                continue
            fs = F // s
            sl = [(X[:, i * fs:(i + 1) * fs], Y2[:, i * fs:(i + 1) * fs]) for i in range(s)]

            def split():
                for xa, ya in sl:
                    api.spmm(P, xa, ya, F=fs, part="sptc")
                for xa, ya in sl:
                    api.spmm(P, xa, ya, F=fs, part="residual")

            def slabwise():
                for xa, ya in sl:
                    api.spmm(P, xa, ya, F=fs)

            res["split%d_ms" % s] = timed(split, flush)
            res["slabwise%d_ms" % s] = timed(slabwise, flush)
            res["split%d_sptc_ms" % s] = timed(lambda: [api.spmm(P, xa, ya, F=fs, part="sptc") for xa, ya in sl],
                                               flush)
            res["split%d_res_ms" % s] = timed(lambda: [api.spmm(P, xa, ya, F=fs, part="residual") for xa, ya in sl],
                                              flush)
            split()
            torch.cuda.synchronize()
            res["split%d_maxdiff" % s] = float((Y - Y2).abs().max())
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
