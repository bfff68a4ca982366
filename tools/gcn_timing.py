"""Per-layer GCN timing on the GNN-shaped configs (the layer wrapper timed per
layer; Table 3's LYR column = the aggregation layer).  For each config: one pack of Ahat
(permuted order, nm_reorder_gpu with the bench's caps), then CUDA-event timing of nm_gcn_layer
(cuBLASLt XW + the packed SpMM + bias/ReLU) and of its aggregation alone, L2 flushed between
reps.  usage: python tools/gcn_timing.py [out.jsonl]"""
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

# (workload, layer dims, order) -- C3: 602 -> 128 (linear first, H padded to 608 columns);
# C4: two 256 -> 256 layers; C5: 100 -> 256 aggregate first (H padded to 104 columns)
CASES = [("c3-reddit-f128-1:2:4", [(608, 128)], "linear"),
         ("c4-proteins-f256-128:2:16", [(256, 256), (256, 256)], "linear"),
         ("c5-products-f100-128:2:8", [(104, 256)], "aggregate")]


def timed(fn, reps, flush):
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
    out = open(sys.argv[1], "w") if len(sys.argv) > 1 else None
    dev = torch.device("cuda:0")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    for wl, layers, order in CASES:
        w = bench.parse_workload(wl)
        ip, ic = graphs.gnn_graph(w["graph"])
        n = len(ip) - 1
        vals = graphs.gcn_norm_values(ip, ic)
        perm, rst = api.reorder(ip, ic, w["V"], 2, w["M"], device=True, **bench.default_reorder_opts(w))
        P = api.pack(ip, ic, perm, w["V"], 2, w["M"], dtype="bf16", val=vals, tau=api.hybrid_tau(w["F"]))
        rng = np.random.default_rng(0)
        H = torch.from_numpy(graphs.round16(rng.standard_normal((n, layers[0][0])).astype(np.float32), "bf16")[0]
                             .view(np.int16)).to(dev).view(torch.bfloat16)
        nnz = int(ip[-1])
        for li, (fi, fo) in enumerate(layers):
            W = torch.from_numpy(graphs.round16((rng.standard_normal((fi, fo)) / np.sqrt(fi)).astype(np.float32),
                                                "bf16")[0].view(np.int16)).to(dev).view(torch.bfloat16)
            b = torch.zeros(fo, device=dev)
            Hout = torch.empty((n, fo), dtype=torch.bfloat16, device=dev)
            ws = torch.empty(api.gcn_workspace_bytes(n, fi, fo), dtype=torch.uint8, device=dev)
            ms = timed(lambda: api.gcn_layer(P, H, W, b, Hout, ws, relu=True, order=order), 20, flush)
            fa = fo if order == "linear" else fi
            Xa = torch.empty((n, fa), dtype=torch.bfloat16, device=dev).normal_()
            Ya = torch.empty((n, fa), device=dev)
            ms_agg = timed(lambda: api.spmm(P, Xa, Ya), 20, flush)
            rec = {"workload": wl, "layer": li, "F_in": fi, "F_out": fo, "order": order, "n": n, "nnz": nnz,
                   "layer_ms": ms, "aggregation_ms": ms_agg, "aggregation_gflops": 2.0 * nnz * fa / (ms_agg * 1e-3) / 1e9,
                   "dense_flop": 2.0 * n * fi * fo, "reorder_s": rst["seconds"]}
            print(json.dumps(rec), flush=True)
            if out:
                out.write(json.dumps(rec) + "\n")
                out.flush()
            H = Hout if fo == layers[min(li + 1, len(layers) - 1)][0] else H


if __name__ == "__main__":
    main()
