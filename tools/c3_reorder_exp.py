"""Does the full MAXITER = 10 reorder (Alg. 1-3) pay off on the C3 (Reddit-shaped)
headline?  Reorders with nm_reorder_gpu at max_outer 0 (the bench's cap) and 10, then packs each
layout (natural, reordered) at several tau and times nm_spmm (L2 flushed, CUDA events).
usage: python tools/c3_reorder_exp.py [out.jsonl]"""
import json
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
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
    out = open(sys.argv[1], "w") if len(sys.argv) > 1 else None
    dev = torch.device("cuda:0")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    ip, ic = graphs.gnn_graph("reddit")
    n, F = len(ip) - 1, 128
    vals = graphs.gcn_norm_values(ip, ic)
    X = torch.empty((n, F), dtype=torch.bfloat16, device=dev).normal_()
    Y = torch.empty((n, F), dtype=torch.float32, device=dev)
    perms = {"natural": (np.arange(n, dtype=np.int32), 0.0, None)}
    for mo in (0, 10):
        t = time.time()
        perm, st = api.reorder(ip, ic, 1, 2, 4, device=True, max_outer=mo, max_stage1=10,
                               max_stage2=0 if mo == 0 else 10)
        perms["reorder_outer%d" % mo] = (perm, time.time() - t, st)
        if mo == 10:
            np.save(os.path.join(ROOT, "gpurun_out", "c3_perm_outer10.npy"), perm)
    for name, (perm, rs, st) in perms.items():
        for tau in (4, 6, 8, 12):
            P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals, tau=tau, order="original")
            ps = P.stats()
            ms = timed(lambda: api.spmm(P, X, Y), flush)
            ms_s = timed(lambda: api.spmm(P, X, Y, part="sptc"), flush)
            rec = {"layout": name, "tau": tau, "ms": ms, "sptc_ms": ms_s, "gflops": 2.0 * ip[-1] * F / ms / 1e6,
                   "n_chunks": ps["n_chunks"], "residual_nnz": ps["residual_nnz"], "reorder_s": rs,
                   "omega": [st["omega_init"], st["omega_final"]] if st else None}
            print(json.dumps(rec), flush=True)
            if out:
                out.write(json.dumps(rec) + "\n")
                out.flush()
            P.free()


if __name__ == "__main__":
    main()
