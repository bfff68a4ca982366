"""Debug aid: locate rows where the GPU SpMM disagrees with the oracle on a bench workload."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import bench  # noqa: E402
import oracle  # noqa: E402
from paper_conf_ppopp_chensz0s25_b200 import api, graphs  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "c2-powerlaw-n262k-d16-f128-1:2:4"
w = bench.parse_workload(wl)
ip, ic, vals, X32 = bench.make_graph(w)
n = w["n"]
perm, st = api.reorder(ip, ic, w["V"], 2, w["M"])
print("reorder", st)
xbits, x64 = graphs.round16(X32, w["dtype"])
_, v64 = graphs.round16(vals, w["dtype"])
X = torch.from_numpy(xbits.view(np.int16)).cuda().view(torch.float16)
for order in ("permuted", "original"):
    P = api.pack(ip, ic, perm, w["V"], 2, w["M"], dtype=w["dtype"], val=vals, order=order)
    print(order, P.info())
    pd = torch.from_numpy(perm).cuda()
    for part in ("sptc", "all"):
        if order == "permuted":
            PX = torch.empty_like(X)
            api.permute_rows(X, PX, pd, "f16")
            Yp = torch.full((n, w["F"]), float("nan"), device="cuda")
            api.spmm(P, PX, Yp, part="sptc")
            if part == "all":
                api.spmm(P, PX, Yp, part="residual")
            Y = torch.empty_like(Yp)
            api.unpermute_rows(Yp, Y, pd, "f32")
        else:
            Y = torch.full((n, w["F"]), float("nan"), device="cuda")
            api.spmm(P, X, Y, part="sptc")
            if part == "all":
                api.spmm(P, X, Y, part="residual")
        torch.cuda.synchronize()
        Yh = Y.cpu().numpy().astype(np.float64)
        rows = np.arange(0, n, 7)
        Yr, Er = oracle.spmm_rows(rows, ip, ic, v64, x64)
        bad = (np.abs(Yh[rows] - Yr) > 1e-3 * Er + 1e-30).any(axis=1)
        br = rows[bad]
        inv = np.empty(n, np.int64)
        inv[perm] = np.arange(n)
        print(order, part, "bad rows %d / %d" % (bad.sum(), len(rows)))
        if bad.any():
            pos = inv[br]  # position in B
            print("  positions in B (first 20):", pos[:20])
            print("  panels:", np.unique(pos // 128)[:20], "of", (n + 127) // 128)
            print("  degrees:", np.diff(ip)[br][:20])
