"""Small nm_spmm runs for compute-sanitizer (racecheck / synccheck / memcheck):
C1 (ER n=2048, 2:4, F=32, hybrid tau -> both kernels) and a multi-unit banded case
(n = 300*128+77, 64:2:8, F=128, several units per CTA).  usage:
    compute-sanitizer --tool racecheck python tools/sanitize_spmm.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_chensz0s25_b200 import api, graphs  # noqa: E402


def run(ip, ic, V, M, F, dtype, tau):
    n = len(ip) - 1
    vals = graphs.symmetric_values(ip, ic, 5)
    perm = np.random.default_rng(1).permutation(n).astype(np.int32)
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=vals, order="original", tau=tau)
    xb, _ = graphs.round16(graphs.features(n, F, 6), dtype)
    X = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.float16 if dtype == "f16" else torch.bfloat16)
    Y = torch.empty((n, F), device="cuda")
    for fmt in (1, 2, 3):
        api.spmm(P, X, Y, part="sptc", format=fmt)
    api.spmm(P, X, Y)
    torch.cuda.synchronize()
    st = P.stats()
    print("n=%d chunks=%d residual=%d split=%d finite=%s" % (n, st["n_chunks"], st["residual_nnz"],
                                                            st["residual_split_rows"], bool(torch.isfinite(Y).all())))


def run_gcn_fused():
    """nm_gcn_layer on a pack without residual (fused epilogue) and nm_gcn_layer_bcast."""
    n, fin, fout = 2600, 96, 64
    ip, ic = graphs.banded_graph(n, 6, 11, self_loops=True)
    vals = graphs.gcn_norm_values(ip, ic)
    perm, _ = api.reorder(ip, ic, 1, 2, 4)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals)
    H = torch.randn((n, fin), device="cuda").to(torch.bfloat16)
    W = (torch.randn((fin, fout), device="cuda") / 10).to(torch.bfloat16)
    b = torch.randn(fout, device="cuda")
    ws = torch.empty(api.gcn_workspace_bytes(n, fin, fout), dtype=torch.uint8, device="cuda")
    out = torch.empty((n, fout), dtype=torch.bfloat16, device="cuda")
    api.gcn_layer(P, H, W, b, out, ws, relu=True)
    dsts = [torch.empty((n + 100, fout), dtype=torch.bfloat16, device="cuda") for _ in range(2)]
    api.gcn_layer_bcast(P, H, W, b, [d.data_ptr() for d in dsts], 100, fout, ws, relu=True)
    torch.cuda.synchronize()
    print("gcn fused residual=%d equal=%s" % (P.info()["residual_nnz"], bool(torch.equal(out, dsts[0][100:]))))


if __name__ == "__main__":
    run_gcn_fused()
    ip, ic = graphs.er_graph(2048, 16384, 1)
    run(ip, ic, 1, 4, 32, "f16", 4)
    ip, ic = graphs.banded_graph(300 * 128 + 77, 12, 91)
    run(ip, ic, 64, 8, 128, "bf16", 4)
    print("SANITIZE RUN DONE")
