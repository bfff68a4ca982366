"""GPU parity of nm_gcn_layer (Eq. 1: H' = ReLU(Ahat (H W) + b), linear first
as GCN does, L564).  The aggregation is checked against the oracle's fp64 SpMM applied to the
exact bf16 operand H W the GPU consumed (read back from the layer's workspace):
|H' - relu(Ahat XW + b)| <= 1e-3 * (|Ahat| |XW|) + one bf16 rounding of the output."""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _gcn_norm(ip, ic):
    """Ahat = D^-1/2 (A + I) D^-1/2 on a graph that already contains its self-loops."""
    n = len(ip) - 1
    deg = np.diff(ip).astype(np.float64)
    rows = np.repeat(np.arange(n), np.diff(ip))
    return (1.0 / np.sqrt(deg[rows] * deg[ic])).astype(np.float32)


@pytest.mark.parametrize("n,fin,fout,V,M", [(2048, 64, 32, 1, 4), (3000, 128, 64, 8, 8), (1500, 96, 128, 1, 4)])
@pytest.mark.parametrize("relu", [True, False])
def test_gcn_layer(n, fin, fout, V, M, relu):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dev = torch.device("cuda:0")
    ip, ic = graphs.er_graph(n, 6 * n, 3, self_loops=True)
    vals = _gcn_norm(ip, ic)
    vbits, v64 = graphs.round16(vals, "bf16")
    perm, _ = api.reorder(ip, ic, V, 2, M)
    P = api.pack(ip, ic, perm, V, 2, M, dtype="bf16", val=vals)
    rng = np.random.default_rng(1)
    H32 = rng.standard_normal((n, fin)).astype(np.float32)
    W32 = (rng.standard_normal((fin, fout)) / np.sqrt(fin)).astype(np.float32)
    b = rng.standard_normal(fout).astype(np.float32)
    hb, _ = graphs.round16(H32, "bf16")
    wb, _ = graphs.round16(W32, "bf16")
    H = torch.from_numpy(hb.view(np.int16)).to(dev).view(torch.bfloat16)
    W = torch.from_numpy(wb.view(np.int16)).to(dev).view(torch.bfloat16)
    pd = torch.from_numpy(perm).to(dev)
    PH = torch.empty_like(H)
    api.permute_rows(H, PH, pd, "bf16")
    ws = torch.empty(api.gcn_workspace_bytes(n, fin, fout), dtype=torch.uint8, device=dev)
    Hout_p = torch.empty((n, fout), dtype=torch.bfloat16, device=dev)
    bias = torch.from_numpy(b).to(dev)
    api.gcn_layer(P, PH, W, bias, Hout_p, ws, relu=relu)
    torch.cuda.synchronize()
    # the bf16 XW the aggregation consumed (permuted order), from the workspace
    xw_bits = ws[: n * fout * 2].view(torch.int16).cpu().numpy().view(np.uint16).reshape(n, fout)
    xw_p = graphs.bf16_bits_to_f64(xw_bits)
    # sanity: XW is H W (permuted) up to bf16 rounding of a fp32-accumulated GEMM
    ref_xw = (graphs.bf16_bits_to_f64(hb) @ graphs.bf16_bits_to_f64(wb))[perm]
    assert np.abs(xw_p - ref_xw).max() <= 1e-2 * np.abs(ref_xw).max()
    xw = np.empty_like(xw_p)
    xw[perm] = xw_p  # back to the original order
    Y, E, _ = oracle.spmm(ip, ic, v64, xw)
    ref = Y + b
    if relu:
        ref = np.maximum(ref, 0.0)
    Hout = torch.empty_like(Hout_p)
    api.unpermute_rows(Hout_p, Hout, pd, "bf16")
    torch.cuda.synchronize()
    got = graphs.bf16_bits_to_f64(Hout.view(torch.int16).cpu().numpy().view(np.uint16))
    bound = 1e-3 * E + 2.0 ** -8 * np.abs(ref) + 1e-30
    assert (np.abs(got - ref) <= bound).all(), np.abs(got - ref).max()


@pytest.mark.parametrize("n,fin,fout,V,M,shards", [(2048, 32, 64, 1, 4, 1), (3000, 104, 256, 128, 8, 3),
                                                   (1500, 64, 64, 1, 4, 2)])
def test_gcn_layer_aggregate_first_and_row_shards(n, fin, fout, V, M, shards):
    """Aggregate-first order (ogbn-products shape, F 100(->104) -> 256, 128:2:8) and
    panel-aligned row shards (nm_pack_rows) whose outputs tile the full result.
    Bound: SpMM 1e-3*(|Ahat||H|)|W| + bf16 rounding of Ahat H (2^-9 relative) propagated through
    W + bf16 rounding of the output (2^-8 relative)."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_chensz0s25_b200.dist import shard_rows
    dev = torch.device("cuda:0")
    ip, ic = graphs.er_graph(n, 5 * n, 4, self_loops=True)
    vals = _gcn_norm(ip, ic)
    _, v64 = graphs.round16(vals, "bf16")
    perm, _ = api.reorder(ip, ic, V, 2, M)
    rng = np.random.default_rng(2)
    hb, h64 = graphs.round16(rng.standard_normal((n, fin)).astype(np.float32), "bf16")
    wb, w64 = graphs.round16((rng.standard_normal((fin, fout)) / np.sqrt(fin)).astype(np.float32), "bf16")
    b = rng.standard_normal(fout).astype(np.float32)
    H = torch.from_numpy(hb.view(np.int16)).to(dev).view(torch.bfloat16)
    W = torch.from_numpy(wb.view(np.int16)).to(dev).view(torch.bfloat16)
    pd = torch.from_numpy(perm).to(dev)
    PH = torch.empty_like(H)
    api.permute_rows(H, PH, pd, "bf16")
    bias = torch.from_numpy(b).to(dev)
    ws = torch.empty(api.gcn_workspace_bytes(n, fin, fout), dtype=torch.uint8, device=dev)
    Hout_p = torch.empty((n, fout), dtype=torch.bfloat16, device=dev)
    for r in range(shards):
        rb, re = shard_rows(n, shards, r)
        P = api.pack(ip, ic, perm, V, 2, M, dtype="bf16", val=vals, row_begin=rb, row_end=re)
        api.gcn_layer(P, PH, W, bias, Hout_p[rb:re], ws, relu=True, order="aggregate")
        torch.cuda.synchronize()
    Hout = torch.empty_like(Hout_p)
    api.unpermute_rows(Hout_p, Hout, pd, "bf16")
    torch.cuda.synchronize()
    got = graphs.bf16_bits_to_f64(Hout.view(torch.int16).cpu().numpy().view(np.uint16))
    Ya, Ea, _ = oracle.spmm(ip, ic, v64, h64)
    ref = np.maximum(Ya @ w64 + b, 0.0)
    bound = 3e-3 * (Ea @ np.abs(w64)) + 2.0 ** -8 * np.abs(ref) + 1e-30
    assert (np.abs(got - ref) <= bound).all(), np.abs(got - ref).max()


@pytest.mark.parametrize("n,fin,fout,V,M", [(2048, 64, 32, 1, 4), (1500, 96, 128, 8, 8)])
@pytest.mark.parametrize("relu", [True, False])
def test_gcn_layer_backward(n, fin, fout, V, M, relu):
    """nm_gcn_layer_backward vs the oracle's fp64 backward, which forms
    Ahat^T explicitly (the GPU reuses the same pack: Ahat^T = Ahat).  The ReLU mask is the
    GPU's Hout > 0 on both sides; db within 1e-3 of sum |dZ|; dW, dH (dT rounded to bf16 once)
    within a relative Frobenius error of 1e-2."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dev = torch.device("cuda:0")
    ip, ic = graphs.er_graph(n, 6 * n, 7, self_loops=True)
    vals = _gcn_norm(ip, ic)
    vbits, v64 = graphs.round16(vals, "bf16")
    perm, _ = api.reorder(ip, ic, V, 2, M)
    P = api.pack(ip, ic, perm, V, 2, M, dtype="bf16", val=vals)
    rng = np.random.default_rng(2)
    hb, h64 = graphs.round16(rng.standard_normal((n, fin)).astype(np.float32), "bf16")
    wb, w64 = graphs.round16((rng.standard_normal((fin, fout)) / np.sqrt(fin)).astype(np.float32), "bf16")
    gb, g64 = graphs.round16(rng.standard_normal((n, fout)).astype(np.float32), "bf16")
    b = rng.standard_normal(fout).astype(np.float32)
    tb = lambda a: torch.from_numpy(a.view(np.int16)).to(dev).view(torch.bfloat16)
    pd = torch.from_numpy(perm).to(dev)
    H, W, G = tb(hb), tb(wb), tb(gb)
    PH, PG = torch.empty_like(H), torch.empty_like(G)
    api.permute_rows(H, PH, pd, "bf16")
    api.permute_rows(G, PG, pd, "bf16")
    ws = torch.empty(api.gcn_workspace_bytes(n, fin, fout), dtype=torch.uint8, device=dev)
    Hout = torch.empty((n, fout), dtype=torch.bfloat16, device=dev)
    api.gcn_layer(P, PH, W, torch.from_numpy(b).to(dev), Hout, ws, relu=relu)
    wsb = torch.empty(api.gcn_backward_workspace_bytes(n, fin, fout), dtype=torch.uint8, device=dev)
    dH = torch.empty((n, fin), dtype=torch.bfloat16, device=dev)
    dW = torch.empty((fin, fout), dtype=torch.float32, device=dev)
    db = torch.empty(fout, dtype=torch.float32, device=dev)
    api.gcn_layer_backward(P, PH, W, Hout, PG, dH, dW, db, wsb, relu=relu)
    torch.cuda.synchronize()
    hout_p = graphs.bf16_bits_to_f64(Hout.view(torch.int16).cpu().numpy().view(np.uint16))
    hout = np.empty_like(hout_p)
    hout[perm] = hout_p
    dH_ref, dW_ref, db_ref, _ = oracle.gcn_layer_backward(ip, ic, v64, h64, w64, hout, g64, relu)
    dZ = g64 * ((hout > 0) if relu else 1.0)
    assert np.all(np.abs(db.cpu().numpy() - db_ref) <= 1e-3 * np.abs(dZ).sum(0) + 1e-6)
    got_dw = dW.cpu().numpy().astype(np.float64)
    assert np.linalg.norm(got_dw - dW_ref) <= 1e-2 * np.linalg.norm(dW_ref)
    dh_p = graphs.bf16_bits_to_f64(dH.view(torch.int16).cpu().numpy().view(np.uint16))
    got_dh = np.empty_like(dh_p)
    got_dh[perm] = dh_p
    assert np.linalg.norm(got_dh - dH_ref) <= 1e-2 * np.linalg.norm(dH_ref)


@pytest.mark.parametrize("fout,relu", [(64, True), (200, False), (128, True)])
def test_gcn_layer_fused_epilogue_without_residual(fout, relu):
    """A pack with an empty residual (banded graph, reordered to conform at 1:2:4, tau = 0):
    nm_gcn_layer applies bias, activation and the bf16 down-convert in the tensor-core kernel's
    epilogue.  The result equals the unfused path (nm_spmm to fp32 + the separate bias/act
    kernel, here through nm_gcn_layer_bcast with one destination) bitwise, and the oracle within
    the GCN bound."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dev = torch.device("cuda:0")
    n, fin = 2600, 96
    ip, ic = graphs.banded_graph(n, 6, 11, self_loops=True)
    vals = _gcn_norm(ip, ic)
    vbits, v64 = graphs.round16(vals, "bf16")
    perm, _ = api.reorder(ip, ic, 1, 2, 4)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals)
    assert P.info()["residual_nnz"] == 0
    rng = np.random.default_rng(4)
    hb, _ = graphs.round16(rng.standard_normal((n, fin)).astype(np.float32), "bf16")
    wb, _ = graphs.round16((rng.standard_normal((fin, fout)) / np.sqrt(fin)).astype(np.float32), "bf16")
    b = rng.standard_normal(fout).astype(np.float32)
    H = torch.from_numpy(hb.view(np.int16)).to(dev).view(torch.bfloat16)
    W = torch.from_numpy(wb.view(np.int16)).to(dev).view(torch.bfloat16)
    pd = torch.from_numpy(perm).to(dev)
    PH = torch.empty_like(H)
    api.permute_rows(H, PH, pd, "bf16")
    ws = torch.empty(api.gcn_workspace_bytes(n, fin, fout), dtype=torch.uint8, device=dev)
    bias = torch.from_numpy(b).to(dev)
    fused = torch.empty((n, fout), dtype=torch.bfloat16, device=dev)
    api.gcn_layer(P, PH, W, bias, fused, ws, relu=relu)
    unfused = torch.empty((n, fout), dtype=torch.bfloat16, device=dev)
    api.gcn_layer_bcast(P, PH, W, bias, [unfused.data_ptr()], 0, fout, ws, relu=relu)
    torch.cuda.synchronize()
    assert torch.equal(fused.view(torch.int16), unfused.view(torch.int16))
    xw_bits = ws[: n * fout * 2].view(torch.int16).cpu().numpy().view(np.uint16).reshape(n, fout)
    xw = np.empty((n, fout))
    xw[perm] = graphs.bf16_bits_to_f64(xw_bits)
    Y, E, _ = oracle.spmm(ip, ic, v64, xw)
    ref = Y + b
    if relu:
        ref = np.maximum(ref, 0.0)
    out = torch.empty_like(fused)
    api.unpermute_rows(fused, out, pd, "bf16")
    torch.cuda.synchronize()
    got = graphs.bf16_bits_to_f64(out.view(torch.int16).cpu().numpy().view(np.uint16))
    bound = 1e-3 * E + 2.0 ** -8 * np.abs(ref) + 1e-30
    assert (np.abs(got - ref) <= bound).all(), np.abs(got - ref).max()
