"""Parity on the GNN-shaped configs of BASELINE.json (configs[2..4]) at reduced vertex count,
same shape parameters (degree distribution, communities, locality, feature widths, V:N:M and
dtype):

* C3 Reddit-shaped   : GCN aggregation at F = 128 (H 602 -> 608 padded, W 608 x 128), bf16,
                       1:2:4 and 128:2:16.
* C4 proteins-shaped : 2-layer GCN 256 -> 256 -> 256, 128:2:16, driven by dist.gcn_forward
                       (one row-sharded all-gather per layer) with the libnm layer.
* C5 products-shaped : F 100 (104 padded) -> 256 aggregate-first, 128:2:8, 8 row shards.

The full-size graphs (57-124M edges) take minutes to generate on the host; the kernels, the
packing and the launch configuration are the same.  Reordering uses a capped pass count
(max_outer = 1) -- its bit-exact parity is covered in test_parity_reorder.py.
Bound: aggregation 1e-3 * E (E = |Ahat| |operand|) propagated through the dense layer, plus
bf16 roundings of the intermediate (2^-9) and of the output (2^-8)."""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs
from paper_conf_ppopp_chensz0s25_b200.dist import gcn_forward, shard_rows

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _gcn_norm(ip, ic):
    deg = np.diff(ip).astype(np.float64)
    rows = np.repeat(np.arange(len(ip) - 1), np.diff(ip))
    return (1.0 / np.sqrt(deg[rows] * deg[ic])).astype(np.float32)


def _bf16(t_np, dev):
    b, v = graphs.round16(t_np.astype(np.float32), "bf16")
    return torch.from_numpy(b.view(np.int16)).to(dev).view(torch.bfloat16), v


def _unbf16(t):
    return graphs.bf16_bits_to_f64(t.view(torch.int16).cpu().numpy().view(np.uint16))


@pytest.mark.parametrize("V,M", [(1, 4), (128, 16)])
def test_c3_reddit_shaped_aggregation(V, M):
    dev = _cuda()
    n = 232965 // 32
    m = int(n * 493 / 2)
    ip, ic = graphs.lmcl_graph(n, m, 2.3, 41, 0.6, 13, self_loops=True)
    vals = _gcn_norm(ip, ic)
    _, v64 = graphs.round16(vals, "bf16")
    perm, st = api.reorder(ip, ic, V, 2, M, max_outer=1, max_stage2=2)
    P = api.pack(ip, ic, perm, V, 2, M, dtype="bf16", val=vals)
    rng = np.random.default_rng(3)
    H = np.zeros((n, 608), np.float32)
    H[:, :602] = rng.standard_normal((n, 602))
    W = np.zeros((608, 128), np.float32)
    W[:602] = rng.standard_normal((602, 128)) * np.sqrt(2.0 / (602 + 128))  # Glorot
    Hd, h64 = _bf16(H, dev)
    Wd, w64 = _bf16(W, dev)
    pd = torch.from_numpy(perm).to(dev)
    PH = torch.empty_like(Hd)
    api.permute_rows(Hd, PH, pd, "bf16")
    ws = torch.empty(api.gcn_workspace_bytes(n, 608, 128), dtype=torch.uint8, device=dev)
    out = torch.empty((n, 128), dtype=torch.bfloat16, device=dev)
    api.gcn_layer(P, PH, Wd, None, out, ws, relu=False, order="linear")
    torch.cuda.synchronize()
    # aggregation checked against the exact bf16 XW the GPU consumed (workspace, permuted)
    xw_p = graphs.bf16_bits_to_f64(ws[: n * 128 * 2].view(torch.int16).cpu().numpy().view(np.uint16)).reshape(n, 128)
    xw = np.empty_like(xw_p)
    xw[perm] = xw_p
    Y, E, _ = oracle.spmm(ip, ic, v64, xw)
    got = np.empty((n, 128))
    got[perm] = _unbf16(out)
    assert (np.abs(got - Y) <= 1e-3 * E + 2.0 ** -8 * np.abs(Y) + 1e-30).all()


def test_c4_proteins_shaped_two_layer_gcn():
    dev = _cuda()
    n = 132534 // 32
    m = int(n * 597 / 2)
    ip, ic = graphs.lmcl_graph(n, m, 3.0, 8, 0.8, 14, self_loops=True)
    vals = _gcn_norm(ip, ic)
    _, v64 = graphs.round16(vals, "bf16")
    perm, _ = api.reorder(ip, ic, 128, 2, 16, max_outer=1, max_stage2=2)
    P = api.pack(ip, ic, perm, 128, 2, 16, dtype="bf16", val=vals)
    rng = np.random.default_rng(4)
    H0 = rng.standard_normal((n, 256)).astype(np.float32)
    Ws = [(rng.standard_normal((256, 256)) / 16.0).astype(np.float32) for _ in range(2)]
    bs = [rng.standard_normal(256).astype(np.float32) * 0.1 for _ in range(2)]
    pd = torch.from_numpy(perm).to(dev)
    H0d, h64 = _bf16(H0, dev)
    PH0 = torch.empty_like(H0d)
    api.permute_rows(H0d, PH0, pd, "bf16")
    Wd = [_bf16(w, dev) for w in Ws]
    bd = [torch.from_numpy(b).to(dev) for b in bs]
    ws = torch.empty(api.gcn_workspace_bytes(n, 256, 256), dtype=torch.uint8, device=dev)

    def local_layer(li, Hf, W, b, relu, rb, re):
        out = torch.empty((re - rb, 256), dtype=torch.bfloat16, device=dev)
        api.gcn_layer(P, Hf, W, b, out, ws, relu=relu, order="linear")
        return out

    layers = [(Wd[0][0], bd[0], True), (Wd[1][0], bd[1], False)]
    out_p = gcn_forward(PH0, layers, local_layer)
    torch.cuda.synchronize()
    got = np.empty((n, 256))
    got[perm] = _unbf16(out_p)
    # fp64 reference of the same network on the same bf16 inputs; each layer's bf16 round
    # trips bound the end-to-end error, checked as a relative Frobenius error <= 1e-2
    h = h64
    for li, (w, b) in enumerate(zip(Wd, bs)):
        y, _, _ = oracle.spmm(ip, ic, v64, h @ w[1])
        h = y + b
        if li == 0:
            h = np.maximum(h, 0.0)
    rel = np.linalg.norm(got - h) / np.linalg.norm(h)
    assert rel <= 1e-2, rel


def test_c5_products_shaped_aggregate_first_8_shards():
    dev = _cuda()
    n = 2449029 // 256
    m = int(n * 50.5 / 2)
    ip, ic = graphs.lmcl_graph(n, m, 2.5, 47, 0.7, 15, self_loops=True)
    vals = _gcn_norm(ip, ic)
    _, v64 = graphs.round16(vals, "bf16")
    perm, _ = api.reorder(ip, ic, 128, 2, 8, max_outer=1, max_stage2=2)
    rng = np.random.default_rng(5)
    H = np.zeros((n, 104), np.float32)
    H[:, :100] = rng.standard_normal((n, 100))
    W = np.zeros((104, 256), np.float32)
    W[:100] = rng.standard_normal((100, 256)) / 10.0
    b = rng.standard_normal(256).astype(np.float32)
    Hd, h64 = _bf16(H, dev)
    Wd, w64 = _bf16(W, dev)
    pd = torch.from_numpy(perm).to(dev)
    PH = torch.empty_like(Hd)
    api.permute_rows(Hd, PH, pd, "bf16")
    bias = torch.from_numpy(b).to(dev)
    ws = torch.empty(api.gcn_workspace_bytes(n, 104, 256), dtype=torch.uint8, device=dev)
    out = torch.empty((n, 256), dtype=torch.bfloat16, device=dev)
    for r in range(8):
        rb, re = shard_rows(n, 8, r)
        if re <= rb:
            continue
        P = api.pack(ip, ic, perm, 128, 2, 8, dtype="bf16", val=vals, row_begin=rb, row_end=re)
        api.gcn_layer(P, PH, Wd, bias, out[rb:re], ws, relu=True, order="auto")
    torch.cuda.synchronize()
    got = np.empty((n, 256))
    got[perm] = _unbf16(out)
    Ya, Ea, _ = oracle.spmm(ip, ic, v64, h64)
    ref = np.maximum(Ya @ w64 + b, 0.0)
    bound = 3e-3 * (Ea @ np.abs(w64)) + 2.0 ** -8 * np.abs(ref) + 1e-30
    assert (np.abs(got - ref) <= bound).all(), np.abs(got - ref).max()
