"""Full-size parity at the GNN-shaped configs of BASELINE.json (configs[2..4]) in the launch
configuration bench.py times (fused original-order pack, nm_pack_auto's hybrid split, both
tensor-core kernels the bench's trial chooses from (bitwise equal),
bench's reorder options), plus multi-unit parity of the wide-M patterns: sampled output rows
(random + the heaviest rows + first/last) are recomputed one by one by the oracle in fp64 and
must satisfy |Y - Y_ref| <= 1e-3 * (|A| |X|) (north star); every row of Y must be finite and
packed + residual entries must equal nnz (lossless)."""
import numpy as np
import pytest

import oracle

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
torch = pytest.importorskip("torch")


def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _sampled_parity(ip, ic, vals, X32, perm, V, M, dtype, tau, order="original", nsample=3000, seed=7,
                    formats=False):
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs
    dev = _cuda()
    n, F = X32.shape
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=vals, order=order, tau=tau, F=F)
    info = P.info()
    assert info["packed_nnz"] + info["residual_nnz"] == ip[-1]
    xbits, x64 = graphs.round16(X32, dtype)
    _, v64 = graphs.round16(vals, dtype)
    Fp = (F + 7) // 8 * 8
    Xb = torch.zeros((n, Fp), dtype=torch.int16, device=dev)
    Xb[:, :F] = torch.from_numpy(xbits.view(np.int16)).to(dev)
    tdt = torch.float16 if dtype == "f16" else torch.bfloat16
    X = Xb.view(tdt)[:, :F]
    if order == "original":
        Y = torch.full((n, Fp), float("nan"), device=dev)[:, :F]
        api.spmm(P, X, Y)
        Yh = Y.cpu().numpy()
        if formats:  # the other tensor-core kernel the bench may pick (A in TMEM): bitwise equal
            Y3 = torch.full((n, Fp), float("nan"), device=dev)[:, :F]
            api.spmm(P, X, Y3, part="sptc", format=3)
            api.spmm(P, X, Y3, part="residual")
            torch.cuda.synchronize()
            assert torch.equal(Y, Y3)
    else:
        pd = torch.from_numpy(perm).to(dev)
        PXb = torch.zeros_like(Xb)
        PX = PXb.view(tdt)[:, :F]
        api.permute_rows(X, PX, pd, dtype)
        Yp = torch.full((n, Fp), float("nan"), device=dev)[:, :F]
        api.spmm(P, PX, Yp)
        Yh = np.empty((n, F), np.float32)
        Yh[perm] = Yp.cpu().numpy()
    torch.cuda.synchronize()
    assert np.isfinite(Yh).all()
    rng = np.random.default_rng(seed)
    rows = np.unique(np.concatenate([rng.integers(0, n, nsample), [0, n - 1], np.argsort(np.diff(ip))[-64:]]))
    Yr, Er = oracle.spmm_rows(rows, ip, ic, v64, x64)
    err = np.abs(Yh[rows].astype(np.float64) - Yr)
    assert (err <= 1e-3 * Er + 1e-30).all(), err.max()
    return P


@pytest.mark.parametrize("workload", ["c3-reddit-f128-1:2:4", "c3-reddit-f128-128:2:16", "c4-proteins-f256-128:2:16",
                                      "c5-products-f100-128:2:8"])
def test_gnn_config_bench_launch(workload):
    import bench
    from paper_conf_ppopp_chensz0s25_b200 import api
    _cuda()
    w = bench.parse_workload(workload)
    ip, ic, vals, X32 = bench.make_graph(w)
    perm, _ = api.reorder(ip, ic, w["V"], 2, w["M"], device=True, **bench.default_reorder_opts(w))
    tau = w["tau"] if w["tau"] is not None else "auto"  # bench.py: nm_pack_auto
    P = _sampled_parity(ip, ic, vals, X32, perm, w["V"], w["M"], w["dtype"], tau, formats=True)
    st = P.stats()
    assert st["n_chunks"] > 4 * 148  # many chunks per CTA: stage ring wrap-around, parity flips


@pytest.mark.parametrize("V,M", [(64, 8), (128, 16)])
@pytest.mark.parametrize("F", [256, 300])
@pytest.mark.parametrize("tau", [0, 4])
def test_wide_patterns_many_units_bf16(V, M, F, tau):
    """>= 300 panels (>= 2 units per CTA of the persistent grid) for the V = 64 / 128 patterns,
    bf16, F = 256 (one full tile) and 300 (two tiles, ragged)."""
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs
    _cuda()
    n = 300 * 128 + 77
    ip, ic = graphs.banded_graph(n, 12, 91)
    vals = graphs.symmetric_values(ip, ic, 92)
    X32 = graphs.features(n, F, 93)
    perm, _ = api.reorder(ip, ic, V, 2, M, max_outer=1, max_stage2=1, device=True)
    for order in ("original", "permuted"):
        P = _sampled_parity(ip, ic, vals, X32, perm, V, M, "bf16", tau, order=order, nsample=1500)
        assert P.stats()["n_panels"] >= 300
