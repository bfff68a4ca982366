"""GPU parity: nm_count_violations, nm_pack (canonical export) and nm_spmm through the C ABI
vs the CPU oracle.

Bars: counts, permutation, packed arrays and residual CSR are bit-exact;
Y (fp32) satisfies |Y - Y_ref| <= 1e-3 * (|A| |X|) elementwise, Y_ref = fp64 A X on the same
16-bit-rounded inputs (BASELINE.json north_star tolerance).
"""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

TOL = 1e-3


def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _graph(kind, seed):
    if kind == "c1":
        return graphs.er_graph(2048, 16384, 1)
    if kind == "er":
        return graphs.er_graph(700, 5000, seed, self_loops=True)
    if kind == "pl":
        return graphs.lmcl_graph(1500, 12000, 2.1, 1, 0.0, seed, scramble=True)
    if kind == "band":
        return graphs.banded_graph(1300, 10, seed)
    if kind == "tiny":
        return graphs.fixture_f1()
    raise ValueError(kind)


CASES = [("tiny", 1, 1, 4), ("c1", 1, 1, 4), ("er", 2, 1, 4), ("pl", 3, 1, 4), ("band", 4, 1, 4),
         ("band", 5, 64, 8), ("pl", 6, 128, 16), ("er", 7, 8, 8), ("band", 8, 128, 8)]


@pytest.mark.parametrize("kind,seed,V,M", CASES)
def test_counts(kind, seed, V, M):
    _cuda()
    ip, ic = _graph(kind, seed)
    n = len(ip) - 1
    perm = np.random.default_rng(seed).permutation(n).astype(np.int32)
    for pm in (None, perm):
        w0, mb0, ps0 = oracle.counts(ip, ic, pm, V, 2, M)
        w1, mb1, ps1 = api.count_violations(ip, ic, pm, V, 2, M)
        assert (w0, mb0) == (w1, mb1)
        assert np.array_equal(ps0, ps1)


def _vp(V):
    """nm_pack's automatic panel height (nm.h): V for V = 16, 32, 64 patterns, else 128."""
    return V if V in (16, 32, 64) else 128


def _values(ip, ic, dtype, seed):
    v = graphs.symmetric_values(ip, ic, seed)
    bits, v64 = graphs.round16(v, dtype)
    return v, bits, v64


@pytest.mark.parametrize("kind,seed,V,M", CASES)
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_pack_canonical_bit_exact(kind, seed, V, M, dtype):
    _cuda()
    ip, ic = _graph(kind, seed)
    perm, _ = api.reorder(ip, ic, V, 2, M)
    v32, bits, _ = _values(ip, ic, dtype, seed)
    Mp = 4 if V == 1 else M
    ref = oracle.pack(ip, ic, bits, 0, perm, _vp(V), Mp)
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=v32)  # device rounds f32 -> 16 bit
    got = P.export_canonical()
    for k in ("panel_ptr", "mb_seg", "sel", "nib", "vals", "res_rowptr", "res_col", "res_val"):
        assert np.array_equal(ref[k], got[k]), k
    inf = P.info()
    assert inf["packed_nnz"] + inf["residual_nnz"] == ip[-1]


def test_pack_rows_shards_match_oracle_rows():
    _cuda()
    ip, ic = _graph("pl", 11)
    n = len(ip) - 1
    perm, _ = api.reorder(ip, ic, 1, 2, 4)
    ref = oracle.pack(ip, ic, None, 0x3C00, perm, 128, 4)
    cuts = [0, 512, 1024, n]
    for a, b in zip(cuts[:-1], cuts[1:]):
        P = api.pack(ip, ic, perm, 1, 2, 4, row_begin=a, row_end=b)
        got = P.export_canonical()
        pa, pb = a // 128, (b + 127) // 128
        m0, m1 = ref["panel_ptr"][pa], ref["panel_ptr"][pb]
        assert np.array_equal(got["panel_ptr"], ref["panel_ptr"][pa:pb + 1] - m0)
        assert np.array_equal(got["mb_seg"], ref["mb_seg"][m0:m1])
        assert np.array_equal(got["nib"], ref["nib"][m0 * 128:m1 * 128])
        assert np.array_equal(got["vals"], ref["vals"][m0 * 256:m1 * 256])
        r0, r1 = ref["res_rowptr"][a], ref["res_rowptr"][b]
        assert np.array_equal(got["res_rowptr"], ref["res_rowptr"][a:b + 1] - r0)
        assert np.array_equal(got["res_col"], ref["res_col"][r0:r1])


def _spmm_check(ip, ic, perm, V, M, F, dtype, seed, part_check=True):
    dev = _cuda()
    n = len(ip) - 1
    v32, bits, v64 = _values(ip, ic, dtype, seed)
    X32 = graphs.features(n, F, seed + 1)
    xbits, x64 = graphs.round16(X32, dtype)
    Y_ref, E, _ = oracle.spmm(ip, ic, v64, x64)
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=v32)
    tdt = torch.float16 if dtype == "f16" else torch.bfloat16
    ldx = (F + 7) // 8 * 8
    X = torch.zeros((n, ldx), dtype=torch.int16, device=dev)
    X[:, :F] = torch.from_numpy(xbits.view(np.int16)).to(dev)
    X = X.view(tdt)
    PX = torch.empty_like(X)
    perm_d = torch.from_numpy(perm.astype(np.int32)).to(dev)
    api.permute_rows(X, PX, perm_d, dtype)
    Yp = torch.full((n, F), float("nan"), dtype=torch.float32, device=dev)
    api.spmm(P, PX, Yp, F=F)
    Y = torch.empty_like(Yp)
    api.unpermute_rows(Yp, Y, perm_d, "f32")
    torch.cuda.synchronize()
    Yh = Y.cpu().numpy().astype(np.float64)
    assert np.isfinite(Yh).all()
    err = np.abs(Yh - Y_ref)
    bad = err > TOL * E + 1e-30
    assert not bad.any(), "max err %g at %s (bound %g)" % (err.max(), np.argwhere(bad)[0], (TOL * E)[bad][0])
    return P


@pytest.mark.parametrize("kind,seed,V,M", CASES)
@pytest.mark.parametrize("F", [32, 128])
def test_spmm_parity(kind, seed, V, M, F):
    ip, ic = _graph(kind, seed)
    perm, _ = api.reorder(ip, ic, V, 2, M)
    _spmm_check(ip, ic, perm, V, M, F, "f16", seed)


@pytest.mark.parametrize("F", [1, 8, 17, 64, 100, 192, 200, 256, 300, 520])
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_spmm_feature_widths(F, dtype):
    ip, ic = _graph("er", 21)
    n = len(ip) - 1
    perm = np.random.default_rng(3).permutation(n).astype(np.int32)
    _spmm_check(ip, ic, perm, 1, 4, F, dtype, 21)


def test_spmm_identity_perm_and_residual_heavy():
    # random order without reorder: many violations -> large residual at 128:2:16
    ip, ic = _graph("pl", 31)
    n = len(ip) - 1
    P = _spmm_check(ip, ic, np.arange(n, dtype=np.int32), 128, 16, 64, "f16", 31)
    assert P.info()["residual_nnz"] > 0


def test_spmm_sptc_plus_residual_equals_total():
    dev = _cuda()
    ip, ic = _graph("band", 41)
    n = len(ip) - 1
    perm, _ = api.reorder(ip, ic, 8, 2, 8)
    P = api.pack(ip, ic, perm, 8, 2, 8)
    X = torch.randn((n, 64), device=dev).to(torch.float16)
    Y1 = torch.empty((n, 64), device=dev)
    Y2 = torch.empty((n, 64), device=dev)
    api.spmm(P, X, Y1)
    api.spmm(P, X, Y2, part="sptc")
    api.spmm(P, X, Y2, part="residual")
    torch.cuda.synchronize()
    assert torch.equal(Y1, Y2)


def test_dense_conforming_panel_equals_dense_gemm():
    """A fully 2:4-dense panel (every 4-group of every row holds 2 nonzeros) is a plain
    structured-sparse GEMM: compare with torch's dense fp32 matmul of the same operands."""
    dev = _cuda()
    n = 256
    rows, cols = [], []
    rng = np.random.default_rng(5)
    for i in range(n):
        for g in range(n // 4):
            for j in sorted(rng.choice(4, 2, replace=False)):
                rows.append(i)
                cols.append(4 * g + j)
    A = np.zeros((n, n), bool)
    A[rows, cols] = True
    A = A | A.T  # symmetric (may exceed 2 per group -> residual keeps it exact)
    ip = np.concatenate([[0], np.cumsum(A.sum(1))]).astype(np.int64)
    ic = np.nonzero(A)[1].astype(np.int32)
    _spmm_check(ip, ic, np.arange(n, dtype=np.int32), 1, 4, 128, "bf16", 5)


def test_empty_rows_and_isolated_vertices():
    # vertices 300..399 isolated: their rows of Y must be exactly 0
    dev = _cuda()
    ipa, ica = graphs.er_graph(300, 1500, 9)
    n = 400
    ip = np.concatenate([ipa, np.full(100, ipa[-1])]).astype(np.int64)
    P = _spmm_check(ip, ica, np.arange(n, dtype=np.int32), 1, 4, 64, "f16", 9)
    X = torch.ones((n, 64), device=dev, dtype=torch.float16)
    Y = torch.full((n, 64), 7.0, device=dev)
    api.spmm(P, X, Y)
    torch.cuda.synchronize()
    assert torch.all(Y[300:] == 0)


@pytest.mark.parametrize("kind,seed,V,M", [("c1", 1, 1, 4), ("pl", 3, 1, 4), ("band", 5, 64, 8),
                                           ("pl", 6, 128, 16)])
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_spmm_original_order_fused(kind, seed, V, M, dtype):
    """NM_PACK_ORIGINAL_ORDER: X in original order in, Y = A X in original order out, same
    canonical pack; also row shards writing disjoint rows of one Y."""
    dev = _cuda()
    ip, ic = _graph(kind, seed)
    n = len(ip) - 1
    F = 96
    perm, _ = api.reorder(ip, ic, V, 2, M)
    v32, bits, v64 = _values(ip, ic, dtype, seed)
    xbits, x64 = graphs.round16(graphs.features(n, F, seed + 2), dtype)
    Y_ref, E, _ = oracle.spmm(ip, ic, v64, x64)
    tdt = torch.float16 if dtype == "f16" else torch.bfloat16
    X = torch.from_numpy(xbits.view(np.int16)).to(dev).view(tdt)
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=v32, order="original")
    ref = oracle.pack(ip, ic, bits, 0, perm, _vp(V), 4 if V == 1 else M)
    got = P.export_canonical()
    for k in ("panel_ptr", "mb_seg", "nib", "vals", "res_rowptr", "res_col", "res_val"):
        assert np.array_equal(ref[k], got[k]), k
    Y = torch.full((n, F), float("nan"), device=dev)
    api.spmm(P, X, Y)
    torch.cuda.synchronize()
    err = np.abs(Y.cpu().numpy().astype(np.float64) - Y_ref)
    assert (err <= TOL * E).all(), err.max()
    # two row shards into one buffer
    Y2 = torch.full((n, F), float("nan"), device=dev)
    cut = ((n // 2) // 128) * 128
    for a, b in ((0, cut), (cut, n)):
        Ps = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=v32, order="original", row_begin=a, row_end=b)
        api.spmm(Ps, X, Y2)
    torch.cuda.synchronize()
    assert torch.equal(Y, Y2)


# ------------------------------------------------------------------------------------------
# hybrid split (nm_pack_hybrid, reading #27): thin meta-blocks go to the residual
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("kind,seed,V,M,tau", [("c1", 1, 1, 4, 3), ("pl", 3, 1, 4, 8), ("pl", 6, 128, 16, 2),
                                               ("band", 5, 64, 8, 5), ("er", 7, 8, 8, 40),
                                               ("band", 4, 1, 4, 10 ** 6)])
@pytest.mark.parametrize("order", ["permuted", "original"])
def test_pack_hybrid_canonical_bit_exact(kind, seed, V, M, tau, order):
    _cuda()
    ip, ic = _graph(kind, seed)
    perm, _ = api.reorder(ip, ic, V, 2, M)
    v32, bits, _ = _values(ip, ic, "f16", seed)
    Mp = 4 if V == 1 else M
    ref = oracle.pack(ip, ic, bits, 0, perm, _vp(V), Mp, tau=tau)
    P = api.pack(ip, ic, perm, V, 2, M, dtype="f16", val=v32, tau=tau, order=order)
    got = P.export_canonical()
    for k in ("panel_ptr", "mb_seg", "sel", "nib", "vals", "res_rowptr", "res_col", "res_val"):
        assert np.array_equal(ref[k], got[k]), k
    inf = P.info()
    assert inf["n_mb"] == ref["n_mb"] and inf["residual_nnz"] == ref["res_nnz"]
    assert inf["packed_nnz"] + inf["residual_nnz"] == ip[-1]


@pytest.mark.parametrize("kind,seed,V,M,tau", [("pl", 3, 1, 4, 8), ("band", 5, 64, 8, 5), ("c1", 1, 1, 4, 10 ** 6)])
def test_spmm_hybrid_parity(kind, seed, V, M, tau):
    """Y of the hybrid pack (original order, fused permutation) within the north-star bound."""
    dev = _cuda()
    ip, ic = _graph(kind, seed)
    n = len(ip) - 1
    F = 128
    perm, _ = api.reorder(ip, ic, V, 2, M)
    v32, bits, v64 = _values(ip, ic, "f16", seed)
    xbits, x64 = graphs.round16(graphs.features(n, F, seed + 2), "f16")
    Y_ref, E, _ = oracle.spmm(ip, ic, v64, x64)
    X = torch.from_numpy(xbits.view(np.int16)).to(dev).view(torch.float16)
    P = api.pack(ip, ic, perm, V, 2, M, dtype="f16", val=v32, order="original", tau=tau)
    Y = torch.full((n, F), float("nan"), device=dev)
    api.spmm(P, X, Y)
    torch.cuda.synchronize()
    err = np.abs(Y.cpu().numpy().astype(np.float64) - Y_ref)
    assert (err <= TOL * E).all(), err.max()


def _star_plus_er(n=3000, hubs=(0, 17), m=6000, seed=51):
    """ER graph plus hub vertices adjacent to every other vertex: hub rows of degree ~n split
    into several residual work items (kResSeg = 256 entries each)."""
    ip, ic = graphs.er_graph(n, m, seed)
    A = set()
    for i in range(n):
        for k in range(ip[i], ip[i + 1]):
            A.add((i, int(ic[k])))
    for h in hubs:
        for v in range(n):
            if v != h:
                A.add((h, v))
                A.add((v, h))
    rows = np.array(sorted(A), dtype=np.int64)
    ip2 = np.concatenate([[0], np.cumsum(np.bincount(rows[:, 0], minlength=n))]).astype(np.int64)
    return ip2, rows[:, 1].astype(np.int32)


@pytest.mark.parametrize("F", [32, 128, 300])
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_residual_split_hub_rows(F, dtype):
    """Everything in the residual (tau = inf): hub rows are cut into several work items whose
    partials are combined deterministically -- parity and bitwise-identical repeats."""
    dev = _cuda()
    ip, ic = _star_plus_er()
    n = len(ip) - 1
    perm = np.random.default_rng(2).permutation(n).astype(np.int32)
    v32, bits, v64 = _values(ip, ic, dtype, 3)
    xbits, x64 = graphs.round16(graphs.features(n, F, 4), dtype)
    Y_ref, E, _ = oracle.spmm(ip, ic, v64, x64)
    tdt = torch.float16 if dtype == "f16" else torch.bfloat16
    ldx = (F + 7) // 8 * 8
    X = torch.zeros((n, ldx), dtype=torch.int16, device=dev)
    X[:, :F] = torch.from_numpy(xbits.view(np.int16)).to(dev)
    X = X.view(tdt)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype=dtype, val=v32, order="original", tau=10 ** 9)
    assert P.info()["n_mb"] == 0 and P.info()["residual_nnz"] == ip[-1]
    outs = []
    for _ in range(3):
        Y = torch.full((n, F), float("nan"), device=dev)
        api.spmm(P, X, Y, F=F)
        torch.cuda.synchronize()
        outs.append(Y.cpu().numpy())
    err = np.abs(outs[0].astype(np.float64) - Y_ref)
    assert (err <= TOL * E).all(), err.max()
    assert all(np.array_equal(outs[0], o) for o in outs[1:])


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_concurrent_spmm_on_one_handle(dtype):
    """nm.h "Handles": the packed matrix is immutable after nm_pack, so two nm_spmm calls on
    the SAME handle on two streams (hub rows split over several residual work items, plus the
    tensor-core part) must both be right -- repeated many times with the launches interleaved."""
    dev = _cuda()
    ip, ic = _star_plus_er(n=6000, hubs=(0, 17, 999), m=18000, seed=52)
    n = len(ip) - 1
    F = 128
    perm = np.random.default_rng(5).permutation(n).astype(np.int32)
    v32, bits, v64 = _values(ip, ic, dtype, 6)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype=dtype, val=v32, order="original", tau=2)
    st = P.stats()
    assert st["residual_split_rows"] > 0 and st["n_mb"] > 0
    tdt = torch.float16 if dtype == "f16" else torch.bfloat16
    Xs, refs = [], []
    for seed in (7, 8):
        xbits, x64 = graphs.round16(graphs.features(n, F, seed), dtype)
        Xs.append(torch.from_numpy(xbits.view(np.int16)).to(dev).view(tdt))
        refs.append(oracle.spmm(ip, ic, v64, x64)[:2])
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    Ys = [torch.empty((n, F), device=dev) for _ in range(2)]
    for it in range(20):
        for k in (0, 1) if it % 2 == 0 else (1, 0):
            Ys[k].fill_(float("nan"))
        torch.cuda.synchronize()
        for k in (0, 1):
            api.spmm(P, Xs[k], Ys[k], stream=streams[k])
        torch.cuda.synchronize()
        for k in (0, 1):
            Y_ref, E = refs[k]
            err = np.abs(Ys[k].cpu().numpy().astype(np.float64) - Y_ref)
            assert (err <= TOL * E).all(), (it, k, err.max())


@pytest.mark.parametrize("kind,seed,V,M", CASES)
@pytest.mark.parametrize("F", [32, 128, 300])
def test_sptc_formats_agree_bitwise(kind, seed, V, M, F):
    """The full-record kernel (format 1), the compressed-record kernel (format 2) and the
    compressed-record kernel with A in tensor memory (format 3) feed the tensor core identical
    operands in the same order: Yp must agree bitwise, and all must meet the oracle bound."""
    dev = _cuda()
    ip, ic = _graph(kind, seed)
    n = len(ip) - 1
    perm = np.random.default_rng(seed + 100).permutation(n).astype(np.int32)
    dtype = "bf16" if seed % 2 else "f16"
    v32, bits, v64 = _values(ip, ic, dtype, seed)
    xbits, x64 = graphs.round16(graphs.features(n, F, seed + 1), dtype)
    tdt = torch.float16 if dtype == "f16" else torch.bfloat16
    ldx = (F + 7) // 8 * 8
    Xb = torch.zeros((n, ldx), dtype=torch.int16, device=dev)
    Xb[:, :F] = torch.from_numpy(xbits.view(np.int16)).to(dev)
    X = Xb.view(tdt)[:, :F]
    P = api.pack(ip, ic, perm, V, 2, M, dtype=dtype, val=v32, order="original")
    outs = []
    for fmt in (1, 2, 3):
        Y = torch.full((n, F), float("nan"), device=dev)
        api.spmm(P, X, Y, part="sptc", format=fmt)
        api.spmm(P, X, Y, part="residual")
        torch.cuda.synchronize()
        outs.append(Y.cpu().numpy())
    assert np.array_equal(outs[0], outs[1])
    assert np.array_equal(outs[0], outs[2])
    Y_ref, E, _ = oracle.spmm(ip, ic, v64, x64)
    err = np.abs(outs[0].astype(np.float64) - Y_ref)
    assert (err <= TOL * E).all(), err.max()


# ------------------------------------------------------------------------------------------
# panel height V_p (nm.h: Vp in {64, 128}; at 64 two canonical panels share a 128-row kernel
# panel's chunks, each k-group holding one half's values)
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("kind,seed,V,M,Vp", [("band", 5, 64, 8, 64), ("band", 5, 64, 8, 128), ("pl", 3, 1, 4, 64),
                                              ("pl", 6, 128, 16, 64), ("er", 7, 8, 8, 64), ("tiny", 1, 1, 4, 64),
                                              ("band", 4, 16, 8, 16), ("pl", 3, 32, 8, 32), ("er", 2, 32, 16, 16)])
@pytest.mark.parametrize("order", ["permuted", "original"])
def test_panel_height_vp(kind, seed, V, M, Vp, order):
    dev = _cuda()
    ip, ic = _graph(kind, seed)
    n = len(ip) - 1
    F = 72
    perm, _ = api.reorder(ip, ic, V, 2, M)
    v32, bits, v64 = _values(ip, ic, "bf16", seed)
    Mp = 4 if V == 1 else M
    ref = oracle.pack(ip, ic, bits, 0, perm, Vp, Mp)
    P = api.pack(ip, ic, perm, V, 2, M, dtype="bf16", val=v32, order=order, Vp=Vp)
    assert P.stats()["Vp"] == Vp
    got = P.export_canonical()
    for k in ("panel_ptr", "mb_seg", "sel", "nib", "vals", "res_rowptr", "res_col", "res_val"):
        assert np.array_equal(ref[k], got[k]), k
    xbits, x64 = graphs.round16(graphs.features(n, F, seed + 2), "bf16")
    Y_ref, E, _ = oracle.spmm(ip, ic, v64, x64)
    X = torch.from_numpy(xbits.view(np.int16)).to(dev).view(torch.bfloat16)
    if order == "permuted":
        perm_d = torch.from_numpy(perm.astype(np.int32)).to(dev)
        PX = torch.empty_like(X)
        api.permute_rows(X, PX, perm_d, "bf16")
        Yp = torch.full((n, F), float("nan"), device=dev)
        api.spmm(P, PX, Yp, F=F)
        Y = torch.empty_like(Yp)
        api.unpermute_rows(Yp, Y, perm_d, "f32")
    else:
        Y = torch.full((n, F), float("nan"), device=dev)
        api.spmm(P, X, Y, F=F)
        # row shards starting at an odd multiple of 64 (legal at Vp = 64 only).  The shard's
        # 128-row kernel panels pair different 64-row panels than the whole pack's, so the
        # chunking (and the fp32 summation grouping inside each MMA) differs: checked against
        # the oracle bound, not bitwise against Y.
        if Vp < 128 and n > 256:
            cut = ((n // 2) // 128) * 128 + Vp
            Y2 = torch.full((n, F), float("nan"), device=dev)
            for a, b in ((0, cut), (cut, n)):
                Ps = api.pack(ip, ic, perm, V, 2, M, dtype="bf16", val=v32, order="original", Vp=Vp,
                              row_begin=a, row_end=b)
                api.spmm(Ps, X, Y2, F=F)
            torch.cuda.synchronize()
            err2 = np.abs(Y2.cpu().numpy().astype(np.float64) - Y_ref)
            assert (err2 <= TOL * E).all(), err2.max()
    torch.cuda.synchronize()
    err = np.abs(Y.cpu().numpy().astype(np.float64) - Y_ref)
    assert (err <= TOL * E).all(), err.max()


@pytest.mark.parametrize("V", [16, 64])
def test_vp64_conforming_v64_has_empty_residual(V):
    """A V:2:8-conforming matrix (every V-row x 8-column meta-block uses <= 4 columns, every
    row <= 2 per 8-segment, L194 / L226-230) packs losslessly into the tensor-core form at
    Vp = V, where 128-row panels would merge the blocks' column sets and spill."""
    _cuda()
    rng = np.random.default_rng(5)
    n, M = 1024, 8
    rows = [[] for _ in range(n)]
    for p in range(n // V):
        for s in range(n // M):
            if rng.random() < 0.25:
                cols = s * M + np.sort(rng.choice(M, 4, replace=False))
                for i in range(p * V, p * V + V):
                    if rng.random() < 0.5:
                        rows[i].extend(rng.choice(cols, 2, replace=False).tolist())
    ip = np.zeros(n + 1, np.int64)
    ic = []
    for i in range(n):
        r = sorted(set(rows[i]))
        ic.extend(r)
        ip[i + 1] = ip[i] + len(r)
    ic = np.array(ic, np.int32)
    ident = np.arange(n, dtype=np.int32)
    P64 = api.pack(ip, ic, ident, V, 2, M)
    P128 = api.pack(ip, ic, ident, V, 2, M, Vp=128)
    assert P64.stats()["Vp"] == V and P128.stats()["Vp"] == 128
    assert P64.info()["residual_nnz"] == 0
    assert P128.info()["residual_nnz"] > 0
    ref = oracle.pack(ip, ic, None, 0x3C00, ident, V, M)
    assert ref["res_nnz"] == 0
    got = P64.export_canonical()
    for k in ("panel_ptr", "mb_seg", "sel", "nib", "vals"):
        assert np.array_equal(ref[k], got[k]), k
