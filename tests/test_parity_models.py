"""GPU parity of the SGC / SAGE / Cheb aggregations against
the oracle's fp64 references (tests/test_oracle_models.py pins them), elementwise:

* SGC: hop by hop.  Hop k's operand is hop k-1's result rounded to bf16 (returned by the K=k-1
  call as Y16); hop k must satisfy the north-star bound 1e-3 * (|Ahat| |operand|) against the
  oracle SpMM of exactly that operand.
* SAGE / Cheb: the error of every 16-bit intermediate is propagated through the layer in fp64
  (|L| e + 1e-3 |L||T| per SpMM, 2^-8 |T| per bf16 rounding) and through |W|; the output adds its
  own bf16 rounding.  The bound is elementwise.
"""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
U = 2.0 ** -8  # bf16 unit roundoff (8 significant bits)


def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _bf(a, dev):
    bits, v = graphs.round16(np.asarray(a, np.float32), "bf16")
    return torch.from_numpy(bits.view(np.int16)).to(dev).view(torch.bfloat16), v


def _un(t):
    return graphs.bf16_bits_to_f64(t.contiguous().view(torch.int16).cpu().numpy().view(np.uint16))


def _graph():
    n = 3000
    ip, ic = graphs.lmcl_graph(n, 30000, 2.3, 4, 0.6, 21, self_loops=True)
    return n, ip, ic


@pytest.mark.parametrize("order", ["permuted", "original"])
def test_sgc_hop_by_hop(order):
    dev = _cuda()
    n, ip, ic = _graph()
    vals = graphs.gcn_norm_values(ip, ic)
    _, v64 = graphs.round16(vals, "bf16")
    perm = np.random.default_rng(1).permutation(n).astype(np.int32)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals, order=order, tau=4)
    F = 64
    X, x64 = _bf(np.random.default_rng(2).standard_normal((n, F)), dev)
    # permuted-order packs chain in permuted order: feed P X, compare against P (A^k X)
    if order == "permuted":
        X = X[torch.from_numpy(perm.astype(np.int64)).to(dev)].contiguous()
    prev = x64
    for K in (1, 2, 3):
        Y = torch.empty((n, F), device=dev)
        Y16 = torch.empty((n, F), dtype=torch.bfloat16, device=dev)
        api.sgc_propagate(P, X, Y, K, Y16=Y16)
        torch.cuda.synchronize()
        y = Y.cpu().numpy().astype(np.float64)
        y16 = _un(Y16)
        if order == "permuted":
            y_o, y16_o = np.empty_like(y), np.empty_like(y16)
            y_o[perm], y16_o[perm] = y, y16
            y, y16 = y_o, y16_o
        ref, E, _ = oracle.spmm(ip, ic, v64, prev)
        assert (np.abs(y - ref) <= 1e-3 * E + 1e-30).all(), (K, np.abs(y - ref).max())
        assert np.array_equal(y16, graphs.round16(y.astype(np.float32), "bf16")[1])
        prev = y16


def test_sage_mean_layer():
    dev = _cuda()
    n, ip, ic = _graph()
    deg = np.diff(ip)
    vmean = (1.0 / np.repeat(deg, deg)).astype(np.float32)  # D^-1 A
    _, vm64 = graphs.round16(vmean, "bf16")
    perm = np.random.default_rng(3).permutation(n).astype(np.int32)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vmean)
    rng = np.random.default_rng(4)
    F_in, F_out = 64, 32
    H, h64 = _bf(rng.standard_normal((n, F_in)), dev)
    Ws, ws64 = _bf(rng.standard_normal((F_in, F_out)) / 8, dev)
    Wn, wn64 = _bf(rng.standard_normal((F_in, F_out)) / 8, dev)
    b = (rng.standard_normal(F_out) * 0.1).astype(np.float32)
    pd = torch.from_numpy(perm.astype(np.int64)).to(dev)
    out = torch.empty((n, F_out), dtype=torch.bfloat16, device=dev)
    api.sage_layer(P, H[pd].contiguous(), Ws, Wn, torch.from_numpy(b).to(dev), out, relu=True)
    torch.cuda.synchronize()
    got = np.empty((n, F_out))
    got[perm] = _un(out)
    ref, agg = oracle.sage_layer(ip, ic, vm64, h64, ws64, wn64, b.astype(np.float64), relu=True)
    _, Eagg, _ = oracle.spmm(ip, ic, np.abs(vm64), np.abs(h64))
    e_agg = 1e-3 * Eagg + U * np.abs(agg)                       # SpMM bound + bf16 rounding of the mean
    bound = e_agg @ np.abs(wn64) + U * np.abs(ref) + 1e-6 * (np.abs(h64) @ np.abs(ws64) + np.abs(agg) @ np.abs(wn64))
    assert (np.abs(got - ref) <= bound + 1e-30).all(), np.abs(got - ref).max()


@pytest.mark.parametrize("K", [1, 2, 3, 4])
def test_cheb_layer(K):
    dev = _cuda()
    n, ip, ic = _graph()
    rows = np.repeat(np.arange(n), np.diff(ip))
    keep = rows != ic                                            # Lhat = -D^-1/2 A D^-1/2 (no self-loops)
    ip2 = np.concatenate([[0], np.cumsum(np.bincount(rows[keep], minlength=n))]).astype(np.int64)
    ic2 = ic[keep]
    vL = -graphs.gcn_norm_values(ip2, ic2)
    _, vL64 = graphs.round16(vL, "bf16")
    perm = np.random.default_rng(5).permutation(n).astype(np.int32)
    P = api.pack(ip2, ic2, perm, 1, 2, 4, dtype="bf16", val=vL)
    rng = np.random.default_rng(6)
    F_in, F_out = 32, 16
    H, h64 = _bf(rng.standard_normal((n, F_in)), dev)
    W, w64 = _bf(rng.standard_normal((K * F_in, F_out)) / 8, dev)
    b = (rng.standard_normal(F_out) * 0.1).astype(np.float32)
    pd = torch.from_numpy(perm.astype(np.int64)).to(dev)
    out = torch.empty((n, F_out), dtype=torch.bfloat16, device=dev)
    api.cheb_layer(P, H[pd].contiguous(), W, torch.from_numpy(b).to(dev), out, K, relu=False)
    torch.cuda.synchronize()
    got = np.empty((n, F_out))
    got[perm] = _un(out)
    Ws = [w64[k * F_in:(k + 1) * F_in] for k in range(K)]
    ref, T = oracle.cheb_layer(ip2, ic2, vL64, h64, Ws, b.astype(np.float64), relu=False)
    aL = np.abs(vL64)
    e = [np.zeros_like(h64)]                                     # elementwise error bound of each T_k
    for k in range(1, K):
        prop, _, _ = oracle.spmm(ip2, ic2, aL, e[k - 1])          # |L| e_{k-1}
        _, EL, _ = oracle.spmm(ip2, ic2, aL, np.abs(T[k - 1]) + e[k - 1])
        spmm_err = prop + 1e-3 * EL
        if k == 1:
            e.append(spmm_err + U * (np.abs(T[1]) + spmm_err))
        else:
            ek = 2.0 * spmm_err + e[k - 2]
            e.append(ek + U * (np.abs(T[k]) + ek))
    bound = sum(e[k] @ np.abs(Ws[k]) for k in range(K)) + U * (np.abs(ref) + 1e-3) + \
        1e-6 * sum((np.abs(T[k]) + e[k]) @ np.abs(Ws[k]) for k in range(K))
    assert (np.abs(got - ref) <= bound).all(), np.abs(got - ref).max()
