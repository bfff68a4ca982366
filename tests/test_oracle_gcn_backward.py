"""Pins of the oracle's GCN-layer backward against central finite
differences of L = sum(G * Hout) on tiny problems -- independent of the backward formulas --
and of its explicit CSR transpose against a dense transpose."""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import graphs


def _problem(seed, n=24, fin=5, fout=4, sym=True):
    rng = np.random.default_rng(seed)
    if sym:
        ip, ic = graphs.er_graph(n, 40, seed, self_loops=True)
    else:  # a non-symmetric pattern: the transpose matters
        A = (rng.random((n, n)) < 0.15)
        ip = np.concatenate([[0], np.cumsum(A.sum(1))]).astype(np.int64)
        ic = np.nonzero(A)[1].astype(np.int32)
    val = rng.uniform(-1, 1, ip[-1])
    H = rng.standard_normal((n, fin))
    W = rng.standard_normal((fin, fout))
    b = rng.standard_normal(fout)
    G = rng.standard_normal((n, fout))
    return ip, ic, val, H, W, b, G


def test_csr_transpose_dense():
    ip, ic, val, *_ = _problem(3, sym=False)
    n = len(ip) - 1
    D = np.zeros((n, n))
    D[np.repeat(np.arange(n), np.diff(ip)), ic] = val
    tp, ti, tv = oracle.csr_transpose(ip, ic, val)
    T = np.zeros((n, n))
    T[np.repeat(np.arange(n), np.diff(tp)), ti] = tv
    assert np.array_equal(T, D.T)


@pytest.mark.parametrize("seed,sym,relu", [(1, True, False), (2, False, False), (4, True, True), (5, False, True)])
def test_backward_matches_finite_differences(seed, sym, relu):
    ip, ic, val, H, W, b, G = _problem(seed, sym=sym)
    Hout, Z = oracle.gcn_layer(ip, ic, val, H, W, b, relu)
    dH, dW, db, _ = oracle.gcn_layer_backward(ip, ic, val, H, W, Z, G, relu)

    def loss(H_, W_, b_):
        return float((G * oracle.gcn_layer(ip, ic, val, H_, W_, b_, relu)[0]).sum())

    eps = 1e-6
    for name, arr, grad in (("W", W, dW), ("b", b, db), ("H", H, dH)):
        num = np.zeros_like(arr)
        for idx in np.ndindex(arr.shape):
            p, m = arr.copy(), arr.copy()
            p[idx] += eps
            m[idx] -= eps
            args_p = {"H": (p, W, b), "W": (H, p, b), "b": (H, W, p)}[name]
            args_m = {"H": (m, W, b), "W": (H, m, b), "b": (H, W, m)}[name]
            num[idx] = (loss(*args_p) - loss(*args_m)) / (2 * eps)
        if relu:  # a ReLU kink within eps of some Z would spoil the difference quotient
            assert np.abs(Z).min() > 1e-4
        np.testing.assert_allclose(grad, num, rtol=1e-5, atol=1e-6, err_msg=name)
