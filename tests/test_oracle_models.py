"""Pins for the oracle's SGC / SAGE / Cheb references:
closed forms that do not reuse the references' own recurrences.

* SGC on Ahat = lambda I: Ahat^K X = lambda^K X.
* Cheb on Lhat = lambda I: T_k = cos(k arccos lambda) H (Chebyshev polynomials of the first
  kind), so the layer is sum_k cos(k acos lambda) H W_k + b.
* Cheb with K = 1 is the dense layer H W_0 + b; on a graph with no edges T_1 = 0, T_2 = -H.
* SAGE: with W_neigh = 0 the layer is H W_self + b; on a d-regular graph whose vertices all
  carry the same feature row h, the neighbour mean is h.
"""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import graphs


def _diag(n):
    return np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32)


@pytest.mark.parametrize("lam,K", [(0.5, 1), (-0.7, 3), (0.9, 5)])
def test_sgc_on_scaled_identity(lam, K):
    n, F = 40, 6
    ip, ic = _diag(n)
    X = np.random.default_rng(1).standard_normal((n, F))
    Y = oracle.sgc_propagate(ip, ic, np.full(n, lam), X, K)
    np.testing.assert_allclose(Y, lam ** K * X, rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("lam", [-0.9, -0.3, 0.0, 0.4, 0.95])
@pytest.mark.parametrize("K", [1, 2, 3, 5])
def test_cheb_on_scaled_identity_is_the_chebyshev_polynomial(lam, K):
    n, F, Fo = 30, 8, 5
    ip, ic = _diag(n)
    rng = np.random.default_rng(2)
    H = rng.standard_normal((n, F))
    Ws = [rng.standard_normal((F, Fo)) for _ in range(K)]
    b = rng.standard_normal(Fo)
    out, T = oracle.cheb_layer(ip, ic, np.full(n, lam), H, Ws, b, relu=False)
    expect = sum(np.cos(k * np.arccos(lam)) * H @ Ws[k] for k in range(K)) + b
    np.testing.assert_allclose(out, expect, rtol=1e-10, atol=1e-10)


def test_cheb_degenerate_cases():
    n, F, Fo = 50, 8, 4
    rng = np.random.default_rng(3)
    H = rng.standard_normal((n, F))
    W0 = rng.standard_normal((F, Fo))
    b = rng.standard_normal(Fo)
    ip, ic = graphs.er_graph(n, 120, 4)
    out, _ = oracle.cheb_layer(ip, ic, graphs.symmetric_values(ip, ic, 5), H, [W0], b, relu=True)
    np.testing.assert_allclose(out, np.maximum(H @ W0 + b, 0.0), rtol=1e-12)
    ip0, ic0 = np.zeros(n + 1, np.int64), np.zeros(0, np.int32)   # no edges: L = 0
    _, T = oracle.cheb_layer(ip0, ic0, np.zeros(0), H, [W0] * 3, b, relu=False)
    assert np.all(T[1] == 0.0) and np.allclose(T[2], -H)


def test_sage_closed_forms():
    rng = np.random.default_rng(4)
    n, F, Fo = 64, 8, 6
    ip, ic = graphs.banded_graph(n, 4, 7)
    deg = np.diff(ip)
    vmean = (1.0 / np.repeat(deg, deg)).astype(np.float64)
    H = rng.standard_normal((n, F))
    Ws, Wn, b = rng.standard_normal((F, Fo)), rng.standard_normal((F, Fo)), rng.standard_normal(Fo)
    out, _ = oracle.sage_layer(ip, ic, vmean, H, Ws, np.zeros((F, Fo)), b, relu=False)
    np.testing.assert_allclose(out, H @ Ws + b, rtol=1e-12)
    # ring graph (2-regular) with identical rows: the neighbour mean is the row itself
    ring = [(i, (i + 1) % n) for i in range(n)]
    a = np.array([min(u, v) for u, v in ring]), np.array([max(u, v) for u, v in ring])
    ipr, icr = graphs._symmetric_csr(n, a[0], a[1])
    h = rng.standard_normal(F)
    Hh = np.tile(h, (n, 1))
    out, agg = oracle.sage_layer(ipr, icr, np.full(len(icr), 0.5), Hh, Ws, Wn, b, relu=False)
    np.testing.assert_allclose(agg, Hh, rtol=1e-12)
    np.testing.assert_allclose(out, Hh @ Ws + Hh @ Wn + b, rtol=1e-12)
