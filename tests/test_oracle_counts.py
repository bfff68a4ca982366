"""Pins for the oracle's violation counts and the Stage-1 sort key (brute force on dense
matrices, written here independently of the oracle).

omega, PScore (L396), MBscore (L382, Fig. 3 caption L370, reading #5),
Stage-1 order (Alg. 2 lines 4-13, L326-362; reading #6: ascending lexicographic order of the
per-row code vectors, stable).
"""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import graphs


def dense_B(indptr, indices, perm):
    n = len(indptr) - 1
    A = np.zeros((n, n), bool)
    for i in range(n):
        A[i, indices[indptr[i]:indptr[i + 1]]] = True
    p = np.asarray(perm)
    return A[np.ix_(p, p)]


def brute_counts(B, V, N, M):
    n = B.shape[0]
    S = (n + M - 1) // M
    omega = 0
    ps = np.zeros(S, np.int64)
    for i in range(n):
        for s in range(S):
            c = int(B[i, s * M:(s + 1) * M].sum())
            if c > N:
                omega += 1
                ps[s] += 1
    mb = 0
    for r in range(0, n, V):
        for s in range(S):
            cols = B[r:r + V, s * M:(s + 1) * M].any(axis=0).sum()
            if cols > 4:
                mb += 1
    return omega, mb, ps


def _graphs():
    out = []
    for n, m, seed in [(16, 20, 1), (37, 120, 2), (64, 300, 3), (50, 400, 4)]:
        out.append(graphs.er_graph(n, m, seed))
    out.append(graphs.lmcl_graph(80, 400, 2.1, 1, 0.0, 5, scramble=True))
    out.append(graphs.banded_graph(90, 8, 6))
    out.append(graphs.er_graph(40, 100, 7, self_loops=True))
    return out


@pytest.mark.parametrize("gi", range(7))
@pytest.mark.parametrize("V,N,M", [(1, 2, 4), (1, 2, 8), (4, 2, 8), (8, 2, 4), (16, 2, 16),
                                   (3, 1, 4), (1, 2, 5)])
def test_counts_match_brute_force(gi, V, N, M):
    indptr, indices = _graphs()[gi]
    n = len(indptr) - 1
    rng = np.random.default_rng(100 + gi)
    for perm in (np.arange(n), rng.permutation(n)):
        w, mb, ps = oracle.counts(indptr, indices, perm, V, N, M)
        bw, bmb, bps = brute_counts(dense_B(indptr, indices, perm), V, N, M)
        assert (w, mb) == (bw, bmb)
        assert np.array_equal(ps, bps)


def _reflected_rank(M):
    seq = ["0", "1"]
    for _ in range(M - 1):
        seq = ["0" + s for s in seq] + ["1" + s for s in reversed(seq)]
    return {int(s, 2): r for r, s in enumerate(seq)}


@pytest.mark.parametrize("gi", range(7))
@pytest.mark.parametrize("M", [4, 8])
def test_stage1_order_is_stable_lexicographic_sort_of_dense_code_vectors(gi, M):
    indptr, indices = _graphs()[gi]
    n = len(indptr) - 1
    N = 2
    rank = _reflected_rank(M)
    rng = np.random.default_rng(7 + gi)
    perm = rng.permutation(n).astype(np.int32)
    B = dense_B(indptr, indices, perm)
    S = (n + M - 1) // M
    vec = []
    for i in range(n):
        row = []
        for s in range(S):
            bits = 0
            for j in range(M):
                q = s * M + j
                bits = (bits << 1) | (1 if q < n and B[i, q] else 0)  # first column -> MSB
            c = rank[bits]
            if bin(bits).count("1") > N:
                c = -c
            row.append(c)
        vec.append(tuple(row))
    order = sorted(range(n), key=lambda i: vec[i])  # Python's sort is stable
    expect = perm[np.array(order)]
    got = oracle.stage1_once(indptr, indices, perm, N, M)
    assert np.array_equal(got, expect)


def test_validate():
    indptr, indices = graphs.er_graph(30, 60, 3)
    assert oracle.validate(indptr, indices) == 0
    bad = indices.copy()
    bad[0], bad[1] = bad[1], bad[0]
    assert oracle.validate(indptr, bad) == 1
    # drop one direction of an edge -> not symmetric
    ip = indptr.copy()
    ind = np.delete(indices, 0)
    ip[1:] -= 1
    assert oracle.validate(ip, ind) == 2
