"""Pins for the oracle's canonical packing (reading #19) and fp64 SpMM (the exact result
Y = A X the lossless method reaches)."""
import os

import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import graphs

from test_oracle_counts import dense_B

GOLD = os.path.join(os.path.dirname(__file__), "golden", "f1_figure1.txt")


def dense_bits(indptr, indices, val16, perm):
    n = len(indptr) - 1
    D = np.zeros((n, n), np.uint16)
    P = np.zeros((n, n), bool)
    for i in range(n):
        cols = indices[indptr[i]:indptr[i + 1]]
        D[i, cols] = val16[indptr[i]:indptr[i + 1]]
        P[i, cols] = True
    p = np.asarray(perm)
    return D[np.ix_(p, p)], P[np.ix_(p, p)]


def test_f1_pack_nibbles():
    indptr, indices = graphs.fixture_f1()
    perm = np.array([0, 1, 2, 4, 3, 5, 6, 7], np.int32)
    val16 = np.full(indices.size, 0x3C00, np.uint16)
    pk = oracle.pack(indptr, indices, val16, 0x3C00, perm, 128, 4)
    assert pk["n_mb"] == 2 and pk["res_nnz"] == 0
    assert list(pk["mb_seg"]) == [0, 1]
    rows = {}
    for line in open(GOLD):
        if line.startswith("row"):
            p = line.split()
            rows[int(p[1])] = p[2:]
    for r in range(8):
        for g in range(2):
            nib_hex, slots = rows[r][g].split(":")
            assert pk["nib"][g * 128 + r] == int(nib_hex, 16)
            v0 = pk["vals"][(g * 128 + r) * 2]
            v1 = pk["vals"][(g * 128 + r) * 2 + 1]
            assert (v0 != 0, v1 != 0) == (slots[0] == "a", slots[1] == "b")


def _pack_cases():
    return [
        graphs.er_graph(150, 900, 1),
        graphs.lmcl_graph(260, 1500, 2.1, 1, 0.0, 2, scramble=True),
        graphs.banded_graph(300, 12, 3),
        graphs.er_graph(97, 700, 4, self_loops=True),
    ]


@pytest.mark.parametrize("ci", range(4))
@pytest.mark.parametrize("Vp,Mp", [(64, 4), (128, 4), (64, 8), (128, 16), (128, 8), (16, 8), (32, 4)])
def test_unpack_plus_residual_is_B_bitwise(ci, Vp, Mp):
    indptr, indices = _pack_cases()[ci]
    n = len(indptr) - 1
    rng = np.random.default_rng(ci)
    perm = rng.permutation(n).astype(np.int32)
    vals = graphs.symmetric_values(indptr, indices, seed=5 + ci)
    val16, _ = graphs.round16(vals, "f16")
    pk = oracle.pack(indptr, indices, val16, 0x3C00, perm, Vp, Mp)
    Bd, present = oracle.unpack(pk, n)
    ref, refp = dense_bits(indptr, indices, val16, perm)
    assert np.array_equal(present, refp)
    assert np.array_equal(Bd, ref)
    kept = int(np.count_nonzero(pk["vals"]))
    assert kept + pk["res_nnz"] == indptr[-1]
    # meta-blocks: ascending non-empty segments per panel
    P = (n + Vp - 1) // Vp
    for r in range(P):
        segs = pk["mb_seg"][pk["panel_ptr"][r]:pk["panel_ptr"][r + 1]]
        rows = refp[r * Vp:(r + 1) * Vp]
        expect = sorted({c // Mp for c in np.nonzero(rows.any(axis=0))[0]})
        assert list(segs) == expect
    # sel = 4 largest column counts, ties to smaller offset, ascending (brute force)
    for mb in range(pk["n_mb"]):
        r = np.searchsorted(pk["panel_ptr"], mb, side="right") - 1
        s = pk["mb_seg"][mb]
        cnt = [int(refp[r * Vp:(r + 1) * Vp, s * Mp + j].sum()) if s * Mp + j < n else 0
               for j in range(Mp)]
        exp = sorted(sorted(range(Mp), key=lambda j: (-cnt[j], j))[:4])
        assert list(pk["sel"][mb * 4:mb * 4 + 4]) == exp
    # every nibble is one of the six legal 2:4 codes
    assert set(np.unique(pk["nib"]).tolist()) <= {0x4, 0x8, 0xC, 0x9, 0xD, 0xE}


def test_conforming_matrix_has_empty_residual():
    # each vertex i links to i +- 4: every 4-group of every row holds <= 1 nonzero
    n = 256
    a = np.arange(n - 4)
    indptr, indices = graphs._symmetric_csr(n, a, a + 4)
    w, _, _ = oracle.counts(indptr, indices, np.arange(n), 1, 2, 4)
    assert w == 0
    pk = oracle.pack(indptr, indices, None, 0x3C00, np.arange(n, dtype=np.int32), 128, 4)
    assert pk["res_nnz"] == 0
    # and at 128:2:8 after the reorder of F1-style fixes: vertical conformity => all selected
    pk8 = oracle.pack(indptr, indices, None, 0x3C00, np.arange(n, dtype=np.int32), 128, 8)
    w8, mb8, _ = oracle.counts(indptr, indices, np.arange(n), 128, 2, 8)
    if w8 == 0 and mb8 == 0:
        assert pk8["res_nnz"] == 0


def test_reorder_then_pack_residual_shrinks():
    indptr, indices = graphs.banded_graph(512, 6, 9)
    n = 512
    ident = np.arange(n, dtype=np.int32)
    perm, st = oracle.reorder(indptr, indices, 1, 2, 4)
    r0 = oracle.pack(indptr, indices, None, 0x3C00, ident, 128, 4)["res_nnz"]
    r1 = oracle.pack(indptr, indices, None, 0x3C00, perm, 128, 4)["res_nnz"]
    assert r1 <= r0
    # at Mp = 4 the residual is exactly the overflow of violating 4-vectors
    B = dense_B(indptr, indices, perm)
    over = sum(max(0, int(B[i, s:s + 4].sum()) - 2) for i in range(n) for s in range(0, n, 4))
    assert r1 == over


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_spmm_matches_dense(seed):
    indptr, indices = graphs.er_graph(120, 700, seed, self_loops=bool(seed % 2))
    n = 120
    vals = graphs.uniform_values(indices.size, seed + 10).astype(np.float64)
    X = graphs.features(n, 24, seed + 20).astype(np.float64)
    Y, E, _ = oracle.spmm(indptr, indices, vals, X)
    A = np.zeros((n, n))
    for i in range(n):
        A[i, indices[indptr[i]:indptr[i + 1]]] = vals[indptr[i]:indptr[i + 1]]
    np.testing.assert_allclose(Y, A @ X, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(E, np.abs(A) @ np.abs(X), rtol=1e-12, atol=1e-12)
    Y4, E4, used = oracle.spmm(indptr, indices, vals, X, nthreads=4)
    assert np.array_equal(Y4, Y) and np.array_equal(E4, E)
    rows = np.array([0, 5, 119, 5])
    Yr, Er = oracle.spmm_rows(rows, indptr, indices, vals, X)
    assert np.array_equal(Yr, Y[rows]) and np.array_equal(Er, E[rows])


def test_spmm_identity_and_ones():
    n = 50
    indptr = np.arange(n + 1, dtype=np.int64)
    indices = np.arange(n, dtype=np.int32)
    X = graphs.features(n, 8, 3).astype(np.float64)
    Y, E, _ = oracle.spmm(indptr, indices, None, X)
    assert np.array_equal(Y, X) and np.array_equal(E, np.abs(X))
    # all-ones rows: Y = row sums of X over neighbours, E >= |Y|
    ip, ic = graphs.er_graph(n, 200, 4)
    Y, E, _ = oracle.spmm(ip, ic, None, np.ones((n, 3)))
    deg = np.diff(ip).astype(np.float64)
    assert np.array_equal(Y[:, 0], deg) and (E >= np.abs(Y)).all()


@pytest.mark.parametrize("ci", range(4))
@pytest.mark.parametrize("Vp,Mp,tau", [(128, 4, 3), (128, 4, 40), (64, 8, 5), (128, 16, 2), (128, 4, 10 ** 9)])
def test_hybrid_tau_drops_thin_blocks_whole(ci, Vp, Mp, tau):
    """Reading #27: the tau-pack is the tau=0 pack with exactly the blocks that keep fewer than
    tau values removed (brute-force filter of the plain pack), and stays lossless."""
    indptr, indices = _pack_cases()[ci]
    n = len(indptr) - 1
    perm = np.random.default_rng(10 + ci).permutation(n).astype(np.int32)
    val16, _ = graphs.round16(graphs.symmetric_values(indptr, indices, seed=ci), "f16")
    full = oracle.pack(indptr, indices, val16, 0x3C00, perm, Vp, Mp)
    pk = oracle.pack(indptr, indices, val16, 0x3C00, perm, Vp, Mp, tau=tau)
    kept = [int(np.count_nonzero(full["vals"][m * Vp * 2:(m + 1) * Vp * 2])) for m in range(full["n_mb"])]
    keep = [m for m in range(full["n_mb"]) if kept[m] >= tau]
    assert pk["n_mb"] == len(keep)
    assert list(pk["mb_seg"]) == [full["mb_seg"][m] for m in keep]
    for i, m in enumerate(keep):
        assert np.array_equal(pk["sel"][i * 4:i * 4 + 4], full["sel"][m * 4:m * 4 + 4])
        assert np.array_equal(pk["nib"][i * Vp:(i + 1) * Vp], full["nib"][m * Vp:(m + 1) * Vp])
        assert np.array_equal(pk["vals"][i * Vp * 2:(i + 1) * Vp * 2], full["vals"][m * Vp * 2:(m + 1) * Vp * 2])
    # panel pointers count the surviving blocks of each panel
    P = (n + Vp - 1) // Vp
    for r in range(P):
        exp = sum(1 for m in keep if full["panel_ptr"][r] <= m < full["panel_ptr"][r + 1])
        assert pk["panel_ptr"][r + 1] - pk["panel_ptr"][r] == exp
    assert pk["res_nnz"] == full["res_nnz"] + sum(kept[m] for m in range(full["n_mb"]) if kept[m] < tau)
    Bd, present = oracle.unpack(pk, n)
    ref, refp = dense_bits(indptr, indices, val16, perm)
    assert np.array_equal(present, refp) and np.array_equal(Bd, ref)
    if tau >= 10 ** 9:
        assert pk["n_mb"] == 0 and pk["res_nnz"] == indptr[-1]
