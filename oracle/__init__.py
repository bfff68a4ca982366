"""CPU oracle for the V:N:M SpMM hot path -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously correct CPU reference of what the hot path of Chen et al.,
"Accelerating GNNs on GPU Sparse Tensor Cores through N:M Sparsity-Oriented Graph
Reordering" (PPoPP'25) computes.  The arithmetic lives in ``oracle/oracle.c`` (plain C,
fp64 for floating point); this module marshals numpy arrays through ctypes, except for the
dense parts of the GCN layer reference (``gcn_layer`` / ``gcn_layer_backward``: fp64 numpy
matmul and elementwise steps around the C SpMM, plus ``csr_transpose``) and the canonical
``unpack`` used by the pack invariants.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with the CUDA path
(``paper_conf_ppopp_chensz0s25_b200``) and neither imports the other.

Pins (see tests/test_oracle_*.py): worked values of PAPER.md:L286-319 (§4.2), brute-force
minimal cumulative-Hamming orders, brute-force violation counts, the Figure-1 fixture F1,
four hand-derived Stage-2 passes (tests/golden/s2_fixture_*.txt), brute-force optimum
bounds on tiny graphs, pack/unpack invariants, dense A@X.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
_lib_handle = None

P64 = ctypes.POINTER(ctypes.c_int64)
P32 = ctypes.POINTER(ctypes.c_int32)
PU8 = ctypes.POINTER(ctypes.c_uint8)
PU16 = ctypes.POINTER(ctypes.c_uint16)
PF64 = ctypes.POINTER(ctypes.c_double)


class _Opts(ctypes.Structure):
    _fields_ = [("max_outer", ctypes.c_int), ("max_stage1", ctypes.c_int),
                ("max_stage2", ctypes.c_int), ("gain_rule", ctypes.c_int),
                ("keep_best", ctypes.c_int)]


class _Stats(ctypes.Structure):
    _fields_ = [("omega_init", ctypes.c_int64), ("omega_final", ctypes.c_int64),
                ("mb_init", ctypes.c_int64), ("mb_final", ctypes.c_int64),
                ("outer_iters", ctypes.c_int64), ("stage1_iters", ctypes.c_int64),
                ("stage2_passes", ctypes.c_int64), ("max_pairs_per_primary", ctypes.c_int64)]


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (building the checker is not using it)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-fopenmp", "-o", tmp, _SRC])
        os.replace(tmp, _SO)
    return _SO


def _lib():
    global _lib_handle
    if _lib_handle is None:
        build()
        L = ctypes.CDLL(_SO)
        L.or_hamming_code.restype = ctypes.c_int64
        L.or_hamming_code.argtypes = [ctypes.c_uint64]
        L.or_position_code.restype = ctypes.c_int64
        L.or_position_code.argtypes = [ctypes.c_uint64, ctypes.c_int]
        L.or_validate.restype = ctypes.c_int
        L.or_validate.argtypes = [ctypes.c_int64, P64, P32]
        L.or_counts.restype = ctypes.c_int
        L.or_counts.argtypes = [ctypes.c_int64, P64, P32, P32, ctypes.c_int, ctypes.c_int,
                                ctypes.c_int, P64, P64, P32]
        L.or_reorder.restype = ctypes.c_int
        L.or_reorder.argtypes = [ctypes.c_int64, P64, P32, ctypes.c_int, ctypes.c_int,
                                 ctypes.c_int, ctypes.POINTER(_Opts), P32,
                                 ctypes.POINTER(_Stats)]
        L.or_pack_count.restype = ctypes.c_int
        L.or_pack_count.argtypes = [ctypes.c_int64, P64, P32, P32, ctypes.c_int, ctypes.c_int,
                                    ctypes.c_int, P64, P64]
        L.or_pack_fill.restype = ctypes.c_int
        L.or_pack_fill.argtypes = [ctypes.c_int64, P64, P32, PU16, ctypes.c_uint16, P32,
                                   ctypes.c_int, ctypes.c_int, ctypes.c_int, P64, P64, P64, P32, PU8, PU8,
                                   PU16, P64, P32, PU16]
        L.or_spmm_f64.restype = ctypes.c_int
        L.or_spmm_f64.argtypes = [ctypes.c_int64, P64, P32, PF64, PF64, ctypes.c_int64,
                                  ctypes.c_int, PF64, PF64, ctypes.c_int]
        L.or_spmm_rows_f64.restype = ctypes.c_int
        L.or_spmm_rows_f64.argtypes = [ctypes.c_int64, P64, P64, P32, PF64, PF64,
                                       ctypes.c_int64, ctypes.c_int, PF64, PF64]
        L.or_stage2_trace.restype = ctypes.c_int64
        L.or_stage2_trace.argtypes = [ctypes.c_int64, P64, P32, P32, ctypes.c_int, ctypes.c_int,
                                      ctypes.c_int, P64]
        L.or_stage1_once.restype = ctypes.c_int
        L.or_stage1_once.argtypes = [ctypes.c_int64, P64, P32, P32, ctypes.c_int, ctypes.c_int,
                                     P32]
        _lib_handle = L
    return _lib_handle


def _p(a, ptype):
    return None if a is None else a.ctypes.data_as(ptype)


def _csr(indptr, indices):
    rp = np.ascontiguousarray(indptr, dtype=np.int64)
    ci = np.ascontiguousarray(indices, dtype=np.int32)
    return rp, ci, len(rp) - 1


def hamming_code(b: int) -> int:
    """Rank of bit string b in the Hamming-distance order."""
    return int(_lib().or_hamming_code(int(b)))


def position_code(b: int, N: int) -> int:
    """Hamming position code, negated for an N:M-violating string (L313-319)."""
    return int(_lib().or_position_code(int(b), int(N)))


def validate(indptr, indices) -> int:
    """0 = ok, 1 = malformed CSR (unsorted/dup/out of range), 2 = pattern not symmetric."""
    rp, ci, n = _csr(indptr, indices)
    return int(_lib().or_validate(n, _p(rp, P64), _p(ci, P32)))


def counts(indptr, indices, perm, V: int, N: int, M: int):
    """(omega, MBscore, PScore[ceil(n/M)]) of B = P A P^T (L203, L382, L396)."""
    rp, ci, n = _csr(indptr, indices)
    pm = None if perm is None else np.ascontiguousarray(perm, dtype=np.int32)
    S = (n + M - 1) // M
    ps = np.zeros(max(S, 1), dtype=np.int32)
    w = ctypes.c_int64()
    mb = ctypes.c_int64()
    _lib().or_counts(n, _p(rp, P64), _p(ci, P32), _p(pm, P32), V, N, M, ctypes.byref(w),
                     ctypes.byref(mb), _p(ps, P32))
    return int(w.value), int(mb.value), ps[:S]


def reorder(indptr, indices, V: int, N: int, M: int, max_outer: int = 10, max_stage1: int = 10,
            max_stage2: int = 10, gain_rule: int = 0, keep_best: int = 1):
    """Alg. 1 with Stage-1 (Alg. 2) and Stage-2 (Alg. 3).
    Returns (perm, stats) with perm[new position] = old vertex."""
    rp, ci, n = _csr(indptr, indices)
    perm = np.zeros(max(n, 1), dtype=np.int32)
    o = _Opts(max_outer, max_stage1, max_stage2, gain_rule, keep_best)
    st = _Stats()
    _lib().or_reorder(n, _p(rp, P64), _p(ci, P32), V, N, M, ctypes.byref(o), _p(perm, P32),
                      ctypes.byref(st))
    stats = {f: int(getattr(st, f)) for f, _ in _Stats._fields_}
    return perm[:n], stats


def select_pattern(indptr, indices, max_M=32, max_V=32, **kw):
    """Best-V:N:M search, step by step as PAPER.md:L496 (§5) describes it: try 1:2:M with M
    initialised to 4 and doubled while the graph can be reordered to conform; then fix M and
    try V:2:M with V doubling from 1 up to max_V in the same way.  Returns (V, M, perm, stats)
    of the last conforming pattern (1:2:4 when even that does not conform)."""
    def conforms(st):
        return st["omega_final"] == 0 and st["mb_final"] == 0

    perm, st = reorder(indptr, indices, 1, 2, 4, **kw)
    best = (1, 4, perm, st)
    if not conforms(st):
        return best
    M = 8
    while M <= max_M:
        p, s = reorder(indptr, indices, 1, 2, M, **kw)
        if not conforms(s):
            break
        best = (1, M, p, s)
        M *= 2
    bestM = best[1]
    V = 2
    while V <= max_V:
        p, s = reorder(indptr, indices, V, 2, bestM, **kw)
        if not conforms(s):
            break
        best = (V, bestM, p, s)
        V *= 2
    return best


def stage1_once(indptr, indices, perm, N: int, M: int):
    """One Stage-1 sort (Alg. 2 lines 4-13) starting from perm; returns the new perm."""
    rp, ci, n = _csr(indptr, indices)
    pm = np.ascontiguousarray(perm, dtype=np.int32)
    out = np.zeros(max(n, 1), np.int32)
    _lib().or_stage1_once(n, _p(rp, P64), _p(ci, P32), _p(pm, P32), N, M, _p(out, P32))
    return out[:n]


def stage2_trace(indptr, indices, perm, N: int, M: int, gain_rule: int = 0):
    """ONE Stage-2 pass (Alg. 3 lines 1-23) from perm: the recorded pairs in recording order
    as a list of (primary segment, target segment, u, v) -- u, v positions of the pass-start
    order -- or None when the pass stops before recording anything."""
    rp, ci, n = _csr(indptr, indices)
    pm = np.ascontiguousarray(perm, dtype=np.int32)
    out = np.zeros(4 * max(n, 1), np.int64)
    k = int(_lib().or_stage2_trace(n, _p(rp, P64), _p(ci, P32), _p(pm, P32), N, M, gain_rule,
                                   _p(out, P64)))
    if k < 0:
        return None
    return [tuple(int(x) for x in out[4 * i:4 * i + 4]) for i in range(k)]


def pack(indptr, indices, val16, one_bits: int, perm, Vp: int, Mp: int, tau: int = 0):
    """Canonical V:N:M packing of B = P A P^T (reading #19).  val16: uint16 bits
    of A's values per CSR entry (None -> one_bits).  tau: meta-blocks keeping fewer than tau
    values go to the residual whole (hybrid split, reading #27; 0 = off)."""
    rp, ci, n = _csr(indptr, indices)
    pm = np.ascontiguousarray(perm, dtype=np.int32)
    v16 = None if val16 is None else np.ascontiguousarray(val16, dtype=np.uint16)
    nmb = ctypes.c_int64()
    rnz = ctypes.c_int64()
    L = _lib()
    L.or_pack_count(n, _p(rp, P64), _p(ci, P32), _p(pm, P32), Vp, Mp, tau, ctypes.byref(nmb),
                    ctypes.byref(rnz))
    P = (n + Vp - 1) // Vp
    m, r = nmb.value, rnz.value
    out = dict(
        panel_ptr=np.zeros(P + 1, np.int64), mb_seg=np.zeros(max(m, 1), np.int32),
        sel=np.zeros(max(m, 1) * 4, np.uint8), nib=np.zeros(max(m, 1) * Vp, np.uint8),
        vals=np.zeros(max(m, 1) * Vp * 2, np.uint16), res_rowptr=np.zeros(n + 1, np.int64),
        res_col=np.zeros(max(r, 1), np.int32), res_val=np.zeros(max(r, 1), np.uint16))
    L.or_pack_fill(n, _p(rp, P64), _p(ci, P32), _p(v16, PU16), one_bits, _p(pm, P32), Vp, Mp,
                   tau, ctypes.byref(nmb), ctypes.byref(rnz), _p(out["panel_ptr"], P64),
                   _p(out["mb_seg"], P32), _p(out["sel"], PU8), _p(out["nib"], PU8),
                   _p(out["vals"], PU16), _p(out["res_rowptr"], P64), _p(out["res_col"], P32),
                   _p(out["res_val"], PU16))
    out["mb_seg"] = out["mb_seg"][:m]
    out["sel"] = out["sel"][:m * 4]
    out["nib"] = out["nib"][:m * Vp]
    out["vals"] = out["vals"][:m * Vp * 2]
    out["res_col"] = out["res_col"][:r]
    out["res_val"] = out["res_val"][:r]
    out["n_mb"] = m
    out["res_nnz"] = r
    out["Vp"] = Vp
    out["Mp"] = Mp
    return out


def spmm(indptr, indices, val, X, nthreads: int = 1):
    """fp64 CSR SpMM Y = A X and E = |A| |X| (the exact result, L128/L560).
    Returns (Y, E, threads_used)."""
    rp, ci, n = _csr(indptr, indices)
    v = None if val is None else np.ascontiguousarray(val, dtype=np.float64)
    Xd = np.ascontiguousarray(X, dtype=np.float64)
    F = Xd.shape[1]
    Y = np.empty((n, F), np.float64)
    E = np.empty((n, F), np.float64)
    used = _lib().or_spmm_f64(n, _p(rp, P64), _p(ci, P32), _p(v, PF64), _p(Xd, PF64), F, F,
                              _p(Y, PF64), _p(E, PF64), nthreads)
    return Y, E, int(used)


def spmm_rows(rows, indptr, indices, val, X):
    """Y and E for the sampled rows only (full-size parity)."""
    rp, ci, n = _csr(indptr, indices)
    rr = np.ascontiguousarray(rows, dtype=np.int64)
    v = None if val is None else np.ascontiguousarray(val, dtype=np.float64)
    Xd = np.ascontiguousarray(X, dtype=np.float64)
    F = Xd.shape[1]
    Y = np.empty((len(rr), F), np.float64)
    E = np.empty((len(rr), F), np.float64)
    _lib().or_spmm_rows_f64(len(rr), _p(rr, P64), _p(rp, P64), _p(ci, P32), _p(v, PF64),
                            _p(Xd, PF64), F, F, _p(Y, PF64), _p(E, PF64))
    return Y, E


def unpack(pk: dict, n: int):
    """Rebuild B (dense fp16/bf16 bits, n x n, uint16) from the canonical pack + residual.
    Plain loops -- for the small pack invariants only."""
    Vp, Mp = pk["Vp"], pk["Mp"]
    Bd = np.zeros((n, n), np.uint16)
    present = np.zeros((n, n), bool)
    P = len(pk["panel_ptr"]) - 1
    for r in range(P):
        for mb in range(int(pk["panel_ptr"][r]), int(pk["panel_ptr"][r + 1])):
            s = int(pk["mb_seg"][mb])
            sel = pk["sel"][mb * 4:mb * 4 + 4]
            for li in range(Vp):
                i = r * Vp + li
                nb = int(pk["nib"][mb * Vp + li])
                i0, i1 = nb & 3, (nb >> 2) & 3
                for slot, j in ((0, i0), (1, i1)):
                    v = int(pk["vals"][(mb * Vp + li) * 2 + slot])
                    col = s * Mp + int(sel[j])
                    if v != 0:
                        assert i < n and col < n
                        assert not present[i, col]
                        Bd[i, col] = v
                        present[i, col] = True
    rp, rc, rv = pk["res_rowptr"], pk["res_col"], pk["res_val"]
    for i in range(n):
        for k in range(int(rp[i]), int(rp[i + 1])):
            assert not present[i, rc[k]]
            Bd[i, rc[k]] = rv[k]
            present[i, rc[k]] = True
    return Bd, present


def csr_transpose(indptr, indices, val):
    """A^T of a CSR matrix (plain counting sort; no symmetry assumed)."""
    indptr = np.asarray(indptr, dtype=np.int64)
    indices = np.asarray(indices, dtype=np.int64)
    val = np.asarray(val, dtype=np.float64)
    n = indptr.shape[0] - 1
    rows = np.repeat(np.arange(n), np.diff(indptr))
    order = np.lexsort((rows, indices))  # by column, then row
    tp = np.concatenate([[0], np.cumsum(np.bincount(indices, minlength=n))]).astype(np.int64)
    return tp, rows[order].astype(np.int32), val[order]


def gcn_layer(indptr, indices, val, H, W, b, relu: bool):
    """Eq. 1 in fp64: Hout = act(A (H W) + b); returns (Hout, Z)."""
    XW = np.asarray(H, dtype=np.float64) @ np.asarray(W, dtype=np.float64)
    Z, _, _ = spmm(indptr, indices, val, XW)
    Z = Z + np.asarray(b, dtype=np.float64)
    return (np.maximum(Z, 0.0) if relu else Z), Z


def gcn_layer_backward(indptr, indices, val, H, W, Z, dHout, relu: bool):
    """Gradients of gcn_layer for the upstream gradient dHout, step by step in fp64 (SURVEY
    §8(f) item 4): dZ = dHout * act'(Z); db = sum over rows of dZ; dT = A^T dZ (the transpose
    is formed explicitly -- the oracle does not assume A symmetric); dW = H^T dT; dH = dT W^T.
    Pinned by central finite differences (tests/test_oracle_gcn_backward.py)."""
    dZ = np.asarray(dHout, dtype=np.float64) * ((np.asarray(Z) > 0) if relu else 1.0)
    db = dZ.sum(axis=0)
    tp, ti, tv = csr_transpose(indptr, indices, val)
    dT, _, _ = spmm(tp, ti, tv, dZ)
    dW = np.asarray(H, dtype=np.float64).T @ dT
    dH = dT @ np.asarray(W, dtype=np.float64).T
    return dH, dW, db, dT


def sgc_propagate(indptr, indices, val, X, K: int):
    """SGC propagation (Table 3 "SGC" L546-553): Ahat^K X in fp64 (K SpMMs)."""
    Y = np.asarray(X, dtype=np.float64)
    for _ in range(K):
        Y, _, _ = spmm(indptr, indices, val, Y)
    return Y


def sage_layer(indptr, indices, val_mean, H, W_self, W_neigh, b, relu: bool):
    """GraphSAGE layer with the mean aggregator (Table 3 "SAGE"), fp64:
    act(H W_self + (Amean H) W_neigh + b) with Amean = D^-1 A given as CSR values."""
    Hd = np.asarray(H, dtype=np.float64)
    agg, _, _ = spmm(indptr, indices, val_mean, Hd)
    Z = Hd @ np.asarray(W_self, np.float64) + agg @ np.asarray(W_neigh, np.float64) + np.asarray(b, np.float64)
    return (np.maximum(Z, 0.0) if relu else Z), agg


def cheb_layer(indptr, indices, val_L, H, Ws, b, relu: bool):
    """Chebyshev convolution (Table 3 "Cheb"), fp64: act(sum_k T_k Ws[k] + b) with
    T_0 = H, T_1 = L H, T_k = 2 L T_{k-1} - T_{k-2} (Defferrard et al.'s recurrence)."""
    T = [np.asarray(H, dtype=np.float64)]
    for k in range(1, len(Ws)):
        LT, _, _ = spmm(indptr, indices, val_L, T[k - 1])
        T.append(LT if k == 1 else 2.0 * LT - T[k - 2])
    Z = sum(T[k] @ np.asarray(Ws[k], np.float64) for k in range(len(Ws))) + np.asarray(b, np.float64)
    return (np.maximum(Z, 0.0) if relu else Z), T
