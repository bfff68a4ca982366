"""Thin Pythonic layer over the C ABI (argument marshalling only; every step runs in libnm).

numpy arrays are passed for host-side graph data, torch CUDA tensors for device buffers
(torch is used for device memory and streams only).
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _lib as L

_DT = {"f16": L.NM_F16, "bf16": L.NM_BF16, "f32": L.NM_F32}


def _ptr(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return ctypes.c_void_p(a.ctypes.data)
    return ctypes.c_void_p(a.data_ptr())  # torch tensor


def _csr_struct(indptr, indices, val=None, val_dtype="f16"):
    rp = np.ascontiguousarray(indptr, dtype=np.int64)
    ci = np.ascontiguousarray(indices, dtype=np.int32)
    keep = [rp, ci]
    c = L.nm_csr()
    c.n = len(rp) - 1
    c.nnz = int(rp[-1])
    c.rowptr = rp.ctypes.data
    c.col = ci.ctypes.data
    if val is not None:
        v = np.ascontiguousarray(val)
        keep.append(v)
        c.val = v.ctypes.data
    else:
        c.val = None
    c.val_dtype = _DT[val_dtype]
    c.on_device = 0
    return c, keep


def _stream_ptr(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def reorder(indptr, indices, V: int, N: int, M: int, max_outer=10, max_stage1=10, max_stage2=10,
            gain_rule=0, keep_best=1, device=False, stream=None):
    """nm_reorder (host) or, with device=True, nm_reorder_gpu (Stage-1 sort and the counts on
    the current CUDA device): returns (perm int32[n], stats dict)."""
    c, keep = _csr_struct(indptr, indices)
    perm = np.zeros(c.n, np.int32)
    o = L.nm_reorder_opts(max_outer, max_stage1, max_stage2, gain_rule, keep_best)
    st = L.nm_reorder_stats()
    if device:
        L.check(L.load().nm_reorder_gpu(ctypes.byref(c), V, N, M, ctypes.byref(o),
                                        perm.ctypes.data_as(L.P32), ctypes.byref(st),
                                        _stream_ptr(stream)), "nm_reorder_gpu")
    else:
        L.check(L.load().nm_reorder(ctypes.byref(c), V, N, M, ctypes.byref(o),
                                    perm.ctypes.data_as(L.P32), ctypes.byref(st)), "nm_reorder")
    return perm, {f: getattr(st, f) for f, _ in L.nm_reorder_stats._fields_}


def select_pattern(indptr, indices, max_M=32, max_V=32, max_outer=10, max_stage1=10, max_stage2=10,
                   gain_rule=0, keep_best=1):
    """nm_select_pattern: returns (V, M, perm, stats) of the best conforming
    V:2:M pattern found by the paper's doubling search."""
    c, keep = _csr_struct(indptr, indices)
    perm = np.zeros(c.n, np.int32)
    o = L.nm_reorder_opts(max_outer, max_stage1, max_stage2, gain_rule, keep_best)
    st = L.nm_reorder_stats()
    V = ctypes.c_int()
    M = ctypes.c_int()
    L.check(L.load().nm_select_pattern(ctypes.byref(c), max_M, max_V, ctypes.byref(o),
                                       perm.ctypes.data_as(L.P32), ctypes.byref(V), ctypes.byref(M),
                                       ctypes.byref(st)), "nm_select_pattern")
    return V.value, M.value, perm, {f: getattr(st, f) for f, _ in L.nm_reorder_stats._fields_}


def score_patterns(indptr, indices, candidates, F, dtype="bf16", val=None, val_dtype=None, stream=None,
                   max_outer=10, max_stage1=10, max_stage2=10, gain_rule=0, keep_best=1):
    """nm_score_patterns: candidates = [(V, M), ...] (N = 2).  Returns (best index, perm of the
    best, [{"V", "M", "score_ns", "n_chunks", "residual_nnz"}, ...])."""
    if val is not None and val_dtype is None:
        val_dtype = "f32" if val.dtype == np.float32 else ("f16" if val.dtype == np.float16 else "bf16")
    c, keep = _csr_struct(indptr, indices, val, val_dtype or "f16")
    k = len(candidates)
    Vs = (ctypes.c_int * k)(*[int(v) for v, _ in candidates])
    Ms = (ctypes.c_int * k)(*[int(m) for _, m in candidates])
    sc = (ctypes.c_double * k)()
    ch = np.zeros(k, np.int64)
    rs = np.zeros(k, np.int64)
    best = ctypes.c_int()
    perm = np.zeros(c.n, np.int32)
    o = L.nm_reorder_opts(max_outer, max_stage1, max_stage2, gain_rule, keep_best)
    L.check(L.load().nm_score_patterns(ctypes.byref(c), k, Vs, Ms, int(F), _DT[dtype], ctypes.byref(o),
                                       _stream_ptr(stream), sc, ch.ctypes.data_as(L.P64), rs.ctypes.data_as(L.P64),
                                       ctypes.byref(best), perm.ctypes.data_as(L.P32)), "nm_score_patterns")
    rows = [{"V": int(v), "M": int(m), "score_ns": float(sc[i]), "n_chunks": int(ch[i]), "residual_nnz": int(rs[i])}
            for i, (v, m) in enumerate(candidates)]
    return best.value, perm, rows


def count_violations(indptr, indices, perm, V: int, N: int, M: int):
    """nm_count_violations (GPU): returns (omega, mbscore, pscore int32[ceil(n/M)])."""
    c, keep = _csr_struct(indptr, indices)
    S = (c.n + M - 1) // M
    ps = np.zeros(S, np.int32)
    w = ctypes.c_int64()
    mb = ctypes.c_int64()
    pm = None if perm is None else np.ascontiguousarray(perm, np.int32)
    L.check(L.load().nm_count_violations(ctypes.byref(c), None if pm is None else pm.ctypes.data_as(L.P32),
                                         V, N, M, ctypes.byref(w), ctypes.byref(mb),
                                         ps.ctypes.data_as(L.P32)), "nm_count_violations")
    return int(w.value), int(mb.value), ps


class Packed:
    """Owns an nm_packed handle (device memory on the current device)."""

    def __init__(self, handle, n, row_begin, row_end, dtype):
        self.handle = handle
        self.n = n
        self.row_begin = row_begin
        self.row_end = row_end
        self.dtype = dtype

    @property
    def rows(self):
        return self.row_end - self.row_begin

    def info(self):
        vals = [ctypes.c_int64() for _ in range(5)]
        L.check(L.load().nm_packed_info(self.handle, *[ctypes.byref(v) for v in vals]),
                "nm_packed_info")
        keys = ("n_mb", "packed_nnz", "residual_nnz", "device_bytes", "n_chunks")
        return {k: int(v.value) for k, v in zip(keys, vals)}

    def stats(self):
        """nm_packed_stats: every size of the packed matrix as a dict."""
        st = L.nm_packed_stat()
        L.check(L.load().nm_packed_stats(self.handle, ctypes.byref(st)), "nm_packed_stats")
        return {f: getattr(st, f) for f, _ in L.nm_packed_stat._fields_}

    def export_canonical(self, residual_only=False):
        """nm_export_canonical -> dict of host arrays (residual_only: just the residual CSR)."""
        inf = self.info()
        m, r = inf["n_mb"], inf["residual_nnz"]
        Vp = int(self.stats()["Vp"])
        P = (self.rows + Vp - 1) // Vp
        out = dict(res_rowptr=np.zeros(self.rows + 1, np.int64), res_col=np.zeros(max(r, 1), np.int32),
                   res_val=np.zeros(max(r, 1), np.uint16))
        if not residual_only:
            out.update(panel_ptr=np.zeros(P + 1, np.int64), mb_seg=np.zeros(max(m, 1), np.int32),
                       sel=np.zeros(max(m, 1) * 4, np.uint8), nib=np.zeros(max(m, 1) * Vp, np.uint8),
                       vals=np.zeros(max(m, 1) * Vp * 2, np.uint16))
        ptr = lambda k, t: out[k].ctypes.data_as(t) if k in out else None
        L.check(L.load().nm_export_canonical(
            self.handle, ptr("panel_ptr", L.P64), ptr("mb_seg", L.P32), ptr("sel", L.PU8), ptr("nib", L.PU8),
            ptr("vals", L.PU16), ptr("res_rowptr", L.P64), ptr("res_col", L.P32), ptr("res_val", L.PU16)),
            "nm_export_canonical")
        if not residual_only:
            out["mb_seg"] = out["mb_seg"][:m]
            out["sel"] = out["sel"][:m * 4]
            out["nib"] = out["nib"][:m * Vp]
            out["vals"] = out["vals"][:m * Vp * 2]
        out["res_col"] = out["res_col"][:r]
        out["res_val"] = out["res_val"][:r]
        out["n_mb"], out["res_nnz"], out["Vp"] = m, r, Vp
        return out

    def free(self):
        if self.handle:
            L.load().nm_packed_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def pack(indptr, indices, perm, V: int, N: int, M: int, dtype="f16", val=None, val_dtype=None,
         row_begin=None, row_end=None, stream=None, order="permuted", tau=0, Vp=0, F=None):
    """nm_pack / nm_pack_rows / nm_pack_ex / nm_pack_hybrid of B = P A P^T.  val: values per CSR
    entry (numpy, dtype val_dtype in {'f16','bf16' (uint16 bits),'f32'}) or None for a binary
    adjacency.  order='original' folds the permutation into the SpMM (NM_PACK_ORIGINAL_ORDER).
    tau > 0: hybrid split (meta-blocks keeping fewer than tau values go to the residual).
    Vp: panel height, 16, 32, 64 or 128 (0 = the library's choice: V for V in 16/32/64, else 128).
    tau="auto": nm_pack_auto for F feature columns (the tau minimising the library's time model)."""
    if val is not None and val_dtype is None:
        val_dtype = "f32" if val.dtype == np.float32 else ("f16" if val.dtype == np.float16 else "bf16")
    c, keep = _csr_struct(indptr, indices, val, val_dtype or "f16")
    pm = None if perm is None else np.ascontiguousarray(perm, np.int32)
    h = ctypes.c_void_p()
    pp = None if pm is None else pm.ctypes.data_as(L.P32)
    sp = _stream_ptr(stream)
    rb = 0 if row_begin is None else int(row_begin)
    re = c.n if row_end is None else int(row_end)
    flags = L.NM_PACK_ORIGINAL_ORDER if order == "original" else 0
    lib = L.load()
    if tau == "auto":
        if F is None:
            raise ValueError("tau='auto' needs F")
        t = ctypes.c_int()
        L.check(lib.nm_pack_auto(ctypes.byref(c), pp, V, N, M, int(Vp), _DT[dtype], rb, re, flags, int(F), sp,
                                 ctypes.byref(h), ctypes.byref(t)), "nm_pack_auto")
        P = Packed(h, c.n, rb, re, dtype)
        P.order = order
        P.tau = int(t.value)
        return P
    if tau:
        L.check(lib.nm_pack_hybrid(ctypes.byref(c), pp, V, N, M, int(Vp), _DT[dtype], rb, re, flags, int(tau), sp,
                                   ctypes.byref(h)), "nm_pack_hybrid")
    elif order == "original":
        L.check(lib.nm_pack_ex(ctypes.byref(c), pp, V, N, M, int(Vp), _DT[dtype], rb, re, flags, sp,
                               ctypes.byref(h)), "nm_pack_ex")
    elif row_begin is None:
        L.check(lib.nm_pack(ctypes.byref(c), pp, V, N, M, int(Vp), _DT[dtype], sp, ctypes.byref(h)), "nm_pack")
    else:
        L.check(lib.nm_pack_rows(ctypes.byref(c), pp, V, N, M, int(Vp), _DT[dtype], rb, re, sp, ctypes.byref(h)),
                "nm_pack_rows")
    P = Packed(h, c.n, rb, re, dtype)
    P.order = order
    P.tau = int(tau)
    return P


def hybrid_tau(F: int) -> int:
    """nm_hybrid_tau: the library's break-even hybrid-split threshold for F feature columns."""
    return int(L.load().nm_hybrid_tau(int(F)))


def spmm(P: Packed, PX, Yp, F=None, stream=None, part="all", format=None):
    """Yp (fp32 CUDA tensor, rows x F) = packed B * PX (16-bit CUDA tensor, n x F).
    part: 'all' | 'sptc' | 'residual'; format (part='sptc' only): None / 0 = the pack's choice,
    1 = full-record kernel, 2 = compressed-record kernel (nm_spmm_sptc_format)."""
    F = PX.shape[1] if F is None else F
    if format is not None:
        assert part == "sptc"
        L.check(L.load().nm_spmm_sptc_format(P.handle, _ptr(PX), PX.stride(0), _ptr(Yp), Yp.stride(0), F,
                                             int(format), _stream_ptr(stream)), "nm_spmm_sptc_format")
        return
    fn = {"all": "nm_spmm", "sptc": "nm_spmm_sptc", "residual": "nm_spmm_residual"}[part]
    L.check(getattr(L.load(), fn)(P.handle, _ptr(PX), PX.stride(0), _ptr(Yp), Yp.stride(0), F,
                                  _stream_ptr(stream)), fn)


def permute_rows(X, PX, perm_dev, dtype, stream=None):
    L.check(L.load().nm_permute_rows(_ptr(X), _ptr(PX), _ptr(perm_dev), X.shape[0], X.shape[1],
                                     X.stride(0), _DT[dtype], _stream_ptr(stream)), "nm_permute_rows")


def unpermute_rows(Yp, Y, perm_dev, dtype, stream=None):
    L.check(L.load().nm_unpermute_rows(_ptr(Yp), _ptr(Y), _ptr(perm_dev), Yp.shape[0], Yp.shape[1],
                                       Yp.stride(0), _DT[dtype], _stream_ptr(stream)),
            "nm_unpermute_rows")


def gcn_workspace_bytes(n, F_in, F_out):
    return int(L.load().nm_gcn_workspace_bytes(n, F_in, F_out))


_ORDERS = {"linear": L.NM_LINEAR_FIRST, "aggregate": L.NM_AGG_FIRST, "auto": L.NM_ORDER_AUTO}


def gcn_layer(P: Packed, H, W, bias, Hout, ws, relu=True, order="linear", stream=None):
    """nm_gcn_layer: Hout (rows of P) = act(Ahat (H W) + bias); order 'linear' | 'aggregate' |
    'auto'."""
    flags = (L.NM_RELU if relu else 0) | _ORDERS[order]
    L.check(L.load().nm_gcn_layer(P.handle, _ptr(H), _ptr(W), _ptr(bias), _ptr(Hout), H.shape[1],
                                  W.shape[1], flags, _ptr(ws), ws.numel(), _stream_ptr(stream)),
            "nm_gcn_layer")


def gcn_layer_bcast(P: Packed, H, W, bias, dst_ptrs, dst_row0, F_out, ws, relu=True, order="linear",
                    stream=None):
    """nm_gcn_layer_bcast: this shard's output rows stored at rows [dst_row0, +rows) of every
    buffer in dst_ptrs (device addresses, e.g. every rank's symmetric-memory buffer)."""
    flags = (L.NM_RELU if relu else 0) | _ORDERS[order]
    arr = (ctypes.c_void_p * len(dst_ptrs))(*[int(p) for p in dst_ptrs])
    L.check(L.load().nm_gcn_layer_bcast(P.handle, _ptr(H), _ptr(W), _ptr(bias), arr, len(dst_ptrs), int(dst_row0),
                                        H.shape[1], int(F_out), flags, _ptr(ws), ws.numel(), _stream_ptr(stream)),
            "nm_gcn_layer_bcast")


def gcn_backward_workspace_bytes(n, F_in, F_out):
    return int(L.load().nm_gcn_backward_workspace_bytes(n, F_in, F_out))


def gcn_layer_backward(P: Packed, H, W, Hout, dHout, dH, dW, db, ws, relu=True, stream=None):
    """nm_gcn_layer_backward: dW (fp32), db (fp32, optional) and dH (16-bit, optional) of
    Hout = act(Ahat (H W) + b) for the upstream gradient dHout (Ahat^T = Ahat)."""
    L.check(L.load().nm_gcn_layer_backward(P.handle, _ptr(H), _ptr(W), _ptr(Hout), _ptr(dHout), _ptr(dH),
                                           _ptr(dW), _ptr(db), H.shape[1], W.shape[1],
                                           L.NM_RELU if relu else 0, _ptr(ws), ws.numel(),
                                           _stream_ptr(stream)),
            "nm_gcn_layer_backward")


def sgc_propagate(P: Packed, X, Y, K: int, Y16=None, ws=None, stream=None):
    """nm_sgc_propagate: Y (fp32, n x F) = Ahat^K X (SGC propagation)."""
    import torch
    F = X.shape[1]
    if ws is None:
        ws = torch.empty(int(L.load().nm_sgc_workspace_bytes(P.n, F)), dtype=torch.uint8, device=X.device)
    L.check(L.load().nm_sgc_propagate(P.handle, _ptr(X), X.stride(0), _ptr(Y), Y.stride(0), _ptr(Y16), F, int(K),
                                      _ptr(ws), ws.numel(), _stream_ptr(stream)), "nm_sgc_propagate")


def sage_layer(P: Packed, H, W_self, W_neigh, bias, Hout, relu=True, ws=None, stream=None):
    """nm_sage_layer: Hout = act([H | Amean H] [W_self; W_neigh] + bias) (GraphSAGE mean)."""
    import torch
    F_in, F_out = W_self.shape
    if ws is None:
        ws = torch.empty(int(L.load().nm_sage_workspace_bytes(P.n, F_in, F_out)), dtype=torch.uint8, device=H.device)
    L.check(L.load().nm_sage_layer(P.handle, _ptr(H), _ptr(W_self), _ptr(W_neigh), _ptr(bias), _ptr(Hout), F_in, F_out,
                                   L.NM_RELU if relu else 0, _ptr(ws), ws.numel(), _stream_ptr(stream)),
            "nm_sage_layer")


def cheb_layer(P: Packed, H, W, bias, Hout, K: int, relu=True, ws=None, stream=None):
    """nm_cheb_layer: Hout = act(sum_k T_k(Lhat) H W_k + bias); W is (K F_in) x F_out."""
    import torch
    F_in = H.shape[1]
    F_out = W.shape[1]
    if ws is None:
        ws = torch.empty(int(L.load().nm_cheb_workspace_bytes(P.n, F_in, F_out, K)), dtype=torch.uint8,
                         device=H.device)
    L.check(L.load().nm_cheb_layer(P.handle, _ptr(H), _ptr(W), _ptr(bias), _ptr(Hout), F_in, F_out, int(K),
                                   L.NM_RELU if relu else 0, _ptr(ws), ws.numel(), _stream_ptr(stream)),
            "nm_cheb_layer")
