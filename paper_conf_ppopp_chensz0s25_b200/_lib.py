"""ctypes binding of libnm (include/nm.h) -- argument marshalling only.

Every entry point of the C ABI is exposed under its C name.  The library is loaded from
this package directory (built in-tree by ``build.py``); if it is missing the import fails
loudly -- there is no CPU fallback anywhere in the product path.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libnm.so")

NM_OK, NM_ERR_INVALID_ARG, NM_ERR_UNSUPPORTED, NM_ERR_BAD_CSR, NM_ERR_NOT_SYMMETRIC, \
    NM_ERR_CUDA, NM_ERR_OOM = range(7)
NM_F16, NM_BF16, NM_F32 = 0, 1, 2
NM_RELU = 1
NM_LINEAR_FIRST, NM_AGG_FIRST, NM_ORDER_AUTO = 0, 2, 4
NM_PACK_ORIGINAL_ORDER = 1

P64 = ctypes.POINTER(ctypes.c_int64)
P32 = ctypes.POINTER(ctypes.c_int32)
PU8 = ctypes.POINTER(ctypes.c_uint8)
PU16 = ctypes.POINTER(ctypes.c_uint16)
VP = ctypes.c_void_p


class nm_csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("rowptr", VP), ("col", VP),
                ("val", VP), ("val_dtype", ctypes.c_int), ("on_device", ctypes.c_int)]


class nm_reorder_opts(ctypes.Structure):
    _fields_ = [("max_outer", ctypes.c_int), ("max_stage1", ctypes.c_int),
                ("max_stage2", ctypes.c_int), ("gain_rule", ctypes.c_int),
                ("keep_best", ctypes.c_int)]


class nm_reorder_stats(ctypes.Structure):
    _fields_ = [("omega_init", ctypes.c_int64), ("omega_final", ctypes.c_int64),
                ("mb_init", ctypes.c_int64), ("mb_final", ctypes.c_int64),
                ("outer_iters", ctypes.c_int64), ("stage1_iters", ctypes.c_int64),
                ("stage2_passes", ctypes.c_int64), ("max_pairs_per_primary", ctypes.c_int64),
                ("seconds", ctypes.c_double)]


class nm_packed_stat(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int64) for k in ("n", "row_begin", "row_end", "n_panels", "n_mb", "n_chunks",
                                              "packed_nnz", "residual_nnz", "image_bytes", "device_bytes",
                                              "residual_items", "residual_split_rows")] + \
               [(k, ctypes.c_int32) for k in ("V", "M", "Mp", "Vp", "tau", "flags")] + \
               [(k, ctypes.c_int64) for k in ("full_image_bytes", "gather_rows")]


# name -> (restype, argtypes); mirrors include/nm.h exactly
SIGNATURES = {
    "nm_reorder": (ctypes.c_int, [ctypes.POINTER(nm_csr), ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                  ctypes.POINTER(nm_reorder_opts), P32,
                                  ctypes.POINTER(nm_reorder_stats)]),
    "nm_reorder_gpu": (ctypes.c_int, [ctypes.POINTER(nm_csr), ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                      ctypes.POINTER(nm_reorder_opts), P32,
                                      ctypes.POINTER(nm_reorder_stats), ctypes.c_void_p]),
    "nm_select_pattern": (ctypes.c_int, [ctypes.POINTER(nm_csr), ctypes.c_int, ctypes.c_int,
                                         ctypes.POINTER(nm_reorder_opts), P32,
                                         ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.c_int),
                                         ctypes.POINTER(nm_reorder_stats)]),
    "nm_pack_auto": (ctypes.c_int, [ctypes.POINTER(nm_csr), P32, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                    ctypes.c_int, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int, VP,
                                    ctypes.POINTER(VP), ctypes.POINTER(ctypes.c_int)]),
    "nm_score_patterns": (ctypes.c_int, [ctypes.POINTER(nm_csr), ctypes.c_int, ctypes.POINTER(ctypes.c_int),
                                         ctypes.POINTER(ctypes.c_int), ctypes.c_int, ctypes.c_int,
                                         ctypes.POINTER(nm_reorder_opts), ctypes.c_void_p,
                                         ctypes.POINTER(ctypes.c_double), P64, P64, ctypes.POINTER(ctypes.c_int),
                                         P32]),
    "nm_count_violations": (ctypes.c_int, [ctypes.POINTER(nm_csr), P32, ctypes.c_int, ctypes.c_int,
                                           ctypes.c_int, P64, P64, P32]),
    "nm_pack": (ctypes.c_int, [ctypes.POINTER(nm_csr), P32, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                               ctypes.c_int, ctypes.c_int, VP, ctypes.POINTER(VP)]),
    "nm_pack_rows": (ctypes.c_int, [ctypes.POINTER(nm_csr), P32, ctypes.c_int, ctypes.c_int,
                                    ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int64,
                                    ctypes.c_int64, VP, ctypes.POINTER(VP)]),
    "nm_pack_ex": (ctypes.c_int, [ctypes.POINTER(nm_csr), P32, ctypes.c_int, ctypes.c_int,
                                  ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int64,
                                  ctypes.c_int64, ctypes.c_int, VP, ctypes.POINTER(VP)]),
    "nm_pack_hybrid": (ctypes.c_int, [ctypes.POINTER(nm_csr), P32, ctypes.c_int, ctypes.c_int,
                                      ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int64,
                                      ctypes.c_int64, ctypes.c_int, ctypes.c_int, VP, ctypes.POINTER(VP)]),
    "nm_hybrid_tau": (ctypes.c_int, [ctypes.c_int]),
    "nm_packed_info": (ctypes.c_int, [VP, P64, P64, P64, P64, P64]),
    "nm_packed_stats": (ctypes.c_int, [VP, ctypes.POINTER(nm_packed_stat)]),
    "nm_export_canonical": (ctypes.c_int, [VP, P64, P32, PU8, PU8, PU16, P64, P32, PU16]),
    "nm_packed_free": (None, [VP]),
    "nm_permute_rows": (ctypes.c_int, [VP, VP, VP, ctypes.c_int64, ctypes.c_int, ctypes.c_int64,
                                       ctypes.c_int, VP]),
    "nm_unpermute_rows": (ctypes.c_int, [VP, VP, VP, ctypes.c_int64, ctypes.c_int, ctypes.c_int64,
                                         ctypes.c_int, VP]),
    "nm_spmm": (ctypes.c_int, [VP, VP, ctypes.c_int64, VP, ctypes.c_int64, ctypes.c_int, VP]),
    "nm_spmm_sptc": (ctypes.c_int, [VP, VP, ctypes.c_int64, VP, ctypes.c_int64, ctypes.c_int, VP]),
    "nm_spmm_sptc_format": (ctypes.c_int, [VP, VP, ctypes.c_int64, VP, ctypes.c_int64, ctypes.c_int, ctypes.c_int,
                                           VP]),
    "nm_spmm_residual": (ctypes.c_int, [VP, VP, ctypes.c_int64, VP, ctypes.c_int64, ctypes.c_int,
                                        VP]),
    "nm_gcn_workspace_bytes": (ctypes.c_size_t, [ctypes.c_int64, ctypes.c_int, ctypes.c_int]),
    "nm_gcn_layer": (ctypes.c_int, [VP, VP, VP, VP, VP, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                    VP, ctypes.c_size_t, VP]),
    "nm_gcn_layer_bcast": (ctypes.c_int, [VP, VP, VP, VP, ctypes.POINTER(VP), ctypes.c_int, ctypes.c_int64,
                                          ctypes.c_int, ctypes.c_int, ctypes.c_int, VP, ctypes.c_size_t, VP]),
    "nm_gcn_backward_workspace_bytes": (ctypes.c_size_t, [ctypes.c_int64, ctypes.c_int, ctypes.c_int]),
    "nm_sgc_workspace_bytes": (ctypes.c_size_t, [ctypes.c_int64, ctypes.c_int]),
    "nm_sgc_propagate": (ctypes.c_int, [VP, VP, ctypes.c_int64, VP, ctypes.c_int64, VP, ctypes.c_int, ctypes.c_int,
                                        VP, ctypes.c_size_t, VP]),
    "nm_sage_workspace_bytes": (ctypes.c_size_t, [ctypes.c_int64, ctypes.c_int, ctypes.c_int]),
    "nm_sage_layer": (ctypes.c_int, [VP, VP, VP, VP, VP, VP, ctypes.c_int, ctypes.c_int, ctypes.c_int, VP,
                                     ctypes.c_size_t, VP]),
    "nm_cheb_workspace_bytes": (ctypes.c_size_t, [ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_int]),
    "nm_cheb_layer": (ctypes.c_int, [VP, VP, VP, VP, VP, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, VP,
                                     ctypes.c_size_t, VP]),
    "nm_gcn_layer_backward": (ctypes.c_int, [VP, VP, VP, VP, VP, VP, VP, VP, ctypes.c_int, ctypes.c_int,
                                             ctypes.c_int, VP, ctypes.c_size_t, VP]),
    "nm_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "nm_last_error": (ctypes.c_char_p, []),
    "nm_version": (ctypes.c_int, []),
}


class NMError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        super().__init__("%s failed: %s (%s)" % (where, _status_name(status), detail))


_lib = None


def load():
    """Load libnm.so from the package directory; raise if it has not been built."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError("libnm.so not built: run `python -m paper_conf_ppopp_chensz0s25_b200"
                              ".build` (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _status_name(s: int) -> str:
    try:
        return load().nm_status_string(s).decode()
    except Exception:  # pragma: no cover
        return str(s)


def check(status: int, where: str):
    if status != NM_OK:
        raise NMError(status, where, load().nm_last_error().decode(errors="replace"))


def __getattr__(name):
    if name in SIGNATURES:
        return getattr(load(), name)
    raise AttributeError(name)
