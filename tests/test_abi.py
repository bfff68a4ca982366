"""The C-ABI library loads and exports every symbol include/nm.h declares (no GPU needed,
no device compute)."""
import ctypes
import os
import re

import pytest

from paper_conf_ppopp_chensz0s25_b200 import _lib, build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "nm.h")).read()
    return sorted(set(re.findall(r"^NM_API\s+[\w\s\*]+?\b(nm_\w+)\s*\(", src, flags=re.M)))


def test_build_and_load():
    build.build()
    lib = _lib.load()
    assert lib.nm_version() == 1


def test_every_declared_symbol_is_exported_and_bound():
    names = _declared()
    assert len(names) >= 17
    lib = ctypes.CDLL(_lib.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
        assert n in _lib.SIGNATURES, "binding missing for " + n
    assert set(_lib.SIGNATURES) == set(names)


def test_status_strings_and_errors():
    lib = _lib.load()
    for s in range(7):
        assert lib.nm_status_string(s).decode().startswith("NM_")
    # invalid arguments are rejected without touching a device
    st = lib.nm_reorder(None, 1, 2, 4, None, None, None)
    assert st == _lib.NM_ERR_INVALID_ARG
    assert b"NULL" in lib.nm_last_error()


def test_reorder_rejects_bad_csr_and_asymmetric():
    import numpy as np
    from paper_conf_ppopp_chensz0s25_b200 import api
    ip = np.array([0, 1, 1], np.int64)
    ic = np.array([1], np.int32)  # (0,1) without (1,0)
    with pytest.raises(_lib.NMError) as e:
        api.reorder(ip, ic, 1, 2, 4)
    assert e.value.status == _lib.NM_ERR_NOT_SYMMETRIC
    ip = np.array([0, 2, 2], np.int64)
    ic = np.array([1, 1], np.int32)  # duplicate
    with pytest.raises(_lib.NMError) as e:
        api.reorder(ip, ic, 1, 2, 4)
    assert e.value.status == _lib.NM_ERR_BAD_CSR


def test_pack_support_set_rejected_cleanly():
    """nm.h's support set for nm_pack: Vp in {16, 32, 64, 128} (0 = auto), N = 2,
    M in {4, 8, 16}, 16-bit dtypes.  Anything else is NM_ERR_UNSUPPORTED before any device work."""
    import ctypes

    import numpy as np
    from paper_conf_ppopp_chensz0s25_b200 import api
    lib = _lib.load()
    ip, ic = np.array([0, 1, 2], np.int64), np.array([1, 0], np.int32)
    c, keep = api._csr_struct(ip, ic)
    h = ctypes.c_void_p()
    for V, N, M, Vp, dt in [(1, 2, 4, 8, _lib.NM_F16), (64, 2, 8, 256, _lib.NM_BF16), (1, 2, 4, 48, _lib.NM_F16), (1, 3, 4, 128, _lib.NM_F16),
                            (1, 2, 32, 128, _lib.NM_F16), (1, 2, 4, 128, _lib.NM_F32)]:
        st = lib.nm_pack(ctypes.byref(c), None, V, N, M, Vp, dt, None, ctypes.byref(h))
        assert st == _lib.NM_ERR_UNSUPPORTED, (V, N, M, Vp, dt, st)
        assert not h.value
