"""LAPACK pins for the oracle, reached by ctypes in scipy's bundled OpenBLAS.

Only tests use this.  ``dsytrd_sy2sb`` is LAPACK's own dense -> band reduction
(the routine the paper's MAGMA baseline ``ssytrd_sy2sb`` mirrors, P:311 fn. 2);
with UPLO='L' it uses the dlarfg sign convention and the same reflector range as
the oracle, so B agrees entry by entry.
"""
from __future__ import annotations

import ctypes
import glob
import os

import numpy as np
import scipy

_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        d = os.path.join(os.path.dirname(scipy.__file__), "..", "scipy.libs")
        cands = sorted(glob.glob(os.path.join(d, "libscipy_openblas*.so")))
        if not cands:
            raise RuntimeError("scipy's OpenBLAS not found")
        _LIB = ctypes.CDLL(cands[0])
    return _LIB


def have_sy2sb() -> bool:
    try:
        return hasattr(_lib(), "scipy_dsytrd_sy2sb_")
    except Exception:
        return False


def sytrd_sy2sb(a: np.ndarray, kd: int, dtype=np.float64):
    """LAPACK ?sytrd_sy2sb with UPLO='L'.  Returns ``(AB, tau, A_out)``.

    AB is LAPACK lower band storage ``(kd+1) x n``: ``AB[i-j, j] = B[i, j]``.
    """
    lib = _lib()
    fn = lib.scipy_dsytrd_sy2sb_ if dtype == np.float64 else lib.scipy_ssytrd_sy2sb_
    n = a.shape[0]
    af = np.asfortranarray(a.astype(dtype))
    ldab = kd + 1
    ab = np.zeros((ldab, n), dtype=dtype, order="F")
    tau = np.zeros(max(1, n - kd), dtype=dtype)
    info = ctypes.c_int(0)
    uplo = ctypes.c_char(b"L")
    i32 = ctypes.c_int
    ptr = lambda x: x.ctypes.data_as(ctypes.c_void_p)  # noqa: E731
    work_q = np.zeros(1, dtype=dtype)
    args = [ctypes.byref(uplo), ctypes.byref(i32(n)), ctypes.byref(i32(kd)), ptr(af),
            ctypes.byref(i32(n)), ptr(ab), ctypes.byref(i32(ldab)), ptr(tau)]
    fn(*args, ptr(work_q), ctypes.byref(i32(-1)), ctypes.byref(info), ctypes.c_size_t(1))
    lwork = max(1, int(work_q[0]))
    work = np.zeros(lwork, dtype=dtype)
    fn(*args, ptr(work), ctypes.byref(i32(lwork)), ctypes.byref(info), ctypes.c_size_t(1))
    if info.value != 0:
        raise RuntimeError(f"sytrd_sy2sb info={info.value}")
    return ab, tau, af
