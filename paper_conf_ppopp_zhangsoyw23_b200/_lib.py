"""ctypes binding of libsbr.so (include/sbr.h): argument marshalling only.

Every step of the reduction runs in libsbr's CUDA kernels; this module only
converts torch tensors / numpy arrays to pointers and sizes.  There is no
fallback: if the shared library is missing the import of the binding fails.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libsbr.so")

# status codes / constants (mirror include/sbr.h)
SBR_OK = 0
SBR_ERR_NONFINITE = 1
SBR_ERR_CUDA = 2
SBR_ERR_NCCL = 3
SBR_ERR_NOMEM = 4
SBR_ERR_UNSUPPORTED = 5
SBR_FP16_FP32ACC = 0
SBR_3XTF32 = 1
SBR_BF16_FP32ACC = 2   # ablation: the FP16 path with bfloat16 operands (sbr.h)
SBR_OUT_BAND, SBR_OUT_Y, SBR_OUT_W = 1, 2, 4
KERNEL_CLASSES = {"panel": 0, "lazy": 1, "wmerge": 2, "pass": 3, "syr2k": 4, "other": 5, "stage2": 6}

# symbol -> (restype, argtypes): the complete exported surface of include/sbr.h
_h = ctypes.c_void_p
_i = ctypes.c_int
_i64 = ctypes.c_int64
_p = ctypes.c_void_p
SIGNATURES = {
    "sbr_create": (_i, [ctypes.POINTER(ctypes.c_void_p), _i, _p]),
    "sbr_set_stream": (_i, [_h, _p]),
    "sbr_destroy": (_i, [_h]),
    "sbr_workspace_query": (_i, [_h, _i64, _i, _i, _i, ctypes.POINTER(ctypes.c_size_t)]),
    "sbr_reduce": (_i, [_h, _i, _i64, _i, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_reduce_host": (_i, [_h, _i, _i64, _i, _i, _p, _i64, _p, _i64, _p, _i64, _i]),
    "sbr_sync": (_i, [_h]),
    "sbr_status_string": (ctypes.c_char_p, [_i]),
    "sbr_generate_symmetric": (_i, [_h, ctypes.c_uint64, _i64, _p, _i64]),
    "sbr_set_kernel_timing": (_i, [_h, _i]),
    "sbr_reset_kernel_stats": (_i, [_h]),
    "sbr_kernel_stats": (_i, [_h, _i, ctypes.POINTER(_i64), ctypes.POINTER(ctypes.c_double),
                              ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]),
    "sbr_launch_count": (_i64, [_h]),
    "sbr_version": (ctypes.c_char_p, []),
    "sbr_get_unique_id": (_i, [_p]),
    "sbr_create_dist": (_i, [ctypes.POINTER(ctypes.c_void_p), _i, _p, _p, _i, _i]),
    "sbr_create_dist_local": (_i, [ctypes.POINTER(ctypes.c_void_p), _i, _p, _i, _i, _i]),
    "sbr_local_cols": (_i64, [_i64, _i, _i, _i]),
    "sbr_reduce_dist": (_i, [_h, _i, _i64, _i, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_form_q": (_i, [_h, _i64, _i, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_form_w": (_i, [_h, _i64, _i, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_apply_q": (_i, [_h, _i64, _i, _i, _p, _i64, _p, _i64, _p, _i64, _i64]),
    "sbr_band_to_tridiag": (_i, [_h, _i64, _i, _p, _i64, _p, _p]),
    "sbr_tridiag_eigenvalues": (_i, [_h, _i64, _p, _p, _p]),
    "sbr_band_eigenvalues": (_i, [_h, _i64, _i, _p, _i64, _p]),
    "sbr_eigenvalues": (_i, [_h, _i, _i64, _i, _i, _p, _i64, _p]),
    "sbr_rank": (_i, [_h]),
    "sbr_nranks": (_i, [_h]),
    # kernel-level test hooks (include/sbr_testing.h)
    "sbr_test_pass_fp16": (_i, [_h, _i64, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_test_pass_fp16_part": (_i, [_h, _i64, _i, _i, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_test_syr2k_fp16": (_i, [_h, _i64, _i, _p, _i64, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_test_zform_fp16": (_i, [_h, _i64, _i, _p, _i64, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_test_panel": (_i, [_h, _i64, _i, _p, _i64, _p, _p, _i64, _p]),
    "sbr_test_panel_trace": (_i, [_h, _i, _p, _p]),
    "sbr_test_pass_tf32": (_i, [_h, _i64, _i, _p, _i64, _p, _i64, _i64, _p, _i64, _p, _i64]),
    "sbr_test_syr2k_tf32": (_i, [_h, _i64, _i, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_test_zform_tf32": (_i, [_h, _i64, _i, _p, _i64, _p, _i64, _p, _i64, _p, _i64]),
    "sbr_test_pass_partition": (_i, [_i64, _i, _i, _i, ctypes.POINTER(_i64), ctypes.POINTER(_i64),
                                     ctypes.POINTER(_i64)]),
    "sbr_test_pass_tiles": (_i, [_i64, _i, _i64, _i64, _p]),
    "sbr_test_set_knob": (_i, [_i, _i]),
    "sbr_test_pass_owned_tiles": (_i64, [_i64, _i, _i, _i64, _i, _i, _p, _i64]),
    "sbr_test_panel_declines": (_i, [_h, _i, ctypes.POINTER(_i64)]),
}

_LIB = None


def lib():
    """Load libsbr.so (once).  Raises if it is missing -- there is no fallback."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
        handle = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(handle, name)
            fn.restype = res
            fn.argtypes = args
        _LIB = handle
    return _LIB


class SbrError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = lib().sbr_status_string(status).decode()
        super().__init__(f"{where}: status {status}: {msg}")


def check(status: int, where: str) -> None:
    if status != SBR_OK:
        raise SbrError(status, where)
