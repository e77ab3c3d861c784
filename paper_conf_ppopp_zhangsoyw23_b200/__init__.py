"""B200-native WY-based successive band reduction (Zhang et al., PPoPP'23).

Public Python surface (a thin layer over the C ABI in ``include/sbr.h``):

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    h = sbr.Handle(device=0)                 # binds torch's current stream
    ab, w = h.reduce(A, b=32, nb=1024, mode="fp16")   # A: (n, n) float32 CUDA tensor

Memory layout: libsbr is column-major.  A torch (n, n) contiguous tensor ``A`` is
passed as the column-major matrix ``A.T``; for a symmetric input that is the same
matrix.  On return ``A`` holds (column-major) the LAPACK sy2sb layout: the band
and, below it, the Householder vectors -- in torch indexing reflector column c's
tail is ``A[c, c+b+1:]``.  ``ab`` has torch shape (n, b+1): ``ab[j, d] = B[j+d, j]``
(``ab.T`` is LAPACK lower band storage).  ``w`` has torch shape (n-b, n):
``w[c, r] = W(r, c)``.
"""
from .api import (Handle, reduce, reduce_host, generate_symmetric, band_to_dense, get_unique_id,  # noqa: F401
                  pass_partition, pass_tiles, local_cols, local_columns, pass_owned_tiles)
from ._lib import lib, LIB_PATH, SbrError  # noqa: F401

__all__ = ["Handle", "reduce", "reduce_host", "generate_symmetric", "band_to_dense", "get_unique_id",
           "pass_partition", "pass_tiles", "local_cols", "local_columns", "pass_owned_tiles", "lib", "LIB_PATH",
           "SbrError"]
