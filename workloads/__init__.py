"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the band-reduction method: it only produces
input matrices (and the prescribed spectra they are built from).  Both the
oracle (``oracle/``) and the CUDA path consume what it returns; neither imports
the other.

Recipes:

* ``random_symmetric(n, seed)`` -- the paper's "Uniform" type (PAPER.md:376,
  Table 3): ``a_ij = a_ji ~ U[-1, 1)`` from a counter-based hash so the host
  and the device generator (``sbr_generate_symmetric`` in ``include/sbr.h``)
  are bit-identical:
  ``h = splitmix64(seed ^ ((max(i,j) << 32) | min(i,j)))``; the top 24 bits
  ``u`` give ``a = (u - 2**23) * 2**-23`` (exact in fp32).
* ``normal_symmetric(n, seed)`` -- the paper's "Normal" type:
  N(0,1) lower triangle from numpy's PCG64, mirrored.
* ``prescribed_spectrum(n, kind, kappa, seed)`` -- the SVD_* types of
  PAPER.md:377-384 (magma_generate conventions, recalled):
  ``A = Q diag(lam) Q^T`` with Haar ``Q`` (QR of a Gaussian with the sign fix),
  built in fp64 and stored fp32 (bit-symmetric).
"""
from __future__ import annotations

import numpy as np

BASE_SEED = 20230225
MASK64 = np.uint64(0xFFFFFFFFFFFFFFFF)

__all__ = [
    "BASE_SEED",
    "config_seed",
    "splitmix64",
    "random_symmetric",
    "random_symmetric_columns",
    "normal_symmetric",
    "spectrum",
    "prescribed_spectrum",
    "SPECTRUM_KINDS",
]


def config_seed(k: int) -> int:
    """Seed of BASELINE.json config k (1-based): 20230225 + k."""
    return BASE_SEED + int(k)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)) & MASK64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & MASK64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & MASK64
        return z ^ (z >> np.uint64(31))


def _hash_entries(i: np.ndarray, j: np.ndarray, seed: int) -> np.ndarray:
    hi = np.maximum(i, j).astype(np.uint64)
    lo = np.minimum(i, j).astype(np.uint64)
    key = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) ^ ((hi << np.uint64(32)) | lo)
    u = (splitmix64(key) >> np.uint64(40)).astype(np.int64)  # top 24 bits
    return ((u - (1 << 23)).astype(np.float64) * 2.0 ** -23).astype(np.float32)


def random_symmetric_columns(n: int, seed: int, c0: int, c1: int) -> np.ndarray:
    """Columns [c0, c1) of ``random_symmetric(n, seed)`` as an (n, c1-c0) fp32 array."""
    i = np.arange(n, dtype=np.int64)[:, None]
    j = np.arange(c0, c1, dtype=np.int64)[None, :]
    return _hash_entries(i, j, seed)


def random_symmetric(n: int, seed: int) -> np.ndarray:
    """n x n fp32, bit-symmetric, entries U[-1,1) on a 2^-23 grid.

    Hashes only the lower triangle (column blocks, rows >= the block's first
    column) and mirrors it block by block."""
    out = np.empty((n, n), dtype=np.float32)
    step = 256
    for c0 in range(0, n, step):
        c1 = min(n, c0 + step)
        i = np.arange(c0, n, dtype=np.uint64)[:, None]
        j = np.arange(c0, c1, dtype=np.uint64)[None, :]
        hi = np.maximum(i, j)
        lo = np.minimum(i, j)
        key = (hi << np.uint64(32)) | lo
        key ^= np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
        h = splitmix64(key)
        h >>= np.uint64(40)
        v = h.astype(np.int64)
        v -= 1 << 23
        blk = v.astype(np.float32)
        blk *= np.float32(2.0 ** -23)
        out[c0:, c0:c1] = blk
        out[c0:c1, c0:] = blk.T
    return out


def normal_symmetric(n: int, seed: int) -> np.ndarray:
    """n x n fp32 with N(0,1) lower triangle, mirrored ("Normal")."""
    g = np.random.Generator(np.random.PCG64(seed)).standard_normal((n, n))
    low = np.tril(g)
    a = low + np.tril(low, -1).T
    return a.astype(np.float32)


SPECTRUM_KINDS = ("geo", "arith", "cluster0", "cluster1")


def spectrum(n: int, kind: str, kappa: float) -> np.ndarray:
    """Prescribed eigenvalues, descending, max 1, min 1/kappa."""
    if n == 1:
        return np.ones(1)
    i = np.arange(n, dtype=np.float64)
    if kind == "geo":
        lam = kappa ** (-i / (n - 1))
    elif kind == "arith":
        lam = 1.0 - i / (n - 1) * (1.0 - 1.0 / kappa)
    elif kind == "cluster0":
        lam = np.full(n, 1.0 / kappa)
        lam[0] = 1.0
    elif kind == "cluster1":
        lam = np.ones(n)
        lam[-1] = 1.0 / kappa
    else:
        raise ValueError(f"unknown spectrum kind {kind!r}")
    return lam


def haar_orthogonal(n: int, seed: int) -> np.ndarray:
    """Haar-distributed orthogonal matrix (fp64): QR of a Gaussian, columns sign-fixed."""
    g = np.random.Generator(np.random.PCG64(seed)).standard_normal((n, n))
    q, r = np.linalg.qr(g)
    return q * np.where(np.diag(r) < 0, -1.0, 1.0)[None, :]


def prescribed_spectrum(n: int, kind: str = "geo", kappa: float = 1e5, seed: int = BASE_SEED):
    """Return (A fp32 bit-symmetric, lam fp64 descending) with A = Q diag(lam) Q^T."""
    lam = spectrum(n, kind, kappa)
    q = haar_orthogonal(n, seed)
    a = (q * lam[None, :]) @ q.T
    low = np.tril(a)
    a = low + np.tril(low, -1).T
    return a.astype(np.float32), lam
