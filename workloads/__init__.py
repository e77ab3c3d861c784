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
    "haar_orthogonal",
    "prescribed_spectrum_device",
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


def prescribed_spectrum_device(n: int, kind: str = "geo", kappa: float = 1e5, seed: int = BASE_SEED,
                               a_device: str = "cuda:0", haar_max: int = 16384):
    """Prescribed-spectrum input on the device (torch fp32 (n, n), bit-symmetric) and a one-line
    description.  n <= haar_max: the host recipe ``prescribed_spectrum`` (Haar Q).  Larger n
    (config 5): Q = H D1 H D2 H D3 / n^{3/2} -- H the n x n Walsh-Hadamard matrix
    (fast transform), D_i seeded random +-1 diagonals -- so A = Q diag(lam) Q^T is dense, exactly
    orthogonally similar to diag(lam) in exact arithmetic, and built in O(n^2 log n) on the GPU
    (fp32; n a power of two).  Input generation only: none of the method's arithmetic."""
    import torch

    if n <= haar_max:
        a, _ = prescribed_spectrum(n, kind, kappa, seed)
        return torch.from_numpy(a).to(a_device), f"prescribed spectrum SVD_{kind} kappa={kappa:g}, Haar Q (seed {seed})"
    if n & (n - 1):
        raise ValueError("the Hadamard recipe needs n a power of two")
    lam = torch.from_numpy(spectrum(n, kind, kappa)).to(device=a_device, dtype=torch.float32)
    g = torch.Generator(device="cpu").manual_seed(seed)
    d = [(torch.randint(0, 2, (n,), generator=g).to(a_device, torch.float32) * 2 - 1) for _ in range(3)]

    def fwht_rows_(x):   # x (n, m): x <- H x (unnormalised), in place, column block by block
        h = 1
        while h < n:
            v = x.view(n // (2 * h), 2, h, -1)
            a = v[:, 0].clone()
            v[:, 0].add_(v[:, 1])
            v[:, 1].neg_().add_(a)
            del a
            h *= 2
        return x

    def apply_q_(x):     # x <- Q x, column blocks of 4096 to bound the temporaries
        for c0 in range(0, x.shape[1], 4096):
            blk = x[:, c0:c0 + 4096]
            t = blk.contiguous()
            for di in (d[2], d[1], d[0]):
                t.mul_(di[:, None])
                fwht_rows_(t)
            t.mul_(float(n) ** -1.5)
            blk.copy_(t)
        return x

    t = torch.diag(lam)                  # T = Q diag(lam)
    apply_q_(t)
    a = t.t().contiguous()               # diag(lam) Q^T
    del t
    apply_q_(a)                          # A = Q diag(lam) Q^T
    low = torch.tril(a)
    a = low + torch.tril(low, -1).t()
    return a.contiguous(), (f"prescribed spectrum SVD_{kind} kappa={kappa:g}, randomised Hadamard "
                            f"Q = H D1 H D2 H D3 / n^1.5 (seed {seed})")
