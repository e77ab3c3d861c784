"""Band -> tridiagonal and Sturm bisection (oracle; test infrastructure only).

Stage two of the two-stage EVD (Fig. 1) is out of scope for the GPU
path; the oracle needs eigenvalues of B to check the band reduction.  Band ->
tridiagonal is the same plain definition with b = 1 (``sbr_unblocked(B, 1)``);
eigenvalues follow by bisection on Sturm counts ("bisection [10]").
"""
from __future__ import annotations

import numpy as np

from .sbr import sbr_unblocked


def tridiagonalize(bmat: np.ndarray):
    """Return ``(d, e)``, diagonal and sub-diagonal of ``T = Q^T B Q`` (b = 1 reduction)."""
    t = sbr_unblocked(bmat, 1, want_q=False)["B"]
    return np.diagonal(t).copy(), np.diagonal(t, -1).copy()


def sturm_count(d: np.ndarray, e: np.ndarray, x: np.ndarray) -> np.ndarray:
    """Number of eigenvalues of tridiag(d, e) strictly below each shift in ``x``.

    LDL^T of ``T - x I``: ``q_0 = d_0 - x``, ``q_i = d_i - x - e_{i-1}^2 / q_{i-1}``;
    the count is the number of negative pivots (Sylvester's law of inertia).  A
    zero pivot is replaced by ``-pivmin`` as in LAPACK dstebz.
    """
    x = np.asarray(x, dtype=np.float64)
    n = d.shape[0]
    scale = max(float(np.max(np.abs(d))) if n else 0.0,
                float(np.max(np.abs(e))) if n > 1 else 0.0, 1e-300)
    pivmin = np.finfo(np.float64).tiny * max(1.0, scale * scale)
    count = np.zeros(x.shape, dtype=np.int64)
    q = d[0] - x
    q = np.where(np.abs(q) < pivmin, -pivmin, q)
    count += q < 0
    for i in range(1, n):
        q = d[i] - x - (e[i - 1] * e[i - 1]) / q
        q = np.where(np.abs(q) < pivmin, -pivmin, q)
        count += q < 0
    return count


def bisection_eigenvalues(d: np.ndarray, e: np.ndarray, tol: float | None = None) -> np.ndarray:
    """All eigenvalues of tridiag(d, e), ascending, by bisection on Gershgorin bounds.

    Eigenvalue k (0-based) is the smallest x with ``sturm_count(x) > k``; each
    interval is halved until ITS width is at most ``tol`` (default
    ``2 eps max(|lo|, |hi|)`` of the Gershgorin bounds) -- per-interval
    convergence, as LAPACK dstebz tests each interval on its own.
    """
    d = np.asarray(d, dtype=np.float64)
    e = np.asarray(e, dtype=np.float64)
    n = d.shape[0]
    if n == 0:
        return np.zeros(0)
    ae = np.abs(e)
    rad = np.zeros(n)
    rad[:-1] += ae
    rad[1:] += ae
    lo_b = float(np.min(d - rad))
    hi_b = float(np.max(d + rad))
    span = max(abs(lo_b), abs(hi_b), 1e-300)
    if tol is None:
        tol = 2.0 * np.finfo(np.float64).eps * span
    lo = np.full(n, lo_b - tol)
    hi = np.full(n, hi_b + tol)
    k = np.arange(n)
    for _ in range(200):                    # ~ log2(span / tol) halvings suffice
        active = (hi - lo) > tol
        if not np.any(active):
            break
        mid = 0.5 * (lo + hi)
        below = sturm_count(d, e, mid) > k
        hi = np.where(active & below, mid, hi)
        lo = np.where(active & ~below, mid, lo)
    return 0.5 * (lo + hi)


def band_eigenvalues(bmat: np.ndarray) -> np.ndarray:
    """Eigenvalues of a symmetric band matrix: tridiagonalise, then bisection."""
    d, e = tridiagonalize(bmat)
    return bisection_eigenvalues(d, e)
