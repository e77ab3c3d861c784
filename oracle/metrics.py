"""Accuracy metrics and Q formation from the block output (oracle; test infrastructure only).

P:395 ``E_b = ||A - Q B Q^-1||_F / (N ||A||_F)``, P:399 ``E_o = ||I - Q^-1 Q||_F / N``
and P:421 ``E_s = ||D_s - D_tc||_2 / (N ||D_s||_2)`` are garbled (reading C9):
the printed Table 3/4 values match only without the 1/N and with Q^T in place
of Q^-1, which is BASELINE.json's definition:

* backward error  ``||A - Q B Q^T||_F / ||A||_F``
* orthogonality   ``||Q^T Q - I||_F / sqrt(n)``
* eigenvalues     ``max_k |lambda_k(B) - lambda_k(ref)| / ||A||_2`` (both sorted)

The paper-normalised variants (with the 1/N) are reported alongside.
"""
from __future__ import annotations

import numpy as np

from .sbr import symmetrize_lower


def backward_error(a: np.ndarray, q: np.ndarray, bmat: np.ndarray) -> float:
    a = symmetrize_lower(a)
    r = a - q @ bmat @ q.T
    return float(np.linalg.norm(r) / np.linalg.norm(a))


def orthogonality(q: np.ndarray) -> float:
    n = q.shape[0]
    return float(np.linalg.norm(q.T @ q - np.eye(n)) / np.sqrt(n))


def eigenvalue_error(lam: np.ndarray, lam_ref: np.ndarray, norm_a2: float) -> float:
    return float(np.max(np.abs(np.sort(lam) - np.sort(lam_ref))) / norm_a2)


def paper_normalised(eb: float, eo_sqrt_n: float, n: int) -> tuple[float, float]:
    """The literal P:395/P:399 normalisations, for reporting beside the gates."""
    return eb / n, eo_sqrt_n * np.sqrt(n) / n


def q_from_blocks(n: int, b: int, blocks) -> np.ndarray:
    """``Q = prod_J (I - W_J Y_J^T)`` with block J acting on rows/cols ``c0_J + b ..``.

    ``blocks`` is a list of ``(c0, W_J, Y_J)``; this is the representation that
    ``sbr_reduce`` returns (W_J in the W array, Y_J below the band of A).
    """
    q = np.eye(n)
    for c0, w, y in blocks:
        r0 = c0 + b
        q[:, r0:] = q[:, r0:] - (q[:, r0:] @ np.asarray(w, np.float64)) @ np.asarray(y, np.float64).T
    return q


def blocks_from_output(a_out: np.ndarray, w_out: np.ndarray, n: int, b: int, nb: int):
    """Unpack ``sbr_reduce``'s (A, W) output into ``[(c0, W_J, Y_J)]``.

    Block J (c0 = J nb) has reflector columns ``c0 .. c0+k_J-1`` (c < n - b; the
    last one, c = n-b-1, has length 1); reflector column c has its unit at row
    ``c + b`` and its tail below it in column c of A (LAPACK dsytrd_sy2sb
    layout); W_J is ``W[c0+b:, c0:c0+k_J]``.
    """
    a_out = np.asarray(a_out, dtype=np.float64)
    w_out = np.asarray(w_out, dtype=np.float64)
    ncols = max(0, n - b)                        # reflector columns c = 0 .. n-b-1
    blocks = []
    for c0 in range(0, ncols, nb):
        k = min(nb, ncols - c0)
        r0 = c0 + b
        m = n - r0
        y = np.zeros((m, k))
        for jj in range(k):
            c = c0 + jj
            y[jj, jj] = 1.0
            y[jj + 1:, jj] = a_out[c + b + 1:, c]
        w = w_out[r0:, c0:c0 + k].copy()
        blocks.append((c0, w, y))
    return blocks
