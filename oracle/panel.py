"""Panel factorisation pieces (oracle; test infrastructure only).

* ``householder_qr``   -- Householder QR of a tall m x k panel, column by column
                          with ``dlarfg`` (the "Householder transformation ... on
                          each small block" of P:311), LAPACK dgeqr2 order.
* ``larft``            -- the triangular factor T with ``H_1 ... H_k = I - V T V^T``
                          (memory-efficient WY; Schreiber & Van Loan [34]).
* ``tsqr``             -- Tall-Skinny QR (Sec. 5.1): a reduction tree of
                          local Householder QRs returning the explicit thin Q and R
                          (signs arbitrary, as TSQR produces them).
* ``reconstruct_wy``   -- Householder reconstruction from an explicit Q
                          (Alg. 3, with Ballard et al.'s sign matrix S,
                          P:339; reading C7):
                          ``Q_1 - S = L U`` (non-pivoted, s_j = -sign(d_j) chosen
                          on the fly), ``Y = [L; Q_2 U^-1]``, ``T = -U S L^-T``,
                          ``W = Y T = (E - Q S) L^-T``, ``R_h = S R``.
"""
from __future__ import annotations

import numpy as np
import scipy.linalg as sla

from .householder import dlarfg, apply_left


def householder_qr(p: np.ndarray):
    """Return ``(V, tau, R)`` for the m x k panel ``p`` (m >= 1).

    ``V`` is m x r unit lower trapezoidal (r = min(m, k) reflectors),
    ``R`` is r x k upper trapezoidal, and ``p = (H_1 ... H_r) [R; 0]``.
    """
    a = np.array(p, dtype=np.float64, copy=True)
    m, k = a.shape
    r = min(m, k)
    v_all = np.zeros((m, r))
    tau = np.zeros(r)
    for j in range(r):
        beta, v, t = dlarfg(a[j:, j])
        a[j, j] = beta
        a[j + 1:, j] = 0.0
        apply_left(t, v, a[j:, j + 1:])
        v_all[j:, j] = v
        tau[j] = t
    return v_all, tau, np.triu(a[:r, :])


def larft(v: np.ndarray, tau: np.ndarray) -> np.ndarray:
    """Forward, column-wise T (LAPACK dlarft 'F','C'): ``H_1...H_k = I - V T V^T``."""
    k = tau.shape[0]
    t = np.zeros((k, k))
    for j in range(k):
        t[j, j] = tau[j]
        if j > 0:
            t[:j, j] = -tau[j] * (t[:j, :j] @ (v[:, :j].T @ v[:, j]))
    return t


def apply_q_thin(v: np.ndarray, tau: np.ndarray, c_top: np.ndarray) -> np.ndarray:
    """``(H_1 ... H_r) [C_top; 0]`` for an m x r reflector block V (explicit-Q formation)."""
    m = v.shape[0]
    out = np.zeros((m, c_top.shape[1]))
    out[: c_top.shape[0], :] = c_top
    for j in reversed(range(tau.shape[0])):
        apply_left(tau[j], v[:, j], out)
    return out


def tsqr(p: np.ndarray, leaf_rows: int = 256, arity: int = 8):
    """Tall-Skinny QR by a reduction tree.  Returns ``(Q, R)``, ``p = Q R``.

    Leaves are row blocks of ``leaf_rows`` (the last absorbs the remainder); the
    stacked leaf R factors are reduced recursively, ``arity`` at a time.  Q is
    thin (m x k) and explicit; column signs are whatever the tree produces.
    """
    p = np.asarray(p, dtype=np.float64)
    m, k = p.shape
    if m < k:
        raise ValueError("tsqr needs m >= k")
    leaf_rows = max(leaf_rows, k)
    nleaf = max(1, m // leaf_rows)
    if nleaf == 1:
        v, tau, r = householder_qr(p)
        return apply_q_thin(v, tau, np.eye(k)), r
    bounds = [i * leaf_rows for i in range(nleaf)] + [m]
    leaves = []
    for i in range(nleaf):
        v, tau, r = householder_qr(p[bounds[i]:bounds[i + 1]])
        leaves.append((v, tau, r))
    stacked = np.vstack([r for (_, _, r) in leaves])          # (nleaf*k) x k
    q_up, r = tsqr(stacked, leaf_rows=arity * k, arity=arity)
    q = np.zeros((m, k))
    for i, (v, tau, _) in enumerate(leaves):
        q[bounds[i]:bounds[i + 1]] = apply_q_thin(v, tau, q_up[i * k:(i + 1) * k])
    return q, r


def reconstruct_wy(q: np.ndarray):
    """Householder reconstruction from an explicit thin Q (Alg. 3 + S).

    Returns ``(Y, T, W, s)``: ``Y`` m x k unit lower trapezoidal, ``T`` k x k upper,
    ``W = Y T``, and the signs ``s`` (diagonal of S) such that
    ``I - Y T Y^T`` restricted to its first k columns equals ``Q diag(s)``.
    """
    q = np.asarray(q, dtype=np.float64)
    m, k = q.shape
    a = q[:k, :].copy()
    s = np.zeros(k)
    lmat = np.eye(k)
    umat = np.zeros((k, k))
    for j in range(k):                      # non-pivoted LU of Q_1 - S
        s[j] = -1.0 if a[j, j] >= 0.0 else 1.0   # s_j = -sign(d_j), sign(0) = +1
        a[j, j] -= s[j]
        umat[j, j:] = a[j, j:]
        lmat[j + 1:, j] = a[j + 1:, j] / a[j, j]
        a[j + 1:, j + 1:] -= np.outer(lmat[j + 1:, j], umat[j, j + 1:])
    y = np.zeros((m, k))
    y[:k] = lmat
    if m > k:                               # L_2 = Q_2 U^-1
        y[k:] = sla.solve_triangular(umat, q[k:].T, trans="T", lower=False).T
    lt_inv_t = sla.solve_triangular(lmat, np.eye(k), lower=True, unit_diagonal=True).T
    t = -(umat * s[None, :]) @ lt_inv_t     # T = -U S L^-T
    e = np.zeros((m, k))
    e[:k] = np.eye(k)
    w = (e - q * s[None, :]) @ lt_inv_t     # W = (E - Q S) L^-T (Alg. 3 l.8 read as C7)
    return y, t, w, s
