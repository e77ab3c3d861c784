"""Householder reflector, LAPACK ``dlarfg`` convention (oracle; test infrastructure only).

PAPER.md:119 (Sec. 3.2): ``H(v) = I - 2 v v^T / (v^T v)`` maps x to a multiple of
e_1.  The paper's text picks ``v = ||x|| e_1 - x``; its reconstruction step
 requires matching "the sign choices made inside the Householder QR
algorithm", i.e. LAPACK's.  DESIGN.md reading C1: ``H = I - tau v v^T`` with
``v[0] = 1``, ``beta = -sign(alpha) * ||x||`` (sign(+0) = +1) and ``tau = 0``
(H = I) when ``x[1:] == 0``.
"""
from __future__ import annotations

import math

import numpy as np


def dlarfg(x: np.ndarray):
    """Return ``(beta, v, tau)`` with ``(I - tau v v^T) x = beta e_1`` and ``v[0] = 1``.

    Follows LAPACK dlarfg (without its underflow-rescaling loop, which never
    triggers for the O(1)-scaled inputs used here).
    """
    x = np.asarray(x, dtype=np.float64)
    alpha = float(x[0])
    sigma = float(np.linalg.norm(x[1:])) if x.shape[0] > 1 else 0.0
    v = np.zeros_like(x)
    v[0] = 1.0
    if sigma == 0.0:
        return alpha, v, 0.0
    beta = -math.copysign(math.hypot(alpha, sigma), alpha)
    tau = (beta - alpha) / beta
    v[1:] = x[1:] / (alpha - beta)
    return beta, v, tau


def apply_left(tau: float, v: np.ndarray, c: np.ndarray) -> None:
    """In place: ``C <- (I - tau v v^T) C``."""
    if tau != 0.0:
        c -= tau * np.outer(v, v @ c)


def apply_right(tau: float, v: np.ndarray, c: np.ndarray) -> None:
    """In place: ``C <- C (I - tau v v^T)``."""
    if tau != 0.0:
        c -= tau * np.outer(c @ v, v)
