"""Pins for oracle.householder and oracle.panel (CPU only).

dlarfg      -> scipy.linalg.lapack.dlarfg (library) + the reflection identity.
householder_qr / larft -> numpy.linalg.qr(mode='raw') (LAPACK dgeqrf) and the
               brute-force product of explicit reflectors.
tsqr + reconstruct_wy (Alg. 3 + S) -> dgeqrf's (V, T, R) entry by entry
               (SURVEY SC3), and the square-panel edge case (SC4/SC9).
"""
import numpy as np
import pytest
import scipy.linalg.lapack as lapack

from oracle import householder, panel


@pytest.mark.parametrize("m", [1, 2, 5, 33, 200])
def test_dlarfg_matches_lapack(m):
    rng = np.random.default_rng(m)
    for trial in range(5):
        x = rng.standard_normal(m)
        if trial == 1 and m > 1:
            x[0] = 0.0                       # sign(+0) = +1 branch
        if trial == 2:
            x[1:] = 0.0                      # tau = 0 branch
        beta, v, tau = householder.dlarfg(x)
        alpha_l, xtail_l, tau_l = lapack.dlarfg(m, x[0], x[1:].copy() if m > 1 else np.zeros(1), 1)
        assert np.isclose(beta, alpha_l, rtol=1e-14, atol=0)
        assert np.isclose(tau, tau_l, rtol=1e-14, atol=1e-300)
        if m > 1:
            np.testing.assert_allclose(v[1:], xtail_l[: m - 1], rtol=1e-13, atol=1e-15)
        h = np.eye(m) - tau * np.outer(v, v)
        e1 = np.zeros(m)
        e1[0] = beta
        np.testing.assert_allclose(h @ x, e1, atol=1e-13 * (1 + np.linalg.norm(x)))
        np.testing.assert_allclose(h @ h.T, np.eye(m), atol=1e-14)


@pytest.mark.parametrize("m,k", [(64, 8), (300, 32), (33, 32), (32, 32), (20, 32)])
def test_householder_qr_matches_dgeqrf(m, k):
    rng = np.random.default_rng(m * 100 + k)
    p = rng.standard_normal((m, k))
    v, tau, r = panel.householder_qr(p)
    h_raw, tau_l = np.linalg.qr(p, mode="raw")        # LAPACK dgeqrf
    h_raw = h_raw.T
    kk = min(m, k)
    np.testing.assert_allclose(tau, tau_l[:kk], rtol=1e-12, atol=1e-14)
    np.testing.assert_allclose(np.tril(v[:, :kk], -1), np.tril(h_raw[:, :kk], -1), rtol=1e-11, atol=1e-13)
    np.testing.assert_allclose(r, np.triu(h_raw[:kk, :]), rtol=1e-11, atol=1e-12)
    # brute force: product of explicit reflectors reproduces the panel
    qfull = np.eye(m)
    for j in range(kk):
        qfull = qfull @ (np.eye(m) - tau[j] * np.outer(v[:, j], v[:, j]))
    rr = np.zeros((m, k))
    rr[:kk] = r
    np.testing.assert_allclose(qfull @ rr, p, atol=1e-12)
    # compact WY: H_1..H_k = I - V T V^T
    t = panel.larft(v, tau)
    np.testing.assert_allclose(np.eye(m) - v @ t @ v.T, qfull, atol=1e-13)


@pytest.mark.parametrize("m,k,leaf,arity", [(512, 32, 64, 4), (1000, 8, 100, 8), (4096, 64, 256, 8),
                                            (64, 32, 32, 2), (40, 32, 32, 8)])
def test_tsqr_reconstruction_reproduces_dgeqrf(m, k, leaf, arity):
    """SC3: TSQR explicit Q -> modified LU with on-the-fly S -> LAPACK's V, T, R."""
    rng = np.random.default_rng(k + m)
    p = rng.standard_normal((m, k)) * np.logspace(0, -3, k)[None, :]   # graded columns
    q, rt = panel.tsqr(p, leaf_rows=leaf, arity=arity)
    np.testing.assert_allclose(q.T @ q, np.eye(k), atol=1e-13)
    np.testing.assert_allclose(q @ rt, p, atol=1e-13)
    y, t, w, s = panel.reconstruct_wy(q)
    v, tau, r = panel.householder_qr(p)
    np.testing.assert_allclose(y, v, atol=1e-12)
    np.testing.assert_allclose(t, panel.larft(v, tau), atol=1e-12)
    np.testing.assert_allclose(w, y @ t, atol=1e-12)
    np.testing.assert_allclose(s[:, None] * rt, r, atol=1e-12 * np.abs(r).max())
    # (I - Y T Y^T)[:, :k] = Q S   (the identity the reconstruction inverts)
    e = np.zeros((m, k))
    e[:k] = np.eye(k)
    np.testing.assert_allclose(e - y @ (t @ y[:k].T), q * s[None, :], atol=1e-12)


def test_reconstruction_square_panel_sign_variant():
    """SC4/SC9: on a square panel the last reflector has length 1.  dlarfg gives tau = 0,
    the reconstruction gives tau = 2 (H = I - 2 e e^T): a valid reflector set that
    differs by D = diag(1,..,1,-1) (reading C1).  Both factor the panel exactly."""
    rng = np.random.default_rng(5)
    k = 32
    p = rng.standard_normal((k, k))
    q, rt = panel.tsqr(p, leaf_rows=k)
    y, t, w, s = panel.reconstruct_wy(q)
    assert np.isclose(t[-1, -1], 2.0)
    v, tau, r = panel.householder_qr(p)
    assert tau[-1] == 0.0
    np.testing.assert_allclose(y[:, :-1], v[:, :-1], atol=1e-12)
    h = np.eye(k) - y @ t @ y.T
    rh = s[:, None] * rt
    np.testing.assert_allclose(h @ rh, p, atol=1e-12)
    d = np.ones(k)
    d[-1] = -1.0
    np.testing.assert_allclose(rh, d[:, None] * r, atol=1e-12 * np.abs(r).max())
