"""Pins for oracle.sbr, oracle.tridiag and oracle.metrics (CPU only).

sbr_unblocked  -> LAPACK dsytrd_sy2sb entry by entry (SC1); b = 1 -> dgehrd
                  (scipy.linalg.hessenberg); invariants (A = Q B Q^T, Q^T Q = I,
                  exact band); eigenvalues -> dsyevd (numpy eigvalsh) and the
                  closed-form prescribed spectrum; special cases (b >= n-1,
                  diagonal A); brute force on tiny n.
sbr_wy_blocked -> equals sbr_unblocked for any nb (SC2), incl. ragged n and nb = b.
tridiag        -> dstebz (scipy eigvalsh_tridiagonal) and dense eigvalsh.
metrics        -> closed forms on constructed examples.
"""
import numpy as np
import pytest
import scipy.linalg as sla

import workloads
from lapack_ref import have_sy2sb, sytrd_sy2sb
from oracle import metrics, sbr, tridiag

needs_sy2sb = pytest.mark.skipif(not have_sy2sb(), reason="scipy OpenBLAS lacks dsytrd_sy2sb")

CASES = [(64, 1), (64, 4), (96, 8), (128, 32), (50, 7), (100, 8), (130, 16)]


@needs_sy2sb
@pytest.mark.parametrize("n,b", CASES)
def test_unblocked_matches_lapack_sy2sb(n, b):
    a = workloads.random_symmetric(n, workloads.config_seed(1) + n).astype(np.float64)
    o = sbr.sbr_unblocked(a, b)
    ab, _, _ = sytrd_sy2sb(a, b)
    ref = sbr.lapack_band_to_dense(ab)
    scale = np.abs(a).max() * np.sqrt(n)
    assert np.abs(o["B"] - ref).max() <= 1e-13 * scale
    assert o["residue"] <= 1e-14 * np.linalg.norm(a)
    np.testing.assert_allclose(sbr.dense_to_lapack_band(o["B"], b), ab, atol=1e-13 * scale)


def test_unblocked_b1_matches_dgehrd():
    n = 80
    a = workloads.random_symmetric(n, 11).astype(np.float64)
    o = sbr.sbr_unblocked(a, 1)
    h = sla.hessenberg(a)                 # LAPACK dgehrd: same dlarfg convention
    t = np.triu(np.tril(h, 1), -1)
    t = np.tril(t) + np.tril(t, -1).T
    assert np.abs(o["B"] - t).max() <= 1e-12


@pytest.mark.parametrize("n,b", CASES)
def test_unblocked_invariants(n, b):
    a = workloads.normal_symmetric(n, n + b).astype(np.float64)
    o = sbr.sbr_unblocked(a, b)
    bm, q = o["B"], o["Q"]
    assert metrics.backward_error(a, q, bm) <= 1e-14
    assert metrics.orthogonality(q) <= 1e-14
    i, j = np.indices((n, n))
    assert np.all(bm[np.abs(i - j) > b] == 0.0)
    np.testing.assert_array_equal(bm, bm.T)
    lam = np.linalg.eigvalsh(bm)
    lam_ref = np.linalg.eigvalsh(a)
    assert np.max(np.abs(lam - lam_ref)) <= 1e-13 * np.linalg.norm(a, 2)


@pytest.mark.parametrize("kind", workloads.SPECTRUM_KINDS)
def test_prescribed_spectrum_recovered(kind):
    n, b = 96, 8
    a, lam = workloads.prescribed_spectrum(n, kind, 1e5, seed=3)
    o = sbr.sbr_unblocked(a, b, want_q=False)
    got = tridiag.band_eigenvalues(o["B"])
    # A is stored fp32: eigenvalues move by at most ||A32 - A64||_2 <= n * 2^-24 * max|a|
    tol = n * 2.0 ** -24 * float(np.abs(a).max()) + 1e-13
    assert np.max(np.abs(np.sort(got) - np.sort(lam))) <= tol


def test_special_cases():
    n = 20
    a = workloads.random_symmetric(n, 1).astype(np.float64)
    for b in (n - 1, n, n + 3):                     # nothing to reduce: B = A, Q = I
        o = sbr.sbr_unblocked(a, b)
        np.testing.assert_array_equal(o["B"], sbr.symmetrize_lower(a))
        np.testing.assert_array_equal(o["Q"], np.eye(n))
    d = np.diag(np.arange(1.0, n + 1))              # already banded: every tau = 0
    o = sbr.sbr_unblocked(d, 3)
    np.testing.assert_array_equal(o["B"], d)
    assert np.all(o["tau"] == 0.0)


def test_brute_force_tiny():
    """n <= 12: Q built from the explicit reflector matrices; Q^T A Q == B."""
    for n, b in [(6, 1), (9, 2), (12, 3)]:
        a = workloads.random_symmetric(n, 100 + n).astype(np.float64)
        o = sbr.sbr_unblocked(a, b)
        q = np.eye(n)
        for c, (v, tau) in enumerate(zip(o["V"], o["tau"])):
            h = np.eye(n)
            h[c + b:, c + b:] -= tau * np.outer(v, v)
            q = q @ h
        np.testing.assert_allclose(q, o["Q"], atol=1e-14)
        np.testing.assert_allclose(q.T @ a @ q, o["B"], atol=1e-13)


@pytest.mark.parametrize("n,b,nb", [(64, 4, 16), (96, 8, 32), (100, 8, 32), (130, 16, 64),
                                    (64, 4, 4), (50, 7, 14), (256, 8, 32), (70, 8, 64)])
def test_blocked_alg1_equals_unblocked(n, b, nb):
    """SC2: Algorithm 1 (lazy WY) reaches the unblocked result for any nb."""
    a = workloads.random_symmetric(n, 7 * n + b).astype(np.float64)
    o = sbr.sbr_unblocked(a, b)
    w = sbr.sbr_wy_blocked(a, b, nb)
    scale = np.linalg.norm(a)
    assert np.abs(w["B"] - o["B"]).max() <= 1e-12 * scale
    assert np.abs(w["Q"] - o["Q"]).max() <= 1e-12 * np.sqrt(n)
    qb = metrics.q_from_blocks(n, b, w["blocks"])
    np.testing.assert_allclose(qb, o["Q"], atol=1e-12 * np.sqrt(n))
    for c0, wj, yj in w["blocks"]:
        # W_J = Y_J T_J with T_J upper triangular, Y_J unit lower staircase
        k = yj.shape[1]
        np.testing.assert_array_equal(np.triu(yj[:k], 1), 0.0)
        np.testing.assert_array_equal(np.diagonal(yj[:k]), 1.0)


def test_bisection_matches_dstebz_and_dense():
    rng = np.random.default_rng(0)
    for n in (1, 2, 7, 60):
        d = rng.standard_normal(n)
        e = rng.standard_normal(max(n - 1, 0))
        lam = tridiag.bisection_eigenvalues(d, e)
        if n > 1:
            ref = sla.eigvalsh_tridiagonal(d, e, lapack_driver="stebz")
        else:
            ref = d.copy()
        t = np.diag(d) + np.diag(e, -1) + np.diag(e, 1)
        scale = max(1.0, np.abs(ref).max())
        assert np.max(np.abs(lam - ref)) <= 1e-13 * scale
        assert np.max(np.abs(lam - np.linalg.eigvalsh(t))) <= 1e-13 * scale
    # Wilkinson W21+: close eigenvalue pairs are resolved
    m = 10
    d = np.abs(np.arange(-m, m + 1, dtype=float))
    e = np.ones(2 * m)
    lam = tridiag.bisection_eigenvalues(d, e)
    ref = np.linalg.eigvalsh(np.diag(d) + np.diag(e, 1) + np.diag(e, -1))
    assert np.max(np.abs(lam - ref)) <= 1e-13 * 11


def test_tridiagonalize_preserves_spectrum():
    n, b = 40, 5
    a = workloads.random_symmetric(n, 3).astype(np.float64)
    bm = sbr.sbr_unblocked(a, b, want_q=False)["B"]
    d, e = tridiag.tridiagonalize(bm)
    t = np.diag(d) + np.diag(e, -1) + np.diag(e, 1)
    np.testing.assert_allclose(np.linalg.eigvalsh(t), np.linalg.eigvalsh(a), atol=1e-13 * n)


def test_metrics_closed_forms():
    n = 16
    q = np.eye(n)
    a = np.diag(np.arange(1.0, n + 1))
    assert metrics.backward_error(a, q, a) == 0.0
    assert metrics.orthogonality(q) == 0.0
    q2 = 2.0 * np.eye(n)                          # Q^T Q - I = 3 I  ->  3 sqrt(n)/sqrt(n)
    assert np.isclose(metrics.orthogonality(q2), 3.0)
    b2 = a.copy()
    b2[0, 0] += 1.0                               # ||A - B||_F = 1
    assert np.isclose(metrics.backward_error(a, q, b2), 1.0 / np.linalg.norm(a))
    assert np.isclose(metrics.eigenvalue_error(np.array([1.0, 3.0]), np.array([3.0, 1.5]), 2.0), 0.25)


def test_band_storage_roundtrip():
    n, b = 30, 4
    a = workloads.random_symmetric(n, 9).astype(np.float64)
    bm = sbr.band_part(a, b)
    ab = sbr.dense_to_lapack_band(bm, b)
    np.testing.assert_array_equal(sbr.lapack_band_to_dense(ab), bm)
    assert ab[0, 3] == bm[3, 3] and ab[2, 5] == bm[7, 5]


def test_blocks_from_output_roundtrip():
    """The (A, W) output layout (Y below the band, LAPACK style) reproduces Q."""
    n, b, nb = 64, 4, 16
    a = workloads.random_symmetric(n, 5).astype(np.float64)
    w = sbr.sbr_wy_blocked(a, b, nb)
    a_out = np.zeros((n, n))
    w_out = np.zeros((n, n - b))
    for c0, wj, yj in w["blocks"]:
        k = yj.shape[1]
        for jj in range(k):
            a_out[c0 + jj + b + 1:, c0 + jj] = yj[jj + 1:, jj]
        w_out[c0 + b:, c0:c0 + k] = wj
    blocks = metrics.blocks_from_output(a_out, w_out, n, b, nb)
    np.testing.assert_allclose(metrics.q_from_blocks(n, b, blocks), w["Q"], atol=1e-13)


@needs_sy2sb
def test_only_lower_triangle_referenced():
    """Reading C14 pinned against LAPACK: dsytrd_sy2sb(UPLO='L') reads only the lower triangle,
    so an input with garbage above the diagonal must give the same band in the oracle as in
    LAPACK -- a mirrored upper triangle (or a transposed read) would fail."""
    n, b = 90, 6
    a = workloads.random_symmetric(n, 1234).astype(np.float64)
    junk = a.copy()
    iu = np.triu_indices(n, 1)
    junk[iu] = np.random.default_rng(5).standard_normal(len(iu[0])) * 100.0
    o = sbr.sbr_unblocked(junk, b)
    ab, _, _ = sytrd_sy2sb(junk, b)
    ref = sbr.lapack_band_to_dense(ab)
    assert np.abs(o["B"] - ref).max() <= 1e-12 * np.linalg.norm(np.tril(a))
    w = sbr.sbr_wy_blocked(junk, b, 18)
    assert np.abs(w["B"] - ref).max() <= 1e-12 * np.linalg.norm(np.tril(a))
    np.testing.assert_array_equal(sbr.symmetrize_lower(junk), sbr.symmetrize_lower(np.tril(junk)))
