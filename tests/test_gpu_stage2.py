"""Stage two on the GPU (include/sbr.h sbr_band_to_tridiag, sbr_tridiag_eigenvalues,
sbr_band_eigenvalues, sbr_eigenvalues), against the oracle (oracle.tridiag, pinned to LAPACK
dstebz / dense eigvalsh in tests/test_oracle_sbr.py) and the mathematics:

  * bisection: the GPU multisection keeps the oracle bisection's invariant (same bounds,
    tolerance, pivmin, recurrence and operation order, IEEE fp64) -> within tol of it;
  * bulge chase: T = Q2^T B Q2 is tridiagonal with the spectrum of B (fp64, backward stable:
    |lam(T) - lam(B)| <= 1e-11 ||B||), ||T||_F = ||B||_F, and (Q2 e_0 = e_0, implicit-Q theorem)
    T equals the oracle's b = 1 reduction up to the signs of e on small cases;
  * the pipeline: sbr_eigenvalues(A) against eigvalsh(A) within the reduction's gate.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _handle():
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    return sbr.Handle(0)


def _random_band(n, b, seed, zero_cols=()):
    rng = np.random.default_rng(seed)
    ab = rng.uniform(-1, 1, (n, b + 1)).astype(np.float32)
    for j in range(n):
        ab[j, max(0, n - j):] = 0.0          # entries below row n-1 do not exist
    for j in zero_cols:
        ab[j, 1:] = 0.0
    return ab


def _band_dense(ab):
    n, bp1 = ab.shape
    m = np.zeros((n, n))
    for d in range(bp1):
        for j in range(n - d):
            m[j + d, j] = m[j, j + d] = ab[j, d]
    return m


@pytest.mark.parametrize("n", [1, 2, 3, 17, 257, 1000, 5000])
def test_multisection_matches_oracle_bisection(n):
    """Both keep count(lo) <= k < count(hi) and stop at width <= tol = 2 eps max|Gershgorin|; the
    GPU's Sturm recurrence divides with a refined reciprocal (a few ulps), which can move a count
    transition by a few ulps of the spectrum: the midpoints agree within 4 tol."""
    import torch

    from oracle.tridiag import bisection_eigenvalues

    rng = np.random.default_rng(7 + n)
    d = rng.uniform(-2, 2, n)
    e = rng.uniform(-1, 1, max(n - 1, 0))
    if n > 10:
        e[n // 3] = 0.0                      # a split: block-diagonal T
        d[n // 2] = d[n // 2 + 1]            # repeated diagonal entries
    h = _handle()
    lam = h.tridiag_eigenvalues(torch.from_numpy(d).cuda(), torch.from_numpy(e).cuda()).cpu().numpy()
    ref = bisection_eigenvalues(d, e)
    rad = np.zeros(n)
    rad[:-1] += np.abs(e)
    rad[1:] += np.abs(e)
    tol = 2 * np.finfo(np.float64).eps * max(abs(np.min(d - rad)), abs(np.max(d + rad)))
    err = float(np.max(np.abs(lam - ref)))
    print(f"multisection n={n}: max|gpu - oracle| {err:.1e} (tol {tol:.1e})")
    assert err <= 4 * tol
    assert np.all(np.diff(lam) >= 0)
    h.close()


def test_bisection_closed_form():
    """tridiag(-1, 2, -1): lam_k = 2 - 2 cos(k pi / (n+1)), k = 1..n."""
    import torch

    n = 500
    h = _handle()
    d = torch.full((n,), 2.0, dtype=torch.float64, device="cuda")
    e = torch.full((n - 1,), -1.0, dtype=torch.float64, device="cuda")
    lam = h.tridiag_eigenvalues(d, e).cpu().numpy()
    k = np.arange(1, n + 1)
    ref = 2.0 - 2.0 * np.cos(k * np.pi / (n + 1))
    assert np.max(np.abs(lam - ref)) <= 1e-14
    h.close()


@pytest.mark.parametrize("n,b", [(3, 2), (40, 8), (257, 32), (1000, 32), (2050, 64), (777, 17), (300, 2), (65, 64)])
def test_band_to_tridiag_spectrum(n, b):
    import torch

    from oracle.tridiag import bisection_eigenvalues

    ab = _random_band(n, b, 100 + n + b, zero_cols=(n // 2,))
    bm = _band_dense(ab)
    h = _handle()
    d, e = h.band_to_tridiag(torch.from_numpy(ab).cuda())
    d, e = d.cpu().numpy(), e.cpu().numpy()
    nb_ = max(np.max(np.abs(np.linalg.eigvalsh(bm))), 1e-300)
    lam_t = bisection_eigenvalues(d, e)
    lam_b = np.linalg.eigvalsh(bm)
    fro_t = np.sqrt(np.sum(d * d) + 2 * np.sum(e * e))
    err = np.max(np.abs(lam_t - lam_b)) / nb_
    print(f"band_to_tridiag n={n} b={b}: eig err {err:.1e}  |T|_F/|B|_F - 1 {fro_t / np.linalg.norm(bm) - 1:.1e}")
    assert err <= 1e-11
    assert abs(fro_t / np.linalg.norm(bm) - 1.0) <= 1e-12
    assert abs(np.sum(d) - np.trace(bm)) <= 1e-10 * max(1.0, np.abs(np.diag(bm)).sum())
    h.close()


@pytest.mark.parametrize("n,b", [(40, 4), (60, 8)])
def test_band_to_tridiag_equals_oracle_reduction(n, b):
    """Q2 e_0 = e_0 on both sides, so T is unique up to the signs of e (implicit-Q theorem)."""
    import torch

    from oracle.tridiag import tridiagonalize

    ab = _random_band(n, b, 5 + n)
    h = _handle()
    d, e = h.band_to_tridiag(torch.from_numpy(ab).cuda())
    d0, e0 = tridiagonalize(_band_dense(ab))
    assert np.max(np.abs(d.cpu().numpy() - d0)) <= 1e-9
    assert np.max(np.abs(np.abs(e.cpu().numpy()) - np.abs(e0))) <= 1e-9
    h.close()


def test_band_to_tridiag_b1_is_identity():
    import torch

    n = 100
    ab = _random_band(n, 1, 3)
    h = _handle()
    d, e = h.band_to_tridiag(torch.from_numpy(ab).cuda())
    assert np.array_equal(d.cpu().numpy(), ab[:, 0].astype(np.float64))
    assert np.array_equal(e.cpu().numpy(), ab[: n - 1, 1].astype(np.float64))
    h.close()


def test_band_eigenvalues_of_diagonal_band():
    """All off-diagonals zero: no reflector anywhere (tau = 0), eigenvalues = sorted diagonal."""
    import torch

    n, b = 300, 16
    ab = np.zeros((n, b + 1), dtype=np.float32)
    ab[:, 0] = np.random.default_rng(1).uniform(-3, 3, n).astype(np.float32)
    h = _handle()
    lam = h.band_eigenvalues(torch.from_numpy(ab).cuda()).cpu().numpy()
    assert np.max(np.abs(lam - np.sort(ab[:, 0].astype(np.float64)))) <= 1e-14 * 3
    h.close()


@pytest.mark.parametrize("n,b,nb,mode,gate", [(2048, 32, 256, "3xtf32", 1e-5), (3000, 32, 512, "fp16", 1e-3),
                                              (4096, 64, 1024, "fp16", 1e-3)])
def test_eigenvalues_pipeline(n, b, nb, mode, gate):
    """A -> sbr_reduce -> band -> GPU stage two, against eigvalsh(A) in fp64 (P:421 metric)."""
    import torch

    import workloads

    a_host = workloads.random_symmetric(n, 31 + n)
    ref = np.linalg.eigvalsh(a_host.astype(np.float64))
    h = _handle()
    a = torch.from_numpy(a_host).cuda()
    lam = h.eigenvalues(a, b, nb, mode=mode).cpu().numpy()
    h.sync()
    err = np.max(np.abs(lam - ref)) / np.max(np.abs(ref))
    # stage two alone on the same band in fp64 on the host: the GPU stage two adds ~nothing
    a2 = torch.from_numpy(a_host).cuda()
    ab, _ = h.reduce(a2, b, nb, mode=mode, want_w=False)
    lam_b = np.linalg.eigvalsh(_band_dense(ab.cpu().numpy()))
    lam2 = h.band_eigenvalues(ab).cpu().numpy()
    err2 = np.max(np.abs(lam2 - lam_b)) / np.max(np.abs(ref))
    print(f"eigenvalues n={n} b={b} {mode}: |lam - eig(A)| {err:.2e}; stage two vs eig(B) {err2:.1e}")
    assert err <= gate
    assert err2 <= 1e-11
    h.close()


def test_stage2_argument_errors():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    h = _handle()
    lib = _lib.lib()
    ab = torch.zeros((10, 3), dtype=torch.float32, device="cuda")
    d = torch.zeros(10, dtype=torch.float64, device="cuda")
    assert lib.sbr_band_to_tridiag(h._h, 10, 2, ab.data_ptr(), 2, d.data_ptr(), d.data_ptr()) == -5
    assert lib.sbr_band_to_tridiag(h._h, 10, 65, ab.data_ptr(), 66, d.data_ptr(), d.data_ptr()) == -3
    assert lib.sbr_band_to_tridiag(h._h, 10, 2, ab.data_ptr(), 3, None, d.data_ptr()) == -6
    assert lib.sbr_tridiag_eigenvalues(h._h, 10, d.data_ptr(), None, d.data_ptr()) == -4
    assert lib.sbr_tridiag_eigenvalues(h._h, 0, None, None, None) == 0
    assert lib.sbr_eigenvalues(h._h, 0, 64, 8, 32, ab.data_ptr(), 64, None) == -8
    assert sbr.SbrError is not None
    h.close()
