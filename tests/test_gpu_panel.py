"""GPU parity of the panel factorisation (steps a1-a2: CholeskyQR / TSQR + Householder
reconstruction, reading R1) through sbr_test_panel, against the definition:

  * R_h (upper b x b of the compact panel) equals LAPACK dgeqrf's R (numpy.linalg.qr, reading C1)
    entry-wise within 2e-5 relative to ||P||;
  * Q^T P = [R_h; 0] with Q = I - W Y^T, in fp64 on the device's fp32 outputs (residual <= 1e-5 ||P||);
  * Q is orthogonal: probe vectors keep their norm and Q Q^T x = x (<= 1e-5);
  * Y is unit lower trapezoidal and its tail is what the compact panel stores.
Cases span the TSQR-only sizes, CholeskyQR with resident rows, and the STREAMED CholeskyQR for
panels taller than 148 CTAs x the shared-memory row capacity (m > 75776 at b = 32, m > 18944 at
b = 64), which is what config 5 (n = 65536, b = 64) needs.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _rank_deficient(m, b, kind, rng):
    """Panels CholeskyQR must decline: exact zero columns, duplicated columns, exact zeros."""
    p0 = rng.uniform(-1, 1, (m, b)).astype(np.float32)
    if kind == "dup":          # columns b/2.. repeat the first half: rank b/2, Gram singular
        p0[:, b // 2:] = p0[:, : b - b // 2]
    elif kind == "zerocols":   # every third column zero
        p0[:, ::3] = 0.0
    elif kind == "zero":       # the already-banded case: the whole panel is zero (tau = 0, H = I)
        p0[:] = 0.0
    return p0


@pytest.mark.parametrize("m,b", [(300, 32), (1000, 8), (2000, 16), (4000, 32), (4000, 64), (33000, 32),
                                 (80000, 32), (20000, 64), (65472, 64)])
def test_panel_vs_dgeqrf(m, b):
    _check_panel(m, b, np.random.default_rng(m + b).uniform(-1, 1, (m, b)).astype(np.float32), m + b, declines=0)


@pytest.mark.parametrize("m,b,kind", [(1000, 32, "dup"), (4000, 32, "zerocols"), (4000, 64, "dup"),
                                      (2000, 16, "zero"), (33000, 32, "dup"), (80000, 32, "zerocols"),
                                      (65472, 64, "dup"), (65472, 64, "zero")])
def test_panel_fallback(m, b, kind):
    """CholeskyQR declines (singular Gram) and the same kernel factors the panel by Householder
    QR (dgeqr2 order, dlarfg sign convention C1), at any height -- including the streamed
    panels beyond the shared-memory row capacity (80000 x 32, 65472 x 64: config 5's tallest),
    which the paper's TSQR tree (148 x 256-row leaves) cannot hold.  Same gates as above: R
    against dgeqrf, Q^T P = [R; 0], orthogonality, Y structure."""
    rng = np.random.default_rng(7 * m + b)
    _check_panel(m, b, _rank_deficient(m, b, kind, rng), m + b, declines=1)


def _check_panel(m, b, p0, seed, declines):
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(seed)
    h = sbr.Handle(0)
    h.panel_declines(reset=True)
    P = torch.from_numpy(np.ascontiguousarray(p0.T)).cuda()        # column-major m x b
    Y = torch.zeros((b, m), device="cuda")
    W = torch.zeros((b, m), device="cuda")
    _lib.check(_lib.lib().sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, None), "panel")
    pc = P.cpu().numpy().T.astype(np.float64)
    y = Y.cpu().numpy().T.astype(np.float64)
    w = W.cpu().numpy().T.astype(np.float64)
    a = p0.astype(np.float64)
    nrm = max(np.linalg.norm(a), 1.0)
    r_h = np.triu(pc[:b])
    r_ref = np.linalg.qr(a, mode="r")
    dr = np.abs(r_h - r_ref).max() / nrm
    # Q^T P = P - Y (W^T P)
    qtp = a - y @ (w.T @ a)
    res = max(np.abs(qtp[:b] - r_h).max(), np.abs(qtp[b:]).max()) / nrm
    # orthogonality on probes: Q^T x (norm), Q (Q^T x) = x
    x = rng.standard_normal((m, 4))
    qt = x - y @ (w.T @ x)
    back = qt - w @ (y.T @ qt)
    eo = max(np.abs(np.linalg.norm(qt, axis=0) / np.linalg.norm(x, axis=0) - 1).max(),
             np.abs(back - x).max() / np.abs(x).max())
    # Y structure and the compact panel's tail
    ys = np.abs(np.triu(y[:b], 1)).max() + np.abs(np.diag(y[:b]) - 1).max()
    tail = np.abs(np.tril(pc, -1) - np.tril(y, -1)).max()
    print(f"panel m={m} b={b}: |R - R_dgeqrf| {dr:.1e}  |Q^T P - [R;0]| {res:.1e}  orth {eo:.1e}  Y {ys:.0e} tail {tail:.0e}")
    assert dr <= 2e-5 and res <= 1e-5 and eo <= 1e-5
    assert ys == 0.0 and tail == 0.0
    if m > 512:   # the CholeskyQR kernel ran (TSQR below): declined exactly when expected
        assert h.panel_declines(reset=True) == declines
    h.close()
