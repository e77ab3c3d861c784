"""GPU parity of sbr_form_q: the explicit Q = prod_J (I - W_J Y_J^T)
built on tcgen05 (3xTF32) from sbr_reduce's outputs, against

  * the oracle's fp64 product of the SAME (W, Y) blocks (oracle.metrics.q_from_blocks) --
    entry-wise, |dQ| <= 2e-5 (FP32-accurate products over K <= n terms of |Q| <= 1 entries);
  * invariants: ||Q^T Q - I||_F / sqrt(n) and ||A - Q B Q^T||_F / ||A||_F within the mode's
    gates (the same gates as the reduction, BASELINE.json);
  * in 3xTF32 mode, the oracle's own Q (unblocked Householder, fp64) within 1e-4 -- Q is
    unique given reading C1.
"""
import numpy as np
import pytest

import workloads
from oracle import metrics
from oracle import sbr as osbr

pytestmark = pytest.mark.gpu

TOL = {"fp16": 5e-3, "3xtf32": 1e-5}


@pytest.mark.parametrize("mode", ["fp16", "3xtf32"])
@pytest.mark.parametrize("n,b,nb", [(256, 8, 32), (300, 8, 32), (1000, 32, 128), (1024, 64, 128), (96, 32, 32),
                                    (40, 32, 32), (2048, 32, 256)])
def test_form_q(n, b, nb, mode):
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    a = workloads.random_symmetric(n, workloads.config_seed(1) + 3 * n + b)
    h = sbr.Handle(0)
    A = torch.from_numpy(a).cuda()
    ab, w = h.reduce(A, b, nb, mode=mode)
    q = h.form_q(A, w, b, nb)
    torch.cuda.synchronize()
    q_gpu = q.cpu().numpy().T.astype(np.float64)
    a_out = A.cpu().numpy().T
    w_out = w.cpu().numpy().T
    q_ref = metrics.q_from_blocks(n, b, metrics.blocks_from_output(a_out, w_out, n, b, nb))
    dq = np.abs(q_gpu - q_ref).max()
    bmat = sbr.band_to_dense(ab.double()).cpu().numpy()
    eo = metrics.orthogonality(q_gpu)
    eb = metrics.backward_error(a, q_gpu, bmat)
    msg = f"form_q n={n} b={b} nb={nb} {mode}: |Q - Q_blocks| {dq:.2e} orth {eo:.2e} backward {eb:.2e}"
    if mode == "3xtf32":
        q_or = osbr.sbr_unblocked(a, b, want_q=True)["Q"]
        dqo = np.abs(q_gpu - q_or).max()
        msg += f" |Q - Q_oracle| {dqo:.2e}"
    print(msg)
    assert dq <= 2e-5
    assert eo <= TOL[mode] and eb <= TOL[mode]
    if mode == "3xtf32":
        assert dqo <= 1e-4
    h.close()


def test_form_q_errors():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    h = sbr.Handle(0)
    x = torch.zeros((64, 64), device="cuda")
    L = _lib.lib()
    p = x.data_ptr()
    assert L.sbr_form_q(None, 64, 8, 32, p, 64, p, 64, p, 64) == -1
    assert L.sbr_form_q(h._h, 0, 8, 32, p, 64, p, 64, p, 64) == -2
    assert L.sbr_form_q(h._h, 64, 0, 32, p, 64, p, 64, p, 64) == -3
    assert L.sbr_form_q(h._h, 64, 8, 12, p, 64, p, 64, p, 64) == -4
    assert L.sbr_form_q(h._h, 64, 8, 32, None, 64, p, 64, p, 64) == -5
    assert L.sbr_form_q(h._h, 64, 8, 32, p, 63, p, 64, p, 64) == -6
    assert L.sbr_form_q(h._h, 64, 8, 32, p, 64, None, 64, p, 64) == -7
    assert L.sbr_form_q(h._h, 64, 8, 32, p, 64, p, 64, None, 64) == -9
    # n <= b + 1: Q = I
    q = torch.full((8, 8), 7.0, device="cuda")
    _lib.check(L.sbr_form_q(h._h, 8, 8, 8, p, 8, p, 8, q.data_ptr(), 8), "form_q trivial")
    assert torch.equal(q.cpu(), torch.eye(8))
    h.close()


@pytest.mark.parametrize("mode", ["fp16", "3xtf32"])
@pytest.mark.parametrize("n,b,nb", [(300, 8, 32), (1000, 32, 128), (2048, 32, 256), (1024, 64, 128), (96, 32, 32)])
def test_form_w_and_apply_q(n, b, nb, mode):
    """Alg. 2 (sbr_form_w) vs the oracle's Alg. 2 on the SAME blocks, entry-wise; X <- Q X
    (sbr_apply_q) vs the oracle product of the blocks times X."""
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from oracle import backtransform

    a = workloads.random_symmetric(n, 71 * n + b)
    h = sbr.Handle(0)
    A = torch.from_numpy(a).cuda()
    ab, w = h.reduce(A, b, nb, mode=mode)
    wm = h.form_w(A, w, b, nb)
    X0 = np.random.default_rng(n).standard_normal((16, n)).astype(np.float32)   # torch (kx, n) = column-major n x kx
    X = torch.from_numpy(X0).cuda()
    h.apply_q(A, w, b, nb, X)
    torch.cuda.synchronize()
    blocks = metrics.blocks_from_output(A.cpu().numpy().T, w.cpu().numpy().T, n, b, nb)
    W_ref, Y_ref = backtransform.form_w(n, b, blocks)
    dw = np.abs(wm.cpu().numpy().T.astype(np.float64) - W_ref).max() / max(1.0, np.abs(W_ref).max())
    qx_ref = backtransform.apply_q(W_ref, Y_ref, X0.T.astype(np.float64))
    dx = np.abs(X.cpu().numpy().T - qx_ref).max() / np.abs(qx_ref).max()
    print(f"form_w/apply_q n={n} b={b} nb={nb} {mode}: |W - W_Alg2| {dw:.2e} |QX - QX_ref| {dx:.2e}")
    assert dw <= 5e-5
    assert dx <= 2e-5
