"""Helpers for the GPU parity tests: run sbr_reduce through the C ABI and turn its
output into (B, Q) for the invariant checks.  Test infrastructure only."""
from __future__ import annotations

import numpy as np


def run_reduce(a_host: np.ndarray, b: int, nb: int, mode: str, handle=None):
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    h = handle or sbr.Handle(0)
    a = torch.from_numpy(np.ascontiguousarray(a_host, dtype=np.float32)).cuda()
    ab, w = h.reduce(a, b, nb, mode=mode)
    torch.cuda.synchronize()
    return a, ab, w


def sign_normalise(bmat: np.ndarray, b: int) -> np.ndarray:
    """D B D with D = diag(+-1) making every outermost band entry B[i, i-b] >= 0.

    TSQR reconstruction may pick H = I - 2 e e^T where dlarfg picks H = I (reading C1);
    the two B differ exactly by such a D, so normalised bands are comparable."""
    n = bmat.shape[0]
    d = np.ones(n)
    for i in range(b, n):
        s = np.sign(bmat[i, i - b])
        d[i] = (s if s != 0 else 1.0) * d[i - b]
    return d[:, None] * bmat * d[None, :]


def q_from_output_torch(a_dev, w_dev, n: int, b: int, nb: int):
    """Q = prod_J (I - W_J Y_J^T) from the device outputs, in fp64 on the GPU."""
    import torch

    acm = a_dev.double().T       # column-major view -> natural indexing A[i, j]
    wcm = w_dev.double().T
    q = torch.eye(n, dtype=torch.float64, device=a_dev.device)
    ncols = n - b
    rows = torch.arange(n, device=a_dev.device)
    for c0 in range(0, ncols, nb):
        k = min(nb, ncols - c0)
        r0 = c0 + b
        y = acm[r0:, c0:c0 + k].clone()
        # unit at local row jj for column jj, zeros above, tail below (from A)
        jj = torch.arange(k, device=a_dev.device)
        rr = rows[: n - r0, None]
        y = torch.where(rr > jj[None, :], y, torch.zeros_like(y))
        y[jj, jj] = 1.0
        wj = wcm[r0:, c0:c0 + k]
        q[:, r0:] -= (q[:, r0:] @ wj) @ y.T
    return q


def invariants_torch(a_host: np.ndarray, a_dev, ab, w, n: int, b: int, nb: int):
    """(backward error, orthogonality, eigenvalues of B ascending) in fp64 on the GPU."""
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    q = q_from_output_torch(a_dev, w, n, b, nb)
    bm = sbr.band_to_dense(ab.double())
    a64 = torch.from_numpy(np.asarray(a_host, dtype=np.float64)).cuda()
    a64 = torch.tril(a64) + torch.tril(a64, -1).T
    eb = (torch.linalg.norm(a64 - q @ bm @ q.T) / torch.linalg.norm(a64)).item()
    eo = (torch.linalg.norm(q.T @ q - torch.eye(n, dtype=torch.float64, device=q.device)) / np.sqrt(n)).item()
    lam = torch.linalg.eigvalsh(bm).cpu().numpy()
    return eb, eo, lam, bm.cpu().numpy()
