"""Probe the 3xTF32 pass kernel's two directions separately (M = 256: tiles (0,0), (1,0), (1,1))."""
import numpy as np
import torch

import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib

h = sbr.Handle(0)


def run(oa, w):
    M, b = w.shape
    d_oa = torch.from_numpy(np.ascontiguousarray(oa.T)).cuda()
    d_w = torch.from_numpy(np.ascontiguousarray(w.T)).cuda()
    d_x = torch.zeros((b, M), dtype=torch.float32, device="cuda")
    _lib.check(_lib.lib().sbr_test_pass_tf32(h._h, M, b, d_oa.data_ptr(), M, None, M, 0, d_w.data_ptr(), M,
                                            d_x.data_ptr(), M), "pass")
    return d_x.cpu().numpy().T.astype(np.float64)


rng = np.random.default_rng(1)
M, b = 256, 32
B = rng.uniform(-1, 1, (128, 128)).astype(np.float32)
W0 = rng.uniform(-1, 1, (128, b)).astype(np.float32)
Z = np.zeros((128, b), np.float32)
oa = np.zeros((M, M), np.float32)
oa[128:, :128] = B


def rep(name, got, cands):
    for cn, c in cands.items():
        print(f"  {name} vs {cn}: {np.abs(got - c).max():.3e}")


x = run(oa, np.vstack([W0, Z]))          # dir1 only: X_1 = B W0
print("dir1: |X0| =", np.abs(x[:128]).max())
rep("X1", x[128:], {"B W0": B @ W0, "B^T W0": B.T @ W0})
x = run(oa, np.vstack([Z, W0]))          # dir2 only: X_0 = B^T W0
print("dir2: |X1| =", np.abs(x[128:]).max())
rep("X0", x[:128], {"B^T W0": B.T @ W0, "B W0": B @ W0})
# diagonal tile only
D = rng.uniform(-1, 1, (128, 128)).astype(np.float32)
D = np.tril(D) + np.tril(D, -1).T
oa = np.zeros((128, 128), np.float32) + D
x = run(oa, W0)
rep("diag", x, {"D W0": D @ W0, "tril(D) W0": np.tril(D) @ W0, "2 tril(D,-1)+diag": (np.tril(D, -1) + np.tril(D, -1).T) @ W0})
x = run(np.eye(128, dtype=np.float32), W0)
rep("eye", x, {"W0": W0, "0.5 W0": 0.5 * W0})
# single entries
for (i, j) in [(5, 3), (40, 3), (100, 70), (3, 3)]:
    e = np.zeros((128, 128), np.float32); e[i, j] = 1; e[j, i] = 1
    x = run(e, W0)
    nz = np.argwhere(np.abs(x).max(axis=1) > 1e-6).ravel()
    print(f"entry ({i},{j}): nonzero X rows {nz[:10]}  X[i]~W0[j]? {np.abs(x[i] - W0[j]).max():.2e}  X[j]~W0[i]? {np.abs(x[j] - W0[i]).max():.2e}")
