import sys, numpy as np, torch
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
import workloads
from oracle import panel
from gpu_helpers import run_reduce
cases = [(64, m) for m in (400, 450, 520, 560, 700, 1000)] + [(48, 520), (48, 700), (32, 1100), (32, 1600), (32, 4000), (16, 1100)]
for b, m in cases:
    n = b + m
    a = workloads.random_symmetric(n, 5)
    a_dev, ab, w = run_reduce(a, b, b, "fp16")
    acm = a_dev.cpu().numpy().T.astype(np.float64)
    wcm = w.cpu().numpy().T.astype(np.float64)
    P = a.astype(np.float64)[b:, :b]
    V, tau, R = panel.householder_qr(P)
    T = panel.larft(V, tau)
    Y = np.tril(acm[b:, :b], -1) + np.eye(m, b)
    Wg = wcm[b:, :b]
    Rg = np.triu(acm[b:2*b, :b])
    d = np.abs(Y - V)
    bad = np.where(d.max(0) > 1e-3)[0]
    print(b, m, "dY %.1e dW %.1e dR %.1e" % (d.max(), np.abs(Wg - V @ T).max(), np.abs(Rg - R).max()), "badcols", bad[:3], flush=True)
