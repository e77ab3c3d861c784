import sys, numpy as np, torch
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
import workloads
from gpu_helpers import run_reduce, invariants_torch
for n, b, nb in [(264, 64, 64), (700, 64, 64), (1024, 64, 64), (1024, 64, 128), (700, 32, 32), (1024, 48, 96), (600, 40, 80)]:
    a = workloads.random_symmetric(n, 5)
    for mode in ["fp16"]:
        a_dev, ab, w = run_reduce(a, b, nb, mode)
        eb, eo, lam, bm = invariants_torch(a, a_dev, ab, w, n, b, nb)
        print(n, b, nb, mode, f"backward {eb:.2e} orth {eo:.2e}", flush=True)
