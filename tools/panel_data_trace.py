"""Standalone CholeskyQR panel (sbr_test_panel) phase stamps on randn data vs the first panel of the
config-4 input (rows [b, n) of columns [0, b) of a U[-1,1) symmetric matrix), same m and ld."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib
n = 32768; b = 32; m = n - b
names = ["start", "loaded", "gram0", "wait0", "chol0", "solve0", "gram1", "LU", "wait1", "checked", "LUread", "end"]
h = sbr.Handle(0); lib = _lib.lib()
g = torch.Generator(device="cuda").manual_seed(1)
A0 = torch.rand(b, n, device="cuda", generator=g) * 2 - 1          # columns 0..b-1 (column-major)
cases = {"randn": torch.randn(b, n, device="cuda"), "uniform": A0, "uniform*1e-3": A0 * 1e-3,
         "randn_rows_b..": torch.randn(b, n, device="cuda")}
Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
for name, P0 in cases.items():
    tr = (ctypes.c_int64 * 16)()
    res = []
    for rep in range(5):
        P = P0.clone()
        _lib.check(lib.sbr_test_panel(h._h, m, b, P.data_ptr() + 4 * b, n, Y.data_ptr(), W.data_ptr(), m, tr), "panel")
        t = np.array([tr[i] for i in range(12)], dtype=np.float64)
        res.append(np.diff(t) / 1e3)
    md = np.median(np.array(res), axis=0)
    print(f"{name:14s} " + " ".join(f"{names[i]}->{names[i+1]}={md[i]:.1f}" for i in range(11)) + f" total {md.sum():.1f}", flush=True)
h.close()
