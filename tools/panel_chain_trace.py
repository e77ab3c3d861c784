"""Phase stamps of the CholeskyQR panel kernel INSIDE sbr_reduce (config 4 by default), next to
the same kernel run standalone (sbr_test_panel) on a panel of the same m and leading dimension.
Stamps (CTA 0, globaltimer ns): 0 start (before the PDL wait), 1 rows loaded, 2 Gram-0 arrive,
3 barrier-0 passed, 4 chol-0, 5 solve-0, 6 Gram-1 arrive, 7 speculative LU done, 8 barrier-1 passed,
9 check passed, 10 LU read, 11 outputs written."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import __graft_entry__
__graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib

n = int(os.environ.get("N", 32768)); b = 32; nb = 1024
names = ["start", "loaded", "gram0", "wait0", "chol0", "solve0", "gram1", "LU", "wait1", "checked", "LUread", "end"]
h = sbr.Handle(0)
g = torch.Generator(device="cuda").manual_seed(1)
A0 = torch.rand(n, n, device="cuda", generator=g) * 2 - 1
A0 = torch.tril(A0) + torch.tril(A0, -1).T
A = A0.clone(); h.reduce(A, b, nb, mode="fp16"); torch.cuda.synchronize()   # warm-up (allocation)
npan = (n - b + b - 1) // b
lib = _lib.lib()
_lib.check(lib.sbr_test_panel_trace(h._h, npan + 8, None, None), "arm")
A = A0.clone(); torch.cuda.synchronize()
h.reduce(A, b, nb, mode="fp16")
buf = (ctypes.c_int64 * (32 * (npan + 8)))(); cnt = ctypes.c_int(0)
_lib.check(lib.sbr_test_panel_trace(h._h, 0, buf, ctypes.byref(cnt)), "read")
T = np.frombuffer(buf, dtype=np.int64)[: 32 * cnt.value].reshape(cnt.value, 32)[:, :12].astype(np.float64)
print(f"n={n}: {cnt.value} CholeskyQR panels traced")
rel = (T - T[:, :1]) / 1e3
rel[T == 0] = np.nan
d = np.diff(np.where(np.isnan(rel), np.nan, rel), axis=1)
for lo, hi in ((0, 32), (480, 512), (960, 992)):
    if hi <= cnt.value:
        md = np.nanmedian(d[lo:hi], axis=0)
        print(f"panels {lo}-{hi}: total {np.nanmedian(rel[lo:hi, 11]):.1f} us; " +
              " ".join(f"{names[i]}->{names[i+1]}={md[i]:.1f}" for i in range(11)))
# output phase detail (stamps 12-15): factor tables, thread 0's first row W / Y, all rows, rows above
T2 = np.frombuffer(buf, dtype=np.int64)[: 32 * cnt.value].reshape(cnt.value, 32)[:, :16].astype(np.float64)
o = T2[:, [10, 12, 13, 14, 15, 11]]
o[o <= 0] = np.nan
if True:
    do = np.diff(o, axis=1) / 1e3
    for lo, hi in ((0, 32), (480, 512), (960, 992)):
        if hi <= cnt.value:
            md = np.nanmedian(do[lo:hi], axis=0)
            print(f"  output phase {lo}-{hi}: tables {md[0]:.1f} row0-W {md[1]:.1f} row0-Y {md[2]:.1f} "
                  f"other rows {md[3]:.1f} rows-above {md[4]:.1f} us")
gap = (T[1:, 0] - T[:-1, 11]) / 1e3
print(f"end(panel t) -> start(panel t+1): median {np.median(gap):.1f} us (the rest of the chain)")
for m in (32000, 16000, 4000):
    P0 = torch.randn(b, n, device="cuda")   # column-major m x b with ld n (rows [0, m) used)
    Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
    tr = (ctypes.c_int64 * 16)()
    for rep in range(3):
        P = P0.clone()
        _lib.check(lib.sbr_test_panel(h._h, m, b, P.data_ptr(), n, Y.data_ptr(), W.data_ptr(), m, tr), "panel")
    t = np.array([tr[i] for i in range(12)], dtype=np.float64)
    r = (t - t[0]) / 1e3
    print(f"standalone m={m}: " + " ".join(f"{names[i]}->{names[i+1]}={r[i+1]-r[i]:.1f}" for i in range(11)) + f" total {r[11]:.1f}")
h.close()
