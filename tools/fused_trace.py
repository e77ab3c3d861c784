"""Phase stamps of the fused chain kernel (k_chain_fused.cu) inside sbr_reduce, config 4 by default.
CTA 0's globaltimer stamps, printed in time order as segment durations (us, median over panels)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import __graft_entry__
__graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib

n = int(os.environ.get("N", 32768)); b = 32; nb = int(os.environ.get("NB", 1024))
NAMES = {25: "A.stage", 26: "A.part", 22: "B.stage", 23: "F.stage", 24: "F.comp", 0: "start", 1: "pdl", 2: "A", 3: "B", 4: "C", 5: "gram0", 6: "bar0", 15: "gread0", 16: "chol0",
         17: "rinv0", 18: "solve0", 7: "gram1", 19: "q1", 20: "lu", 8: "inv", 9: "bar1", 21: "gread1",
         10: "out", 11: "barW", 12: "E", 13: "F", 14: "end"}
ORDER = [0, 1, 25, 26, 2, 22, 3, 4, 5, 6, 15, 16, 17, 18, 7, 19, 20, 8, 9, 21, 10, 11, 12, 23, 24, 13, 14]
h = sbr.Handle(0)
A0 = h.generate_symmetric(20230229, n)
A = A0.clone(); h.reduce(A, b, nb, mode="fp16"); torch.cuda.synchronize()
npan = (n - b + b - 1) // b
lib = _lib.lib()
_lib.check(lib.sbr_test_panel_trace(h._h, npan + 8, None, None), "arm")
A = A0.clone(); torch.cuda.synchronize()
h.reduce(A, b, nb, mode="fp16")
buf = (ctypes.c_int64 * (32 * (npan + 8)))(); cnt = ctypes.c_int(0)
_lib.check(lib.sbr_test_panel_trace(h._h, 0, buf, ctypes.byref(cnt)), "read")
T = np.frombuffer(buf, dtype=np.int64)[: 32 * cnt.value].reshape(cnt.value, 32).astype(np.float64)
T[T == 0] = np.nan
T = T[:, ORDER]
print(f"n={n} nb={nb}: {cnt.value} fused launches traced")
tpb = nb // b
rows = {"t>=1 early": [i for i in range(1, 40) if i % tpb], "t>=1 mid": [i for i in range(480, 520) if i % tpb],
        "t>=1 late": [i for i in range(960, min(cnt.value, 1000)) if i % tpb],
        "t=0": [i for i in range(cnt.value) if i % tpb == 0]}
for label, sel in rows.items():
    sel = [i for i in sel if i < cnt.value]
    if not sel:
        continue
    R = T[sel] - T[sel][:, :1]
    segs = []
    for j in range(1, len(ORDER)):
        prev = np.nanmax(R[:, :j], axis=1)
        d = R[:, j] - prev
        md = np.nanmedian(d) if np.any(~np.isnan(d)) else np.nan
        if not np.isnan(md):
            segs.append(f"{NAMES[ORDER[j]]}={md / 1e3:.1f}")
    tot = np.nanmedian(np.nanmax(R, axis=1))
    print(f"{label}: total {tot / 1e3:.1f} us; " + " ".join(segs))
last = np.nanmax(T, axis=1)
gap = (T[1:, 0] - last[:-1]) / 1e3
print(f"end(launch i) -> start(launch i+1): median {np.nanmedian(gap):.1f} us (pass + launch)")
h.close()
