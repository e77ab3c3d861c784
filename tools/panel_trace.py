"""Time one panel (a1-a2) at several m and print the kernel's phase timestamps."""
import ctypes, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import __graft_entry__; __graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib
h = sbr.Handle(0)
names = ["start", "loaded", "gram0", "wait0", "chol0", "solve0", "gram1", "LU(cta0)", "wait1", "checked", "LUread", "rows", "x12", "x13", "x14", "x15"]
for b in (32,):
    for m in (4000, 16000, 32000):
        P0 = torch.randn(b, m, device="cuda")   # column-major m x b
        Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
        tr = (ctypes.c_int64 * 16)()
        for rep in range(3):
            P = P0.clone()
            _lib.check(_lib.lib().sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, tr), "panel")
        t = [tr[i] for i in range(16)]
        rel = [(t[i] - t[0]) / 1e3 if t[i] else None for i in range(16)]
        st = torch.cuda.Event(enable_timing=True); en = torch.cuda.Event(enable_timing=True)
        P = P0.clone(); st.record()
        for _ in range(10):
            _lib.lib().sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, None)
        en.record(); torch.cuda.synchronize()
        print(f"b={b} m={m}: total {st.elapsed_time(en)/10*1e3:.1f} us/call ;", " ".join(f"{n}={r:.1f}" for n, r in sorted(zip(names, rel), key=lambda z: z[1] if z[1] is not None else 1e9) if r is not None), flush=True)
