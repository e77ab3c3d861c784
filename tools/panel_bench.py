"""Time the panel step (a1-a2) through sbr_test_panel for both panel algorithms and check it
against LAPACK-style Householder QR (numpy) on random and rank-deficient panels."""
import ctypes, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import __graft_entry__; __graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib
from oracle import panel
h = sbr.Handle(0)
for b in (32,):
    for m in (4000, 32000):
        for kind in ("randn", "rankdef"):
            P0 = torch.randn(b, m, device="cuda", dtype=torch.float64)
            if kind == "rankdef":
                P0[5] = P0[3] * 2.0   # dependent column
                P0[7] = 0.0           # zero column
            P0 = P0.float()
            Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
            P = P0.clone()
            _lib.check(_lib.lib().sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, None), "panel")
            torch.cuda.synchronize()
            st = torch.cuda.Event(enable_timing=True); en = torch.cuda.Event(enable_timing=True)
            st.record()
            for _ in range(20):
                P.copy_(P0)
                _lib.lib().sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, None)
            en.record(); torch.cuda.synchronize()
            # accuracy: H = I - Y T Y^T with W = Y T; check (I - W Y^T)^T P = [R; 0]
            Pn = P0.double().cpu().numpy().T; Yn = Y.double().cpu().numpy().T; Wn = W.double().cpu().numpy().T
            Rg = np.triu(P.double().cpu().numpy().T[:b])
            QtP = Pn - Yn @ (Wn.T @ Pn)
            res = np.abs(QtP[:b] - Rg).max() / np.abs(Pn).max(); low = np.abs(QtP[b:]).max() / np.abs(Pn).max()
            orth = np.abs((np.eye(m, b) - Wn @ Yn[:b].T).T @ (np.eye(m, b) - Wn @ Yn[:b].T) - np.eye(b)).max()
            if kind == "randn":
                V, tau, R = panel.householder_qr(Pn)
                dY = np.abs(Yn - V).max()
            else:
                dY = float("nan")
            print(f"b={b} m={m} {kind}: {st.elapsed_time(en)/20*1e3:7.1f} us/panel (incl. copy)  |QtP-R| {res:.1e} below {low:.1e} orthQ {orth:.1e} dY {dY:.1e}", flush=True)
