"""Experiment: why is the CholeskyQR panel slower inside sbr_reduce than standalone?
Times the standalone panel (m = 32000, b = 32, ld 32768) with its phase stamps (a) warm,
(b) right after a 1 GiB device read sweep (evicts L2 data and TLB entries, as the pass does),
(c) after a 1 GiB sweep over the SAME 2 MiB pages re-read (L2 evicted, pages few: TLB warm-ish).
Diagnostic only."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import __graft_entry__
__graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib

names = ["start", "loaded", "gram0", "wait0", "chol0", "solve0", "gram1", "LU", "wait1", "checked", "LUread", "end"]
h = sbr.Handle(0)
lib = _lib.lib()
n, m, b = 32768, 32000, 32
P0 = torch.randn(b, n, device="cuda")
Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
big = torch.empty(1 << 28, device="cuda")          # 1 GiB, 512 pages of 2 MiB
small = torch.empty(1 << 22, device="cuda")        # 16 MiB: 8 pages
mid = torch.empty(40 << 20, device="cuda")         # 160 MiB: 80 pages, more than the 126 MB L2
tlb_idx = torch.arange(0, 1 << 28, 1 << 19, device="cuda")   # one float per 2 MiB page of big
sink = torch.empty(1, device="cuda")

def run(pre):
    out = []
    for rep in range(5):
        P = P0.clone()
        if pre == "sweep":
            torch.sum(big, out=sink[0:1].view(())) if False else big.sum()
        elif pre == "l2only":
            for _ in range(64):
                small.sum()
        elif pre == "write":
            big.fill_(1.0)
        elif pre == "l2sweep":   # evicts the L2 through 80 pages only
            mid.sum()
        elif pre == "tlbsweep":  # touches 512 pages, one 4-byte load each: TLB churn, L2 intact
            big.index_select(0, tlb_idx).sum()
        tr = (ctypes.c_int64 * 16)()
        _lib.check(lib.sbr_test_panel(h._h, m, b, P.data_ptr(), n, Y.data_ptr(), W.data_ptr(), m, tr), "panel")
        t = np.array([tr[i] for i in range(16)], dtype=np.float64)
        out.append(t)
    t = np.median(np.stack(out[1:]), axis=0)
    r = (t[:12] - t[0]) / 1e3
    print(f"{pre:8s}: " + " ".join(f"{names[i]}->{names[i+1]}={r[i+1]-r[i]:.1f}" for i in range(11)) + f" total {r[11]:.1f}")

for pre in ("warm", "sweep", "l2sweep", "tlbsweep", "write", "warm"):
    run(pre)
h.close()
