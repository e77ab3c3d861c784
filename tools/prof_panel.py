"""Run the panel step (a1-a2) a few times at one size (for ncu): python tools/prof_panel.py m b."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import __graft_entry__; __graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib
m = int(sys.argv[1]) if len(sys.argv) > 1 else 32000
b = int(sys.argv[2]) if len(sys.argv) > 2 else 32
h = sbr.Handle(0)
P0 = torch.randn(b, m, device="cuda")
Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
for _ in range(3):
    P = P0.clone()
    _lib.check(_lib.lib().sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, None), "panel")
torch.cuda.synchronize()
print("done")
