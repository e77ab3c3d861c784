"""Run one reduction (debug): python tools/smallb.py n b nb mode [banded|rank8]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch, workloads
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from oracle import sbr as osbr
n, b, nb, mode = [int(x) if x.isdigit() else x for x in sys.argv[1:5]]
kind = sys.argv[5] if len(sys.argv) > 5 else "uniform"
a = workloads.random_symmetric(n, 3)
if kind == "banded":
    a = osbr.band_part(a.astype(np.float64), b).astype(np.float32)
h = sbr.Handle(0)
t = torch.from_numpy(a).cuda()
ab, w = h.reduce(t, b, nb, mode=mode)
h.sync()
print("ok", n, b, nb, mode, kind, "declines", h.panel_declines(), "finite", bool(torch.isfinite(ab).all()))
