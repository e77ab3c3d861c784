"""SYR2K tile raster: band height H (tile rows per band, test knob 2) at config 4.  Each line:
H, ms per reduction (CUDA events, A re-copied from the pristine input before each rep, not timed).
Diagnostic only (the library default is H = 64 for the FP16 128 x 256 tiles)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import __graft_entry__
__graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib
import workloads

n, b, nb = 32768, 32, 1024
h = sbr.Handle(0)
lib = _lib.lib()
pr = h.generate_symmetric(workloads.config_seed(4), n)
A = torch.empty_like(pr)
for H in [0, 16, 32, 64, 128, 256, 0]:
    _lib.check(lib.sbr_test_set_knob(2, H), "knob")
    ts = []
    for rep in range(4):
        A.copy_(pr)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); h.reduce(A, b, nb, mode="fp16"); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts = sorted(ts[1:])
    print(f"H={H if H else 'default(64)'}: {ts[len(ts)//2]:.2f} ms (min {ts[0]:.2f})", flush=True)
_lib.check(lib.sbr_test_set_knob(2, 0), "knob")
