"""Where does the 3xTF32 mode's error come from?  (VERDICT r1 weak item 3.)  Runs the same inputs
through (a) the tensor-core 3xTF32 reduction, (b) the same with the SIMT fp32 pass in place of
the tcgen05 3xTF32 pass (test knob 1), (c) the all-SIMT fp32 reduction (SBR_TF32_TC=0), and
prints backward error, orthogonality and eigenvalue error against fp64 eigvalsh.  Diagnostic."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import __graft_entry__
__graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib
import workloads
from gpu_helpers import invariants_torch

lib = _lib.lib()
h_tc = sbr.Handle(0)
os.environ["SBR_TF32_TC"] = "0"
h_simt = sbr.Handle(0)
del os.environ["SBR_TF32_TC"]
for n, b, nb in ((256, 8, 32), (1024, 32, 128), (2048, 32, 256), (4096, 32, 256)):
    a = workloads.random_symmetric(n, workloads.config_seed(1) + n)
    lam_ref = np.linalg.eigvalsh(a.astype(np.float64))
    norm2 = float(np.max(np.abs(lam_ref)))
    for name, h, kn in (("tc", h_tc, 0), ("tc+simt-pass", h_tc, 1), ("all-simt", h_simt, 0)):
        _lib.check(lib.sbr_test_set_knob(1, kn), "knob")
        A = torch.from_numpy(a).cuda()
        ab, w = h.reduce(A, b, nb, mode="3xtf32")
        torch.cuda.synchronize()
        eb, eo, lam, _ = invariants_torch(a, A, ab, w, n, b, nb)
        ee = float(np.max(np.abs(np.sort(lam) - lam_ref))) / norm2
        print(f"n={n} b={b} nb={nb} {name:13s}: backward {eb:.2e} orth {eo:.2e} eig {ee:.2e}", flush=True)
_lib.check(lib.sbr_test_set_knob(1, 0), "knob")
