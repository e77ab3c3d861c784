"""One reduction + sbr_form_q at n (3xTF32), for ncu launch lists of form_q."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
ap = argparse.ArgumentParser(); ap.add_argument("--n", type=int, default=16384); ap.add_argument("--nb", type=int, default=1024)
a = ap.parse_args()
import __graft_entry__; __graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr, workloads
h = sbr.Handle(0)
A = h.generate_symmetric(workloads.config_seed(3), a.n)
ab, w = h.reduce(A, 32, a.nb, mode="3xtf32")
q = h.form_q(A, w, 32, a.nb)
torch.cuda.synchronize()
print("done")
