"""One sbr_reduce on the bench workload, for ncu captures (no timing here)."""
import argparse, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768); ap.add_argument("--b", type=int, default=32)
ap.add_argument("--nb", type=int, default=1024); ap.add_argument("--mode", default="fp16")
ap.add_argument("--reps", type=int, default=1)
a = ap.parse_args()
import __graft_entry__; __graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr, workloads
h = sbr.Handle(0)
pr = h.generate_symmetric(workloads.config_seed(4), a.n)
A = torch.empty_like(pr)
for _ in range(a.reps):
    A.copy_(pr)
    h.reduce(A, a.b, a.nb, mode=a.mode)
torch.cuda.synchronize()
print("done")
