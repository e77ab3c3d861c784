import sys, os
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import numpy as np, torch, workloads
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
n, b, nb, mode = [int(x) if x.isdigit() else x for x in sys.argv[1:5]]
h = sbr.Handle(0)
a = torch.from_numpy(workloads.random_symmetric(n, 3)).cuda()
h.reduce(a, b, nb, mode=mode)
h.sync()
print("ok", n, b, nb, mode)
