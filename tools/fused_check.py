"""Quick A/B of the fused FP16 chain vs the per-kernel chain (SBR_FUSED=0 in a subprocess):
invariants (backward error, orthogonality, eigenvalues vs fp64) at a few sizes."""
import os, subprocess, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import torch

CASES = [(320, 32, 64), (1024, 32, 256), (2100, 32, 256), (4096, 32, 1024), (8192, 32, 1024)]


def run():
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    import workloads
    from gpu_helpers import invariants_torch, run_reduce

    h = sbr.Handle(0)
    for n, b, nb in CASES:
        a = workloads.random_symmetric(n, 1234 + n)
        t0 = time.time()
        h.panel_declines(reset=True)
        a_dev, ab, w = run_reduce(a, b, nb, "fp16", handle=h)
        try:
            h.sync()
            st = "ok"
        except Exception as e:  # noqa
            st = str(e)[:120]
        dec = h.panel_declines(reset=True)
        eb, eo, lam, _ = invariants_torch(a, a_dev, ab, w, n, b, nb)
        ref = torch.linalg.eigvalsh(torch.from_numpy(a.astype(np.float64)).cuda()).cpu().numpy()
        ee = np.max(np.abs(np.sort(lam) - ref)) / np.max(np.abs(ref))
        print(f"FUSED={os.environ.get('SBR_FUSED', '1')} n={n} b={b} nb={nb}: {st} declines {dec} "
              f"backward {eb:.2e} orth {eo:.2e} eig {ee:.2e} ({time.time() - t0:.1f}s)", flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1:
        run()
    else:
        for f in ("1", "0"):   # fused chain kernel vs the per-kernel chain
            env = dict(os.environ, SBR_FUSED=f)
            subprocess.run([sys.executable, __file__, "run"], env=env, timeout=600)
