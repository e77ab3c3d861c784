"""Stage two timing on one B200: the two-stage eigenvalue pipeline
(sbr_reduce -> sbr_band_to_tridiag -> sbr_tridiag_eigenvalues) against torch.linalg.eigvalsh
(cuSOLVER syevd) on the same matrix.  Prints one JSON line per n.

    python tools/stage2_bench.py [--n 4096 8192 16384 32768] [--b 32] [--nb 1024] [--mode fp16]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, nargs="+", default=[4096, 8192, 16384, 32768])
    ap.add_argument("--b", type=int, default=32)
    ap.add_argument("--nb", type=int, default=1024)
    ap.add_argument("--mode", default="fp16")
    ap.add_argument("--cusolver-max", type=int, default=32768)
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    st = torch.cuda.Stream()
    h = sbr.Handle(0, stream=st)
    for n in args.n:
        b, nb = args.b, args.nb
        with torch.cuda.stream(st):
            a0 = h.generate_symmetric(1234 + n, n)
            a = torch.empty_like(a0)
            ab = torch.empty((n, b + 1), dtype=torch.float32, device="cuda")
            d = torch.empty(n, dtype=torch.float64, device="cuda")
            e = torch.empty(n - 1, dtype=torch.float64, device="cuda")
            lam = torch.empty(n, dtype=torch.float64, device="cuda")
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            best = None
            for rep in range(args.reps + 1):
                a.copy_(a0)
                st.synchronize()
                ev[0].record(st)
                h.reduce(a, b, nb, mode=args.mode, want_w=False, ab=ab)
                ev[1].record(st)
                h.band_to_tridiag(ab, d, e)
                ev[2].record(st)
                h.tridiag_eigenvalues(d, e, lam)
                ev[3].record(st)
                h.sync()
                t = [ev[i].elapsed_time(ev[i + 1]) for i in range(3)]
                if rep > 0 and (best is None or sum(t) < sum(best)):
                    best = t
            ours = lam.clone()
        rec = {"n": n, "b": b, "nb": nb, "mode": args.mode, "ms_reduce": round(best[0], 2),
               "ms_band_to_tridiag": round(best[1], 2), "ms_bisection": round(best[2], 2),
               "ms_total": round(sum(best), 2)}
        if n <= args.cusolver_max:
            torch.cuda.synchronize()
            ref = None
            tb = None
            for rep in range(2 if n > 16384 else 3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.copy_(a0)
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                e0.record()
                ref = torch.linalg.eigvalsh(a)
                e1.record()
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1)
                if rep > 0 or n > 16384:
                    tb = ms if tb is None else min(tb, ms)
            rec["ms_cusolver_eigvalsh_fp32"] = round(tb, 2)
            rec["speedup_vs_cusolver"] = round(tb / sum(best), 2)
            rel = (ours - ref.double()).abs().max().item() / ref.double().abs().max().item()
            rec["max_rel_diff_vs_cusolver"] = float(f"{rel:.3e}")
        print(json.dumps(rec), flush=True)
        del a0, a
        torch.cuda.empty_cache()
    h.close()


if __name__ == "__main__":
    main()
