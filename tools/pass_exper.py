"""Timing-only pass experiments (results invalid): config-4 reductions with the pass experiment knob
(include/sbr_testing.h knob 0) set to each value given, per-kernel-class device time per reduction.

    python tools/pass_exper.py 0 8 16 3
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    import workloads
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    vals = [int(v) for v in sys.argv[1:]] or [0]
    n, b, nb = 32768, 32, 1024
    st = torch.cuda.Stream()
    h = sbr.Handle(0, stream=st)
    with torch.cuda.stream(st):
        a0 = h.generate_symmetric(workloads.config_seed(4), n)
        a = torch.empty_like(a0)
        ab = torch.empty((n, b + 1), dtype=torch.float32, device="cuda")
    for v in vals:
        _lib.lib().sbr_test_set_knob(0, v)
        with torch.cuda.stream(st):
            a.copy_(a0)
            h.reduce(a, b, nb, want_w=False, ab=ab)   # warm-up
            h.sync()
            h.set_kernel_timing(True)
            h.reset_kernel_stats()
            reps = 2
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            tot = 0.0
            for _ in range(reps):
                a.copy_(a0)
                ev0.record(st)
                h.reduce(a, b, nb, want_w=False, ab=ab)
                ev1.record(st)
                h.sync()
                tot += ev0.elapsed_time(ev1)
            ks = {c: h.kernel_stats(c)["ms"] / reps for c in ("panel", "lazy", "wmerge", "pass", "syr2k", "other")}
            h.set_kernel_timing(False)
        print(f"exper={v}: {tot / reps:.1f} ms/reduction (events on)  " +
              "  ".join(f"{k} {x:.1f}" for k, x in ks.items()), flush=True)
    _lib.lib().sbr_test_set_knob(0, 0)
    h.close()


if __name__ == "__main__":
    main()
