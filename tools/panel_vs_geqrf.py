"""SURVEY §8(f) f4 / paper Fig. 8: the panel factorisation against cuSOLVER's
Householder QR on the same tall-skinny panels, on the B200.

Rows: m x b fp32 panels (uniform [-1, 1)), b in {32, 64}, m from 4096 to 65536.
  * chol  -- this repo's default panel (CholeskyQR in fp64 + Householder reconstruction into
             Y, W = Y T and the compact [R; V] panel: everything the next SBR step needs);
  * tsqr  -- the paper's TSQR + reconstruction (SBR_PANEL=tsqr; capacity 148 leaves of 256 rows);
  * geqrf -- torch.geqrf (cuSOLVER sgeqrf): V and tau only, no T and no W = V T, so it is a
             LOWER bound on what one SBR panel step needs from cuSOLVER.
Times are CUDA-event medians over 20 repetitions after 3 warm-ups, one line of JSON per case."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import __graft_entry__
__graft_entry__.build()
import paper_conf_ppopp_zhangsoyw23_b200 as sbr
from paper_conf_ppopp_zhangsoyw23_b200 import _lib


def ev_time(fn, reps=20, warm=3):
    for _ in range(warm):
        fn()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def ours(h, m, b, P0, Y, W):
    lib = _lib.lib()
    P = P0.clone()
    def f():
        P.copy_(P0)
        _lib.check(lib.sbr_test_panel(h._h, m, b, P.data_ptr(), m, Y.data_ptr(), W.data_ptr(), m, None), "panel")
    t_all = ev_time(f)
    t_copy = ev_time(lambda: P.copy_(P0))
    return t_all - t_copy


def main():
    g = torch.Generator(device="cuda").manual_seed(11)
    h = sbr.Handle(0)
    os.environ["SBR_PANEL"] = "tsqr"
    ht = sbr.Handle(0)          # the env knob is read when a handle is created
    del os.environ["SBR_PANEL"]
    for b in (32, 64):
        for m in (4096, 8192, 16384, 32768, 65536):
            P0 = (torch.rand(b, m, device="cuda", generator=g) * 2 - 1).contiguous()   # column-major m x b
            Y = torch.zeros(b, m, device="cuda"); W = torch.zeros(b, m, device="cuda")
            rec = {"m": m, "b": b}
            rec["chol_ms"] = ours(h, m, b, P0, Y, W)
            try:
                rec["tsqr_ms"] = ours(ht, m, b, P0, Y, W)
            except Exception as e:   # beyond the TSQR tree's capacity
                rec["tsqr_ms"] = None
                rec["tsqr_note"] = str(e).splitlines()[0][:80]
            A = P0.t().contiguous()                 # row-major m x b for torch (cuSOLVER takes its own copy)
            rec["geqrf_ms"] = ev_time(lambda: torch.geqrf(A))
            rec["chol_vs_geqrf"] = rec["geqrf_ms"] / rec["chol_ms"]
            if rec["tsqr_ms"]:
                rec["tsqr_vs_geqrf"] = rec["geqrf_ms"] / rec["tsqr_ms"]
            print(json.dumps(rec), flush=True)
    h.close(); ht.close()


if __name__ == "__main__":
    main()
