"""One sbr_band_eigenvalues call on a seeded random band (for ncu captures of the stage-two kernels).

    python tools/stage2_once.py [n] [b]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
    b = int(sys.argv[2]) if len(sys.argv) > 2 else 32
    g = torch.Generator(device="cuda").manual_seed(n + b)
    ab = torch.rand((n, b + 1), generator=g, device="cuda", dtype=torch.float32) * 2 - 1
    h = sbr.Handle(0)
    lam = h.band_eigenvalues(ab)
    h.sync()
    print("lam range", float(lam[0]), float(lam[-1]))
    h.close()


if __name__ == "__main__":
    main()
