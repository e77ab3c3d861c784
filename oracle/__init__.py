"""CPU oracle for WY-based successive band reduction (SBR) -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct numpy float64 implementations of what the CUDA path
computes, each function citing the PAPER.md passage it follows (``P:n`` = line n
of the paper text).  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``
(its ``cpu_baseline`` leg and ``--impl reference`` arm) may import this package.
The product path (``paper_conf_ppopp_zhangsoyw23_b200``) never imports it and
shares no code with it; the only shared module is ``workloads`` (seeded inputs,
none of the method's arithmetic).

Contents
--------
householder  -- Householder reflector in LAPACK ``dlarfg`` convention.
sbr          -- the plain definition: unblocked Householder band reduction
                (Fig. 2), and the paper's Algorithm 1 (lazy WY,
                P:211-231) written step by step; both are pinned to LAPACK.
panel        -- Householder QR of a tall panel, its T factor, TSQR
                and the Householder reconstruction of Alg. 3 + sign matrix S
                (P:315-339).
tridiag      -- band -> tridiagonal (unblocked SBR with b = 1) and Sturm
                bisection for eigenvalues.
metrics      -- backward error / orthogonality / eigenvalue error (P:395,
                P:399, P:421 as read in DESIGN.md C9), and Q from the
                per-block (W, Y) output.
backtransform -- Alg. 2 FormW and X <- Q X.

Every function is pinned by ``tests/test_oracle_*.py`` against LAPACK,
closed forms, brute force or invariants; none is "parity unpinned".
"""
from . import householder, sbr, panel, tridiag, metrics, backtransform  # noqa: F401
