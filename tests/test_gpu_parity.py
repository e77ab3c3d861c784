"""GPU parity: sbr_reduce (C ABI, CUDA kernels) vs the CPU oracle on the same seeded inputs.

Gates (BASELINE.json north_star):
  FP16 mode   : backward error <= 5e-3, orthogonality <= 5e-3
  3xTF32 mode : backward error <= 1e-5, orthogonality <= 1e-5,
                eigenvalues of B within 1e-5 ||A||_2 of the oracle's
  entry-wise  : sign-normalised B vs the oracle's B within 2e-4 ||A||_2 (3xTF32) --
                B is unique up to D B D.
"""
import numpy as np
import pytest

import workloads
from gpu_helpers import invariants_torch, run_reduce, sign_normalise
from oracle import sbr as osbr
from oracle import tridiag

pytestmark = pytest.mark.gpu

TOL = {"fp16": 5e-3, "3xtf32": 1e-5}


def _oracle(a, b):
    ref = osbr.sbr_unblocked(a, b, want_q=False)
    lam = tridiag.band_eigenvalues(ref["B"])
    return ref["B"], lam


@pytest.mark.parametrize("mode", ["fp16", "3xtf32"])
@pytest.mark.parametrize("n,b,nb", [
    (256, 8, 32),     # config 1 (BASELINE.json configs[0])
    (300, 8, 32),     # n not a multiple of nb (ragged last block)
    (257, 8, 16),     # n not a multiple of b (last panel has m < b)
    (1000, 32, 128),  # multi-leaf TSQR (first panel m = 968 > 512) + reconstruction
    (1024, 64, 128),  # b = 64 (config-5 bandwidth): 4 leaves, arity 4
    (96, 32, 32),     # nb = b (non-lazy degenerate case)
    (1500, 16, 256),  # tile-contiguous FP16 shadow over several blocks, ragged last tile (n - b = 1484)
])
def test_parity_vs_oracle(n, b, nb, mode):
    a = workloads.random_symmetric(n, workloads.config_seed(1) + n + b)
    b_ref, lam_ref = _oracle(a, b)
    norm2 = float(np.max(np.abs(lam_ref)))
    a_dev, ab, w = run_reduce(a, b, nb, mode)
    eb, eo, lam, bm = invariants_torch(a, a_dev, ab, w, n, b, nb)
    ee = float(np.max(np.abs(np.sort(lam) - np.sort(lam_ref)))) / norm2
    db = float(np.max(np.abs(sign_normalise(bm, b) - sign_normalise(b_ref, b)))) / norm2
    print(f"n={n} b={b} nb={nb} {mode}: backward {eb:.2e} orth {eo:.2e} eig {ee:.2e} dB {db:.2e}")
    assert eb <= TOL[mode] and eo <= TOL[mode]
    # exact band structure (C13): AB is the band; nothing else is stored
    assert np.all(np.isfinite(bm))
    if mode == "3xtf32":
        assert ee <= 1e-5
        assert db <= 2e-4
    else:   # FP16: observed <= 2.1e-4 (n = 256 .. 1500); the paper's Table 4 reports ~1e-4
        assert ee <= 1e-3


def test_generator_bit_identical():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    h = sbr.Handle(0)
    for n, seed in [(300, 5), (1031, workloads.config_seed(4))]:
        dev = h.generate_symmetric(seed, n)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(dev.cpu().numpy(), workloads.random_symmetric(n, seed))


def test_prescribed_spectrum_config2_fp16():
    """Config 2: n=4096 SVD_Geo kappa=1e5, b=32, nb=256, FP16 mode (BASELINE configs[1])."""
    n, b, nb = 4096, 32, 256
    a, lam = workloads.prescribed_spectrum(n, "geo", 1e5, seed=workloads.config_seed(2))
    a_dev, ab, w = run_reduce(a, b, nb, "fp16")
    eb, eo, lam_b, _ = invariants_torch(a, a_dev, ab, w, n, b, nb)
    ee = float(np.max(np.abs(np.sort(lam_b) - np.sort(lam))))
    print(f"config2 fp16: backward {eb:.2e} orth {eo:.2e} eig-vs-prescribed {ee:.2e}")
    assert eb <= 5e-3 and eo <= 5e-3
    assert ee <= 5e-3


def test_trivial_and_error_cases():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from paper_conf_ppopp_zhangsoyw23_b200 import SbrError

    h = sbr.Handle(0)
    a_host = workloads.random_symmetric(40, 3)
    a = torch.from_numpy(a_host).cuda()
    ab, _ = h.reduce(a, 39, 39, mode="fp16")        # n <= b+1: AB = band of A
    torch.cuda.synchronize()
    got = sbr.band_to_dense(ab.double()).cpu().numpy()
    np.testing.assert_array_equal(got, osbr.band_part(a_host.astype(np.float64), 39))
    bad = torch.from_numpy(a_host).cuda()
    bad[3, 2] = float("nan")      # both triangles (only the lower one is referenced)
    bad[2, 3] = float("nan")
    h.reduce(bad, 8, 16)                # no host sync: the device latches the error ...
    with pytest.raises(SbrError) as ei:
        h.sync()                        # ... and sbr_sync reports it (include/sbr.h)
    assert ei.value.status == 1
    h.sync()                            # reported once
    with pytest.raises(SbrError) as ei:
        h.reduce(torch.from_numpy(a_host).cuda(), 2, 3)   # nb % b != 0
    assert ei.value.status == -5


@pytest.mark.parametrize("mode", ["fp16", "3xtf32"])
def test_reduce_host_matches_device(mode):
    """sbr_reduce_host (host buffers, copies inside) against sbr_reduce (device buffers) and against
    the oracle.  The fp32 / fp64 reductions of the kernels (atomics) sum in a run-dependent order and
    SBR is backward- not forward-stable, so the two runs' bands are compared entry-wise AFTER the sign
    normalisation of reading C1 to the ORACLE's band B (unique given dlarfg's signs), each within the
    mode's forward tolerance, plus their spectra against each other."""
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    n, b, nb = 512, 16, 64
    a_host = workloads.random_symmetric(n, 77)
    b_ref, lam_ref = _oracle(a_host, b)
    norm2 = float(np.max(np.abs(lam_ref)))
    h = sbr.Handle(0)
    a_dev = torch.from_numpy(a_host).cuda()
    ab_dev, _ = h.reduce(a_dev, b, nb, mode=mode)
    pinned = torch.from_numpy(a_host.copy()).pin_memory()
    ab_host, _ = h.reduce_host(pinned, b, nb, mode=mode)
    torch.cuda.synchronize()
    bd = sbr.band_to_dense(ab_dev.double().cpu()).numpy()
    bh = sbr.band_to_dense(ab_host.double()).numpy()
    ref = sign_normalise(b_ref, b)
    dd = float(np.max(np.abs(sign_normalise(bd, b) - ref))) / norm2
    dh = float(np.max(np.abs(sign_normalise(bh, b) - ref))) / norm2
    tol = 1e-4 if mode == "3xtf32" else 3e-2   # observed 9e-6 / 8.5e-3
    print(f"host vs device {mode}: |B_dev - B_oracle| {dd:.1e}  |B_host - B_oracle| {dh:.1e}")
    assert dd <= tol and dh <= tol
    lam_h = np.linalg.eigvalsh(bh)
    lam_d = np.linalg.eigvalsh(bd)
    assert np.max(np.abs(lam_h - lam_d)) <= (1e-5 if mode == "3xtf32" else 1e-3) * norm2
    assert np.all(np.isfinite(ab_host.numpy()))
