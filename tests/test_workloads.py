"""The seeded input generators (shared by oracle and CUDA tests): determinism and recipe."""
import numpy as np

import workloads


def test_splitmix64_known_values():
    # Reference values of the splitmix64 finaliser for x = 0, 1 (Vigna's splitmix64
    # with state increment folded in: next() of a generator seeded with x).
    out = workloads.splitmix64(np.array([0, 1], dtype=np.uint64))
    assert int(out[0]) == 0xE220A8397B1DCDAF
    assert int(out[1]) == 0x910A2DEC89025CC1


def test_random_symmetric_properties():
    a = workloads.random_symmetric(300, 42)
    assert a.dtype == np.float32
    np.testing.assert_array_equal(a, a.T)
    assert a.min() >= -1.0 and a.max() < 1.0
    # values on the 2^-23 grid
    np.testing.assert_array_equal(a.astype(np.float64) * 2.0 ** 23, np.round(a.astype(np.float64) * 2.0 ** 23))
    assert abs(float(a.mean())) < 0.01
    assert abs(float(a.var()) - 1.0 / 3.0) < 0.01
    b = workloads.random_symmetric(300, 42)
    np.testing.assert_array_equal(a, b)
    c = workloads.random_symmetric(300, 43)
    assert np.mean(a == c) < 0.01
    cols = workloads.random_symmetric_columns(300, 42, 17, 40)
    np.testing.assert_array_equal(cols, a[:, 17:40])


def test_prescribed_spectrum():
    for kind in workloads.SPECTRUM_KINDS:
        a, lam = workloads.prescribed_spectrum(64, kind, 1e3, seed=9)
        np.testing.assert_array_equal(a, a.T)
        assert np.isclose(lam.max(), 1.0) and np.isclose(lam.min(), 1e-3)
        got = np.linalg.eigvalsh(a.astype(np.float64))
        assert np.max(np.abs(np.sort(got) - np.sort(lam))) < 1e-6


def test_hadamard_prescribed_spectrum_cpu():
    """Config-5 recipe (randomised Hadamard Q) on CPU at small n: bit-symmetric,
    dense, spectrum = the prescribed one to fp32 accuracy."""
    import numpy as np

    import workloads

    n = 512
    a, desc = workloads.prescribed_spectrum_device(n, "geo", 1e5, 11, a_device="cpu", haar_max=16)
    a = a.numpy()
    assert "Hadamard" in desc
    np.testing.assert_array_equal(a, a.T)
    assert np.count_nonzero(a) > 0.99 * n * n
    lam = np.linalg.eigvalsh(a.astype(np.float64))
    assert np.max(np.abs(lam - np.sort(workloads.spectrum(n, "geo", 1e5)))) <= 1e-6
