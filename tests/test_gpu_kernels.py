"""Kernel-level parity of the tcgen05/TMA kernels (include/sbr_testing.h) against fp64
products of the SAME fp16-rounded operands (|err| <= 2^-22 * K * max|a||b|
for fp32 accumulation of exact fp16 products, plus the fp16 rounding of outputs where stated)."""
import ctypes

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _h():
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    return sbr.Handle(0)


def _cm(t):
    """torch (rows, cols) -> column-major device buffer = contiguous tensor of the transpose."""
    return t.t().contiguous()


def _r16(x):
    return x.astype(np.float16).astype(np.float64)


@pytest.mark.parametrize("M,b", [(128, 32), (300, 32), (1000, 32), (2050, 32), (777, 64), (640, 16), (513, 8)])
def test_pass_fp16(M, b):
    import torch
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M + b)
    oa = rng.uniform(-1, 1, (M, M)).astype(np.float32)
    oa = np.tril(oa) + np.tril(oa, -1).T
    w = rng.uniform(-1, 1, (M, b)).astype(np.float32)
    h = _h()
    d_oa = _cm(torch.from_numpy(oa).cuda())
    d_w = _cm(torch.from_numpy(w).cuda())
    d_x = torch.zeros((b, M), dtype=torch.float32, device="cuda")
    _lib.check(_lib.lib().sbr_test_pass_fp16(h._h, M, b, d_oa.data_ptr(), M, d_w.data_ptr(), M, d_x.data_ptr(), M),
               "pass")
    x = d_x.cpu().numpy().T
    # shadow: strict lower fp16, diagonal halved in fp16 (exact), doubled back by symmetry
    low = np.tril(oa, -1)
    ref_oa = _r16(low) + _r16(low).T + np.diag(2.0 * _r16(0.5 * np.diag(oa)))
    ref = ref_oa @ _r16(w)
    tol = 2.0 ** -22 * M * 2 + 1e-6
    err = np.abs(x - ref).max()
    print(f"pass M={M} b={b}: max err {err:.2e} (tol {tol:.1e})")
    assert err <= tol


@pytest.mark.parametrize("M,K", [(128, 64), (256, 32), (700, 128), (1100, 256), (2100, 1024), (333, 96)])
def test_syr2k_fp16(M, K):
    import torch
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M * 7 + K)
    y = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    z = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    c = rng.uniform(-1, 1, (M, M)).astype(np.float32)
    h = _h()
    d_y, d_z, d_c = _cm(torch.from_numpy(y).cuda()), _cm(torch.from_numpy(z).cuda()), _cm(torch.from_numpy(c).cuda())
    d_s = torch.zeros((M, M), dtype=torch.float32, device="cuda")
    _lib.check(_lib.lib().sbr_test_syr2k_fp16(h._h, M, K, d_y.data_ptr(), M, d_z.data_ptr(), M, d_c.data_ptr(), M,
                                             d_s.data_ptr(), M), "syr2k")
    got = d_c.cpu().numpy().T
    sh = d_s.cpu().numpy().T
    y16, z16 = _r16(y), _r16(z)
    ref = c.astype(np.float64) - (y16 @ z16.T + z16 @ y16.T)
    low = np.tril(np.ones((M, M), dtype=bool))
    tol = 2.0 ** -22 * 2 * K * 1.0 + 1e-5
    err = np.abs(got - ref)[low].max()
    print(f"syr2k M={M} K={K}: max err {err:.2e} (tol {tol:.1e})")
    assert err <= tol
    np.testing.assert_array_equal(got[~low], c[~low])            # upper triangle untouched
    # shadow = fp16 of the new lower triangle, diagonal halved, upper zero
    exp_sh = np.tril(got, -1).astype(np.float16).astype(np.float32) + \
        np.diag((0.5 * np.diag(got)).astype(np.float16).astype(np.float32))
    np.testing.assert_array_equal(sh, exp_sh)


@pytest.mark.parametrize("M,K", [(128, 64), (500, 96), (1500, 256), (2048, 1024)])
def test_zform_fp16(M, K):
    import torch
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M + 3 * K)
    y = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    g = rng.uniform(-1, 1, (K, K)).astype(np.float32)
    g = (g + g.T).astype(np.float32)
    x = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    h = _h()
    d_y, d_g, d_x = _cm(torch.from_numpy(y).cuda()), _cm(torch.from_numpy(g).cuda()), _cm(torch.from_numpy(x).cuda())
    d_z = torch.zeros((K, M), dtype=torch.float32, device="cuda")
    _lib.check(_lib.lib().sbr_test_zform_fp16(h._h, M, K, d_y.data_ptr(), M, d_g.data_ptr(), K, d_x.data_ptr(), M,
                                             d_z.data_ptr(), M), "zform")
    z = d_z.cpu().numpy().T
    ref = x.astype(np.float64) - 0.5 * (_r16(y) @ _r16(g))
    # fp32 accumulation error, then the fp16 rounding of Z (relative 2^-11)
    tol = 2.0 ** -22 * K * 2 + np.abs(ref) * 2.0 ** -11 + 1e-6
    err = np.abs(z - ref)
    print(f"zform M={M} K={K}: max err {err.max():.2e}")
    assert np.all(err <= tol)


# ---------------------------------------------------------------- 3xTF32 (reading C11 / R4)
def _tf32_rna(x):
    """numpy emulation of cvt.rna.tf32.f32 (add 0x1000, mask 0xFFFFE000)."""
    u = np.asarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    return ((u + 0x1000) & 0xFFFFE000).astype(np.uint32).view(np.float32).astype(np.float64)


def _gate_3xtf32(err, err1, K, scale, what):
    """3xTF32 must be far below a single TF32 product (|err| <= err_1xTF32 / 16) and inside
    the worst-case 3xTF32 bound (3 * 2^-20 per product, fp32 accumulation 2^-23 per term)."""
    bound = K * scale * (3 * 2.0 ** -20 + 2.0 ** -23)
    print(f"{what}: max err {err:.2e}  (1xTF32 {err1:.2e}, bound {bound:.1e})")
    assert err <= err1 / 16
    assert err <= bound


@pytest.mark.parametrize("M,b,sw", [(128, 32, 0), (300, 32, 0), (1000, 32, 0), (2052, 32, 200), (780, 64, 0),
                                    (640, 16, 96), (516, 8, 0), (1024, 32, 1000), (8192, 32, 992)])
def test_pass_tf32(M, b, sw):
    import torch
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M + b + 11)
    oa = rng.uniform(-1, 1, (M, M)).astype(np.float32)
    oa = np.tril(oa) + np.tril(oa, -1).T
    w = rng.uniform(-1, 1, (M, b)).astype(np.float32)
    # the kernel must read only the lower triangle: poison the upper one
    a_dev = np.tril(oa) + np.triu(np.full((M, M), np.nan, np.float32), 1)
    strip = None
    if sw:
        swc = min((sw + 127) // 128 * 128, M)
        strip = np.asfortranarray(a_dev[:, :swc])
        a_dev[:, :swc] = np.nan            # those columns must come from the strip
    h = _h()
    d_oa = _cm(torch.from_numpy(a_dev).cuda())
    d_w = _cm(torch.from_numpy(w).cuda())
    d_x = torch.zeros((b, M), dtype=torch.float32, device="cuda")
    d_s = _cm(torch.from_numpy(np.ascontiguousarray(strip)).cuda()) if sw else None
    _lib.check(_lib.lib().sbr_test_pass_tf32(h._h, M, b, d_oa.data_ptr(), M, d_s.data_ptr() if sw else None, M, sw,
                                            d_w.data_ptr(), M, d_x.data_ptr(), M), "pass_tf32")
    x = d_x.cpu().numpy().T
    ref = oa.astype(np.float64) @ w.astype(np.float64)
    err = np.abs(x - ref).max()
    err1 = np.abs(_tf32_rna(oa) @ _tf32_rna(w) - ref).max()
    _gate_3xtf32(err, err1, M, 1.0, f"pass_tf32 M={M} b={b} sw={sw}")


@pytest.mark.parametrize("M,K", [(128, 64), (256, 32), (700, 128), (1100, 256), (2100, 1024), (333, 96), (400, 40)])
def test_syr2k_tf32(M, K):
    import torch
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M * 5 + K)
    y = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    z = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    c = rng.uniform(-1, 1, (M, M)).astype(np.float32)
    h = _h()
    d_y, d_z, d_c = _cm(torch.from_numpy(y).cuda()), _cm(torch.from_numpy(z).cuda()), _cm(torch.from_numpy(c).cuda())
    _lib.check(_lib.lib().sbr_test_syr2k_tf32(h._h, M, K, d_y.data_ptr(), M, d_z.data_ptr(), M, d_c.data_ptr(), M),
               "syr2k_tf32")
    got = d_c.cpu().numpy().T
    y64, z64 = y.astype(np.float64), z.astype(np.float64)
    ref = c.astype(np.float64) - (y64 @ z64.T + z64 @ y64.T)
    low = np.tril(np.ones((M, M), dtype=bool))
    err = np.abs(got - ref)[low].max()
    yt, zt = _tf32_rna(y), _tf32_rna(z)
    err1 = np.abs((c.astype(np.float64) - (yt @ zt.T + zt @ yt.T)) - ref)[low].max()
    _gate_3xtf32(err, err1, 2 * K, 1.0, f"syr2k_tf32 M={M} K={K}")
    np.testing.assert_array_equal(got[~low], c[~low])            # upper triangle untouched


@pytest.mark.parametrize("M,K", [(128, 64), (500, 96), (1500, 256), (2048, 1024), (300, 40)])
def test_zform_tf32(M, K):
    import torch
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M + 7 * K)
    y = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    g = rng.uniform(-1, 1, (K, K)).astype(np.float32)
    g = (g + g.T).astype(np.float32)
    x = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    h = _h()
    d_y, d_g, d_x = _cm(torch.from_numpy(y).cuda()), _cm(torch.from_numpy(g).cuda()), _cm(torch.from_numpy(x).cuda())
    d_z = torch.zeros((K, M), dtype=torch.float32, device="cuda")
    _lib.check(_lib.lib().sbr_test_zform_tf32(h._h, M, K, d_y.data_ptr(), M, d_g.data_ptr(), K, d_x.data_ptr(), M,
                                             d_z.data_ptr(), M), "zform_tf32")
    z = d_z.cpu().numpy().T
    ref = x.astype(np.float64) - 0.5 * (y.astype(np.float64) @ g.astype(np.float64))
    err = np.abs(z - ref).max()
    err1 = np.abs(x.astype(np.float64) - 0.5 * (_tf32_rna(y) @ _tf32_rna(g)) - ref).max()
    _gate_3xtf32(err, err1, K, 2.0, f"zform_tf32 M={M} K={K}")
