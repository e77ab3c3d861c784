"""Pins for oracle.backtransform (CPU only): Alg. 2's merged W reproduces the product of the
per-block factors (a different formula, metrics.q_from_blocks), for several block counts
(recursion depths, odd splits) and ragged last blocks; apply_q equals that Q times X."""
import numpy as np
import pytest

import workloads
from oracle import backtransform, metrics, sbr


@pytest.mark.parametrize("n,b,nb", [(64, 4, 8), (100, 8, 16), (130, 16, 16), (96, 8, 32), (40, 8, 8), (20, 4, 32)])
def test_form_w_equals_block_product(n, b, nb):
    a = workloads.random_symmetric(n, 5 * n + b).astype(np.float64)
    o = sbr.sbr_wy_blocked(a, b, nb)
    blocks = o["blocks"]
    W, Y = backtransform.form_w(n, b, blocks)
    q_merged = np.eye(n) - W @ Y.T
    q_blocks = metrics.q_from_blocks(n, b, blocks)
    assert np.abs(q_merged - q_blocks).max() <= 1e-12
    assert np.abs(q_blocks - o["Q"]).max() <= 1e-12
    # the merged W is the block W where there is a single block
    if len(blocks) == 1:
        np.testing.assert_allclose(W[b:, :], blocks[0][1], atol=0)
    rng = np.random.default_rng(n)
    X = rng.standard_normal((n, 7))
    np.testing.assert_allclose(backtransform.apply_q(W, Y, X), q_blocks @ X, atol=1e-12)
