"""Multi-GPU path (include/sbr.h sbr_*_dist).

CPU (world_size 2, gloo, 127.0.0.1): the host logic the sharded reduction relies on --
  * the pass's tile partition (sbr_test_pass_partition / sbr_test_pass_tiles, the host mirror
    of the kernel's tile order) covers every lower 128x128 tile of OA exactly once over the
    ranks, for several M, b and world sizes;
  * the sharded pass itself: each gloo rank forms ITS tiles' contributions
    X_I += L_IJ W_J, X_J += L_IJ^T W_I (half-diagonal shadow convention of the kernel) in
    fp64, an all-reduce sums them, and the sum equals OA W (the definition);
  * the NCCL unique-id exchange the ranks use to build their communicator.
GPU (one B200): the device-side share of every rank (sbr_test_pass_fp16_part summed over
ranks = the full pass) and sbr_reduce_dist through a real NCCL communicator with the
exchanges forced on (SBR_DIST_COLLECTIVES=1), checked against the parity invariants.
"""
import os
import socket

import numpy as np
import pytest


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("M,b", [(128, 32), (1000, 32), (4000, 32), (3000, 64), (2500, 16)])
@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_pass_partition_covers_lower_tiles_once(M, b, P):
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    NT = (M + 127) // 128
    seen = {}
    ends = []
    for r in range(P):
        t0, t1, tot = sbr.pass_partition(M, b, r, P)
        assert tot == NT * (NT + 1) // 2
        ends.append((t0, t1))
        for ij in sbr.pass_tiles(M, b, t0, t1):
            seen[ij] = seen.get(ij, 0) + 1
    assert ends[0][0] == 0 and ends[-1][1] == NT * (NT + 1) // 2
    assert all(ends[i][1] == ends[i + 1][0] for i in range(P - 1))
    assert max(t1 - t0 for t0, t1 in ends) - min(t1 - t0 for t0, t1 in ends) <= 1   # balanced to one tile
    assert set(seen) == {(i, j) for i in range(NT) for j in range(i + 1)}
    assert all(v == 1 for v in seen.values())


def _sharded_pass_worker(rank, world, port, M, b, q):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rng = np.random.default_rng(1234)                 # same inputs on every rank
        a = rng.uniform(-1, 1, (M, M))
        oa = np.tril(a) + np.tril(a, -1).T
        w = rng.uniform(-1, 1, (M, b))
        # the kernel's shadow: strict lower + half diagonal, zero above
        sh = np.tril(oa, -1) + np.diag(0.5 * np.diag(oa))
        t0, t1, _ = sbr.pass_partition(M, b, rank, world)
        x = np.zeros((M, b))
        for (I, J) in sbr.pass_tiles(M, b, t0, t1):
            i0, i1, j0, j1 = I * 128, min(M, I * 128 + 128), J * 128, min(M, J * 128 + 128)
            L = sh[i0:i1, j0:j1]
            x[i0:i1] += L @ w[j0:j1]
            x[j0:j1] += L.T @ w[i0:i1]
        xt = torch.from_numpy(x)
        dist.all_reduce(xt)
        # unique-id exchange (what bench.py / users do before sbr_create_dist)
        obj = [sbr.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ids = [None] * world
        dist.all_gather_object(ids, obj[0])
        if rank == 0:
            err = float(np.max(np.abs(xt.numpy() - oa @ w)))
            q.put((err, len(set(ids)), len(ids[0])))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("M,b", [(700, 32), (1300, 64)])
def test_sharded_pass_world2_gloo(M, b):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sharded_pass_worker, args=(r, 2, port, M, b, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs)
    err, distinct, nbytes = q.get(timeout=10)
    assert err <= 1e-10
    assert distinct == 1 and nbytes == 128


@pytest.mark.gpu
@pytest.mark.parametrize("M,b,P", [(1000, 32, 2), (2050, 32, 3), (777, 64, 4)])
def test_pass_rank_shares_sum_to_full_pass(M, b, P):
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    rng = np.random.default_rng(M + P)
    oa = rng.uniform(-1, 1, (M, M)).astype(np.float32)
    oa = np.tril(oa) + np.tril(oa, -1).T
    w = rng.uniform(-1, 1, (M, b)).astype(np.float32)
    h = sbr.Handle(0)
    d_oa = torch.from_numpy(oa.T.copy()).cuda()
    d_w = torch.from_numpy(w.T.copy()).cuda()
    full = torch.zeros((b, M), dtype=torch.float32, device="cuda")
    _lib.check(_lib.lib().sbr_test_pass_fp16(h._h, M, b, d_oa.data_ptr(), M, d_w.data_ptr(), M, full.data_ptr(), M),
               "pass")
    acc = torch.zeros((b, M), dtype=torch.float64, device="cuda")
    for r in range(P):
        part = torch.zeros((b, M), dtype=torch.float32, device="cuda")
        _lib.check(_lib.lib().sbr_test_pass_fp16_part(h._h, M, b, r, P, d_oa.data_ptr(), M, d_w.data_ptr(), M,
                                                      part.data_ptr(), M), "pass part")
        acc += part.double()
    err = float((acc - full.double()).abs().max())
    assert err <= 2.0 ** -20 * M   # same fp16 products, fp32 sums in another order


@pytest.mark.gpu
def test_reduce_dist_one_rank_with_collectives(monkeypatch):
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    import workloads
    from gpu_helpers import invariants_torch

    monkeypatch.setenv("SBR_DIST_COLLECTIVES", "1")
    n, b, nb = 1024, 32, 128
    a_host = workloads.random_symmetric(n, 99)
    h = sbr.Handle(0, unique_id=sbr.get_unique_id(), rank=0, nranks=1)
    a = torch.from_numpy(a_host).cuda()
    ab, w = h.reduce_dist(a, b, nb, mode="fp16")
    torch.cuda.synchronize()
    eb, eo, lam, _ = invariants_torch(a_host, a, ab, w, n, b, nb)
    lam_ref = np.linalg.eigvalsh(a_host.astype(np.float64))
    ee = float(np.max(np.abs(np.sort(lam) - lam_ref))) / float(np.max(np.abs(lam_ref)))
    print(f"reduce_dist(1 rank, NCCL exchanges on): backward {eb:.2e} orth {eo:.2e} eig {ee:.2e}")
    assert eb <= 5e-3 and eo <= 5e-3 and ee <= 1e-2
    h.close()
