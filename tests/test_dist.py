"""Multi-GPU path (north star: 1D block-cyclic columns; include/sbr.h sbr_*_dist).

CPU (world_size 2-3, gloo, 127.0.0.1): the host logic of the sharded reduction --
  * the column ownership: every column belongs to exactly one rank, local layouts concatenate
    the owned nb-blocks in order (sbr_local_cols / local_columns);
  * the distributed pass's tile walk (sbr_test_pass_owned_tiles, the host mirror of the
    kernel's walk): over the ranks it covers every lower 128x128 tile of the block's
    128-aligned grid exactly once, each rank only tiles of its own column blocks;
  * the sharded pass itself: each gloo rank forms ITS tiles' contributions
    X_I += L_IJ W_J, X_J += L_IJ^T W_I (half-diagonal shadow, OA starting b rows into the
    grid, W zero-padded in front) in fp64, an all-reduce sums them, and the sum equals
    OA W (the definition);
  * the NCCL unique-id exchange the ranks use to build their communicator.
GPU (one B200): sbr_reduce_dist with P in-process ranks (sbr_create_dist_local: one thread per
rank, the same kernels and call sequence as NCCL ranks) -- the gathered outputs pass the parity
invariants and match the single-GPU reduction; each rank holds only its columns.
"""
import os
import socket
import threading

import numpy as np
import pytest


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("n,nb,P", [(4096, 1024, 2), (5000, 1024, 3), (9000, 2048, 4), (700, 1024, 2)])
def test_column_ownership_partitions_columns(n, nb, P):
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    seen = np.zeros(n, dtype=int)
    for r in range(P):
        cols = sbr.local_columns(n, nb, r, P)
        assert len(cols) == sbr.local_cols(n, nb, r, P)
        assert np.all(np.diff(cols) > 0)
        assert np.all((cols // nb) % P == r)
        seen[cols] += 1
    assert np.all(seen == 1)


@pytest.mark.parametrize("n,b,nb", [(4096, 32, 1024), (5200, 32, 1024), (9000, 64, 2048)])
@pytest.mark.parametrize("P", [1, 2, 3])
def test_owned_pass_tiles_cover_lower_tiles_once(n, b, nb, P):
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    for c0 in range(0, n - b - 1, nb):
        M = n - c0 - b
        NT = (M + b + 127) // 128
        seen = {}
        for r in range(P):
            for (I, J) in sbr.pass_owned_tiles(n, b, nb, c0, r, P):
                assert I >= J
                assert ((c0 + 128 * J) // nb) % P == r      # only the rank's column blocks
                seen[(I, J)] = seen.get((I, J), 0) + 1
        assert set(seen) == {(i, j) for i in range(NT) for j in range(i + 1)}
        assert all(v == 1 for v in seen.values())


def _sharded_pass_worker(rank, world, port, n, b, nb, c0, q):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        M = n - c0 - b
        rng = np.random.default_rng(1234)                 # same inputs on every rank
        a = rng.uniform(-1, 1, (M, M))
        oa = np.tril(a) + np.tril(a, -1).T
        w = rng.uniform(-1, 1, (M, b))
        off = b
        G = M + off                                       # grid rows: OA starts `off` rows in
        sh = rng.uniform(-5, 5, (G, G))                   # junk: stale panel columns / rows above OA
        sh[off:, off:] = np.tril(oa, -1) + np.diag(0.5 * np.diag(oa))   # the shadow convention on OA
        wp = np.zeros((G, b))
        wp[off:] = w                                      # W with `off` zero rows in front
        xp = np.zeros((G, b))
        for (I, J) in sbr.pass_owned_tiles(n, b, nb, c0, rank, world):
            i0, i1, j0, j1 = I * 128, min(G, I * 128 + 128), J * 128, min(G, J * 128 + 128)
            L = sh[i0:i1, j0:j1]
            xp[i0:i1] += L @ wp[j0:j1]
            xp[j0:j1] += L.T @ wp[i0:i1]
        xt = torch.from_numpy(xp[off:].copy())            # X rows = grid rows - off
        dist.all_reduce(xt)
        obj = [sbr.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ids = [None] * world
        dist.all_gather_object(ids, obj[0])
        if rank == 0:
            err = float(np.max(np.abs(xt.numpy() - oa @ w)))
            q.put((err, len(set(ids)), len(ids[0])))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,b,nb,c0,world", [(2600, 32, 1024, 0, 2), (3500, 32, 1024, 1024, 3), (5000, 64, 2048, 0, 2)])
def test_sharded_pass_gloo(n, b, nb, c0, world):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sharded_pass_worker, args=(r, world, port, n, b, nb, c0, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(180)
    assert all(p.exitcode == 0 for p in procs)
    err, distinct, nbytes = q.get(timeout=10)
    assert err <= 1e-9
    assert distinct == 1 and nbytes == 128


def _run_virtual_ranks(a_host, n, b, nb, P, mode="fp16", group=None):
    """sbr_reduce_dist with P in-process ranks on cuda:0; returns per-rank (A_local, W_local),
    the band of rank 0 and the local column lists."""
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr

    group = group if group is not None else (os.getpid() * 131 + P) % 100000
    out = [None] * P
    errs = []
    a_full = torch.from_numpy(a_host)

    def work(r):
        try:
            torch.cuda.set_device(0)
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                h = sbr.Handle(0, stream=st, local_group=group, rank=r, nranks=P)
                cols = sbr.local_columns(n, nb, r, P)
                a_loc = a_full[torch.from_numpy(cols)].contiguous().cuda()
                ab, w = h.reduce_dist(a_loc, n, b, nb, mode=mode)
                h.sync()
                out[r] = (a_loc.cpu(), None if w is None else w.cpu(), None if ab is None else ab.cpu(), cols)
                h.close()
        except Exception as e:  # pragma: no cover
            errs.append(f"rank {r}: {e!r}")

    th = [threading.Thread(target=work, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(600)
    assert not errs, errs
    return out


def _gather(out, n):
    import torch

    a = torch.zeros((n, n), dtype=torch.float32)
    w = torch.zeros((n, n), dtype=torch.float32)
    for a_loc, w_loc, _, cols in out:
        idx = torch.from_numpy(cols)
        a[idx] = a_loc
        w[idx] = w_loc
    return a, w


@pytest.mark.gpu
@pytest.mark.parametrize("n,P,mode", [(4096, 2, "fp16"), (5200, 3, "fp16"), (3072, 1, "fp16"),
                                      (4096, 2, "3xtf32"), (5200, 3, "3xtf32")])
def test_reduce_dist_virtual_ranks(n, P, mode):
    """P ranks (threads, one B200): gathered outputs pass the parity gates and match the
    single-GPU reduction's spectrum; the band is the same matrix up to D B D."""
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    import workloads
    from gpu_helpers import invariants_torch, run_reduce, sign_normalise

    b, nb = 32, 1024
    a_host = workloads.random_symmetric(n, 4242 + n)
    out = _run_virtual_ranks(a_host, n, b, nb, P, mode=mode)
    a_out, w_out = _gather(out, n)
    ab = out[0][2]
    eb, eo, lam, bm = invariants_torch(a_host, a_out.cuda(), ab.cuda(), w_out[: n - b].cuda(), n, b, nb)
    ref = np.linalg.eigvalsh(a_host.astype(np.float64))
    ee = float(np.max(np.abs(np.sort(lam) - ref))) / float(np.max(np.abs(ref)))
    a1, ab1, w1 = run_reduce(a_host, b, nb, mode)
    bm1 = sbr.band_to_dense(ab1.double()).cpu().numpy()
    db = float(np.max(np.abs(sign_normalise(bm, b) - sign_normalise(bm1, b)))) / float(np.max(np.abs(ref)))
    print(f"reduce_dist P={P} n={n} {mode}: backward {eb:.2e} orth {eo:.2e} eig {ee:.2e} |dB| vs 1 GPU {db:.2e}")
    if mode == "fp16":
        assert eb <= 5e-3 and eo <= 5e-3 and ee <= 1e-3
        # entry-wise B is a forward error (cond x backward error): two single-GPU FP16 runs already
        # differ by ~2e-2 ||A||_2 (fp32 atomics in the pass sum in another order), so this only
        # checks that the distributed band is the same matrix, not a different reduction
        assert db <= 5e-2
    else:
        assert eb <= 1e-5 and eo <= 1e-5 and ee <= 1e-5
        assert db <= 1e-3
    for r, (a_loc, _, _, cols) in enumerate(out):   # each rank held only its columns
        assert a_loc.shape[0] == len(cols) == sbr.local_cols(n, nb, r, P)


@pytest.mark.gpu
def test_reduce_dist_unsupported_args():
    import torch

    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    from paper_conf_ppopp_zhangsoyw23_b200 import SbrError

    n = 2048
    errs = []

    def work(r):
        try:
            h = sbr.Handle(0, stream=torch.cuda.Stream(), local_group=777, rank=r, nranks=2)
            a = torch.zeros((sbr.local_cols(n, 256, r, 2), n), dtype=torch.float32, device="cuda")
            with pytest.raises(SbrError) as ei:
                h.reduce_dist(a, n, 32, 256)        # nb not a multiple of 1024
            assert ei.value.status == 5
            with pytest.raises(SbrError) as ei:
                h.reduce_dist(a, n, 2, 256, mode="3xtf32")   # b % 4 != 0
            assert ei.value.status == 5
            h.close()
        except Exception as e:  # pragma: no cover
            errs.append(repr(e))

    th = [threading.Thread(target=work, args=(r,)) for r in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join(60)
    assert not errs, errs
