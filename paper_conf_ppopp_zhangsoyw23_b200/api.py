"""Python API over libsbr (marshalling only; see include/sbr.h for semantics)."""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import check, lib

MODES = {"fp16": _lib.SBR_FP16_FP32ACC, "3xtf32": _lib.SBR_3XTF32, "bf16": _lib.SBR_BF16_FP32ACC}


def _mode(mode) -> int:
    if isinstance(mode, int):
        return mode
    try:
        return MODES[mode.lower()]
    except KeyError:
        raise ValueError(f"mode must be one of {sorted(MODES)}") from None


def _ptr(t) -> int | None:
    if t is None:
        return None
    if hasattr(t, "data_ptr"):
        return t.data_ptr()
    return t.ctypes.data  # numpy


def get_unique_id() -> bytes:
    """128-byte NCCL unique id for ``Handle(..., unique_id=..., rank=..., nranks=...)`` (rank 0 creates it)."""
    buf = ctypes.create_string_buffer(128)
    check(lib().sbr_get_unique_id(buf), "sbr_get_unique_id")
    return buf.raw


def pass_partition(M: int, b: int, rank: int, nranks: int):
    """Host-only: (t0, t1, total) -- the tiles of the per-panel pass that ``rank`` streams (sbr_testing.h)."""
    t0, t1, tot = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    check(lib().sbr_test_pass_partition(M, b, rank, nranks, ctypes.byref(t0), ctypes.byref(t1), ctypes.byref(tot)),
          "sbr_test_pass_partition")
    return t0.value, t1.value, tot.value


def local_cols(n: int, nb: int, rank: int, nranks: int) -> int:
    """Columns rank ``rank`` holds under the 1D block-cyclic distribution (sbr_local_cols)."""
    return int(lib().sbr_local_cols(int(n), int(nb), int(rank), int(nranks)))


def local_columns(n: int, nb: int, rank: int, nranks: int):
    """Global column indices of the rank's local columns, in local order (numpy int64)."""
    import numpy as np

    cols = [np.arange(c0, min(n, c0 + nb)) for c0 in range(rank * nb, n, nranks * nb)]
    return np.concatenate(cols) if cols else np.zeros(0, dtype=np.int64)


def pass_owned_tiles(n: int, b: int, nb: int, c0: int, rank: int, nranks: int):
    """Host-only: (I, J) tiles of the distributed pass that ``rank`` streams for block origin c0."""
    cnt = int(lib().sbr_test_pass_owned_tiles(n, b, nb, c0, rank, nranks, None, 0))
    if cnt < 0:
        raise ValueError("unsupported arguments")
    buf = (ctypes.c_int * (2 * cnt + 1))()
    lib().sbr_test_pass_owned_tiles(n, b, nb, c0, rank, nranks, buf, cnt)
    return [(buf[2 * k], buf[2 * k + 1]) for k in range(cnt)]


def pass_tiles(M: int, b: int, t0: int, t1: int):
    """Host-only: list of (I, J) lower 128x128 tiles [t0, t1) in the pass's order."""
    n = max(0, t1 - t0)
    buf = (ctypes.c_int * (2 * n + 1))()
    check(lib().sbr_test_pass_tiles(M, b, t0, t1, buf), "sbr_test_pass_tiles")
    return [(buf[2 * k], buf[2 * k + 1]) for k in range(n)]


class Handle:
    """One libsbr handle: a device, a CUDA stream (torch's current stream by default)
    and the reduction workspace it owns.  With ``unique_id``/``rank``/``nranks`` it also owns
    an NCCL communicator (one process per GPU) for :meth:`reduce_dist`."""

    def __init__(self, device: int = 0, stream=None, unique_id: bytes | None = None, rank: int = 0,
                 nranks: int = 1, local_group: int | None = None):
        """``unique_id``: NCCL communicator (one process per GPU).  ``local_group``: the in-process
        communicator -- ``nranks`` handles of one process (one thread each) with the same key."""
        import torch

        self.device = int(device)
        if stream is None:
            stream = torch.cuda.current_stream(self.device)
        self._stream = stream
        h = ctypes.c_void_p()
        if local_group is not None:
            check(lib().sbr_create_dist_local(ctypes.byref(h), self.device, ctypes.c_void_p(stream.cuda_stream),
                                              int(local_group), int(rank), int(nranks)), "sbr_create_dist_local")
        elif unique_id is None:
            check(lib().sbr_create(ctypes.byref(h), self.device, ctypes.c_void_p(stream.cuda_stream)), "sbr_create")
        else:
            uid = ctypes.create_string_buffer(bytes(unique_id), 128)
            check(lib().sbr_create_dist(ctypes.byref(h), self.device, ctypes.c_void_p(stream.cuda_stream), uid,
                                        int(rank), int(nranks)), "sbr_create_dist")
        self._h = h
        self.rank, self.nranks = int(rank), int(nranks)

    # -- lifecycle
    def close(self) -> None:
        if getattr(self, "_h", None) is not None and self._h.value:
            lib().sbr_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def set_stream(self, stream) -> None:
        self._stream = stream
        check(lib().sbr_set_stream(self._h, ctypes.c_void_p(stream.cuda_stream)), "sbr_set_stream")

    # -- the reduction
    def workspace_bytes(self, n: int, b: int, nb: int, mode="fp16") -> int:
        out = ctypes.c_size_t()
        check(lib().sbr_workspace_query(self._h, n, b, nb, _mode(mode), ctypes.byref(out)), "workspace_query")
        return int(out.value)

    def reduce(self, A, b: int, nb: int, mode="fp16", want_w: bool = True, ab=None, w=None):
        """Reduce the symmetric (n, n) float32 CUDA tensor ``A`` in place to bandwidth b.

        Returns ``(ab, w)``: ``ab`` (n, b+1) with ``ab[j, d] = B[j+d, j]``; ``w``
        (n-b, n) with ``w[c, r] = W(r, c)`` (None if ``want_w`` is False).  A is
        overwritten with the sy2sb layout (see the package docstring).  Enqueued on
        the handle's stream without host synchronisation: device-detected errors (non-finite
        input, fp16 range) are latched and raised by :meth:`sync` or the next call.
        """
        import torch

        n = int(A.shape[0])
        if A.dim() != 2 or A.shape[1] != n or A.dtype != torch.float32 or not A.is_cuda or not A.is_contiguous():
            raise ValueError("A must be a contiguous square float32 CUDA tensor")
        if ab is None:
            ab = torch.empty((n, b + 1), dtype=torch.float32, device=A.device)
        if want_w and w is None and n > b:   # zeros: entries the reduction does not reference stay 0
            w = torch.zeros((max(n - b, 1), n), dtype=torch.float32, device=A.device)
        if not want_w:
            w = None
        check(lib().sbr_reduce(self._h, _mode(mode), n, int(b), int(nb), _ptr(A), n, _ptr(ab), b + 1,
                               _ptr(w), n), "sbr_reduce")
        return ab, w

    def form_q(self, A, w, b: int, nb: int, q=None):
        """Explicit Q = prod_J (I - W_J Y_J^T) from :meth:`reduce`'s outputs (A holding Y, and ``w``)
        with the same b, nb (sbr_form_q; 3xTF32 on tcgen05).  Returns the (n, n) float32 tensor
        ``q`` with ``q[c, r] = Q(r, c)`` (column-major Q, i.e. ``Q = q.T``)."""
        import torch

        n = int(A.shape[0])
        if A.dim() != 2 or A.shape[1] != n or A.dtype != torch.float32 or not A.is_cuda or not A.is_contiguous():
            raise ValueError("A must be a contiguous square float32 CUDA tensor")
        if w is None or w.dtype != torch.float32 or not w.is_contiguous() or w.shape[-1] != n:
            raise ValueError("w must be the (n-b, n) float32 tensor returned by reduce")
        if q is None:
            q = torch.empty((n, n), dtype=torch.float32, device=A.device)
        check(lib().sbr_form_q(self._h, n, int(b), int(nb), _ptr(A), n, _ptr(w), n, _ptr(q), n), "sbr_form_q")
        return q

    def form_w(self, A, w, b: int, nb: int, out=None):
        """Alg. 2 (sbr_form_w): the merged W (torch shape (n-b, n), ``out[c, r] = W(r, c)``) with
        Q = I - W Y^T, from :meth:`reduce`'s outputs."""
        import torch

        n = int(A.shape[0])
        if out is None:
            out = torch.empty((max(n - b, 1), n), dtype=torch.float32, device=A.device)
        check(lib().sbr_form_w(self._h, n, int(b), int(nb), _ptr(A), n, _ptr(w), n, _ptr(out), n), "sbr_form_w")
        return out

    def apply_q(self, A, w, b: int, nb: int, X):
        """X <- Q X in place (sbr_apply_q); X: torch (kx, n) contiguous float32 CUDA (= column-major n x kx)."""
        n = int(A.shape[0])
        if X.dim() != 2 or X.shape[1] != n or not X.is_contiguous():
            raise ValueError("X must be a contiguous (kx, n) float32 CUDA tensor")
        check(lib().sbr_apply_q(self._h, n, int(b), int(nb), _ptr(A), n, _ptr(w), n, _ptr(X), n, int(X.shape[0])),
              "sbr_apply_q")
        return X

    # ---- stage two (include/sbr.h sbr_band_to_tridiag ...)
    def band_to_tridiag(self, ab, d=None, e=None):
        """Band (torch (n, b+1) float32 CUDA, ``ab[j, k] = B[j+k, j]``, :meth:`reduce`'s output) ->
        tridiagonal ``(d, e)`` (float64, n and n-1 entries) by bulge chasing on the GPU."""
        import torch

        n, bp1 = int(ab.shape[0]), int(ab.shape[1])
        if ab.dtype != torch.float32 or not ab.is_cuda or not ab.is_contiguous():
            raise ValueError("ab must be a contiguous (n, b+1) float32 CUDA tensor")
        d = torch.empty(n, dtype=torch.float64, device=ab.device) if d is None else d
        e = torch.empty(max(n - 1, 0), dtype=torch.float64, device=ab.device) if e is None else e
        check(lib().sbr_band_to_tridiag(self._h, n, bp1 - 1, _ptr(ab), bp1, _ptr(d), _ptr(e)), "sbr_band_to_tridiag")
        return d, e

    def tridiag_eigenvalues(self, d, e, lam=None):
        """Eigenvalues (ascending, float64 CUDA) of tridiag(d, e) by Sturm bisection on the GPU."""
        import torch

        n = int(d.shape[0])
        if d.dtype != torch.float64 or e.dtype != torch.float64 or not d.is_cuda or not e.is_cuda:
            raise ValueError("d, e must be float64 CUDA tensors")
        lam = torch.empty(n, dtype=torch.float64, device=d.device) if lam is None else lam
        check(lib().sbr_tridiag_eigenvalues(self._h, n, _ptr(d.contiguous()), _ptr(e.contiguous()), _ptr(lam)),
              "sbr_tridiag_eigenvalues")
        return lam

    def band_eigenvalues(self, ab, lam=None):
        """All eigenvalues of the band ``ab`` (stage two on the GPU: bulge chase + bisection)."""
        import torch

        n, bp1 = int(ab.shape[0]), int(ab.shape[1])
        if ab.dtype != torch.float32 or not ab.is_cuda or not ab.is_contiguous():
            raise ValueError("ab must be a contiguous (n, b+1) float32 CUDA tensor")
        lam = torch.empty(n, dtype=torch.float64, device=ab.device) if lam is None else lam
        check(lib().sbr_band_eigenvalues(self._h, n, bp1 - 1, _ptr(ab), bp1, _ptr(lam)), "sbr_band_eigenvalues")
        return lam

    def eigenvalues(self, A, b: int, nb: int, mode="fp16", lam=None):
        """Two-stage EVD, eigenvalues only (sbr_eigenvalues): A (overwritten) -> band -> lam (float64)."""
        import torch

        n = int(A.shape[0])
        if A.dim() != 2 or A.shape[1] != n or A.dtype != torch.float32 or not A.is_cuda or not A.is_contiguous():
            raise ValueError("A must be a contiguous square float32 CUDA tensor")
        lam = torch.empty(n, dtype=torch.float64, device=A.device) if lam is None else lam
        check(lib().sbr_eigenvalues(self._h, _mode(mode), n, int(b), int(nb), _ptr(A), n, _ptr(lam)),
              "sbr_eigenvalues")
        return lam

    def reduce_dist(self, A_local, n: int, b: int, nb: int, mode="fp16", want_w: bool = True, ab=None, w=None):
        """One n x n matrix across the handle's ranks (collective; include/sbr.h sbr_reduce_dist).

        ``A_local``: this rank's columns -- a contiguous float32 CUDA tensor of torch shape
        (ncols_loc, n) whose row lc is global column ``local_columns(n, nb, rank, nranks)[lc]``
        (``A[cols]`` for a symmetric torch matrix ``A``).  Returns ``(ab, w_local)``: the band
        (rank 0; None elsewhere, torch shape (n, b+1)) and this rank's W columns (same local
        layout as ``A_local``; None if ``want_w`` is False)."""
        import torch

        n = int(n)
        ncl = local_cols(n, nb, self.rank, self.nranks)
        if (A_local.dim() != 2 or tuple(A_local.shape) != (ncl, n) or A_local.dtype != torch.float32
                or not A_local.is_cuda or not A_local.is_contiguous()):
            raise ValueError(f"A_local must be a contiguous ({ncl}, {n}) float32 CUDA tensor")
        lead = self.rank == 0
        if lead and ab is None:
            ab = torch.empty((n, b + 1), dtype=torch.float32, device=A_local.device)
        if want_w and w is None and ncl > 0:
            w = torch.zeros((ncl, n), dtype=torch.float32, device=A_local.device)
        if not want_w:
            w = None
        check(lib().sbr_reduce_dist(self._h, _mode(mode), n, int(b), int(nb), _ptr(A_local), n,
                                    _ptr(ab) if lead else None, b + 1, _ptr(w), n), "sbr_reduce_dist")
        return (ab if lead else None), w

    def reduce_host(self, A, b: int, nb: int, mode="fp16", outputs: int = _lib.SBR_OUT_BAND, ab=None, w=None):
        """End-to-end variant on HOST buffers (torch CPU tensors, ideally pinned, or numpy).

        Copies A in, reduces, copies back the band (and A / W if selected in
        ``outputs``); returns after the results are on the host."""
        import torch

        n = int(A.shape[0])
        if ab is None:
            ab = torch.empty((n, b + 1), dtype=torch.float32, pin_memory=True)
        if (outputs & _lib.SBR_OUT_W) and w is None and n > b:
            w = torch.empty((n - b, n), dtype=torch.float32, pin_memory=True)
        check(lib().sbr_reduce_host(self._h, _mode(mode), n, int(b), int(nb), _ptr(A), n, _ptr(ab), b + 1,
                                    _ptr(w), n, int(outputs)), "sbr_reduce_host")
        return ab, w

    def generate_symmetric(self, seed: int, n: int, out=None):
        """Device twin of ``workloads.random_symmetric`` (bit-identical)."""
        import torch

        if out is None:
            out = torch.empty((n, n), dtype=torch.float32, device=f"cuda:{self.device}")
        check(lib().sbr_generate_symmetric(self._h, ctypes.c_uint64(seed & (2**64 - 1)), n, _ptr(out), n),
              "sbr_generate_symmetric")
        return out

    def sync(self) -> None:
        check(lib().sbr_sync(self._h), "sbr_sync")

    # -- instrumentation
    def set_kernel_timing(self, enable: bool) -> None:
        check(lib().sbr_set_kernel_timing(self._h, int(bool(enable))), "set_kernel_timing")

    def reset_kernel_stats(self) -> None:
        check(lib().sbr_reset_kernel_stats(self._h), "reset_kernel_stats")

    def kernel_stats(self, name: str) -> dict:
        kid = _lib.KERNEL_CLASSES[name]
        n = ctypes.c_int64()
        ms, by, fl = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
        check(lib().sbr_kernel_stats(self._h, kid, ctypes.byref(n), ctypes.byref(ms), ctypes.byref(by),
                                     ctypes.byref(fl)), "kernel_stats")
        return {"launches": n.value, "ms": ms.value, "bytes": by.value, "flops": fl.value}

    def panel_declines(self, reset: bool = True) -> int:
        """Test hook: CholeskyQR panels that declined (TSQR fallback) since the last reset."""
        c = ctypes.c_int64()
        check(lib().sbr_test_panel_declines(self._h, int(bool(reset)), ctypes.byref(c)), "panel_declines")
        return int(c.value)

    def launch_count(self) -> int:
        return int(lib().sbr_launch_count(self._h))


_DEFAULT = {}


def _default_handle(device: int) -> Handle:
    h = _DEFAULT.get(device)
    if h is None:
        h = _DEFAULT[device] = Handle(device)
    return h


def reduce(A, b: int, nb: int, mode="fp16", want_w: bool = True):
    """Module-level convenience: ``Handle(A.device.index).reduce(...)``."""
    return _default_handle(A.device.index or 0).reduce(A, b, nb, mode=mode, want_w=want_w)


def reduce_host(A, b: int, nb: int, mode="fp16", outputs: int = _lib.SBR_OUT_BAND, device: int = 0):
    return _default_handle(device).reduce_host(A, b, nb, mode=mode, outputs=outputs)


def generate_symmetric(seed: int, n: int, device: int = 0):
    return _default_handle(device).generate_symmetric(seed, n)


def band_to_dense(ab):
    """(n, b+1) band tensor (``ab[j, d] = B[j+d, j]``) -> dense symmetric (n, n) tensor (same device/dtype)."""
    import torch

    n, bp1 = ab.shape
    out = torch.zeros((n, n), dtype=ab.dtype, device=ab.device)
    j = torch.arange(n, device=ab.device)
    for d in range(bp1):
        jj = j[: n - d]
        out[jj + d, jj] = ab[: n - d, d]
        out[jj, jj + d] = ab[: n - d, d]
    return out
