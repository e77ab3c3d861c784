"""Python API over libsbr (marshalling only; see include/sbr.h for semantics)."""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import check, lib

MODES = {"fp16": _lib.SBR_FP16_FP32ACC, "3xtf32": _lib.SBR_3XTF32}


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


class Handle:
    """One libsbr handle: a device, a CUDA stream (torch's current stream by default)
    and the reduction workspace it owns."""

    def __init__(self, device: int = 0, stream=None):
        import torch

        self.device = int(device)
        if stream is None:
            stream = torch.cuda.current_stream(self.device)
        self._stream = stream
        h = ctypes.c_void_p()
        check(lib().sbr_create(ctypes.byref(h), self.device, ctypes.c_void_p(stream.cuda_stream)), "sbr_create")
        self._h = h

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
        the handle's stream; no host synchronisation except the input check.
        """
        import torch

        n = int(A.shape[0])
        if A.dim() != 2 or A.shape[1] != n or A.dtype != torch.float32 or not A.is_cuda or not A.is_contiguous():
            raise ValueError("A must be a contiguous square float32 CUDA tensor")
        if ab is None:
            ab = torch.empty((n, b + 1), dtype=torch.float32, device=A.device)
        if want_w and w is None and n > b:
            w = torch.empty((max(n - b, 1), n), dtype=torch.float32, device=A.device)
        if not want_w:
            w = None
        check(lib().sbr_reduce(self._h, _mode(mode), n, int(b), int(nb), _ptr(A), n, _ptr(ab), b + 1,
                               _ptr(w), n), "sbr_reduce")
        return ab, w

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
