"""B200-native batched spline-coefficient builder.

Python face of ``include/spline_builder.h``: :class:`SplineBuilder` wraps one
handle (one collocation matrix, factored once at create) and
solves batches of right-hand sides in place on the GPU (Algorithm 1,
P:86-91).  torch is used only for device memory and streams; the names
mirror the C ABI and every call is argument marshalling into
``libsplinebuilder.so``.
"""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import (SB_F32, SB_F64, SB_FLAG_DEVICE_UPDATE, SB_FLAG_HOST_ONLY, SB_GREVILLE, SB_HERMITE, SB_PERIODIC, SplineBuilderError,
                   SplineBuilderInfo)

PERIODIC, GREVILLE, HERMITE = SB_PERIODIC, SB_GREVILLE, SB_HERMITE


def bc_mixed(lo: int, hi: int) -> int:
    """SB_BC(lo, hi) of include/spline_builder.h: different conditions at x_0 / x_N."""
    return lo if lo == hi else lo | (hi << 4)

last_kernel = _lib.last_kernel

__all__ = ["last_kernel", "SplineBuilder", "SplineBuilderError", "PERIODIC", "GREVILLE", "HERMITE", "load_library", "solve_2d_", "bc_mixed"]


def n_cells_of(degree: int, n_points: int, bc: int) -> int:
    """Number of cells N (so N+1 breakpoints) fixed by (degree, n_points, bc),
    as stated for spline_builder_create in include/spline_builder.h."""
    p = int(degree)
    nbc = (p - 1) // 2 if p % 2 else p // 2
    if bc == PERIODIC:
        return int(n_points)
    if bc == GREVILLE:
        return int(n_points) - p
    if bc == HERMITE:
        return int(n_points) - 1 if p % 2 else int(n_points)
    lo, hi = bc & 15, (bc >> 4) & 15
    return int(n_points) - p + (nbc if lo == HERMITE else 0) + (nbc if hi == HERMITE else 0)


def _knots_arg(knots, n_cells: int):
    """Contiguous fp64 copy of the breakpoints, checked to hold N+1 values
    (the C side reads exactly that many)."""
    import numpy as np
    kn = np.ascontiguousarray(knots, dtype=np.float64)
    if kn.ndim != 1 or kn.shape[0] != n_cells + 1:
        raise ValueError(f"knots must be a 1-D array of N+1 = {n_cells + 1} breakpoints, got shape {kn.shape}")
    return kn


def _check_extent(t, last_index: int, what: str = "rhs"):
    """The C side addresses elements [0, last_index] from t.data_ptr(): they
    must lie inside t's storage."""
    avail = (t.untyped_storage().nbytes() - t.storage_offset() * t.element_size()) // t.element_size()
    if last_index >= avail:
        raise ValueError(f"{what}: strides address element {last_index} but only {avail} are allocated")


def load_library():
    """Load the native library (raises ImportError if it was not built)."""
    return _lib.load()


def _stream_handle(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


class SplineBuilder:
    """One spline space (degree, points, boundary condition, breakpoints).

    ``split`` = (split_lo, split_hi) forces the Schur split of Eq. 3
    (default: chosen at create).  ``host_only`` factors without touching the
    GPU (inspection / CPU tests)."""

    def __init__(self, degree: int, n_points: int, bc: int = PERIODIC, knots=None, split=None,
                 host_only: bool = False, device_update: bool = False):
        lib = _lib.load()
        self._lib = lib
        kbuf = None
        if knots is not None:
            self._knots = _knots_arg(knots, n_cells_of(degree, n_points, bc))
            kbuf = ctypes.c_void_p(self._knots.ctypes.data)
        lo, hi = (-1, -1) if split is None else split
        flags = (SB_FLAG_HOST_ONLY if host_only else 0) | (SB_FLAG_DEVICE_UPDATE if device_update else 0)
        h = lib.spline_builder_create_ex(int(degree), int(n_points), int(bc), kbuf, int(lo), int(hi), flags)
        if not h:
            raise SplineBuilderError(lib.spline_builder_last_status(), _lib.last_error())
        self._h = ctypes.c_void_p(h)
        self.degree, self.n_points, self.bc = degree, n_points, bc
        self.n = int(lib.spline_builder_nbasis(self._h))

    # ------------------------------------------------------------ lifetime
    def close(self):
        if getattr(self, "_h", None):
            self._lib.spline_builder_destroy(self._h)
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

    def update(self, knots=None):
        """New breakpoints for the same degree / n_points / bc / split request
        (``spline_builder_update``): the factors are rebuilt and replaced in
        the handle.  Synchronise streams that use this handle first.  On
        error the handle keeps its previous mesh."""
        kbuf = None
        if knots is not None:
            kn = _knots_arg(knots, self.info()["n_cells"])
            kbuf = ctypes.c_void_p(kn.ctypes.data)
        _lib.check(self._lib.spline_builder_update(self._h, kbuf))
        if knots is not None:
            self._knots = kn

    def update_device_(self, knots=None, stream=None):
        """New breakpoints factorised on the device (``spline_builder_update_device``;
        handle created with ``device_update=True``): ``knots`` is a CUDA fp64
        tensor of N+1 breakpoints (None: uniform).  Asynchronous on ``stream``;
        :meth:`update_status` returns the outcome (the previous mesh is kept on
        failure)."""
        import torch
        kp = None
        if knots is not None:
            if not (isinstance(knots, torch.Tensor) and knots.is_cuda and knots.dtype == torch.float64):
                raise TypeError("knots must be a CUDA float64 tensor")
            if knots.dim() != 1 or not knots.is_contiguous() or knots.numel() != self.info()["n_cells"] + 1:
                raise ValueError(f"knots must be a contiguous 1-D tensor of N+1 = {self.info()['n_cells'] + 1} values")
            self._dev_knots = knots  # kept alive until the kernel has read it
            kp = ctypes.c_void_p(knots.data_ptr())
        _lib.check(self._lib.spline_builder_update_device(self._h, kp, _stream_handle(stream)))
        return self

    def update_status(self) -> None:
        """Wait for the last :meth:`update_device_`; raises SplineBuilderError if it
        was rejected (the previous mesh stays in place)."""
        try:
            _lib.check(self._lib.spline_builder_update_status(self._h))
        finally:
            self._dev_knots = None

    # ------------------------------------------------------------- queries
    def info(self) -> dict:
        inf = SplineBuilderInfo()
        _lib.check(self._lib.spline_builder_get_info(self._h, ctypes.byref(inf)))
        return inf.as_dict()

    def blocks(self):
        """(lambda COO, beta COO, delta') as numpy arrays (host copies)."""
        import numpy as np
        inf = self.info()
        k, nl, nb = inf["k"], inf["nnz_lambda"], inf["nnz_beta"]
        lr, lc, lv = np.empty(nl, np.int32), np.empty(nl, np.int32), np.empty(nl)
        br, bc, bv = np.empty(nb, np.int32), np.empty(nb, np.int32), np.empty(nb)
        dp = np.empty((k, k))
        p = lambda a: ctypes.c_void_p(a.ctypes.data)  # noqa: E731
        _lib.check(self._lib.spline_builder_get_blocks(self._h, p(lr), p(lc), p(lv), p(br), p(bc), p(bv), p(dp)))
        return (lr, lc, lv), (br, bc, bv), dp

    # -------------------------------------------------------------- solves
    def solve_(self, rhs, batch_stride: int | None = None, stream=None):
        """In-place solve of a CUDA tensor (fp64 or fp32).  Layouts:
        (n, batch) contiguous -> batch-contiguous; (batch, n) contiguous ->
        point-contiguous.  Anything else: :meth:`solve_strided_`."""
        import torch
        if not rhs.is_cuda:
            raise ValueError("rhs must be a CUDA tensor (use solve_host for host data)")
        if rhs.dtype not in (torch.float64, torch.float32):
            raise TypeError("rhs must be float64 or float32")
        if rhs.dim() != 2 or not rhs.is_contiguous():
            raise ValueError("rhs must be a contiguous 2-D tensor")
        if batch_stride is None:
            if rhs.shape[0] == self.n:
                batch, bs = rhs.shape[1], 1
            elif rhs.shape[1] == self.n:
                batch, bs = rhs.shape[0], self.n
            else:
                raise ValueError(f"no dimension of size n={self.n}")
        else:
            bs = int(batch_stride)
            if bs == 1:
                if rhs.shape[0] != self.n:
                    raise ValueError(f"batch_stride=1 needs shape (n={self.n}, batch), got {tuple(rhs.shape)}")
                batch = rhs.shape[1]
            else:
                if bs != rhs.shape[1] or rhs.shape[1] < self.n:
                    raise ValueError(f"batch_stride={bs} needs shape (batch, {bs}) with {bs} >= n={self.n}, "
                                     f"got {tuple(rhs.shape)}")
                batch = rhs.shape[0]
        fn = self._lib.spline_builder_solve if rhs.dtype == torch.float64 else self._lib.spline_builder_solve_f32
        _lib.check(fn(self._h, ctypes.c_void_p(rhs.data_ptr()), int(batch), int(bs), _stream_handle(stream)))
        return rhs

    def solve_strided_(self, rhs, batch: int, batch_stride: int, point_stride: int, stream=None):
        import torch
        if not rhs.is_cuda:
            raise ValueError("rhs must be a CUDA tensor")
        if rhs.dtype not in (torch.float64, torch.float32):
            raise TypeError("rhs must be float64 or float32")
        if batch > 0:
            _check_extent(rhs, (batch - 1) * batch_stride + (self.n - 1) * point_stride)
        dt = SB_F64 if rhs.dtype == torch.float64 else SB_F32
        _lib.check(self._lib.spline_builder_solve_strided(self._h, ctypes.c_void_p(rhs.data_ptr()), dt, int(batch),
                                                          int(batch_stride), int(point_stride),
                                                          _stream_handle(stream)))
        return rhs

    def solve_slabs_(self, rhs, batch: int, ld: int, nslab: int, slab_stride: int, stream=None):
        """In-place solve of nslab batch-contiguous (n, batch) blocks, element
        (j, r, q) at rhs[q*slab_stride + j*ld + r] (spline_builder_solve_slabs)."""
        import torch
        if not rhs.is_cuda:
            raise ValueError("rhs must be a CUDA tensor")
        if rhs.dtype not in (torch.float64, torch.float32):
            raise TypeError("rhs must be float64 or float32")
        if batch > 0 and nslab > 0:
            _check_extent(rhs, (nslab - 1) * slab_stride + (self.n - 1) * ld + batch - 1)
        dt = SB_F64 if rhs.dtype == torch.float64 else SB_F32
        _lib.check(self._lib.spline_builder_solve_slabs(self._h, ctypes.c_void_p(rhs.data_ptr()), dt, int(batch),
                                                        int(ld), int(nslab), int(slab_stride),
                                                        _stream_handle(stream)))
        return rhs

    def advect_(self, f, shift, batch_stride: int | None = None, stream=None):
        """One semi-Lagrangian step of Algorithm 2, in
        place: every RHS line of f (CUDA tensor, layouts as :meth:`solve_`) is
        replaced by its spline evaluated at xi_i - shift[r] (periodic spaces).
        ``shift``: CUDA fp64 tensor of batch displacements."""
        import torch
        if not (f.is_cuda and shift.is_cuda):
            raise ValueError("f and shift must be CUDA tensors")
        if shift.dtype != torch.float64 or not shift.is_contiguous():
            raise TypeError("shift must be a contiguous float64 tensor")
        if f.dim() != 2 or not f.is_contiguous():
            raise ValueError("f must be a contiguous 2-D tensor")
        if batch_stride is None:
            if f.shape[0] == self.n:
                batch, bs, pst = f.shape[1], 1, f.shape[1]
            elif f.shape[1] == self.n:
                batch, bs, pst = f.shape[0], self.n, 1
            else:
                raise ValueError(f"no dimension of size n={self.n}")
        else:
            bs = int(batch_stride)
            if bs == 1 and f.shape[0] != self.n:
                raise ValueError(f"batch_stride=1 needs shape (n={self.n}, batch), got {tuple(f.shape)}")
            if bs != 1 and (bs != f.shape[1] or bs < self.n):
                raise ValueError(f"batch_stride={bs} needs shape (batch, {bs}) with {bs} >= n={self.n}")
            batch, pst = (f.shape[1], f.shape[1]) if bs == 1 else (f.shape[0], 1)
        if shift.numel() != batch:
            raise ValueError("shift must have one entry per right-hand side")
        dt = SB_F64 if f.dtype == torch.float64 else SB_F32
        _lib.check(self._lib.spline_builder_advect(self._h, ctypes.c_void_p(f.data_ptr()), dt, int(batch), int(bs),
                                                   int(pst), ctypes.c_void_p(shift.data_ptr()),
                                                   _stream_handle(stream)))
        return f

    def solve_host_(self, arr, ld: int | None = None):
        """End-to-end solve of host memory (numpy array or CPU tensor of shape
        (n, >=batch), row-major).  Pinned memory gives full PCIe bandwidth."""
        try:
            import torch
            is_t = isinstance(arr, torch.Tensor)
        except ImportError:  # pragma: no cover
            is_t = False
        if is_t:
            if arr.is_cuda:
                raise ValueError("solve_host_ takes host memory (use solve_ for CUDA tensors)")
            if arr.dtype not in (torch.float64, torch.float32):
                raise TypeError("host array must be float64 or float32")
            if arr.dim() != 2 or arr.stride(1) != 1:
                raise ValueError("host array must be 2-D (n, batch) with unit inner stride")
            dt = SB_F64 if arr.dtype == torch.float64 else SB_F32
            ptr, batch, ld0 = arr.data_ptr(), arr.shape[1], arr.stride(0)
        else:
            import numpy as np
            if arr.dtype not in (np.float64, np.float32):
                raise TypeError("host array must be float64 or float32")
            if arr.ndim != 2 or arr.strides[1] != arr.itemsize or arr.strides[0] % arr.itemsize:
                raise ValueError("host array must be 2-D (n, batch) with unit inner stride")
            if not arr.flags.writeable:
                raise ValueError("host array must be writeable (the solve is in place)")
            dt = SB_F64 if arr.dtype == np.float64 else SB_F32
            ptr, batch, ld0 = arr.ctypes.data, arr.shape[1], arr.strides[0] // arr.itemsize
        if arr.shape[0] != self.n:
            raise ValueError(f"host array must have n={self.n} rows, got {arr.shape[0]}")
        if ld is not None and ld != ld0:
            raise ValueError(f"ld={ld} differs from the array's row stride {ld0}")
        _lib.check(self._lib.spline_builder_solve_host(self._h, ctypes.c_void_p(ptr), dt, int(batch),
                                                       int(ld if ld is not None else ld0)))
        return arr

    def solve_cpu_plan_(self, arr):
        """Host fp64 run of the same factorisation (create's self-check path;
        for tests of the host plan only, not a product solve path)."""
        import numpy as np
        assert arr.dtype == np.float64 and arr.flags.c_contiguous and arr.shape[0] == self.n
        _lib.check(self._lib.spline_builder_solve_cpu_plan(self._h, ctypes.c_void_p(arr.ctypes.data),
                                                           int(arr.shape[1]), 1, int(arr.shape[1])))
        return arr


def solve_2d_(h1: SplineBuilder, h2: SplineBuilder, f, stream=None):
    """Tensor-product coefficients in place (spline_builder_solve_2d):
    f is a contiguous CUDA tensor of shape (batch, n2, n1) or (n2, n1), dim 1
    (h1, size n1) fastest; on exit C = A1^{-1} F A2^{-T} for every grid."""
    import torch
    if not f.is_cuda or not f.is_contiguous():
        raise ValueError("f must be a contiguous CUDA tensor")
    if f.dtype not in (torch.float64, torch.float32):
        raise TypeError("f must be float64 or float32")
    shp = tuple(f.shape)
    if len(shp) == 2:
        shp = (1,) + shp
    if len(shp) != 3 or shp[1] != h2.n or shp[2] != h1.n:
        raise ValueError(f"f must have shape (batch, {h2.n}, {h1.n})")
    dt = SB_F64 if f.dtype == torch.float64 else SB_F32
    _lib.check(h1._lib.spline_builder_solve_2d(h1._h, h2._h, ctypes.c_void_p(f.data_ptr()), dt, int(shp[0]),
                                               int(shp[1] * shp[2]), _stream_handle(stream)))
    return f
