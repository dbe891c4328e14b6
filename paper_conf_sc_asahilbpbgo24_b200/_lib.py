"""Thin ctypes binding of include/spline_builder.h -- argument marshalling
only.  Every step of the solve runs in libsplinebuilder.so (host create in
C++, the solve in the sm_100a kernels).  There is no CPU fallback: if the
library is missing or was built without the kernels, loading fails loudly.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# SB_LIB_PATH: load another build of the same library (A/B experiments)
LIB_PATH = os.environ.get("SB_LIB_PATH") or os.path.join(HERE, "libsplinebuilder.so")

SB_PERIODIC, SB_GREVILLE, SB_HERMITE = 0, 1, 2
SB_F64, SB_F32 = 0, 1
SB_OK, SB_INVALID_ARG, SB_SINGULAR, SB_CUDA, SB_NOMEM, SB_UNSUPPORTED = range(6)
SB_FLAG_HOST_ONLY, SB_FLAG_DEVICE_UPDATE = 1, 2

# every symbol include/spline_builder.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "spline_builder_create", "spline_builder_create_ex", "spline_builder_update", "spline_builder_update_device",
    "spline_builder_update_status", "spline_builder_solve", "spline_builder_solve_f32",
    "spline_builder_solve_strided", "spline_builder_solve_slabs", "spline_builder_solve_2d", "spline_builder_advect", "spline_builder_solve_host", "spline_builder_destroy",
    "spline_builder_get_info", "spline_builder_nbasis", "spline_builder_get_blocks",
    "spline_builder_solve_cpu_plan", "spline_builder_last_error", "spline_builder_last_status",
    "spline_builder_last_kernel",
    "spline_builder_version",
]


class SplineBuilderInfo(ctypes.Structure):
    _fields_ = [(name, ctypes.c_int) for name in (
        "degree", "bc", "n_cells", "nbasis", "split_lo", "split_hi", "k", "q_kl", "q_ku", "q_type",
        "nnz_lambda", "nnz_beta", "beta_rows_head", "beta_rows_tail", "nnz_Lambda", "nnz_gamma", "n_segments",
        "seg_len",
        "carry_fwd", "carry_bwd")] + [("max_pivot_growth", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class SplineBuilderError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"spline_builder status {status}: {msg}")
        self.status = status


_lib = None


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libsplinebuilder.so; raises if it is absent (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not found: build it with `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(path)
    vp, i32, i64, dp = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_void_p
    lib.spline_builder_create.restype = vp
    lib.spline_builder_create.argtypes = [i32, i32, i32, dp]
    lib.spline_builder_create_ex.restype = vp
    lib.spline_builder_create_ex.argtypes = [i32, i32, i32, dp, i32, i32, i32]
    for name in ("spline_builder_solve", "spline_builder_solve_f32"):
        getattr(lib, name).restype = i32
        getattr(lib, name).argtypes = [vp, dp, i64, i64, vp]
    lib.spline_builder_solve_strided.restype = i32
    lib.spline_builder_solve_strided.argtypes = [vp, dp, i32, i64, i64, i64, vp]
    lib.spline_builder_solve_slabs.restype = i32
    lib.spline_builder_solve_slabs.argtypes = [vp, dp, i32, i64, i64, i64, i64, vp]
    lib.spline_builder_solve_2d.restype = i32
    lib.spline_builder_solve_2d.argtypes = [vp, vp, dp, i32, i64, i64, vp]
    lib.spline_builder_advect.restype = i32
    lib.spline_builder_advect.argtypes = [vp, dp, i32, i64, i64, i64, dp, vp]
    lib.spline_builder_solve_host.restype = i32
    lib.spline_builder_solve_host.argtypes = [vp, dp, i32, i64, i64]
    lib.spline_builder_update.restype = i32
    lib.spline_builder_update.argtypes = [vp, dp]
    lib.spline_builder_update_device.restype = i32
    lib.spline_builder_update_device.argtypes = [vp, dp, vp]
    lib.spline_builder_update_status.restype = i32
    lib.spline_builder_update_status.argtypes = [vp]
    lib.spline_builder_destroy.restype = None
    lib.spline_builder_destroy.argtypes = [vp]
    lib.spline_builder_get_info.restype = i32
    lib.spline_builder_get_info.argtypes = [vp, ctypes.POINTER(SplineBuilderInfo)]
    lib.spline_builder_nbasis.restype = i64
    lib.spline_builder_nbasis.argtypes = [vp]
    lib.spline_builder_get_blocks.restype = i32
    lib.spline_builder_get_blocks.argtypes = [vp] + [dp] * 7
    lib.spline_builder_solve_cpu_plan.restype = i32
    lib.spline_builder_solve_cpu_plan.argtypes = [vp, dp, i64, i64, i64]
    lib.spline_builder_last_error.restype = ctypes.c_char_p
    lib.spline_builder_last_error.argtypes = []
    lib.spline_builder_last_status.restype = i32
    lib.spline_builder_last_status.argtypes = []
    lib.spline_builder_last_kernel.restype = ctypes.c_char_p
    lib.spline_builder_last_kernel.argtypes = []
    lib.spline_builder_version.restype = ctypes.c_char_p
    lib.spline_builder_version.argtypes = []
    _lib = lib
    return lib


def last_error() -> str:
    return load().spline_builder_last_error().decode()


def last_kernel() -> str:
    """Kernel (and configuration) of the calling thread's last solve."""
    return load().spline_builder_last_kernel().decode()


def check(status: int) -> None:
    if status != SB_OK:
        raise SplineBuilderError(status, last_error())
