"""CPU oracle for the batched spline-coefficient build -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_sc_asahilbpbgo24_b200``) never imports it and shares
no code with it.

The arithmetic lives in ``spline_oracle.c`` (plain C, fp64; see its header for
the PAPER.md passages each step follows).  This module only builds that file
with gcc and marshals numpy arrays through ctypes.

Parity status: every oracle function is pinned by tests/test_oracle_pins.py
(closed forms, scipy, brute force, invariants); none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "spline_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

PERIODIC, GREVILLE, HERMITE = 0, 1, 2

_lib = None


def build(force: bool = False) -> str:
    """Compile spline_oracle.c -> liboracle.so (gcc, -O2, no fast-math)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        cmd = ["gcc", "-O2", "-fno-fast-math", "-fopenmp", "-std=c99", "-shared", "-fPIC",
               SRC, "-o", LIB + ".tmp", "-lm"]
        subprocess.check_call(cmd)
        os.replace(LIB + ".tmp", LIB)
    return LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(LIB)
        vp, i32, i64, dp = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_void_p
        lib.oracle_create.restype = vp
        lib.oracle_create.argtypes = [i32, i32, i32, dp, ctypes.POINTER(ctypes.c_int)]
        lib.oracle_destroy.argtypes = [vp]
        lib.oracle_nbasis.argtypes = [vp]
        lib.oracle_ncells.argtypes = [vp]
        lib.oracle_get_matrix.argtypes = [vp, dp]
        lib.oracle_get_row_scale.argtypes = [vp, dp]
        lib.oracle_get_rows.argtypes = [vp, dp, dp, dp]
        lib.oracle_handle_solve.argtypes = [vp, dp, i64, i64, i64, i32]
        lib.oracle_eval.argtypes = [vp, dp, i32, dp, i64, dp]
        lib.oracle_advect.argtypes = [vp, dp, i64, i64, i64, dp, i32]
        lib.oracle_solve_2d.argtypes = [vp, vp, dp, i64, i64, i32]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


class Oracle:
    """Collocation matrix + dense GEPP factorisation of one spline space."""

    def __init__(self, degree: int, n_points: int, bc: int, knots=None):
        lib = _load()
        self._knots = None if knots is None else np.ascontiguousarray(knots, dtype=np.float64)
        st = ctypes.c_int(0)
        kp = None if self._knots is None else _ptr(self._knots)
        self._h = lib.oracle_create(degree, n_points, bc, kp, ctypes.byref(st))
        if not self._h:
            raise ValueError(f"oracle_create failed with status {st.value}")
        self.degree, self.bc = degree, bc
        self.n = lib.oracle_nbasis(self._h)
        self.N = lib.oracle_ncells(self._h)

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.oracle_destroy(self._h)
            self._h = None

    def matrix(self) -> np.ndarray:
        A = np.empty((self.n, self.n), dtype=np.float64)
        _lib.oracle_get_matrix(self._h, _ptr(A))
        return A

    def row_scale(self) -> np.ndarray:
        s = np.empty(self.n, dtype=np.float64)
        _lib.oracle_get_row_scale(self._h, _ptr(s))
        return s

    def rows(self):
        """(points, cells, derivative orders) of the n interpolation rows."""
        x = np.empty(self.n, dtype=np.float64)
        c = np.empty(self.n, dtype=np.int32)
        d = np.empty(self.n, dtype=np.int32)
        _lib.oracle_get_rows(self._h, _ptr(x), _ptr(c), _ptr(d))
        return x, c, d

    def solve_(self, rhs: np.ndarray, batch_stride: int | None = None, point_stride: int | None = None,
               batch: int | None = None, nthreads: int = 0) -> np.ndarray:
        """In-place solve.  Default layout: rhs of shape (n, batch), C order
        (batch contiguous: batch_stride=1, point_stride=batch)."""
        assert rhs.dtype == np.float64 and rhs.flags.c_contiguous
        if batch is None:
            assert rhs.ndim == 2 and rhs.shape[0] == self.n
            batch = rhs.shape[1]
        if batch_stride is None:
            batch_stride, point_stride = 1, rhs.shape[1]
        st = _lib.oracle_handle_solve(self._h, _ptr(rhs), int(batch), int(batch_stride), int(point_stride),
                                      int(nthreads))
        if st:
            raise RuntimeError(f"oracle solve failed: {st}")
        return rhs

    def solve(self, b: np.ndarray, nthreads: int = 0) -> np.ndarray:
        """x = A^{-1} b for b of shape (n,) or (n, batch) (batch contiguous)."""
        x = np.array(b, dtype=np.float64, order="C", copy=True)
        if x.ndim == 1:
            x = x.reshape(self.n, 1)
            return self.solve_(x, nthreads=nthreads)[:, 0]
        return self.solve_(x, nthreads=nthreads)

    def eval(self, coef: np.ndarray, xs: np.ndarray, deriv: int = 0) -> np.ndarray:
        coef = np.ascontiguousarray(coef, dtype=np.float64)
        xs = np.ascontiguousarray(xs, dtype=np.float64)
        out = np.empty(xs.shape[0], dtype=np.float64)
        _lib.oracle_eval(self._h, _ptr(coef), int(deriv), _ptr(xs), int(xs.shape[0]), _ptr(out))
        return out

    def advect(self, f: np.ndarray, shift: np.ndarray, nthreads: int = 0) -> np.ndarray:
        """One Algorithm-2 step on f of shape (n, batch)
        (batch contiguous): spline build + evaluation at xi_i - shift[r]."""
        out = np.array(f, dtype=np.float64, order="C", copy=True)
        sh = np.ascontiguousarray(shift, dtype=np.float64)
        assert out.ndim == 2 and out.shape[0] == self.n and sh.shape == (out.shape[1],)
        st = _lib.oracle_advect(self._h, _ptr(out), int(out.shape[1]), 1, int(out.shape[1]), _ptr(sh), int(nthreads))
        if st:
            raise RuntimeError(f"oracle advect failed: {st}")
        return out

    def residual(self, x: np.ndarray, b: np.ndarray) -> float:
        """Interpolation residual on the equilibrated rows (R8):
        max_i |s_i (A x - b)_i| / max_i |s_i b_i|, per RHS, max over RHS."""
        A = self.matrix()
        s = self.row_scale()[:, None]
        x2 = x.reshape(self.n, -1)
        b2 = b.reshape(self.n, -1)
        r = np.abs(s * (A @ x2 - b2)).max(axis=0)
        den = np.abs(s * b2).max(axis=0)
        den[den == 0] = 1.0
        return float((r / den).max())


def solve_2d(o1: Oracle, o2: Oracle, f: np.ndarray, nthreads: int = 0) -> np.ndarray:
    """Tensor-product coefficients: f of shape (batch, n2, n1)
    or (n2, n1), dim 1 (o1) fastest; returns C = A1^{-1} F A2^{-T} per grid."""
    c = np.array(f, dtype=np.float64, order="C", copy=True)
    g = c.reshape((1,) + c.shape) if c.ndim == 2 else c
    assert g.ndim == 3 and g.shape[1] == o2.n and g.shape[2] == o1.n
    st = _lib.oracle_solve_2d(o1._h, o2._h, _ptr(g), int(g.shape[0]), int(o1.n * o2.n), int(nthreads))
    if st:
        raise RuntimeError(f"oracle solve_2d failed: {st}")
    return c


def eval_2d(o1: Oracle, o2: Oracle, coef: np.ndarray, xs: np.ndarray, ys: np.ndarray) -> np.ndarray:
    """S(x, y) = sum_{j1,j2} C[j2][j1] B1_{j1}(x) B2_{j2}(y) on the grid xs x ys
    (result [len(ys)][len(xs)]), by 1-D evaluations along each dimension."""
    coef = np.asarray(coef, dtype=np.float64)
    # along dim 2 first: G[y][j1] = sum_{j2} C[j2][j1] B2_{j2}(y)
    G = np.stack([o2.eval(np.ascontiguousarray(coef[:, j1]), ys) for j1 in range(o1.n)], axis=1)
    return np.stack([o1.eval(np.ascontiguousarray(G[q]), xs) for q in range(len(ys))], axis=0)


def rel_coef_error(x: np.ndarray, ref: np.ndarray) -> float:
    """Max over RHS of max_j |x - ref| / max_j |ref| (R7)."""
    x2 = np.asarray(x, dtype=np.float64).reshape(ref.shape[0], -1)
    r2 = np.asarray(ref, dtype=np.float64).reshape(ref.shape[0], -1)
    num = np.abs(x2 - r2).max(axis=0)
    den = np.abs(r2).max(axis=0)
    den[den == 0] = 1.0
    return float((num / den).max())
