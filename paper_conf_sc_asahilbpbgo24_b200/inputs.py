"""Seeded synthetic input generators shared by the tests, the bench and the
oracle legs.

This module holds NONE of the method's arithmetic (no B-splines, no
factorisation, no solve): only breakpoint recipes and random right-hand
sides, stated in DESIGN.md "Input recipe".  It imports neither ``oracle/`` nor
the CUDA binding, so both sides can draw the same inputs from it.

* breakpoints: uniform on [0, 1]; the deterministic "sin map"
  x_i = u_i + 0.5 sin(2 pi u_i) / (2 pi), u_i = i/N (cell-width
  ratio ~3, "non-uniform mesh ... steep gradients"); seeded
  jitter +-0.3 h of the interior breakpoints.
* right-hand sides: U(-1, 1) from numpy's counter-based Philox generator,
  keyed by the seed; column r of the (n, batch) array is RHS r.  Hermite
  derivative rows are scaled by (2 pi)^d.
* GYSELA-like 4-D slice f[y][v][mu][x]: smooth
  Maxwellian-like values plus 1e-3 U(-1, 1) noise.
"""
from __future__ import annotations

import numpy as np

PERIODIC, GREVILLE, HERMITE = 0, 1, 2
RHS_BLOCK = 4096


def bc_mixed(lo: int, hi: int) -> int:
    """Boundary-condition code of include/spline_builder.h for (lo, hi) ends."""
    return lo if lo == hi else lo | (hi << 4)


def bc_ends(bc: int) -> tuple[int, int]:
    return (bc, bc) if bc < 16 else (bc & 15, (bc >> 4) & 15)


def n_hermite_rows(degree: int, bc: int) -> tuple[int, int]:
    """Derivative rows at (x_0, x_N) -- the header's row-order convention."""
    nbc = (degree - 1) // 2 if degree % 2 else degree // 2
    lo, hi = bc_ends(bc)
    return (nbc if lo == HERMITE else 0, nbc if hi == HERMITE else 0)


def n_cells(degree: int, n_points: int, bc: int) -> int:
    """Number of cells N implied by (degree, n_points, bc) -- the counting
    convention of include/spline_builder.h, not method arithmetic."""
    if bc >= 16:
        lo, hi = n_hermite_rows(degree, bc)
        return n_points - degree + lo + hi
    if bc == PERIODIC:
        return n_points
    if bc == GREVILLE:
        return n_points - degree
    if bc == HERMITE:
        return n_points - 1 if degree % 2 else n_points
    raise ValueError(bc)


def nbasis(degree: int, n_points: int, bc: int) -> int:
    N = n_cells(degree, n_points, bc)
    return N if bc == PERIODIC else N + degree


def breakpoints(N: int, kind: str = "uniform", seed: int = 42) -> np.ndarray | None:
    """N+1 breakpoints on [0, 1].  ``uniform`` returns None (the library's
    knots == NULL convention); ``uniform_array`` returns them explicitly."""
    u = np.arange(N + 1, dtype=np.float64) / N
    if kind == "uniform":
        return None
    if kind == "uniform_array":
        return u
    if kind == "sin":
        x = u + 0.5 * np.sin(2.0 * np.pi * u) / (2.0 * np.pi)
        x[0], x[-1] = 0.0, 1.0
        return x
    if kind == "jitter":
        rng = np.random.Generator(np.random.Philox(key=seed))
        x = u.copy()
        x[1:-1] += rng.uniform(-0.3, 0.3, N - 1) / N
        return x
    raise ValueError(kind)


def rhs(n: int, batch: int, seed: int = 1234, dtype=np.float64, degree: int = 3, bc: int = PERIODIC,
        first: int = 0) -> np.ndarray:
    """(n, batch) batch-contiguous RHS, U(-1, 1).  RHS are drawn in blocks of
    RHS_BLOCK columns, block q from Philox keyed by (seed, q), so column r
    depends only on (seed, n, r): a shard [first, first+batch) of a global
    batch draws exactly the columns of the unsharded array."""
    b = np.empty((batch, n), dtype=np.float64)
    q0, q1 = first // RHS_BLOCK, (first + batch + RHS_BLOCK - 1) // RHS_BLOCK
    for q in range(q0, q1):
        g = np.random.Generator(np.random.Philox(key=(q << 64) | seed))
        blk = g.uniform(-1.0, 1.0, size=(RHS_BLOCK, n))
        lo, hi = max(first, q * RHS_BLOCK), min(first + batch, (q + 1) * RHS_BLOCK)
        b[lo - first:hi - first] = blk[lo - q * RHS_BLOCK:hi - q * RHS_BLOCK]
    b = b.T.copy()
    if bc != PERIODIC:
        nlo, nhi = n_hermite_rows(degree, bc)
        for d in range(1, nlo + 1):
            b[d - 1, :] *= (2.0 * np.pi) ** d
        for d in range(1, nhi + 1):
            b[n - nhi + d - 1, :] *= (2.0 * np.pi) ** d
    return np.ascontiguousarray(b.astype(dtype))


def rhs_device(n: int, batch: int, seed: int = 1234, first: int = 0, dtype=None, device="cuda",
               out=None):
    """Device-side twin of :func:`rhs` for batches too large for the host
    (C5: 8e6 RHS = 64 GB).  Same block structure: block q of RHS_BLOCK
    columns is U(-1, 1) from torch's CUDA Philox seeded with (seed, q), so a
    shard [first, first+batch) holds exactly the columns of the unsharded
    array.  (Values differ from the numpy generator of :func:`rhs`; parity
    tests copy the sampled input columns to the host.)  Returns (n, batch)."""
    import torch
    dtype = dtype or torch.float64
    x = out if out is not None else torch.empty((n, batch), dtype=dtype, device=device)
    g = torch.Generator(device=device)
    q0, q1 = first // RHS_BLOCK, (first + batch + RHS_BLOCK - 1) // RHS_BLOCK
    for q in range(q0, q1):
        g.manual_seed((seed * 1_000_003 + q) & 0x7FFFFFFFFFFFFFFF)
        blk = torch.rand((n, RHS_BLOCK), generator=g, dtype=torch.float64, device=device).mul_(2.0).sub_(1.0)
        lo, hi = max(first, q * RHS_BLOCK), min(first + batch, (q + 1) * RHS_BLOCK)
        x[:, lo - first:hi - first].copy_(blk[:, lo - q * RHS_BLOCK:hi - q * RHS_BLOCK])
    return x


def gysela_slice(ny: int = 64, nv: int = 64, nmu: int = 32, nx: int = 1024, seed: int = 7,
                 dtype=np.float64) -> np.ndarray:
    """f[y][v][mu][x], x contiguous."""
    g = np.random.Generator(np.random.Philox(key=seed))
    y = np.arange(ny) / ny
    v = np.linspace(-4.0, 4.0, nv)
    mu = np.linspace(0.0, 4.0, nmu)
    x = np.arange(nx) / nx
    base = np.exp(-0.5 * v[None, :, None, None] ** 2 - mu[None, None, :, None])
    mod = 1.0 + 0.1 * np.cos(2 * np.pi * x)[None, None, None, :] * np.cos(2 * np.pi * y)[:, None, None, None]
    f = base * mod + 1e-3 * g.uniform(-1.0, 1.0, size=(ny, nv, nmu, nx))
    return np.ascontiguousarray(f.astype(dtype))
