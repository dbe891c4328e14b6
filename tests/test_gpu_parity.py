"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs (BASELINE.json tolerances):
max relative coefficient error <= 1e-12 (fp64) / 1e-5 (fp32), interpolation
residual <= 1e-12 (fp64).  Run on a B200 with ``pytest -m gpu``.
"""
import numpy as np
import pytest

import oracle
from oracle import GREVILLE, HERMITE, PERIODIC, Oracle, rel_coef_error
from paper_conf_sc_asahilbpbgo24_b200 import inputs

pytestmark = pytest.mark.gpu

TOL64 = 1e-12
TOL32 = 1e-5


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def make(p, n_points, bc, kind):
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    N = inputs.n_cells(p, n_points, bc)
    x = inputs.breakpoints(N, kind)
    return SplineBuilder(p, n_points, bc, x), Oracle(p, n_points, bc, x)


def gpu_solve(torch, sb, b, dtype=None):
    t = torch.from_numpy(b if dtype is None else b.astype(dtype)).cuda()
    sb.solve_(t)
    torch.cuda.synchronize()
    return t.cpu().numpy()


CASES = [
    # (degree, n_points, bc, mesh)
    (3, 16, PERIODIC, "uniform"),      # C1
    (3, 1000, PERIODIC, "uniform"),    # C2 shape
    (4, 1000, PERIODIC, "uniform"),
    (5, 1000, PERIODIC, "uniform"),
    (3, 1000, PERIODIC, "sin"),
    (4, 1000, PERIODIC, "jitter"),
    (5, 1000, PERIODIC, "jitter"),
    (5, 1000, GREVILLE, "sin"),        # C3 Greville
    (5, 996, HERMITE, "sin"),          # C3 Hermite
    (3, 1024, PERIODIC, "uniform"),    # C4 shape
    (3, 200, GREVILLE, "jitter"),
    (3, 200, HERMITE, "uniform"),
    (4, 200, HERMITE, "sin"),
    (1, 50, PERIODIC, "uniform"),
    (2, 50, PERIODIC, "jitter"),
    (2, 40, GREVILLE, "sin"),
    (3, 5, PERIODIC, "uniform"),
    (5, 8, GREVILLE, "uniform"),
    (3, 33, PERIODIC, "uniform"),
    (3, 64, PERIODIC, "jitter"),
    # mixed ends (NEXT row f4): Hermite at one end, Greville at the other
    (5, 998, HERMITE | (GREVILLE << 4), "sin"),
    (3, 200, GREVILLE | (HERMITE << 4), "jitter"),
    (4, 150, HERMITE | (GREVILLE << 4), "uniform"),
    (2, 60, GREVILLE | (HERMITE << 4), "sin"),
]


@pytest.mark.parametrize("case", CASES, ids=[f"p{c[0]}-n{c[1]}-bc{c[2]}-{c[3]}" for c in CASES])
@pytest.mark.parametrize("batch", [1, 37, 256, 1000])
def test_parity_fp64_batch_contiguous(torch_cuda, case, batch):
    p, npts, bc, kind = case
    sb, o = make(p, npts, bc, kind)
    b = inputs.rhs(sb.n, batch, seed=1234 + batch, degree=p, bc=bc)
    ref = o.solve(b)
    got = gpu_solve(torch_cuda, sb, b)
    err = rel_coef_error(got, ref)
    assert err <= TOL64, (case, batch, err)
    assert o.residual(got, b) <= TOL64


@pytest.mark.parametrize("case", [c for c in CASES if c[1] >= 16][:10])
def test_parity_fp32(torch_cuda, case):
    p, npts, bc, kind = case
    sb, o = make(p, npts, bc, kind)
    b = inputs.rhs(sb.n, 300, seed=77, degree=p, bc=bc)
    b32 = b.astype(np.float32)
    ref = o.solve(b32.astype(np.float64))  # oracle on the fp32-rounded inputs
    got = gpu_solve(torch_cuda, sb, b32)
    assert got.dtype == np.float32
    assert rel_coef_error(got.astype(np.float64), ref) <= TOL32


@pytest.mark.parametrize("n_points,dtype", [(1024, np.float64), (1024, np.float32), (1000, np.float64)])
def test_parity_point_contiguous(torch_cuda, n_points, dtype):
    """C4 layout: x contiguous, batch_stride = n (transpose path)."""
    torch = torch_cuda
    sb, o = make(3, n_points, PERIODIC, "uniform")
    f = inputs.gysela_slice(4, 8, 4, n_points, dtype=np.float64).reshape(-1, n_points)  # (batch, n)
    ref = o.solve(np.ascontiguousarray(f.T.astype(dtype).astype(np.float64)))
    t = torch.from_numpy(np.ascontiguousarray(f.astype(dtype))).cuda()
    sb.solve_(t)  # (batch, n) -> point-contiguous
    torch.cuda.synchronize()
    got = t.cpu().numpy().T.astype(np.float64)
    assert rel_coef_error(got, ref) <= (TOL64 if dtype == np.float64 else TOL32)


@pytest.mark.parametrize("case", [(5, 1000, GREVILLE, "sin"), (5, 996, HERMITE, "sin"), (5, 1000, PERIODIC, "jitter"),
                                  (4, 1000, PERIODIC, "uniform"), (3, 200, GREVILLE | (HERMITE << 4), "jitter"),
                                  (2, 40, GREVILLE, "sin")],
                         ids=lambda c: f"p{c[0]}-n{c[1]}-bc{c[2]}-{c[3]}")
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_parity_point_contiguous_corners(torch_cuda, case, dtype):
    """Point layout (warp kernel) for delta orders k = 2..6 and mixed ends:
    the fp64 corner runs on registers of every lane (getrs + gamma rows on
    parallel lanes), the fp32 one on lane 0."""
    torch = torch_cuda
    p, npts, bc, kind = case
    sb, o = make(p, npts, bc, kind)
    B = 333
    b = inputs.rhs(sb.n, B, seed=808, degree=p, bc=bc).astype(dtype)
    t = torch.from_numpy(np.ascontiguousarray(b.T)).cuda()
    sb.solve_(t)
    torch.cuda.synchronize()
    got = t.cpu().numpy().T.astype(np.float64)
    b64 = b.astype(np.float64)
    ref = o.solve(b64)
    assert rel_coef_error(got, ref) <= (TOL64 if dtype == np.float64 else TOL32), sb.info()["k"]
    if dtype == np.float64:
        assert o.residual(got, b64) <= TOL64


def test_strided_matches_contiguous(torch_cuda):
    """The same RHS in batch-contiguous (tile kernel) and point-contiguous
    (warp kernel) layouts agree to rounding.  The two kernels use different
    segment lengths, so the bits may differ."""
    torch = torch_cuda
    sb, o = make(3, 1024, PERIODIC, "uniform")
    b = inputs.rhs(sb.n, 96, seed=5)
    t1 = torch.from_numpy(b).cuda()
    t2 = torch.from_numpy(np.ascontiguousarray(b.T)).cuda()
    sb.solve_(t1)
    sb.solve_(t2)
    torch.cuda.synchronize()
    x1, x2 = t1.cpu().numpy(), t2.cpu().numpy().T
    assert rel_coef_error(x1, x2) <= 1e-14
    assert rel_coef_error(x2, o.solve(b)) <= TOL64


def test_general_strided_subslice(torch_cuda):
    """_strided: a sub-slice of a wider array (ld != batch), untouched columns
    unchanged."""
    torch = torch_cuda
    sb, o = make(3, 1000, PERIODIC, "uniform")
    b = inputs.rhs(sb.n, 500, seed=9)
    t = torch.from_numpy(b).cuda()
    view = t[:, 100:300]
    sb.solve_strided_(view, batch=200, batch_stride=1, point_stride=500)
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    assert np.array_equal(got[:, :100], b[:, :100]) and np.array_equal(got[:, 300:], b[:, 300:])
    assert rel_coef_error(got[:, 100:300], o.solve(b[:, 100:300])) <= TOL64


def test_batch_zero_and_errors(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, SplineBuilderError
    sb = SplineBuilder(3, 100, PERIODIC)
    t = torch.zeros(100, 0, dtype=torch.float64, device="cuda")
    sb.solve_(t)
    with pytest.raises(SplineBuilderError):
        sb.solve_strided_(torch.zeros(100, 10, dtype=torch.float64, device="cuda"), 10, 3, 5)


def test_solve_host_end_to_end(torch_cuda):
    torch = torch_cuda
    sb, o = make(3, 1000, PERIODIC, "uniform")
    b = inputs.rhs(sb.n, 3001, seed=11)
    pinned = torch.from_numpy(b.copy()).pin_memory()
    sb.solve_host_(pinned)
    assert rel_coef_error(pinned.numpy(), o.solve(b)) <= TOL64


def _threads():
    import os
    return len(os.sched_getaffinity(0))


def test_c2_full_size_every_rhs(torch_cuda):
    """C2 at full size (n=1000, 1e5 RHS) in the bench's launch configuration
    (tile kernel, TMA), EVERY right-hand side against the oracle, plus the
    interpolation residual of every RHS (BASELINE.json tolerances)."""
    torch = torch_cuda
    sb, o = make(3, 1000, PERIODIC, "uniform")
    B = 100000
    b = inputs.rhs(sb.n, B, seed=1234)
    t = torch.from_numpy(b).cuda()
    sb.solve_(t)
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    ref = o.solve(b, nthreads=_threads())
    assert rel_coef_error(got, ref) <= TOL64
    assert o.residual(got, b) <= TOL64


@pytest.mark.parametrize("bc,npts", [(GREVILLE, 1000), (HERMITE, 996)])
def test_c3_full_size_every_rhs(torch_cuda, bc, npts):
    torch = torch_cuda
    sb, o = make(5, npts, bc, "sin")
    B = 100000
    b = inputs.rhs(sb.n, B, seed=4321, degree=5, bc=bc)
    t = torch.from_numpy(b).cuda()
    sb.solve_(t)
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    ref = o.solve(b, nthreads=_threads())
    assert rel_coef_error(got, ref) <= TOL64
    assert o.residual(got, b) <= TOL64


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_c4_full_size_every_rhs(torch_cuda, dtype):
    """C4 at full size in the bench's configuration: n = 1024, 64*64*32 =
    131072 right-hand sides, x contiguous (point layout: the warp kernel's
    bulk-copy pipeline), every RHS; fp32 against the oracle run on the
    fp32-rounded inputs."""
    torch = torch_cuda
    sb, o = make(3, 1024, PERIODIC, "uniform")
    B = 64 * 64 * 32
    host = np.ascontiguousarray(inputs.rhs(sb.n, B, seed=1234).T.astype(np.float64 if dtype == "f64" else np.float32))
    t = torch.from_numpy(host).cuda()
    sb.solve_(t)
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    b_s = np.ascontiguousarray(host.T.astype(np.float64))
    ref = o.solve(b_s, nthreads=_threads())
    x = np.ascontiguousarray(got.T.astype(np.float64))
    assert rel_coef_error(x, ref) <= (TOL64 if dtype == "f64" else TOL32)
    if dtype == "f64":
        assert o.residual(x, b_s) <= TOL64


@pytest.mark.parametrize("kind", ["uniform", "sin"])
def test_advect_full_size_every_rhs(torch_cuda, kind):
    """The advection workloads at full size (Nx = 1024, Nv = 1e5, x
    contiguous, |shift| <= 2.5 cells as in bench.py), every row against the
    oracle's solve + evaluation at the feet (Algorithm 2)."""
    torch = torch_cuda
    sb, o = make(3, 1024, PERIODIC, kind)
    B = 100000
    b = inputs.rhs(sb.n, B, seed=1234)
    v = -1.0 + 2.0 * np.arange(B, dtype=np.float64) / B
    shift = v * (2.5 / o.N)
    t = torch.from_numpy(np.ascontiguousarray(b.T)).cuda()
    sb.advect_(t, torch.from_numpy(shift).cuda())
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    ref = o.advect(b, shift, nthreads=_threads())
    assert rel_coef_error(np.ascontiguousarray(got.T), ref) <= TOL64


def test_c5_full_size_device_inputs_sampled(torch_cuda):
    """C5 at its full single-GPU size: 8e6 right-hand sides (64 GB fp64,
    row pitch 64 MB) generated on the device (inputs.rhs_device), solved in ONE
    call in the bench's configuration; the first and last RHS of every 1e6
    block plus a seeded sample of 512 are compared with the oracle (the
    oracle cannot take 8e6 RHS in a test: ~5 min on 16 cores)."""
    torch = torch_cuda
    sb, o = make(3, 1000, PERIODIC, "uniform")
    total = 8_000_000
    free, _ = torch.cuda.mem_get_info()
    if free < total * sb.n * 8 * 1.05:
        pytest.skip(f"needs {total * sb.n * 8 / 1e9:.0f} GB of free device memory")
    x = inputs.rhs_device(sb.n, total, seed=1234)
    edges = [q * 1_000_000 + d for q in range(8) for d in (0, 999_999)]
    idx = np.unique(np.concatenate([edges, np.random.default_rng(8).choice(total, 512, replace=False)]))
    it = torch.from_numpy(idx).cuda()
    b_s = x.index_select(1, it).cpu().numpy()
    sb.solve_(x)
    torch.cuda.synchronize()
    got = x.index_select(1, it).cpu().numpy()
    del x
    torch.cuda.empty_cache()
    assert rel_coef_error(got, o.solve(b_s)) <= TOL64
    assert o.residual(got, b_s) <= TOL64


def test_c5_shards_bitwise_equal_and_sampled_parity(torch_cuda):
    """C5 recipe: device-generated RHS (inputs.rhs_device), sharded into
    contiguous slices; each shard solved on its own equals the unsharded solve
    bit for bit (per-RHS arithmetic is independent of the shard), and a seeded
    sample matches the oracle."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200.shard import shard_bounds
    sb, o = make(3, 1000, PERIODIC, "uniform")
    total = 20000
    full = inputs.rhs_device(sb.n, total, seed=99)
    b_host = full.cpu().numpy()
    sb.solve_(full)
    for world in (2, 3):
        parts = []
        for rank in range(world):
            a, b = shard_bounds(rank, world, total)
            x = inputs.rhs_device(sb.n, b - a, seed=99, first=a)
            assert torch.equal(x.cpu(), torch.from_numpy(b_host[:, a:b]))
            sb.solve_(x)
            parts.append(x)
        assert torch.equal(torch.cat(parts, dim=1), full)
    torch.cuda.synchronize()
    idx = np.unique(np.concatenate([[0, total - 1], np.random.default_rng(5).choice(total, 512, replace=False)]))
    got = full.cpu().numpy()[:, idx]
    assert rel_coef_error(got, o.solve(np.ascontiguousarray(b_host[:, idx]))) <= TOL64


@pytest.mark.parametrize("n_points,bc,p", [(1500, PERIODIC, 3), (2000, GREVILLE, 5), (3000, PERIODIC, 3),
                                           (4100, HERMITE, 5)])
@pytest.mark.parametrize("layout", ["batch", "point"])
def test_large_n_paths(torch_cuda, n_points, bc, p, layout):
    """n beyond the 1-CTA tile: R=8 tiles, the warp kernel with L=63, and the
    serial fallback (one thread per RHS) for Q longer than 32 x 63 rows."""
    torch = torch_cuda
    sb, o = make(p, n_points, bc, "sin")
    b = inputs.rhs(sb.n, 70, seed=21, degree=p, bc=bc)
    ref = o.solve(b)
    t = torch.from_numpy(b if layout == "batch" else np.ascontiguousarray(b.T)).cuda()
    sb.solve_(t)
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    got = got if layout == "batch" else got.T
    assert rel_coef_error(got, ref) <= TOL64


@pytest.mark.parametrize("p,kind", [(1, "uniform"), (2, "uniform"), (3, "uniform"), (4, "uniform"), (5, "uniform"),
                                    (3, "sin"), (4, "sin"), (5, "sin"), (3, "jitter"), (5, "jitter"),
                                    (2, "sin"), (3, "uniform_array")])
@pytest.mark.parametrize("layout", ["point", "batch"])
def test_advect_step_parity(torch_cuda, p, kind, layout):
    """NEXT f1: one Algorithm-2 advection step (spline build + evaluation at
    the feet of the characteristics) fused in the warp kernel,
    against the oracle's solve + evaluation."""
    torch = torch_cuda
    N = 1024 if kind == "uniform" else 1000
    sb, o = make(p, N, PERIODIC, kind)
    B = 300
    f = inputs.rhs(sb.n, B, seed=31)
    v = np.linspace(-4.0, 4.0, B)
    shift = 0.37 * v / N * 3.0  # up to ~4.4 cells
    ref = o.advect(f, shift)
    sh = torch.from_numpy(shift).cuda()
    t = torch.from_numpy(f if layout == "batch" else np.ascontiguousarray(f.T)).cuda()
    sb.advect_(t, sh)
    torch.cuda.synchronize()
    got = t.cpu().numpy()
    got = got if layout == "batch" else got.T
    assert rel_coef_error(got, ref) <= TOL64


def test_advect_fp32_and_errors(torch_cuda):
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, SplineBuilderError
    sb, o = make(3, 1024, PERIODIC, "uniform")
    f = inputs.rhs(sb.n, 64, seed=32)
    shift = np.linspace(-0.01, 0.01, 64)
    ref = o.advect(f.astype(np.float32).astype(np.float64), shift)
    t = torch.from_numpy(np.ascontiguousarray(f.T.astype(np.float32))).cuda()
    sb.advect_(t, torch.from_numpy(shift).cuda())
    torch.cuda.synchronize()
    assert rel_coef_error(t.cpu().numpy().T.astype(np.float64), ref) <= TOL32
    g = SplineBuilder(5, 1000, GREVILLE)
    with pytest.raises(SplineBuilderError):
        g.advect_(torch.zeros(1000, 4, dtype=torch.float64, device="cuda"),
                  torch.zeros(4, dtype=torch.float64, device="cuda"))


@pytest.mark.parametrize("kind", ["uniform", "sin"])
def test_advect_shifts_beyond_period(torch_cuda, kind):
    """Feet more than one period away (|shift| up to 5.3 domain lengths) and
    exact cell multiples wrap like the oracle's periodic evaluation."""
    torch = torch_cuda
    sb, o = make(3, 512, PERIODIC, kind)
    B = 96
    f = inputs.rhs(sb.n, B, seed=33)
    shift = np.concatenate([np.linspace(-5.3, 5.3, B - 32), np.arange(-16, 16) / 512.0])
    ref = o.advect(f, shift)
    t = torch.from_numpy(np.ascontiguousarray(f.T)).cuda()
    sb.advect_(t, torch.from_numpy(shift).cuda())
    torch.cuda.synchronize()
    assert rel_coef_error(t.cpu().numpy().T, ref) <= TOL64


# ------------------------------------------- slabs (spline_builder_solve_slabs)
@pytest.mark.parametrize("p,npts,bc,kind", [(3, 1000, PERIODIC, "uniform"), (5, 1000, GREVILLE, "sin"),
                                            (5, 996, HERMITE, "sin"), (4, 200, PERIODIC, "jitter")])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_slabs_stacked_parity(torch_cuda, p, npts, bc, kind, dtype):
    """nslab stacked (n, batch) blocks with padding (ld > batch, slab gap): one
    launch of the tile kernel over a 3-D tensor map; each slab matches the oracle,
    padding untouched."""
    torch = torch_cuda
    sb, orc = make(p, npts, bc, kind)
    n, B, ld, nslab = sb.n, 37, 48, 5
    sstride = n * ld + 16
    buf = np.full(nslab * sstride, 7.0)
    blocks = []
    for q in range(nslab):
        b = inputs.rhs(n, B, seed=50 + q, degree=p, bc=bc)
        blocks.append(b)
        for j in range(n):
            buf[q * sstride + j * ld: q * sstride + j * ld + B] = b[j]
    t = torch.from_numpy(buf.astype(dtype)).cuda()
    sb.solve_slabs_(t, B, ld, nslab, sstride)
    torch.cuda.synchronize()
    out = t.cpu().numpy().astype(np.float64)
    tol = TOL64 if dtype == np.float64 else TOL32
    mask = np.ones_like(out, dtype=bool)
    for q in range(nslab):
        got = np.stack([out[q * sstride + j * ld: q * sstride + j * ld + B] for j in range(n)])
        for j in range(n):
            mask[q * sstride + j * ld: q * sstride + j * ld + B] = False
        ref = orc.solve(blocks[q].astype(dtype).astype(np.float64))
        assert rel_coef_error(got, ref) <= tol
    assert np.all(out[mask] == 7.0)


def test_slabs_side_by_side_and_errors(torch_cuda):
    """Slabs interleaved inside each row (f[x][y][v], slab y): equals one
    batch-contiguous solve; aliasing strides are rejected."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilderError
    sb, orc = make(3, 500, PERIODIC, "sin")
    n, B, nslab = sb.n, 24, 6
    b = inputs.rhs(n, B * nslab, seed=61)
    t = torch.from_numpy(b.copy()).cuda()
    sb.solve_slabs_(t, B, B * nslab, nslab, B)
    torch.cuda.synchronize()
    assert rel_coef_error(t.cpu().numpy(), orc.solve(b)) <= TOL64
    with pytest.raises(SplineBuilderError):
        sb.solve_slabs_(t, B, B * nslab, nslab, B - 1)


def test_c4m_middle_layout_matches_point_layout(torch_cuda):
    """C4's second layout f[y][x][v] (x in the middle) via slabs gives the same
    coefficients as the x-contiguous layout solved by the warp kernel."""
    torch = torch_cuda
    sb, orc = make(3, 1024, PERIODIC, "uniform")
    n, Y, V = sb.n, 8, 256
    b = inputs.rhs(n, Y * V, seed=62)                     # (n, Y*V)
    mid = np.ascontiguousarray(b.reshape(n, Y, V).transpose(1, 0, 2))  # f[y][x][v]
    t = torch.from_numpy(mid).cuda()
    sb.solve_slabs_(t, V, V, Y, n * V)
    pt = torch.from_numpy(np.ascontiguousarray(b.T)).cuda()  # f[r][x]
    sb.solve_(pt)
    torch.cuda.synchronize()
    got = t.cpu().numpy().transpose(1, 0, 2).reshape(n, Y * V)
    ref = orc.solve(b)
    assert rel_coef_error(got, ref) <= TOL64
    assert rel_coef_error(pt.cpu().numpy().T, ref) <= TOL64


# ----------------------------------------- 2-D tensor product (solve_2d, f3)
CASES_2D = [
    # (dim-1 space, dim-2 space, grids)
    ((3, 64, PERIODIC, "uniform"), (3, 48, PERIODIC, "uniform"), 5),
    ((3, 200, PERIODIC, "sin"), (5, 150, GREVILLE, "sin"), 3),
    ((5, 120, HERMITE, "jitter"), (4, 100, PERIODIC, "jitter"), 3),
    ((4, 33, GREVILLE, "uniform"), (3, 1000, PERIODIC, "uniform"), 2),
    ((3, 1024, PERIODIC, "uniform"), (3, 17, PERIODIC, "uniform"), 2),
]


def rel_grid_error(got, ref):
    return float(max(np.abs(g - r).max() / np.abs(r).max() for g, r in zip(got, ref)))


@pytest.mark.parametrize("c1,c2,G", CASES_2D, ids=[f"{a[0]}{a[2]}{a[1]}x{b[0]}{b[2]}{b[1]}" for a, b, _ in CASES_2D])
def test_2d_parity(torch_cuda, c1, c2, G):
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import solve_2d_
    sb1, o1 = make(*c1)
    sb2, o2 = make(*c2)
    F = inputs.rhs(sb1.n, G * sb2.n, seed=70).T.reshape(G, sb2.n, sb1.n).copy()
    ref = oracle.solve_2d(o1, o2, F)
    t = torch.from_numpy(F).cuda()
    solve_2d_(sb1, sb2, t)
    torch.cuda.synchronize()
    assert rel_grid_error(t.cpu().numpy(), ref) <= TOL64
    t32 = torch.from_numpy(F.astype(np.float32)).cuda()
    solve_2d_(sb1, sb2, t32)
    torch.cuda.synchronize()
    ref32 = oracle.solve_2d(o1, o2, F.astype(np.float32).astype(np.float64))
    assert rel_grid_error(t32.cpu().numpy(), ref32) <= TOL32


def test_2d_full_size_chunked_sampled(torch_cuda):
    """C6 shape (1024 x 1024 grids, 16 of them: 128 MB, several L2 chunks):
    sampled grids against the oracle, interpolation property on one grid."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import solve_2d_
    sb1, o1 = make(3, 1024, PERIODIC, "uniform")
    sb2, o2 = make(3, 1024, PERIODIC, "uniform")
    G = 16
    F = inputs.rhs(1024, G * 1024, seed=71).T.reshape(G, 1024, 1024).copy()
    t = torch.from_numpy(F).cuda()
    solve_2d_(sb1, sb2, t)
    torch.cuda.synchronize()
    out = t.cpu().numpy()
    for g in (0, 7, 15):
        ref = oracle.solve_2d(o1, o2, F[g])
        assert rel_grid_error(out[g:g + 1], ref[None]) <= TOL64
    # A1 C A2^T = F on grid 3
    A1, A2 = o1.matrix(), o2.matrix()
    res = np.abs(A2 @ out[3] @ A1.T - F[3]).max() / np.abs(F[3]).max()
    assert res <= 1e-12


@pytest.mark.parametrize("p,npts,bc", [(3, 1000, PERIODIC), (5, 1000, GREVILLE), (5, 996, HERMITE),
                                       (4, 1024, PERIODIC)])
def test_update_new_mesh_parity(torch_cuda, p, npts, bc):
    """NEXT f4 (matrices that change): spline_builder_update moves a device
    handle to a new mesh; batch-contiguous solves, point-contiguous solves and
    (periodic) the advection step then match the oracle on the new mesh and
    a handle created on it bit for bit."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    N = inputs.n_cells(p, npts, bc)
    sb = SplineBuilder(p, npts, bc, inputs.breakpoints(N, "uniform"))
    b = inputs.rhs(sb.n, 333, seed=17, degree=p, bc=bc)
    gpu_solve(torch, sb, b.copy())
    for kind, seed in (("sin", 42), ("jitter", 3), ("uniform", 42)):
        x = inputs.breakpoints(N, kind, seed=seed)
        sb.update(x)
        o = Oracle(p, npts, bc, x)
        fresh = SplineBuilder(p, npts, bc, x)
        got = gpu_solve(torch, sb, b.copy())
        assert rel_coef_error(got, o.solve(b)) <= TOL64
        assert np.array_equal(got, gpu_solve(torch, fresh, b.copy()))
        t = torch.from_numpy(np.ascontiguousarray(b.T)).cuda()
        sb.solve_(t)
        torch.cuda.synchronize()
        assert rel_coef_error(t.cpu().numpy().T, o.solve(b)) <= TOL64
        if bc == PERIODIC:
            shift = np.linspace(-2.5, 2.5, b.shape[1]) / N
            t = torch.from_numpy(b.copy()).cuda()
            sb.advect_(t, torch.from_numpy(shift).cuda())
            torch.cuda.synchronize()
            assert rel_coef_error(t.cpu().numpy(), o.advect(b, shift)) <= TOL64
        fresh.close()


def test_two_host_threads_two_streams_one_handle(torch_cuda):
    """Concurrent solves with ONE handle from two host threads on two streams
    (include/spline_builder.h: allowed): both take the TMA tile kernel (the
    tensor-map encoder is resolved once, thread-safely) and both match the
    oracle."""
    import threading
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import last_kernel
    sb, o = make(5, 1000, GREVILLE, "sin")
    bs = [inputs.rhs(sb.n, 4096 + 16 * i, seed=600 + i, degree=5, bc=GREVILLE) for i in range(2)]
    ts = [torch.from_numpy(b).cuda() for b in bs]
    streams = [torch.cuda.Stream() for _ in range(2)]
    kernels, errors = [None, None], []
    barrier = threading.Barrier(2)

    def work(i):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(streams[i]):
                src = torch.from_numpy(bs[i]).cuda()
                barrier.wait()
                for rep in range(3):
                    ts[i].copy_(src)
                    sb.solve_(ts[i], stream=streams[i])
                    kernels[i] = last_kernel()
            streams[i].synchronize()
        except Exception as e:  # pragma: no cover
            errors.append(e)

    th = [threading.Thread(target=work, args=(i,)) for i in range(2)]
    [t.start() for t in th]
    [t.join() for t in th]
    assert not errors, errors
    torch.cuda.synchronize()
    for i in range(2):
        assert kernels[i].startswith("tile<f64") and "TMA" in kernels[i], kernels[i]
        assert rel_coef_error(ts[i].cpu().numpy(), o.solve(bs[i])) <= TOL64


# ------------------------------------------------------------ device-side refactorisation
DEV_UPDATE_CASES = [
    # (degree, n_points, bc, create mesh, new meshes)
    (3, 1000, PERIODIC, "sin", ["jitter", "sin2", "uniform_array"]),
    (3, 1000, PERIODIC, "uniform", ["jitter"]),
    (4, 600, PERIODIC, "jitter", ["sin"]),
    (5, 1000, GREVILLE, "sin", ["jitter", "sin2"]),
    (5, 996, HERMITE, "sin", ["jitter", "sin2"]),
    (3, 200, GREVILLE | (HERMITE << 4), "jitter", ["sin"]),
]


def _mesh(N, kind):
    if kind == "sin2":  # the sin map with a smaller amplitude: another smooth non-uniform mesh
        u = np.arange(N + 1, dtype=np.float64) / N
        x = u + 0.3 * np.sin(2.0 * np.pi * u) / (2.0 * np.pi)
        x[0], x[-1] = 0.0, 1.0
        return x
    x = inputs.breakpoints(N, kind)
    return x if x is not None else inputs.breakpoints(N, "uniform_array")


@pytest.mark.parametrize("case", DEV_UPDATE_CASES, ids=lambda c: f"p{c[0]}-n{c[1]}-bc{c[2]}-{c[3]}")
def test_update_device_new_meshes_parity(torch_cuda, case):
    """spline_builder_update_device: the factorisation of a new
    mesh is computed by a kernel on the device; the batched solve (tile kernel,
    batch-contiguous, and warp kernel, point layout) then matches the oracle
    built on the new breakpoints, element by element at 1e-12, plus the
    interpolation residual."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    p, npts, bc, m0, news = case
    N = inputs.n_cells(p, npts, bc)
    sb = SplineBuilder(p, npts, bc, _mesh(N, m0), device_update=True)
    b = inputs.rhs(sb.n, 777, seed=31, degree=p, bc=bc)
    for kind in news:
        x = _mesh(N, kind)
        sb.update_device_(torch.from_numpy(x).cuda())
        sb.update_status()
        o = Oracle(p, npts, bc, x)
        ref = o.solve(b)
        got = gpu_solve(torch, sb, b)
        assert rel_coef_error(got, ref) <= TOL64, (kind, rel_coef_error(got, ref))
        assert o.residual(got, b) <= TOL64
        t = torch.from_numpy(np.ascontiguousarray(b.T)).cuda()
        sb.solve_(t)
        torch.cuda.synchronize()
        assert rel_coef_error(np.ascontiguousarray(t.cpu().numpy().T), ref) <= TOL64, kind


def test_update_device_advection_and_graph_replay(torch_cuda):
    """After a device update the advection step (non-uniform evaluation data
    rebuilt on the device) matches the oracle on the new mesh, and a solve
    captured in a CUDA graph BEFORE the update replays with the new mesh (the
    launch arguments point at constants updated in place)."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    N = 1024
    x0, x1 = _mesh(N, "sin"), _mesh(N, "jitter")
    sb = SplineBuilder(3, N, PERIODIC, x0, device_update=True)
    b = inputs.rhs(N, 4096, seed=41)
    t = torch.from_numpy(b).cuda()
    pristine = t.clone()
    g = torch.cuda.CUDAGraph()
    sb.solve_(t)  # warm-up outside the capture
    with torch.cuda.graph(g):
        sb.solve_(t)
    sb.update_device_(torch.from_numpy(x1).cuda())
    sb.update_status()
    t.copy_(pristine)
    g.replay()
    torch.cuda.synchronize()
    o1 = Oracle(3, N, PERIODIC, x1)
    assert rel_coef_error(t.cpu().numpy(), o1.solve(b)) <= TOL64
    B = 300
    f = inputs.rhs(N, B, seed=43)
    shift = np.linspace(-2.0, 2.0, B) / N
    tf = torch.from_numpy(np.ascontiguousarray(f.T)).cuda()
    sb.advect_(tf, torch.from_numpy(shift).cuda())
    torch.cuda.synchronize()
    assert rel_coef_error(np.ascontiguousarray(tf.cpu().numpy().T), o1.advect(f, shift)) <= TOL64


def test_update_device_rejections_keep_previous_mesh(torch_cuda):
    """The status path of the device update: knots that are not increasing
    (SB_INVALID_ARG), a periodic mesh that moves its end points
    (SB_INVALID_ARG), and a mesh whose matrix leaves the structure frozen at
    create (SB_UNSUPPORTED: a Lambda entry above 1e-14 outside the pattern) are
    rejected on the device; the previous mesh stays live and solves still
    match its oracle."""
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, SplineBuilderError
    N = 500
    x0 = _mesh(N, "sin")
    sb = SplineBuilder(3, N, PERIODIC, x0, device_update=True)
    o0 = Oracle(3, N, PERIODIC, x0)
    b = inputs.rhs(N, 64, seed=51)
    bad = x0.copy()
    bad[10], bad[11] = bad[11], bad[10]
    moved = x0 * 2.0
    # cells shrinking geometrically towards x = 0.5: far slower decay of Lambda
    # than the create-time mesh, so entries above 1e-14 appear outside the pattern
    u = np.arange(N + 1) / N
    steep = 0.5 + 0.5 * np.sign(u - 0.5) * np.abs(2 * u - 1) ** 6
    expected = [(bad, 1), (moved, 1), (steep, 5)]
    for x, status in expected:
        sb.update_device_(torch.from_numpy(x).cuda())
        with pytest.raises(SplineBuilderError) as ei:
            sb.update_status()
        assert ei.value.status == status, (status, str(ei.value))
        assert rel_coef_error(gpu_solve(torch, sb, b), o0.solve(b)) <= TOL64


def test_update_device_faster_than_host_replan(torch_cuda):
    """The device refactorisation of a C3 Greville mesh (n = 1000, p = 5) takes
    less time than the host re-plan + upload of spline_builder_update (the
    point of the device path: meshes that change every step)."""
    import time
    torch = torch_cuda
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder
    N = inputs.n_cells(5, 1000, GREVILLE)
    xs = [_mesh(N, k) for k in ("sin", "sin2")]
    sb = SplineBuilder(5, 1000, GREVILLE, xs[0], device_update=True)
    dx = [torch.from_numpy(x).cuda() for x in xs]
    for i in range(3):
        sb.update_device_(dx[i % 2])
        sb.update_status()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    reps = 20
    for i in range(reps):
        sb.update_device_(dx[i % 2])
    sb.update_status()
    t_dev = (time.perf_counter() - t0) / reps
    t0 = time.perf_counter()
    for i in range(5):
        sb.update(xs[i % 2])
    t_host = (time.perf_counter() - t0) / 5
    print(f"device update {t_dev * 1e3:.3f} ms, host re-plan {t_host * 1e3:.3f} ms")
    assert t_dev < t_host


PAIR_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, %(root)r)
import oracle
from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, inputs, last_kernel
cases = [(3, 1000, 0, "uniform"), (5, 1000, 1, "sin"), (5, 996, 2, "sin"), (4, 1000, 0, "jitter"),
         (3, 200, 1 | (2 << 4), "jitter"), (3, 1024, 0, "sin")]
for deg, npts, bc, mesh in cases:
    N = inputs.n_cells(deg, npts, bc)
    x = inputs.breakpoints(N, mesh)
    sb, o = SplineBuilder(deg, npts, bc, x), oracle.Oracle(deg, npts, bc, x)
    for B in (32, 96, 32 * 74 * 2 + 6):
        b = inputs.rhs(sb.n, B, seed=B, degree=deg, bc=bc)
        t = torch.from_numpy(b).cuda()
        sb.solve_(t)
        torch.cuda.synchronize()
        kern = last_kernel()
        assert kern.startswith("pair<"), (deg, npts, bc, B, kern)
        err = oracle.rel_coef_error(t.cpu().numpy(), o.solve(b))
        assert err <= 1e-12, (deg, npts, bc, B, err)
        assert o.residual(t.cpu().numpy(), b) <= 1e-12
print("pair ok")
"""


def test_pair_tile_parity_forced(torch_cuda):
    """The 2-CTA-cluster tile kernel (pair.cuh; 32-RHS tiles split in row halves,
    carries and the corner exchanged through distributed shared memory) on
    every band / boundary family, 1 to several tiles per cluster, forced with
    SB_TILE_PAIR=2 in a subprocess (the dispatch reads it once per process)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, SB_TILE_PAIR="2")
    r = subprocess.run([sys.executable, "-c", PAIR_SCRIPT % {"root": root}], env=env, capture_output=True, text=True,
                       timeout=300)
    assert r.returncode == 0 and "pair ok" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]
