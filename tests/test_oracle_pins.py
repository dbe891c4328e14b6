"""Pins for the CPU oracle: the oracle is checked
against things other than itself -- values the paper prints, textbook closed
forms (cardinal B-spline values, circulant FFT), an independent library
(scipy's B-splines and interpolation, LAPACK through numpy) and invariants.
All tests are CPU only.
"""
import json
import os

import numpy as np
import pytest
import scipy.interpolate as si
import scipy.linalg as sl

import oracle
from oracle import GREVILLE, HERMITE, PERIODIC, Oracle, rel_coef_error
from paper_conf_sc_asahilbpbgo24_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

# textbook cardinal B-spline values at the centre and integer offsets
# (Schoenberg; SURVEY S-5): first column of the uniform periodic matrix.
CARDINAL = {
    1: [1.0],
    2: [6 / 8, 1 / 8],
    3: [4 / 6, 1 / 6],
    4: [230 / 384, 76 / 384, 1 / 384],
    5: [66 / 120, 26 / 120, 1 / 120],
}


def circulant_first_col(p, n):
    c = np.zeros(n)
    vals = CARDINAL[p]
    c[0] = vals[0]
    for m, v in enumerate(vals[1:], start=1):
        c[m] += v
        c[-m] += v
    return c


def rng(seed=0):
    return np.random.Generator(np.random.Philox(key=seed))


# ---------------------------------------------------------------- helpers
# Independent constructions with scipy, in GLOBAL coordinates (fine at the
# small N used here).

def periodic_ext_knots(x, p):
    N = len(x) - 1
    L = x[-1] - x[0]
    g = np.arange(-2 * p - 2, N + 2 * p + 3)
    return g, x[g % N] + np.floor_divide(g, N) * L


def scipy_periodic_matrix(x, p):
    """A[i, j] = B_j(xi_i) with B_j centred (support [t_{j-s}, t_{j-s+p+1}],
    s = floor((p+1)/2)) and xi_i its Greville abscissa, periodic images summed."""
    N = len(x) - 1
    L = x[-1] - x[0]
    s = (p + 1) // 2
    g, t = periodic_ext_knots(x, p)
    off = -g[0]
    xi = np.array([t[off + j - s + 1: off + j - s + p + 1].mean() for j in range(N)])
    xi = x[0] + np.mod(xi - x[0], L)
    A = np.zeros((N, N))
    for j in range(N):
        kn = t[off + j - s: off + j - s + p + 2]
        be = si.BSpline.basis_element(kn, extrapolate=False)
        for shift in (-2 * L, -L, 0.0, L, 2 * L):
            v = np.nan_to_num(be(xi + shift))
            A[:, j] += v
    return A, xi


def clamped_knots(x, p):
    return np.concatenate([np.full(p, x[0]), x, np.full(p, x[-1])])


def greville(t, p, n):
    return np.array([t[j + 1: j + p + 1].mean() for j in range(n)])


def scipy_clamped_matrix(x, p, bc):
    """Raw collocation matrix built with scipy.BSpline (values and derivatives)."""
    N = len(x) - 1
    t = clamped_knots(x, p)
    n = N + p
    if bc == GREVILLE:
        pts = greville(t, p, n)
        pts[-1] = x[-1]
        rows = [(xx, 0) for xx in pts]
    else:
        nbc = (p - 1) // 2 if p % 2 else p // 2
        vals = list(x) if p % 2 else list(0.5 * (x[1:] + x[:-1]))
        rows = [(x[0], d) for d in range(1, nbc + 1)] + [(v, 0) for v in vals] + \
               [(x[-1], d) for d in range(1, nbc + 1)]
    A = np.zeros((n, n))
    for j in range(n):
        c = np.zeros(n)
        c[j] = 1.0
        spl = si.BSpline(t, c, p, extrapolate=True)
        for i, (xx, d) in enumerate(rows):
            A[i, j] = spl.derivative(d)(xx) if d else spl(xx)
    return A, t, rows


MESHES = ["uniform", "sin", "jitter"]


def mesh(N, kind):
    return inputs.breakpoints(N, kind if kind != "uniform" else "uniform_array", seed=42)


# ------------------------------------------------------------------ P2

@pytest.mark.parametrize("p", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("n", [16, 1000, 1024])
def test_uniform_periodic_matrix_is_cardinal_circulant(p, n):
    o = Oracle(p, n, PERIODIC)
    A = o.matrix()
    c = circulant_first_col(p, n)
    ref = sl.circulant(c)
    assert np.abs(A - ref).max() < 4e-16


@pytest.mark.parametrize("p", [2, 3, 4, 5])
@pytest.mark.parametrize("n", [16, 1000, 1024])
def test_uniform_periodic_solve_matches_fft(p, n):
    """P2: A circulant => x = ifft(fft(b) / fft(c))."""
    o = Oracle(p, n, PERIODIC)
    b = rng(1).uniform(-1, 1, size=(n, 8))
    x = o.solve(b)
    c = circulant_first_col(p, n)
    xf = np.real(np.fft.ifft(np.fft.fft(b, axis=0) / np.fft.fft(c)[:, None], axis=0))
    assert rel_coef_error(x, xf) < 2e-15


# ------------------------------------------------------------------ P3

@pytest.mark.parametrize("p", [3, 5])
@pytest.mark.parametrize("N", [12, 40])
def test_uniform_periodic_odd_matches_scipy_interp(p, N):
    """scipy's periodic interpolant at the breakpoints; its basis j starts at
    x_{j-p}, ours at x_{j-s}: ours[j] = scipy.c[j + p - s]."""
    x = np.arange(N + 1) / N
    y = rng(2).uniform(-1, 1, N)
    spl = si.make_interp_spline(x, np.append(y, y[0]), k=p, bc_type="periodic")
    s = (p + 1) // 2
    ours = Oracle(p, N, PERIODIC).solve(y)
    theirs = spl.c[np.arange(N) + p - s]
    assert rel_coef_error(ours, theirs) < 1e-14


@pytest.mark.parametrize("p", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("kind", MESHES)
def test_periodic_matrix_matches_scipy_basis(p, kind):
    N = 24
    x = mesh(N, kind)
    A_ref, xi = scipy_periodic_matrix(x, p)
    o = Oracle(p, N, PERIODIC, None if kind == "uniform" else x)
    A = o.matrix()
    assert np.abs(A - A_ref).max() < 1e-13
    pts, _, _ = o.rows()
    d = np.abs(pts - xi)
    assert np.minimum(d, 1.0 - d).max() < 1e-14  # compare on the circle of period 1


@pytest.mark.parametrize("p", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("kind", MESHES)
def test_greville_matches_scipy_interp(p, kind):
    N = 30
    x = mesh(N, kind)
    t = clamped_knots(x, p)
    n = N + p
    xi = greville(t, p, n)
    y = rng(3).uniform(-1, 1, n)
    spl = si.make_interp_spline(xi, y, k=p, t=t)
    o = Oracle(p, n, GREVILLE, x)
    pts, _, _ = o.rows()
    assert np.abs(pts - xi).max() < 1e-15
    assert pts[0] == x[0] and pts[-1] == x[-1]
    assert rel_coef_error(o.solve(y), spl.c) < 1e-13


@pytest.mark.parametrize("p", [3, 5])
@pytest.mark.parametrize("kind", MESHES)
def test_hermite_odd_matches_scipy_interp(p, kind):
    """scipy bc_type=([(1,a),(2,b)],[(1,c),(2,d)]): knots = clamped(breaks)
    (SURVEY S8); RHS order [d1..dnbc at x0][values][d1..dnbc at xN]."""
    N = 30
    x = mesh(N, kind)
    nbc = (p - 1) // 2
    r = rng(4)
    y = r.uniform(-1, 1, N + 1)
    dl = r.uniform(-5, 5, nbc)
    dr = r.uniform(-5, 5, nbc)
    spl = si.make_interp_spline(x, y, k=p, bc_type=([(d + 1, dl[d]) for d in range(nbc)],
                                                    [(d + 1, dr[d]) for d in range(nbc)]))
    assert np.allclose(spl.t, clamped_knots(x, p))
    b = np.concatenate([dl, y, dr])
    o = Oracle(p, N + 1, HERMITE, x)
    assert o.n == N + p
    assert rel_coef_error(o.solve(b), spl.c) < 1e-12


@pytest.mark.parametrize("p,bc", [(q, GREVILLE) for q in range(1, 6)] + [(q, HERMITE) for q in range(2, 6)])
@pytest.mark.parametrize("kind", MESHES)
def test_clamped_matrix_matches_scipy_basis(p, bc, kind):
    N = 20
    x = mesh(N, kind)
    A_ref, _, rows = scipy_clamped_matrix(x, p, bc)
    n_points = N + p if bc == GREVILLE else (N + 1 if p % 2 else N)
    o = Oracle(p, n_points, bc, x)
    A = o.matrix()
    scale = np.abs(A_ref).max(axis=1, keepdims=True)
    assert np.abs((A - A_ref) / scale).max() < 1e-12


# ------------------------------------------------------------------ P4

@pytest.mark.parametrize("case", [(3, 16, PERIODIC, "uniform"), (5, 16, PERIODIC, "jitter"),
                                  (4, 16, PERIODIC, "sin"), (5, 21, GREVILLE, "sin"),
                                  (5, 17, HERMITE, "jitter"), (4, 16, HERMITE, "uniform"),
                                  (3, 8, PERIODIC, "uniform"), (2, 5, PERIODIC, "jitter")])
def test_brute_force_tiny(case):
    """P4: dense LAPACK solve (numpy) of the scipy-built matrix, n <= 32."""
    p, n_points, bc, kind = case
    N = inputs.n_cells(p, n_points, bc)
    x = mesh(N, kind)
    A = scipy_periodic_matrix(x, p)[0] if bc == PERIODIC else scipy_clamped_matrix(x, p, bc)[0]
    b = rng(5).uniform(-1, 1, size=(A.shape[0], 8))
    ref = np.linalg.solve(A, b)
    o = Oracle(p, n_points, bc, None if kind == "uniform" else x)
    assert rel_coef_error(o.solve(b), ref) < 1e-13


# ------------------------------------------------------------------ P7

@pytest.mark.parametrize("p,bc", [(q, GREVILLE) for q in range(1, 6)] + [(q, HERMITE) for q in range(2, 6)])
@pytest.mark.parametrize("kind", MESHES)
def test_polynomial_reproduction(p, bc, kind):
    """P7: data of a polynomial of degree <= p is reproduced exactly
    everywhere (evaluated with scipy and with the oracle's evaluator)."""
    N = 25
    x = mesh(N, kind)
    n_points = N + p if bc == GREVILLE else (N + 1 if p % 2 else N)
    o = Oracle(p, n_points, bc, x)
    poly = np.polynomial.Polynomial(rng(6).uniform(-1, 1, p + 1))
    pts, _, der = o.rows()
    b = np.array([poly.deriv(d)(xx) if d else poly(xx) for xx, d in zip(pts, der)])
    c = o.solve(b)
    xs = np.sort(rng(7).uniform(0, 1, 200))
    spl = si.BSpline(clamped_knots(x, p), c, p)
    assert np.abs(spl(xs) - poly(xs)).max() < 1e-12
    assert np.abs(o.eval(c, xs) - poly(xs)).max() < 1e-12
    if p >= 2:
        assert np.abs(o.eval(c, xs, deriv=1) - poly.deriv(1)(xs)).max() < 1e-9


# ------------------------------------------------------------------ P5

@pytest.mark.parametrize("p,bc,kind", [(3, PERIODIC, "uniform"), (5, PERIODIC, "jitter"), (4, PERIODIC, "sin"),
                                       (5, GREVILLE, "sin"), (5, HERMITE, "sin"), (3, HERMITE, "jitter")])
def test_interpolation_property(p, bc, kind):
    """P5: the spline evaluated (scipy) at the interpolation points gives b."""
    N = 40
    x = mesh(N, kind)
    n_points = N if bc == PERIODIC else (N + p if bc == GREVILLE else N + 1)
    o = Oracle(p, n_points, bc, None if kind == "uniform" else x)
    b = rng(8).uniform(-1, 1, o.n)
    c = o.solve(b)
    pts, _, der = o.rows()
    if bc == PERIODIC:
        A = scipy_periodic_matrix(x, p)[0]
        got = A @ c
    else:
        spl = si.BSpline(clamped_knots(x, p), c, p)
        got = np.array([spl.derivative(d)(xx) if d else spl(xx) for xx, d in zip(pts, der)])
    scale = np.abs(o.matrix()).max(axis=1)
    assert np.abs((got - b) / scale).max() < 1e-13
    assert o.residual(c, b) < 1e-14


# ------------------------------------------------------------- P8 / P9

@pytest.mark.parametrize("p", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("kind", MESHES)
def test_partition_of_unity(p, kind):
    """P8: sum_j B_j == 1 => b == 1 gives x == 1 (periodic and Greville)."""
    N = 50
    x = mesh(N, kind)
    for bc, npts in ((PERIODIC, N), (GREVILLE, N + p)):
        o = Oracle(p, npts, bc, None if kind == "uniform" else x)
        assert np.abs(o.solve(np.ones(o.n)) - 1.0).max() < 1e-14


@pytest.mark.parametrize("p", [3, 4, 5])
def test_shift_invariance(p):
    """P9: uniform periodic: roll(b, s) -> roll(x, s)."""
    n = 200
    o = Oracle(p, n, PERIODIC)
    b = rng(9).uniform(-1, 1, n)
    x = o.solve(b)
    for s in (1, 7, 123):
        assert rel_coef_error(o.solve(np.roll(b, s)), np.roll(x, s)) < 1e-15


# ------------------------------------------------------- paper pins P1

def test_paper_worked_example_corner_nnz():
    """P1: cubic uniform periodic n=1000 -> top-right
    (999,1) block has 48 non-zeros, bottom-left (1,999) has 2."""
    g = json.load(open(os.path.join(GOLDEN, "paper_p249_corner_nnz.json")))
    n, k = g["n"], g["k"]
    A = Oracle(g["degree"], n, PERIODIC).matrix()
    Q, gam, lam = A[:n - k, :n - k], A[:n - k, n - k:], A[n - k:, :n - k]
    beta = np.linalg.solve(Q, gam)
    assert beta.shape == tuple(g["top_right_shape"])
    assert lam.shape == tuple(g["bottom_left_shape"])
    assert int((np.abs(beta) > g["beta_drop_threshold"]).sum()) == g["top_right_nnz"]
    assert int((lam != 0).sum()) == g["bottom_left_nnz"]


def test_paper_table1_q_types():
    """PAPER.md P:95-101 (Table I): type of Q by degree and uniformity."""
    g = json.load(open(os.path.join(GOLDEN, "paper_table1_q_types.json")))
    N = 64
    for row in g["rows"]:
        p = row["degree"]
        x = None if row["mesh"] == "uniform" else inputs.breakpoints(N, "jitter", seed=3)
        A = Oracle(p, N, PERIODIC, x).matrix()
        offs = [((j - i + N // 2) % N) - N // 2 for i, j in zip(*np.nonzero(A))]
        k = max(max(offs), -min(offs))
        Q = A[:N - k, :N - k]
        sym = np.abs(Q - Q.T).max() < 1e-15
        assert sym == row["symmetric"], row
        if sym:
            np.linalg.cholesky(Q)  # positive definite
            ii, jj = np.nonzero(Q)
            assert [int((ii - jj).max()), int((jj - ii).max())] == row["band"], row


# ---------------------------------------------------------- layout check

def test_oracle_layouts_agree():
    o = Oracle(3, 64, PERIODIC)
    b = rng(10).uniform(-1, 1, size=(64, 33))
    x1 = o.solve(b)
    bt = np.ascontiguousarray(b.T)  # point-contiguous: rhs r at r*64
    o.solve_(bt, batch_stride=64, point_stride=1, batch=33)
    assert np.array_equal(bt.T, x1)


def test_oracle_bc_row_counts():
    for p in (3, 5):
        assert Oracle(p, 996 if p == 5 else 998, HERMITE).n == 1000
    assert Oracle(5, 1000, GREVILLE).n == 1000
    with pytest.raises(ValueError):
        Oracle(3, 10, GREVILLE, np.array([0.0, 0.5, 0.4, 1.0, 1.1, 1.2, 1.3, 1.4]))


# ------------------------------------------------ advection step (NEXT f1)

@pytest.mark.parametrize("p", [2, 3, 4, 5])
def test_advect_integer_cell_shift_is_exact_roll(p):
    """Algorithm 2 on a uniform periodic mesh: shifting by m whole
    cells maps the spline space onto itself, so f_new = roll(f, m) exactly."""
    N = 64
    o = Oracle(p, N, PERIODIC)
    f = rng(11).uniform(-1, 1, size=(N, 3))
    h = 1.0 / N
    for m in (0, 1, 5, -3):
        out = o.advect(f, np.full(3, m * h))
        assert np.abs(out - np.roll(f, m, axis=0)).max() < 1e-13


@pytest.mark.parametrize("p", [3, 5])
@pytest.mark.parametrize("kind", ["uniform", "jitter"])
def test_advect_matches_scipy_spline_evaluation(p, kind):
    """fractional shifts: the oracle's evaluation equals scipy's BSpline of the
    same coefficients at the feet of the characteristics."""
    N = 40
    x = mesh(N, kind)
    o = Oracle(p, N, PERIODIC, None if kind == "uniform" else x)
    f = rng(12).uniform(-1, 1, size=(N, 4))
    shift = np.array([0.0123, -0.37, 0.5, 1.77])
    out = o.advect(f, shift)
    c = o.solve(f)
    g, t = periodic_ext_knots(x, p)
    s = (p + 1) // 2
    pts, _, _ = o.rows()
    for r in range(4):
        # our basis j has first knot j-s; scipy's BSpline(t, c', p) basis i has first knot t[i]
        off = -g[0]
        cext = np.zeros(len(t) - p - 1)
        for j in range(-2 * N, 3 * N):
            i = off + j - s
            if 0 <= i < len(cext):
                cext[i] = c[j % N, r]
        spl = si.BSpline(t, cext, p, extrapolate=False)
        feet = np.mod(pts - shift[r], 1.0)
        assert np.abs(spl(feet) - out[:, r]).max() < 1e-12


def test_advect_smooth_profile_is_accurate():
    """a smooth periodic profile is transported to ~h^4 accuracy (cubic)."""
    N = 128
    o = Oracle(3, N, PERIODIC)
    xs = np.arange(N) / N
    f = np.sin(2 * np.pi * xs)[:, None]
    out = o.advect(f, np.array([0.2345]))
    assert np.abs(out[:, 0] - np.sin(2 * np.pi * (xs - 0.2345))).max() < 1e-6


# ------------------------------------------------- 2-D tensor product
# Pins of oracle.solve_2d (NEXT row f3): the 2-D interpolation system
# sum C[j2][j1] B1_j1(xi1) B2_j2(xi2) = F, written out as one big matrix from
# scipy-built 1-D collocation matrices, a 2-D FFT closed form, scipy's own
# per-axis interpolation, and tensor-product polynomial reproduction.

def test_2d_kronecker_brute_force_scipy_matrices():
    """vec(C) = (A2 (x) A1)^{-1} vec(F) with A1, A2 built by scipy (not the oracle)."""
    x1 = mesh(7, "jitter")
    x2 = mesh(5, "sin")
    A1, _ = scipy_periodic_matrix(x1, 3)
    A2, _, _ = scipy_clamped_matrix(x2, 4, GREVILLE)
    o1, o2 = Oracle(3, 7, PERIODIC, x1), Oracle(4, 5 + 4, GREVILLE, x2)
    F = rng(5).uniform(-1, 1, size=(3, o2.n, o1.n))
    C = oracle.solve_2d(o1, o2, F)
    big = np.kron(A2, A1)
    for b in range(3):
        ref = np.linalg.solve(big, F[b].reshape(-1)).reshape(o2.n, o1.n)
        assert np.abs(C[b] - ref).max() <= 1e-12 * np.abs(ref).max()


@pytest.mark.parametrize("p1,p2", [(3, 3), (4, 5), (5, 3)])
def test_2d_uniform_periodic_fft_closed_form(p1, p2):
    """Uniform periodic x uniform periodic: A1, A2 circulant, so A1 C A2^T = F is
    a 2-D cyclic convolution: C = ifft2(fft2(F) / (fft(c2)[:, None] fft(c1)[None, :]))."""
    n1, n2 = 24, 20
    F = rng(6).uniform(-1, 1, size=(n2, n1))
    c1, c2 = circulant_first_col(p1, n1), circulant_first_col(p2, n2)
    ref = np.real(np.fft.ifft2(np.fft.fft2(F) / (np.fft.fft(c2)[:, None] * np.fft.fft(c1)[None, :])))
    C = oracle.solve_2d(Oracle(p1, n1, PERIODIC), Oracle(p2, n2, PERIODIC), F)
    assert np.abs(C - ref).max() <= 1e-13 * np.abs(ref).max()


def test_2d_matches_scipy_per_axis_interpolation():
    """Greville x Greville: scipy make_interp_spline along axis 1 then axis 0
    (scipy's own batched-over-the-other-axis solves) gives the same coefficients."""
    p1, p2, N1, N2 = 3, 5, 9, 11
    x1, x2 = mesh(N1, "sin"), mesh(N2, "jitter")
    t1, t2 = clamped_knots(x1, p1), clamped_knots(x2, p2)
    g1, g2 = greville(t1, p1, N1 + p1), greville(t2, p2, N2 + p2)
    g1[-1], g2[-1] = x1[-1], x2[-1]
    F = rng(7).uniform(-1, 1, size=(N2 + p2, N1 + p1))
    s1 = si.make_interp_spline(g1, F, k=p1, t=t1, axis=1)
    s1c = np.moveaxis(s1.c, 0, 1)  # scipy keeps the interpolation axis first
    s2 = si.make_interp_spline(g2, s1c, k=p2, t=t2, axis=0)
    C = oracle.solve_2d(Oracle(p1, N1 + p1, GREVILLE, x1), Oracle(p2, N2 + p2, GREVILLE, x2), F)
    assert np.abs(C - s2.c).max() <= 1e-12 * np.abs(C).max()


@pytest.mark.parametrize("bc1,bc2", [(GREVILLE, HERMITE), (HERMITE, GREVILLE)])
def test_2d_tensor_polynomial_reproduction(bc1, bc2):
    """Data from P(x, y) = sum a_ab x^a y^b, a <= p1, b <= p2: the tensor spline
    equals P everywhere (Hermite rows take the polynomial's derivatives)."""
    p1, p2, N1, N2 = 3, 5, 8, 6
    x1, x2 = mesh(N1, "jitter"), mesh(N2, "sin")
    npts1 = N1 + p1 if bc1 == GREVILLE else N1 + 1
    npts2 = N2 + p2 if bc2 == GREVILLE else N2 + 1
    o1, o2 = Oracle(p1, npts1, bc1, x1), Oracle(p2, npts2, bc2, x2)
    a = rng(8).uniform(-1, 1, size=(p1 + 1, p2 + 1))
    P1 = [np.polynomial.Polynomial(np.eye(p1 + 1)[i]) for i in range(p1 + 1)]
    P2 = [np.polynomial.Polynomial(np.eye(p2 + 1)[i]) for i in range(p2 + 1)]
    r1, _, d1 = o1.rows()
    r2, _, d2 = o2.rows()
    F = np.zeros((o2.n, o1.n))
    for ia in range(p1 + 1):
        u = np.array([P1[ia].deriv(d)(x) if d else P1[ia](x) for x, d in zip(r1, d1)])
        for ib in range(p2 + 1):
            v = np.array([P2[ib].deriv(d)(y) if d else P2[ib](y) for y, d in zip(r2, d2)])
            F += a[ia, ib] * np.outer(v, u)
    C = oracle.solve_2d(o1, o2, F)
    xs = rng(9).uniform(x1[0], x1[-1], size=7)
    ys = rng(10).uniform(x2[0], x2[-1], size=5)
    S = oracle.eval_2d(o1, o2, C, xs, ys)
    ref = sum(a[ia, ib] * np.outer(P2[ib](ys), P1[ia](xs)) for ia in range(p1 + 1) for ib in range(p2 + 1))
    assert np.abs(S - ref).max() <= 1e-12 * max(1.0, np.abs(ref).max())


def test_2d_interpolation_property_periodic_nonuniform():
    """S(xi1_i1, xi2_i2) = F[i2][i1] on a non-uniform periodic x periodic grid."""
    o1 = Oracle(4, 12, PERIODIC, mesh(12, "jitter"))
    o2 = Oracle(3, 10, PERIODIC, mesh(10, "sin"))
    F = rng(11).uniform(-1, 1, size=(o2.n, o1.n))
    C = oracle.solve_2d(o1, o2, F)
    S = oracle.eval_2d(o1, o2, C, o1.rows()[0], o2.rows()[0])
    assert np.abs(S - F).max() <= 1e-12


# ------------------------------------- mixed boundary conditions (NEXT row f4)
# bc = lo | (hi << 4): Hermite derivative rows at one end, Greville abscissae
# elsewhere (the nbc abscissae next to a Hermite end are dropped; R13).

def mixed_case(p, N, lo, hi, kind):
    nbc = (p - 1) // 2 if p % 2 else p // 2
    x = mesh(N, kind)
    n_hermite = (lo == HERMITE) + (hi == HERMITE)
    o = Oracle(p, N + p - nbc * n_hermite, lo | (hi << 4), x)
    t = clamped_knots(x, p)
    n = N + p
    g = greville(t, p, n)
    g[-1] = x[-1]
    keep = [j for j in range(n) if not ((lo == HERMITE and 1 <= j <= nbc) or (hi == HERMITE and n - 1 - nbc <= j <= n - 2))]
    return o, x, t, g[keep], nbc


@pytest.mark.parametrize("p", [2, 3, 4, 5])
@pytest.mark.parametrize("lo,hi", [(HERMITE, GREVILLE), (GREVILLE, HERMITE)])
@pytest.mark.parametrize("kind", ["uniform", "jitter"])
def test_mixed_bc_matches_scipy(p, lo, hi, kind):
    """scipy make_interp_spline on the clamped knots with the derivative
    conditions on one side only (bc_type=(derivs, None) / (None, derivs))."""
    o, x, t, pts, nbc = mixed_case(p, 20, lo, hi, kind)
    g = rng(12)
    y = g.uniform(-1, 1, len(pts))
    dv = g.uniform(-1, 1, nbc)
    conds = [(d + 1, dv[d]) for d in range(nbc)]
    spl = si.make_interp_spline(pts, y, k=p, t=t, bc_type=(conds, None) if lo == HERMITE else (None, conds))
    b = np.concatenate([dv, y]) if lo == HERMITE else np.concatenate([y, dv])
    c = o.solve(b)
    assert np.abs(c - spl.c).max() <= 1e-12 * max(1.0, np.abs(spl.c).max())


@pytest.mark.parametrize("p", [3, 4, 5])
@pytest.mark.parametrize("lo,hi", [(HERMITE, GREVILLE), (GREVILLE, HERMITE)])
def test_mixed_bc_polynomial_reproduction(p, lo, hi):
    o, x, t, pts, nbc = mixed_case(p, 17, lo, hi, "sin")
    poly = np.polynomial.Polynomial(rng(13).uniform(-1, 1, p + 1))
    xr, _, dr = o.rows()
    b = np.array([poly.deriv(d)(xx) if d else poly(xx) for xx, d in zip(xr, dr)])
    c = o.solve(b)
    xs = rng(14).uniform(x[0], x[-1], 50)
    assert np.abs(o.eval(c, xs) - poly(xs)).max() <= 1e-12
