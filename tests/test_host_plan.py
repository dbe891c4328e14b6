"""The host create step (C++ plan behind the C ABI, SB_FLAG_HOST_ONLY -- no
GPU): Schur split, factor types, corner blocks, segment data, and the host
run of the same factorisation against the oracle.  CPU only.

Pins: P1 the paper's worked example, Table I
(P:95-101), P6 closed-form factors, P10 block identity against the oracle's
independently built matrix."""
import json
import os

import numpy as np
import pytest

from oracle import GREVILLE, HERMITE, PERIODIC, Oracle, rel_coef_error
from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def host(p, npts, bc, kind="uniform", split=None):
    N = inputs.n_cells(p, npts, bc)
    x = inputs.breakpoints(N, kind)
    return SplineBuilder(p, npts, bc, x, split=split, host_only=True), x


def test_paper_worked_example_p249():
    g = json.load(open(os.path.join(GOLDEN, "paper_p249_corner_nnz.json")))
    sb, _ = host(g["degree"], g["n"], PERIODIC)
    inf = sb.info()
    assert inf["k"] == g["k"]
    assert inf["nnz_beta"] == g["top_right_nnz"]      # beta = Q^-1 gamma, |beta| > 1e-14
    assert inf["nnz_lambda"] == g["bottom_left_nnz"]
    (lr, lc, lv), (br, bc, bv), dp = sb.blocks()
    n, k = g["n"], g["k"]
    assert lr.max() < k and lc.max() < n - k          # lambda is (1, 999)
    assert br.max() < n - k and bc.max() < k          # beta is (999, 1)


def test_table1_q_types():
    g = json.load(open(os.path.join(GOLDEN, "paper_table1_q_types.json")))
    want = {"pttrs": 0, "pbtrs": 1, "gbtrs": 2}
    for row in g["rows"]:
        sb, _ = host(row["degree"], 200, PERIODIC, "uniform" if row["mesh"] == "uniform" else "jitter")
        inf = sb.info()
        assert inf["q_type"] == want[row["lapack"]], row
        if "band" in row:
            assert [inf["q_kl"], inf["q_ku"]] == row["band"]


def test_closed_form_factors_p6():
    """cubic uniform: delta' = 1/sqrt(3); p=4/5 delta' entries."""
    sb, _ = host(3, 1000, PERIODIC)
    _, _, dp = sb.blocks()
    assert abs(dp[0, 0] - 1 / np.sqrt(3)) < 1e-15
    sb, _ = host(4, 1000, PERIODIC)
    _, _, dp = sb.blocks()
    assert np.allclose(dp, [[0.525067, 0.195963], [0.195963, 0.525067]], atol=1e-6)
    sb, _ = host(5, 1000, PERIODIC)
    _, _, dp = sb.blocks()
    assert np.allclose(dp, [[0.448932, 0.208772], [0.208772, 0.448932]], atol=1e-6)


@pytest.mark.parametrize("p,npts,bc,kind", [(3, 1000, PERIODIC, "uniform"), (5, 1000, PERIODIC, "jitter"),
                                            (5, 1000, GREVILLE, "sin"), (5, 996, HERMITE, "sin"),
                                            (4, 300, HERMITE, "jitter"), (3, 60, GREVILLE, "uniform")])
def test_block_identity_p10(p, npts, bc, kind):
    """[[Q,0],[lambda,delta']] [[I,beta],[0,I]] = A (equilibrated rows),
    with A from the ORACLE (independent construction)."""
    sb, x = host(p, npts, bc, kind)
    inf = sb.info()
    o = Oracle(p, npts, bc, x)
    A = o.matrix()
    n, lo, hi, k = o.n, inf["split_lo"], inf["split_hi"], inf["k"]
    # the library equilibrates Hermite derivative rows by h^d; rescale the oracle's raw rows
    scale = np.ones(n)
    if bc == HERMITE:
        nbc = (p - 1) // 2 if p % 2 else p // 2
        h0, h1 = x[1] - x[0], x[-1] - x[-2]
        for d in range(1, nbc + 1):
            scale[d - 1] = h0 ** d
            scale[n - nbc + d - 1] = h1 ** d
    A = A * scale[:, None]
    D = np.r_[np.arange(lo), np.arange(n - hi, n)].astype(int)
    Qi = np.arange(lo, n - hi)
    Q, gam, lam, dlt = A[np.ix_(Qi, Qi)], A[np.ix_(Qi, D)], A[np.ix_(D, Qi)], A[np.ix_(D, D)]
    (lr, lc, lv), (br, bc_, bv), dp = sb.blocks()
    lam_lib = np.zeros((k, n - k))
    lam_lib[lr, lc] = lv
    assert np.abs(lam_lib - lam).max() < 1e-13 * max(1, np.abs(lam).max())
    beta = np.linalg.solve(Q, gam)
    beta_lib = np.zeros_like(beta)
    beta_lib[br, bc_] = bv
    assert np.abs(beta_lib - beta).max() < 1e-13            # thresholded at 1e-14 + rounding
    assert np.abs(dp - (dlt - lam @ beta)).max() < 1e-12
    # block identity with the library's blocks
    L_ = np.block([[Q, np.zeros((n - k, k))], [lam_lib, dp]])
    U_ = np.block([[np.eye(n - k), beta_lib], [np.zeros((k, n - k)), np.eye(k)]])
    Ap = A[np.ix_(np.r_[Qi, D], np.r_[Qi, D])]
    assert np.abs(L_ @ U_ - Ap).max() < 1e-12


def test_default_splits():
    """Greville p=5 -> (2,2) with Q band (3,3); Hermite p=5 ->
    (3,3) with Q band (2,2) and no interchanges."""
    sb, _ = host(5, 1000, GREVILLE, "sin")
    inf = sb.info()
    assert (inf["split_lo"], inf["split_hi"], inf["q_kl"], inf["q_ku"]) == (2, 2, 3, 3)
    sb, _ = host(5, 996, HERMITE, "sin")
    inf = sb.info()
    assert (inf["split_lo"], inf["split_hi"], inf["q_kl"], inf["q_ku"]) == (3, 3, 2, 2)
    assert inf["max_pivot_growth"] < 10


CASES = [(p, N, PERIODIC, kind) for p in (1, 2, 3, 4, 5) for N, kind in ((16, "uniform"), (200, "jitter"))] + \
        [(p, 100 + p, GREVILLE, kind) for p in (1, 2, 3, 4, 5) for kind in ("uniform", "sin")] + \
        [(p, 101 if p % 2 else 100, HERMITE, kind) for p in (2, 3, 4, 5) for kind in ("uniform", "sin")] + \
        [(3, 5, PERIODIC, "uniform"), (5, 8, GREVILLE, "uniform"), (3, 1000, PERIODIC, "uniform"),
         (5, 1000, GREVILLE, "sin"), (5, 996, HERMITE, "sin"), (3, 1024, PERIODIC, "uniform")]


@pytest.mark.parametrize("case", CASES, ids=[f"p{c[0]}-n{c[1]}-bc{c[2]}-{c[3]}" for c in CASES])
def test_host_plan_solve_matches_oracle(case):
    """the plan (split, factors, Lambda/gamma corners -- the kernels' order)
    run on the host reproduces the oracle to fp64 rounding."""
    p, npts, bc, kind = case
    sb, x = host(p, npts, bc, kind)
    o = Oracle(p, npts, bc, x)
    b = inputs.rhs(o.n, 9, seed=3, degree=p, bc=bc)
    assert rel_coef_error(sb.solve_cpu_plan_(b.copy()), o.solve(b)) < 1e-13


@pytest.mark.parametrize("split", [(0, 0), (1, 1), (2, 2), (3, 3), (2, 3)])
def test_explicit_split_override(split):
    sb, x = host(5, 1000, GREVILLE, "sin", split=split)
    inf = sb.info()
    assert (inf["split_lo"], inf["split_hi"]) == split
    o = Oracle(5, 1000, GREVILLE, x)
    b = inputs.rhs(o.n, 5, seed=4, degree=5, bc=GREVILLE)
    assert rel_coef_error(sb.solve_cpu_plan_(b.copy()), o.solve(b)) < 1e-13


def test_segment_plan_c2():
    sb, _ = host(3, 1000, PERIODIC)
    inf = sb.info()
    assert inf["seg_len"] == 36 and inf["n_segments"] == 28  # 999 Q rows -> 28 x 36 (9 padding rows)
    assert 1 <= inf["carry_fwd"] <= 2 and 1 <= inf["carry_bwd"] <= 2
    assert inf["nnz_Lambda"] == 48 and inf["nnz_gamma"] == 2


def test_hermite_rejects_derivative_rows_in_q():
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilderError
    with pytest.raises(SplineBuilderError):
        host(5, 996, HERMITE, "sin", split=(1, 1))


MIXED = [(p, N, lo, hi, kind) for p in (1, 2, 3, 4, 5) for (lo, hi) in ((HERMITE, GREVILLE), (GREVILLE, HERMITE))
         for N, kind in ((60, "uniform"), (995, "sin"))]


@pytest.mark.parametrize("case", MIXED, ids=[f"p{c[0]}-N{c[1]}-{c[2]}{c[3]}-{c[4]}" for c in MIXED])
def test_mixed_bc_host_plan_matches_oracle(case):
    """Mixed ends (NEXT row f4): the plan's split keeps every derivative row in
    delta and reproduces the oracle."""
    p, N, lo, hi, kind = case
    bc = inputs.bc_mixed(lo, hi)
    nlo, nhi = inputs.n_hermite_rows(p, bc)
    npts = N + p - nlo - nhi
    sb, x = host(p, npts, bc, kind)
    inf = sb.info()
    assert inf["n_cells"] == N and inf["nbasis"] == N + p
    assert inf["split_lo"] >= nlo and inf["split_hi"] >= nhi
    o = Oracle(p, npts, bc, x)
    b = inputs.rhs(o.n, 9, seed=3, degree=p, bc=bc)
    assert rel_coef_error(sb.solve_cpu_plan_(b.copy()), o.solve(b)) < 1e-13


UPDATE = [(3, 1000, PERIODIC), (4, 200, PERIODIC), (5, 1000, GREVILLE), (5, 996, HERMITE),
          (3, 60 + 3 - 1, inputs.bc_mixed(HERMITE, GREVILLE))]


@pytest.mark.parametrize("case", UPDATE, ids=[f"p{c[0]}-n{c[1]}-bc{c[2]}" for c in UPDATE])
def test_update_new_mesh_matches_oracle(case):
    """spline_builder_update (NEXT row f4, matrices that change): a handle
    moved from one mesh to another solves like the oracle on the new mesh and
    carries the same factors as a handle created on it."""
    p, npts, bc = case
    sb, _ = host(p, npts, bc, "uniform")
    N = inputs.n_cells(p, npts, bc)
    for kind, seed in (("sin", 42), ("jitter", 7), ("uniform", 42)):
        x = inputs.breakpoints(N, kind, seed=seed)
        sb.update(x)
        fresh = SplineBuilder(p, npts, bc, x, host_only=True)
        assert sb.info() == fresh.info()
        o = Oracle(p, npts, bc, x)
        b = inputs.rhs(o.n, 7, seed=5, degree=p, bc=bc)
        got = sb.solve_cpu_plan_(b.copy())
        assert rel_coef_error(got, o.solve(b)) < 1e-13
        assert np.array_equal(got, fresh.solve_cpu_plan_(b.copy()))


def test_update_failure_keeps_previous_mesh():
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilderError
    p, npts = 3, 100
    x = inputs.breakpoints(npts, "sin")
    sb = SplineBuilder(p, npts, PERIODIC, x, host_only=True)
    o = Oracle(p, npts, PERIODIC, x)
    b = inputs.rhs(o.n, 3, seed=9, degree=p)
    want = sb.solve_cpu_plan_(b.copy())
    bad = x.copy()
    bad[10] = bad[12]                                  # not strictly increasing
    with pytest.raises(SplineBuilderError):
        sb.update(bad)
    assert np.array_equal(sb.solve_cpu_plan_(b.copy()), want)
    assert rel_coef_error(want, o.solve(b)) < 1e-13
