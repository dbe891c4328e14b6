// plan.hpp -- host-side "create" step of the spline builder: collocation
// matrix, Schur split, one-time factorisation, sparse corner blocks and the
// segment coupling data of the in-CTA parallel recurrences.
//
// "the factorization is only done once at
// initialization ... we take advantage of existing CPU libraries to
// factorize the matrix and copy the result to the device".  There is no
// LAPACK on the target box, so the banded factorisations (pttrf / pbtrf-like
// LDL^T, gbtrf without interchanges, getrf for delta') are written here.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace sb {

enum Bc { PERIODIC = 0, GREVILLE = 1, HERMITE = 2 };
enum QType { Q_PTTRS = 0, Q_PBTRS = 1, Q_GBTRS = 2 };

constexpr int KMAX_BAND = 4;          // largest Q half-band the kernels are built for
constexpr int KMAX_DELTA = 32;        // largest delta' order
constexpr double CORNER_DROP = 1e-14; // keep |beta|, |Lambda| > 1e-14 (DESIGN R4)

// What an interpolation row is, independent of the mesh (device-side
// refactorisation recomputes its point for new breakpoints):
//   GREVILLE  Greville abscissa of basis idx        BREAK  value at x_idx (idx < N)
//   END       value at x_N                           MID    value at the midpoint of cell idx
//   DER0/DERN derivative of order deriv at x_0 / x_N
enum RowKind { ROW_GREVILLE = 0, ROW_BREAK = 1, ROW_END = 2, ROW_MID = 3, ROW_DER0 = 4, ROW_DERN = 5 };
struct RowDesc {
    int kind, idx, deriv;
};

// build_plan flags
enum PlanFlags {
    PLAN_DEVICE_UPDATE = 1  // structure frozen for device-side refactorisation: corner patterns dilated by
                            // CORNER_MARGIN, carry walks one segment deeper, no slot sharing, generic
                            // (non-uniform) advection geometry with a 2x finer bucket table
};
constexpr int CORNER_MARGIN = 24;  // Lambda columns / gamma rows kept around the create-time pattern

struct SparseRow {
    std::vector<int> col;
    std::vector<double> val;
};

// segment partition of the padded Q recurrences for one register segment
// length L: S segments of exactly L rows, Q padded with
// identity rows to nQp = S*L.
struct SegPlan {
    int L = 0, S = 0, nQp = 0;
    int carry_f = 0, carry_b = 0;  // predecessor segments in the carry walks
    std::vector<double> G;         // S*K*K forward transfer  G_t[j][m]
    std::vector<double> H;         // S*K*K backward transfer H_t[j][m]
};

struct Plan {
    // ---- spline space
    int p = 0, bc = 0, N = 0, n = 0, nbc = 0;
    int bc_lo = 0, bc_hi = 0, nbc_lo = 0, nbc_hi = 0;  // per end (mixed boundary conditions)
    std::vector<double> h;          // cell widths
    std::vector<double> xb;         // N+1 breakpoints (xb[N] = xb[0] + period for periodic)
    std::vector<double> xi;         // n interpolation points (row positions; derivative rows: the end point)
    std::vector<double> xe;         // periodic: extended knots t_c, c in [-p, N+p] at xe[c+p]
    bool adv_uniform = false;       // periodic uniform mesh (stencil evaluation of Algorithm 2)
    double adv_invh = 0.0, adv_q0 = 0.0;  // 1/h and (xi_0 - x_0)/h
    int adv_steps = 0;              // forward steps from the bucket's cell to the point's cell (<= 2 typically)
    std::vector<int> adv_tbl;       // periodic: buckets of [x_0, x_N) no wider than the smallest cell -> cell
    std::vector<double> adv_rcp;    // periodic: 1/(t_{m+w} - t_m) at [(m+p)*(p|1) + w-1], m in [-p, N+p), w = 1..p
    std::vector<RowDesc> rowdesc;   // n row descriptors (mesh independent)
    bool dev_update = false;        // PLAN_DEVICE_UPDATE
    std::vector<SparseRow> A;       // equilibrated collocation matrix rows
    std::vector<double> rowscale;   // A_eq = diag(rowscale) * A_raw
    // ---- Schur split (Eq. 3)
    int s_lo = 0, s_hi = 0, k = 0, nQ = 0;
    std::vector<int> drow;          // delta index -> row of A
    int kl = 0, ku = 0, K = 1;      // Q band, kernel band (max, >=1)
    int qtype = Q_GBTRS;
    double growth = 0.0;
    // ---- factors of Q, Q-local indices (forward unit-lower L, backward
    //      x_i = y_i*dinv_i - sum_m up_{i,m} x_{i+m})
    std::vector<double> Lb;         // nQ*K : Lb[i*K+m-1] = L(i, i-m)
    std::vector<double> Ub;         // nQ*K : Ub[i*K+m-1] = U(i, i+m)/U(i,i)
    std::vector<double> dinv;       // nQ
    // ---- corners (Eq. 4 and its transposed twin)
    std::vector<int> lam_r, lam_c;   std::vector<double> lam_v;    // lambda COO (delta row, Q col)
    std::vector<int> gam_r, gam_c;   std::vector<double> gam_v;    // gamma COO (Q row, delta col), sorted by row
    std::vector<int> beta_r, beta_c; std::vector<double> beta_v;   // beta = Q^-1 gamma, thresholded COO
    std::vector<int> Lam_ptr, Lam_c; std::vector<double> Lam_v;    // Lambda = lambda Q^-1, thresholded CSR by delta row
    std::vector<double> dprime;     // k*k delta' = delta - lambda beta
    std::vector<double> dlu;        // k*k LU of delta' (getrf, partial pivoting)
    std::vector<int> dpiv;          // k
    // ---- segment plans: [0] batch-contiguous fp64 kernel (L=36), [1] batch-
    //      contiguous fp32 kernel (L=72), [2] point-contiguous warp-per-RHS
    //      kernel (32 lanes = segments, odd L; S = 0 if nQ is too large)
    SegPlan seg[3];
};

struct Status {
    int code = 0;
    std::string msg;
};

// Build the spline space, the (equilibrated) collocation matrix, choose the
// split, factor, compute corners and segment data.  split_lo/hi = -1: default.
Status build_plan(Plan &P, int degree, int n_points, int bc, const double *knots, int split_lo, int split_hi,
                  int flags = 0);

// Algorithm 1 on the CPU with the plan's factors (serial, fp64), in the same
// order as the kernels (Lambda / gamma form).  Used by create's self-check.
void plan_solve_cpu(const Plan &P, double *rhs, int64_t batch, int64_t bstride, int64_t pstride);

}  // namespace sb
