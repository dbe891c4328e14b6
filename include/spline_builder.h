/*
 * spline_builder.h -- C ABI of the B200-native batched spline-coefficient
 * builder (PAPER.md: Asahi et al., "Development of performance portable
 * spline solver for exa-scale plasma turbulence simulation", SC'24-W).
 *
 * The problem (Sec. II.B, Eq. 2): one B-spline collocation
 * matrix A, fixed in time, solved against a huge batch of right-hand sides
 * b ("a fixed single matrix A and multiple right-hand sides"), in place
 * ("b stores the right-hand side vectors on entry and stores the solution
 * vectors on exit").  A is factored once at create time on the host
 * with the Schur-complement block split of Eq. 3-4,
 * and every solve runs Algorithm 1 in one fused sm_100a kernel:
 *   x0' = Q^{-1} b0            (banded LDL^T / LU: pttrs, pbtrs or gbtrs, Table I)
 *   x1  = delta'^{-1} (b1 - lambda x0')   (COO spmv + getrs)
 *   x0  = x0' - beta x1                     (COO spmv, beta = Q^{-1} gamma)
 *
 * All functions are extern "C", take plain pointers and sizes, and never
 * throw.  No torch type appears here.  Status codes are the SB_* values
 * below; the message of the last failure on the calling thread is returned
 * by spline_builder_last_error().
 */
#ifndef SPLINE_BUILDER_H
#define SPLINE_BUILDER_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct spline_builder *spline_builder_t; /* opaque; changed only by spline_builder_update */

/* boundary conditions (PAPER.md P:55 periodic; non-periodic per BASELINE C3) */
enum { SB_PERIODIC = 0, SB_GREVILLE = 1, SB_HERMITE = 2 };
/* different conditions at the two ends (Greville / Hermite only; R13) */
#define SB_BC(lo, hi) ((lo) == (hi) ? (lo) : ((lo) | ((hi) << 4)))
/* element types of the right-hand sides */
enum { SB_F64 = 0, SB_F32 = 1 };
/* status codes */
enum {
    SB_OK = 0,
    SB_INVALID_ARG = 1, /* bad argument; nothing was launched                 */
    SB_SINGULAR = 2,    /* A (or Q / delta') could not be factored             */
    SB_CUDA = 3,        /* a CUDA runtime / driver call or launch failed       */
    SB_NOMEM = 4,       /* host or device allocation failed                    */
    SB_UNSUPPORTED = 5  /* valid request outside what this build implements   */
};
/* create flags */
enum {
    SB_FLAG_HOST_ONLY = 1,    /* factor on the host only; no device upload (solve_* then
                                 return SB_UNSUPPORTED).  For inspection / CPU tests. */
    SB_FLAG_DEVICE_UPDATE = 2 /* structure frozen for spline_builder_update_device: the
                                 gamma / Lambda patterns are dilated by 24 rows / columns,
                                 segment carries one deeper, no factor sharing between
                                 segments (uniform meshes solve slightly slower) */
};

/*
 * spline_builder_create -- one-time construction and factorisation
 * ("the factorization is only done once at
 * initialization ... and copy the result to the device").
 *
 *   degree   spline degree p, 1..5.
 *   n_points number of interpolation conditions, which fixes the number of
 *            cells N:   periodic  N = n_points          (nbasis n = N)
 *                       Greville  N = n_points - p      (n = N + p)
 *                       Hermite   N = n_points - 1 (odd p) or N = n_points
 *                                 (even p, values at cell midpoints); n = N + p
 *   bc       SB_PERIODIC, SB_GREVILLE or SB_HERMITE (both ends alike), or
 *            SB_BC(lo, hi) with lo != hi in {SB_GREVILLE, SB_HERMITE}: mixed,
 *            N = n_points - p + nbc(lo) + nbc(hi), nbc(Hermite end) = nbc
 *            below, nbc(Greville end) = 0; the value rows are the Greville
 *            abscissae of the clamped basis without the nbc next to a Hermite
 *            end (the end point itself stays).
 *   knots    NULL -> uniform mesh on [0, 1] (all cells of width 1/N exactly);
 *            else N+1 strictly increasing breakpoints (host pointer, read
 *            during the call only; the periodic period is knots[N]-knots[0]).
 *
 * Row order of every right-hand side (length n):
 *   periodic / Greville: b_j = f(xi_j), xi_j the Greville abscissa of basis j
 *     (periodic basis j is centred on xi_j; uniform: xi_j = x_j for odd p,
 *     x_j + h/2 for even p).
 *   Hermite: [f^(1..nbc)(x_0), f(x_0) ... f(x_N), f^(1..nbc)(x_N)] with raw
 *     derivatives (odd p, nbc = (p-1)/2); even p: values at the N cell
 *     midpoints, nbc = p/2.
 *   mixed: [f^(1..nbc)(x_0) if lo is Hermite, values at the kept Greville
 *     abscissae in increasing order, f^(1..nbc)(x_N) if hi is Hermite].
 * The handle owns host and device copies of the factors on the CUDA device
 * current at the call.  Returns NULL on failure (see last_error / the
 * status in spline_builder_last_status()).
 */
spline_builder_t spline_builder_create(int degree, int n_points, int bc, const double *knots);

/* Same as create, with an explicit Schur split: the delta index set is the
 * first split_lo and the last split_hi rows/columns of A.
 * split_lo = split_hi = -1 selects the default.  Periodic requires
 * split_lo = 0 and split_hi >= the circulant half-bandwidth (or -1). */
spline_builder_t spline_builder_create_ex(int degree, int n_points, int bc, const double *knots,
                                          int split_lo, int split_hi, int flags);

/* spline_builder_update -- new mesh, same handle (SURVEY 8(f)4 "matrices
 * that change"; the factorisation is done once per mesh on the host and
 * copied to the device).  Rebuilds the collocation matrix, the Schur
 * split of Eq. 3 and every factor for the breakpoints `knots` (host
 * pointer, N+1 values, same meaning as in create; NULL = uniform), keeping
 * the create-time degree, n_points, bc and split request.  The device
 * constants are replaced synchronously; the caller ensures no solve on h is
 * in flight (as for destroy).  On any error (bad knots, singular factor,
 * out of memory) the handle keeps its previous mesh and factors and the
 * status code is returned.
 * CUDA graphs: a solve captured before the update keeps the OLD mesh's
 * constants (its launch arguments point into the previous device blob, which
 * stays allocated until destroy, so replay is memory-safe but uses the old
 * matrix).  Re-capture graphs after an update to solve with the new mesh.
 * Each host update retires one blob (~10-200 KB) until destroy. */
int spline_builder_update(spline_builder_t h, const double *knots);

/*
 * spline_builder_update_device -- new mesh, factorised ON THE DEVICE (SURVEY
 * 8(f)4; BASELINE north_star "one-time host or device factorisation"), for a
 * handle created with SB_FLAG_DEVICE_UPDATE.  One kernel on `stream`
 * recomputes, for the breakpoints `knots` (DEVICE pointer, N+1 strictly
 * increasing values, read by the kernel; NULL = uniform on [0,1]), the
 * collocation matrix (de Boor BSPLVB/BSPLVD), the Schur blocks of Eq. 3
 * (P:69-78), the banded LU of Q without interchanges (Table I), beta = Q^-1 gamma,
 * Lambda = lambda Q^-1, delta' = delta - lambda beta and its LU (Eq. 4-6), and
 * every layout the solve kernels read, into a staging copy of the handle's
 * device constants; the copy replaces the live constants in stream order only
 * if every check passed.  Asynchronous: solves enqueued later on the same
 * stream use the new mesh; solves on other streams must be ordered by the
 * caller.  Kernels captured in a CUDA graph keep valid arguments and see the
 * new mesh on replay.  Checks (reported by spline_builder_update_status, the
 * previous mesh kept on failure): knots strictly increasing (SB_INVALID_ARG);
 * a periodic mesh keeps its end points (SB_INVALID_ARG); Q / delta' factor
 * without breakdown or growth > 1e3 (SB_SINGULAR); the new matrix fits the
 * frozen band, gamma / Lambda (|Lambda| > 1e-14) patterns, carry depths and
 * advection buckets (SB_UNSUPPORTED: re-plan with spline_builder_update).
 * Host-side queries (get_info, get_blocks, solve_cpu_plan) keep describing the
 * mesh of the last host create/update.  Returns SB_UNSUPPORTED for handles
 * without the flag.
 */
int spline_builder_update_device(spline_builder_t h, const double *knots, void *stream);

/* Waits for the last spline_builder_update_device on h and returns its
 * outcome (SB_OK: the new mesh is live; else the previous mesh is kept and
 * spline_builder_last_error() says why).  SB_OK if none is pending. */
int spline_builder_update_status(spline_builder_t h);

/*
 * spline_builder_solve -- in-place batched solve of fp64 right-hand sides
 * (Algorithm 1; fused kernel of Listing 6).
 *
 *   rhs           DEVICE pointer on the handle's device, caller owned.  On
 *                 entry b, on exit the spline coefficients x (same layout).
 *   batch         number of right-hand sides (>= 0; 0 is a no-op).
 *   batch_stride  elements between consecutive right-hand sides:
 *                   1   -> batch-contiguous (the paper's layout, P:143,
 *                          P:391): element (row j, rhs r) at rhs[j*batch + r]
 *                   >=n -> point-contiguous: element (j, r) at
 *                          rhs[r*batch_stride + j]   (GYSELA slice, C4)
 *                 anything else -> SB_INVALID_ARG (use _strided).
 *   stream        cudaStream_t (NULL = legacy default stream) on which the
 *                 kernel is enqueued; the call is asynchronous.
 * Concurrent solves on different streams with one handle are allowed.
 */
int spline_builder_solve(spline_builder_t h, double *rhs, int64_t batch, int64_t batch_stride, void *stream);

/* fp32 storage, same semantics (compute in fp32). */
int spline_builder_solve_f32(spline_builder_t h, float *rhs, int64_t batch, int64_t batch_stride, void *stream);

/* General strided layout: element (row j, rhs r) at
 * rhs[r*batch_stride + j*point_stride]; dtype SB_F64 or SB_F32.  Strides
 * in elements, > 0, and the (j, r) -> offset map must be one-to-one. */
int spline_builder_solve_strided(spline_builder_t h, void *rhs, int dtype, int64_t batch, int64_t batch_stride,
                                 int64_t point_stride, void *stream);

/*
 * spline_builder_solve_slabs -- in-place solve of nslab independent
 * batch-contiguous (n, batch) blocks in ONE launch: element (row j, rhs r,
 * slab q) at rhs[q*slab_stride + j*ld + r].  This is the layout of a
 * dimension that is neither the fastest nor the slowest of a higher-
 * dimensional array (e.g. f[y][x][v] solved along x, slabs y), and pass 2 of
 * the tensor-product builder below.  PAPER.md P:59: "batched over the other
 * dimensions".
 *   rhs          DEVICE pointer, SB_F64 or SB_F32 (dtype), caller owned.
 *   ld >= batch  elements between rows;  slab_stride: elements between slabs,
 *                either >= n*ld (stacked slabs) or >= batch with
 *                ld >= (nslab-1)*slab_stride + batch (slabs side by side in
 *                each row); anything that aliases -> SB_INVALID_ARG.
 * nslab == 0 or batch == 0 is a no-op.  Asynchronous on stream.
 */
int spline_builder_solve_slabs(spline_builder_t h, void *rhs, int dtype, int64_t batch, int64_t ld, int64_t nslab,
                               int64_t slab_stride, void *stream);

/*
 * spline_builder_solve_2d -- tensor-product spline coefficients (PAPER.md
 * "Higher dimensional B-splines can be obtained by a tensor product of
 * 1D splines.  For N-D splines, N equations in the form of equation (2) must
 * be solved ... batched over the other dimensions"):  for each of the batch
 * 2-D grids F (n2 x n1, dim 1 contiguous), in place
 *     C = A1^{-1} F A2^{-T},   i.e. vec(C) = (A2 (x) A1)^{-1} vec(F),
 * A1 / A2 the collocation matrices of h1 (along dim 1) and h2 (along dim 2).
 * Element (i1, i2, b) at rhs[b*batch_stride + i2*n1 + i1], n1 = nbasis(h1),
 * n2 = nbasis(h2); batch_stride >= n1*n2 (ignored when batch == 1).
 * Two fused 1-D passes: dim 1 by the warp-per-RHS kernel (rows contiguous),
 * dim 2 by the tile kernel over slabs (3-D TMA).  Both handles on the same
 * device.  Asynchronous on stream.
 */
int spline_builder_solve_2d(spline_builder_t h1, spline_builder_t h2, void *rhs, int dtype, int64_t batch,
                            int64_t batch_stride, void *stream);

/*
 * spline_builder_advect -- one step of the 1-D semi-Lagrangian advection of
 * Algorithm 2 for a PERIODIC space, fused in one kernel:
 * for every right-hand side r (one v_j line of f(x_i, v_j), same layout rules
 * as spline_builder_solve_strided), the spline eta of f(., v_j) is built
 * (Algorithm 1) and f is overwritten, in place, with eta evaluated at the feet
 * of the characteristics:  f(xi_i, v_j) <- S_eta(xi_i - shift[r])  (periodic
 * wrap), xi_i the interpolation points.  No transposes: the point-contiguous
 * layout (batch_stride >= n, point_stride 1) is the fast path.
 *   f      DEVICE pointer, SB_F64 or SB_F32 (dtype)
 *   shift  DEVICE pointer to batch fp64 displacements (dt * v_j), in units of x
 * Returns SB_UNSUPPORTED for non-periodic spaces.  Asynchronous on stream.
 */
int spline_builder_advect(spline_builder_t h, void *f, int dtype, int64_t batch, int64_t batch_stride,
                          int64_t point_stride, const double *shift, void *stream);

/*
 * spline_builder_solve_host -- end-to-end solve of HOST data (fp64 or fp32,
 * batch-contiguous (n, batch) layout with leading dimension ld >= batch):
 * the batch is cut into chunks that are copied host->device, solved and
 * copied back on a pipeline of streams so that the copies overlap the
 * kernels.  host_rhs should be pinned (cudaHostRegister / cudaMallocHost)
 * for full PCIe bandwidth.  Synchronous: returns when the data is back.
 */
int spline_builder_solve_host(spline_builder_t h, void *host_rhs, int dtype, int64_t batch, int64_t ld);

void spline_builder_destroy(spline_builder_t h); /* caller syncs first; NULL ok */

/* ------------------------------------------------------------ queries */
typedef struct {
    int degree, bc, n_cells, nbasis;
    int split_lo, split_hi, k;      /* delta' is k x k, k = split_lo + split_hi */
    int q_kl, q_ku;                 /* band of Q (Table I type below)            */
    int q_type;                     /* 0 pttrs (sym tridiag), 1 pbtrs (sym band),
                                       2 gbtrs (general band, no interchanges)   */
    int nnz_lambda, nnz_beta;       /* COO sizes; beta kept if > 1e-14   */
    int beta_rows_head, beta_rows_tail; /* Q rows at each end touched by beta     */
    int nnz_Lambda, nnz_gamma;      /* Lambda = lambda Q^-1 (kept if > 1e-14) and
                                       gamma: the corner data the kernel uses      */
    int n_segments, seg_len;        /* in-CTA segment split of the Q recurrences
                                       (fp64 kernels)                             */
    int carry_fwd, carry_bwd;       /* predecessor segments in the carry walks    */
    double max_pivot_growth;        /* max |U| / max |Q| of the no-pivot LU        */
} spline_builder_info_t;

int spline_builder_get_info(spline_builder_t h, spline_builder_info_t *info);
int64_t spline_builder_nbasis(spline_builder_t h);

/* Host copies of the Schur blocks for inspection (any pointer may be NULL):
 * lambda COO (rows in [0,k), cols in [0,n-k)) and beta COO (rows in
 * [0,n-k), cols in [0,k)), indices are delta-/Q-local; delta' (k*k,
 * row-major, before LU).  Arrays must hold nnz / k*k entries. */
int spline_builder_get_blocks(spline_builder_t h, int *lam_rows, int *lam_cols, double *lam_vals, int *beta_rows,
                              int *beta_cols, double *beta_vals, double *delta_prime);

/* Host-side fp64 reference solve of the SAME factorisation (Algorithm 1 on
 * the CPU, serial).  Used by create's self-check; exported for tests of the
 * host plan.  Layout as spline_builder_solve_strided. */
int spline_builder_solve_cpu_plan(spline_builder_t h, double *rhs, int64_t batch, int64_t batch_stride,
                                  int64_t point_stride);

const char *spline_builder_last_error(void); /* thread-local; never NULL */
/* Kernel the last solve call on the calling thread launched, with its
 * configuration, e.g. "tile<f64,K=1,R=16,TMA>" (batch-contiguous tile kernel
 * fed by TMA), "warp<f64,K=1,L=33,BULK>", "serial<f64,K=3>"; "" before the
 * first solve.  Thread-local, never NULL; for tests and diagnostics. */
const char *spline_builder_last_kernel(void);
int spline_builder_last_status(void);        /* status of the last failed call */
const char *spline_builder_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPLINE_BUILDER_H */
