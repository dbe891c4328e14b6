// refactor.cu -- device-side refactorisation for a new mesh (SURVEY 8(f)4,
// BASELINE north_star "one-time host or device factorisation").
//
// A handle created with SB_FLAG_DEVICE_UPDATE has its structure frozen at
// create: degree, boundary conditions, Schur split, Q band, the sparsity
// patterns of gamma and Lambda (dilated by CORNER_MARGIN), the segment plans
// and carry-walk depths (one deeper), and the advection bucket table.  For new
// breakpoints (a DEVICE pointer) one single-block kernel recomputes every
// number the solve kernels read, in stream order, without a host round trip:
//   1. cell widths, interpolation points (Greville abscissae, end points,
//      midpoints) and the collocation rows by de Boor's BSPLVB / BSPLVD in
//      local coordinates (the same construction as the host
//      create, csrc/host/plan.cpp)
//   2. the Schur blocks of Eq. 3: Q band, gamma, lambda, delta
//   3. banded LU of Q without interchanges (Table I gbtrf; growth checked)
//   4. Lambda = lambda Q^{-1} (the transposed twin of Eq. 4's beta = Q^{-1} gamma,
//      DESIGN.md R6; beta itself is not read by the kernels)
//   5. delta' = delta - lambda beta = delta - Lambda gamma and getrf(delta') (Eq. 4-6)
//   6. the kernels' layouts: per-segment factor blocks, segment transfer
//      matrices G/H (and their carry depths), the serial-fallback rows, the
//      corner data (Lambda CSR / dense window, gamma COO, delta' LU), fp32
//      copies, and the periodic advection geometry
// into a staging copy of the handle's device blob; only if every check passed
// (a status word in device memory) is the staging copy committed over the
// live blob.  The DevPlan scalars (sizes, patterns) do not change, so kernels
// already captured in a CUDA graph keep working and see the new mesh.
#include <algorithm>
#include <cstdio>

#include "device.hpp"
#include "refactor.hpp"

namespace sb {
namespace {

constexpr double CORNER_DROP_D = 1e-14;  // |Lambda| kept above this (host plan: CORNER_DROP)

// ------------------------------------------------------- spline space (device)
struct DSpace {
    int p, periodic, N;
    const double *h;  // cell widths
    __device__ long lmod(long a, long m) const {
        long r = a % m;
        return r < 0 ? r + m : r;
    }
    __device__ double width(long g) const {
        if (periodic) return h[lmod(g, N)];
        return (g >= p && g < N + p) ? h[g - p] : 0.0;
    }
    __device__ double kd(long a, long b) const {  // t_a - t_b, a >= b, as a sum of widths
        double s = 0.0;
        for (long g = b; g < a; ++g) s += width(g);
        return s;
    }
    __device__ long first_knot(int j) const { return periodic ? j - (p + 1) / 2 : j; }
    __device__ int basis_of(long q, int n) const { return periodic ? (int)lmod(q + (p + 1) / 2, N) : (int)q; }
    __device__ long span_of_cell(int c) const { return periodic ? c : (long)c + p; }
};

// BSPLVB: the q+1 degree-q B-splines with first knots span-q .. span at t_span + u
__device__ void d_bsplvb(const DSpace &S, long mu, double u, int q, double *b) {
    double dl[8], dr[8];
    b[0] = 1.0;
    for (int j = 0; j < q; ++j) {
        dr[j] = S.kd(mu + 1 + j, mu) - u;
        dl[j] = u + S.kd(mu, mu - j);
        double saved = 0.0;
        for (int r = 0; r <= j; ++r) {
            const double den = dr[r] + dl[j - r];
            const double term = den > 0.0 ? b[r] / den : 0.0;
            b[r] = saved + dr[r] * term;
            saved = dl[j - r] * term;
        }
        b[j + 1] = saved;
    }
}

// d-th derivative of the p+1 degree-p B-splines (values of degree p-d, then d
// applications of the derivative recursion)
__device__ void d_bsplvd(const DSpace &S, long mu, double u, int d, double *out) {
    const int p = S.p;
    double v[8], w[8];
    d_bsplvb(S, mu, u, p - d, v);
    for (int q = p - d + 1; q <= p; ++q) {
        for (int r = 0; r <= q; ++r) {
            const long i = mu - q + r;
            double acc = 0.0;
            if (r - 1 >= 0) {
                const double den = S.kd(i + q, i);
                if (den > 0.0) acc += v[r - 1] / den;
            }
            if (r <= q - 1) {
                const double den = S.kd(i + q + 1, i + 1);
                if (den > 0.0) acc -= v[r] / den;
            }
            w[r] = q * acc;
        }
        for (int r = 0; r <= q; ++r) v[r] = w[r];
    }
    for (int r = 0; r <= p; ++r) out[r] = v[r];
}

// Greville abscissa of basis j as (span, u), snapped to a knot within rounding
__device__ void d_greville(const DSpace &S, int j, long &span, double &u) {
    const long q = S.first_knot(j);
    double off = 0.0;
    for (int l = 1; l <= S.p; ++l) off += S.kd(q + l, q);
    off /= S.p;
    {
        const double sp = S.kd(q + S.p + 1, q);
        for (int l = 0; l <= S.p + 1; ++l) {
            const double t = S.kd(q + l, q);
            if (fabs(off - t) <= 8.0 * 2.220446049250313e-16 * sp) { off = t; break; }
        }
    }
    long last = -1;
    double lastlo = 0.0;
    for (int l = 0; l <= S.p; ++l) {
        const long g = q + l;
        const double w = S.width(g);
        if (w <= 0.0) continue;
        const double lo = S.kd(g, q);
        last = g;
        lastlo = lo;
        if (off >= lo && off < lo + w) { span = g; u = off - lo; return; }
    }
    span = last;
    u = off - lastlo;
}

__device__ __forceinline__ void fail(int *st, int code) { atomicCAS(st, 0, code); }

// 7. commit: copy the staging blob over the live one iff every check passed
__global__ void sb_refactor_commit(const uint4 *__restrict__ src, uint4 *__restrict__ dst, size_t n16,
                                   const int *status) {
    if (*status != 0) return;
    for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < n16; e += (size_t)gridDim.x * blockDim.x)
        dst[e] = src[e];
}

// Banded LU of Q without interchanges (Table I gbtrf path) on one thread with
// the active (K+1) x (K+1) window in registers: at step j, A[r][c] = W(j+r, j+c).
// The window moves one row/column per step; the new row and column come from
// Q's original entries (no earlier step touched them).  W holds Q's band by
// rows, W[i*BW + (c - i + K)]; on exit it holds L below the diagonal and U on
// and above it.  Returns max |l| and max |u| for the growth check.
template <int K>
__device__ void band_lu_window(double *W, int nQ, double qmax, int *st, double &lmax, double &umax) {
    constexpr int BW = 2 * K + 1;
    double A[K + 1][K + 1];
#pragma unroll
    for (int r = 0; r <= K; ++r)
#pragma unroll
        for (int c = 0; c <= K; ++c) A[r][c] = (r < nQ && c < nQ) ? W[r * BW + (c - r + K)] : 0.0;
    lmax = umax = 0.0;
    for (int j = 0; j < nQ; ++j) {
        // the entries entering the window after this step (never written by it): loaded
        // first, so they are in flight during the step's dependent reciprocal / FMAs
        const int nr = j + K + 1;
        double nrow[K + 1], ncol[K];
#pragma unroll
        for (int c = 0; c <= K; ++c) nrow[c] = nr < nQ ? W[(size_t)nr * BW + c] : 0.0;
#pragma unroll
        for (int r = 0; r < K; ++r) {
            const int row = j + 1 + r;
            ncol[r] = (row < nQ && nr < nQ) ? W[(size_t)row * BW + K + (K - r)] : 0.0;
        }
        const double pv = A[0][0];
        if (!(fabs(pv) > 1e-13 * qmax)) { fail(st, SB_RF_SINGULAR); return; }
        const double rp = 1.0 / pv;
#pragma unroll
        for (int r = 1; r <= K; ++r) {
            const double l = A[r][0] * rp;
            if (j + r < nQ) {
                W[(size_t)(j + r) * BW + (K - r)] = l;  // L(j+r, j)
                lmax = fmax(lmax, fabs(l));
            }
#pragma unroll
            for (int c = 1; c <= K; ++c) A[r][c] = fma(-l, A[0][c], A[r][c]);
        }
#pragma unroll
        for (int c = 0; c <= K; ++c)
            if (j + c < nQ) {
                W[(size_t)j * BW + K + c] = A[0][c];  // U(j, j+c)
                umax = fmax(umax, fabs(A[0][c]));
            }
#pragma unroll
        for (int r = 0; r < K; ++r)
#pragma unroll
            for (int c = 0; c < K; ++c) A[r][c] = A[r + 1][c + 1];
        // new last row j+K+1 (columns j+1 .. j+K+1) and new last column j+K+1 (rows j+1 .. j+K)
#pragma unroll
        for (int c = 0; c <= K; ++c) A[K][c] = nrow[c];
#pragma unroll
        for (int r = 0; r < K; ++r) A[r][K] = ncol[r];
    }
}

// ================================================================= kernel
template <int K>
__global__ void __launch_bounds__(256, 1) sb_refactor_kernel(const RefactorArgs a) {
    const DevPlan &P = a.P;
    const int tid = threadIdx.x, nth = blockDim.x;
    const int p = a.p, N = P.N, n = P.n, nQ = P.nQ, k = P.k, s_lo = P.s_lo;
    constexpr int BW = 2 * K + 1;
    int *st = a.status;
    if (tid == 0) *st = 0;
    // every thread takes the same branch: read the status word between two barriers
#define SB_RF_CHECK()                 \
    do {                              \
        __syncthreads();              \
        const int bad_ = *st;         \
        __syncthreads();              \
        if (bad_) goto done;          \
    } while (0)
    // global scratch: mesh and rows (parallel phases); the mesh (read by every
    // knot-difference sum of the BSPLVB recursions) is mirrored in shared memory
    double *hg = a.scr, *xbg = hg + N, *rows = xbg + N + 1;  // rows: 8 doubles per collocation row
    double *rsc = rows + (size_t)n * 8;                   // n row scales
    double *del = rsc + n, *dp = del + (size_t)k * k, *lu = dp + (size_t)k * k;
    int *piv = reinterpret_cast<int *>(lu + (size_t)k * k);
    double *gcopy = reinterpret_cast<double *>(piv + 64);  // gamma (for delta' and the pattern check)
    // the sequential working set (Q band -> its LU in place, lambda -> Lambda) lives in shared memory when it fits (a.smem_bytes > 0), else in scratch
    extern __shared__ __align__(16) double rf_smem[];
    double *wbase = a.smem_bytes ? rf_smem : gcopy + (size_t)nQ * k;
    double *Qb = wbase, *gam = Qb + (size_t)nQ * BW, *lam = gam + (size_t)nQ * k;
    const bool mesh_smem = a.smem_bytes >= ((size_t)nQ * BW + (size_t)nQ * k * 2 + (size_t)(2 * N + 1)) * 8;
    double *h = mesh_smem ? lam + (size_t)k * nQ : hg, *xb = mesh_smem ? h + N : xbg;
    double *Lam = lam;  // solved in place
    // factors in place in Qb after step 3: L(i, i-m), 1/U(i,i), U(i,i+m)/U(i,i)
#define LB(i, m) Qb[(size_t)(i) * BW + K - (m)]
#define UB(i, m) Qb[(size_t)(i) * BW + K + (m)]
#define DINV(i) Qb[(size_t)(i) * BW + K]
    __syncthreads();
    // ---------------------------------------------------------- 1. mesh
    for (int c = tid; c <= N; c += nth) xb[c] = a.knots ? a.knots[c] : (double)c / (double)N;
    __syncthreads();
    for (int c = tid; c < N; c += nth) {
        h[c] = a.knots ? xb[c + 1] - xb[c] : 1.0 / (double)N;
        if (!(h[c] > 0.0) || !isfinite(h[c])) fail(st, SB_RF_BADKNOTS);
    }
    if (tid == 0 && P.periodic && (xb[0] != a.x0 || xb[N] != a.xN)) fail(st, SB_RF_DOMAIN);
    for (int i = tid; i < nQ * BW; i += nth) Qb[i] = 0.0;
    for (int i = tid; i < nQ * k; i += nth) gam[i] = lam[i] = 0.0;
    for (int i = tid; i < k * k; i += nth) del[i] = 0.0;
    SB_RF_CHECK();
    {
        const DSpace S{p, P.periodic, N, h};
        // ------------------------------------------------ collocation rows
        for (int i = tid; i < n; i += nth) {
            const int kind = a.rowdesc[3 * i], idx = a.rowdesc[3 * i + 1], der = a.rowdesc[3 * i + 2];
            long span = 0;
            double u = 0.0, sc = 1.0;
            switch (kind) {
                case 0: d_greville(S, idx, span, u); break;                                  // ROW_GREVILLE
                case 1: span = S.span_of_cell(idx); u = 0.0; break;                          // ROW_BREAK
                case 2: span = S.span_of_cell(N - 1); u = h[N - 1]; break;                   // ROW_END
                case 3: span = S.span_of_cell(idx); u = 0.5 * h[idx]; break;                 // ROW_MID
                case 4: span = S.span_of_cell(0); u = 0.0; sc = pow(h[0], der); break;       // ROW_DER0
                default: span = S.span_of_cell(N - 1); u = h[N - 1]; sc = pow(h[N - 1], der); break;
            }
            double v[8];
            if (der == 0) d_bsplvb(S, span, u, p, v);
            else d_bsplvd(S, span, u, der, v);
            rsc[i] = sc;
            for (int r = 0; r <= p; ++r) rows[(size_t)i * 8 + r] = v[r] * sc;
            // interpolation point (advection data)
            const long cell = P.periodic ? S.lmod(span, N) : span - p;
            rows[(size_t)i * 8 + 7] = xb[cell] + u;
            // scatter into the Schur blocks (the row is owned by this thread)
            const int dg = i < s_lo ? i : (i >= n - (k - s_lo) ? s_lo + (i - (n - (k - s_lo))) : -1);
            for (int r = 0; r <= p; ++r) {
                const int c = S.basis_of(span - p + r, n);
                const double val = v[r] * sc;
                const int dc = c < s_lo ? c : (c >= n - (k - s_lo) ? s_lo + (c - (n - (k - s_lo))) : -1);
                if (dg < 0 && dc < 0) {
                    const int o = c - i;
                    if (o < -K || o > K) { if (val != 0.0) fail(st, SB_RF_STRUCTURE); }
                    else Qb[(size_t)(i - s_lo) * BW + (o + K)] += val;
                } else if (dg < 0) {
                    gam[(size_t)(i - s_lo) * k + dc] += val;
                } else if (dc < 0) {
                    lam[(size_t)dg * nQ + (c - s_lo)] += val;
                } else {
                    del[(size_t)dg * k + dc] += val;
                }
            }
            // every scaled (derivative) row must be a delta row
            if (dg < 0 && sc != 1.0) fail(st, SB_RF_SCALED);
        }
    }
    SB_RF_CHECK();
    for (int i = tid; i < nQ * k; i += nth) gcopy[i] = gam[i];
    // ---------------------------------------------- 3. LU of Q, no interchanges
    {
        __shared__ double red[256];
        double m = 0.0;
        for (int i = tid; i < nQ * BW; i += nth) m = fmax(m, fabs(Qb[i]));
        red[tid] = m;
        __syncthreads();
        for (int w = nth / 2; w > 0; w >>= 1) {
            if (tid < w) red[tid] = fmax(red[tid], red[tid + w]);
            __syncthreads();
        }
        const double qmax = red[0];
        if (tid == 0) {
            double lmax, umax;
            band_lu_window<K>(Qb, nQ, qmax, st, lmax, umax);
            if (!*st && (lmax > 1e3 || umax > 1e3 * qmax)) fail(st, SB_RF_SINGULAR);
        }
    }
    SB_RF_CHECK();
    // scale U rows by 1/U(i,i) and keep 1/U(i,i) on the diagonal
    for (int i = tid; i < nQ; i += nth) {
        const double d = 1.0 / Qb[(size_t)i * BW + K];
        Qb[(size_t)i * BW + K] = d;
#pragma unroll
        for (int m = 1; m <= K; ++m) Qb[(size_t)i * BW + K + m] *= d;
    }
    __syncthreads();
    // ---------------------------------------------- 4. Lambda = lambda Q^-1 (one thread per row;
    // the last K values of each recurrence stay in registers).  beta = Q^-1 gamma is not
    // needed on the device: the kernels use Lambda and gamma, and delta' = delta - Lambda gamma
    if (tid < k) {  // Lambda(c, :) in place of lambda(c, :)
        const int c = tid;
        double win[K];
        {  // Lambda(c, :): Q^T w = lambda(c, :)^T with Q = L D (I + U'), in place in lam
            double *__restrict__ w = Lam + (size_t)c * nQ;
            const double *__restrict__ Qr = Qb;  // the factors: loads may run ahead of the stores to w
#pragma unroll
            for (int m = 0; m < K; ++m) win[m] = 0.0;  // win[m] = w_{j-1-m}
            for (int j = 0; j < nQ; ++j) {
                double acc = w[j];
#pragma unroll
                for (int m = K; m >= 1; --m) acc = j - m >= 0 ? fma(-Qr[(size_t)(j - m) * BW + K + m], win[m - 1], acc) : acc;
#pragma unroll
                for (int m = K - 1; m > 0; --m) win[m] = win[m - 1];
                win[0] = acc;
                w[j] = acc * Qr[(size_t)j * BW + K];
            }
#pragma unroll
            for (int m = 0; m < K; ++m) win[m] = 0.0;  // win[m] = w_{j+1+m}
            for (int j = nQ - 1; j >= 0; --j) {
                double acc = w[j];
#pragma unroll
                for (int m = K; m >= 1; --m) acc = j + m < nQ ? fma(-Qr[(size_t)(j + m) * BW + K - m], win[m - 1], acc) : acc;
#pragma unroll
                for (int m = K - 1; m > 0; --m) win[m] = win[m - 1];
                win[0] = acc;
                w[j] = acc;
            }
        }
    }
    __syncthreads();
    // ---------------------------------------------- 5. delta' = delta - lambda beta = delta - Lambda gamma
    for (int e = tid; e < k * k; e += nth) {
        const int r = e / k, c = e % k;
        double acc = 0.0;
        for (int i = 0; i < nQ; ++i) acc = fma(Lam[(size_t)r * nQ + i], gcopy[(size_t)i * k + c], acc);
        dp[e] = del[e] - acc;
    }
    __syncthreads();
    if (tid == 0 && k > 0) {
        double dmax = 0.0;
        for (int e = 0; e < k * k; ++e) { lu[e] = dp[e]; dmax = fmax(dmax, fabs(dp[e])); }
        for (int j = 0; j < k; ++j) {
            int pr = j;
            double best = fabs(lu[j * k + j]);
            for (int i = j + 1; i < k; ++i)
                if (fabs(lu[i * k + j]) > best) { best = fabs(lu[i * k + j]); pr = i; }
            piv[j] = pr;
            if (!(best > 1e-13 * dmax)) { fail(st, SB_RF_SINGULAR); break; }
            if (pr != j)
                for (int c = 0; c < k; ++c) { const double t = lu[j * k + c]; lu[j * k + c] = lu[pr * k + c]; lu[pr * k + c] = t; }
            for (int i = j + 1; i < k; ++i) {
                const double l = lu[i * k + j] / lu[j * k + j];
                lu[i * k + j] = l;
                for (int c = j + 1; c < k; ++c) lu[i * k + c] -= l * lu[j * k + c];
            }
        }
    }
    SB_RF_CHECK();
    {
        // ------------------------------------------ 6. the kernels' layouts
        auto S8 = [&](const void *live) { return reinterpret_cast<double *>(a.stage + ((const unsigned char *)live - a.live)); };
        auto S4 = [&](const void *live) { return reinterpret_cast<float *>(a.stage + ((const unsigned char *)live - a.live)); };
        auto SI = [&](const void *live) { return reinterpret_cast<int *>(a.stage + ((const unsigned char *)live - a.live)); };
        // segment plans: factor blocks (identity padding) and transfer matrices
        for (int g = 0; g < 3; ++g) {
            const DevSeg &G = P.seg[g];
            if (G.S == 0) continue;
            const int L = G.L, Sg = G.S, LP = G.LP;
            // transfer-matrix layout as in upload (capi.cpp): warp plan [j][m][t], tile plans [t][j][m]
            auto gidx = [&](int t, int j, int m) -> size_t {
                return g == 2 ? ((size_t)j * K + m) * Sg + t : ((size_t)t * K + j) * K + m;
            };
            double *F8 = S8(G.F[0]);
            float *F4 = S4(G.F[1]);
            const size_t BS = (size_t)BW * LP;
            for (int sb = tid; sb < G.nslots * BW; sb += nth) {  // one factor row (slot s, band b) per thread
                const int s = sb / BW, b = sb - s * BW;
                const size_t e0 = (size_t)s * BS + (size_t)b * LP;
                for (int i = 0; i < LP; ++i) {
                    const int row = s * L + i;
                    double v = b == 2 * K ? 1.0 : 0.0;
                    if (i < L && row < nQ) {
                        if (b < K) v = LB(row, b + 1);
                        else if (b < 2 * K) v = UB(row, b - K + 1);
                        else v = DINV(row);
                    }
                    F8[e0 + i] = v;
                    F4[e0 + i] = (float)v;
                }
            }
            double *G8 = S8(G.G[0]), *H8 = S8(G.H[0]);
            float *G4 = S4(G.G[1]), *H4 = S4(G.H[1]);
            for (int e = tid; e < Sg * K; e += nth) {
                const int t = e / K, m = e % K + 1;
                // forward: response of segment t to inflow unit m, at rows a+L-1-j
                if (t >= 1) {
                    double yf[8];  // rolling window: yf[q] = y_{a+i-1-q}
                    for (int q = 0; q < K; ++q) yf[q] = q == m - 1 ? 1.0 : 0.0;  // inflow unit: y_{a-m} = 1
                    double last[8];
                    for (int q = 0; q < K; ++q) last[q] = 0.0;
                    const int a0 = t * L;
                    for (int i = 0; i < L; ++i) {
                        const int row = a0 + i;
                        double acc = 0.0;
                        for (int mm = 1; mm <= K; ++mm) acc -= (row < nQ ? LB(row, mm) : 0.0) * yf[mm - 1];
                        for (int q = K - 1; q > 0; --q) yf[q] = yf[q - 1];
                        yf[0] = acc;
                        if (i >= L - K) last[L - 1 - i] = acc;
                    }
                    for (int j = 0; j < K; ++j) {
                        G8[gidx(t, j, m - 1)] = last[j];
                        G4[gidx(t, j, m - 1)] = (float)last[j];
                    }
                } else {
                    for (int j = 0; j < K; ++j) { G8[gidx(0, j, m - 1)] = 0.0; G4[gidx(0, j, m - 1)] = 0.f; }
                }
                // backward: response of segment t to outflow unit m, at rows a+j
                if (t + 1 < Sg) {
                    double yb[8];  // yb[q] = x_{a+i+1+q}
                    for (int q = 0; q < K; ++q) yb[q] = (q == m - 1) ? 1.0 : 0.0;
                    double first[8];
                    const int a0 = t * L;
                    for (int i = L - 1; i >= 0; --i) {
                        const int row = a0 + i;
                        double acc = 0.0;
                        for (int mm = 1; mm <= K; ++mm) acc -= (row < nQ ? UB(row, mm) : 0.0) * yb[mm - 1];
                        for (int q = K - 1; q > 0; --q) yb[q] = yb[q - 1];
                        yb[0] = acc;
                        if (i < K) first[i] = acc;
                    }
                    for (int j = 0; j < K; ++j) {
                        H8[gidx(t, j, m - 1)] = first[j];
                        H4[gidx(t, j, m - 1)] = (float)first[j];
                    }
                } else {
                    for (int j = 0; j < K; ++j) {
                        H8[gidx(t, j, m - 1)] = 0.0;
                        H4[gidx(t, j, m - 1)] = 0.f;
                    }
                }
            }
        }
        __syncthreads();
        // carry depths: the frozen walks must still reach the 2^-60 bound
        for (int g = 0; g < 3; ++g)
        for (int s = tid; s < P.seg[g].S; s += nth) {
            const DevSeg &G = P.seg[g];
            const double *G8 = S8(G.G[0]), *H8 = S8(G.H[0]);
            auto nrm = [&](const double *M, int t) {
                double r = 0.0;
                for (int j = 0; j < K; ++j) {
                    double sum = 0.0;
                    for (int m = 0; m < K; ++m) sum += fabs(M[g == 2 ? ((size_t)j * K + m) * G.S + t : ((size_t)t * K + j) * K + m]);
                    r = fmax(r, sum);
                }
                return r;
            };
            const double eps = 8.673617379884035e-19;  // 2^-60
            if (s >= 1) {
                int T = 0;
                double prod = 1.0;
                while (true) {
                    ++T;
                    const int t = s - T;
                    if (t == 0) break;
                    prod *= nrm(G8, t);
                    if (prod <= eps) break;
                }
                if (T > G.carry_f) fail(st, SB_RF_CARRY);
            }
            if (s + 1 < G.S) {
                int T = 0;
                double prod = 1.0;
                while (true) {
                    ++T;
                    const int t = s + T;
                    if (t == G.S - 1) break;
                    prod *= nrm(H8, t);
                    if (prod <= eps) break;
                }
                if (T > G.carry_b) fail(st, SB_RF_CARRY);
            }
        }
        // serial-fallback rows
        {
            double *R8 = S8(P.rowf[0]);
            float *R4 = S4(P.rowf[1]);
            for (int e = tid; e < nQ * BW; e += nth) {
                const int i = e / BW, b = e % BW;
                const double v = b < K ? LB(i, b + 1) : (b < 2 * K ? UB(i, b - K + 1) : DINV(i));
                R8[e] = v;
                R4[e] = (float)v;
            }
        }
        // corner data: Lambda CSR values on the frozen pattern (+ pattern check),
        // its dense window, gamma COO values (+ check), delta' LU, row scales
        {   // values on the pattern, then: no entry above the threshold off the pattern
            // (the pattern's entries of Lambda are zeroed after being read)
            double *LV8 = S8(P.lam_v[0]);
            float *LV4 = S4(P.lam_v[1]);
            for (int d = 0; d < k; ++d)
                for (int e = a.lam_ptr[d] + tid; e < a.lam_ptr[d + 1]; e += nth) {
                    const double v = Lam[(size_t)d * nQ + a.lam_c[e]];
                    LV8[e] = v;
                    LV4[e] = (float)v;
                }
        }
        {
            const int lh = P.lw_head, lw = P.lw_head + P.lw_tail;
            double *W8 = S8(P.lw_v[0]);
            float *W4 = S4(P.lw_v[1]);
            for (int e = tid; e < lw * k; e += nth) { W8[e] = 0.0; W4[e] = 0.f; }
            __syncthreads();
            for (int d = 0; d < k; ++d) {
                for (int e = a.lam_ptr[d] + tid; e < a.lam_ptr[d + 1]; e += nth) {
                    const int c = a.lam_c[e];
                    const int j = c < lh ? c : lh + (c - (nQ - P.lw_tail));
                    const double v = Lam[(size_t)d * nQ + c];
                    if (j >= 0 && j < lw) { W8[(size_t)j * k + d] = v; W4[(size_t)j * k + d] = (float)v; }
                }
            }
            __syncthreads();
            for (int d = 0; d < k; ++d)
                for (int e = a.lam_ptr[d] + tid; e < a.lam_ptr[d + 1]; e += nth) Lam[(size_t)d * nQ + a.lam_c[e]] = 0.0;
            __syncthreads();
            for (int i = tid; i < k * nQ; i += nth)
                if (fabs(Lam[i]) > CORNER_DROP_D) fail(st, SB_RF_LAMBDA);
        }
        {
            double *GV8 = S8(P.gam_v[0]);
            float *GV4 = S4(P.gam_v[1]);
            for (int e = tid; e < P.gam_nnz; e += nth) {
                const double v = gcopy[(size_t)a.gam_r[e] * k + a.gam_c[e]];
                GV8[e] = v;
                GV4[e] = (float)v;
            }
            // every structural nonzero of gamma must be in the frozen pattern: zero the
            // pattern's entries of the copy, then no nonzero may remain
            __syncthreads();
            for (int e = tid; e < P.gam_nnz; e += nth) gcopy[(size_t)a.gam_r[e] * k + a.gam_c[e]] = 0.0;
            __syncthreads();
            for (int i = tid; i < nQ * k; i += nth)
                if (gcopy[i] != 0.0) fail(st, SB_RF_GAMMA);
        }
        if (tid == 0) {
            double *D8 = S8(P.dlu[0]), *DS8 = S8(P.dscale[0]);
            float *D4 = S4(P.dlu[1]), *DS4 = S4(P.dscale[1]);
            int *DP = SI(P.dpiv);
            for (int e = 0; e < k * k; ++e) { D8[e] = lu[e]; D4[e] = (float)lu[e]; }
            for (int d = 0; d < k; ++d) {
                DP[d] = piv[d];
                const double sc = rsc[a.drow[d]];
                DS8[d] = sc;
                DS4[d] = (float)sc;
            }
        }
        // interpolation points and, for periodic spaces, the advection geometry
        {
            double *XI = S8(P.xi);
            for (int i = tid; i < n; i += nth) XI[i] = rows[(size_t)i * 8 + 7];
        }
        if (P.periodic) {
            const double Lp = xb[N] - xb[0];
            double *XE = S8(P.xe);
            for (int c = -p + tid; c <= N + p; c += nth)
                XE[c + p] = c < 0 ? xb[c + N] - Lp : (c > N ? xb[c - N] + Lp : xb[c]);
            __syncthreads();
            double *RC = S8(P.adv_rcp);
            const int RS = p | 1;
            for (int e = tid; e < (N + 2 * p) * RS; e += nth) {
                const int m = e / RS - p, w = e % RS + 1;
                double v = 0.0;
                if (w <= p && m + w <= N + p) v = 1.0 / (XE[m + w + p] - XE[m + p]);
                RC[e] = v;
            }
            int *TB = SI(P.adv_tbl);
            const int MT = P.adv_nbkt;
            const double w = Lp / MT, margin = 1e-9 * w;
            auto cell_of = [&](double x) {
                int lo = 0, hi = N - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) / 2;
                    if (xb[mid] <= x) lo = mid;
                    else hi = mid - 1;
                }
                return lo;
            };
            for (int b = tid; b < MT; b += nth) {
                const int lo = cell_of(xb[0] + b * w - margin);
                const int hi = cell_of(xb[0] + (b + 1) * w + margin);
                TB[b] = lo;
                if (hi - lo > P.adv_steps) fail(st, SB_RF_BUCKETS);
            }
        }
    }
    __syncthreads();
done:
    __syncthreads();
    // (7. the commit of the staging copy is a separate, grid-wide kernel)
#undef SB_RF_CHECK
#undef LB
#undef UB
#undef DINV
}

}  // namespace

size_t refactor_scratch_bytes(int n, int N, int nQ, int k, int K) {
    const size_t BW = 2 * K + 1;
    const size_t d = (size_t)N + (N + 1) + (size_t)n * 8 + n + (size_t)k * k * 3;  // h, xb, rows, rsc, del, dp, lu
    const size_t w = (size_t)nQ * BW + (size_t)nQ * k * 2;                            // Q band, gamma, lambda
    return (d + 32) * 8 + (size_t)nQ * k * 8 + w * 8 + 256;
}

size_t refactor_smem_bytes(int nQ, int k, int K) {
    return ((size_t)nQ * (2 * K + 1) + (size_t)nQ * k * 2) * 8;
}

namespace {
template <int K>
int launch_refactor_K(RefactorArgs a, cudaStream_t stream) {
    // the sequential working set in shared memory when it fits (else global scratch)
    // (plus the mesh, h and breakpoints, when that fits too)
    const size_t need0 = refactor_smem_bytes(a.P.nQ, a.P.k, K);
    const size_t mesh = (size_t)(2 * a.P.N + 1) * 8;
    int dev = 0, maxs = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    a.smem_bytes = need0 + mesh + 4096 <= (size_t)maxs ? need0 + mesh : (need0 + 4096 <= (size_t)maxs ? need0 : 0);
    if (a.smem_bytes) {
        static bool set[64] = {false};
        if (dev >= 0 && dev < 64 && !set[dev]) {
            cudaFuncSetAttribute(sb_refactor_kernel<K>, cudaFuncAttributeMaxDynamicSharedMemorySize, maxs - 4096);
            set[dev] = true;
        }
    }
    sb_refactor_kernel<K><<<1, 256, a.smem_bytes, stream>>>(a);
    const size_t n16 = a.blob_bytes / 16;
    const int blocks = (int)std::min<size_t>(148, (n16 + 255) / 256);
    sb_refactor_commit<<<std::max(blocks, 1), 256, 0, stream>>>(reinterpret_cast<const uint4 *>(a.stage),
                                                                reinterpret_cast<uint4 *>(a.live), n16, a.status);
    return 0;
}

}  // namespace

int launch_refactor(const RefactorArgs &a, cudaStream_t stream, char *err, int errlen) {
    switch (a.P.K) {
        case 1: launch_refactor_K<1>(a, stream); break;
        case 2: launch_refactor_K<2>(a, stream); break;
        case 3: launch_refactor_K<3>(a, stream); break;
        case 4: launch_refactor_K<4>(a, stream); break;
        default: snprintf(err, errlen, "refactor: unsupported band K=%d", a.P.K); return 5;
    }
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        snprintf(err, errlen, "refactor kernel launch: %s", cudaGetErrorString(e));
        return 3;
    }
    return 0;
}

}  // namespace sb
