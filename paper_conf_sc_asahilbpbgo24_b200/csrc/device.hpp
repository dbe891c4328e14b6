// device.hpp -- interface between the C ABI (capi.cpp) and the CUDA kernels
// (solve_kernels.cu).  Plain structs only; no torch, no host STL in kernels.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sb {

// Segment plan of one kernel family: Q padded to S*L rows, split into S
// register segments of L rows.  The factors of a segment form one block of
// (2K+1) rows of pitch LP (16-B aligned pairs; tile kernels LP = L+2 fp64 /
// L+4 fp32, warp kernel LP = L odd), so a thread needs ONE base address and
// every factor offset is a compile-time immediate:
//   F + slot[s]*(2K+1)*LP:  L(a+i, a+i-1-m)  at [m*LP + i]        (a = s*L)
//                           U'(a+i, a+i+1+m) at [(K+m)*LP + i]
//                           dinv(a+i)        at [2K*LP + i]         (1 on padding rows)
// Segments with bitwise-identical factors share a slot (broadcast reads).
// Floating-point arrays exist in fp64 ([0]) and fp32 ([1]).
struct DevSeg {
    int L, S, LP, carry_f, carry_b;
    int nslots;               // distinct factor blocks; segment s reads block slot[s]
    const int *slot;
    const void *F[2];         // nslots factor blocks of (2K+1)*LP, fp64 [0] / fp32 [1]
    const void *G[2], *H[2];  // S*K*K forward / backward segment transfer matrices
    const int *gptr;          // S+1: gamma COO entries of segment s are [gptr[s], gptr[s+1])
};

// Packed constants uploaded once at create ("copy the result
// to the device").
struct DevPlan {
    int n, nQ, s_lo, k, K;   // order, Q order, Q offset, delta order, kernel band
    int lam_nnz, gam_nnz;    // Lambda CSR / gamma COO sizes
    int corner_rows;         // rows [0,c) and [n-c,n) hold every row the corner reads (0: none/unbounded)
    const void *lam_v[2], *gam_v[2], *dlu[2], *dscale[2];
    const void *rowf[2];     // nQ x (2K+1): L(i,i-1..i-K), U'(i,i+1..i+K), dinv(i) -- serial fallback
    int p, N, periodic;      // spline degree, cells, periodic flag (advection / evaluation)
    const double *xe, *xi;   // periodic extended knots t_c at xe[c+p] (N+2p+1), n row positions
    int adv_uniform;         // uniform periodic mesh: Algorithm 2's evaluation is a per-row stencil
    double adv_invh, adv_q0; // 1/h, (xi_0 - x_0)/h
    const double *adv_rcp;   // non-uniform: 1/(t_{m+w} - t_m) at [(m+p)*(p|1) + w-1], m in [-p, N+p), w = 1..p
    const int *adv_tbl;      // non-uniform: bucket b of [x_0, x_N) -> cell of its left edge (bucket <= min cell)
    int adv_nbkt, adv_steps;
    double adv_bscale;       // adv_nbkt / (x_N - x_0)
    const int *lam_ptr, *lam_c, *gam_r, *gam_c, *dpiv, *drow;
    // Tile-kernel corner: Lambda on a dense column window, Q columns [0, lw_head)
    // then [nQ-lw_tail, nQ); lw_v[j*k + d] = Lambda(d, column j of the window)
    // (0 where dropped), so every shared-memory load of the spmv is independent
    // of the others (no column-index load in front of each b load)
    int lw_head, lw_tail;
    const void *lw_v[2];
    DevSeg seg[3];           // [0] tile kernel fp64 (L=36), [1] tile kernel fp32 (L=72),
                             // [2] warp-per-RHS kernel (odd L; S == 0 if unavailable)
};

struct SolveArgs {
    void *rhs;
    int64_t batch;
    int64_t bstride;   // elements between RHS
    int64_t pstride;   // elements between rows
    int dtype;         // 0 fp64, 1 fp32
    cudaStream_t stream;
    const double *shift = nullptr;  // advect: per-RHS displacement (device, fp64); nullptr = plain solve
    int64_t nslab = 1;              // independent (n, batch) blocks, slab_stride elements apart
    int64_t slab_stride = 0;
};

// name + configuration of the kernel the last launch_solve on this thread chose
const char *last_kernel();

// returns 0 on success, else an SB_* status; fills err on failure
int launch_solve(const DevPlan &P, const SolveArgs &a, int num_sms, char *err, int errlen);

}  // namespace sb
