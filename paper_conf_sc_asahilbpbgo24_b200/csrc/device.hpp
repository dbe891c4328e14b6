// device.hpp -- interface between the C ABI (capi.cpp) and the CUDA kernels
// (solve_kernels.cu).  Plain structs only; no torch, no host STL in kernels.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sb {

// segment plan of one compute precision (register segment length L)
struct DevSeg {
    int L, S, nQp, carry_f, carry_b;
    const void *G, *H;    // S*K*K forward / backward transfer matrices (compute type)
    const int *gptr;      // S+1: gamma COO entries of segment s are [gptr[s], gptr[s+1])
};

// Packed constants uploaded once at create ("copy the result
// to the device").  Floating-point sections exist in fp64 ([0]) and fp32 ([1]).
struct DevPlan {
    int n, nQ, s_lo, k, K;         // order, Q order, Q offset, delta order, kernel band
    int nQpa;                      // stride of the padded factor arrays
    int lam_nnz, gam_nnz;          // Lambda CSR / gamma COO sizes
    const void *Lr[2];             // K arrays of nQpa: L(i, i-1-m) at [m*nQpa + i]
    const void *Ur[2];             // K arrays of nQpa: U'(i, i+1+m) at [m*nQpa + i]
    const void *dinv[2];           // nQpa (1 on padding rows)
    const void *lam_v[2], *gam_v[2], *dlu[2], *dscale[2];
    const int *lam_ptr, *lam_c, *gam_r, *gam_c, *dpiv, *drow;
    DevSeg seg[2];                 // [0] fp64 kernels, [1] fp32 kernels
};

struct SolveArgs {
    void *rhs;
    int64_t batch;
    int64_t bstride;   // elements between RHS
    int64_t pstride;   // elements between rows
    int dtype;         // 0 fp64, 1 fp32
    cudaStream_t stream;
};

// returns 0 on success, else an SB_* status; fills err on failure
int launch_solve(const DevPlan &P, const SolveArgs &a, int num_sms, char *err, int errlen);

}  // namespace sb
