// device.hpp -- interface between the C ABI (capi.cpp) and the CUDA kernels
// (solve_kernels.cu).  Plain structs only; no torch, no host STL in kernels.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sb {

// Packed constant blob uploaded once at create ("copy the
// result to the device").  Offsets are in bytes from the blob base; each
// section is 16-byte aligned.  Both an fp64 and an fp32 copy of the
// floating-point sections are stored (fp32 compute path).
struct DevPlan {
    int n, nQ, s_lo, k, K;          // order, Q order, Q offset, delta order, band
    int S, seg_base, seg_rem;       // segments of the Q recurrences
    int carry_f, carry_b;           // carry-walk depths
    int Wh, Wt, nlam;               // window sizes, nnz(lambda)
    // record strides (elements): forward = 2K (L, g), backward = 2K+2 (dinv, U', h, pad)
    int fstride, bstride;
    // device pointers (fp64 then fp32 copies)
    const void *fwd[2], *bwd[2], *betaW[2], *lam_v[2], *dlu[2], *dscale[2];
    const int *lam_r, *lam_slot, *dpiv, *drow;
};

enum LayoutKind { LAYOUT_BATCH_CONTIG = 0, LAYOUT_STRIDED = 1 };

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

// bytes of dynamic shared memory the constant sections need (for validation)
size_t const_smem_bytes(const DevPlan &P, int dtype);

}  // namespace sb
