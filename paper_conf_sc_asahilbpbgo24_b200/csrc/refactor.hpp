// refactor.hpp -- device-side refactorisation of a handle for a new mesh
// (refactor.cu).  Plain structs; no torch, no host STL in the kernel.
#pragma once
#include <cstddef>
#include <cuda_runtime.h>

#include "device.hpp"

namespace sb {

// reasons in the device status word (0: committed)
enum {
    SB_RF_OK = 0, SB_RF_BADKNOTS = 1, SB_RF_DOMAIN = 2, SB_RF_STRUCTURE = 3, SB_RF_SINGULAR = 4, SB_RF_CARRY = 5,
    SB_RF_LAMBDA = 6, SB_RF_GAMMA = 7, SB_RF_BUCKETS = 8, SB_RF_SCALED = 9
};

struct RefactorArgs {
    DevPlan P;                  // live layout: pointers into the live blob (patterns read from there)
    int p;                      // degree
    double x0, xN;              // periodic: the domain ends fixed at create
    const double *knots;        // DEVICE, N+1 breakpoints (nullptr: uniform on [0, 1])
    const int *rowdesc;         // DEVICE, 3 ints per row: kind, index, derivative order (host/plan.hpp)
    const int *lam_ptr, *lam_c, *gam_r, *gam_c, *drow;  // frozen patterns (live blob)
    double *scr;                // DEVICE scratch of refactor_scratch_bytes()
    unsigned char *stage;       // DEVICE staging copy of the blob (same layout)
    unsigned char *live;        // the live blob
    size_t blob_bytes;
    int *status;                // DEVICE status word (SB_RF_*), written by the kernel
    size_t smem_bytes;          // set by the launcher: working set in shared memory (0: in scr)
};

size_t refactor_scratch_bytes(int n, int N, int nQ, int k, int K);
size_t refactor_smem_bytes(int nQ, int k, int K);
int launch_refactor(const RefactorArgs &a, cudaStream_t stream, char *err, int errlen);

}  // namespace sb
