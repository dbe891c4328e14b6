// warp_f64.cu -- instantiations of the warp-per-RHS kernel (double).
#include "kernels.cuh"

namespace sb {
int launch_warp_f64(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    return warp_K<double>(K, L, kp, grid, st, err, errlen);
}
}  // namespace sb
