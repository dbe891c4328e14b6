// warp_f32.cu -- instantiations of the warp-per-RHS kernel (float).
#include "kernels.cuh"

namespace sb {
int launch_warp_f32(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    return warp_K<float>(K, L, kp, grid, st, err, errlen);
}
}  // namespace sb
