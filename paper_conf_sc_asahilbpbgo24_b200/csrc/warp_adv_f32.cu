// warp_adv_f32.cu -- instantiations of the warp-per-RHS kernel (float) with the
// fused Algorithm-2 evaluation (spline_builder_advect); own TU for build parallelism.
#include "kernels.cuh"

namespace sb {
int launch_warp_adv_f32(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    return warp_K<float, true>(K, L, kp, grid, st, err, errlen);
}
}  // namespace sb
