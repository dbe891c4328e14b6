// warp_f32.cu -- instantiations of the warp-per-RHS kernel (float), plain solve.
#include "kernels.cuh"

namespace sb {
int launch_warp_f32(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    if (kp.adv) return launch_warp_adv_f32(K, L, kp, grid, st, err, errlen);
    return warp_K<float, false>(K, L, kp, grid, st, err, errlen);
}
}  // namespace sb
