// warp_f64.cu -- instantiations of the warp-per-RHS kernel (double), plain solve.
#include "kernels.cuh"

namespace sb {
int launch_warp_f64(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    if (kp.adv) return launch_warp_adv_f64(K, L, kp, grid, st, err, errlen);
    return warp_K<double, false>(K, L, kp, grid, st, err, errlen);
}
}  // namespace sb
