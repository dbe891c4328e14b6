// tile_f64.cu -- instantiations of the batch-contiguous tile kernel (double).
#include "kernels.cuh"

namespace sb {
int launch_tile_f64(int R, int loader, int K, const KParams &kp, const CUtensorMap *tm, int grid, int threads,
                    cudaStream_t st, char *err, int errlen) {
    const bool tma = loader == LOAD_TMA;
    if (R == 16) return tma ? tile_K<double, 36, 16, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen)
                          : tile_K<double, 36, 16, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
    if (R == 8) return tma ? tile_K<double, 36, 8, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen)
                         : tile_K<double, 36, 8, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
    snprintf(err, errlen, "unsupported tile width R=%d", R);
    return 5;
}
}  // namespace sb

#ifdef SB_TRACE
extern "C" int sb_trace_dump(long long *host, size_t bytes) {
    return (int)cudaMemcpyFromSymbol(host, sb::g_sb_trace, bytes);
}
#endif
