// tile_pair_f64.cu -- instantiations and launcher of the 2-CTA-cluster tile
// kernel (pair.cuh), fp64, segment length 36.
#include "pair.cuh"

namespace sb {

template <int K>
static int launch_pair_K(const KParams &kp, const CUtensorMap *tm, int grid, int threads, cudaStream_t st, char *err,
                         int errlen) {
    auto fn = sb_pair_kernel<K, 36>;
    if (smem_attr_once(fn) != cudaSuccess) return check_launch("cudaFuncSetAttribute(pair)", err, errlen);
    fn<<<grid, threads, kp.smem_total, st>>>(kp, tm[0]);
    return check_launch("pair tile kernel launch", err, errlen);
}

int launch_pair_f64(int K, const KParams &kp, const CUtensorMap *tm, int grid, int threads, cudaStream_t st, char *err,
                    int errlen) {
    switch (K) {
        case 1: return launch_pair_K<1>(kp, tm, grid, threads, st, err, errlen);
        case 2: return launch_pair_K<2>(kp, tm, grid, threads, st, err, errlen);
        case 3: return launch_pair_K<3>(kp, tm, grid, threads, st, err, errlen);
        case 4: return launch_pair_K<4>(kp, tm, grid, threads, st, err, errlen);
    }
    snprintf(err, errlen, "pair tile: unsupported band K=%d", K);
    return 5;
}

}  // namespace sb
