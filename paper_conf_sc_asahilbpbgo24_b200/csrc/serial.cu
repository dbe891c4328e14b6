// serial.cu -- instantiations of the serial (one thread per RHS) fallback kernel.
#include "kernels.cuh"

namespace sb {
template <typename T, int K>
static int launch_serial_t(const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    sb_serial_kernel<T, K><<<grid, 128, 0, st>>>(kp);
    return check_launch("serial kernel launch", err, errlen);
}

int launch_serial(int dtype, int K, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    switch (K * 2 + dtype) {
        case 2: return launch_serial_t<double, 1>(kp, grid, st, err, errlen);
        case 3: return launch_serial_t<float, 1>(kp, grid, st, err, errlen);
        case 4: return launch_serial_t<double, 2>(kp, grid, st, err, errlen);
        case 5: return launch_serial_t<float, 2>(kp, grid, st, err, errlen);
        case 6: return launch_serial_t<double, 3>(kp, grid, st, err, errlen);
        case 7: return launch_serial_t<float, 3>(kp, grid, st, err, errlen);
        case 8: return launch_serial_t<double, 4>(kp, grid, st, err, errlen);
        case 9: return launch_serial_t<float, 4>(kp, grid, st, err, errlen);
    }
    snprintf(err, errlen, "unsupported band K=%d", K);
    return 5;
}
}  // namespace sb
