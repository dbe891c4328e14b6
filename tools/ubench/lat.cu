// Latency microbenchmark (diagnostic): dependent DFMA chain, dependent LDS
// chain, and a K=3 banded forward recurrence over smem factors, one warp and
// 16 warps per SM.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 lat.cu -o lat
#include <cstdio>
#include <cuda_runtime.h>

__global__ void dfma_chain(double *out, long long *cyc, int n) {
    double a = out[threadIdx.x], b = 1.0000001, c = 1e-9;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u) a = fma(a, b, c);
    }
    long long t1 = clock64();
    out[threadIdx.x] = a;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void lds_chain(double *out, long long *cyc, int n) {
    __shared__ int idx[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) idx[i] = (i + 1) & 1023;
    __syncthreads();
    int j = threadIdx.x & 1;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u) j = idx[j];
    }
    long long t1 = clock64();
    out[threadIdx.x] = j;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// independent DFMA chains: throughput of the fp64 pipe
template <int CH>
__global__ void dfma_tput(double *out, long long *cyc, int n) {
    double a[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) a[c] = out[threadIdx.x] + c;
    const double b = 1.0000001, d = 1e-9;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int c = 0; c < CH; ++c) a[c] = fma(a[c], b, d);
    }
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += a[c];
    out[threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// y_i = b_i - l0 y_{i-1} - l1 y_{i-2} - l2 y_{i-3}, factors from smem (pairs), 36 rows, repeated
template <int K>
__global__ void band_fwd(double *out, long long *cyc, int reps) {
    __shared__ __align__(16) double f[K * 38 * 2];
    for (int i = threadIdx.x; i < K * 38 * 2; i += blockDim.x) f[i] = 0.01 * (i % 7);
    __syncthreads();
    double v[36];
#pragma unroll
    for (int i = 0; i < 36; ++i) v[i] = out[i * blockDim.x + threadIdx.x];
    const double *fl = f + (threadIdx.x >> 4 & 1) * K * 38;
    long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
        double st[K];
#pragma unroll
        for (int m = 0; m < K; ++m) st[m] = 0.0;
#pragma unroll
        for (int i = 0; i < 36; i += 2) {
            double l0[K], l1[K];
#pragma unroll
            for (int m = 0; m < K; ++m) {
                double2 w = *reinterpret_cast<const double2 *>(fl + m * 38 + i);
                l0[m] = w.x; l1[m] = w.y;
            }
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                double acc = v[i + h];
#pragma unroll
                for (int m = K - 1; m >= 0; --m) acc = fma(-(h ? l1[m] : l0[m]), st[m], acc);
#pragma unroll
                for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
                st[0] = acc;
                v[i + h] = acc;
            }
        }
    }
    long long t1 = clock64();
#pragma unroll
    for (int i = 0; i < 36; ++i) out[i * blockDim.x + threadIdx.x] = v[i];
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
    double *out; long long *cyc, h[1024];
    cudaMalloc(&out, 1 << 24); cudaMalloc(&cyc, 8 * 1024);
    cudaMemset(out, 0, 1 << 24);
    for (int w : {1, 4, 16}) {
        dfma_chain<<<148, 32 * w>>>(out, cyc, 256); cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("dfma chain, %2d warps/SM: %.2f cycles per dependent DFMA\n", w, h[0] / (256.0 * 16));
        lds_chain<<<148, 32 * w>>>(out, cyc, 256); cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("lds chain,  %2d warps/SM: %.2f cycles per dependent LDS\n", w, h[0] / (256.0 * 16));
    }
    for (int w : {1, 4, 8, 16, 32}) {
        dfma_tput<8><<<148, 32 * w>>>(out, cyc, 256); cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("dfma tput 8 chains, %2d warps/SM: %.1f DFMA lanes/clk/SM (%s)\n", w, 256.0 * 4 * 8 * 32 * w / h[0],
               cudaGetErrorString(cudaGetLastError()));
    }
    for (int w : {1, 2, 4, 8}) {
        band_fwd<1><<<148, 32 * w>>>(out, cyc, 64); cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("band fwd K=1, %2d warps/SM: %.1f cycles per row\n", w, h[0] / (64.0 * 36));
        band_fwd<2><<<148, 32 * w>>>(out, cyc, 64); cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("band fwd K=2, %2d warps/SM: %.1f cycles per row\n", w, h[0] / (64.0 * 36));
        band_fwd<3><<<148, 32 * w>>>(out, cyc, 64); cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        if (cudaGetLastError() != cudaSuccess) printf("launch error\n");
        printf("band fwd K=3, %2d warps/SM: %.1f cycles per row\n", w, h[0] / (64.0 * 36));
    }
    return 0;
}
