// stream_probe.cu -- diagnostic microbenchmarks (NOT product code): how fast
// can the (n rows x B RHS) batch-contiguous fp64 array be read and written in
// place with the access patterns the solver kernel can use?
//   flat   : grid-stride double2 read+write (copy-like ceiling)
//   tma    : per-CTA TMA 2D tiles [n x R] into NBUF smem buffers, threads pull
//            their column segment from smem and STG it back
//   direct : per-thread LDG of its column segment into registers, STG back
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o stream_probe stream_probe.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d: %s\n", #x, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void flat_kernel(double2 *x, size_t n2) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n2; i += (size_t)gridDim.x * blockDim.x) {
        double2 v = x[i];
        v.x *= 1.0000001; v.y *= 1.0000001;
        x[i] = v;
    }
}

template <int R, int NBUF, int L>
__global__ void __launch_bounds__(1024, 1) tma_kernel(const __grid_constant__ CUtensorMap tm, double *x, int n, int64_t B,
                                                    int ntiles, int nbox, int boxr) {
    extern __shared__ __align__(1024) unsigned char smem[];
    double *buf = (double *)smem;
    uint64_t *mbar = (uint64_t *)(smem + (size_t)NBUF * nbox * boxr * R * 8);
    const int tid = threadIdx.x, r = tid % R, s = tid / R;
    const size_t bufel = (size_t)nbox * boxr * R;
    const uint32_t bytes = (uint32_t)(bufel * 8);
    if (tid == 0) {
        for (int b = 0; b < NBUF; ++b) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(mbar + b)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](int t, int b) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(mbar + b)), "r"(bytes) : "memory");
        for (int q = 0; q < nbox; ++q)
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                         ::"r"(su32(buf + b * bufel + (size_t)q * boxr * R)), "l"(&tm), "r"(t * R), "r"(q * boxr), "r"(su32(mbar + b)) : "memory");
    };
    int it = 0;
    if (tid == 0)
        for (int b = 0; b < NBUF; ++b) if (blockIdx.x + b * gridDim.x < ntiles) issue(blockIdx.x + b * gridDim.x, b);
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
        const int b = it % NBUF;
        const uint32_t par = (it / NBUF) & 1;
        asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W;\n}\n" ::"r"(su32(mbar + b)), "r"(par) : "memory");
        double v[L];
        const int a = s * L;
#pragma unroll
        for (int i = 0; i < L; ++i) v[i] = (a + i < n) ? buf[b * bufel + (size_t)(a + i) * R + r] : 0.0;
        __syncthreads();
        if (tid == 0) { int nt = t + NBUF * gridDim.x; if (nt < ntiles) issue(nt, b); }
        const int64_t col = (int64_t)t * R + r;
#pragma unroll
        for (int i = 0; i < L; ++i)
            if (a + i < n && col < B) __stcs(x + (int64_t)(a + i) * B + col, v[i] * 1.0000001);
    }
}

template <int R, int L>
__global__ void __launch_bounds__(512) direct_kernel(double *x, int n, int64_t B, int ntiles) {
    const int tid = threadIdx.x, r = tid % R, s = tid / R;
    const int a = s * L;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int64_t col = (int64_t)t * R + r;
        double v[L];
        const double *src = x + (int64_t)a * B + col;
#pragma unroll
        for (int i = 0; i < L; ++i) v[i] = (a + i < n) ? __ldcs(src + (int64_t)i * B) : 0.0;
#pragma unroll
        for (int i = 0; i < L; ++i)
            if (a + i < n) __stcs(x + (int64_t)(a + i) * B + col, v[i] * 1.0000001);
    }
}

static PFN_cuTensorMapEncodeTiled_v12000 enc() {
    void *p = nullptr; cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    return (PFN_cuTensorMapEncodeTiled_v12000)p;
}

template <typename F>
static double timeit(F f, int reps = 20) {
    cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
    for (int i = 0; i < 3; ++i) f();
    CK(cudaEventRecord(a));
    for (int i = 0; i < reps; ++i) f();
    CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    CK(cudaGetLastError());
    return ms / reps;
}

template <int R, int NBUF, int THREADS>
static void run_tma(double *x, int n, int64_t B, int sms, int g = 1) {
    constexpr int S = THREADS / R;
    constexpr int L = 32;
    (void)S;
    int nbox = (n + 255) / 256, boxr = ((n + nbox - 1) / nbox + 7) / 8 * 8;
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)B, (cuuint64_t)n};
    cuuint64_t str[1] = {(cuuint64_t)(B * 8)};
    cuuint32_t box[2] = {R, (cuuint32_t)boxr}, es[2] = {1, 1};
    CUresult cr = enc()(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr) { printf("encode failed %d\n", cr); return; }
    size_t smem = (size_t)NBUF * nbox * boxr * R * 8 + 64;
    auto k = tma_kernel<R, NBUF, L>;
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) { printf("tma R=%d NBUF=%d: smem %zu too big\n", R, NBUF, smem); cudaGetLastError(); return; }
    int ntiles = (int)((B + R - 1) / R);
    int threads = R * ((n + L - 1) / L);
    double ms = timeit([&] { k<<<sms * g, threads, smem>>>(tm, x, n, B, ntiles, nbox, boxr); });
    printf("tma    R=%2d NBUF=%d threads=%4d smem=%6zu ctas/sm=%d : %.3f ms  %.0f GB/s\n", R, NBUF, threads, smem, g, ms, 2.0 * n * B * 8 / ms / 1e6);
}

template <int R, int L>
static void run_direct(double *x, int n, int64_t B, int sms, int ctas_per_sm) {
    int ntiles = (int)((B + R - 1) / R);
    int threads = R * ((n + L - 1) / L);
    double ms = timeit([&] { direct_kernel<R, L><<<sms * ctas_per_sm, threads>>>(x, n, B, ntiles); });
    printf("direct R=%2d L=%d threads=%4d ctas/sm=%d : %.3f ms  %.0f GB/s\n", R, L, threads, ctas_per_sm, ms, 2.0 * n * B * 8 / ms / 1e6);
}

int main() {
    const int n = 1000; const int64_t B = 100000;
    int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    double *x; CK(cudaMalloc(&x, (size_t)n * B * 8));
    CK(cudaMemset(x, 0, (size_t)n * B * 8));
    for (int g : {1, 2, 4, 8}) {
        double ms = timeit([&] { flat_kernel<<<sms * g, 1024>>>((double2 *)x, (size_t)n * B / 2); });
        printf("flat   grid=%d x 1024 : %.3f ms  %.0f GB/s\n", sms * g, ms, 2.0 * n * B * 8 / ms / 1e6);
    }
    run_tma<16, 1, 512>(x, n, B, sms);
    run_tma<8, 1, 256>(x, n, B, sms);
    run_tma<8, 2, 256>(x, n, B, sms);
    run_tma<8, 3, 256>(x, n, B, sms);
    run_tma<4, 4, 128>(x, n, B, sms);
    run_tma<4, 6, 128>(x, n, B, sms);
    run_tma<8, 1, 256>(x, n, B, sms, 2);
    run_tma<8, 1, 256>(x, n, B, sms, 3);
    run_tma<4, 1, 128>(x, n, B, sms, 4);
    run_tma<4, 2, 128>(x, n, B, sms, 3);
    run_direct<16, 32>(x, n, B, sms, 1);
    run_direct<16, 32>(x, n, B, sms, 2);
    run_direct<8, 32>(x, n, B, sms, 2);
    run_direct<8, 32>(x, n, B, sms, 4);
    run_direct<16, 16>(x, n, B, sms, 2);
    CK(cudaFree(x));
    return 0;
}
