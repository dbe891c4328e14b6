// stream_probe2.cu -- diagnostic (NOT product code): variants of the tile
// access pattern of the batch-contiguous layout, (n=1000 rows) x (1e5 RHS)
// fp64, in place.  What limits the TMA-tile skeleton at ~5.4 TB/s?
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d: %s\n", #x, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)
__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

// MODE bit0: do loads, bit1: do stores; STORE: 0 st.cs, 1 st.wb (default), 2 st with L2::evict_first policy
template <int R, int L, int MODE, int STORE, int HALVES = 1>
__global__ void __launch_bounds__(512, 1) tma_kernel(const __grid_constant__ CUtensorMap tm, double *x, int n, int64_t B,
                                                   int ntiles, int nbox, int boxr) {
    extern __shared__ __align__(1024) unsigned char smem[];
    double *buf = (double *)smem;
    uint64_t *mbar = (uint64_t *)(smem + (size_t)nbox * boxr * R * 8);
    const int tid = threadIdx.x, r = tid % R, s = tid / R;
    const uint32_t bytes = (uint32_t)(nbox * boxr * R * 8);
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(mbar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const int half = blockIdx.x % HALVES;
    const int rows0 = half * nbox * boxr;  // this CTA's first row
    auto issue = [&](int t) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(mbar)), "r"(bytes) : "memory");
        for (int q = 0; q < nbox; ++q)
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                         ::"r"(su32(buf + (size_t)q * boxr * R)), "l"(&tm), "r"(t * R), "r"(rows0 + q * boxr), "r"(su32(mbar)) : "memory");
    };
    int it = 0;
    const int g0 = blockIdx.x / HALVES, gstep = gridDim.x / HALVES;
    if ((MODE & 1) && tid == 0 && g0 < ntiles) issue(g0);
    for (int t = g0; t < ntiles; t += gstep, ++it) {
        double v[L];
        const int a = s * L;
        if (MODE & 1) {
            asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W;\n}\n" ::"r"(su32(mbar)), "r"(it & 1) : "memory");
#pragma unroll
            for (int i = 0; i < L; ++i) v[i] = (a + i < n) ? buf[(size_t)(a + i) * R + r] : 0.0;
            __syncthreads();
            if (tid == 0 && t + gstep < ntiles) issue(t + gstep);
        } else {
#pragma unroll
            for (int i = 0; i < L; ++i) v[i] = (double)(t + i);
        }
        const int64_t col = (int64_t)t * R + r;
        if ((MODE & 2) && STORE == 3) {
            // results -> own smem tile (second buffer after the load buffer), TMA store
            double *obuf = buf + (size_t)nbox * boxr * R + 16;  // past the mbarrier
            if (it > 0 && tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            __syncthreads();
#pragma unroll
            for (int i = 0; i < L; ++i)
                if (a + i < nbox * boxr) obuf[(size_t)(a + i) * R + r] = v[i] * 1.0000001;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncthreads();
            if (tid == 0) {
                for (int q = 0; q < nbox; ++q)
                    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                                 ::"l"(&tm), "r"(t * R), "r"(rows0 + q * boxr), "r"(su32(obuf + (size_t)q * boxr * R)) : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
        } else if (MODE & 2) {
#pragma unroll
            for (int i = 0; i < L; ++i)
                if (rows0 + a + i < n && a + i < nbox * boxr && col < B) {
                    double *p = x + (int64_t)(rows0 + a + i) * B + col;
                    double w = v[i] * 1.0000001;
                    if (STORE == 0) __stcs(p, w);
                    else if (STORE == 1) *p = w;
                    else asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(p), "d"(w), "l"(pol) : "memory");
                }
        } else {
            double acc = 0;
#pragma unroll
            for (int i = 0; i < L; ++i) acc += v[i];
            if (acc == 12345.678) x[0] = acc;
        }
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

template <int MODE, int STORE, int R = 16, int HALVES = 1>
static void run(double *x, int n, int64_t B, int sms, int boxr_req, CUtensorMapL2promotion prom, const char *tag) {
    constexpr int L = 32;
    const int nh = n / HALVES;  // rows per CTA
    int nbox = (nh + boxr_req - 1) / boxr_req, boxr = ((nh + nbox - 1) / nbox + 7) / 8 * 8;
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)B, (cuuint64_t)n};
    cuuint64_t str[1] = {(cuuint64_t)(B * 8)};
    cuuint32_t box[2] = {R, (cuuint32_t)boxr}, es[2] = {1, 1};
    CUresult cr = enc()(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, prom, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr) { printf("encode failed %d\n", cr); return; }
    size_t smem = (size_t)nbox * boxr * R * 8 * (STORE == 3 ? 2 : 1) + 256;
    auto k = tma_kernel<R, L, MODE, STORE, HALVES>;
    CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int ntiles = (int)((B + R - 1) / R);
    int threads = R * ((nbox * boxr + L - 1) / L);
    if (threads > 512) { printf("%s: too many threads %d\n", tag, threads); return; }
    double ms = timeit([&] { k<<<(sms / HALVES) * HALVES, threads, smem>>>(tm, x, n, B, ntiles, nbox, boxr); });
    double bytes = (double)n * B * 8 * (((MODE & 1) ? 1 : 0) + ((MODE & 2) ? 1 : 0));
    printf("%-34s boxr=%3d mode=%d store=%d : %.3f ms  %.0f GB/s\n", tag, boxr, MODE, STORE, ms, bytes / ms / 1e6);
}

int main(int argc, char **argv) {
    // argv[1]: batch B (row pitch = B doubles): 1e5 (C2, 800 KB) ... 8e6 (C5 on one GPU, 64 MB);
    // argv[2] = "all": every variant, else the pitch study subset
    const int n = 1000;
    const int64_t B = argc > 1 ? (int64_t)atof(argv[1]) : 100000;
    const bool all = argc > 2;
    int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    double *x; CK(cudaMalloc(&x, (size_t)n * B * 8));
    CK(cudaMemset(x, 0, (size_t)n * B * 8));
    printf("B = %lld (row pitch %.1f MB)\n", (long long)B, B * 8.0 / 1e6);
    auto P256 = CU_TENSOR_MAP_L2_PROMOTION_L2_256B, P128 = CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
         P0 = CU_TENSOR_MAP_L2_PROMOTION_NONE;
    run<3, 0>(x, n, B, sms, 256, P256, "rw st.cs prom256");
    run<3, 0, 32, 2>(x, n, B, sms, 256, P256, "R32 halves rw");
    run<1, 0>(x, n, B, sms, 256, P256, "read only");
    run<1, 0, 32, 2>(x, n, B, sms, 256, P256, "R32 halves read only");
    run<2, 0>(x, n, B, sms, 256, P256, "write only st.cs");
    run<3, 3, 16, 2>(x, n, B, sms, 256, P256, "rw TMA store (R16 halves)");
    if (all) {
        run<2, 3, 16, 2>(x, n, B, sms, 256, P256, "write only TMA store (R16 halves)");
        run<2, 3, 32, 4>(x, n, B, sms, 256, P256, "write only TMA store (R32 quarters)");
        run<3, 0, 32, 2>(x, n, B, sms, 128, P256, "R32 halves rw box128");
        run<3, 0, 16, 2>(x, n, B, sms, 256, P256, "R16 halves rw (2 CTA/tile)");
        run<3, 1>(x, n, B, sms, 256, P256, "rw st.wb prom256");
        run<3, 2>(x, n, B, sms, 256, P256, "rw st.evict_first prom256");
        run<3, 0>(x, n, B, sms, 256, P128, "rw st.cs prom128");
        run<3, 0>(x, n, B, sms, 256, P0, "rw st.cs prom none");
        run<3, 0>(x, n, B, sms, 128, P256, "rw st.cs box128");
        run<3, 0>(x, n, B, sms, 64, P256, "rw st.cs box64");
        run<2, 1>(x, n, B, sms, 256, P256, "write only st.wb");
    }
    CK(cudaFree(x));
    return 0;
}
