// solve_kernels.cu -- fused sm_100a kernels of the batched spline solve.
//
// One launch runs the whole of Algorithm 1 for every
// right-hand side, the B200 counterpart of the paper's fused
// "SerialPttrs_Spmv" kernel (Listing 6):
//   step 2  Q x0' = b0       banded forward/backward recurrences (pttrs /
//                            pbtrs / gbtrs, Listing 1, Table I)
//   step 3  delta' x1 = b1 - lambda x0'   COO spmv + getrs
//   step 4  x0 = x0' - beta x1            COO spmv
//
// B200 design, unlike the paper's one-thread-per-RHS
// walk over HBM (which re-reads every element):
//  * a CTA owns a tile of R right-hand sides; the tile is staged in shared
//    memory by TMA (cp.async.bulk.tensor, mbarrier-tracked) while the previous
//    tile is being solved, so HBM sees exactly one read and one write of each
//    element;
//  * thread (r, s) holds segment s of the Q rows of RHS r in registers; the
//    recurrences run locally with zero inflow and are made exact by the
//    precomputed spike vectors of the segment partition (truncated SPIKE):
//    carries go through shared memory, the fix-up is fused into the next sweep;
//  * factor bands, spikes, corner COO and delta' LU are staged once per CTA
//    in shared memory and read as warp broadcasts;
//  * the corner steps touch only the head/tail windows of Q.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>

#include "device.hpp"

namespace sb {

enum Loader { LOAD_DIRECT = 0, LOAD_TMA = 1 };

struct KParams {
    DevPlan P;
    void *rhs;
    int64_t batch, bstride, pstride;
    int ntiles, nbox, boxr;
    // dynamic shared memory offsets (bytes)
    int off_buf, off_fwd, off_bwd, off_fend, off_bbeg, off_win, off_b1, off_x1, off_betaW, off_lamv, off_lamr,
        off_lams, off_dlu, off_dpiv, off_dscale, off_drow, off_mbar, smem_total;
};

// ------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *m, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *m, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *m, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "SB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra SB_WAIT;\n}\n" ::"r"(smem_u32(m)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, uint64_t *mbar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            smem_u32(dst)),
        "l"(map), "r"(c0), "r"(c1), "r"(smem_u32(mbar))
        : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

template <typename T>
__device__ __forceinline__ void stg_stream(T *p, T v) {
    __stcs(p, v);  // streaming store: written once, not re-read by this kernel
}

// ------------------------------------------------------------------ kernel
template <typename T, int K, int LMAX, int R, int LOADER>
__global__ void __launch_bounds__(512, 1)
    sb_solve_kernel(const __grid_constant__ KParams p, const __grid_constant__ CUtensorMap tmap) {
    using C = T;  // compute in the storage precision (fp64 -> fp64, fp32 -> fp32)
    constexpr int CI = sizeof(C) == 8 ? 0 : 1;
    constexpr int FS = 2 * K;      // forward record: L(i,i-1..i-K), g^(1..K)_i
    constexpr int BS = 2 * K + 2;  // backward record: dinv_i, U'(i,1..K), h^(1..K)_i, pad
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;

    const int tid = threadIdx.x;
    const int r = tid % R;
    const int s = tid / R;
    const int S = P.S, nQ = P.nQ, k = P.k, Wh = P.Wh, Wt = P.Wt, W = P.Wh + P.Wt;
    const int a = s * P.seg_base + min(s, P.seg_rem);
    const int len = P.seg_base + (s < P.seg_rem ? 1 : 0);

    C *sfwd = reinterpret_cast<C *>(smem + p.off_fwd);
    C *sbwd = reinterpret_cast<C *>(smem + p.off_bwd);
    C *sfend = reinterpret_cast<C *>(smem + p.off_fend);
    C *sbbeg = reinterpret_cast<C *>(smem + p.off_bbeg);
    C *swin = reinterpret_cast<C *>(smem + p.off_win);
    C *sb1 = reinterpret_cast<C *>(smem + p.off_b1);
    C *sx1 = reinterpret_cast<C *>(smem + p.off_x1);
    C *sbeta = reinterpret_cast<C *>(smem + p.off_betaW);
    C *slamv = reinterpret_cast<C *>(smem + p.off_lamv);
    int *slamr = reinterpret_cast<int *>(smem + p.off_lamr);
    int *slams = reinterpret_cast<int *>(smem + p.off_lams);
    C *sdlu = reinterpret_cast<C *>(smem + p.off_dlu);
    int *sdpiv = reinterpret_cast<int *>(smem + p.off_dpiv);
    C *sdscale = reinterpret_cast<C *>(smem + p.off_dscale);
    int *sdrow = reinterpret_cast<int *>(smem + p.off_drow);
    uint64_t *mbar = reinterpret_cast<uint64_t *>(smem + p.off_mbar);
    T *buf = reinterpret_cast<T *>(smem + p.off_buf);

    const int nthreads = blockDim.x;
    int tile = blockIdx.x;

    // kick off the first tile before staging the constants (overlap)
    if (LOADER == LOAD_TMA && tid == 0) {
        prefetch_tmap(&tmap);
        mbar_init(mbar, 1);
        fence_mbar_init();
        if (tile < p.ntiles) {
            mbar_arrive_expect_tx(mbar, (uint32_t)(p.nbox * p.boxr * R * sizeof(T)));
            for (int b = 0; b < p.nbox; ++b) tma_load_2d(buf + (size_t)b * p.boxr * R, &tmap, mbar, tile * R, b * p.boxr);
        }
    }
    // stage constants (factor records, corners) once per CTA
    {
        const float4 *src = reinterpret_cast<const float4 *>(P.fwd[CI]);
        float4 *dst = reinterpret_cast<float4 *>(sfwd);
        const int nv = (int)(((size_t)nQ * FS * sizeof(C) + 15) / 16);  // sections padded to 16 B
        for (int i = tid; i < nv; i += nthreads) dst[i] = src[i];
        src = reinterpret_cast<const float4 *>(P.bwd[CI]);
        dst = reinterpret_cast<float4 *>(sbwd);
        const int nb = (int)(((size_t)nQ * BS * sizeof(C) + 15) / 16);
        for (int i = tid; i < nb; i += nthreads) dst[i] = src[i];
        const C *bw = reinterpret_cast<const C *>(P.betaW[CI]);
        for (int i = tid; i < W * k; i += nthreads) sbeta[i] = bw[i];
        const C *lv = reinterpret_cast<const C *>(P.lam_v[CI]);
        for (int i = tid; i < P.nlam; i += nthreads) {
            slamv[i] = lv[i];
            slamr[i] = P.lam_r[i];
            slams[i] = P.lam_slot[i];
        }
        const C *dl = reinterpret_cast<const C *>(P.dlu[CI]);
        for (int i = tid; i < k * k; i += nthreads) sdlu[i] = dl[i];
        const C *ds = reinterpret_cast<const C *>(P.dscale[CI]);
        for (int i = tid; i < k; i += nthreads) {
            sdpiv[i] = P.dpiv[i];
            sdscale[i] = ds[i];
            sdrow[i] = P.drow[i];
        }
    }
    __syncthreads();

    T *gout = reinterpret_cast<T *>(p.rhs);
    uint32_t phase = 0;
    for (; tile < p.ntiles; tile += gridDim.x) {
        const int64_t col = (int64_t)tile * R + r;
        const bool live = col < p.batch;
        T *gcol = gout + col * p.bstride;
        C v[LMAX];
        // ---------------------------------------------------------- load
        if (LOADER == LOAD_TMA) {
            mbar_wait(mbar, phase);
            phase ^= 1u;
            const T *brow = buf + (size_t)(P.s_lo + a) * R + r;
#pragma unroll
            for (int i = 0; i < LMAX; ++i)
                if (i < len) v[i] = (C)brow[(size_t)i * R];
            if (s == 0)
                for (int d = 0; d < k; ++d) sb1[r * k + d] = (C)buf[(size_t)sdrow[d] * R + r] * sdscale[d];
            __syncthreads();  // B1: tile buffer consumed -> refill it with the next tile
            if (tid == 0 && tile + (int)gridDim.x < p.ntiles) {
                const int nt = tile + gridDim.x;
                mbar_arrive_expect_tx(mbar, (uint32_t)(p.nbox * p.boxr * R * sizeof(T)));
                for (int b = 0; b < p.nbox; ++b)
                    tma_load_2d(buf + (size_t)b * p.boxr * R, &tmap, mbar, nt * R, b * p.boxr);
            }
        } else {
            const T *gsrc = gcol + (int64_t)(P.s_lo + a) * p.pstride;
#pragma unroll
            for (int i = 0; i < LMAX; ++i)
                if (i < len) v[i] = live ? (C)__ldcs(gsrc + (int64_t)i * p.pstride) : C(0);
            if (s == 0)
                for (int d = 0; d < k; ++d)
                    sb1[r * k + d] = live ? (C)gcol[(int64_t)sdrow[d] * p.pstride] * sdscale[d] : C(0);
        }
        // ------------------------------- step 2a: local forward sweep (L y = b)
        C st[K];
#pragma unroll
        for (int m = 0; m < K; ++m) st[m] = C(0);
        {
            const C *f = sfwd + (size_t)a * FS;
#pragma unroll
            for (int i = 0; i < LMAX; ++i) {
                if (i < len) {
                    C acc = v[i];
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(-f[i * FS + m], st[m], acc);
#pragma unroll
                    for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
                    st[0] = acc;
                    v[i] = acc;
                }
            }
        }
#pragma unroll
        for (int j = 0; j < K; ++j) sfend[(s * R + r) * K + j] = st[j];
        __syncthreads();  // B2
        // forward carry: true y at rows a-1..a-K (walk over predecessor segments)
        C cin[K];
#pragma unroll
        for (int m = 0; m < K; ++m) cin[m] = C(0);
        if (s > 0) {
            const int t0 = max(0, s - P.carry_f);
            for (int t = t0; t < s; ++t) {
                const int end = t * P.seg_base + min(t, P.seg_rem) + P.seg_base + (t < P.seg_rem ? 1 : 0);
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = sfend[(t * R + r) * K + j];
                    const C *g = sfwd + (size_t)(end - 1 - j) * FS + K;
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(g[m], cin[m], acc);
                    nw[j] = acc;
                }
#pragma unroll
                for (int j = 0; j < K; ++j) cin[j] = nw[j];
            }
        }
        // ---------- step 2b: forward fix-up fused into the local backward sweep
        C st2[K];
#pragma unroll
        for (int m = 0; m < K; ++m) st2[m] = C(0);
        {
            const C *f = sfwd + (size_t)a * FS;
            const C *b = sbwd + (size_t)a * BS;
            const bool fix = s > 0;
#pragma unroll
            for (int i = LMAX - 1; i >= 0; --i) {
                if (i < len) {
                    C y = v[i];
                    if (fix) {
#pragma unroll
                        for (int m = 0; m < K; ++m) y = fma(f[i * FS + K + m], cin[m], y);
                    }
                    C acc = y * b[i * BS];
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(-b[i * BS + 1 + m], st2[m], acc);
#pragma unroll
                    for (int m = K - 1; m > 0; --m) st2[m] = st2[m - 1];
                    st2[0] = acc;
                    v[i] = acc;
                }
            }
        }
#pragma unroll
        for (int j = 0; j < K; ++j) sbbeg[(s * R + r) * K + j] = st2[j];
        __syncthreads();  // B3
        C cout[K];
#pragma unroll
        for (int m = 0; m < K; ++m) cout[m] = C(0);
        if (s < S - 1) {
            const int t0 = min(S - 1, s + P.carry_b);
            for (int t = t0; t > s; --t) {
                const int at = t * P.seg_base + min(t, P.seg_rem);
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = sbbeg[(t * R + r) * K + j];
                    const C *h = sbwd + (size_t)(at + j) * BS + 1 + K;
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(h[m], cout[m], acc);
                    nw[j] = acc;
                }
#pragma unroll
                for (int j = 0; j < K; ++j) cout[j] = nw[j];
            }
        }
        // backward fix-up -> x0'; window rows go to smem, the rest straight to HBM
        const bool inwin = (a < Wh) || (a + len > nQ - Wt);
        {
            const C *b = sbwd + (size_t)a * BS;
            const bool fix = s < S - 1;
            T *grow = gcol + (int64_t)(P.s_lo + a) * p.pstride;
#pragma unroll
            for (int i = 0; i < LMAX; ++i) {
                if (i < len) {
                    if (fix) {
#pragma unroll
                        for (int m = 0; m < K; ++m) v[i] = fma(b[i * BS + 1 + K + m], cout[m], v[i]);
                    }
                    const int q = a + i;
                    const int slot = q < Wh ? q : (q >= nQ - Wt ? Wh + q - (nQ - Wt) : -1);
                    if (slot >= 0) swin[r * W + slot] = v[i];
                    else if (live) stg_stream(grow + (int64_t)i * p.pstride, (T)v[i]);
                }
            }
        }
        __syncthreads();  // B4
        // ------------- step 3: x1 = delta'^{-1} (b1 - lambda x0')  (one thread per RHS)
        if (s == 0 && k > 0) {
            C *x1 = sx1 + r * k;
            for (int d = 0; d < k; ++d) x1[d] = sb1[r * k + d];
            for (int e = 0; e < P.nlam; ++e) x1[slamr[e]] = fma(-slamv[e], swin[r * W + slams[e]], x1[slamr[e]]);
            for (int d = 0; d < k; ++d) {
                const int pv = sdpiv[d];
                if (pv != d) { C t = x1[d]; x1[d] = x1[pv]; x1[pv] = t; }
            }
            for (int i = 1; i < k; ++i)
                for (int j = 0; j < i; ++j) x1[i] = fma(-sdlu[i * k + j], x1[j], x1[i]);
            for (int i = k - 1; i >= 0; --i) {
                C acc = x1[i];
                for (int j = i + 1; j < k; ++j) acc = fma(-sdlu[i * k + j], x1[j], acc);
                x1[i] = acc / sdlu[i * k + i];
            }
            if (live)
                for (int d = 0; d < k; ++d) stg_stream(gcol + (int64_t)sdrow[d] * p.pstride, (T)x1[d]);
        }
        __syncthreads();  // B5
        // ------------------------------------ step 4: x0 = x0' - beta x1 (windows)
        if (inwin) {
            const C *x1 = sx1 + r * k;
            T *grow = gcol + (int64_t)(P.s_lo + a) * p.pstride;
#pragma unroll
            for (int i = 0; i < LMAX; ++i) {
                if (i < len) {
                    const int q = a + i;
                    const int slot = q < Wh ? q : (q >= nQ - Wt ? Wh + q - (nQ - Wt) : -1);
                    if (slot >= 0) {
                        C acc = v[i];
                        for (int c = 0; c < k; ++c) acc = fma(-sbeta[slot * k + c], x1[c], acc);
                        if (live) stg_stream(grow + (int64_t)i * p.pstride, (T)acc);
                    }
                }
            }
        }
    }
}

// ------------------------------------------------------------------ host
namespace {

constexpr int LMAX = 32;
constexpr int MAX_THREADS = 512;

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void *ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
    }
    return fn;
}

template <typename T, int K, int R, int LOADER>
int launch_t(const KParams &kp, const CUtensorMap &tm, int grid, int threads, cudaStream_t st, char *err, int errlen) {
    auto fn = sb_solve_kernel<T, K, LMAX, R, LOADER>;
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kp.smem_total);
    if (e != cudaSuccess) {
        snprintf(err, errlen, "cudaFuncSetAttribute: %s", cudaGetErrorString(e));
        return 3;
    }
    fn<<<grid, threads, kp.smem_total, st>>>(kp, tm);
    e = cudaGetLastError();
    if (e != cudaSuccess) {
        snprintf(err, errlen, "kernel launch: %s", cudaGetErrorString(e));
        return 3;
    }
    return 0;
}

template <typename T, int R, int LOADER>
int dispatch_K(int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads, cudaStream_t st, char *err,
               int errlen) {
    switch (K) {
        case 1: return launch_t<T, 1, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 2: return launch_t<T, 2, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 3: return launch_t<T, 3, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 4: return launch_t<T, 4, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
    }
    snprintf(err, errlen, "unsupported band K=%d", K);
    return 5;
}

template <typename T>
int dispatch(int R, int loader, int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads,
             cudaStream_t st, char *err, int errlen) {
    if (R == 16 && loader == LOAD_TMA) return dispatch_K<T, 16, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen);
    if (R == 8 && loader == LOAD_TMA) return dispatch_K<T, 8, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen);
    if (R == 16) return dispatch_K<T, 16, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
    if (R == 8) return dispatch_K<T, 8, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
    snprintf(err, errlen, "unsupported tile width R=%d", R);
    return 5;
}

// lay out dynamic smem; returns total bytes
int layout_smem(KParams &kp, const DevPlan &P, int R, size_t esz, bool with_buf, int nbox, int boxr) {
    size_t o = 0;
    auto take = [&](size_t bytes, size_t al) {
        o = align_up(o, al);
        size_t r = o;
        o += bytes;
        return (int)r;
    };
    kp.off_buf = with_buf ? take((size_t)nbox * boxr * R * esz, 1024) : 0;
    kp.off_fwd = take((size_t)P.nQ * P.fstride * esz, 16);
    kp.off_bwd = take((size_t)P.nQ * P.bstride * esz, 16);
    kp.off_fend = take((size_t)P.S * R * P.K * esz, 16);
    kp.off_bbeg = take((size_t)P.S * R * P.K * esz, 16);
    kp.off_win = take((size_t)R * (P.Wh + P.Wt) * esz, 16);
    kp.off_b1 = take((size_t)R * P.k * esz, 16);
    kp.off_x1 = take((size_t)R * P.k * esz, 16);
    kp.off_betaW = take((size_t)(P.Wh + P.Wt) * P.k * esz, 16);
    kp.off_lamv = take((size_t)P.nlam * esz, 16);
    kp.off_lamr = take((size_t)P.nlam * 4, 16);
    kp.off_lams = take((size_t)P.nlam * 4, 16);
    kp.off_dlu = take((size_t)P.k * P.k * esz, 16);
    kp.off_dpiv = take((size_t)P.k * 4, 16);
    kp.off_dscale = take((size_t)P.k * esz, 16);
    kp.off_drow = take((size_t)P.k * 4, 16);
    kp.off_mbar = take(8, 8);
    kp.smem_total = (int)align_up(o, 16);
    return kp.smem_total;
}

}  // namespace

size_t const_smem_bytes(const DevPlan &P, int dtype) {
    KParams kp{};
    return (size_t)layout_smem(kp, P, 16, dtype == 0 ? 8 : 4, false, 0, 0);
}

int launch_solve(const DevPlan &P, const SolveArgs &a, int num_sms, char *err, int errlen) {
    if (a.batch == 0) return 0;
    const size_t esz = a.dtype == 0 ? 8 : 4;
    int dev = 0;
    cudaGetDevice(&dev);
    int max_smem = 0;
    cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);

    KParams kp{};
    kp.P = P;
    kp.rhs = a.rhs;
    kp.batch = a.batch;
    kp.bstride = a.bstride;
    kp.pstride = a.pstride;

    // tile width R and loader: TMA for the batch-contiguous layout when the
    // tensor-map constraints hold and the tile fits in shared memory
    const bool contig = a.bstride == 1;
    const bool aligned = ((uintptr_t)a.rhs % 16 == 0) && ((a.pstride * (int64_t)esz) % 16 == 0);
    const int nbox = (P.n + 255) / 256;
    const int boxr = ((P.n + nbox - 1) / nbox + 7) / 8 * 8;
    int R = 0, loader = LOAD_DIRECT;
    CUtensorMap tm;
    memset(&tm, 0, sizeof(tm));
    for (int cand : {16, 8}) {
        if (cand * P.S > MAX_THREADS) continue;
        if (contig && aligned && a.batch >= cand && get_encode()) {
            KParams t = kp;
            if (layout_smem(t, P, cand, esz, true, nbox, boxr) <= max_smem) { R = cand; loader = LOAD_TMA; break; }
        }
        KParams t = kp;
        if (layout_smem(t, P, cand, esz, false, 0, 0) <= max_smem) { R = cand; loader = LOAD_DIRECT; break; }
    }
    if (!R) {
        snprintf(err, errlen, "problem too large for the shared-memory kernel (n=%d, S=%d)", P.n, P.S);
        return 5;
    }
    layout_smem(kp, P, R, esz, loader == LOAD_TMA, nbox, boxr);
    kp.ntiles = (int)((a.batch + R - 1) / R);
    kp.nbox = nbox;
    kp.boxr = boxr;
    if (loader == LOAD_TMA) {
        cuuint64_t dims[2] = {(cuuint64_t)a.batch, (cuuint64_t)P.n};
        cuuint64_t strides[1] = {(cuuint64_t)(a.pstride * (int64_t)esz)};
        cuuint32_t box[2] = {(cuuint32_t)R, (cuuint32_t)boxr};
        cuuint32_t estr[2] = {1, 1};
        CUresult cr = get_encode()(&tm, a.dtype == 0 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                                   2, a.rhs, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (cr != CUDA_SUCCESS) {
            snprintf(err, errlen, "cuTensorMapEncodeTiled failed (%d)", (int)cr);
            return 3;
        }
    }
    const int threads = R * P.S;
    const int grid = (int)std::min<int64_t>((int64_t)kp.ntiles, (int64_t)num_sms);
    if (a.dtype == 0) return dispatch<double>(R, loader, P.K, kp, tm, grid, threads, a.stream, err, errlen);
    return dispatch<float>(R, loader, P.K, kp, tm, grid, threads, a.stream, err, errlen);
}

}  // namespace sb
