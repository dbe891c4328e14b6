// solve_kernels.cu -- fused sm_100a kernel of the batched spline solve.
//
// One launch runs the whole Schur-complement chain (Eq. 3-6,
// Algorithm 1) for every right-hand side -- the B200 counterpart of
// the paper's fused "SerialPttrs_Spmv" kernel (Listing 6).  The
// block LU is applied in its transposed form A = [[I,0],[Lambda,I]] [[Q,gamma],[0,delta']]
// with Lambda = lambda Q^{-1} (R6), which gives the same x:
//   corner  x1 = delta'^{-1} (b1 - Lambda b0)   COO/CSR spmv + getrs
//   gamma   b0 <- b0 - gamma x1                  COO spmv (transposed)
//   Q       x0 = Q^{-1} b0                        banded LDL^T / LU recurrences
//                                                 (pttrs / pbtrs / gbtrs, Listing 1, Table I)
// so the corner work reads only input rows of the tile already in shared
// memory and the Q solution goes straight from registers to HBM.
//
// B200 mapping:
//  * persistent CTA (one per SM) owns a tile of R right-hand sides x all n
//    rows; the next tile is fetched by TMA (cp.async.bulk.tensor 2-D,
//    mbarrier complete_tx) while the current one is solved -> each element is
//    read once and written once (16 B / element in fp64);
//  * thread (r, s) keeps rows [s*L, s*L+L) of RHS r in registers; the
//    recurrences run locally with zero inflow, then the exact inflow /
//    outflow ("carries") is obtained from the neighbours' end states through
//    shared memory and the precomputed segment transfer matrices, and added
//    back by a correction chain (SPIKE-style) -- exact, no overlap, no re-read;
//  * Q is padded with identity rows to S*L so the sweeps carry no predicates;
//  * factors, transfer matrices and corner data are staged once per CTA in
//    shared memory and read as broadcasts.
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
    int off_buf, off_L, off_U, off_dinv, off_G, off_H, off_fend, off_bbeg, off_x1, off_lamptr, off_lamc, off_lamv,
        off_gamr, off_gamc, off_gamv, off_gptr, off_dlu, off_dpiv, off_dscale, off_drow, off_mbar, smem_total;
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
__device__ __forceinline__ void copy_words(T *dst, const T *src, int count, int tid, int nthreads) {
    for (int i = tid; i < count; i += nthreads) dst[i] = src[i];
}

// ------------------------------------------------------------------ kernel
template <typename T, int K, int L, int R, int LOADER>
__global__ void __launch_bounds__(512, 1)
    sb_solve_kernel(const __grid_constant__ KParams p, const __grid_constant__ CUtensorMap tmap) {
    using C = T;  // compute in the storage precision
    constexpr int CI = sizeof(T) == 8 ? 0 : 1;
    constexpr int CP = 32 / R;  // corner lanes per RHS in warp 0
    static_assert(L % 2 == 0, "segment length must be even");
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;
    const DevSeg &G = P.seg[CI];

    const int tid = threadIdx.x;
    const int nthreads = blockDim.x;
    const int r = tid % R;
    const int s = tid / R;
    const int S = G.S, nQ = P.nQ, k = P.k, nQpa = P.nQpa;
    const int a = s * L;
    const bool full = a + L <= nQ;  // segment has no padding rows

    C *sL = reinterpret_cast<C *>(smem + p.off_L);
    C *sU = reinterpret_cast<C *>(smem + p.off_U);
    C *sdinv = reinterpret_cast<C *>(smem + p.off_dinv);
    C *sG = reinterpret_cast<C *>(smem + p.off_G);
    C *sH = reinterpret_cast<C *>(smem + p.off_H);
    C *sfend = reinterpret_cast<C *>(smem + p.off_fend);
    C *sbbeg = reinterpret_cast<C *>(smem + p.off_bbeg);
    C *sx1 = reinterpret_cast<C *>(smem + p.off_x1);
    int *slamptr = reinterpret_cast<int *>(smem + p.off_lamptr);
    int *slamc = reinterpret_cast<int *>(smem + p.off_lamc);
    C *slamv = reinterpret_cast<C *>(smem + p.off_lamv);
    int *sgamr = reinterpret_cast<int *>(smem + p.off_gamr);
    int *sgamc = reinterpret_cast<int *>(smem + p.off_gamc);
    C *sgamv = reinterpret_cast<C *>(smem + p.off_gamv);
    int *sgptr = reinterpret_cast<int *>(smem + p.off_gptr);
    C *sdlu = reinterpret_cast<C *>(smem + p.off_dlu);
    int *sdpiv = reinterpret_cast<int *>(smem + p.off_dpiv);
    C *sdscale = reinterpret_cast<C *>(smem + p.off_dscale);
    int *sdrow = reinterpret_cast<int *>(smem + p.off_drow);
    uint64_t *mbar = reinterpret_cast<uint64_t *>(smem + p.off_mbar);
    T *buf = reinterpret_cast<T *>(smem + p.off_buf);

    int tile = blockIdx.x;
    const uint32_t tile_bytes = (uint32_t)(p.nbox * p.boxr * R * sizeof(T));

    // first tile in flight while the constants are staged
    if (LOADER == LOAD_TMA && tid == 0) {
        prefetch_tmap(&tmap);
        mbar_init(mbar, 1);
        fence_mbar_init();
        if (tile < p.ntiles) {
            mbar_arrive_expect_tx(mbar, tile_bytes);
            for (int b = 0; b < p.nbox; ++b) tma_load_2d(buf + (size_t)b * p.boxr * R, &tmap, mbar, tile * R, b * p.boxr);
        }
    }
    {
        const int nrec = K * nQpa;
        copy_words(sL, reinterpret_cast<const C *>(P.Lr[CI]), nrec, tid, nthreads);
        copy_words(sU, reinterpret_cast<const C *>(P.Ur[CI]), nrec, tid, nthreads);
        copy_words(sdinv, reinterpret_cast<const C *>(P.dinv[CI]), nQpa, tid, nthreads);
        copy_words(sG, reinterpret_cast<const C *>(G.G), S * K * K, tid, nthreads);
        copy_words(sH, reinterpret_cast<const C *>(G.H), S * K * K, tid, nthreads);
        copy_words(slamptr, P.lam_ptr, k + 1, tid, nthreads);
        copy_words(slamc, P.lam_c, P.lam_nnz, tid, nthreads);
        copy_words(slamv, reinterpret_cast<const C *>(P.lam_v[CI]), P.lam_nnz, tid, nthreads);
        copy_words(sgamr, P.gam_r, P.gam_nnz, tid, nthreads);
        copy_words(sgamc, P.gam_c, P.gam_nnz, tid, nthreads);
        copy_words(sgamv, reinterpret_cast<const C *>(P.gam_v[CI]), P.gam_nnz, tid, nthreads);
        copy_words(sgptr, G.gptr, S + 1, tid, nthreads);
        copy_words(sdlu, reinterpret_cast<const C *>(P.dlu[CI]), k * k, tid, nthreads);
        copy_words(sdpiv, P.dpiv, k, tid, nthreads);
        copy_words(sdscale, reinterpret_cast<const C *>(P.dscale[CI]), k, tid, nthreads);
        copy_words(sdrow, P.drow, k, tid, nthreads);
    }
    __syncthreads();

    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    uint32_t phase = 0;
    for (; tile < p.ntiles; tile += gridDim.x) {
        const int64_t col = (int64_t)tile * R + r;
        const bool live = col < p.batch;
        T *gcol = gout + col * p.bstride;
        if (LOADER == LOAD_TMA) {
            mbar_wait(mbar, phase);
            phase ^= 1u;
        }
        // ---------- corner: x1 = delta'^{-1} (s1*b1 - Lambda b0), warp 0 (CP lanes per RHS)
        if (tid < 32 && k > 0) {
            // CTAs with a single segment have only R (< 32) threads: one part
            const int cp = min(CP, nthreads / R);
            const int part = tid / R, rr = tid % R;
            const int64_t ccol = (int64_t)tile * R + rr;
            const bool clive = ccol < p.batch;
            const T *ccolp = gout + ccol * p.bstride;
            auto ldb = [&](int row) -> C {
                if (LOADER == LOAD_TMA) return (C)buf[(size_t)row * R + rr];
                return clive ? (C)ccolp[(int64_t)row * ps] : C(0);
            };
            for (int d = 0; d < k; ++d) {
                C acc = part == 0 ? ldb(sdrow[d]) * sdscale[d] : C(0);
                for (int e = slamptr[d] + part; e < slamptr[d + 1]; e += cp)
                    acc = fma(-slamv[e], ldb(P.s_lo + slamc[e]), acc);
                if (cp > 1) {
#pragma unroll
                    for (int off = R; off < 32; off *= 2) acc += __shfl_xor_sync(0xffffffffu, acc, off);
                }
                if (part == 0) sx1[rr * k + d] = acc;
            }
            if (part == 0) {
                C *x1 = sx1 + rr * k;
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
                if (clive)
                    for (int d = 0; d < k; ++d) __stcs(gout + ccol * p.bstride + (int64_t)sdrow[d] * ps, (T)x1[d]);
            }
        }
        // ---------- own segment of b0 into registers
        C v[L];
        {
            if (LOADER == LOAD_TMA) {
                const T *src = buf + (size_t)(P.s_lo + a) * R + r;
                if (full) {
#pragma unroll
                    for (int i = 0; i < L; ++i) v[i] = (C)src[(size_t)i * R];
                } else {
#pragma unroll
                    for (int i = 0; i < L; ++i) v[i] = (a + i < nQ) ? (C)src[(size_t)i * R] : C(0);
                }
            } else {
                const T *src = gcol + (int64_t)(P.s_lo + a) * ps;
                if (full && live) {
#pragma unroll
                    for (int i = 0; i < L; ++i) v[i] = (C)__ldcs(src + (int64_t)i * ps);
                } else {
#pragma unroll
                    for (int i = 0; i < L; ++i) v[i] = (live && a + i < nQ) ? (C)__ldcs(src + (int64_t)i * ps) : C(0);
                }
            }
        }
        __syncthreads();  // B1: tile buffer consumed, x1 published
        if (LOADER == LOAD_TMA && tid == 0 && tile + (int)gridDim.x < p.ntiles) {
            const int nt = tile + gridDim.x;
            mbar_arrive_expect_tx(mbar, tile_bytes);
            for (int b = 0; b < p.nbox; ++b) tma_load_2d(buf + (size_t)b * p.boxr * R, &tmap, mbar, nt * R, b * p.boxr);
        }
        // ---------- b0 -= gamma x1 on this segment's gamma rows
        for (int e = sgptr[s]; e < sgptr[s + 1]; ++e) {
            const int i = sgamr[e] - a;
            const C dv = sgamv[e] * sx1[r * k + sgamc[e]];
#pragma unroll
            for (int j = 0; j < L; ++j)
                if (j == i) v[j] -= dv;
        }
        // ---------- local forward sweep, zero inflow:  y_i = b_i - sum_m L(i,i-m) y_{i-m}
        C st[K];
#pragma unroll
        for (int m = 0; m < K; ++m) st[m] = C(0);
#pragma unroll
        for (int i = 0; i < L; ++i) {
            C acc = v[i];
#pragma unroll
            for (int m = 0; m < K; ++m) acc = fma(-sL[m * nQpa + a + i], st[m], acc);
#pragma unroll
            for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
            st[0] = acc;
            v[i] = acc;
        }
#pragma unroll
        for (int j = 0; j < K; ++j) sfend[(s * R + r) * K + j] = st[j];
        __syncthreads();  // B2
        // ---------- forward carry (true y at rows a-1..a-K) and correction chain
        if (s > 0) {
            C cin[K];
#pragma unroll
            for (int m = 0; m < K; ++m) cin[m] = C(0);
            for (int t = max(0, s - G.carry_f); t < s; ++t) {
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = sfend[(t * R + r) * K + j];
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(sG[(t * K + j) * K + m], cin[m], acc);
                    nw[j] = acc;
                }
#pragma unroll
                for (int j = 0; j < K; ++j) cin[j] = nw[j];
            }
            // c_i = -sum_m L(i,i-m) c_{i-m}, c_{a-m} = cin ;  y_i += c_i
#pragma unroll
            for (int i = 0; i < L; ++i) {
                C c = C(0);
#pragma unroll
                for (int m = 0; m < K; ++m) c = fma(-sL[m * nQpa + a + i], cin[m], c);
#pragma unroll
                for (int m = K - 1; m > 0; --m) cin[m] = cin[m - 1];
                cin[0] = c;
                v[i] += c;
            }
        }
        // ---------- local backward sweep, zero outflow: x_i = y_i dinv_i - sum_m U'(i,m) x_{i+m}
        C st2[K];
#pragma unroll
        for (int m = 0; m < K; ++m) st2[m] = C(0);
#pragma unroll
        for (int i = L - 1; i >= 0; --i) {
            C acc = v[i] * sdinv[a + i];
#pragma unroll
            for (int m = 0; m < K; ++m) acc = fma(-sU[m * nQpa + a + i], st2[m], acc);
#pragma unroll
            for (int m = K - 1; m > 0; --m) st2[m] = st2[m - 1];
            st2[0] = acc;
            v[i] = acc;
        }
#pragma unroll
        for (int j = 0; j < K; ++j) sbbeg[(s * R + r) * K + j] = st2[j];
        __syncthreads();  // B3
        // ---------- backward carry (true x at rows a+L..a+L+K-1), correction chain, store
        T *dst = gcol + (int64_t)(P.s_lo + a) * ps;
        if (s < S - 1) {
            C co[K];
#pragma unroll
            for (int m = 0; m < K; ++m) co[m] = C(0);
            for (int t = min(S - 1, s + G.carry_b); t > s; --t) {
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = sbbeg[(t * R + r) * K + j];
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(sH[(t * K + j) * K + m], co[m], acc);
                    nw[j] = acc;
                }
#pragma unroll
                for (int j = 0; j < K; ++j) co[j] = nw[j];
            }
#pragma unroll
            for (int i = L - 1; i >= 0; --i) {
                C c = C(0);
#pragma unroll
                for (int m = 0; m < K; ++m) c = fma(-sU[m * nQpa + a + i], co[m], c);
#pragma unroll
                for (int m = K - 1; m > 0; --m) co[m] = co[m - 1];
                co[0] = c;
                v[i] += c;
            }
        }
        if (live) {
            if (full) {
#pragma unroll
                for (int i = 0; i < L; ++i) __stcs(dst + (int64_t)i * ps, (T)v[i]);
            } else {
#pragma unroll
                for (int i = 0; i < L; ++i)
                    if (a + i < nQ) __stcs(dst + (int64_t)i * ps, (T)v[i]);
            }
        }
    }
}

// ------------------------------------------------------------------ host
namespace {

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

template <typename T, int K, int L, int R, int LOADER>
int launch_t(const KParams &kp, const CUtensorMap &tm, int grid, int threads, cudaStream_t st, char *err, int errlen) {
    auto fn = sb_solve_kernel<T, K, L, R, LOADER>;
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

template <typename T, int L, int R, int LOADER>
int dispatch_K(int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads, cudaStream_t st, char *err,
               int errlen) {
    switch (K) {
        case 1: return launch_t<T, 1, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 2: return launch_t<T, 2, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 3: return launch_t<T, 3, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 4: return launch_t<T, 4, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
    }
    snprintf(err, errlen, "unsupported band K=%d", K);
    return 5;
}

// (dtype, R, loader) -> instantiation.  fp64: L=32, R in {16, 8};
// fp32: L=64, R in {32, 16}.
int dispatch(int dtype, int R, int loader, int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads,
             cudaStream_t st, char *err, int errlen) {
    const bool tma = loader == LOAD_TMA;
    if (dtype == 0) {
        if (R == 16) return tma ? dispatch_K<double, 32, 16, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen)
                                : dispatch_K<double, 32, 16, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
        if (R == 8) return tma ? dispatch_K<double, 32, 8, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen)
                               : dispatch_K<double, 32, 8, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
    } else {
        if (R == 32) return tma ? dispatch_K<float, 64, 32, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen)
                                : dispatch_K<float, 64, 32, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
        if (R == 16) return tma ? dispatch_K<float, 64, 16, LOAD_TMA>(K, kp, tm, grid, threads, st, err, errlen)
                                : dispatch_K<float, 64, 16, LOAD_DIRECT>(K, kp, tm, grid, threads, st, err, errlen);
    }
    snprintf(err, errlen, "unsupported tile width R=%d", R);
    return 5;
}

int layout_smem(KParams &kp, const DevPlan &P, int R, size_t esz, bool with_buf, int nbox, int boxr, int S) {
    size_t o = 0;
    auto take = [&](size_t bytes, size_t al) {
        o = align_up(o, al);
        size_t r = o;
        o += align_up(bytes, 16);
        return (int)r;
    };
    const int K = P.K, k = P.k;
    kp.off_buf = with_buf ? take((size_t)nbox * boxr * R * esz, 1024) : 0;
    kp.off_L = take((size_t)K * P.nQpa * esz, 16);
    kp.off_U = take((size_t)K * P.nQpa * esz, 16);
    kp.off_dinv = take((size_t)P.nQpa * esz, 16);
    kp.off_G = take((size_t)S * K * K * esz, 16);
    kp.off_H = take((size_t)S * K * K * esz, 16);
    kp.off_fend = take((size_t)S * R * K * esz, 16);
    kp.off_bbeg = take((size_t)S * R * K * esz, 16);
    kp.off_x1 = take((size_t)R * k * esz, 16);
    kp.off_lamptr = take((size_t)(k + 1) * 4, 16);
    kp.off_lamc = take((size_t)P.lam_nnz * 4, 16);
    kp.off_lamv = take((size_t)P.lam_nnz * esz, 16);
    kp.off_gamr = take((size_t)P.gam_nnz * 4, 16);
    kp.off_gamc = take((size_t)P.gam_nnz * 4, 16);
    kp.off_gamv = take((size_t)P.gam_nnz * esz, 16);
    kp.off_gptr = take((size_t)(S + 1) * 4, 16);
    kp.off_dlu = take((size_t)k * k * esz, 16);
    kp.off_dpiv = take((size_t)k * 4, 16);
    kp.off_dscale = take((size_t)k * esz, 16);
    kp.off_drow = take((size_t)k * 4, 16);
    kp.off_mbar = take(8, 8);
    kp.smem_total = (int)align_up(o, 16);
    return kp.smem_total;
}

}  // namespace

int launch_solve(const DevPlan &P, const SolveArgs &a, int num_sms, char *err, int errlen) {
    if (a.batch == 0) return 0;
    const size_t esz = a.dtype == 0 ? 8 : 4;
    const DevSeg &G = P.seg[a.dtype == 0 ? 0 : 1];
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

    // TMA for the batch-contiguous layout when the tensor-map rules hold
    // (16-B aligned base and row pitch) and the tile fits in shared memory.
    const bool contig = a.bstride == 1;
    const bool aligned = ((uintptr_t)a.rhs % 16 == 0) && ((a.pstride * (int64_t)esz) % 16 == 0);
    const int nbox = (P.n + 255) / 256;
    const int boxr = ((P.n + nbox - 1) / nbox + 7) / 8 * 8;
    const int cands64[2] = {16, 8}, cands32[2] = {32, 16};
    const int *cands = a.dtype == 0 ? cands64 : cands32;
    int R = 0, loader = LOAD_DIRECT;
    for (int ci = 0; ci < 2 && !R; ++ci) {
        const int cand = cands[ci];
        if (cand * G.S > MAX_THREADS) continue;
        KParams t = kp;
        if (contig && aligned && a.batch >= cand && get_encode() &&
            layout_smem(t, P, cand, esz, true, nbox, boxr, G.S) <= max_smem) {
            R = cand;
            loader = LOAD_TMA;
        } else if (layout_smem(t, P, cand, esz, false, 0, 0, G.S) <= max_smem) {
            R = cand;
            loader = LOAD_DIRECT;
        }
    }
    if (!R) {
        snprintf(err, errlen, "problem too large for the shared-memory kernel (n=%d, segments=%d)", P.n, G.S);
        return 5;
    }
    layout_smem(kp, P, R, esz, loader == LOAD_TMA, nbox, boxr, G.S);
    kp.ntiles = (int)((a.batch + R - 1) / R);
    kp.nbox = nbox;
    kp.boxr = boxr;
    CUtensorMap tm;
    memset(&tm, 0, sizeof(tm));
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
    const int threads = R * G.S;
    const int grid = (int)std::min<int64_t>((int64_t)kp.ntiles, (int64_t)num_sms);
    return dispatch(a.dtype, R, loader, P.K, kp, tm, grid, threads, a.stream, err, errlen);
}

}  // namespace sb
