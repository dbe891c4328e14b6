#pragma once
// kernels.cuh -- fused sm_100a kernels of the batched spline solve.
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
// The corner reads only input rows, so nothing is held back for a post-pass.
//
// Two kernels:
//  sb_tile_kernel  batch-contiguous layout (the paper's).  A persistent
//    CTA owns tiles of R right-hand sides x all n rows.  Tiles arrive by TMA
//    (cp.async.bulk.tensor 2-D) box by box; each box has a full and an empty
//    mbarrier, so a box is refilled with the next tile as soon as the warps
//    that read it are done.  One extra warp issues the TMAs and computes the
//    corner step of the NEXT tile while the compute warps solve the current
//    one.  Compute thread (r, s) keeps rows [s*L, s*L+L) of RHS r in
//    registers; the recurrences run locally with zero inflow and are made
//    exact by carries exchanged through shared memory (segment transfer
//    matrices) plus a correction chain (SPIKE).  HBM sees one read and one
//    write per element.
//  sb_warp_kernel  any strided layout, tuned for point-contiguous rows (the
//    GYSELA slice, C4).  One warp owns one RHS: the row is loaded coalesced
//    into a per-warp shared-memory row, lane s takes segment s (odd L makes
//    the transposed reads bank-conflict free), carries travel by warp
//    shuffles, and the row is written back coalesced.  No block barriers.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <type_traits>
#include <cstdio>
#include <cstring>

#include "device.hpp"

namespace sb {

enum Loader { LOAD_DIRECT = 0, LOAD_TMA = 1 };
constexpr int NBOXMAX = 8;
constexpr int TILE_MAX_THREADS = 512;  // <= 15 compute warps + 1 corner/producer warp: 4 warps per
                                       // SM sub-partition keeps the 128-register budget

struct KParams {
    DevPlan P;
    void *rhs;
    int64_t batch, bstride, pstride;
    int ntiles, nbox, boxr, ncw;     // tiles, TMA boxes per tile, rows per box, compute warps
    int empty_count[NBOXMAX];        // arrivals that free box c (reader warps + corner warp)
    // dynamic shared memory offsets (bytes)
    int off_buf, off_L, off_U, off_dinv, off_G, off_H, off_fend, off_bbeg, off_x1, off_lamptr, off_lamc, off_lamv,
        off_gamr, off_gamc, off_gamv, off_gptr, off_dlu, off_dpiv, off_dscale, off_drow, off_mbar, smem_total;
    int wbuf_pitch;                  // warp kernel: elements per per-warp row buffer
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
__device__ __forceinline__ void mbar_arrive(uint64_t *m) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(m)) : "memory");
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
__device__ __forceinline__ void named_bar(int id, int count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}

template <typename T>
__device__ __forceinline__ void copy_words(T *dst, const T *src, int count, int tid, int nthreads) {
    for (int i = tid; i < count; i += nthreads) dst[i] = src[i];
}

template <typename T> struct Vec2;
template <> struct Vec2<double> { using type = double2; };
template <> struct Vec2<float> { using type = float2; };

// ------------------------------------------------- per-thread segment math
// Factor access: f[m*ms + i] for band index m (0..K-1) and local row i.
// PAIRS: rows (i, i+1) are read with one 2-wide load (pitch even, i even).

// local forward sweep, zero inflow: y_i = b_i - sum_m L(i,i-1-m) y_{i-1-m}
template <typename C, int K, int L, bool PAIRS>
__device__ __forceinline__ void fwd_local(C (&v)[L], const C *fL, int ms, C (&st)[K]) {
#pragma unroll
    for (int m = 0; m < K; ++m) st[m] = C(0);
#pragma unroll
    for (int i = 0; i < L; i += (PAIRS ? 2 : 1)) {
        C l0[K], l1[K];
#pragma unroll
        for (int m = 0; m < K; ++m) {
            if constexpr (PAIRS) {
                const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(fL + m * ms + i);
                l0[m] = w.x;
                l1[m] = w.y;
            } else {
                l0[m] = fL[m * ms + i];
            }
        }
#pragma unroll
        for (int q = 0; q < (PAIRS ? 2 : 1); ++q) {
            C acc = v[i + q];
#pragma unroll
            for (int m = 0; m < K; ++m) acc = fma(-(q ? l1[m] : l0[m]), st[m], acc);
#pragma unroll
            for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
            st[0] = acc;
            v[i + q] = acc;
        }
    }
}

// forward correction chain c_i = -sum_m L(i,i-1-m) c_{i-1-m}, c(a-1-m) = cin[m];  y_i += c_i
template <typename C, int K, int L, bool PAIRS>
__device__ __forceinline__ void fwd_correct(C (&v)[L], const C *fL, int ms, C (&cin)[K]) {
#pragma unroll
    for (int i = 0; i < L; i += (PAIRS ? 2 : 1)) {
        C l0[K], l1[K];
#pragma unroll
        for (int m = 0; m < K; ++m) {
            if constexpr (PAIRS) {
                const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(fL + m * ms + i);
                l0[m] = w.x;
                l1[m] = w.y;
            } else {
                l0[m] = fL[m * ms + i];
            }
        }
#pragma unroll
        for (int q = 0; q < (PAIRS ? 2 : 1); ++q) {
            C c = C(0);
#pragma unroll
            for (int m = 0; m < K; ++m) c = fma(-(q ? l1[m] : l0[m]), cin[m], c);
#pragma unroll
            for (int m = K - 1; m > 0; --m) cin[m] = cin[m - 1];
            cin[0] = c;
            v[i + q] += c;
        }
    }
}

// local backward sweep, zero outflow: x_i = y_i dinv_i - sum_m U'(i,i+1+m) x_{i+1+m}
template <typename C, int K, int L, bool PAIRS>
__device__ __forceinline__ void bwd_local(C (&v)[L], const C *fU, const C *fD, int ms, C (&st)[K]) {
#pragma unroll
    for (int m = 0; m < K; ++m) st[m] = C(0);
#pragma unroll
    for (int i = L - (PAIRS ? 2 : 1); i >= 0; i -= (PAIRS ? 2 : 1)) {
        C u0[K], u1[K], d0, d1 = C(0);
#pragma unroll
        for (int m = 0; m < K; ++m) {
            if constexpr (PAIRS) {
                const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(fU + m * ms + i);
                u0[m] = w.x;
                u1[m] = w.y;
            } else {
                u0[m] = fU[m * ms + i];
            }
        }
        if constexpr (PAIRS) {
            const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(fD + i);
            d0 = w.x;
            d1 = w.y;
        } else {
            d0 = fD[i];
        }
#pragma unroll
        for (int q = (PAIRS ? 1 : 0); q >= 0; --q) {
            C acc = v[i + q] * (q ? d1 : d0);
#pragma unroll
            for (int m = 0; m < K; ++m) acc = fma(-(q ? u1[m] : u0[m]), st[m], acc);
#pragma unroll
            for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
            st[0] = acc;
            v[i + q] = acc;
        }
    }
}

// backward correction chain c_i = -sum_m U'(i,i+1+m) c_{i+1+m}, c(a+L+m) = co[m];  x_i += c_i
template <typename C, int K, int L, bool PAIRS>
__device__ __forceinline__ void bwd_correct(C (&v)[L], const C *fU, int ms, C (&co)[K]) {
#pragma unroll
    for (int i = L - (PAIRS ? 2 : 1); i >= 0; i -= (PAIRS ? 2 : 1)) {
        C u0[K], u1[K];
#pragma unroll
        for (int m = 0; m < K; ++m) {
            if constexpr (PAIRS) {
                const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(fU + m * ms + i);
                u0[m] = w.x;
                u1[m] = w.y;
            } else {
                u0[m] = fU[m * ms + i];
            }
        }
#pragma unroll
        for (int q = (PAIRS ? 1 : 0); q >= 0; --q) {
            C c = C(0);
#pragma unroll
            for (int m = 0; m < K; ++m) c = fma(-(q ? u1[m] : u0[m]), co[m], c);
#pragma unroll
            for (int m = K - 1; m > 0; --m) co[m] = co[m - 1];
            co[0] = c;
            v[i + q] += c;
        }
    }
}

// x1 <- delta'^{-1} x1 (getrs: row interchanges, unit-lower L, upper U; k x k row-major LU)
template <typename C>
__device__ __forceinline__ void getrs_small(C *x1, const C *lu, const int *piv, int k) {
    for (int d = 0; d < k; ++d) {
        const int pv = piv[d];
        if (pv != d) { C t = x1[d]; x1[d] = x1[pv]; x1[pv] = t; }
    }
    for (int i = 1; i < k; ++i)
        for (int j = 0; j < i; ++j) x1[i] = fma(-lu[i * k + j], x1[j], x1[i]);
    for (int i = k - 1; i >= 0; --i) {
        C acc = x1[i];
        for (int j = i + 1; j < k; ++j) acc = fma(-lu[i * k + j], x1[j], acc);
        x1[i] = acc / lu[i * k + i];
    }
}

// stage the constants of one segment plan + the corner data into shared memory
template <typename C, int K>
__device__ __forceinline__ void stage_constants(const KParams &p, const DevSeg &G, unsigned char *smem, int tid,
                                                int nthreads) {
    constexpr int CI = sizeof(C) == 8 ? 0 : 1;
    const DevPlan &P = p.P;
    const int k = P.k, S = G.S;
    const int nrec = K * S * G.LP;
    copy_words(reinterpret_cast<C *>(smem + p.off_L), reinterpret_cast<const C *>(G.Lr[CI]), nrec, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_U), reinterpret_cast<const C *>(G.Ur[CI]), nrec, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_dinv), reinterpret_cast<const C *>(G.dinv[CI]), S * G.LP, tid,
               nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_G), reinterpret_cast<const C *>(G.G[CI]), S * K * K, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_H), reinterpret_cast<const C *>(G.H[CI]), S * K * K, tid, nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_lamptr), P.lam_ptr, k + 1, tid, nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_lamc), P.lam_c, P.lam_nnz, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_lamv), reinterpret_cast<const C *>(P.lam_v[CI]), P.lam_nnz, tid,
               nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_gamr), P.gam_r, P.gam_nnz, tid, nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_gamc), P.gam_c, P.gam_nnz, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_gamv), reinterpret_cast<const C *>(P.gam_v[CI]), P.gam_nnz, tid,
               nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_gptr), G.gptr, S + 1, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_dlu), reinterpret_cast<const C *>(P.dlu[CI]), k * k, tid, nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_dpiv), P.dpiv, k, tid, nthreads);
    copy_words(reinterpret_cast<C *>(smem + p.off_dscale), reinterpret_cast<const C *>(P.dscale[CI]), k, tid,
               nthreads);
    copy_words(reinterpret_cast<int *>(smem + p.off_drow), P.drow, k, tid, nthreads);
}

// ========================================================= tile kernel
template <typename T, int K, int L, int R, int LOADER>
__global__ void __launch_bounds__(TILE_MAX_THREADS, 1)
    sb_tile_kernel(const __grid_constant__ KParams p, const __grid_constant__ CUtensorMap tmap) {
    using C = T;  // compute in the storage precision
    constexpr int CI = sizeof(T) == 8 ? 0 : 1;
    constexpr int SPW = 32 / R;  // segments per compute warp
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;
    const DevSeg &G = P.seg[CI];

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int S = G.S, LP = G.LP, nQ = P.nQ, k = P.k, s_lo = P.s_lo;
    const int ncw = p.ncw, nbox = p.nbox, boxr = p.boxr;
    const int ms = S * LP;  // band stride of the factor arrays

    C *sL = reinterpret_cast<C *>(smem + p.off_L);
    C *sU = reinterpret_cast<C *>(smem + p.off_U);
    C *sdinv = reinterpret_cast<C *>(smem + p.off_dinv);
    C *sG = reinterpret_cast<C *>(smem + p.off_G);
    C *sH = reinterpret_cast<C *>(smem + p.off_H);
    C *sfend = reinterpret_cast<C *>(smem + p.off_fend);
    C *sbbeg = reinterpret_cast<C *>(smem + p.off_bbeg);
    C *sx1 = reinterpret_cast<C *>(smem + p.off_x1);  // [2][R*k]
    const int *slamptr = reinterpret_cast<const int *>(smem + p.off_lamptr);
    const int *slamc = reinterpret_cast<const int *>(smem + p.off_lamc);
    const C *slamv = reinterpret_cast<const C *>(smem + p.off_lamv);
    const int *sgamr = reinterpret_cast<const int *>(smem + p.off_gamr);
    const int *sgamc = reinterpret_cast<const int *>(smem + p.off_gamc);
    const C *sgamv = reinterpret_cast<const C *>(smem + p.off_gamv);
    const int *sgptr = reinterpret_cast<const int *>(smem + p.off_gptr);
    const C *sdlu = reinterpret_cast<const C *>(smem + p.off_dlu);
    const int *sdpiv = reinterpret_cast<const int *>(smem + p.off_dpiv);
    const C *sdscale = reinterpret_cast<const C *>(smem + p.off_dscale);
    const int *sdrow = reinterpret_cast<const int *>(smem + p.off_drow);
    uint64_t *full = reinterpret_cast<uint64_t *>(smem + p.off_mbar);
    uint64_t *empty = full + NBOXMAX;
    uint64_t *x1full = empty + NBOXMAX;
    T *buf = reinterpret_cast<T *>(smem + p.off_buf);
    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    const uint32_t box_bytes = (uint32_t)(boxr * R * sizeof(T));

    if (tid == 0) {
        for (int c = 0; c < nbox; ++c) {
            mbar_init(full + c, 1);
            mbar_init(empty + c, p.empty_count[c]);
        }
        mbar_init(x1full + 0, 1);
        mbar_init(x1full + 1, 1);
        fence_mbar_init();
        if (LOADER == LOAD_TMA) prefetch_tmap(&tmap);
    }
    stage_constants<C, K>(p, G, smem, tid, blockDim.x);
    __syncthreads();

    if (warp == ncw) {
        // ===================== corner + producer warp (runs one tile ahead)
        const int part = lane / R, rr = lane % R;
        int it = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x, ++it) {
            if (LOADER == LOAD_TMA) {
                if (lane == 0)
                    for (int c = 0; c < nbox; ++c) {
                        if (it > 0) mbar_wait(empty + c, (it - 1) & 1);
                        mbar_arrive_expect_tx(full + c, box_bytes);
                        tma_load_2d(buf + (size_t)c * boxr * R, &tmap, full + c, tile * R, c * boxr);
                    }
                for (int c = 0; c < nbox; ++c) mbar_wait(full + c, it & 1);
            } else if (it > 0) {
                mbar_wait(empty + 0, (it - 1) & 1);  // all compute warps finished tile it-1
            }
            const int64_t ccol = (int64_t)tile * R + rr;
            const bool clive = ccol < p.batch;
            const T *ccolp = gout + ccol * p.bstride;
            auto ldb = [&](int row) -> C {
                if (LOADER == LOAD_TMA) return (C)buf[(size_t)row * R + rr];
                return clive ? (C)ccolp[(int64_t)row * ps] : C(0);
            };
            C *x1 = sx1 + (it & 1) * R * k + rr * k;
            for (int d = 0; d < k; ++d) {
                C acc = part == 0 ? ldb(sdrow[d]) * sdscale[d] : C(0);
                int e = slamptr[d] + part;
                const int e1 = slamptr[d + 1];
                // 4 independent partial sums keep the dependent smem loads in flight
                C a1 = C(0), a2 = C(0), a3 = C(0);
                for (; e + 3 * SPW < e1; e += 4 * SPW) {
                    acc = fma(-slamv[e], ldb(s_lo + slamc[e]), acc);
                    a1 = fma(-slamv[e + SPW], ldb(s_lo + slamc[e + SPW]), a1);
                    a2 = fma(-slamv[e + 2 * SPW], ldb(s_lo + slamc[e + 2 * SPW]), a2);
                    a3 = fma(-slamv[e + 3 * SPW], ldb(s_lo + slamc[e + 3 * SPW]), a3);
                }
                for (; e < e1; e += SPW) acc = fma(-slamv[e], ldb(s_lo + slamc[e]), acc);
                acc += (a1 + a2) + a3;
#pragma unroll
                for (int off = R; off < 32; off *= 2) acc += __shfl_xor_sync(0xffffffffu, acc, off);
                if (part == 0) x1[d] = acc;
            }
            if (part == 0 && k > 0) {
                getrs_small(x1, sdlu, sdpiv, k);
                if (clive)
                    for (int d = 0; d < k; ++d) __stcs(gout + ccol * p.bstride + (int64_t)sdrow[d] * ps, (T)x1[d]);
            }
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(x1full + (it & 1));
                if (LOADER == LOAD_TMA)
                    for (int c = 0; c < nbox; ++c) mbar_arrive(empty + c);
            }
        }
        return;
    }

    // ============================================== compute warps
    const int r = tid % R;
    const int s = tid / R;
    const bool active = s < S;
    const int a = s * L;
    const bool full_seg = a + L <= nQ;
    const int sc = active ? s : 0;  // idle threads of the last warp alias segment 0
    const C *fL = sL + (size_t)sc * LP;
    const C *fU = sU + (size_t)sc * LP;
    const C *fD = sdinv + (size_t)sc * LP;
    // boxes this warp reads (rows of its real segments)
    int c_lo = 0, c_hi = -1;
    {
        const int s0 = warp * SPW;
        const int r0 = s_lo + s0 * L;
        const int r1 = s_lo + min((s0 + SPW) * L, nQ) - 1;
        if (s0 < S && r1 >= r0) {
            c_lo = r0 / boxr;
            c_hi = r1 / boxr;
        }
    }
    const int nthr_c = ncw * 32;
    int it = 0;
    for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x, ++it) {
        const int64_t col = (int64_t)tile * R + r;
        const bool live = active && col < p.batch;
        T *gcol = gout + col * p.bstride;
        C v[L];
        // ---------- own segment of b0 into registers
        if (LOADER == LOAD_TMA) {
            for (int c = c_lo; c <= c_hi; ++c) mbar_wait(full + c, it & 1);
            const T *src = buf + (size_t)(s_lo + a) * R + r;
            if (full_seg) {
#pragma unroll
                for (int i = 0; i < L; ++i) v[i] = (C)src[(size_t)i * R];
            } else {
#pragma unroll
                for (int i = 0; i < L; ++i) v[i] = (active && a + i < nQ) ? (C)src[(size_t)i * R] : C(0);
            }
            __syncwarp();
            if (lane == 0)
                for (int c = c_lo; c <= c_hi; ++c) mbar_arrive(empty + c);
        } else {
            const T *src = gcol + (int64_t)(s_lo + a) * ps;
            if (full_seg && live) {
#pragma unroll
                for (int i = 0; i < L; ++i) v[i] = (C)__ldcs(src + (int64_t)i * ps);
            } else {
#pragma unroll
                for (int i = 0; i < L; ++i) v[i] = (live && a + i < nQ) ? (C)__ldcs(src + (int64_t)i * ps) : C(0);
            }
        }
        // ---------- b0 -= gamma x1 (only segments holding gamma rows wait for the corner warp)
        if (active && sgptr[s] < sgptr[s + 1]) {
            mbar_wait(x1full + (it & 1), (it >> 1) & 1);
            const C *x1 = sx1 + (it & 1) * R * k + r * k;
            for (int e = sgptr[s]; e < sgptr[s + 1]; ++e) {
                const int i = sgamr[e] - a;
                const C dv = sgamv[e] * x1[sgamc[e]];
#pragma unroll
                for (int j = 0; j < L; ++j)
                    if (j == i) v[j] -= dv;
            }
        }
        // ---------- local forward sweep, publish end state
        C st[K];
        fwd_local<C, K, L, true>(v, fL, ms, st);
        if (active)
#pragma unroll
            for (int j = 0; j < K; ++j) sfend[(s * R + r) * K + j] = st[j];
        named_bar(1, nthr_c);  // B2
        // ---------- forward carry (true y at rows a-1..a-K) + correction chain
        if (active && s > 0) {
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
            fwd_correct<C, K, L, true>(v, fL, ms, cin);
        }
        // ---------- local backward sweep, publish begin state
        bwd_local<C, K, L, true>(v, fU, fD, ms, st);
        if (active)
#pragma unroll
            for (int j = 0; j < K; ++j) sbbeg[(s * R + r) * K + j] = st[j];
        named_bar(1, nthr_c);  // B3
        // ---------- backward carry (true x at rows a+L..a+L+K-1) + correction chain
        if (active && s < S - 1) {
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
            bwd_correct<C, K, L, true>(v, fU, ms, co);
        }
        // ---------- store x0 straight from registers.  DIRECT mode: the corner warp
        // reads b0 from HBM, so no row of this tile is overwritten before x1 is done.
        if (LOADER == LOAD_DIRECT && k > 0) mbar_wait(x1full + (it & 1), (it >> 1) & 1);
        if (live) {
            T *dst = gcol + (int64_t)(s_lo + a) * ps;
            if (full_seg) {
#pragma unroll
                for (int i = 0; i < L; ++i) __stcs(dst + (int64_t)i * ps, (T)v[i]);
            } else {
#pragma unroll
                for (int i = 0; i < L; ++i)
                    if (a + i < nQ) __stcs(dst + (int64_t)i * ps, (T)v[i]);
            }
        }
        if (LOADER == LOAD_DIRECT) {  // tile done: lets the corner warp move to tile it+1
            __syncwarp();
            if (lane == 0) mbar_arrive(empty + 0);
        }
    }
}

// ========================================================= warp kernel
// One warp per RHS; lane s owns segment s (rows [s*L, s*L+L) of Q).
template <typename T, int K, int L>
__global__ void __launch_bounds__(256)
    sb_warp_kernel(const __grid_constant__ KParams p) {
    using C = T;
    constexpr int CI = sizeof(T) == 8 ? 0 : 1;
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;
    const DevSeg &G = P.seg[2];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int S = G.S, LP = G.LP, nQ = P.nQ, k = P.k, s_lo = P.s_lo, n = P.n;
    const int ms = S * LP;

    stage_constants<C, K>(p, G, smem, tid, blockDim.x);
    __syncthreads();

    const C *sL = reinterpret_cast<const C *>(smem + p.off_L);
    const C *sU = reinterpret_cast<const C *>(smem + p.off_U);
    const C *sdinv = reinterpret_cast<const C *>(smem + p.off_dinv);
    const C *sG = reinterpret_cast<const C *>(smem + p.off_G);
    const C *sH = reinterpret_cast<const C *>(smem + p.off_H);
    const int *slamptr = reinterpret_cast<const int *>(smem + p.off_lamptr);
    const int *slamc = reinterpret_cast<const int *>(smem + p.off_lamc);
    const C *slamv = reinterpret_cast<const C *>(smem + p.off_lamv);
    const int *sgamr = reinterpret_cast<const int *>(smem + p.off_gamr);
    const int *sgamc = reinterpret_cast<const int *>(smem + p.off_gamc);
    const C *sgamv = reinterpret_cast<const C *>(smem + p.off_gamv);
    const C *sdlu = reinterpret_cast<const C *>(smem + p.off_dlu);
    const int *sdpiv = reinterpret_cast<const int *>(smem + p.off_dpiv);
    const C *sdscale = reinterpret_cast<const C *>(smem + p.off_dscale);
    const int *sdrow = reinterpret_cast<const int *>(smem + p.off_drow);
    C *rowbuf = reinterpret_cast<C *>(smem + p.off_buf) + (size_t)warp * p.wbuf_pitch;  // n values + k spare
    C *x1 = rowbuf + n;  // k values after the row

    const int s = lane;
    const bool active = s < S;
    const int a = s * L;
    const C *fL = sL + (size_t)(active ? s : 0) * LP;
    const C *fU = sU + (size_t)(active ? s : 0) * LP;
    const C *fD = sdinv + (size_t)(active ? s : 0) * LP;
    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    const bool vec = (ps == 1) && ((p.bstride * (int64_t)sizeof(T)) % 16 == 0) &&
                     ((uintptr_t)p.rhs % 16 == 0) && (n % (16 / (int)sizeof(T)) == 0);
    constexpr int VW = 16 / sizeof(T);  // elements per 16-B vector

    const int64_t gw = (int64_t)blockIdx.x * (blockDim.x >> 5) + warp;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t rhs = gw; rhs < p.batch; rhs += nw) {
        T *g = gout + rhs * p.bstride;
        // ---------- coalesced load of the whole row
        if (vec) {
            using V = typename std::conditional<sizeof(T) == 8, double2, float4>::type;
            const V *gv = reinterpret_cast<const V *>(g);
            for (int q = lane; q < n / VW; q += 32) {
                const V w = __ldcs(gv + q);
                const T *pw = reinterpret_cast<const T *>(&w);
#pragma unroll
                for (int e = 0; e < VW; ++e) rowbuf[q * VW + e] = (C)pw[e];
            }
        } else {
            for (int j = lane; j < n; j += 32) rowbuf[j] = (C)__ldcs(g + (int64_t)j * ps);
        }
        __syncwarp();
        // ---------- corner: x1 = delta'^{-1} (s1*b1 - Lambda b0), then b0 -= gamma x1
        if (k > 0) {
            for (int d = 0; d < k; ++d) {
                C acc = lane == 0 ? rowbuf[sdrow[d]] * sdscale[d] : C(0);
                for (int e = slamptr[d] + lane; e < slamptr[d + 1]; e += 32)
                    acc = fma(-slamv[e], rowbuf[s_lo + slamc[e]], acc);
#pragma unroll
                for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
                if (lane == 0) x1[d] = acc;
            }
            if (lane == 0) {
                getrs_small(x1, sdlu, sdpiv, k);
                for (int e = 0; e < P.gam_nnz; ++e) rowbuf[s_lo + sgamr[e]] -= sgamv[e] * x1[sgamc[e]];
                for (int d = 0; d < k; ++d) rowbuf[sdrow[d]] = x1[d];
            }
            __syncwarp();
        }
        // ---------- own segment into registers (odd L: conflict-free)
        C v[L];
#pragma unroll
        for (int i = 0; i < L; ++i) v[i] = (active && a + i < nQ) ? rowbuf[s_lo + a + i] : C(0);
        // ---------- forward: local sweep, carry by shuffles, correction chain
        C st[K];
        fwd_local<C, K, L, false>(v, fL, ms, st);
        {
            C cin[K];
#pragma unroll
            for (int m = 0; m < K; ++m) cin[m] = C(0);
            for (int w = G.carry_f; w >= 1; --w) {  // from segment s-w up to s-1
                const int t = s - w;
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = __shfl_up_sync(0xffffffffu, st[j], w);
                    if (t >= 0)
#pragma unroll
                        for (int m = 0; m < K; ++m) acc = fma(sG[(t * K + j) * K + m], cin[m], acc);
                    nw[j] = t >= 0 ? acc : C(0);
                }
#pragma unroll
                for (int j = 0; j < K; ++j) cin[j] = nw[j];
            }
            if (active && s > 0) fwd_correct<C, K, L, false>(v, fL, ms, cin);
        }
        // ---------- backward: local sweep, carry by shuffles, correction chain
        bwd_local<C, K, L, false>(v, fU, fD, ms, st);
        {
            C co[K];
#pragma unroll
            for (int m = 0; m < K; ++m) co[m] = C(0);
            for (int w = G.carry_b; w >= 1; --w) {  // from segment s+w down to s+1
                const int t = s + w;
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = __shfl_down_sync(0xffffffffu, st[j], w);
                    if (t < S)
#pragma unroll
                        for (int m = 0; m < K; ++m) acc = fma(sH[(t * K + j) * K + m], co[m], acc);
                    nw[j] = t < S ? acc : C(0);
                }
#pragma unroll
                for (int j = 0; j < K; ++j) co[j] = nw[j];
            }
            if (active && s < S - 1) bwd_correct<C, K, L, false>(v, fU, ms, co);
        }
        // ---------- back to the row buffer, coalesced store
#pragma unroll
        for (int i = 0; i < L; ++i)
            if (active && a + i < nQ) rowbuf[s_lo + a + i] = v[i];
        __syncwarp();
        if (vec) {
            using V = typename std::conditional<sizeof(T) == 8, double2, float4>::type;
            V *gv = reinterpret_cast<V *>(g);
            for (int q = lane; q < n / VW; q += 32) {
                V w;
                T *pw = reinterpret_cast<T *>(&w);
#pragma unroll
                for (int e = 0; e < VW; ++e) pw[e] = (T)rowbuf[q * VW + e];
                __stcs(gv + q, w);
            }
        } else {
            for (int j = lane; j < n; j += 32) __stcs(g + (int64_t)j * ps, (T)rowbuf[j]);
        }
        __syncwarp();
    }
}

}  // namespace sb

namespace sb {
// per-TU launchers (tile_f64.cu, tile_f32.cu, warp_f64.cu, warp_f32.cu)
int launch_tile_f64(int R, int loader, int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads,
                    cudaStream_t st, char *err, int errlen);
int launch_tile_f32(int R, int loader, int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads,
                    cudaStream_t st, char *err, int errlen);
int launch_warp_f64(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);
int launch_warp_f32(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);

inline int check_launch(const char *what, char *err, int errlen) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        snprintf(err, errlen, "%s: %s", what, cudaGetErrorString(e));
        return 3;
    }
    return 0;
}

template <typename T, int K, int L, int R, int LOADER>
int launch_tile(const KParams &kp, const CUtensorMap &tm, int grid, int threads, cudaStream_t st, char *err,
                int errlen) {
    auto fn = sb_tile_kernel<T, K, L, R, LOADER>;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kp.smem_total) != cudaSuccess)
        return check_launch("cudaFuncSetAttribute(tile)", err, errlen);
    fn<<<grid, threads, kp.smem_total, st>>>(kp, tm);
    return check_launch("tile kernel launch", err, errlen);
}

template <typename T, int L, int R, int LOADER>
int tile_K(int K, const KParams &kp, const CUtensorMap &tm, int grid, int threads, cudaStream_t st, char *err,
           int errlen) {
    switch (K) {
        case 1: return launch_tile<T, 1, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 2: return launch_tile<T, 2, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 3: return launch_tile<T, 3, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
        case 4: return launch_tile<T, 4, L, R, LOADER>(kp, tm, grid, threads, st, err, errlen);
    }
    snprintf(err, errlen, "unsupported band K=%d", K);
    return 5;
}

template <typename T, int K, int L>
int launch_warp1(const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    auto fn = sb_warp_kernel<T, K, L>;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kp.smem_total) != cudaSuccess)
        return check_launch("cudaFuncSetAttribute(warp)", err, errlen);
    fn<<<grid, 256, kp.smem_total, st>>>(kp);
    return check_launch("warp kernel launch", err, errlen);
}

// odd segment lengths instantiated for the warp kernel (the plan picks from this set)
template <typename T, int K>
int warp_L(int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    switch (L) {
        case 3: return launch_warp1<T, K, 3>(kp, grid, st, err, errlen);
        case 5: return launch_warp1<T, K, 5>(kp, grid, st, err, errlen);
        case 9: return launch_warp1<T, K, 9>(kp, grid, st, err, errlen);
        case 17: return launch_warp1<T, K, 17>(kp, grid, st, err, errlen);
        case 33: return launch_warp1<T, K, 33>(kp, grid, st, err, errlen);
        case 63: return launch_warp1<T, K, 63>(kp, grid, st, err, errlen);
    }
    snprintf(err, errlen, "warp kernel: no instantiation for segment length %d", L);
    return 5;
}

template <typename T>
int warp_K(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    switch (K) {
        case 1: return warp_L<T, 1>(L, kp, grid, st, err, errlen);
        case 2: return warp_L<T, 2>(L, kp, grid, st, err, errlen);
        case 3: return warp_L<T, 3>(L, kp, grid, st, err, errlen);
        case 4: return warp_L<T, 4>(L, kp, grid, st, err, errlen);
    }
    snprintf(err, errlen, "unsupported band K=%d", K);
    return 5;
}
}  // namespace sb
