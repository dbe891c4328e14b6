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
#include <mutex>
#include <set>
#include <utility>
#include <type_traits>
#include <cstdio>
#include <cstring>

#include "device.hpp"

namespace sb {

enum Loader { LOAD_DIRECT = 0, LOAD_TMA = 1 };

// shared-memory layout of the non-uniform advection geometry (doubles from
// off_geo; every array 16-B aligned for the bulk copies):
//   xe[N+2p+1] (t_c at xe[c+p]) | xi[n] | rcp[(N+2p) p] | bucket table (int)
struct GeoLayout {
    int o_xi, o_rc, o_tbl, total_doubles;
    __host__ __device__ GeoLayout(const DevPlan &P) {
        auto even = [](int x) { return (x + 1) & ~1; };
        o_xi = even(P.N + 2 * P.p + 1);
        o_rc = o_xi + even(P.n);
        o_tbl = o_rc + even((P.N + 2 * P.p) * (P.p | 1));
        total_doubles = o_tbl + (P.adv_nbkt + 1) / 2 + 2;
    }
};
constexpr int NBOXMAX = 8;
constexpr int WB_FRONT = 4;
constexpr int WARP_MAX_WARPS = 16;  // warp kernel: <= 16 warps per block / per SM (128 registers each)  // warp kernel: elements in front of each row buffer (advection wrap pad)
constexpr int TILE_MAX_THREADS = 512;  // <= 15 compute warps + 1 corner/producer warp: 4 warps per
                                       // SM sub-partition keeps the 128-register budget

struct KParams {
    DevPlan P;
    void *rhs;
    int64_t batch, bstride, pstride;
    int ntiles, nbox, boxr, ncw;     // tiles, TMA boxes per tile, rows per box, compute warps
    int tps;                         // tile kernel: tiles per slab (ntiles = nslab * tps)
    int64_t slab_stride;             // tile kernel: elements between slabs of (n, batch) blocks
    int empty_count[NBOXMAX];        // arrivals that free box c (reader warps; corner warp if none)
    int corner_arrive_mask;          // boxes without a compute-warp reader: the corner warp frees them
    int corner_need_mask;            // (no corner boxes) boxes holding the rows the corner reads
    int box_order[NBOXMAX];          // TMA issue order of the boxes: the corner's boxes first
    int cbox;                        // rows of each corner box (0: corner reads the main tile)
    // dynamic shared memory offsets (bytes)
    int off_lw;                      // tile corner: Lambda window (DevPlan::lw_*)
    // pair tile (pair.cuh): per CTA of the cluster: first row, rows, first segment,
    // segments, boxes, and the arrivals that free each box
    int pr_rb[2], pr_nrows[2], pr_seg0[2], pr_nseg[2], pr_nbox[2];
    int pr_empty[2][NBOXMAX];
    int off_buf, off_L, off_U, off_dinv, off_G, off_H, off_fend, off_bbeg, off_x1, off_lamptr, off_lamc, off_lamv,
        off_gamr, off_gamc, off_gamv, off_gptr, off_dlu, off_dpiv, off_dscale, off_drow, off_mbar, off_cbuf,
        smem_total;
    int wbuf_pitch;                  // warp kernel: elements per per-warp row buffer
    int bulk, warp_threads;          // warp kernel: bulk-copy pipeline on/off, threads per block
    const double *shift;             // advect: per-RHS displacement (nullptr: plain solve)
                                     // (wbuf_pitch includes WB_FRONT + n + max(k, 3) + slack)
    int adv, off_geo;                // advect flag; smem offset of xe[N+2p+1], xi[n], rcp[(N+2p) p] (fp64)
};

// SB_TRACE (diagnostic builds only, never the shipped library): lane 0 of
// every warp of blocks < 4 records a timestamp at up to 9 points of its first
// TR_TILES tiles into g_sb_trace[block][tile][warp][point] (tools/trace_tile.py).
#ifdef SB_TRACE
constexpr int TR_BLOCKS = 4, TR_TILES = 8, TR_WARPS = 16, TR_PTS = 9;
static __device__ long long g_sb_trace[TR_BLOCKS * TR_TILES * TR_WARPS * TR_PTS];
__device__ __forceinline__ long long sb_trace_clock() {
#ifdef SB_TRACE_GLOBALTIMER
    long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
#else
    return clock64();
#endif
}
#define SB_TR(pt)                                                                                          \
    do {                                                                                                   \
        if (lane == 0 && blockIdx.x < TR_BLOCKS && it < TR_TILES)                                          \
            g_sb_trace[((blockIdx.x * TR_TILES + it) * TR_WARPS + warp) * TR_PTS + (pt)] = sb_trace_clock(); \
    } while (0)
#else
#define SB_TR(pt) \
    do {          \
    } while (0)
#endif

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
// 3-D box (rhs, row, slab): the tile kernel's tensor maps carry a slab
// dimension so one launch covers many (n, batch) blocks (2-D builder, pass 2)
__device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *map, uint64_t *mbar, int c0, int c1,
                                            int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
        "[%5];" ::"r"(smem_u32(dst)),
        "l"(map), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(mbar))
        : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}
__device__ __forceinline__ void named_bar(int id, int count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}


template <typename T> struct Vec2;
template <> struct Vec2<double> { using type = double2; };
template <> struct Vec2<float> { using type = float2; };

// ------------------------------------------------- per-thread segment math
// Each thread runs NV independent chains (NV right-hand sides) over the same
// L rows; v[i][q] is row i of RHS q.  Factor access: f[m*ms + i] for band
// index m (0..K-1) and local row i; one factor load serves all NV chains.
// PAIRS: rows (i, i+1) are read with one 2-wide load (pitch even, i even).
// Inside each row the newest state enters the FMA chain last (1-FMA critical
// path per row).

template <typename C, int K, bool PAIRS>
__device__ __forceinline__ void load_band(const C *f, int ms, int i, C (&f0)[K], C (&f1)[K]) {
#pragma unroll
    for (int m = 0; m < K; ++m) {
        if constexpr (PAIRS) {
            const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(f + m * ms + i);
            f0[m] = w.x;
            f1[m] = w.y;
        } else {
            f0[m] = f[m * ms + i];
            f1[m] = C(0);
        }
    }
}

// local forward sweep, zero inflow: y_i = b_i - sum_m L(i,i-1-m) y_{i-1-m}
template <typename C, int K, int L, int NV, bool PAIRS>
__device__ __forceinline__ void fwd_local(C (&v)[L][NV], const C *fL, int ms, C (&st)[K][NV]) {
#pragma unroll
    for (int m = 0; m < K; ++m)
#pragma unroll
        for (int q = 0; q < NV; ++q) st[m][q] = C(0);
#pragma unroll
    for (int i = 0; i < L; i += (PAIRS ? 2 : 1)) {
        C l0[K], l1[K];
        load_band<C, K, PAIRS>(fL, ms, i, l0, l1);
#pragma unroll
        for (int h = 0; h < (PAIRS ? 2 : 1); ++h) {
#pragma unroll
            for (int q = 0; q < NV; ++q) {
                C acc = v[i + h][q];
#pragma unroll
                for (int m = K - 1; m >= 0; --m) acc = fma(-(h ? l1[m] : l0[m]), st[m][q], acc);
#pragma unroll
                for (int m = K - 1; m > 0; --m) st[m][q] = st[m - 1][q];
                st[0][q] = acc;
                v[i + h][q] = acc;
            }
        }
    }
}

// forward correction chain c_i = -sum_m L(i,i-1-m) c_{i-1-m}, c(a-1-m) = cin[m];  y_i += c_i
template <typename C, int K, int L, int NV, bool PAIRS>
__device__ __forceinline__ void fwd_correct(C (&v)[L][NV], const C *fL, int ms, C (&cin)[K][NV]) {
#pragma unroll
    for (int i = 0; i < L; i += (PAIRS ? 2 : 1)) {
        C l0[K], l1[K];
        load_band<C, K, PAIRS>(fL, ms, i, l0, l1);
#pragma unroll
        for (int h = 0; h < (PAIRS ? 2 : 1); ++h) {
#pragma unroll
            for (int q = 0; q < NV; ++q) {
                C c = C(0);
#pragma unroll
                for (int m = K - 1; m >= 0; --m) c = fma(-(h ? l1[m] : l0[m]), cin[m][q], c);
#pragma unroll
                for (int m = K - 1; m > 0; --m) cin[m][q] = cin[m - 1][q];
                cin[0][q] = c;
                v[i + h][q] += c;
            }
        }
    }
}

// local backward sweep, zero outflow: x_i = y_i dinv_i - sum_m U'(i,i+1+m) x_{i+1+m}
template <typename C, int K, int L, int NV, bool PAIRS>
__device__ __forceinline__ void bwd_local(C (&v)[L][NV], const C *fU, const C *fD, int ms, C (&st)[K][NV]) {
#pragma unroll
    for (int m = 0; m < K; ++m)
#pragma unroll
        for (int q = 0; q < NV; ++q) st[m][q] = C(0);
#pragma unroll
    for (int i = L - (PAIRS ? 2 : 1); i >= 0; i -= (PAIRS ? 2 : 1)) {
        C u0[K], u1[K], d0, d1 = C(0);
        load_band<C, K, PAIRS>(fU, ms, i, u0, u1);
        if constexpr (PAIRS) {
            const auto w = *reinterpret_cast<const typename Vec2<C>::type *>(fD + i);
            d0 = w.x;
            d1 = w.y;
        } else {
            d0 = fD[i];
        }
#pragma unroll
        for (int h = (PAIRS ? 1 : 0); h >= 0; --h) {
#pragma unroll
            for (int q = 0; q < NV; ++q) {
                C acc = v[i + h][q] * (h ? d1 : d0);
#pragma unroll
                for (int m = K - 1; m >= 0; --m) acc = fma(-(h ? u1[m] : u0[m]), st[m][q], acc);
#pragma unroll
                for (int m = K - 1; m > 0; --m) st[m][q] = st[m - 1][q];
                st[0][q] = acc;
                v[i + h][q] = acc;
            }
        }
    }
}

// backward correction chain c_i = -sum_m U'(i,i+1+m) c_{i+1+m}, c(a+L+m) = co[m];  x_i += c_i.
// STORE: row i is final once corrected, so it goes to HBM right there (one
// NV-wide vector per row): the stores trickle out under the chain's FMA latency
// instead of leaving every warp of the tile in one burst.  dst points at row
// L-1 of this segment and walks back by ps per row (one 64-bit add per row,
// not a multiply); rows i >= nvalid are not stored (PRED only: the last segment).
template <typename C, int K, int L, int NV, bool PAIRS, bool STORE = false, bool PRED = false, typename T = C>
__device__ __forceinline__ void bwd_correct(C (&v)[L][NV], const C *fU, int ms, C (&co)[K][NV],
                                            T *dst = nullptr, int64_t ps = 0, int nvalid = 0) {
    using V = typename std::conditional<NV == 1, T,
                                        typename std::conditional<sizeof(T) == 8, double2,
                                                                  typename std::conditional<NV == 2, float2,
                                                                                            float4>::type>::type>::type;
#pragma unroll
    for (int i = L - (PAIRS ? 2 : 1); i >= 0; i -= (PAIRS ? 2 : 1)) {
        C u0[K], u1[K];
        load_band<C, K, PAIRS>(fU, ms, i, u0, u1);
#pragma unroll
        for (int h = (PAIRS ? 1 : 0); h >= 0; --h) {
#pragma unroll
            for (int q = 0; q < NV; ++q) {
                C c = C(0);
#pragma unroll
                for (int m = K - 1; m >= 0; --m) c = fma(-(h ? u1[m] : u0[m]), co[m][q], c);
#pragma unroll
                for (int m = K - 1; m > 0; --m) co[m][q] = co[m - 1][q];
                co[0][q] = c;
                v[i + h][q] += c;
            }
            if constexpr (STORE) {
                if (!PRED || i + h < nvalid) {
                    V w;
                    T *pw = reinterpret_cast<T *>(&w);
#pragma unroll
                    for (int q = 0; q < NV; ++q) pw[q] = (T)v[i + h][q];
                    // plain (write-back) store: measured faster than st.global.cs here
                    // (C2 0.2861 -> 0.2830 ms, C3 Greville 0.3178 -> 0.3162, C5S8 2.874 -> 2.857)
                    *reinterpret_cast<V *>(dst) = w;
                }
                dst -= ps;
            }
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

// x1 <- delta'^{-1} x1 with x1 in registers (warp kernel corner, k <= KR;
// unrolled and guarded by d < k, no dynamic register indexing; the same
// operations in the same order as getrs_small; LAPACK pivots, piv[d] >= d).
// Measured (A/B against the lane-0 corner, two sessions): C4 0.383 -> 0.352
// ms, C6 0.389 -> 0.379 ms, C6NU 0.591 -> 0.618 ms (pass 1 has k = 2).
// Restricting it to k == 1, or instantiating 1 slot, changes the code
// generation of the whole kernel and loses the C4 gain (0.374 ms).
constexpr int WCORNER_KREG = 8;
template <typename C, int KR>
__device__ __forceinline__ void wgetrs_reg(C (&x)[KR], const C *lu, const int *piv, int k) {
#pragma unroll
    for (int d = 0; d < KR; ++d) {
        if (d < k) {
            const int pv = piv[d];
            C xp = x[d];
#pragma unroll
            for (int j = d + 1; j < KR; ++j) xp = j == pv ? x[j] : xp;
            const C t = x[d];
            x[d] = xp;
#pragma unroll
            for (int j = d + 1; j < KR; ++j) x[j] = j == pv ? t : x[j];
        }
    }
#pragma unroll
    for (int i = 1; i < KR; ++i)
        if (i < k)
#pragma unroll
            for (int j = 0; j < i; ++j) x[i] = fma(-lu[i * k + j], x[j], x[i]);
#pragma unroll
    for (int i = KR - 1; i >= 0; --i)
        if (i < k) {
            C acc = x[i];
#pragma unroll
            for (int j = i + 1; j < KR; ++j)
                if (j < k) acc = fma(-lu[i * k + j], x[j], acc);
            x[i] = acc / lu[i * k + i];
        }
}

// Stage the constants of one segment plan + the corner data (+ the advection
// geometry) into shared memory with bulk async copies (cp.async.bulk, one
// instruction per array, completion on one mbarrier) instead of a
// load/store loop: the copies stream at L2 bandwidth and cost the CTA a
// single wait.  Every array starts 16-B aligned in the blob and in shared
// memory and its size is rounded up to 16 B (the blob pads each array).
// Each copy raises the barrier's expected transaction count itself
// (mbarrier.expect_tx), and one arrive closes the list, so no list of copies
// is kept (a local array of them would live on the stack).
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *mbar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(mbar))
                 : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *m, uint32_t bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void stage_one(void *dst, const void *src, size_t nb, uint64_t *bar) {
    const uint32_t b16 = (uint32_t)((nb + 15) & ~(size_t)15);
    if (b16 == 0) return;
    mbar_expect_tx(bar, b16);
    bulk_g2s(dst, src, b16, bar);
}

// one thread: issue every copy, then the single arrival that lets the phase complete
template <typename C, int K>
__device__ __forceinline__ void stage_constants_issue(const KParams &p, const DevSeg &G, unsigned char *smem,
                                                      uint64_t *cbar) {
    constexpr int CI = sizeof(C) == 8 ? 0 : 1;
    const DevPlan &P = p.P;
    const int k = P.k, S = G.S;
    const size_t esz = sizeof(C);
    stage_one(smem + p.off_L, G.F[CI], (size_t)G.nslots * (2 * K + 1) * G.LP * esz, cbar);
    stage_one(smem + p.off_G, G.G[CI], (size_t)S * K * K * esz, cbar);
    stage_one(smem + p.off_H, G.H[CI], (size_t)S * K * K * esz, cbar);
    stage_one(smem + p.off_lamptr, P.lam_ptr, (size_t)(k + 1) * 4, cbar);
    stage_one(smem + p.off_lamc, P.lam_c, (size_t)P.lam_nnz * 4, cbar);
    stage_one(smem + p.off_lamv, P.lam_v[CI], (size_t)P.lam_nnz * esz, cbar);
    stage_one(smem + p.off_lw, P.lw_v[CI], (size_t)(P.lw_head + P.lw_tail) * k * esz, cbar);
    stage_one(smem + p.off_gamr, P.gam_r, (size_t)P.gam_nnz * 4, cbar);
    stage_one(smem + p.off_gamc, P.gam_c, (size_t)P.gam_nnz * 4, cbar);
    stage_one(smem + p.off_gamv, P.gam_v[CI], (size_t)P.gam_nnz * esz, cbar);
    stage_one(smem + p.off_gptr, G.gptr, (size_t)(S + 1) * 4, cbar);
    stage_one(smem + p.off_dlu, P.dlu[CI], (size_t)k * k * esz, cbar);
    stage_one(smem + p.off_dpiv, P.dpiv, (size_t)k * 4, cbar);
    stage_one(smem + p.off_dscale, P.dscale[CI], (size_t)k * esz, cbar);
    stage_one(smem + p.off_drow, P.drow, (size_t)k * 4, cbar);
    if (p.adv && !P.adv_uniform) {  // advection geometry: xe | xi | rcp | bucket table, each 16-B aligned
        const GeoLayout gl(P);
        double *sgeo = reinterpret_cast<double *>(smem + p.off_geo);
        stage_one(sgeo, P.xe, (size_t)(P.N + 2 * P.p + 1) * 8, cbar);
        stage_one(sgeo + gl.o_xi, P.xi, (size_t)P.n * 8, cbar);
        stage_one(sgeo + gl.o_rc, P.adv_rcp, (size_t)(P.N + 2 * P.p) * (P.p | 1) * 8, cbar);
        stage_one(sgeo + gl.o_tbl, P.adv_tbl, (size_t)P.adv_nbkt * 4, cbar);
    }
    mbar_arrive(cbar);
}

// bulk (non-tensor) copies and the generic->async proxy fence
__device__ __forceinline__ void bulk_load(void *dst, const void *src, uint32_t bytes, uint64_t *mbar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(mbar))
                 : "memory");
}
__device__ __forceinline__ void bulk_store(void *dst, const void *src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)),
                 "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ---------------------------------------------------- tile-kernel corner
// x1 = delta'^{-1} (s1 b1 - Lambda b0) for one tile (one RHS per lane pair),
// run by the corner/producer warp one tile ahead of the compute warps.
template <typename C, typename T> struct CornerCtx {
    int part, lh, lw;
    const C *slw, *sdlu, *sdscale;
    const int *sdrow, *sdpiv;
    C *sx1;            // this lane's x1 slot in shared memory (x1[d] at sx1[d * R]: [d][rhs] order)
    T *gout;           // column of this RHS in HBM (nullptr: RHS beyond the batch)
    int64_t ps;
    const T *hb, *tb;  // b at the first row of the Lambda window's head / tail (this RHS)
    int64_t bst;       // elements between consecutive rows there
};

// k = KC <= 8: Lambda on its dense column window (each b row loaded once for
// all KC rows; loads in independent batches), xor-shuffle over the CPR lanes
// of a RHS, getrs on registers, delta rows of x to HBM, x1 to shared memory
// (the compute warps holding gamma rows apply b0 -= gamma x1).
template <typename C, typename T, int KC, int R, typename LDB>
__device__ __forceinline__ void tile_corner(const CornerCtx<C, T> &cx, LDB ldb) {
    constexpr int CPR = 32 / R;
    C xr[KC];
#pragma unroll
    for (int d = 0; d < KC; ++d) xr[d] = C(0);
    // the window's head columns are rows hb[j*bst], its tail columns rows tb[j*bst]
    // (j from 0): batches of JB columns per lane with immediate offsets, the b
    // loads and the Lambda loads of a batch independent of each other
    constexpr int JB = 8;
    auto window = [&](const T *base, const C *lv, int len) {
        base += (int64_t)cx.part * cx.bst;
        lv += cx.part * KC;
        for (int j0 = cx.part; j0 < len; j0 += JB * CPR) {
            C b[JB];
#pragma unroll
            for (int u = 0; u < JB; ++u) b[u] = j0 + u * CPR < len ? (C)base[(int64_t)u * CPR * cx.bst] : C(0);
#pragma unroll
            for (int u = 0; u < JB; ++u)
                if (j0 + u * CPR < len)
#pragma unroll
                    for (int d = 0; d < KC; ++d) xr[d] = fma(-lv[u * CPR * KC + d], b[u], xr[d]);
            base += (int64_t)JB * CPR * cx.bst;
            lv += JB * CPR * KC;
        }
    };
    window(cx.hb, cx.slw, cx.lh);
    window(cx.tb, cx.slw + cx.lh * KC, cx.lw - cx.lh);
#pragma unroll
    for (int d = 0; d < KC; ++d) {
        C acc = xr[d];
#pragma unroll
        for (int off = R; off < 32; off *= 2) acc += __shfl_xor_sync(0xffffffffu, acc, off);
        xr[d] = fma(ldb(cx.sdrow[d]), cx.sdscale[d], acc);
    }
    wgetrs_reg<C, KC>(xr, cx.sdlu, cx.sdpiv, KC);
    if (cx.part == 0 && cx.gout)
#pragma unroll
        for (int d = 0; d < KC; ++d) __stcs(cx.gout + (int64_t)cx.sdrow[d] * cx.ps, (T)xr[d]);
    if (cx.part == 0) {
#pragma unroll
        for (int d = 0; d < KC; ++d) cx.sx1[d * R] = xr[d];
    }
}

// ========================================================= tile kernel
// NV right-hand sides of one row as one vector access
template <typename T, int NV> struct VecN { using type = T; };
template <> struct VecN<double, 2> { using type = double2; };
template <> struct VecN<float, 2> { using type = float2; };
template <> struct VecN<float, 4> { using type = float4; };

// right-hand sides per compute thread of the tile kernel (1: one chain per
// thread; 2/4 were measured slower -- per-segment overheads and carry smem grow)
constexpr int tile_nv(int /*esz*/) { return 1; }

template <typename T, int K, int L, int R, int NV, int LOADER>
__global__ void __launch_bounds__(TILE_MAX_THREADS, 1)
    sb_tile_kernel(const __grid_constant__ KParams p, const __grid_constant__ CUtensorMap tmap,
                   const __grid_constant__ CUtensorMap tmap_c) {
    using C = T;  // compute in the storage precision
    constexpr int CI = sizeof(T) == 8 ? 0 : 1;
    constexpr int CPR = 32 / R;   // corner lanes per RHS
    constexpr int RP = R / NV;    // RHS groups per tile (a thread owns NV adjacent RHS)
    constexpr int SPW = 32 / RP;  // segments per compute warp
    static_assert(NV * (int)sizeof(T) <= 16, "NV RHS form one vector of at most 16 B");
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;
    const DevSeg &G = P.seg[CI];

    const int S = G.S, nQ = P.nQ, k = P.k, s_lo = P.s_lo;
    const int ncw = p.ncw, nbox = p.nbox, boxr = p.boxr;
    // The corner/producer warp runs on hardware warp 0: the warp schedulers favour
    // older warps, and the corner's short dependent chains (x1 for the next tile)
    // must not be starved by the compute warps (as the youngest warp it finished
    // x1 only just before the gamma warps needed it).  Logical numbering: compute
    // warps 0..ncw-1 (hardware warps 1..ncw), corner warp ncw.
    const int hwarp = (int)(threadIdx.x >> 5), lane = (int)(threadIdx.x & 31);
    const int warp = hwarp == 0 ? ncw : hwarp - 1;
    const int tid = warp * 32 + lane;
    constexpr int LP = L + (sizeof(T) == 8 ? 2 : 4);  // factor pitch (capi.cpp upload; checked at launch)
    constexpr int ms = LP;                            // band stride inside a segment's factor block

    C *sF = reinterpret_cast<C *>(smem + p.off_L);  // factor blocks (device.hpp DevSeg)
    C *sG = reinterpret_cast<C *>(smem + p.off_G);
    C *sH = reinterpret_cast<C *>(smem + p.off_H);
    C *sfend = reinterpret_cast<C *>(smem + p.off_fend);
    C *sbbeg = reinterpret_cast<C *>(smem + p.off_bbeg);
    C *sx1 = reinterpret_cast<C *>(smem + p.off_x1);  // [2][R*k]
    const int *slamptr = reinterpret_cast<const int *>(smem + p.off_lamptr);
    const int *slamc = reinterpret_cast<const int *>(smem + p.off_lamc);
    const C *slamv = reinterpret_cast<const C *>(smem + p.off_lamv);
    const C *slw = reinterpret_cast<const C *>(smem + p.off_lw);
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
    uint64_t *cfull = x1full + 2;  // corner boxes, double-buffered (+ [2]: constants staged)
    T *buf = reinterpret_cast<T *>(smem + p.off_buf);
    T *cbuf = reinterpret_cast<T *>(smem + p.off_cbuf);  // [2][2 boxes][cbox rows][R]
    const int cbox = p.cbox;
    const bool use_cbox = LOADER == LOAD_TMA && cbox > 0;
    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    const uint32_t box_bytes = (uint32_t)(boxr * R * sizeof(T));

    if (tid == 0) {
        for (int c = 0; c < nbox; ++c) {
            mbar_init(full + c, 1);
            mbar_init(empty + c, p.empty_count[c]);
        }
        mbar_init(x1full + 0, R);  // every x1-writing corner lane arrives (release of its own writes)
        mbar_init(x1full + 1, R);
        mbar_init(cfull + 0, 1);
        mbar_init(cfull + 1, 1);
        mbar_init(cfull + 2, 1);  // constants staged
        fence_mbar_init();
        if (LOADER == LOAD_TMA) prefetch_tmap(&tmap);
        if (use_cbox) prefetch_tmap(&tmap_c);
        stage_constants_issue<C, K>(p, G, smem, cfull + 2);
    }
    __syncthreads();
    mbar_wait(cfull + 2, 0);

    if (warp == ncw) {
        // ===================== corner + producer warp (runs one tile ahead)
        // The corner of tile t+1 needs only its head/tail rows: they arrive in two
        // small "corner boxes" issued one tile early, so x1(t+1) is ready before
        // the compute warps reach tile t+1 (the main load re-reads those rows from L2).
        const int part = lane / R, rr = lane % R;
        const uint32_t cbytes = (uint32_t)(2 * cbox * R * sizeof(T));
        auto issue_cbox = [&](int t, int b) {
            T *dst = cbuf + (size_t)b * 2 * cbox * R;
            const int sl = t / p.tps, tb = t - sl * p.tps;
            mbar_arrive_expect_tx(cfull + b, cbytes);
            tma_load_3d(dst, &tmap_c, cfull + b, tb * R, 0, sl);
            tma_load_3d(dst + (size_t)cbox * R, &tmap_c, cfull + b, tb * R, P.n - cbox, sl);
        };
        if (use_cbox && lane == 0 && (int)blockIdx.x < p.ntiles) issue_cbox(blockIdx.x, 0);
        int it = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x, ++it) {
            const int slab = tile / p.tps, tb = tile - slab * p.tps;
            T *gs = gout + slab * p.slab_stride;
            SB_TR(0);
            if (LOADER == LOAD_TMA) {
                if (lane == 0) {
                    for (int q = 0; q < nbox; ++q) {
                        const int c = p.box_order[q];  // the corner's boxes first: x1 starts earlier
                        if (it > 0) mbar_wait(empty + c, (it - 1) & 1);
                        mbar_arrive_expect_tx(full + c, box_bytes);
                        tma_load_3d(buf + (size_t)c * boxr * R, &tmap, full + c, tb * R, c * boxr, slab);
                    }
                    if (use_cbox && tile + (int)gridDim.x < p.ntiles) issue_cbox(tile + gridDim.x, (it + 1) & 1);
                }
                // every lane passes lane 0's empty waits: the compute warps have loaded
                // tile it-1, so they are done with tile it-2 and its x1 buffer (it & 1)
                __syncwarp();
                SB_TR(8);
                if (use_cbox) mbar_wait(cfull + (it & 1), (it >> 1) & 1);
                else
                    for (int c = 0; c < nbox; ++c)
                        if ((p.corner_need_mask >> c) & 1) mbar_wait(full + c, it & 1);
            } else if (it > 0) {
                mbar_wait(empty + 0, (it - 1) & 1);  // all compute warps finished tile it-1
            }
            SB_TR(2);
            const T *cb = cbuf + (size_t)(it & 1) * 2 * cbox * R;
            const int64_t ccol = (int64_t)tb * R + rr;
            const bool clive = ccol < p.batch;
            const T *ccolp = gs + ccol * p.bstride;
            auto ldb = [&](int row) -> C {
                if (LOADER == LOAD_TMA) {
                    if (use_cbox) return (C)cb[(size_t)(row < cbox ? row : cbox + row - (P.n - cbox)) * R + rr];
                    return (C)buf[(size_t)row * R + rr];
                }
                return clive ? (C)ccolp[(int64_t)row * ps] : C(0);
            };
            CornerCtx<C, T> cx;
            cx.part = part; cx.lh = P.lw_head; cx.lw = P.lw_head + P.lw_tail;
            cx.slw = slw; cx.sdlu = sdlu; cx.sdscale = sdscale; cx.sdrow = sdrow; cx.sdpiv = sdpiv;
            cx.sx1 = sx1 + (it & 1) * R * k + rr;  // [d][rhs]: consecutive lanes, consecutive banks
            cx.gout = clive ? gs + ccol * p.bstride : nullptr; cx.ps = ps;
            {   // where the window rows of this RHS live: corner boxes, main tile or HBM
                const int hr = s_lo, tr = s_lo + nQ - P.lw_tail;  // first rows of head / tail windows
                if (LOADER == LOAD_TMA) {
                    cx.bst = R;
                    if (use_cbox) {
                        cx.hb = cb + (size_t)hr * R + rr;
                        cx.tb = cb + (size_t)(cbox + tr - (P.n - cbox)) * R + rr;
                    } else {
                        cx.hb = buf + (size_t)hr * R + rr;
                        cx.tb = buf + (size_t)tr * R + rr;
                    }
                } else {
                    cx.bst = clive ? ps : 0;  // beyond the batch: read row 0 of column 0, times 0
                    cx.hb = clive ? ccolp + (int64_t)hr * ps : gout;
                    cx.tb = clive ? ccolp + (int64_t)tr * ps : gout;
                }
            }
            if (k >= 1 && k <= WCORNER_KREG) {
                // x1 in registers with k a compile-time constant (every instruction of the
                // corner warp costs ~4 issue cycles next to the compute warps)
                switch (k) {
                    case 1: tile_corner<C, T, 1, R>(cx, ldb); break;
                    case 2: tile_corner<C, T, 2, R>(cx, ldb); break;
                    case 3: tile_corner<C, T, 3, R>(cx, ldb); break;
                    case 4: tile_corner<C, T, 4, R>(cx, ldb); break;
                    case 5: tile_corner<C, T, 5, R>(cx, ldb); break;
                    case 6: tile_corner<C, T, 6, R>(cx, ldb); break;
                    case 7: tile_corner<C, T, 7, R>(cx, ldb); break;
                    default: tile_corner<C, T, 8, R>(cx, ldb); break;
                }
            } else if (k > 0) {
                // k > 8 (rare): CSR spmv and getrs through shared memory
                C *x1 = sx1 + (it & 1) * R * k + rr * k;
                for (int d = 0; d < k; ++d) {
                    C acc = part == 0 ? ldb(sdrow[d]) * sdscale[d] : C(0);
                    for (int e = slamptr[d] + part; e < slamptr[d + 1]; e += CPR)
                        acc = fma(-slamv[e], ldb(s_lo + slamc[e]), acc);
#pragma unroll
                    for (int off = R; off < 32; off *= 2) acc += __shfl_xor_sync(0xffffffffu, acc, off);
                    if (part == 0) x1[d] = acc;
                }
                SB_TR(3);
                if (part == 0) {
                    getrs_small(x1, sdlu, sdpiv, k);
                    if (clive)
                        for (int d = 0; d < k; ++d) __stcs(gs + ccol * p.bstride + (int64_t)sdrow[d] * ps, (T)x1[d]);
                }
            }
            SB_TR(1);
            __syncwarp();
            if (part == 0) mbar_arrive(x1full + (it & 1));
            if (lane == 0) {
                if (LOADER == LOAD_TMA)
                    for (int c = 0; c < nbox; ++c)
                        if ((p.corner_arrive_mask >> c) & 1) mbar_arrive(empty + c);
            }
        }
        return;
    }

    // ============================================== compute warps
    using V = typename VecN<T, NV>::type;
    const int rp = tid % RP;
    const int s = tid / RP;
    const int r0 = rp * NV;  // first of this thread's NV right-hand sides in the tile
    const bool active = s < S;
    const int a = s * L;
    const bool full_seg = a + L <= nQ;
    const int sc = G.slot[active ? s : 0];  // factor block (idle threads alias segment 0)
    const C *fL = sF + sc * (2 * K + 1) * LP;  // one base register; bands at immediate offsets
    const C *fU = fL + K * LP;
    const C *fD = fL + 2 * K * LP;
    // boxes this warp reads (rows of its real segments)
    int c_lo = 0, c_hi = -1;
    {
        const int s0 = warp * SPW;
        const int rr0 = s_lo + s0 * L;
        const int rr1 = s_lo + min((s0 + SPW) * L, nQ) - 1;
        if (s0 < S && rr1 >= rr0) {
            c_lo = rr0 / boxr;
            c_hi = rr1 / boxr;
        }
    }
    int it = 0;
    for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x, ++it) {
        const int slab = tile / p.tps;
        const int64_t col0 = (int64_t)(tile - slab * p.tps) * R + r0;
        // right-hand sides of this thread that exist (0..NV)
        const int nlive = active ? (int)max((int64_t)0, min((int64_t)NV, p.batch - col0)) : 0;
        T *gcol = gout + slab * p.slab_stride + col0 * p.bstride;
        C v[L][NV];
        SB_TR(0);
        // ---------- own segment of b0 into registers
        if (LOADER == LOAD_TMA) {
            for (int c = c_lo; c <= c_hi; ++c) mbar_wait(full + c, it & 1);
            SB_TR(8);
            // one predicated path for full and partial segments (no divergence in the
            // warp that holds the last, partial segment)
            const T *src = buf + (size_t)(s_lo + a) * R + r0;
#pragma unroll
            for (int i = 0; i < L; ++i) {
                V w;
                if (full_seg || (active && a + i < nQ)) w = *reinterpret_cast<const V *>(src + (size_t)i * R);
                else w = V{};
                const T *pw = reinterpret_cast<const T *>(&w);
#pragma unroll
                for (int q = 0; q < NV; ++q) v[i][q] = (C)pw[q];
            }
            __syncwarp();
            if (lane == 0)
                for (int c = c_lo; c <= c_hi; ++c) mbar_arrive(empty + c);
        } else {
            const T *src = gcol + (int64_t)(s_lo + a) * ps;
#pragma unroll
            for (int i = 0; i < L; ++i)
#pragma unroll
                for (int q = 0; q < NV; ++q)
                    v[i][q] = (q < nlive && a + i < nQ) ? (C)__ldcs(src + (int64_t)i * ps + q * p.bstride) : C(0);
        }
        SB_TR(1);
        // ---------- b0 -= gamma x1 (only segments holding gamma rows wait for the corner warp)
        if (active && sgptr[s] < sgptr[s + 1]) {
            mbar_wait(x1full + (it & 1), (it >> 1) & 1);
            // x1 order: [d][rhs] from the register corner (k <= 8, conflict-free), [rhs][d]
            // from the shared-memory corner (k > 8)
            const int xsr = k <= WCORNER_KREG ? 1 : k, xsd = k <= WCORNER_KREG ? R : 1;
            const C *x1 = sx1 + (it & 1) * R * k + r0 * xsr;
            for (int e = sgptr[s]; e < sgptr[s + 1]; ++e) {
                const int i = sgamr[e] - a;
                const int dc = sgamc[e];
                const C gv = sgamv[e];
#pragma unroll
                for (int j = 0; j < L; ++j)
                    if (j == i)
#pragma unroll
                        for (int q = 0; q < NV; ++q) v[j][q] = fma(-gv, x1[q * xsr + dc * xsd], v[j][q]);
            }
        }
        SB_TR(2);
        // ---------- local forward sweep, publish end state
        C st[K][NV];
        fwd_local<C, K, L, NV, true>(v, fL, ms, st);
        // end states in SoA order [j][segment][rhs]: consecutive lanes hit consecutive banks
        if (active)
#pragma unroll
            for (int q = 0; q < NV; ++q)
#pragma unroll
                for (int j = 0; j < K; ++j) sfend[(j * S + s) * R + r0 + q] = st[j][q];
        SB_TR(3);
        named_bar(1, ncw * 32);  // B2: every local forward end state is published
        SB_TR(4);
        // ---------- forward carry (true y at rows a-1..a-K) + correction chain
        if (active && s > 0) {
            C cin[K][NV];
#pragma unroll
            for (int m = 0; m < K; ++m)
#pragma unroll
                for (int q = 0; q < NV; ++q) cin[m][q] = C(0);
            for (int t = max(0, s - G.carry_f); t < s; ++t) {
                C nw[K][NV];
#pragma unroll
                for (int j = 0; j < K; ++j)
#pragma unroll
                    for (int q = 0; q < NV; ++q) {
                        C acc = sfend[(j * S + t) * R + r0 + q];
#pragma unroll
                        for (int m = 0; m < K; ++m) acc = fma(sG[(t * K + j) * K + m], cin[m][q], acc);
                        nw[j][q] = acc;
                    }
#pragma unroll
                for (int j = 0; j < K; ++j)
#pragma unroll
                    for (int q = 0; q < NV; ++q) cin[j][q] = nw[j][q];
            }
            fwd_correct<C, K, L, NV, true>(v, fL, ms, cin);
        }
        // ---------- local backward sweep, publish begin state
        bwd_local<C, K, L, NV, true>(v, fU, fD, ms, st);
        if (active)
#pragma unroll
            for (int q = 0; q < NV; ++q)
#pragma unroll
                for (int j = 0; j < K; ++j) sbbeg[(j * S + s) * R + r0 + q] = st[j][q];
        SB_TR(5);
        named_bar(1, ncw * 32);  // B3: every local backward begin state is published
        SB_TR(6);
        // ---------- backward carry (true x at rows a+L..a+L+K-1) + correction chain
        // TMA path: every row is stored from inside the chain as soon as it is final
        // (the last segment runs the chain with zero carries, so there is one store
        // path).  Measured: C3 Greville 0.403 -> 0.380 ms, Hermite 0.335 -> 0.326 ms
        // (round 1); band K = 1 took the burst after the chain until the round-2
        // kernel, where the fused stores won too (C2 0.2888 -> 0.2866 ms, C4M 0.3752 ->
        // 0.3724 ms, profiles/r02/ab_experiments.md).
        constexpr bool FUSED = LOADER == LOAD_TMA && NV == 1;
        if (active && (FUSED || s < S - 1)) {
            C co[K][NV];
#pragma unroll
            for (int m = 0; m < K; ++m)
#pragma unroll
                for (int q = 0; q < NV; ++q) co[m][q] = C(0);
            for (int t = min(S - 1, s + G.carry_b); t > s; --t) {
                C nw[K][NV];
#pragma unroll
                for (int j = 0; j < K; ++j)
#pragma unroll
                    for (int q = 0; q < NV; ++q) {
                        C acc = sbbeg[(j * S + t) * R + r0 + q];
#pragma unroll
                        for (int m = 0; m < K; ++m) acc = fma(sH[(t * K + j) * K + m], co[m][q], acc);
                        nw[j][q] = acc;
                    }
#pragma unroll
                for (int j = 0; j < K; ++j)
#pragma unroll
                    for (int q = 0; q < NV; ++q) co[j][q] = nw[j][q];
            }
            if constexpr (FUSED) {
                // one code path for every segment (a full and the partial last segment
                // share warp 13: two instantiations would run one after the other)
                T *dlast = gcol + (int64_t)(s_lo + a + L - 1) * ps;
                const int nvalid = nlive > 0 ? min(L, nQ - a) : 0;
                bwd_correct<C, K, L, NV, true, true, true, T>(v, fU, ms, co, dlast, ps, nvalid);
            } else
                bwd_correct<C, K, L, NV, true>(v, fU, ms, co);
        }
        // ---------- store x0 straight from registers (one 16-B vector per row).
        // DIRECT mode: the corner warp reads b0 from HBM, so no row of this tile is
        // overwritten before x1 is done.
        if (LOADER == LOAD_DIRECT && k > 0) mbar_wait(x1full + (it & 1), (it >> 1) & 1);
        if (!FUSED && nlive > 0) {
            // one predicated path for full and partial segments (no divergence in the
            // warp that holds the last, partial segment); running row pointer
            T *dst = gcol + (int64_t)(s_lo + a) * ps;
            if (LOADER == LOAD_TMA && nlive == NV) {
#pragma unroll
                for (int i = 0; i < L; ++i) {
                    V w;
                    T *pw = reinterpret_cast<T *>(&w);
#pragma unroll
                    for (int q = 0; q < NV; ++q) pw[q] = (T)v[i][q];
                    if (full_seg || a + i < nQ) __stcs(reinterpret_cast<V *>(dst), w);
                    dst += ps;
                }
            } else {
#pragma unroll
                for (int i = 0; i < L; ++i) {
#pragma unroll
                    for (int q = 0; q < NV; ++q)
                        if (q < nlive && a + i < nQ) __stcs(dst + q * p.bstride, (T)v[i][q]);
                    dst += ps;
                }
            }
        }
        SB_TR(7);
        if (LOADER == LOAD_DIRECT) {  // tile done: lets the corner warp move to tile it+1
            __syncwarp();
            if (lane == 0) mbar_arrive(empty + 0);
        }
    }
}

// ========================================================= warp kernel
// One warp per RHS; lane s owns segment s (rows [s*L, s*L+L) of Q).
// BULK: rows are contiguous and 16-B aligned -- lane 0 moves a whole row with
// one cp.async.bulk (global->smem, mbarrier complete_tx) into one of two
// per-warp row buffers, so the next row streams in while this one is solved,
// and writes the result back with one bulk smem->global copy.
// Algorithm 2's interpolation at the feet of the characteristics (PAPER.md
// P:157-163): out[i] = S(xi_i - shift) for the periodic spline S with
// coefficients coef[0..N) just solved for.  The p+1 nonzero B-splines at a
// point come from de Boor's triangular scheme (BSPLVB) with
// dl[j] = x - t_{c-j}, dr[j] = t_{c+1+j} - x; basis j of the centred periodic
// space has its first knot at j - s, s = floor((p+1)/2), so the value is
// sum_r b[r] coef[(c - p + r + s) mod N].
template <int PD>
__device__ __forceinline__ void bspl_values(const double (&dl)[PD], const double (&dr)[PD], double (&b)[PD + 1]) {
    b[0] = 1.0;
#pragma unroll
    for (int j = 0; j < PD; ++j) {
        double saved = 0.0;
#pragma unroll
        for (int r = 0; r <= j; ++r) {
            const double term = b[r] / (dr[r] + dl[j - r]);
            b[r] = saved + dr[r] * term;
            saved = dl[j - r] * term;
        }
        b[j + 1] = saved;
    }
}

// Non-uniform periodic evaluation at a foot x in cell c (Algorithm 2's
// interpolation step): de Boor's triangular recursion (BSPLVB) with the
// denominators t_{c+1+r} - t_{c-j+r} replaced by precomputed reciprocals, so
// no division; knots, reciprocals and the p+1 coefficients come straight from
// shared memory through two base pointers (immediate offsets).  The
// coefficients are coef[(c-p+s+r) mod N]; the row is padded on both sides
// (coef[-2..-1] = coef[N-2..N-1], coef[N..N+2] = coef[0..2]), so no wrap.
template <typename C, int PD>
__device__ __forceinline__ C nu_value(double x, int c, const double *xe, const C *coef, const double *rc) {
    constexpr int s = (PD + 1) / 2;
    const double *tk = xe + c;       // tk[q] = t_{c+q}
    constexpr int RS = PD | 1;       // odd row stride of the reciprocal table (bank-conflict free)
    const double *rk = rc + c * RS;  // rk[m*RS + w-1] = 1/(t_{c+m+w} - t_{c+m})
    double b[PD + 1];
    b[0] = 1.0;
#pragma unroll
    for (int j = 0; j < PD; ++j) {
        double saved = 0.0;
#pragma unroll
        for (int r = 0; r <= j; ++r) {
            // (computing the reciprocals with __drcp_rn instead of loading them,
            // -48 B of shared traffic per point, measured 1.32 vs 1.02 ms for ADVNU)
            const double term = b[r] * rk[(r - j) * RS + j];  // 1/(t_{c+1+r} - t_{c-j+r})
            b[r] = fma(tk[1 + r] - x, term, saved);
            saved = (x - tk[r - j]) * term;
        }
        b[j + 1] = saved;
    }
    const C *cw = coef + (c - PD + s);
    C acc = C(0);
#pragma unroll
    for (int r = 0; r <= PD; ++r) acc = fma((C)b[r], cw[r], acc);
    return acc;
}

// One row of the advection step, uniform mesh: every foot xi_i - shift has
// the same local coordinate u, so the p+1 weights are computed once per row
// and out[i] = sum_r w_r coef[(i+off+r) mod N] is a (p+1)-tap stencil.  Lanes
// take consecutive points (conflict-free shared loads; the row is padded past
// N by the periodic wrap) and store straight to HBM, coalesced.
template <typename C, typename T, int PD>
__device__ __forceinline__ void advect_row(const DevPlan &P, const C *coef, T *g, int64_t ps, double sh, int lane) {
    constexpr int s = (PD + 1) / 2;
    const int N = P.N;
    const double q = P.adv_q0 - sh * P.adv_invh;  // foot of point 0, in cells from x_0
    const double cf = floor(q);
    double dl[PD], dr[PD], b[PD + 1];
#pragma unroll
    for (int j = 0; j < PD; ++j) {
        dl[j] = (q - cf) + j;
        dr[j] = (j + 1) - (q - cf);
    }
    bspl_values<PD>(dl, dr, b);
    C w[PD + 1];
#pragma unroll
    for (int r = 0; r <= PD; ++r) w[r] = (C)b[r];
    int c0 = (int)(cf - (double)N * floor(cf / (double)N));
    c0 = c0 >= N ? c0 - N : (c0 < 0 ? c0 + N : c0);
    int off = c0 - PD + s;  // point i reads coef[i + off .. i + off + PD] (mod N)
    off = off < 0 ? off + N : (off >= N ? off - N : off);
#pragma unroll 4
    for (int i = lane; i < N; i += 32) {
        int idx = i + off;
        idx -= idx >= N ? N : 0;
        const C *cw = coef + idx;
        C acc = C(0);
#pragma unroll
        for (int r = 0; r <= PD; ++r) acc = fma(w[r], cw[r], acc);
        __stcs(g + (int64_t)i * ps, (T)acc);
    }
}

// Non-uniform mesh: lanes take consecutive points (j = lane + 32u, two per
// iteration for ILP); the foot's cell comes from a bucket table (bucket width
// <= the smallest cell, so at most one step to correct) and nu_value
// evaluates the p+1 B-splines there.  Results go straight to HBM, coalesced
// (the row is on chip, so the in-place write is safe): no output buffer.
template <typename C, typename T, int PD>
__device__ __forceinline__ void advect_row_nu(const DevPlan &P, const double *sgeo, const C *coef, T *g,
                                              int64_t ps, double sh, int lane) {
    const int N = P.N;
    const GeoLayout gl(P);
    const double *xe = sgeo + PD;                  // xe[c] = t_c, c in [-PD, N+PD]
    const double *xi = sgeo + gl.o_xi;             // interpolation points (n = N)
    const double *rc = sgeo + gl.o_rc + PD * (PD | 1);  // rc[m*(PD|1) + w-1] = 1/(t_{m+w} - t_m), m in [-PD, N+PD)
    const int *tbl = reinterpret_cast<const int *>(sgeo + gl.o_tbl);
    const int MT = P.adv_nbkt;
    const double x0 = xe[0], xN = xe[N], Lp = xN - x0, invLp = 1.0 / Lp, bscale = P.adv_bscale;
    double shr = sh - floor(sh * invLp) * Lp;  // sh mod L, in [0, L)
    if (shr >= Lp) shr -= Lp;
    if (shr < 0.0) shr += Lp;
    const int nsteps = P.adv_steps;
    auto locate = [&](double x) {  // t_c <= x < t_{c+1}: bucket, then nsteps branch-free steps
        int c = tbl[min(max((int)((x - x0) * bscale), 0), MT - 1)];
        for (int q = 0; q < nsteps; ++q) c += (x >= xe[c + 1]);
        return c;
    };
    // feet: xi_j in [x_0, x_N), shr in [0, L) -> one conditional wrap (x_N itself maps to x_0)
    auto foot = [&](int j) {
        double x = xi[j] - shr;
        if (x < x0) x += Lp;
        if (x >= xN) x -= Lp;
        return x;
    };
    // software pipeline: the cells of the next pair of points are located while
    // the current pair is evaluated
    int j0 = lane;
    double xa = foot(min(j0, N - 1)), xb = foot(min(j0 + 32, N - 1));
    int ca = locate(xa), cb = locate(xb);
    for (; j0 < N; j0 += 64) {
        const int j1 = j0 + 32, jn = j0 + 64;
        const double xan = foot(min(jn, N - 1)), xbn = foot(min(jn + 32, N - 1));
        const int can = locate(xan), cbn = locate(xbn);
        const C ya = nu_value<C, PD>(xa, ca, xe, coef, rc);
        const C yb = nu_value<C, PD>(xb, cb, xe, coef, rc);
        __stcs(g + (int64_t)j0 * ps, (T)ya);
        if (j1 < N) __stcs(g + (int64_t)j1 * ps, (T)yb);
        xa = xan; xb = xbn; ca = can; cb = cbn;
    }
}

template <typename T, int K, int L, bool BULK, bool ADV>
__global__ void __launch_bounds__(32 * WARP_MAX_WARPS)
    sb_warp_kernel(const __grid_constant__ KParams p) {
    using C = T;
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;
    const DevSeg &G = P.seg[2];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int S = G.S, nQ = P.nQ, k = P.k, s_lo = P.s_lo, n = P.n;
    constexpr int LP = L;  // odd factor pitch (conflict-free across the 32 lanes' segments)
    constexpr int ms = LP;
    const int nwarps = blockDim.x >> 5;

    uint64_t *wbar = reinterpret_cast<uint64_t *>(smem + p.off_mbar) + 2 * warp;  // 2 per warp
    uint64_t *cbar = reinterpret_cast<uint64_t *>(smem + p.off_mbar) + 2 * WARP_MAX_WARPS;  // constants staged
    if (BULK && lane == 0) {
        mbar_init(wbar, 1);
        mbar_init(wbar + 1, 1);
        fence_mbar_init();
    }
    if (tid == 0) {
        mbar_init(cbar, 1);
        fence_mbar_init();
        stage_constants_issue<C, K>(p, G, smem, cbar);
    }
    // advect, non-uniform geometry (GeoLayout): xe | xi | rcp | bucket table
    const double *sgeo = reinterpret_cast<const double *>(smem + p.off_geo);
    __syncthreads();
    mbar_wait(cbar, 0);

    const C *sF = reinterpret_cast<const C *>(smem + p.off_L);
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
    // per warp: row buffer(s) of WB_FRONT pad + n values + k spare for x1 (the
    // advection pads the row on both sides with the periodic wrap)
    C *wbuf = reinterpret_cast<C *>(smem + p.off_buf) + (size_t)warp * (BULK ? 2 : 1) * p.wbuf_pitch + WB_FRONT;

    const int s = lane;
    const bool active = s < S;
    const int a = s * L;
    const int slot = G.slot[active ? s : 0];  // identical segments share (and broadcast) one block
    const C *fL = sF + slot * (2 * K + 1) * LP;
    const C *fU = fL + K * LP;
    const C *fD = fL + 2 * K * LP;
    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    const bool vec = (ps == 1) && ((p.bstride * (int64_t)sizeof(T)) % 16 == 0) &&
                     ((uintptr_t)p.rhs % 16 == 0) && (n % (16 / (int)sizeof(T)) == 0);
    constexpr int VW = 16 / sizeof(T);  // elements per 16-B vector
    using V = typename std::conditional<sizeof(T) == 8, double2, float4>::type;
    const uint32_t row_bytes = (uint32_t)(n * sizeof(T));

    const int64_t gw = (int64_t)blockIdx.x * nwarps + warp;
    const int64_t nw = (int64_t)gridDim.x * nwarps;
    if (BULK && lane == 0)
        for (int b = 0; b < 2; ++b) {
            const int64_t r = gw + b * nw;
            if (r < p.batch) {
                mbar_arrive_expect_tx(wbar + b, row_bytes);
                bulk_load(wbuf + (size_t)b * p.wbuf_pitch, gout + r * p.bstride, row_bytes, wbar + b);
            }
        }
    int j = 0;
    for (int64_t rhs = gw; rhs < p.batch; rhs += nw, ++j) {
        T *g = gout + rhs * p.bstride;
        C *rowbuf = wbuf + (BULK ? (size_t)(j & 1) * p.wbuf_pitch : 0);
        C *x1 = rowbuf + n;  // k values after the row
        // ---------- the whole row into shared memory
        if (BULK) {
            mbar_wait(wbar + (j & 1), (j >> 1) & 1);
        } else if (vec) {
            const V *gv = reinterpret_cast<const V *>(g);
            V *sv = reinterpret_cast<V *>(rowbuf);  // C == T: whole 16-B vectors, conflict-free
            for (int q = lane; q < n / VW; q += 32) sv[q] = __ldcs(gv + q);
            __syncwarp();
        } else {
            for (int q = lane; q < n; q += 32) rowbuf[q] = (C)__ldcs(g + (int64_t)q * ps);
            __syncwarp();
        }
        // ---------- corner: x1 = delta'^{-1} (s1*b1 - Lambda b0), then b0 -= gamma x1
        // fp64 solve: x1 in registers on every lane (the xor reduction leaves the
        // sum on all lanes), getrs on registers, then gamma row by row on parallel
        // lanes -- no serial chain of dependent shared-memory round trips on lane 0
        // (measured: C4 fp64 0.383 -> 0.352 ms, C6 0.389 -> 0.379 ms; the same code
        // made the fp32 solve and the advection step slower, 0.182 -> 0.211 and
        // 0.385 -> 0.460 ms, so they keep the lane-0 corner)
        constexpr bool REG_CORNER = sizeof(T) == 8 && !ADV;
        if (REG_CORNER && k > 0 && k <= WCORNER_KREG) {
            C xr[WCORNER_KREG];
#pragma unroll
            for (int d = 0; d < WCORNER_KREG; ++d) {
                C acc = C(0);
                if (d < k) {
                    acc = lane == 0 ? rowbuf[sdrow[d]] * sdscale[d] : C(0);
                    for (int e = slamptr[d] + lane; e < slamptr[d + 1]; e += 32)
                        acc = fma(-slamv[e], rowbuf[s_lo + slamc[e]], acc);
#pragma unroll
                    for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
                }
                xr[d] = acc;
            }
            wgetrs_reg<C, WCORNER_KREG>(xr, sdlu, sdpiv, k);
            auto xsel = [&](int c) {
                C r = xr[0];
#pragma unroll
                for (int j = 1; j < WCORNER_KREG; ++j) r = j == c ? xr[j] : r;
                return r;
            };
            __syncwarp();  // every lane has read its Lambda columns and delta rows of the row buffer
            for (int e = lane; e < P.gam_nnz; e += 32) {
                const int row = sgamr[e];
                if (e > 0 && sgamr[e - 1] == row) continue;  // the lane of the row's first entry does the row
                C val = rowbuf[s_lo + row];
                for (int f = e; f < P.gam_nnz && sgamr[f] == row; ++f) val -= sgamv[f] * xsel(sgamc[f]);
                rowbuf[s_lo + row] = val;
            }
            if (lane < k) rowbuf[sdrow[lane]] = xsel(lane);
            __syncwarp();
        } else if (k > 0) {
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
        C v[L][1];
#pragma unroll
        for (int i = 0; i < L; ++i) v[i][0] = (active && a + i < nQ) ? rowbuf[s_lo + a + i] : C(0);
        // ---------- forward: local sweep, carry by shuffles, correction chain
        C st[K][1];
        fwd_local<C, K, L, 1, false>(v, fL, ms, st);
        {
            C cin[K][1];
#pragma unroll
            for (int m = 0; m < K; ++m) cin[m][0] = C(0);
            for (int w = G.carry_f; w >= 1; --w) {  // from segment s-w up to s-1
                const int t = s - w;
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = __shfl_up_sync(0xffffffffu, st[j][0], w);
                    if (t >= 0)
#pragma unroll
                        for (int m = 0; m < K; ++m) acc = fma(sG[(j * K + m) * S + t], cin[m][0], acc);
                    nw[j] = t >= 0 ? acc : C(0);
                }
#pragma unroll
                for (int j = 0; j < K; ++j) cin[j][0] = nw[j];
            }
            if (active && s > 0) fwd_correct<C, K, L, 1, false>(v, fL, ms, cin);
        }
        // ---------- backward: local sweep, carry by shuffles, correction chain
        bwd_local<C, K, L, 1, false>(v, fU, fD, ms, st);
        {
            C co[K][1];
#pragma unroll
            for (int m = 0; m < K; ++m) co[m][0] = C(0);
            for (int w = G.carry_b; w >= 1; --w) {  // from segment s+w down to s+1
                const int t = s + w;
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    C acc = __shfl_down_sync(0xffffffffu, st[j][0], w);
                    if (t < S)
#pragma unroll
                        for (int m = 0; m < K; ++m) acc = fma(sH[(j * K + m) * S + t], co[m][0], acc);
                    nw[j] = t < S ? acc : C(0);
                }
#pragma unroll
                for (int j = 0; j < K; ++j) co[j][0] = nw[j];
            }
            if (active && s < S - 1) bwd_correct<C, K, L, 1, false>(v, fU, ms, co);
        }
        // ---------- back to the row buffer, then to HBM
#pragma unroll
        for (int i = 0; i < L; ++i)
            if (active && a + i < nQ) rowbuf[s_lo + a + i] = v[i][0];
        C *res = rowbuf;  // row that goes back to HBM
        bool direct = false;  // the result was written to HBM by the evaluation itself
        if (ADV) {
            // ---------- Algorithm 2: f(xi_i) <- S(xi_i - shift) while the coefficients are on chip
            const double sh = p.shift[rhs];
            // wrap pads: rowbuf[-2..-1] = rowbuf[n-2..n-1], rowbuf[n..n+4] = rowbuf[0..4] (mod n)
            __syncwarp();
            if (lane < 2) rowbuf[lane - 2] = rowbuf[n - 1 - ((1 - lane) % n)];
            else if (lane < 7) rowbuf[n + lane - 2] = rowbuf[(lane - 2) % n];
            __syncwarp();
            if (P.adv_uniform) {
                switch (P.p) {  // degrees 1..5 (the library's range)
                    case 1: advect_row<C, T, 1>(P, rowbuf, g, ps, sh, lane); break;
                    case 2: advect_row<C, T, 2>(P, rowbuf, g, ps, sh, lane); break;
                    case 3: advect_row<C, T, 3>(P, rowbuf, g, ps, sh, lane); break;
                    case 4: advect_row<C, T, 4>(P, rowbuf, g, ps, sh, lane); break;
                    default: advect_row<C, T, 5>(P, rowbuf, g, ps, sh, lane); break;
                }
            } else {
                switch (P.p) {
                    case 1: advect_row_nu<C, T, 1>(P, sgeo, rowbuf, g, ps, sh, lane); break;
                    case 2: advect_row_nu<C, T, 2>(P, sgeo, rowbuf, g, ps, sh, lane); break;
                    case 3: advect_row_nu<C, T, 3>(P, sgeo, rowbuf, g, ps, sh, lane); break;
                    case 4: advect_row_nu<C, T, 4>(P, sgeo, rowbuf, g, ps, sh, lane); break;
                    default: advect_row_nu<C, T, 5>(P, sgeo, rowbuf, g, ps, sh, lane); break;
                }
            }
            direct = true;
        }
        if (BULK && direct) {
            __syncwarp();  // every lane is done reading this row buffer
            if (lane == 0) {
                const int64_t nr = rhs + 2 * nw;
                if (nr < p.batch) {
                    fence_proxy_async_smem();  // generic reads before the async refill
                    mbar_arrive_expect_tx(wbar + (j & 1), row_bytes);
                    bulk_load(rowbuf, gout + nr * p.bstride, row_bytes, wbar + (j & 1));
                }
            }
            __syncwarp();
        } else if (direct) {
            __syncwarp();
        } else if (BULK) {
            fence_proxy_async_smem();  // generic smem writes -> visible to the bulk copy
            __syncwarp();
            if (lane == 0) {
                bulk_store(g, res, row_bytes);
                const int64_t nr = rhs + 2 * nw;  // next row for this buffer
                if (ADV || nr < p.batch) bulk_wait_read();  // the store has read its source row
                if (nr < p.batch) {
                    mbar_arrive_expect_tx(wbar + (j & 1), row_bytes);
                    bulk_load(rowbuf, gout + nr * p.bstride, row_bytes, wbar + (j & 1));
                }
            }
            __syncwarp();
        } else if (vec) {
            __syncwarp();
            V *gv = reinterpret_cast<V *>(g);
            const V *sv = reinterpret_cast<const V *>(res);
            for (int q = lane; q < n / VW; q += 32) __stcs(gv + q, sv[q]);
            __syncwarp();
        } else {
            __syncwarp();
            for (int q = lane; q < n; q += 32) __stcs(g + (int64_t)q * ps, (T)res[q]);
            __syncwarp();
        }
    }
    if (BULK && lane == 0) bulk_wait_all();
}

// ========================================================= serial fallback
// One thread per RHS walks all n rows in global memory (the paper's fused
// Listing 6 structure): any n, any strides.  Used only when the
// register-segment kernels do not apply (Q longer than 32 x 63 rows).
template <typename T, int K>
__global__ void __launch_bounds__(128)
    sb_serial_kernel(const __grid_constant__ KParams p) {
    using C = T;
    constexpr int CI = sizeof(T) == 8 ? 0 : 1;
    constexpr int RW = 2 * K + 1;
    const DevPlan &P = p.P;
    const int nQ = P.nQ, k = P.k, s_lo = P.s_lo;
    const C *rowf = reinterpret_cast<const C *>(P.rowf[CI]);
    const C *lamv = reinterpret_cast<const C *>(P.lam_v[CI]);
    const C *gamv = reinterpret_cast<const C *>(P.gam_v[CI]);
    const C *dlu = reinterpret_cast<const C *>(P.dlu[CI]);
    const C *dscale = reinterpret_cast<const C *>(P.dscale[CI]);
    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    C x1[32];
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < p.batch; r += (int64_t)gridDim.x * blockDim.x) {
        T *g = gout + r * p.bstride;
        T *q0 = g + (int64_t)s_lo * ps;
        // corner: x1 = delta'^-1 (s1 b1 - Lambda b0);  b0 -= gamma x1
        for (int d = 0; d < k; ++d) {
            C acc = (C)g[(int64_t)P.drow[d] * ps] * dscale[d];
            for (int e = P.lam_ptr[d]; e < P.lam_ptr[d + 1]; ++e) acc = fma(-lamv[e], (C)q0[(int64_t)P.lam_c[e] * ps], acc);
            x1[d] = acc;
        }
        if (k > 0) getrs_small(x1, dlu, P.dpiv, k);
        for (int e = 0; e < P.gam_nnz; ++e) {
            T *q = q0 + (int64_t)P.gam_r[e] * ps;
            *q = (T)((C)*q - gamv[e] * x1[P.gam_c[e]]);
        }
        // forward sweep in place: y_i = b_i - sum_m L(i,i-1-m) y_{i-1-m}
        C st[K];
#pragma unroll
        for (int m = 0; m < K; ++m) st[m] = C(0);
        for (int i = 0; i < nQ; ++i) {
            const C *f = rowf + (size_t)i * RW;
            C acc = (C)q0[(int64_t)i * ps];
#pragma unroll
            for (int m = K - 1; m >= 0; --m) acc = fma(-__ldg(f + m), st[m], acc);
#pragma unroll
            for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
            st[0] = acc;
            q0[(int64_t)i * ps] = (T)acc;
        }
        // backward sweep in place: x_i = y_i dinv_i - sum_m U'(i,i+1+m) x_{i+1+m}
#pragma unroll
        for (int m = 0; m < K; ++m) st[m] = C(0);
        for (int i = nQ - 1; i >= 0; --i) {
            const C *f = rowf + (size_t)i * RW;
            C acc = (C)q0[(int64_t)i * ps] * __ldg(f + 2 * K);
#pragma unroll
            for (int m = K - 1; m >= 0; --m) acc = fma(-__ldg(f + K + m), st[m], acc);
#pragma unroll
            for (int m = K - 1; m > 0; --m) st[m] = st[m - 1];
            st[0] = acc;
            q0[(int64_t)i * ps] = (T)acc;
        }
        for (int d = 0; d < k; ++d) g[(int64_t)P.drow[d] * ps] = (T)x1[d];
    }
}

}  // namespace sb

namespace sb {
// per-TU launchers (tile_f64.cu, tile_f32.cu, warp_f64.cu, warp_f32.cu)
int launch_tile_f64(int R, int loader, int K, const KParams &kp, const CUtensorMap *tm, int grid, int threads,
                    cudaStream_t st, char *err, int errlen);
int launch_tile_f32(int R, int loader, int K, const KParams &kp, const CUtensorMap *tm, int grid, int threads,
                    cudaStream_t st, char *err, int errlen);
int launch_warp_f64(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);
int launch_warp_f32(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);
int launch_warp_adv_f64(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);
int launch_warp_adv_f32(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);
int launch_serial(int dtype, int K, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen);

// Raise a kernel's dynamic shared-memory limit once per device (the attribute
// call costs microseconds; small batches are launch-bound).  The limit is set
// to the device maximum, which every launch's smem_total respects.
template <typename F>
inline cudaError_t smem_attr_once(F fn) {
    static std::mutex mu;
    static std::set<std::pair<const void *, int>> done;  // (kernel, device)
    int dev = 0;
    cudaGetDevice(&dev);
    const std::pair<const void *, int> key{reinterpret_cast<const void *>(fn), dev};
    {
        std::lock_guard<std::mutex> lk(mu);
        if (done.count(key)) return cudaSuccess;
    }
    int maxs = 0;
    cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    const cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, maxs);
    if (e == cudaSuccess) {
        std::lock_guard<std::mutex> lk(mu);
        done.insert(key);
    }
    return e;
}

inline int check_launch(const char *what, char *err, int errlen) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        snprintf(err, errlen, "%s: %s", what, cudaGetErrorString(e));
        return 3;
    }
    return 0;
}

template <typename T, int K, int L, int R, int LOADER>
int launch_tile(const KParams &kp, const CUtensorMap *tm, int grid, int threads, cudaStream_t st, char *err,
                int errlen) {
    auto fn = sb_tile_kernel<T, K, L, R, tile_nv(sizeof(T)), LOADER>;
    if (smem_attr_once(fn) != cudaSuccess) return check_launch("cudaFuncSetAttribute(tile)", err, errlen);
    fn<<<grid, threads, kp.smem_total, st>>>(kp, tm[0], tm[1]);
    return check_launch("tile kernel launch", err, errlen);
}

template <typename T, int L, int R, int LOADER>
int tile_K(int K, const KParams &kp, const CUtensorMap *tm, int grid, int threads, cudaStream_t st, char *err,
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

template <typename T, int K, int L, bool ADV>
int launch_warp1(const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    auto fn = kp.bulk ? sb_warp_kernel<T, K, L, true, ADV> : sb_warp_kernel<T, K, L, false, ADV>;
    if (smem_attr_once(fn) != cudaSuccess) return check_launch("cudaFuncSetAttribute(warp)", err, errlen);
    fn<<<grid, kp.warp_threads, kp.smem_total, st>>>(kp);
    return check_launch("warp kernel launch", err, errlen);
}

// odd segment lengths instantiated for the warp kernel (the plan picks from this set)
template <typename T, int K, bool ADV>
int warp_L(int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    switch (L) {
        case 3: return launch_warp1<T, K, 3, ADV>(kp, grid, st, err, errlen);
        case 5: return launch_warp1<T, K, 5, ADV>(kp, grid, st, err, errlen);
        case 9: return launch_warp1<T, K, 9, ADV>(kp, grid, st, err, errlen);
        case 17: return launch_warp1<T, K, 17, ADV>(kp, grid, st, err, errlen);
        case 33: return launch_warp1<T, K, 33, ADV>(kp, grid, st, err, errlen);
        case 63: return launch_warp1<T, K, 63, ADV>(kp, grid, st, err, errlen);
    }
    snprintf(err, errlen, "warp kernel: no instantiation for segment length %d", L);
    return 5;
}

// ADV (the advection step) exists for periodic spaces only, whose Q band is <= 3
template <typename T, bool ADV>
int warp_K(int K, int L, const KParams &kp, int grid, cudaStream_t st, char *err, int errlen) {
    switch (K) {
        case 1: return warp_L<T, 1, ADV>(L, kp, grid, st, err, errlen);
        case 2: return warp_L<T, 2, ADV>(L, kp, grid, st, err, errlen);
        case 3: return warp_L<T, 3, ADV>(L, kp, grid, st, err, errlen);
        case 4:
            if constexpr (!ADV) return warp_L<T, 4, ADV>(L, kp, grid, st, err, errlen);
            break;
    }
    snprintf(err, errlen, "unsupported band K=%d", K);
    return 5;
}
}  // namespace sb
