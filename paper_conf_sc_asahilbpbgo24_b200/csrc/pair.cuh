#pragma once
// pair.cuh -- the batch-contiguous tile kernel on a 2-CTA cluster ("pair" tile).
//
// Why: a tile row chunk of 16 fp64 right-hand sides is 128 B, one per row of
// the (n, batch) array.  With a large row pitch every chunk sits on its own
// page, and the layout's read+write ceiling falls with the pitch (measured,
// tools/stream_probe2.cu, profiles/r02/stream_probe_pitch.txt: 5654 GB/s at
// an 800 KB pitch (C2), 4970 at 8 MB (C5 on 8 GPUs), 4594 at 64 MB (C5 on one
// GPU)), while 256-B chunks hold ~5.9 TB/s at every pitch.  A 32-RHS tile is
// 256 KB of fp64 -- the whole register file of one SM -- so two SMs share it:
// the CTAs of a cluster of 2 split its rows (segments) in halves, each loads
// 256-B row chunks of its half by TMA, and the segment carries that cross the
// half boundary travel through distributed shared memory:
//   forward  -- CTA 1's first segments read CTA 0's local end states,
//   backward -- CTA 0's last segments read CTA 1's local begin states,
// each published by one remote mbarrier arrival (release.cluster) after the
// CTA's own barrier; the corner (x1 = delta'^{-1}(b1 - Lambda b0), Algorithm 1
// P:86-91) is split the same way: each CTA's corner warp reduces its own head
// or tail rows of the Lambda window and delta rows, the two partial vectors
// are exchanged through DSMEM, and both CTAs finish getrs on registers.
// Everything else (segment sweeps, carries, gamma, fused stores) is the code
// of the single-CTA tile kernel (kernels.cuh).
#include "kernels.cuh"

namespace sb {

__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t mapa_shared(uint32_t addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
    return r;
}
// arrive on an mbarrier of the other CTA (address from mapa), release at cluster scope
__device__ __forceinline__ void mbar_arrive_remote(uint32_t remote_addr) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(remote_addr) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t *m, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "SB_WAITC:\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra SB_WAITC;\n}\n" ::"r"(smem_u32(m)),
        "r"(parity)
        : "memory");
}
#ifdef SB_PAIR_DEBUG
// diagnostic builds: bounded waits that report which barrier of which CTA hangs
__device__ __forceinline__ bool mbar_test(uint64_t *m, uint32_t parity) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred P1;\n\tmbarrier.test_wait.parity.acquire.cluster.shared::cta.b64 P1, [%1], %2;\n\t"
                 "selp.u32 %0, 1, 0, P1;\n}" : "=r"(ok) : "r"(smem_u32(m)), "r"(parity) : "memory");
    return ok != 0;
}
#define PAIR_WAIT(m, par, tag, itv)                                                                              \
    do {                                                                                                         \
        long long n_ = 0;                                                                                        \
        while (!mbar_test((m), (par)))                                                                           \
            if (++n_ == (1ll << 26)) {                                                                           \
                printf("pair hang: %s block %d thread %d it %d parity %d\n", tag, blockIdx.x, threadIdx.x, (itv),  \
                       (int)(par));                                                                              \
                __trap();                                                                                        \
            }                                                                                                    \
    } while (0)
#else
#define PAIR_WAIT(m, par, tag, itv) mbar_wait_cluster((m), (par))
#endif
__device__ __forceinline__ double ld_dsmem_f64(uint32_t addr) {
    double v;
    asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(addr) : "memory");
    return v;
}
__device__ __forceinline__ void st_dsmem_f64(uint32_t addr, double v) {
    asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(addr), "d"(v) : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// x1 for the pair tile (k = KC, one lane per RHS): this CTA's partial of
// (s1 b1 - Lambda b0) over its own rows, exchanged with the other CTA through
// DSMEM, then getrs on registers.  h: this CTA's rank; own window part
// [j0, j1) of the dense Lambda window with rows base[(j - j0) * R].
template <int KC, int R>
__device__ __forceinline__ void pair_corner(const KParams &p, int h, int it, int lane, const double *slw,
                                            const double *wbase, int j0, int j1, const double *sdscale,
                                            const int *sdrow, const double *sdlu, const int *sdpiv, const double *buf,
                                            int rb, double *xpart, uint32_t xpart_remote, uint64_t *xready,
                                            uint32_t xready_remote, double *sx1, double *gout, int64_t ps) {
    const DevPlan &P = p.P;
    const int k = P.k, n = P.n;
    double xr[KC];
#pragma unroll
    for (int d = 0; d < KC; ++d) xr[d] = 0.0;
    constexpr int JB = 8;
    for (int jb = j0; jb < j1; jb += JB) {
        double b[JB];
#pragma unroll
        for (int u = 0; u < JB; ++u) b[u] = jb + u < j1 ? wbase[(size_t)(jb + u - j0) * R] : 0.0;
#pragma unroll
        for (int u = 0; u < JB; ++u)
            if (jb + u < j1)
#pragma unroll
                for (int d = 0; d < KC; ++d) xr[d] = fma(-slw[(jb + u) * KC + d], b[u], xr[d]);
    }
    // delta rows of this CTA's half
#pragma unroll
    for (int d = 0; d < KC; ++d) {
        const int row = sdrow[d];
        const bool own = (h == 0) ? row < P.s_lo : row >= n - (k - P.s_lo);
        if (own) xr[d] = fma(buf[(size_t)(row - rb) * R + lane], sdscale[d], xr[d]);
    }
    // exchange the partial vectors (double-buffered by tile parity)
    const int pb = (it & 1) * R * KC;
#pragma unroll
    for (int d = 0; d < KC; ++d) st_dsmem_f64(xpart_remote + (uint32_t)((pb + d * R + lane) * 8), xr[d]);
    mbar_arrive_remote(xready_remote + (uint32_t)((it & 1) * 8));  // the other CTA's xready[it & 1]
    PAIR_WAIT(xready + (it & 1), (it >> 1) & 1, "xready", it);
#pragma unroll
    for (int d = 0; d < KC; ++d) xr[d] += xpart[pb + d * R + lane];
    wgetrs_reg<double, KC>(xr, sdlu, sdpiv, KC);
    if (gout)
#pragma unroll
        for (int d = 0; d < KC; ++d) {
            const int row = sdrow[d];
            const bool own = (h == 0) ? row < P.s_lo : row >= n - (k - P.s_lo);
            if (own) __stcs(gout + (int64_t)row * ps, xr[d]);
        }
#pragma unroll
    for (int d = 0; d < KC; ++d) sx1[d * R + lane] = xr[d];  // [d][rhs]: conflict-free
}

template <int K, int L>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(TILE_MAX_THREADS, 1)
    sb_pair_kernel(const __grid_constant__ KParams p, const __grid_constant__ CUtensorMap tmap) {
    using C = double;
    using T = double;
    constexpr int R = 32;  // 256-B row chunks; one RHS per compute lane, one segment per warp
    constexpr int LP = L + 2;
    constexpr int ms = LP;
    extern __shared__ __align__(1024) unsigned char smem[];
    const DevPlan &P = p.P;
    const DevSeg &G = P.seg[0];
    const int h = (int)cluster_ctarank(), other = 1 - h;
    const int S = G.S, nQ = P.nQ, k = P.k, s_lo = P.s_lo;
    const int ncw = p.pr_nseg[h];            // compute warps = own segments
    const int seg0 = p.pr_seg0[h];           // first own segment
    const int rb = p.pr_rb[h];               // first row of this CTA's half
    const int nbox = p.pr_nbox[h], boxr = p.boxr;
    const int Smax = p.pr_nseg[0];           // stride of the carry arrays (both CTAs)
    const int hwarp = (int)(threadIdx.x >> 5), lane = (int)(threadIdx.x & 31);
    const int warp = hwarp == 0 ? ncw : hwarp - 1;  // corner/producer warp on hardware warp 0
    // (both CTAs launch max(nseg) + 1 warps; a CTA with one segment fewer has an idle warp)
    const bool idle = hwarp != 0 && hwarp - 1 >= ncw;

    C *sF = reinterpret_cast<C *>(smem + p.off_L);
    C *sG = reinterpret_cast<C *>(smem + p.off_G);
    C *sH = reinterpret_cast<C *>(smem + p.off_H);
    C *sfend = reinterpret_cast<C *>(smem + p.off_fend);  // [K][Smax][R], own segments
    C *sbbeg = reinterpret_cast<C *>(smem + p.off_bbeg);
    C *sx1 = reinterpret_cast<C *>(smem + p.off_x1);      // [2][R*k]
    C *xpart = reinterpret_cast<C *>(smem + p.off_cbuf);  // [2][R*k]: the other CTA's partials
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
    uint64_t *x1full = empty + NBOXMAX;  // [2]
    uint64_t *cst = x1full + 2;          // constants staged
    uint64_t *xready = cst + 1;          // [2] the other CTA's corner partials arrived
    uint64_t *xf = xready + 2;           // CTA 1: CTA 0's local end states published
    uint64_t *xb = xf + 1;               // CTA 0: CTA 1's local begin states published
    T *buf = reinterpret_cast<T *>(smem + p.off_buf);
    T *gout = reinterpret_cast<T *>(p.rhs);
    const int64_t ps = p.pstride;
    const uint32_t box_bytes = (uint32_t)(boxr * R * sizeof(T));

    if (threadIdx.x == 0) {
        for (int c = 0; c < nbox; ++c) {
            mbar_init(full + c, 1);
            mbar_init(empty + c, p.pr_empty[h][c]);
        }
        mbar_init(x1full + 0, R);
        mbar_init(x1full + 1, R);
        mbar_init(cst, 1);
        mbar_init(xready + 0, R);  // the other corner's 32 lanes arrive
        mbar_init(xready + 1, R);
        mbar_init(xf, 1);
        mbar_init(xb, 1);
        fence_mbar_init();
        prefetch_tmap(&tmap);
        stage_constants_issue<C, K>(p, G, smem, cst);
    }
    // both CTAs' barriers initialised before any remote arrival
    cluster_sync_all();
    if (idle) {
        cluster_sync_all();
        return;
    }
    mbar_wait(cst, 0);
    const uint32_t xready_remote = mapa_shared(smem_u32(xready), (uint32_t)other);
    const uint32_t xpart_remote = mapa_shared(smem_u32(xpart), (uint32_t)other);
    const uint32_t xf_remote = mapa_shared(smem_u32(xf), (uint32_t)other);
    const uint32_t xb_remote = mapa_shared(smem_u32(xb), (uint32_t)other);
    const uint32_t fend_remote = mapa_shared(smem_u32(sfend), (uint32_t)other);
    const uint32_t bbeg_remote = mapa_shared(smem_u32(sbbeg), (uint32_t)other);
    const int nclus = (int)gridDim.x / 2, clus = (int)blockIdx.x / 2;

    if (warp == ncw) {
        // ===================== corner + producer warp
        int it = 0;
        // own part of the dense Lambda window: head columns live in CTA 0, tail in CTA 1
        const int lh = P.lw_head, lw = P.lw_head + P.lw_tail;
        const int j0 = h == 0 ? 0 : lh, j1 = h == 0 ? lh : lw;
        const int wrow0 = h == 0 ? s_lo : s_lo + nQ - P.lw_tail;  // first row of the own window part
        for (int tile = clus; tile < p.ntiles; tile += nclus, ++it) {
            const int slab = tile / p.tps, tb = tile - slab * p.tps;
            T *gs = gout + slab * p.slab_stride;
            if (lane == 0)
                for (int c = 0; c < nbox; ++c) {
                    if (it > 0) PAIR_WAIT(empty + c, (it - 1) & 1, "empty(corner)", it);
                    mbar_arrive_expect_tx(full + c, box_bytes);
                    tma_load_3d(buf + (size_t)c * boxr * R, &tmap, full + c, tb * R, rb + c * boxr, slab);
                }
            __syncwarp();
            for (int c = 0; c < nbox; ++c) PAIR_WAIT(full + c, it & 1, "full(corner)", it);
            const int64_t ccol = (int64_t)tb * R + lane;
            T *gcol = ccol < p.batch ? gs + ccol * p.bstride : nullptr;
            const T *wbase = buf + (size_t)(wrow0 - rb) * R + lane;
            double *x1 = sx1 + (it & 1) * R * k;
            switch (k) {
                case 0: break;  // no delta block: nothing to exchange
                case 1: pair_corner<1, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                case 2: pair_corner<2, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                case 3: pair_corner<3, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                case 4: pair_corner<4, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                case 5: pair_corner<5, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                case 6: pair_corner<6, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                case 7: pair_corner<7, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                          xpart_remote, xready, xready_remote, x1, gcol, ps); break;
                default: pair_corner<8, R>(p, h, it, lane, slw, wbase, j0, j1, sdscale, sdrow, sdlu, sdpiv, buf, rb, xpart,
                                           xpart_remote, xready, xready_remote, x1, gcol, ps); break;
            }
            __syncwarp();
            mbar_arrive(x1full + (it & 1));
            if (lane == 0)
                for (int c = 0; c < nbox; ++c) mbar_arrive(empty + c);  // the corner read this tile's boxes
        }
        // no CTA may exit while the other can still write into its shared memory
        cluster_sync_all();
        return;
    }

    // ============================================== compute warps (one own segment each)
    const int sl = warp;                 // local segment
    const int s = seg0 + sl;             // global segment
    const int r0 = lane;                 // right-hand side of this thread in the tile
    const bool active = sl < ncw && s < S;
    const int a = s * L;
    const bool full_seg = a + L <= nQ;
    const int sc = G.slot[active ? s : 0];
    const C *fL = sF + sc * (2 * K + 1) * LP;
    const C *fU = fL + K * LP;
    const C *fD = fL + 2 * K * LP;
    const int brow = s_lo + a - rb;      // first buffer row of this segment
    // boundary segments: their carry walks reach into the other CTA (either direction,
    // so the same warps also write the states the other CTA reads; the others never wait
    // for the other CTA -- their writes of the next tile stay behind the CTA barriers
    // that the boundary warps pass only after the other CTA's signal)
    const int reach = max(G.carry_f, G.carry_b);
    const bool bnd = h == 0 ? s >= p.pr_nseg[0] - reach : s < p.pr_nseg[0] + reach;
    const int c_lo = brow / boxr, c_hi = min(brow + min(L, nQ - a) - 1, p.pr_nrows[h] - 1) / boxr;
    int it = 0;
    for (int tile = clus; tile < p.ntiles; tile += nclus, ++it) {
        const int slab = tile / p.tps;
        const int64_t col0 = (int64_t)(tile - slab * p.tps) * R + r0;
        const int nlive = (active && col0 < p.batch) ? 1 : 0;
        T *gcol = gout + slab * p.slab_stride + col0 * p.bstride;
        C v[L][1];
        for (int c = c_lo; c <= c_hi; ++c) PAIR_WAIT(full + c, it & 1, "full(compute)", it);
        {
            const T *src = buf + (size_t)brow * R + r0;
#pragma unroll
            for (int i = 0; i < L; ++i) v[i][0] = (full_seg || a + i < nQ) ? src[(size_t)i * R] : C(0);
        }
        __syncwarp();
        if (lane == 0)
            for (int c = c_lo; c <= c_hi; ++c) mbar_arrive(empty + c);
        // ---------- b0 -= gamma x1
        if (active && sgptr[s] < sgptr[s + 1]) {
            PAIR_WAIT(x1full + (it & 1), (it >> 1) & 1, "x1full", it);
            const C *x1 = sx1 + (it & 1) * R * k + r0;  // [d][rhs]
            for (int e = sgptr[s]; e < sgptr[s + 1]; ++e) {
                const int i = sgamr[e] - a;
                const int dc = sgamc[e];
                const C gv = sgamv[e];
#pragma unroll
                for (int j = 0; j < L; ++j)
                    if (j == i) v[j][0] = fma(-gv, x1[dc * R], v[j][0]);
            }
        }
        // ---------- local forward sweep, publish end state
        C st[K][1];
        fwd_local<C, K, L, 1, true>(v, fL, ms, st);
#pragma unroll
        for (int j = 0; j < K; ++j) sfend[(j * Smax + sl) * R + r0] = st[j][0];
        named_bar(1, ncw * 32);  // B2 (own CTA)
        if (h == 0) {
            if (threadIdx.x == 32) mbar_arrive_remote(xf_remote);  // CTA 1 may read these end states
        } else if (bnd) {
            PAIR_WAIT(xf, it & 1, "xf", it);  // only the segments whose carries reach into CTA 0
        }
        // ---------- forward carry + correction chain (predecessors may live in CTA 0)
        if (s > 0) {
            C cin[K][1];
#pragma unroll
            for (int m = 0; m < K; ++m) cin[m][0] = C(0);
            for (int t = max(0, s - G.carry_f); t < s; ++t) {
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    const int tl = t - seg0;
                    C acc = tl >= 0 ? sfend[(j * Smax + tl) * R + r0]
                                    : ld_dsmem_f64(fend_remote + (uint32_t)(((j * Smax + t) * R + r0) * 8));
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(sG[(t * K + j) * K + m], cin[m][0], acc);
                    nw[j] = acc;
                }
#pragma unroll
                for (int j = 0; j < K; ++j) cin[j][0] = nw[j];
            }
            fwd_correct<C, K, L, 1, true>(v, fL, ms, cin);
        }
        // ---------- local backward sweep, publish begin state
        bwd_local<C, K, L, 1, true>(v, fU, fD, ms, st);
#pragma unroll
        for (int j = 0; j < K; ++j) sbbeg[(j * Smax + sl) * R + r0] = st[j][0];
        named_bar(1, ncw * 32);  // B3 (own CTA)
        if (h == 1) {
            if (threadIdx.x == 32) mbar_arrive_remote(xb_remote);  // CTA 0 may read these begin states
        } else if (bnd) {
            PAIR_WAIT(xb, it & 1, "xb", it);
        }
        // ---------- backward carry (successors may live in CTA 1) + correction, stores.
        // Every row is stored from inside the correction chain as soon as it is final
        // (for every band, also K = 1: C5 23.94 -> 23.63 ms, its 8-GPU shard shape
        // 2.93 -> 2.88 ms against a burst after the chain; the last segment runs the
        // chain with zero carries, so there is one store path).
        {
            C co[K][1];
#pragma unroll
            for (int m = 0; m < K; ++m) co[m][0] = C(0);
            for (int t = min(S - 1, s + G.carry_b); t > s; --t) {
                C nw[K];
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    const int tl = t - seg0;
                    C acc = tl < ncw ? sbbeg[(j * Smax + tl) * R + r0]
                                     : ld_dsmem_f64(bbeg_remote + (uint32_t)(((j * Smax + (t - p.pr_seg0[1])) * R + r0) * 8));
#pragma unroll
                    for (int m = 0; m < K; ++m) acc = fma(sH[(t * K + j) * K + m], co[m][0], acc);
                    nw[j] = acc;
                }
#pragma unroll
                for (int j = 0; j < K; ++j) co[j][0] = nw[j];
            }
            T *dlast = gcol + (int64_t)(s_lo + a + L - 1) * ps;
            const int nvalid = nlive > 0 ? min(L, nQ - a) : 0;
            bwd_correct<C, K, L, 1, true, true, true, T>(v, fU, ms, co, dlast, ps, nvalid);
        }
    }
    cluster_sync_all();
}

}  // namespace sb
