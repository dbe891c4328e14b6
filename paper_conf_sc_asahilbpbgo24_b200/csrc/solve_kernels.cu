// solve_kernels.cu -- host-side dispatch of the fused kernels (kernels.cuh):
// layout / tile-width / loader choice, shared-memory layout, TMA descriptor.
#include <atomic>
#include <cstdlib>

#include "kernels.cuh"

namespace sb {

int launch_pair_f64(int K, const KParams &kp, const CUtensorMap *tm, int grid, int threads, cudaStream_t st, char *err,
                    int errlen);

// kernel chosen by the last launch_solve on this thread (spline_builder_last_kernel)
static thread_local char g_last_kernel[96] = "";
const char *last_kernel() { return g_last_kernel; }

// ------------------------------------------------------------------ host
namespace {

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// L2 promotion of the tile kernels' TMA loads.  Measured (same box, two rounds):
// the single-CTA tile with band K = 1 (128-B row chunks) wants 256 B (C2 0.2832 vs
// 0.2861 ms with 128 B or none); band K >= 2 and the pair tile (256-B chunks) want
// none (C3 Greville 0.3159 vs 0.3178, C5S8 2.810 vs 2.853 ms).  SB_TILE_L2PROMO=0..3
// (none, 64 B, 128 B, 256 B) overrides it for A/B runs.
CUtensorMapL2promotion tile_l2_promotion(bool wide) {
    static const int env = [] {
        const char *e = getenv("SB_TILE_L2PROMO");
        return e ? atoi(e) : -1;
    }();
    const int v = env >= 0 ? env : (wide ? 3 : 0);
    switch (v) {
        case 0: return CU_TENSOR_MAP_L2_PROMOTION_NONE;
        case 1: return CU_TENSOR_MAP_L2_PROMOTION_L2_64B;
        case 2: return CU_TENSOR_MAP_L2_PROMOTION_L2_128B;
        default: return CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    }
}


// resolved once, thread-safe (C++11 magic static): concurrent first calls all
// see the same result instead of racing on a half-written pointer
PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static const PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
        void *ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
        return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    }();
    return fn;
}

// opt-in shared memory per block of each device, queried once (atomic: solves
// from several host threads may race on the first query)
int max_smem_of(int dev) {
    static std::atomic<int> cache[64];
    int v = (dev >= 0 && dev < 64) ? cache[dev].load(std::memory_order_relaxed) : 0;
    if (!v) {
        cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        if (dev >= 0 && dev < 64) cache[dev].store(v, std::memory_order_relaxed);
    }
    return v;
}

int layout_smem(KParams &kp, const DevPlan &P, const DevSeg &G, int R, size_t esz, size_t buf_bytes, int cbox = 0,
                int fend_S = -1) {
    const size_t geo_bytes = (kp.adv && !P.adv_uniform) ? (size_t)GeoLayout(P).total_doubles * 8 : 0;
    size_t o = 0;
    auto take = [&](size_t bytes, size_t al) {
        o = align_up(o, al);
        size_t r = o;
        o += align_up(bytes, 16);
        return (int)r;
    };
    const int K = P.K, k = P.k, S = G.S;
    kp.off_buf = take(buf_bytes, 1024);
    kp.off_L = take((size_t)(2 * K + 1) * G.nslots * G.LP * esz, 16);  // factor blocks (DevSeg::F)
    kp.off_U = kp.off_dinv = kp.off_L;
    kp.off_G = take((size_t)S * K * K * esz, 16);
    kp.off_H = take((size_t)S * K * K * esz, 16);
    const int FS = fend_S >= 0 ? fend_S : S;  // carry arrays: segments of this CTA (pair tile: half)
    kp.off_fend = take((size_t)FS * R * K * esz, 16);
    kp.off_bbeg = take((size_t)FS * R * K * esz, 16);
    kp.off_x1 = take((size_t)2 * R * k * esz, 16);
    kp.off_lamptr = take((size_t)(k + 1) * 4, 16);
    kp.off_lamc = take((size_t)P.lam_nnz * 4, 16);
    kp.off_lamv = take((size_t)P.lam_nnz * esz, 16);
    kp.off_lw = take((size_t)(P.lw_head + P.lw_tail) * k * esz, 16);
    kp.off_gamr = take((size_t)P.gam_nnz * 4, 16);
    kp.off_gamc = take((size_t)P.gam_nnz * 4, 16);
    kp.off_gamv = take((size_t)P.gam_nnz * esz, 16);
    kp.off_gptr = take((size_t)(S + 1) * 4, 16);
    kp.off_dlu = take((size_t)k * k * esz, 16);
    kp.off_dpiv = take((size_t)k * 4, 16);
    kp.off_dscale = take((size_t)k * esz, 16);
    kp.off_drow = take((size_t)k * 4, 16);
    kp.off_cbuf = take((size_t)4 * cbox * R * esz, 128);
    kp.off_geo = take(geo_bytes, 16);
    // tile: full/empty per box, x1full[2], cfull[3]; warp kernel: 2 per warp + constants
    kp.off_mbar = take((size_t)std::max(2 * NBOXMAX + 7, 2 * WARP_MAX_WARPS + 1) * 8, 8);
    kp.smem_total = (int)align_up(o, 16);
    return kp.smem_total;
}

int launch_warp(const DevPlan &P, const SolveArgs &a, int num_sms, int max_smem, char *err, int errlen) {
    const size_t esz = a.dtype == 0 ? 8 : 4;
    const DevSeg &G = P.seg[2];
    if (G.S == 0 && a.shift) {
        snprintf(err, errlen, "advect: n=%d too large for the warp kernel", P.n);
        return 5;
    }
    if (G.S == 0) {  // Q too long for 32 register segments: serial fallback
        KParams kp{};
        kp.P = P;
        kp.rhs = a.rhs;
        kp.batch = a.batch;
        kp.bstride = a.bstride;
        kp.pstride = a.pstride;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((a.batch + 127) / 128, (int64_t)num_sms * 16));
        snprintf(g_last_kernel, sizeof(g_last_kernel), "serial<%s,K=%d>", a.dtype == 0 ? "f64" : "f32", P.K);
        return launch_serial(a.dtype, P.K, kp, grid, a.stream, err, errlen);
    }
    KParams kp{};
    kp.P = P;
    kp.rhs = a.rhs;
    kp.batch = a.batch;
    kp.bstride = a.bstride;
    kp.pstride = a.pstride;
    kp.wbuf_pitch = (int)align_up((size_t)WB_FRONT + P.n + std::max(P.k, 3) + 2, 4);
    kp.shift = a.shift;
    kp.adv = a.shift != nullptr;
    // bulk-copy pipeline when every row is one contiguous, 16-B aligned run;
    // fewer warps per block (or no second buffer) when shared memory is short
    const bool can_bulk = a.pstride == 1 && (a.bstride * (int64_t)esz) % 16 == 0 && (uintptr_t)a.rhs % 16 == 0 &&
                          ((int64_t)P.n * (int64_t)esz) % 16 == 0;
    // candidates (bulk pipeline first, measured best for C4), scored by resident
    // warps per SM; the per-block constants (factors, advection geometry) are
    // paid once per block, so large-smem cases prefer fewer, wider blocks.
    // SB_WARP_BULK=0/1 forces the loader (A/B experiments).
    static const int bulk_env = [] {
        const char *e = getenv("SB_WARP_BULK");
        return e ? atoi(e) : -1;
    }();
    struct Cand { bool bulk; int wpb; };
    const Cand cands[] = {{true, 4}, {true, 2}, {true, 1}, {true, 8}, {true, 6}, {true, 3}, {true, 12}, {true, 16},
                          {false, 8}, {false, 6}, {false, 4}, {false, 2}, {false, 1}, {false, 12}, {false, 16}};
    const int out_row = 0;  // the advection stores straight to HBM (no output row buffer)
    int best = -1, best_score = 0;
    for (int ci = 0; ci < (int)(sizeof(cands) / sizeof(cands[0])); ++ci) {
        const Cand &c = cands[ci];
        if (c.bulk && !can_bulk) continue;
        if (bulk_env >= 0 && c.bulk != (bulk_env > 0)) continue;
        // the advection step with band K >= 2 runs better without the bulk pipeline
        // (measured, Fig. 2 uniform p = 4 / 5: 0.592 -> 0.572 ms, 0.628 -> 0.609 ms;
        // p = 3 (K = 1) keeps it: 0.373 vs 0.403 ms)
        if (bulk_env < 0 && c.bulk && kp.adv && P.K >= 2) continue;
        KParams t = kp;
        layout_smem(t, P, G, 1, esz, (size_t)c.wpb * ((c.bulk ? 2 : 1) + out_row) * kp.wbuf_pitch * esz);
        if (t.smem_total > max_smem) continue;
        const int per_sm = std::min(WARP_MAX_WARPS / c.wpb, (int)(228 * 1024 / (t.smem_total + 1024)));
        // the bulk pipeline (double-buffered rows) is worth 1.5x the warps
        // (measured: C4 bulk 12 warps/SM 0.378 ms vs plain 16 warps 0.396 ms)
        const int score = c.wpb * std::max(per_sm, 1) * (c.bulk ? 3 : 2);
        if (score > best_score) {
            best_score = score;
            best = ci;
        }
    }
    const bool fits = best >= 0;
    if (fits) {
        kp.bulk = cands[best].bulk;
        kp.warp_threads = 32 * cands[best].wpb;
        layout_smem(kp, P, G, 1, esz,
                    (size_t)cands[best].wpb * ((kp.bulk ? 2 : 1) + out_row) * kp.wbuf_pitch * esz);
    }
    if (!fits && kp.adv) {
        snprintf(err, errlen, "advect: n=%d needs more shared memory than a block has", P.n);
        return 5;
    }
    if (!fits) {  // factors + one row do not fit: serial fallback
        snprintf(g_last_kernel, sizeof(g_last_kernel), "serial<%s,K=%d>", a.dtype == 0 ? "f64" : "f32", P.K);
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((a.batch + 127) / 128, (int64_t)num_sms * 16));
        return launch_serial(a.dtype, P.K, kp, grid, a.stream, err, errlen);
    }
    const int wpb = kp.warp_threads / 32;
    const int per_sm = std::max(1, std::min(WARP_MAX_WARPS / wpb, (int)(228 * 1024 / (kp.smem_total + 1024))));
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((a.batch + wpb - 1) / wpb, (int64_t)num_sms * per_sm));
    // round L up to an instantiated odd length (the plan chose the smallest odd L >= nQ/32)
    snprintf(g_last_kernel, sizeof(g_last_kernel), "warp<%s,K=%d,L=%d,%s%s>", a.dtype == 0 ? "f64" : "f32", P.K,
             G.L, kp.bulk ? "BULK" : "DIRECT", kp.adv ? ",ADV" : "");
    if (a.dtype == 0) return launch_warp_f64(P.K, G.L, kp, grid, a.stream, err, errlen);
    return launch_warp_f32(P.K, G.L, kp, grid, a.stream, err, errlen);
}

}  // namespace

int launch_solve(const DevPlan &P, const SolveArgs &a_in, int num_sms, char *err, int errlen) {
    SolveArgs a = a_in;
    if (a.batch == 0 || a.nslab == 0) return 0;
    if (a.nslab > 1 && (a.bstride != 1 || a.shift)) {
        // slabs of a strided layout: the warp kernel takes them one launch each
        for (int64_t sl = 0; sl < a.nslab; ++sl) {
            SolveArgs b = a;
            b.nslab = 1;
            b.rhs = (char *)a.rhs + sl * a.slab_stride * (a.dtype == 0 ? 8 : 4);
            const int st = launch_solve(P, b, num_sms, err, errlen);
            if (st) return st;
        }
        return 0;
    }
    if (a.nslab == 1) a.slab_stride = (int64_t)P.n * a.pstride;
    const size_t esz = a.dtype == 0 ? 8 : 4;
    int dev = 0;
    cudaGetDevice(&dev);
    const int max_smem = max_smem_of(dev);

    // point-contiguous / general strided layouts and the advection step: warp-per-RHS kernel
    if (a.bstride != 1 || a.shift) return launch_warp(P, a, num_sms, max_smem, err, errlen);
    auto per_slab_warp = [&]() {  // batch-contiguous slabs the tile kernel cannot take
        for (int64_t sl = 0; sl < a.nslab; ++sl) {
            SolveArgs b = a;
            b.nslab = 1;
            b.rhs = (char *)a.rhs + sl * a.slab_stride * (int64_t)esz;
            const int st = launch_warp(P, b, num_sms, max_smem, err, errlen);
            if (st) return st;
        }
        return 0;
    };

    static const int small_env = [] {  // SB_SMALL_KERNEL=1 serial / 2 warp / 3 tile kernel for batch-contiguous (A/B)
        const char *e = getenv("SB_SMALL_KERNEL");
        return e ? atoi(e) : 0;
    }();
    // tiny problems (C1: 16 x 8) are launch/latency-bound: the warp kernel's lighter
    // prologue wins (C1 graph-timed: warp 5.4 us, serial 6.4 us, tile 7.3 us)
    const bool tiny = a.nslab == 1 && P.n <= 64 && a.batch <= 64 && P.seg[2].S > 0;
    if ((small_env == 2 || (small_env == 0 && tiny)) && a.nslab == 1)
        return launch_warp(P, a, num_sms, max_smem, err, errlen);
    if (small_env == 1 && a.nslab == 1) {
        KParams kp{};
        kp.P = P;
        kp.rhs = a.rhs;
        kp.batch = a.batch;
        kp.bstride = a.bstride;
        kp.pstride = a.pstride;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((a.batch + 127) / 128, (int64_t)num_sms * 16));
        snprintf(g_last_kernel, sizeof(g_last_kernel), "serial<%s,K=%d>", a.dtype == 0 ? "f64" : "f32", P.K);
        return launch_serial(a.dtype, P.K, kp, grid, a.stream, err, errlen);
    }
    // pair tile (pair.cuh): 32-RHS tiles (256-B row chunks) split over a 2-CTA cluster.
    // Worth it where the row pitch is large (C5: 8e6 RHS, 64 MB rows); SB_TILE_PAIR=0
    // never, 2 whenever it applies (A/B), default 1: rows of at least pair_pitch bytes.
    {
        static const int pair_env = [] {
            const char *e = getenv("SB_TILE_PAIR");
            return e ? atoi(e) : 1;
        }();
        static const double pair_pitch = [] {
            const char *e = getenv("SB_TILE_PAIR_PITCH_MB");
            return (e ? atof(e) : 4.0) * 1048576.0;
        }();
        const DevSeg &G0 = P.seg[0];
        const bool want = pair_env == 2 || (pair_env == 1 && (double)a.pstride * esz >= pair_pitch);
        const int nseg0 = (G0.S + 1) / 2, nseg1 = G0.S - nseg0;
        const int rb1 = P.s_lo + nseg0 * G0.L;  // first row of CTA 1
        const bool fits_geom = G0.S >= 2 && nseg1 >= 1 && P.K <= 4 && P.k <= 8 && G0.LP == G0.L + 2 &&
                               P.lw_head <= nseg0 * G0.L && P.nQ - P.lw_tail >= nseg0 * G0.L && rb1 < P.n;
        const bool aligned = ((uintptr_t)a.rhs % 16 == 0) && ((a.pstride * (int64_t)esz) % 16 == 0) &&
                             ((a.slab_stride * (int64_t)esz) % 16 == 0) && a.nslab < (1ll << 31);
        if (want && a.dtype == 0 && fits_geom && aligned && a.batch >= 32 && get_encode()) {
            KParams kp{};
            kp.P = P;
            kp.rhs = a.rhs;
            kp.batch = a.batch;
            kp.bstride = a.bstride;
            kp.pstride = a.pstride;
            kp.pr_rb[0] = 0; kp.pr_rb[1] = rb1;
            kp.pr_nrows[0] = rb1; kp.pr_nrows[1] = P.n - rb1;
            kp.pr_seg0[0] = 0; kp.pr_seg0[1] = nseg0;
            kp.pr_nseg[0] = nseg0; kp.pr_nseg[1] = nseg1;
            const int maxrows = std::max(kp.pr_nrows[0], kp.pr_nrows[1]);
            const int nb = (maxrows + 255) / 256;
            const int boxr = ((maxrows + nb - 1) / nb + 7) / 8 * 8;
            kp.boxr = boxr;
            for (int h = 0; h < 2; ++h) kp.pr_nbox[h] = (kp.pr_nrows[h] + boxr - 1) / boxr;
            const int nbx = std::max(kp.pr_nbox[0], kp.pr_nbox[1]);
            const int64_t tps = (a.batch + 31) / 32;
            if (nbx <= NBOXMAX && tps * a.nslab < (1ll << 31) &&
                layout_smem(kp, P, G0, 32, 8, (size_t)nbx * boxr * 32 * 8, (P.k + 1) / 2, nseg0) <= max_smem) {
                kp.tps = (int)tps;
                kp.ntiles = (int)(tps * a.nslab);
                kp.slab_stride = a.slab_stride;
                for (int h = 0; h < 2; ++h) {
                    for (int c = 0; c < NBOXMAX; ++c) kp.pr_empty[h][c] = 1;  // unused boxes: any valid count
                    for (int c = 0; c < kp.pr_nbox[h]; ++c) kp.pr_empty[h][c] = 1;  // the corner warp reads every box
                    for (int sl = 0; sl < kp.pr_nseg[h]; ++sl) {
                        const int sg = kp.pr_seg0[h] + sl, a0 = sg * G0.L;
                        const int r0 = P.s_lo + a0 - kp.pr_rb[h];
                        const int r1 = std::min(r0 + std::min(G0.L, P.nQ - a0), kp.pr_nrows[h]) - 1;
                        for (int c = r0 / boxr; c <= r1 / boxr; ++c) kp.pr_empty[h][c]++;
                    }
                }
                CUtensorMap tm[1];
                memset(tm, 0, sizeof(tm));
                cuuint64_t dims[3] = {(cuuint64_t)a.batch, (cuuint64_t)P.n, (cuuint64_t)a.nslab};
                cuuint64_t strides[2] = {(cuuint64_t)(a.pstride * 8), (cuuint64_t)(a.slab_stride * 8)};
                cuuint32_t box[3] = {32u, (cuuint32_t)boxr, 1u};
                cuuint32_t estr[3] = {1, 1, 1};
                CUresult cr = get_encode()(&tm[0], CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, a.rhs, dims, strides, box, estr,
                                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                           tile_l2_promotion(false), CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                if (cr != CUDA_SUCCESS) {
                    snprintf(err, errlen, "cuTensorMapEncodeTiled (pair) failed (%d)", (int)cr);
                    return 3;
                }
                const int threads = (std::max(nseg0, nseg1) + 1) * 32;
                const int clusters = (int)std::min<int64_t>((int64_t)kp.ntiles, (int64_t)num_sms / 2);
                snprintf(g_last_kernel, sizeof(g_last_kernel), "pair<f64,K=%d,R=32,TMA,2xCTA>", P.K);
                return launch_pair_f64(P.K, kp, tm, 2 * clusters, threads, a.stream, err, errlen);
            }
        }
    }
    const DevSeg &G = P.seg[a.dtype == 0 ? 0 : 1];
    const int L = G.L;
    if (G.LP != L + (esz == 8 ? 2 : 4)) {  // the tile kernel's compile-time factor pitch
        snprintf(err, errlen, "tile plan pitch %d does not match L=%d", G.LP, L);
        return 5;
    }
    KParams kp{};
    kp.P = P;
    kp.rhs = a.rhs;
    kp.batch = a.batch;
    kp.bstride = a.bstride;
    kp.pstride = a.pstride;
    // TMA needs a 16-B aligned base, row pitch and slab pitch; boxes of <= 256 rows
    const bool aligned = ((uintptr_t)a.rhs % 16 == 0) && ((a.pstride * (int64_t)esz) % 16 == 0) &&
                         ((a.slab_stride * (int64_t)esz) % 16 == 0) && a.nslab < (1ll << 31);
    static const int box_max = [] {  // SB_TILE_BOXROWS: rows per TMA box at most (A/B; TMA limit 256)
        const char *e = getenv("SB_TILE_BOXROWS");
        const int v = e ? atoi(e) : 256;
        return v >= 8 && v <= 256 ? v : 256;
    }();
    int nbox = (P.n + box_max - 1) / box_max;
    if (nbox > NBOXMAX) nbox = (P.n + 255) / 256;
    const int boxr = ((P.n + nbox - 1) / nbox + 7) / 8 * 8;
    const int cands64[2] = {16, 8}, cands32[2] = {32, 16};
    const int *cands = a.dtype == 0 ? cands64 : cands32;
    int R = 0, loader = LOAD_DIRECT;
    for (int ci = 0; ci < 2 && !R; ++ci) {
        const int cand = cands[ci];
        const int ncw = (cand / tile_nv((int)esz) * G.S + 31) / 32;  // RP = R / NV threads per segment
        if ((ncw + 1) * 32 > TILE_MAX_THREADS) continue;
        KParams t = kp;
        if (aligned && a.batch >= cand && nbox <= NBOXMAX && get_encode() &&
            layout_smem(t, P, G, cand, esz, (size_t)nbox * boxr * cand * esz) <= max_smem) {
            R = cand;
            loader = LOAD_TMA;
        } else if (layout_smem(t, P, G, cand, esz, 0) <= max_smem) {
            R = cand;
            loader = LOAD_DIRECT;
        }
    }
    if (!R) return per_slab_warp();  // too large for the tile kernel
    const int RP = R / tile_nv((int)esz);  // a compute thread owns NV right-hand sides
    kp.ncw = (RP * G.S + 31) / 32;
    layout_smem(kp, P, G, R, esz, loader == LOAD_TMA ? (size_t)nbox * boxr * R * esz : 0);
    const int64_t tps = (a.batch + R - 1) / R;
    if (tps * a.nslab >= (1ll << 31)) return per_slab_warp();
    kp.tps = (int)tps;
    kp.ntiles = (int)(tps * a.nslab);
    kp.slab_stride = a.slab_stride;
    kp.nbox = nbox;
    kp.boxr = boxr;
    // corner boxes: the corner reads only rows [0,cbox) and [n-cbox,n); they are
    // fetched one tile early with their own (smaller) tensor map
    int cbox = 0;
    // Off by default since the corner became a k-templated register computation on
    // hardware warp 0 reading a dense Lambda window: it now finishes from the landed
    // tile in time, and the corner boxes only cost shared memory and L2 re-reads
    // (measured: C3 Hermite 0.298 ms with them, 0.276 ms without; C2, C3 Greville,
    // C4M unchanged).  SB_TILE_CBOX=1 enables them where they fit (A/B experiments).
    static const int cbox_env = [] {
        const char *e = getenv("SB_TILE_CBOX");
        return e ? atoi(e) : 0;
    }();
    // worth it only when the corner step is heavy enough to delay the gamma warps
    // (measured: k=1 / 48 nnz C2 loses 4.6 %, k=6 Hermite C3 gains 16 %)
    const int corner_work = P.lam_nnz / (32 / R) + P.k * P.k;
    if (loader == LOAD_TMA && P.corner_rows > 0 && cbox_env && (corner_work > 30 || cbox_env > 1)) {
        cbox = (P.corner_rows + 7) / 8 * 8;
        KParams t = kp;
        if (cbox > 256 || 2 * cbox > P.n ||
            layout_smem(t, P, G, R, esz, (size_t)nbox * boxr * R * esz, cbox) > max_smem)
            cbox = 0;
    }
    kp.cbox = cbox;
    layout_smem(kp, P, G, R, esz, loader == LOAD_TMA ? (size_t)nbox * boxr * R * esz : 0, cbox);
    // arrivals that free box c: compute warps whose real rows touch it (+ the corner
    // warp when it reads the main tile, or when no compute warp reads box c).
    // DIRECT: empty[0] counts the compute warps that finished a tile.
    const int spw = 32 / RP;
    for (int c = 0; c < NBOXMAX; ++c) kp.empty_count[c] = 0;
    kp.corner_arrive_mask = 0;
    if (loader == LOAD_TMA) {
        for (int w = 0; w < kp.ncw; ++w) {
            const int s0 = w * spw;
            if (s0 >= G.S) continue;
            const int r0 = P.s_lo + s0 * L;
            const int r1 = P.s_lo + std::min((s0 + spw) * L, P.nQ) - 1;
            if (r1 < r0) continue;
            for (int c = r0 / boxr; c <= r1 / boxr; ++c) kp.empty_count[c]++;
        }
        // boxes the corner reads from the main tile: delta rows and the Lambda window
        int need = 0;
        for (int d = 0; d < P.k; ++d) {  // delta row d: the head rows first, then the tail rows
            const int row = d < P.s_lo ? d : P.n - (P.k - P.s_lo) + (d - P.s_lo);
            need |= 1 << (row / boxr);
        }
        if (P.lw_head > 0)
            for (int c = P.s_lo / boxr; c <= (P.s_lo + P.lw_head - 1) / boxr; ++c) need |= 1 << c;
        if (P.lw_tail > 0)
            for (int c = (P.s_lo + P.nQ - P.lw_tail) / boxr; c <= (P.s_lo + P.nQ - 1) / boxr; ++c) need |= 1 << c;
        kp.corner_need_mask = cbox == 0 ? need : 0;
        for (int c = 0; c < nbox; ++c)
            if ((cbox == 0 && ((need >> c) & 1)) || kp.empty_count[c] == 0) {
                kp.empty_count[c]++;
                kp.corner_arrive_mask |= 1 << c;
            }
        // issue the corner's boxes first when its work is heavy (C3 Greville, k = 4 over a
        // 45-column window: 0.332 -> 0.320 ms); for a light corner (C2, C4M: k = 1) the
        // natural order is better (0.284 vs 0.293 ms): the tail box's readers are the last
        // warps to free it, and waiting for them first delays the middle boxes
        const bool heavy = P.k * (P.lw_head + P.lw_tail + 1) >= 64;
        int q = 0;
        for (int c = 0; c < nbox; ++c)
            if (!heavy || ((kp.corner_need_mask >> c) & 1)) kp.box_order[q++] = c;
        for (int c = 0; c < nbox && heavy; ++c)
            if (!((kp.corner_need_mask >> c) & 1)) kp.box_order[q++] = c;
    } else {
        kp.empty_count[0] = kp.ncw;
        for (int c = 0; c < NBOXMAX; ++c) kp.box_order[c] = c;
    }
    for (int c = 0; c < NBOXMAX; ++c)
        if (kp.empty_count[c] == 0) kp.empty_count[c] = 1;  // unused boxes: any valid count
    CUtensorMap tm[2];
    memset(tm, 0, sizeof(tm));
    if (loader == LOAD_TMA) {
        for (int q = 0; q < (cbox ? 2 : 1); ++q) {
            cuuint64_t dims[3] = {(cuuint64_t)a.batch, (cuuint64_t)P.n, (cuuint64_t)a.nslab};
            cuuint64_t strides[2] = {(cuuint64_t)(a.pstride * (int64_t)esz), (cuuint64_t)(a.slab_stride * (int64_t)esz)};
            cuuint32_t box[3] = {(cuuint32_t)R, (cuuint32_t)(q == 0 ? boxr : cbox), 1};
            cuuint32_t estr[3] = {1, 1, 1};
            CUresult cr = get_encode()(&tm[q], a.dtype == 0 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64
                                                            : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                                       3, a.rhs, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                       CU_TENSOR_MAP_SWIZZLE_NONE, tile_l2_promotion(P.K == 1),
                                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
            if (cr != CUDA_SUCCESS) {
                snprintf(err, errlen, "cuTensorMapEncodeTiled failed (%d)", (int)cr);
                return 3;
            }
        }
    }
    const int threads = (kp.ncw + 1) * 32;
    const int grid = (int)std::min<int64_t>((int64_t)kp.ntiles, (int64_t)num_sms);
    snprintf(g_last_kernel, sizeof(g_last_kernel), "tile<%s,K=%d,R=%d,%s%s>", a.dtype == 0 ? "f64" : "f32", P.K, R,
             loader == LOAD_TMA ? "TMA" : "DIRECT", cbox ? ",CBOX" : "");
    if (a.dtype == 0) return launch_tile_f64(R, loader, P.K, kp, tm, grid, threads, a.stream, err, errlen);
    return launch_tile_f32(R, loader, P.K, kp, tm, grid, threads, a.stream, err, errlen);
}

}  // namespace sb
