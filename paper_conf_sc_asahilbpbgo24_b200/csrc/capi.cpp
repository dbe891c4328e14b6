// capi.cpp -- the extern "C" boundary declared in include/spline_builder.h.
// Host create (plan.cpp) + one packed device upload + kernel dispatch
// (solve_kernels.cu).  No exception crosses the ABI.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "../../include/spline_builder.h"
#include "device.hpp"
#include "host/plan.hpp"
#include "refactor.hpp"

namespace {

thread_local std::string g_err = "";
thread_local int g_status = 0;

int fail(int code, const std::string &msg) {
    g_err = msg;
    g_status = code;
    return code;
}


}  // namespace

struct spline_builder {
    sb::Plan plan;
    int device = -1;
    int num_sms = 0;
    bool host_only = false;
    int c_degree = 0, c_npoints = 0, c_bc = 0, c_split_lo = -1, c_split_hi = -1;  // create arguments (update)
    void *blob = nullptr;  // device constants
    size_t blob_bytes = 0;
    // blobs replaced by update(): kept until destroy, so kernels captured in a
    // CUDA graph before an update stay memory-safe (they keep the old mesh)
    std::vector<void *> retired;
    sb::DevPlan dp{};
    // device-side refactorisation (SB_FLAG_DEVICE_UPDATE)
    bool dev_update = false;
    void *stage_blob = nullptr;   // staging copy of the blob (same layout)
    void *rf_scratch = nullptr;   // scratch of the refactor kernel
    int *rf_status = nullptr;     // device status word
    int *rf_status_host = nullptr; // pinned copy of it
    int *rf_rowdesc = nullptr;    // row descriptors (device)
    cudaEvent_t rf_event = nullptr;
    bool rf_pending = false;
    double x0 = 0.0, xN = 1.0;    // periodic domain ends at create
    // 2-D builder pipeline: pass 1 and pass 2 on two internal streams, chunk by chunk
    std::mutex pipe_mu;
    cudaStream_t pipe[2] = {nullptr, nullptr};
    std::vector<cudaEvent_t> pipe_ev;
    // staging for solve_host
    std::mutex host_mu;
    void *stage[3] = {nullptr, nullptr, nullptr};
    size_t stage_bytes = 0;
    cudaStream_t streams[3] = {nullptr, nullptr, nullptr};
};

namespace {

struct Packer {
    std::vector<unsigned char> bytes;
    size_t add(const void *src, size_t n) {
        size_t off = (bytes.size() + 15) / 16 * 16;
        bytes.resize(off + (n + 15) / 16 * 16, 0);
        if (n) std::memcpy(bytes.data() + off, src, n);
        return off;
    }
    template <typename T>
    size_t addv(const std::vector<T> &v) { return add(v.data(), v.size() * sizeof(T)); }
};

template <typename C>
std::vector<C> conv(const std::vector<double> &v) {
    return std::vector<C>(v.begin(), v.end());
}

// [t][j][m] (host SegPlan) -> [j][m][t] (device; see upload)
std::vector<double> seg_major(const std::vector<double> &M, int S, int K) {
    std::vector<double> r(M.size(), 0.0);
    for (int t = 0; t < S; ++t)
        for (int j = 0; j < K; ++j)
            for (int m = 0; m < K; ++m) r[((size_t)j * K + m) * S + t] = M[((size_t)t * K + j) * K + m];
    return r;
}

int upload(spline_builder *h) {
    const sb::Plan &P = h->plan;
    const int K = P.K, nQ = P.nQ, k = P.k;
    std::vector<double> dscale(k);
    for (int d = 0; d < k; ++d) dscale[d] = P.rowscale[P.drow[d]];
    Packer pk;
    // per segment plan: factor arrays in the padded per-segment layout of device.hpp
    struct SegOff { size_t F[2], G[2], H[2], gptr, slot; int LP, nslots; };
    SegOff so[3];
    for (int g = 0; g < 3; ++g) {
        const sb::SegPlan &G = P.seg[g];
        // pitch: even (pair loads) and bank-staggered for the tile kernels (+2 fp64 / +4 fp32
        // elements = 16 B); the warp kernel (odd L, lanes read distinct rows) needs no padding
        const int LP = g == 0 ? G.L + 2 : (g == 1 ? G.L + 4 : G.L);
        so[g].LP = LP;
        const int S = G.S;
        // factor data of each segment (identity on padding rows); segments with
        // bitwise-identical data share one storage slot, so lanes reading them
        // broadcast (uniform meshes: the LDL^T factors converge after ~30 rows)
        std::vector<std::vector<double>> segdata(S);
        for (int s = 0; s < S; ++s) {
            std::vector<double> &dsd = segdata[s];
            dsd.assign((size_t)(2 * K + 1) * G.L, 0.0);
            for (int i = 0; i < G.L; ++i) {
                const int row = s * G.L + i;
                dsd[(size_t)2 * K * G.L + i] = 1.0;
                if (row >= nQ) continue;
                for (int m = 0; m < K; ++m) {
                    dsd[(size_t)m * G.L + i] = P.Lb[(size_t)row * K + m];
                    dsd[(size_t)(K + m) * G.L + i] = P.Ub[(size_t)row * K + m];
                }
                dsd[(size_t)2 * K * G.L + i] = P.dinv[row];
            }
        }
        std::vector<int> slot(std::max(S, 1), 0), uniq;
        for (int s = 0; s < S; ++s) {
            int found = -1;
            // (device-updatable handles: one slot per segment, the factors change in place)
            for (size_t u = 0; u < uniq.size() && found < 0 && !P.dev_update; ++u)
                if (segdata[uniq[u]] == segdata[s]) found = (int)u;
            if (found < 0) { found = (int)uniq.size(); uniq.push_back(s); }
            slot[s] = found;
        }
        const int NS = std::max(1, (int)uniq.size());
        so[g].nslots = NS;
        // one block per slot: [L bands K x LP][U bands K x LP][dinv LP] (device.hpp)
        const size_t BS = (size_t)(2 * K + 1) * LP;
        std::vector<double> F(NS * BS, 0.0);
        for (size_t u = 0; u < (size_t)NS; ++u)
            for (int i = 0; i < LP; ++i) F[u * BS + (size_t)2 * K * LP + i] = 1.0;  // padding rows: identity
        for (size_t u = 0; u < uniq.size(); ++u) {
            const std::vector<double> &dsd = segdata[uniq[u]];
            for (int i = 0; i < G.L; ++i)
                for (int b = 0; b <= 2 * K; ++b) F[u * BS + (size_t)b * LP + i] = dsd[(size_t)b * G.L + i];
        }
        so[g].slot = pk.addv(slot);
        std::vector<int> gptr(S + 1, 0);
        for (int s = 0, e = 0; s <= S; ++s) {
            while (e < (int)P.gam_r.size() && P.gam_r[e] < s * G.L) ++e;
            gptr[s] = e;
        }
        if (S > 0) gptr[S] = (int)P.gam_r.size();
        so[g].F[0] = pk.addv(F); so[g].F[1] = pk.addv(conv<float>(F));
        // transfer matrices: the warp plan (g = 2) in [j][m][segment] order -- its lanes
        // walk different segments, so consecutive lanes read consecutive words (the
        // host plan's [segment][j][m] order made every K >= 2 walk load a 4- to 8-way
        // bank conflict); the tile plans keep [segment][j][m] (two segments per warp,
        // and the extra index arithmetic spilled the K = 3 tile kernel)
        const std::vector<double> Gs = g == 2 ? seg_major(G.G, G.S, P.K) : G.G;
        const std::vector<double> Hs = g == 2 ? seg_major(G.H, G.S, P.K) : G.H;
        so[g].G[0] = pk.addv(Gs); so[g].G[1] = pk.addv(conv<float>(Gs));
        so[g].H[0] = pk.addv(Hs); so[g].H[1] = pk.addv(conv<float>(Hs));
        so[g].gptr = pk.addv(gptr);
    }
    std::vector<double> rowf((size_t)std::max(nQ, 1) * (2 * K + 1), 0.0);
    for (int i = 0; i < nQ; ++i) {
        for (int m = 0; m < K; ++m) {
            rowf[(size_t)i * (2 * K + 1) + m] = P.Lb[(size_t)i * K + m];
            rowf[(size_t)i * (2 * K + 1) + K + m] = P.Ub[(size_t)i * K + m];
        }
        rowf[(size_t)i * (2 * K + 1) + 2 * K] = P.dinv[i];
    }
    size_t oRowf[2] = {pk.addv(rowf), pk.addv(conv<float>(rowf))};
    size_t oXe = pk.addv(P.xe), oXi = pk.addv(P.xi), oRcp = pk.addv(P.adv_rcp), oTbl = pk.addv(P.adv_tbl);
    size_t oLam[2], oGam[2], oDlu[2], oDs[2];
    for (int c = 0; c < 2; ++c) {
        auto put = [&](const std::vector<double> &v) { return c == 0 ? pk.addv(v) : pk.addv(conv<float>(v)); };
        oLam[c] = put(P.Lam_v); oGam[c] = put(P.gam_v); oDlu[c] = put(P.dlu); oDs[c] = put(dscale);
    }
    // tile-kernel corner data (device.hpp): Lambda on a dense column window and
    // gamma by distinct row
    int lw_head = 0, lw_tail = 0;
    for (int c : P.Lam_c) {
        if (c < nQ / 2) lw_head = std::max(lw_head, c + 1);
        else lw_tail = std::max(lw_tail, nQ - c);
    }
    const int lw_w = lw_head + lw_tail;
    std::vector<double> lw_v((size_t)std::max(lw_w, 1) * std::max(k, 1), 0.0);
    for (int d = 0; d < k; ++d)
        for (int e = P.Lam_ptr[d]; e < P.Lam_ptr[d + 1]; ++e) {
            const int c = P.Lam_c[e];
            const int j = c < lw_head ? c : lw_head + (c - (nQ - lw_tail));
            lw_v[(size_t)j * k + d] = P.Lam_v[e];
        }
    size_t o_lw[2] = {pk.addv(lw_v), pk.addv(conv<float>(lw_v))};
    size_t o_lamptr = pk.addv(P.Lam_ptr), o_lamc = pk.addv(P.Lam_c), o_gamr = pk.addv(P.gam_r),
           o_gamc = pk.addv(P.gam_c), o_dpiv = pk.addv(P.dpiv), o_drow = pk.addv(P.drow);
    h->blob_bytes = std::max<size_t>(pk.bytes.size(), 16);
    cudaError_t e = cudaMalloc(&h->blob, h->blob_bytes);
    if (e != cudaSuccess) return fail(SB_NOMEM, std::string("cudaMalloc(blob): ") + cudaGetErrorString(e));
    e = cudaMemcpy(h->blob, pk.bytes.data(), pk.bytes.size(), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return fail(SB_CUDA, std::string("cudaMemcpy(blob): ") + cudaGetErrorString(e));
    // a copy from pageable memory may still be in flight when cudaMemcpy returns;
    // solves may be issued on non-blocking streams that do not order against it
    e = cudaStreamSynchronize(0);
    if (e != cudaSuccess) return fail(SB_CUDA, std::string("sync after blob upload: ") + cudaGetErrorString(e));
    auto at = [&](size_t off) { return (const void *)((const unsigned char *)h->blob + off); };
    sb::DevPlan &d = h->dp;
    d.n = P.n; d.nQ = nQ; d.s_lo = P.s_lo; d.k = k; d.K = K;
    d.p = P.p; d.N = P.N; d.periodic = P.bc == sb::PERIODIC;
    d.lam_nnz = (int)P.Lam_v.size(); d.gam_nnz = (int)P.gam_v.size();
    {   // rows the corner step reads: delta rows (b1) and Lambda columns (b0)
        int head = 0, tail = 0;
        auto note = [&](int row) {
            if (row < P.n / 2) head = std::max(head, row + 1);
            else tail = std::max(tail, P.n - row);
        };
        for (int r : P.drow) note(r);
        for (int c : P.Lam_c) note(P.s_lo + c);
        d.corner_rows = k > 0 ? std::max(head, tail) : 0;
    }
    for (int c = 0; c < 2; ++c) {
        d.lam_v[c] = at(oLam[c]); d.gam_v[c] = at(oGam[c]); d.dlu[c] = at(oDlu[c]); d.dscale[c] = at(oDs[c]);
        d.rowf[c] = at(oRowf[c]);
    }
    for (int g = 0; g < 3; ++g) {
        const sb::SegPlan &G = P.seg[g];
        sb::DevSeg &ds = d.seg[g];
        ds.L = G.L; ds.S = G.S; ds.LP = so[g].LP; ds.carry_f = G.carry_f; ds.carry_b = G.carry_b;
        ds.nslots = so[g].nslots; ds.slot = (const int *)at(so[g].slot);
        for (int c = 0; c < 2; ++c) {
            ds.F[c] = at(so[g].F[c]);
            ds.G[c] = at(so[g].G[c]); ds.H[c] = at(so[g].H[c]);
        }
        ds.gptr = (const int *)at(so[g].gptr);
    }
    d.xe = (const double *)at(oXe); d.xi = (const double *)at(oXi);
    d.adv_uniform = P.adv_uniform ? 1 : 0; d.adv_invh = P.adv_invh; d.adv_q0 = P.adv_q0;
    d.adv_rcp = (const double *)at(oRcp);
    d.adv_tbl = (const int *)at(oTbl); d.adv_nbkt = (int)P.adv_tbl.size(); d.adv_steps = P.adv_steps;
    d.adv_bscale = P.xe.empty() ? 0.0 : (double)P.adv_tbl.size() / (P.xb[P.N] - P.xb[0]);
    d.lam_ptr = (const int *)at(o_lamptr); d.lam_c = (const int *)at(o_lamc);
    d.lw_head = lw_head; d.lw_tail = lw_tail;
    for (int c = 0; c < 2; ++c) d.lw_v[c] = at(o_lw[c]);
    d.gam_r = (const int *)at(o_gamr); d.gam_c = (const int *)at(o_gamc);
    d.dpiv = (const int *)at(o_dpiv); d.drow = (const int *)at(o_drow);
    return 0;
}

// device-update resources: a staging copy of the blob (initialised from the
// live one, so the arrays the refactor kernel does not rewrite -- patterns,
// slots -- are already in place), scratch, status word, row descriptors
int init_device_update(spline_builder *h) {
    const sb::Plan &P = h->plan;
    auto bad = [&](cudaError_t e, const char *what) {
        return fail(e == cudaErrorMemoryAllocation ? SB_NOMEM : SB_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
    };
    cudaError_t e;
    if (h->stage_blob) { cudaFree(h->stage_blob); h->stage_blob = nullptr; }
    if ((e = cudaMalloc(&h->stage_blob, h->blob_bytes)) != cudaSuccess) return bad(e, "cudaMalloc(staging blob)");
    if ((e = cudaMemcpy(h->stage_blob, h->blob, h->blob_bytes, cudaMemcpyDeviceToDevice)) != cudaSuccess)
        return bad(e, "staging blob copy");
    if (!h->rf_scratch &&
        (e = cudaMalloc(&h->rf_scratch, sb::refactor_scratch_bytes(P.n, P.N, P.nQ, P.k, P.K))) != cudaSuccess)
        return bad(e, "cudaMalloc(refactor scratch)");
    if (!h->rf_status && (e = cudaMalloc(&h->rf_status, sizeof(int))) != cudaSuccess) return bad(e, "cudaMalloc(status)");
    if (!h->rf_status_host && (e = cudaMallocHost(&h->rf_status_host, sizeof(int))) != cudaSuccess)
        return bad(e, "cudaMallocHost(status)");
    *h->rf_status_host = 0;
    if (!h->rf_event && (e = cudaEventCreateWithFlags(&h->rf_event, cudaEventDisableTiming)) != cudaSuccess)
        return bad(e, "cudaEventCreate");
    std::vector<int> rd(3 * P.n);
    for (int i = 0; i < P.n; ++i) {
        rd[3 * i] = P.rowdesc[i].kind; rd[3 * i + 1] = P.rowdesc[i].idx; rd[3 * i + 2] = P.rowdesc[i].deriv;
    }
    if (h->rf_rowdesc) { cudaFree(h->rf_rowdesc); h->rf_rowdesc = nullptr; }
    if ((e = cudaMalloc(&h->rf_rowdesc, rd.size() * sizeof(int))) != cudaSuccess) return bad(e, "cudaMalloc(rowdesc)");
    if ((e = cudaMemcpy(h->rf_rowdesc, rd.data(), rd.size() * sizeof(int), cudaMemcpyHostToDevice)) != cudaSuccess)
        return bad(e, "rowdesc upload");
    if ((e = cudaStreamSynchronize(0)) != cudaSuccess) return bad(e, "device-update setup");
    h->x0 = P.xb.empty() ? 0.0 : P.xb[0];
    h->xN = P.xb.empty() ? 1.0 : P.xb[P.N];
    return SB_OK;
}

int do_solve(spline_builder *h, void *rhs, int dtype, int64_t batch, int64_t bstride, int64_t pstride,
             cudaStream_t stream, const double *shift = nullptr, int64_t nslab = 1, int64_t slab_stride = 0) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (h->host_only) return fail(SB_UNSUPPORTED, "handle was created with SB_FLAG_HOST_ONLY");
    if (dtype != SB_F64 && dtype != SB_F32) return fail(SB_INVALID_ARG, "dtype must be SB_F64 or SB_F32");
    if (batch < 0) return fail(SB_INVALID_ARG, "batch < 0");
    if (batch == 0) return SB_OK;
    if (!rhs) return fail(SB_INVALID_ARG, "rhs is NULL");
    if (bstride <= 0 || pstride <= 0) return fail(SB_INVALID_ARG, "strides must be positive");
    const int64_t n = h->plan.n;
    // one-to-one map (j, r) -> r*bstride + j*pstride for the two supported families
    bool ok = (bstride == 1 && pstride >= batch) || (pstride == 1 && bstride >= n) ||
              (bstride >= pstride * n) || (pstride >= bstride * batch);
    if (!ok) return fail(SB_INVALID_ARG, "strides alias: (row, rhs) -> offset is not one-to-one");
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != h->device) cudaSetDevice(h->device);
    sb::SolveArgs a{rhs, batch, bstride, pstride, dtype, stream, shift, nslab, slab_stride};
    char err[256] = {0};
    int st = sb::launch_solve(h->dp, a, h->num_sms, err, sizeof(err));
    if (cur != h->device) cudaSetDevice(cur);
    if (st) return fail(st, err);
    return SB_OK;
}

// slabs interleaved inside each row: columns [s*slab_stride, s*slab_stride+batch)
// of one (n, ld) batch-contiguous block; contiguous when slab_stride == batch
int do_solve_cols(spline_builder *h, void *rhs, int dtype, int64_t batch, int64_t ld, int64_t nslab,
                  int64_t slab_stride, cudaStream_t stream) {
    if (slab_stride == batch) return do_solve(h, rhs, dtype, nslab * batch, 1, ld, stream);
    const size_t esz = dtype == SB_F64 ? 8 : 4;
    for (int64_t sl = 0; sl < nslab; ++sl) {
        const int st = do_solve(h, (char *)rhs + (size_t)(sl * slab_stride) * esz, dtype, batch, 1, ld, stream);
        if (st) return st;
    }
    return SB_OK;
}

}  // namespace

extern "C" {

spline_builder_t spline_builder_create_ex(int degree, int n_points, int bc, const double *knots, int split_lo,
                                          int split_hi, int flags) {
    spline_builder *h = new (std::nothrow) spline_builder();
    if (!h) { fail(SB_NOMEM, "out of host memory"); return nullptr; }
    try {
        const int pflags = (flags & SB_FLAG_DEVICE_UPDATE) ? sb::PLAN_DEVICE_UPDATE : 0;
        sb::Status st = sb::build_plan(h->plan, degree, n_points, bc, knots, split_lo, split_hi, pflags);
        if (st.code) { fail(st.code, st.msg); delete h; return nullptr; }
    } catch (const std::bad_alloc &) {
        fail(SB_NOMEM, "out of host memory in create"); delete h; return nullptr;
    } catch (...) {
        fail(SB_INVALID_ARG, "unexpected failure in create"); delete h; return nullptr;
    }
    h->host_only = (flags & SB_FLAG_HOST_ONLY) != 0;
    h->dev_update = (flags & SB_FLAG_DEVICE_UPDATE) != 0;
    h->c_degree = degree; h->c_npoints = n_points; h->c_bc = bc; h->c_split_lo = split_lo; h->c_split_hi = split_hi;
    if (!h->host_only) {
        if (cudaGetDevice(&h->device) != cudaSuccess) { fail(SB_CUDA, "no CUDA device"); delete h; return nullptr; }
        cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, h->device);
        if (upload(h)) { spline_builder_destroy(h); return nullptr; }
        if (h->dev_update && init_device_update(h)) { spline_builder_destroy(h); return nullptr; }
    }
    return h;
}

int spline_builder_update(spline_builder_t h, const double *knots) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    sb::Plan fresh;
    try {
        sb::Status st = sb::build_plan(fresh, h->c_degree, h->c_npoints, h->c_bc, knots, h->c_split_lo, h->c_split_hi,
                                       h->dev_update ? sb::PLAN_DEVICE_UPDATE : 0);
        if (st.code) return fail(st.code, st.msg);
    } catch (const std::bad_alloc &) {
        return fail(SB_NOMEM, "out of host memory in update");
    } catch (...) {
        return fail(SB_INVALID_ARG, "unexpected failure in update");
    }
    if (h->host_only) { h->plan = std::move(fresh); return SB_OK; }
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != h->device) cudaSetDevice(h->device);
    // keep the old state until the new blob is on the device; restore it on failure
    sb::Plan old_plan = std::move(h->plan);
    void *old_blob = h->blob;
    size_t old_bytes = h->blob_bytes;
    sb::DevPlan old_dp = h->dp;
    h->plan = std::move(fresh);
    h->blob = nullptr;
    int rc = upload(h);  // synchronous cudaMemcpy: the new constants are in place on return
    if (rc) {
        if (h->blob) cudaFree(h->blob);
        h->plan = std::move(old_plan); h->blob = old_blob; h->blob_bytes = old_bytes; h->dp = old_dp;
        const std::string msg = g_err;
        if (cur != h->device) cudaSetDevice(cur);
        return fail(rc, msg);
    }
    if (old_blob) h->retired.push_back(old_blob);  // freed at destroy (graphs may still reference it)
    int rc2 = SB_OK;
    if (h->dev_update) rc2 = init_device_update(h);  // new layout: fresh staging copy
    if (cur != h->device) cudaSetDevice(cur);
    return rc2;
}

int spline_builder_update_device(spline_builder_t h, const double *knots, void *stream) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (h->host_only) return fail(SB_UNSUPPORTED, "handle was created with SB_FLAG_HOST_ONLY");
    if (!h->dev_update) return fail(SB_UNSUPPORTED, "handle was not created with SB_FLAG_DEVICE_UPDATE");
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != h->device) cudaSetDevice(h->device);
    sb::RefactorArgs a{};
    a.P = h->dp;
    a.p = h->plan.p;
    a.x0 = h->x0; a.xN = h->xN;
    a.knots = knots;
    a.rowdesc = h->rf_rowdesc;
    a.lam_ptr = h->dp.lam_ptr; a.lam_c = h->dp.lam_c; a.gam_r = h->dp.gam_r; a.gam_c = h->dp.gam_c;
    a.drow = h->dp.drow;
    a.scr = static_cast<double *>(h->rf_scratch);
    a.stage = static_cast<unsigned char *>(h->stage_blob);
    a.live = static_cast<unsigned char *>(h->blob);
    a.blob_bytes = h->blob_bytes / 16 * 16;
    a.status = h->rf_status;
    char err[256] = {0};
    const cudaStream_t st = (cudaStream_t)stream;
    int rc = sb::launch_refactor(a, st, err, sizeof(err));
    cudaError_t e = cudaSuccess;
    if (!rc) e = cudaMemcpyAsync(h->rf_status_host, h->rf_status, sizeof(int), cudaMemcpyDeviceToHost, st);
    if (!rc && e == cudaSuccess) e = cudaEventRecord(h->rf_event, st);
    if (cur != h->device) cudaSetDevice(cur);
    if (rc) return fail(rc, err);
    if (e != cudaSuccess) return fail(SB_CUDA, std::string("update_device: ") + cudaGetErrorString(e));
    h->rf_pending = true;
    return SB_OK;
}

int spline_builder_update_status(spline_builder_t h) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (!h->dev_update || !h->rf_pending) return SB_OK;
    const cudaError_t e = cudaEventSynchronize(h->rf_event);
    if (e != cudaSuccess) return fail(SB_CUDA, std::string("update_status: ") + cudaGetErrorString(e));
    h->rf_pending = false;
    switch (*h->rf_status_host) {
        case sb::SB_RF_OK: return SB_OK;
        case sb::SB_RF_BADKNOTS: return fail(SB_INVALID_ARG, "device update: breakpoints must be strictly increasing");
        case sb::SB_RF_DOMAIN: return fail(SB_INVALID_ARG, "device update: a periodic mesh must keep its end points");
        case sb::SB_RF_SINGULAR: return fail(SB_SINGULAR, "device update: Q or delta' could not be factored");
        case sb::SB_RF_CARRY:
            return fail(SB_UNSUPPORTED, "device update: the new mesh needs deeper segment carries than frozen at create");
        case sb::SB_RF_LAMBDA:
            return fail(SB_UNSUPPORTED, "device update: Lambda has entries above 1e-14 outside the pattern frozen at "
                                        "create (use spline_builder_update)");
        case sb::SB_RF_GAMMA:
            return fail(SB_UNSUPPORTED, "device update: gamma leaves the pattern frozen at create (use spline_builder_update)");
        case sb::SB_RF_BUCKETS:
            return fail(SB_UNSUPPORTED, "device update: the new cells are too small for the advection bucket table "
                                        "frozen at create (use spline_builder_update)");
        case sb::SB_RF_SCALED:
            return fail(SB_UNSUPPORTED, "device update: a derivative row fell into Q (use spline_builder_update)");
        default:
            return fail(SB_UNSUPPORTED, "device update: the new collocation matrix leaves the Q band frozen at create "
                                        "(use spline_builder_update)");
    }
}

spline_builder_t spline_builder_create(int degree, int n_points, int bc, const double *knots) {
    return spline_builder_create_ex(degree, n_points, bc, knots, -1, -1, 0);
}

int spline_builder_solve(spline_builder_t h, double *rhs, int64_t batch, int64_t batch_stride, void *stream) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (batch_stride == 1) return do_solve(h, rhs, SB_F64, batch, 1, batch, (cudaStream_t)stream);
    if (batch_stride >= h->plan.n) return do_solve(h, rhs, SB_F64, batch, batch_stride, 1, (cudaStream_t)stream);
    return fail(SB_INVALID_ARG, "batch_stride must be 1 or >= n (use spline_builder_solve_strided)");
}

int spline_builder_solve_f32(spline_builder_t h, float *rhs, int64_t batch, int64_t batch_stride, void *stream) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (batch_stride == 1) return do_solve(h, rhs, SB_F32, batch, 1, batch, (cudaStream_t)stream);
    if (batch_stride >= h->plan.n) return do_solve(h, rhs, SB_F32, batch, batch_stride, 1, (cudaStream_t)stream);
    return fail(SB_INVALID_ARG, "batch_stride must be 1 or >= n (use spline_builder_solve_strided)");
}

int spline_builder_solve_strided(spline_builder_t h, void *rhs, int dtype, int64_t batch, int64_t batch_stride,
                                 int64_t point_stride, void *stream) {
    return do_solve(h, rhs, dtype, batch, batch_stride, point_stride, (cudaStream_t)stream);
}

int spline_builder_advect(spline_builder_t h, void *f, int dtype, int64_t batch, int64_t batch_stride,
                          int64_t point_stride, const double *shift, void *stream) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (h->plan.bc != sb::PERIODIC) return fail(SB_UNSUPPORTED, "advect needs a periodic spline space");
    if (batch > 0 && !shift) return fail(SB_INVALID_ARG, "shift is NULL");
    return do_solve(h, f, dtype, batch, batch_stride, point_stride, (cudaStream_t)stream, shift);
}

int spline_builder_solve_slabs(spline_builder_t h, void *rhs, int dtype, int64_t batch, int64_t ld, int64_t nslab,
                               int64_t slab_stride, void *stream) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (nslab < 0) return fail(SB_INVALID_ARG, "nslab < 0");
    if (nslab == 0 || batch == 0) return SB_OK;
    if (ld < batch) return fail(SB_INVALID_ARG, "need ld >= batch");
    const int64_t n = h->plan.n;
    // one-to-one: slabs stacked (slab_stride >= n*ld) or interleaved inside each row
    const bool stacked = slab_stride >= n * ld;
    const bool inrow = slab_stride >= batch && ld >= (nslab - 1) * slab_stride + batch;
    if (nslab > 1 && !stacked && !inrow) return fail(SB_INVALID_ARG, "slabs alias: (row, rhs, slab) -> offset is not one-to-one");
    if (nslab > 1 && inrow && !stacked)  // one batch-contiguous block of nslab*slab_stride columns
        return do_solve_cols(h, rhs, dtype, batch, ld, nslab, slab_stride, (cudaStream_t)stream);
    return do_solve(h, rhs, dtype, batch, 1, ld, (cudaStream_t)stream, nullptr, nslab, nslab > 1 ? slab_stride : 0);
}

int spline_builder_solve_2d(spline_builder_t h1, spline_builder_t h2, void *rhs, int dtype, int64_t batch,
                            int64_t batch_stride, void *stream) {
    if (!h1 || !h2) return fail(SB_INVALID_ARG, "null handle");
    if (h1->host_only || h2->host_only) return fail(SB_UNSUPPORTED, "handle was created with SB_FLAG_HOST_ONLY");
    if (h1->device != h2->device) return fail(SB_INVALID_ARG, "the two handles live on different devices");
    if (dtype != SB_F64 && dtype != SB_F32) return fail(SB_INVALID_ARG, "dtype must be SB_F64 or SB_F32");
    if (batch < 0) return fail(SB_INVALID_ARG, "batch < 0");
    if (batch == 0) return SB_OK;
    if (!rhs) return fail(SB_INVALID_ARG, "rhs is NULL");
    const int64_t n1 = h1->plan.n, n2 = h2->plan.n, slice = n1 * n2;
    if (batch > 1 && batch_stride < slice) return fail(SB_INVALID_ARG, "need batch_stride >= n1*n2");
    if (batch == 1) batch_stride = slice;
    const size_t esz = dtype == SB_F64 ? 8 : 4;
    // Pass 1 (dim 1, contiguous rows) then pass 2 (dim 2, rows n1 apart), each one
    // launch over every grid (default).  SB_2D_CHUNK_MB > 0: chunked pipeline -- pass 1
    // of chunk c+1 on one internal stream while pass 2 of chunk c runs on the other
    // (event per chunk; fork/join with the caller's stream, so graph capture works),
    // so pass 2 would read a chunk pass 1 just left in L2.  Measured on C6 (64 grids
    // of 1024^2 fp64): unchunked 0.369 ms; 16 / 32 / 48 / 96 MB chunks 0.751 / 0.577 /
    // 0.502 / 0.448 ms -- every launch pays its pipeline fill and drain (constants
    // staged, first tile loaded before any compute, last tile's compute not overlapped),
    // which the L2 reuse does not repay (profiles/r02/ab_experiments.md).
    static const int64_t chunk_mb = [] {
        const char *e = getenv("SB_2D_CHUNK_MB");
        return e ? (int64_t)atoll(e) : (int64_t)0;
    }();
    auto pass1 = [&](void *base, int64_t nb, cudaStream_t st) {
        if (batch_stride == slice) return do_solve(h1, base, dtype, nb * n2, n1, 1, st);
        return do_solve(h1, base, dtype, n2, n1, 1, st, nullptr, nb, batch_stride);
    };
    auto pass2 = [&](void *base, int64_t nb, cudaStream_t st) {
        return do_solve(h2, base, dtype, n1, 1, n1, st, nullptr, nb, batch_stride);
    };
    const cudaStream_t cs = (cudaStream_t)stream;
    int64_t cb = batch;
    if (chunk_mb > 0) cb = std::max<int64_t>(1, (chunk_mb << 20) / (slice * (int64_t)esz));
    if (cb >= batch) {  // one chunk: the two passes back to back on the caller's stream
        int st = pass1(rhs, batch, cs);
        if (!st) st = pass2(rhs, batch, cs);
        return st;
    }
    std::lock_guard<std::mutex> lock(h1->pipe_mu);
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != h1->device) cudaSetDevice(h1->device);
    const int64_t nchunks = (batch + cb - 1) / cb;
    auto bad = [&](cudaError_t e) {
        if (cur != h1->device) cudaSetDevice(cur);
        return fail(SB_CUDA, std::string("2-D pipeline: ") + cudaGetErrorString(e));
    };
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < 2 && e == cudaSuccess; ++i)
        if (!h1->pipe[i]) e = cudaStreamCreateWithFlags(&h1->pipe[i], cudaStreamNonBlocking);
    while (e == cudaSuccess && (int64_t)h1->pipe_ev.size() < nchunks + 3) {
        cudaEvent_t ev;
        e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
        if (e == cudaSuccess) h1->pipe_ev.push_back(ev);
    }
    if (e != cudaSuccess) return bad(e);
    cudaEvent_t *ev = h1->pipe_ev.data();  // [0] fork, [1] join A, [2] join B, [3 + c] pass 1 of chunk c done
    const cudaStream_t sA = h1->pipe[0], sB = h1->pipe[1];
    if ((e = cudaEventRecord(ev[0], cs)) != cudaSuccess) return bad(e);
    if ((e = cudaStreamWaitEvent(sA, ev[0], 0)) != cudaSuccess || (e = cudaStreamWaitEvent(sB, ev[0], 0)) != cudaSuccess)
        return bad(e);
    int st = SB_OK;
    for (int64_t c = 0; c < nchunks && !st; ++c) {
        const int64_t b0 = c * cb, nb = std::min(cb, batch - b0);
        void *base = (char *)rhs + (size_t)(b0 * batch_stride) * esz;
        st = pass1(base, nb, sA);
        if (st) break;
        if ((e = cudaEventRecord(ev[3 + c], sA)) != cudaSuccess || (e = cudaStreamWaitEvent(sB, ev[3 + c], 0)) != cudaSuccess)
            return bad(e);
        st = pass2(base, nb, sB);
    }
    // join (also after a failed launch, so the caller's stream never runs ahead)
    if ((e = cudaEventRecord(ev[1], sA)) != cudaSuccess || (e = cudaEventRecord(ev[2], sB)) != cudaSuccess ||
        (e = cudaStreamWaitEvent(cs, ev[1], 0)) != cudaSuccess || (e = cudaStreamWaitEvent(cs, ev[2], 0)) != cudaSuccess)
        return bad(e);
    if (cur != h1->device) cudaSetDevice(cur);
    return st;
}

int spline_builder_solve_host(spline_builder_t h, void *host_rhs, int dtype, int64_t batch, int64_t ld) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    if (h->host_only) return fail(SB_UNSUPPORTED, "handle was created with SB_FLAG_HOST_ONLY");
    if (dtype != SB_F64 && dtype != SB_F32) return fail(SB_INVALID_ARG, "dtype must be SB_F64 or SB_F32");
    if (batch < 0 || ld < batch) return fail(SB_INVALID_ARG, "need 0 <= batch <= ld");
    if (batch == 0) return SB_OK;
    if (!host_rhs) return fail(SB_INVALID_ARG, "host_rhs is NULL");
    std::lock_guard<std::mutex> lock(h->host_mu);
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != h->device) cudaSetDevice(h->device);
    const size_t esz = dtype == SB_F64 ? 8 : 4;
    const int64_t n = h->plan.n;
    // chunk of RHS per pipeline stage: ~16 MB (SB_HOST_CHUNK_MB), multiple of 16 columns.
    // Measured (C2, 800 + 800 MB per step over PCIe, whose copy ceiling is 16.1 ms):
    // e2e 5.53-5.59e6 RHS/s at 16 MB vs 5.16e6 at 64 MB and 4.90e6 at 128 MB (shorter
    // pipeline fill and drain); 4-12 MB were no better (profiles/r02/ab_experiments.md)
    static const int64_t chunk_mb = [] {
        const char *e = getenv("SB_HOST_CHUNK_MB");
        return e && atoll(e) > 0 ? (int64_t)atoll(e) : (int64_t)16;
    }();
    int64_t chunk = std::max<int64_t>(16, ((int64_t)(chunk_mb << 20) / (n * (int64_t)esz)) / 16 * 16);
    chunk = std::min<int64_t>(chunk, (batch + 15) / 16 * 16);
    const size_t need = (size_t)chunk * n * esz;
    int rc = SB_OK;
    if (need > h->stage_bytes) {
        for (int i = 0; i < 3; ++i) { if (h->stage[i]) cudaFree(h->stage[i]); h->stage[i] = nullptr; }
        h->stage_bytes = 0;
        for (int i = 0; i < 3; ++i)
            if (cudaMalloc(&h->stage[i], need) != cudaSuccess) rc = fail(SB_NOMEM, "cudaMalloc(staging) failed");
        if (rc) {
            for (int i = 0; i < 3; ++i) { if (h->stage[i]) cudaFree(h->stage[i]); h->stage[i] = nullptr; }
        } else {
            h->stage_bytes = need;
        }
    }
    for (int i = 0; i < 3 && !rc; ++i)
        if (!h->streams[i] && cudaStreamCreateWithFlags(&h->streams[i], cudaStreamNonBlocking) != cudaSuccess)
            rc = fail(SB_CUDA, "cudaStreamCreate failed");
    unsigned char *host = static_cast<unsigned char *>(host_rhs);
    for (int64_t c0 = 0, it = 0; c0 < batch && !rc; c0 += chunk, ++it) {
        const int64_t w = std::min<int64_t>(chunk, batch - c0);
        const int si = (int)(it % 3);
        cudaStream_t st = h->streams[si];
        void *dbuf = h->stage[si];
        cudaError_t e = cudaMemcpy2DAsync(dbuf, w * esz, host + c0 * esz, ld * esz, w * esz, n,
                                          cudaMemcpyHostToDevice, st);
        if (e != cudaSuccess) { rc = fail(SB_CUDA, std::string("H2D: ") + cudaGetErrorString(e)); break; }
        int s = do_solve(h, dbuf, dtype, w, 1, w, st);
        if (s) { rc = s; break; }
        e = cudaMemcpy2DAsync(host + c0 * esz, ld * esz, dbuf, w * esz, w * esz, n, cudaMemcpyDeviceToHost, st);
        if (e != cudaSuccess) { rc = fail(SB_CUDA, std::string("D2H: ") + cudaGetErrorString(e)); break; }
    }
    for (int i = 0; i < 3; ++i)
        if (h->streams[i]) {
            cudaError_t e = cudaStreamSynchronize(h->streams[i]);
            if (e != cudaSuccess && !rc) rc = fail(SB_CUDA, std::string("solve_host: ") + cudaGetErrorString(e));
        }
    if (cur != h->device) cudaSetDevice(cur);
    return rc;
}

void spline_builder_destroy(spline_builder_t h) {
    if (!h) return;
    if (!h->host_only) {
        int cur = -1;
        cudaGetDevice(&cur);
        if (h->device >= 0 && cur != h->device) cudaSetDevice(h->device);
        if (h->blob) cudaFree(h->blob);
        for (void *b : h->retired) cudaFree(b);
        for (int i = 0; i < 2; ++i)
            if (h->pipe[i]) cudaStreamDestroy(h->pipe[i]);
        for (cudaEvent_t e : h->pipe_ev) cudaEventDestroy(e);
        if (h->stage_blob) cudaFree(h->stage_blob);
        if (h->rf_scratch) cudaFree(h->rf_scratch);
        if (h->rf_status) cudaFree(h->rf_status);
        if (h->rf_rowdesc) cudaFree(h->rf_rowdesc);
        if (h->rf_status_host) cudaFreeHost(h->rf_status_host);
        if (h->rf_event) cudaEventDestroy(h->rf_event);
        for (int i = 0; i < 3; ++i) {
            if (h->stage[i]) cudaFree(h->stage[i]);
            if (h->streams[i]) cudaStreamDestroy(h->streams[i]);
        }
        if (h->device >= 0 && cur != h->device) cudaSetDevice(cur);
    }
    delete h;
}

int spline_builder_get_info(spline_builder_t h, spline_builder_info_t *info) {
    if (!h || !info) return fail(SB_INVALID_ARG, "null argument");
    const sb::Plan &P = h->plan;
    info->degree = P.p; info->bc = P.bc; info->n_cells = P.N; info->nbasis = P.n;
    info->split_lo = P.s_lo; info->split_hi = P.s_hi; info->k = P.k;
    info->q_kl = P.kl; info->q_ku = P.ku; info->q_type = P.qtype;
    info->nnz_lambda = (int)P.lam_v.size(); info->nnz_beta = (int)P.beta_v.size();
    int head = 0, tail = 0;
    for (int r : P.beta_r) { if (r < P.nQ / 2) head = std::max(head, r + 1); else tail = std::max(tail, P.nQ - r); }
    info->beta_rows_head = head; info->beta_rows_tail = tail;
    info->nnz_Lambda = (int)P.Lam_v.size(); info->nnz_gamma = (int)P.gam_v.size();
    info->n_segments = P.seg[0].S; info->seg_len = P.seg[0].L;
    info->carry_fwd = P.seg[0].carry_f; info->carry_bwd = P.seg[0].carry_b;
    info->max_pivot_growth = P.growth;
    return SB_OK;
}

int64_t spline_builder_nbasis(spline_builder_t h) { return h ? h->plan.n : -1; }

int spline_builder_get_blocks(spline_builder_t h, int *lam_rows, int *lam_cols, double *lam_vals, int *beta_rows,
                              int *beta_cols, double *beta_vals, double *delta_prime) {
    if (!h) return fail(SB_INVALID_ARG, "null handle");
    const sb::Plan &P = h->plan;
    for (size_t e = 0; e < P.lam_v.size(); ++e) {
        if (lam_rows) lam_rows[e] = P.lam_r[e];
        if (lam_cols) lam_cols[e] = P.lam_c[e];
        if (lam_vals) lam_vals[e] = P.lam_v[e];
    }
    for (size_t e = 0; e < P.beta_v.size(); ++e) {
        if (beta_rows) beta_rows[e] = P.beta_r[e];
        if (beta_cols) beta_cols[e] = P.beta_c[e];
        if (beta_vals) beta_vals[e] = P.beta_v[e];
    }
    if (delta_prime && !P.dprime.empty()) std::memcpy(delta_prime, P.dprime.data(), P.dprime.size() * sizeof(double));
    return SB_OK;
}

int spline_builder_solve_cpu_plan(spline_builder_t h, double *rhs, int64_t batch, int64_t batch_stride,
                                  int64_t point_stride) {
    if (!h || !rhs || batch < 0) return fail(SB_INVALID_ARG, "bad argument");
    sb::plan_solve_cpu(h->plan, rhs, batch, batch_stride, point_stride);
    return SB_OK;
}

const char *spline_builder_last_error(void) { return g_err.c_str(); }
const char *spline_builder_last_kernel(void) { return sb::last_kernel(); }
int spline_builder_last_status(void) { return g_status; }
const char *spline_builder_version(void) { return "b200-spline-build 0.1 (sm_100a)"; }

}  // extern "C"
