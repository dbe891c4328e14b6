// plan.cpp -- host create step (see plan.hpp).
//
// Collocation matrix: span-based de Boor triangular scheme (BSPLVB) and its
// derivative extension, evaluated in local (cell-relative) coordinates: every
// knot difference is a sum of cell widths and every point is (span, offset).
// Schur split / factorisation / corners: PAPER.md Eq. 3-6, Table I
// (P:95-101), COO corners (Listing 5-6).
#include "plan.hpp"

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <map>
#include <random>

namespace sb {
namespace {

long lmod(long a, long m) {
    long r = a % m;
    return r < 0 ? r + m : r;
}

struct Space {
    int p, bc, N, n, nbc;
    const double *h;

    double width(long g) const {
        if (bc == PERIODIC) return h[lmod(g, N)];
        return (g >= p && g < N + p) ? h[g - p] : 0.0;
    }
    // t_a - t_b (a >= b) as a sum of interval widths
    double kd(long a, long b) const {
        double s = 0.0;
        for (long g = b; g < a; ++g) s += width(g);
        return s;
    }
    long first_knot(int j) const { return bc == PERIODIC ? j - (p + 1) / 2 : j; }
    int basis_of(long q) const { return bc == PERIODIC ? (int)lmod(q + (p + 1) / 2, N) : (int)q; }
    long span_of_cell(int c) const { return bc == PERIODIC ? c : (long)c + p; }
};

struct RowPt {
    long span;  // knot interval index containing the point
    double u;   // offset from t_span
    int deriv;
};

// BSPLVB (de Boor): values of the q+1 degree-q B-splines with first knots
// span-q .. span at x = t_span + u.
void bsplvb(const Space &S, long mu, double u, int q, double *b) {
    double dl[16], dr[16];
    b[0] = 1.0;
    for (int j = 0; j < q; ++j) {
        dr[j] = S.kd(mu + 1 + j, mu) - u;
        dl[j] = u + S.kd(mu, mu - j);
        double saved = 0.0;
        for (int r = 0; r <= j; ++r) {
            double den = dr[r] + dl[j - r];
            double term = den > 0.0 ? b[r] / den : 0.0;
            b[r] = saved + dr[r] * term;
            saved = dl[j - r] * term;
        }
        b[j + 1] = saved;
    }
}

// d-th derivative of the p+1 degree-p B-splines with first knots span-p..span:
// values of degree p-d, then d applications of
//   D B_{i,q} = q (B_{i,q-1}/(t_{i+q}-t_i) - B_{i+1,q-1}/(t_{i+q+1}-t_{i+1})).
void bsplvd(const Space &S, long mu, double u, int d, double *out) {
    const int p = S.p;
    double v[16], w[16];
    bsplvb(S, mu, u, p - d, v);
    for (int q = p - d + 1; q <= p; ++q) {
        for (int r = 0; r <= q; ++r) {
            long i = mu - q + r;
            double acc = 0.0;
            if (r - 1 >= 0) {
                double den = S.kd(i + q, i);
                if (den > 0.0) acc += v[r - 1] / den;
            }
            if (r <= q - 1) {
                double den = S.kd(i + q + 1, i + 1);
                if (den > 0.0) acc -= v[r] / den;
            }
            w[r] = q * acc;
        }
        for (int r = 0; r <= q; ++r) v[r] = w[r];
    }
    for (int r = 0; r <= p; ++r) out[r] = v[r];
}

// Greville abscissa (t_{q+1}+...+t_{q+p})/p of the basis with first knot q,
// located as (span, u); the closed right end of the last interval is kept.
RowPt greville(const Space &S, int j) {
    long q = S.first_knot(j);
    double off = 0.0;
    for (int l = 1; l <= S.p; ++l) off += S.kd(q + l, q);
    off /= S.p;
    // snap to a knot when within rounding of it (uniform odd degree: the
    // Greville point IS a knot), so structural zeros of A stay exact
    {
        const double span = S.kd(q + S.p + 1, q);
        for (int l = 0; l <= S.p + 1; ++l) {
            const double t = S.kd(q + l, q);
            if (std::fabs(off - t) <= 8.0 * 2.220446049250313e-16 * span) { off = t; break; }
        }
    }
    long last = -1;
    double lastlo = 0.0;
    for (int l = 0; l <= S.p; ++l) {
        long g = q + l;
        double w = S.width(g);
        if (w <= 0.0) continue;
        double lo = S.kd(g, q);
        last = g;
        lastlo = lo;
        if (off >= lo && off < lo + w) return RowPt{g, off - lo, 0};
    }
    return RowPt{last, off - lastlo, 0};
}

double dmax_abs(const std::vector<double> &v) {
    double m = 0.0;
    for (double x : v) m = std::max(m, std::fabs(x));
    return m;
}

struct SplitResult {
    int code = 0;
    std::string msg;
};

// try one Schur split; fills P on success
SplitResult try_split(Plan &P, int slo, int shi) {
    SplitResult R;
    const int n = P.n;
    const int k = slo + shi;
    if (slo < 0 || shi < 0 || k > KMAX_DELTA || k > n) return {1, "split out of range"};
    const int nQ = n - k;
    // every equilibrated (scaled) row must be a delta row (kernel reads Q rows unscaled)
    for (int i = slo; i < n - shi; ++i)
        if (P.rowscale[i] != 1.0) return {1, "scaled (Hermite derivative) row inside Q"};
    auto dindex = [&](int g) { return g < slo ? g : (g >= n - shi ? slo + (g - (n - shi)) : -1); };
    // Q band
    int kl = 0, ku = 0;
    for (int i = 0; i < nQ; ++i) {
        const SparseRow &row = P.A[slo + i];
        for (size_t e = 0; e < row.col.size(); ++e) {
            int c = row.col[e];
            if (c < slo || c >= n - shi || (row.val[e] == 0.0 && !P.dev_update)) continue;
            int o = (c - slo) - i;
            kl = std::max(kl, -o);
            ku = std::max(ku, o);
        }
    }
    if (kl > KMAX_BAND || ku > KMAX_BAND) return {5, "Q band too wide"};
    const int K = std::max(1, std::max(kl, ku));
    // dense band of Q: Qb[i*(2K+1) + (o+K)]
    const int BW = 2 * K + 1;
    std::vector<double> Qb((size_t)nQ * BW, 0.0);
    std::vector<double> gam((size_t)nQ * k, 0.0), lam((size_t)k * nQ, 0.0), del((size_t)k * k, 0.0);
    for (int g = 0; g < n; ++g) {
        const SparseRow &row = P.A[g];
        int dg = dindex(g);
        for (size_t e = 0; e < row.col.size(); ++e) {
            int c = row.col[e];
            double v = row.val[e];
            int dc = dindex(c);
            if (dg < 0 && dc < 0) Qb[(size_t)(g - slo) * BW + ((c - slo) - (g - slo) + K)] += v;
            else if (dg < 0) gam[(size_t)(g - slo) * k + dc] += v;
            else if (dc < 0) lam[(size_t)dg * nQ + (c - slo)] += v;
            else del[(size_t)dg * k + dc] += v;
        }
    }
    auto Q = [&](int i, int j) -> double & { return Qb[(size_t)i * BW + (j - i + K)]; };
    const double qmax = dmax_abs(Qb);
    std::vector<double> Lb((size_t)nQ * K, 0.0), Ub((size_t)nQ * K, 0.0), dinv(nQ, 0.0);
    int qtype = Q_GBTRS;
    double growth = 1.0;
    bool done = false;
    if (nQ > 0) {
        // symmetric up to rounding of the entries?  (PAPER Table I: uniform -> PDS; the
        // LDL^T below reads the lower triangle, the self-check bounds the effect)
        bool sym = true;
        for (int i = 0; i < nQ && sym; ++i)
            for (int m = 1; m <= K && i + m < nQ; ++m)
                if (std::fabs(Q(i, i + m) - Q(i + m, i)) > 1e-13 * qmax) { sym = false; break; }
        if (sym) {
            // banded LDL^T (pttrf for K=1, pbtrf-equivalent otherwise), no pivoting
            std::vector<double> L((size_t)nQ * K, 0.0), d(nQ, 0.0);  // L[i*K+m-1] = L(i,i-m)
            bool pd = true;
            for (int j = 0; j < nQ && pd; ++j) {
                double dj = Q(j, j);
                for (int m = 1; m <= K && j - m >= 0; ++m) dj -= L[(size_t)j * K + m - 1] * L[(size_t)j * K + m - 1] * d[j - m];
                if (!(dj > 0.0)) { pd = false; break; }
                d[j] = dj;
                for (int i = j + 1; i <= j + K && i < nQ; ++i) {
                    double v = Q(i, j);
                    // sum over c < j inside both bands: L(i,c) L(j,c) d_c
                    for (int c = std::max(0, i - K); c < j; ++c) {
                        if (j - c > K) continue;
                        v -= L[(size_t)i * K + (i - c) - 1] * L[(size_t)j * K + (j - c) - 1] * d[c];
                    }
                    L[(size_t)i * K + (i - j) - 1] = v / dj;
                }
            }
            if (pd) {
                for (int i = 0; i < nQ; ++i) {
                    dinv[i] = 1.0 / d[i];
                    for (int m = 1; m <= K; ++m) {
                        Lb[(size_t)i * K + m - 1] = L[(size_t)i * K + m - 1];
                        Ub[(size_t)i * K + m - 1] = (i + m < nQ) ? L[(size_t)(i + m) * K + m - 1] : 0.0;
                    }
                }
                qtype = (K == 1) ? Q_PTTRS : Q_PBTRS;
                growth = 1.0;
                done = true;
            }
        }
        if (!done) {
            // banded LU without row interchanges (gbtrf path).  Accepted only if
            // it is stable here (collocation matrices are totally positive, so
            // elimination without pivoting is stable; R5).
            std::vector<double> W = Qb;
            auto Wa = [&](int i, int j) -> double & { return W[(size_t)i * BW + (j - i + K)]; };
            double lmax = 0.0, umax = 0.0;
            for (int j = 0; j < nQ; ++j) {
                double piv = Wa(j, j);
                if (!(std::fabs(piv) > 1e-13 * qmax)) return {2, "zero pivot in Q"};
                for (int i = j + 1; i <= std::min(nQ - 1, j + kl); ++i) {
                    double l = Wa(i, j) / piv;
                    Wa(i, j) = l;
                    lmax = std::max(lmax, std::fabs(l));
                    if (l != 0.0)
                        for (int c = j + 1; c <= std::min(nQ - 1, j + ku); ++c) Wa(i, c) -= l * Wa(j, c);
                }
            }
            for (int i = 0; i < nQ; ++i)
                for (int c = i; c <= std::min(nQ - 1, i + ku); ++c) umax = std::max(umax, std::fabs(Wa(i, c)));
            growth = umax / qmax;
            if (lmax > 1e3 || growth > 1e3) return {2, "no-pivot LU of Q unstable"};
            for (int i = 0; i < nQ; ++i) {
                double u = Wa(i, i);
                dinv[i] = 1.0 / u;
                for (int m = 1; m <= K; ++m) {
                    Lb[(size_t)i * K + m - 1] = (i - m >= 0 && m <= kl) ? Wa(i, i - m) : 0.0;
                    Ub[(size_t)i * K + m - 1] = (i + m < nQ && m <= ku) ? Wa(i, i + m) / u : 0.0;
                }
            }
            qtype = Q_GBTRS;
        }
    }
    // banded solves with the factors: Q v = w (in place) and Q^T v = w
    auto qsolve = [&](std::vector<double> &v) {
        for (int i = 0; i < nQ; ++i)
            for (int m = 1; m <= K && i - m >= 0; ++m) v[i] -= Lb[(size_t)i * K + m - 1] * v[i - m];
        for (int i = nQ - 1; i >= 0; --i) {
            double acc = v[i] * dinv[i];
            for (int m = 1; m <= K && i + m < nQ; ++m) acc -= Ub[(size_t)i * K + m - 1] * v[i + m];
            v[i] = acc;
        }
    };
    // Q = L D (I + U'),  Q^T = (I + U')^T D L^T
    auto qtsolve = [&](std::vector<double> &v) {
        for (int j = 0; j < nQ; ++j)
            for (int m = 1; m <= K && j - m >= 0; ++m) v[j] -= Ub[(size_t)(j - m) * K + m - 1] * v[j - m];
        for (int j = 0; j < nQ; ++j) v[j] *= dinv[j];
        for (int j = nQ - 1; j >= 0; --j)
            for (int m = 1; m <= K && j + m < nQ; ++m) v[j] -= Lb[(size_t)(j + m) * K + m - 1] * v[j + m];
    };
    // beta = Q^{-1} gamma (Eq. 4), one banded solve per delta column
    std::vector<double> beta((size_t)nQ * k, 0.0), v(nQ);
    for (int c = 0; c < k; ++c) {
        for (int i = 0; i < nQ; ++i) v[i] = gam[(size_t)i * k + c];
        qsolve(v);
        for (int i = 0; i < nQ; ++i) beta[(size_t)i * k + c] = v[i];
    }
    // Lambda = lambda Q^{-1} (transposed twin of beta): Lambda_d^T = Q^{-T} lambda_d^T
    std::vector<double> Lam((size_t)k * nQ, 0.0);
    for (int d = 0; d < k; ++d) {
        for (int i = 0; i < nQ; ++i) v[i] = lam[(size_t)d * nQ + i];
        qtsolve(v);
        for (int i = 0; i < nQ; ++i) Lam[(size_t)d * nQ + i] = v[i];
    }
    // delta' = delta - lambda beta (Eq. 4)
    std::vector<double> dp = del;
    for (int r = 0; r < k; ++r)
        for (int c = 0; c < k; ++c) {
            double acc = 0.0;
            for (int i = 0; i < nQ; ++i) acc += lam[(size_t)r * nQ + i] * beta[(size_t)i * k + c];
            dp[(size_t)r * k + c] -= acc;
        }
    // getrf(delta') with partial pivoting (first max, like idamax)
    std::vector<double> lu = dp;
    std::vector<int> piv(k);
    double dmax = dmax_abs(dp);
    for (int j = 0; j < k; ++j) {
        int pr = j;
        double best = std::fabs(lu[(size_t)j * k + j]);
        for (int i = j + 1; i < k; ++i)
            if (std::fabs(lu[(size_t)i * k + j]) > best) { best = std::fabs(lu[(size_t)i * k + j]); pr = i; }
        piv[j] = pr;
        if (!(best > 1e-13 * dmax)) return {2, "delta' singular"};
        if (pr != j)
            for (int c = 0; c < k; ++c) std::swap(lu[(size_t)j * k + c], lu[(size_t)pr * k + c]);
        for (int i = j + 1; i < k; ++i) {
            double l = lu[(size_t)i * k + j] / lu[(size_t)j * k + j];
            lu[(size_t)i * k + j] = l;
            for (int c = j + 1; c < k; ++c) lu[(size_t)i * k + c] -= l * lu[(size_t)j * k + c];
        }
    }
    // commit
    P.s_lo = slo; P.s_hi = shi; P.k = k; P.nQ = nQ;
    P.drow.resize(k);
    for (int d = 0; d < k; ++d) P.drow[d] = d < slo ? d : n - shi + (d - slo);
    P.kl = kl; P.ku = ku; P.K = K; P.qtype = qtype; P.growth = growth;
    P.Lb.swap(Lb); P.Ub.swap(Ub); P.dinv.swap(dinv);
    P.dprime = dp; P.dlu.swap(lu); P.dpiv.swap(piv);
    P.lam_r.clear(); P.lam_c.clear(); P.lam_v.clear();
    for (int r = 0; r < k; ++r)
        for (int i = 0; i < nQ; ++i)
            if (lam[(size_t)r * nQ + i] != 0.0) {
                P.lam_r.push_back(r); P.lam_c.push_back(i); P.lam_v.push_back(lam[(size_t)r * nQ + i]);
            }
    P.gam_r.clear(); P.gam_c.clear(); P.gam_v.clear();
    // PLAN_DEVICE_UPDATE: the gamma pattern is frozen at create, so it covers every
    // delta column of the rows within CORNER_MARGIN of a structural nonzero (a new
    // mesh may move a collocation point into a neighbouring span)
    std::vector<char> grow(nQ, 0);
    for (int i = 0; i < nQ; ++i)
        for (int c = 0; c < k; ++c)
            if (gam[(size_t)i * k + c] != 0.0) grow[i] = 1;
    if (P.dev_update) {
        std::vector<char> g2(nQ, 0);
        for (int i = 0; i < nQ; ++i)
            if (grow[i])
                for (int j = std::max(0, i - CORNER_MARGIN); j <= std::min(nQ - 1, i + CORNER_MARGIN); ++j) g2[j] = 1;
        grow.swap(g2);
    }
    for (int i = 0; i < nQ; ++i)
        for (int c = 0; c < k; ++c)
            if (gam[(size_t)i * k + c] != 0.0 || (P.dev_update && grow[i])) {
                P.gam_r.push_back(i); P.gam_c.push_back(c); P.gam_v.push_back(gam[(size_t)i * k + c]);
            }
    P.beta_r.clear(); P.beta_c.clear(); P.beta_v.clear();
    for (int i = 0; i < nQ; ++i)
        for (int c = 0; c < k; ++c) {
            double b = beta[(size_t)i * k + c];
            if (std::fabs(b) > CORNER_DROP) { P.beta_r.push_back(i); P.beta_c.push_back(c); P.beta_v.push_back(b); }
        }
    P.Lam_ptr.assign(k + 1, 0); P.Lam_c.clear(); P.Lam_v.clear();
    // PLAN_DEVICE_UPDATE: one frozen column set for every row of Lambda (the union
    // of the rows' columns above the threshold, dilated by CORNER_MARGIN columns):
    // a row whose entries at one end fall just under 1e-14 on this mesh may have
    // them above it on the next
    std::vector<char> uni(nQ, 0);
    if (P.dev_update)
        for (int d = 0; d < k; ++d)
            for (int i = 0; i < nQ; ++i)
                if (std::fabs(Lam[(size_t)d * nQ + i]) > CORNER_DROP)
                    for (int j = std::max(0, i - CORNER_MARGIN); j <= std::min(nQ - 1, i + CORNER_MARGIN); ++j) uni[j] = 1;
    for (int d = 0; d < k; ++d) {
        for (int i = 0; i < nQ; ++i)
            if (P.dev_update ? uni[i] != 0 : std::fabs(Lam[(size_t)d * nQ + i]) > CORNER_DROP) {
                P.Lam_c.push_back(i);
                P.Lam_v.push_back(Lam[(size_t)d * nQ + i]);
            }
        P.Lam_ptr[d + 1] = (int)P.Lam_c.size();
    }
    return R;
}

// segment partition of the padded Q for register segment length L: transfer
// matrices of each segment and the carry-walk depths.
void build_segplan(const Plan &P, SegPlan &G, int L) {
    const int nQ = P.nQ, K = P.K;
    G.L = L;
    G.S = nQ > 0 ? (nQ + L - 1) / L : 1;
    G.nQp = G.S * L;
    const int S = G.S;
    auto Lf = [&](int row, int m) { return row < nQ ? P.Lb[(size_t)row * K + m - 1] : 0.0; };  // pad: identity
    auto Uf = [&](int row, int m) { return row < nQ ? P.Ub[(size_t)row * K + m - 1] : 0.0; };
    G.G.assign((size_t)S * K * K, 0.0);
    G.H.assign((size_t)S * K * K, 0.0);
    std::vector<double> y(L + 2 * K);
    for (int t = 1; t < S; ++t) {  // forward: segment t's response to inflow unit m, at rows a+L-1-j
        const int a = t * L;
        for (int m = 1; m <= K; ++m) {
            std::fill(y.begin(), y.end(), 0.0);
            y[K - m] = 1.0;  // y[K+i] = y_{a+i}
            for (int i = 0; i < L; ++i) {
                double acc = 0.0;
                for (int mm = 1; mm <= K; ++mm) acc -= Lf(a + i, mm) * y[K + i - mm];
                y[K + i] = acc;
            }
            for (int j = 0; j < K; ++j) G.G[((size_t)t * K + j) * K + (m - 1)] = y[K + L - 1 - j];
        }
    }
    for (int t = 0; t + 1 < S; ++t) {  // backward: response to outflow unit m, at rows a+j
        const int a = t * L;
        for (int m = 1; m <= K; ++m) {
            std::fill(y.begin(), y.end(), 0.0);
            y[L + m - 1] = 1.0;  // y[i] = x_{a+i}
            for (int i = L - 1; i >= 0; --i) {
                double acc = 0.0;
                for (int mm = 1; mm <= K; ++mm) acc -= Uf(a + i, mm) * y[i + mm];
                y[i] = acc;
            }
            for (int j = 0; j < K; ++j) G.H[((size_t)t * K + j) * K + (m - 1)] = y[j];
        }
    }
    // carry depths: smallest T with prod ||transfer||_inf <= 2^-60, or an exact end
    const double eps = std::ldexp(1.0, -60);
    auto nrm = [&](const std::vector<double> &M, int t) {
        double r = 0.0;
        for (int j = 0; j < K; ++j) {
            double s = 0.0;
            for (int m = 0; m < K; ++m) s += std::fabs(M[((size_t)t * K + j) * K + m]);
            r = std::max(r, s);
        }
        return r;
    };
    G.carry_f = 0;
    for (int s = 1; s < S; ++s) {
        int T = 0;
        double prod = 1.0;
        while (true) {
            ++T;
            int t = s - T;
            if (t == 0) break;
            prod *= nrm(G.G, t);
            if (prod <= eps) break;
        }
        G.carry_f = std::max(G.carry_f, T + (P.dev_update && T < s ? 1 : 0));  // device update: one deeper
    }
    G.carry_b = 0;
    for (int s = 0; s + 1 < S; ++s) {
        int T = 0;
        double prod = 1.0;
        while (true) {
            ++T;
            int t = s + T;
            if (t == S - 1) break;
            prod *= nrm(G.H, t);
            if (prod <= eps) break;
        }
        G.carry_b = std::max(G.carry_b, T + (P.dev_update && s + T < S - 1 ? 1 : 0));
    }
}

}  // namespace

void plan_solve_cpu(const Plan &P, double *rhs, int64_t batch, int64_t bstride, int64_t pstride) {
    const int nQ = P.nQ, k = P.k, K = P.K;
    std::vector<double> v(nQ), x1(k);
    for (int64_t r = 0; r < batch; ++r) {
        double *col = rhs + r * bstride;
        for (int i = 0; i < nQ; ++i) v[i] = col[(int64_t)(P.s_lo + i) * pstride];
        // x1 = delta'^{-1} (b1 - Lambda b0),  Lambda = lambda Q^{-1}
        for (int d = 0; d < k; ++d) {
            double acc = col[(int64_t)P.drow[d] * pstride] * P.rowscale[P.drow[d]];
            for (int e = P.Lam_ptr[d]; e < P.Lam_ptr[d + 1]; ++e) acc -= P.Lam_v[e] * v[P.Lam_c[e]];
            x1[d] = acc;
        }
        for (int d = 0; d < k; ++d)
            if (P.dpiv[d] != d) std::swap(x1[d], x1[P.dpiv[d]]);
        for (int i = 1; i < k; ++i)
            for (int j = 0; j < i; ++j) x1[i] -= P.dlu[(size_t)i * k + j] * x1[j];
        for (int i = k - 1; i >= 0; --i) {
            for (int j = i + 1; j < k; ++j) x1[i] -= P.dlu[(size_t)i * k + j] * x1[j];
            x1[i] /= P.dlu[(size_t)i * k + i];
        }
        // x0 = Q^{-1} (b0 - gamma x1)
        for (size_t e = 0; e < P.gam_v.size(); ++e) v[P.gam_r[e]] -= P.gam_v[e] * x1[P.gam_c[e]];
        for (int i = 0; i < nQ; ++i)
            for (int m = 1; m <= K && i - m >= 0; ++m) v[i] -= P.Lb[(size_t)i * K + m - 1] * v[i - m];
        for (int i = nQ - 1; i >= 0; --i) {
            double acc = v[i] * P.dinv[i];
            for (int m = 1; m <= K && i + m < nQ; ++m) acc -= P.Ub[(size_t)i * K + m - 1] * v[i + m];
            v[i] = acc;
        }
        for (int i = 0; i < nQ; ++i) col[(int64_t)(P.s_lo + i) * pstride] = v[i];
        for (int d = 0; d < k; ++d) col[(int64_t)P.drow[d] * pstride] = x1[d];
    }
}

Status build_plan(Plan &P, int degree, int n_points, int bc, const double *knots, int split_lo, int split_hi,
                  int flags) {
    P = Plan();
    P.dev_update = (flags & PLAN_DEVICE_UPDATE) != 0;
    if (degree < 1 || degree > 5) return {1, "degree must be in 1..5"};
    // bc < 16: both ends alike; else lo | (hi << 4) (mixed, R13)
    int bc_lo = bc, bc_hi = bc;
    if (bc >= 16) {
        bc_lo = bc & 15;
        bc_hi = (bc >> 4) & 15;
        if ((bc >> 8) || bc_lo == PERIODIC || bc_hi == PERIODIC) return {1, "unknown boundary condition"};
        if (bc_lo == bc_hi) bc = bc_lo;
    }
    if (bc_lo != PERIODIC && bc_lo != GREVILLE && bc_lo != HERMITE) return {1, "unknown boundary condition"};
    if (bc_hi != PERIODIC && bc_hi != GREVILLE && bc_hi != HERMITE) return {1, "unknown boundary condition"};
    const bool mixed = bc_lo != bc_hi;
    P.p = degree;
    P.bc = bc;
    P.bc_lo = bc_lo;
    P.bc_hi = bc_hi;
    const int nbc_p = (degree % 2) ? (degree - 1) / 2 : degree / 2;
    if (bc == PERIODIC) { P.N = n_points; P.n = P.N; }
    else if (bc == GREVILLE) { P.N = n_points - degree; P.n = P.N + degree; }
    else if (!mixed) {
        P.N = (degree % 2) ? n_points - 1 : n_points;
        P.nbc = nbc_p;
        P.n = P.N + degree;
    } else {
        P.nbc_lo = bc_lo == HERMITE ? nbc_p : 0;
        P.nbc_hi = bc_hi == HERMITE ? nbc_p : 0;
        P.nbc = std::max(P.nbc_lo, P.nbc_hi);
        P.N = n_points - degree + P.nbc_lo + P.nbc_hi;
        P.n = P.N + degree;
        if (P.n < P.nbc_lo + P.nbc_hi + 2) return {1, "too few points for this degree / boundary condition"};
    }
    if (!mixed) P.nbc_lo = P.nbc_hi = (bc == HERMITE) ? P.nbc : 0;
    if (P.N < 1) return {1, "too few points for this degree / boundary condition"};
    if (bc == PERIODIC && P.N < 2) return {1, "periodic spline needs at least 2 cells"};
    const int N = P.N, n = P.n, p = P.p;
    P.h.resize(N);
    for (int c = 0; c < N; ++c) {
        P.h[c] = knots ? knots[c + 1] - knots[c] : 1.0 / (double)N;  // uniform: exact equal widths (R1)
        if (!(P.h[c] > 0.0) || !std::isfinite(P.h[c])) return {1, "breakpoints must be strictly increasing"};
    }
    Space S{p, bc == PERIODIC ? PERIODIC : GREVILLE, N, n, P.nbc, P.h.data()};  // clamped knots unless periodic
    // rows: mesh-independent descriptors first (device refactorisation reuses them)
    P.rowdesc.clear();
    if (mixed) {
        // derivative rows at a Hermite end; the Greville abscissae minus the nbc
        // next to a Hermite end (the end point itself stays)
        for (int d = 1; d <= P.nbc_lo; ++d) P.rowdesc.push_back({ROW_DER0, 0, d});
        for (int j = 0; j < n; ++j) {
            if (j >= 1 && j <= P.nbc_lo) continue;
            if (j >= n - 1 - P.nbc_hi && j <= n - 2) continue;
            P.rowdesc.push_back({ROW_GREVILLE, j, 0});
        }
        for (int d = 1; d <= P.nbc_hi; ++d) P.rowdesc.push_back({ROW_DERN, 0, d});
        if ((int)P.rowdesc.size() != n) return {1, "mixed boundary rows do not add up"};
    } else if (bc != HERMITE) {
        for (int j = 0; j < n; ++j) P.rowdesc.push_back({ROW_GREVILLE, j, 0});
    } else {
        for (int d = 1; d <= P.nbc; ++d) P.rowdesc.push_back({ROW_DER0, 0, d});
        if (p % 2) {
            for (int i = 0; i < N; ++i) P.rowdesc.push_back({ROW_BREAK, i, 0});
            P.rowdesc.push_back({ROW_END, N, 0});
        } else {
            for (int c = 0; c < N; ++c) P.rowdesc.push_back({ROW_MID, c, 0});
        }
        for (int d = 1; d <= P.nbc; ++d) P.rowdesc.push_back({ROW_DERN, 0, d});
    }
    std::vector<RowPt> rows(n);
    P.rowscale.assign(n, 1.0);
    for (int i = 0; i < n; ++i) {
        const RowDesc &d = P.rowdesc[i];
        switch (d.kind) {
            case ROW_GREVILLE: rows[i] = greville(S, d.idx); break;
            case ROW_BREAK: rows[i] = RowPt{S.span_of_cell(d.idx), 0.0, 0}; break;
            case ROW_END: rows[i] = RowPt{S.span_of_cell(N - 1), P.h[N - 1], 0}; break;
            case ROW_MID: rows[i] = RowPt{S.span_of_cell(d.idx), 0.5 * P.h[d.idx], 0}; break;
            case ROW_DER0: rows[i] = RowPt{S.span_of_cell(0), 0.0, d.deriv}; P.rowscale[i] = std::pow(P.h[0], d.deriv); break;
            default: rows[i] = RowPt{S.span_of_cell(N - 1), P.h[N - 1], d.deriv}; P.rowscale[i] = std::pow(P.h[N - 1], d.deriv); break;
        }
    }
    // breakpoints and row positions (advection / evaluation data)
    // (uniform: x_c = c/N on [0,1], not a running sum of widths, R1)
    P.xb.assign(N + 1, 0.0);
    for (int c = 0; c <= N; ++c) P.xb[c] = knots ? knots[c] : (double)c / (double)N;
    P.xi.resize(n);
    for (int i = 0; i < n; ++i) {
        const long cell = bc == PERIODIC ? lmod(rows[i].span, N) : rows[i].span - p;
        P.xi[i] = P.xb[cell] + rows[i].u;
    }
    if (bc == PERIODIC) {
        // periodic extension t_c, c in [-p, N+p]: xe[c + p] (evaluation at the feet, Algorithm 2)
        const double Lp = P.xb[N] - P.xb[0];
        P.xe.resize(N + 2 * p + 1);
        for (int c = -p; c <= N + p; ++c)
            P.xe[c + p] = c < 0 ? P.xb[c + N] - Lp : (c > N ? P.xb[c - N] + Lp : P.xb[c]);
        // uniform within one ulp: every foot of a row shares its local coordinate,
        // so the evaluation is a (p+1)-tap stencil with weights computed once per row
        const double hu = Lp / N;
        double dev = 0.0, xmax = 1.0;
        for (int c = 0; c <= N; ++c) {
            dev = std::max(dev, std::fabs(P.xb[c] - (P.xb[0] + c * hu)));
            xmax = std::max(xmax, std::fabs(P.xb[c]));
        }
        for (int i = 0; i < n; ++i) dev = std::max(dev, std::fabs((P.xi[i] - P.xi[0]) - i * hu));
        P.adv_uniform = dev <= 2.3e-16 * xmax && !P.dev_update;  // device update: generic geometry
        P.adv_invh = 1.0 / hu;
        P.adv_q0 = (P.xi[0] - P.xb[0]) / hu;
        // bucket table: buckets no wider than the smallest cell (up to 8N of them);
        // tbl[b] = cell holding the bucket's left edge minus a margin that covers
        // the rounding of b = floor((x - x_0) * scale) on the device, so the true
        // cell is tbl[b] + 0..adv_steps, found by adv_steps branch-free steps
        {
            double hmin = Lp;
            for (int c = 0; c < N; ++c) hmin = std::min(hmin, P.xb[c + 1] - P.xb[c]);
            // (device update: twice as many buckets, so a new mesh whose smallest cell
            // is down to half of this one keeps the frozen step count)
            const double fine = P.dev_update ? 2.0 : 1.0;
            const int MT = std::max(1, (int)std::min<double>(8.0 * N, std::ceil(fine * Lp / hmin * (1.0 + 1e-12))));
            const double w = Lp / MT, margin = 1e-9 * w;
            auto cell_of = [&](double x) {  // t_c <= x < t_{c+1}, clamped to [0, N)
                int lo = 0, hi = N - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) / 2;
                    if (P.xb[mid] <= x) lo = mid;
                    else hi = mid - 1;
                }
                return lo;
            };
            P.adv_tbl.resize(MT);
            P.adv_steps = 0;
            for (int b = 0; b < MT; ++b) {
                const int lo = cell_of(P.xb[0] + b * w - margin);
                const int hi = cell_of(P.xb[0] + (b + 1) * w + margin);
                P.adv_tbl[b] = lo;
                P.adv_steps = std::max(P.adv_steps, hi - lo);
            }
            // device update: two more locate steps, so cells down to a third of the
            // bucket width (jitter +-0.3h on a 2x finer table) keep the frozen table
            if (P.dev_update) P.adv_steps += 2;
        }
        // reciprocal knot differences 1/(t_{m+w} - t_m), m in [-p, N+p), w = 1..p:
        // the denominators of de Boor's recursion depend on the knots only, so the
        // non-uniform evaluation multiplies instead of dividing
        const int RS = p | 1;  // odd row stride: lanes at consecutive cells hit distinct banks
        P.adv_rcp.assign((size_t)(N + 2 * p) * RS, 0.0);
        for (int m = -p; m < N + p; ++m)
            for (int w = 1; w <= p; ++w)
                if (m + w <= N + p) P.adv_rcp[(size_t)(m + p) * RS + (w - 1)] = 1.0 / (P.xe[m + w + p] - P.xe[m + p]);
    }
    // equilibrated sparse rows: rowscale * (d^deriv B_j)(point)
    P.A.assign(n, SparseRow());
    for (int i = 0; i < n; ++i) {
        double vals[16];
        if (rows[i].deriv == 0) bsplvb(S, rows[i].span, rows[i].u, p, vals);
        else bsplvd(S, rows[i].span, rows[i].u, rows[i].deriv, vals);
        std::map<int, double> acc;
        for (int r = 0; r <= p; ++r) acc[S.basis_of(rows[i].span - p + r)] += vals[r] * P.rowscale[i];
        if (P.dev_update) {
            // structure frozen for later meshes: a Greville point that sits ON a knot
            // (uniform odd-degree meshes put every one there) moves into the
            // neighbouring span under any perturbation, so the basis function on that
            // side is a structural entry (value 0 here) of the band and the split
            const double w = S.width(rows[i].span), u = rows[i].u;
            if (P.rowdesc[i].kind == ROW_GREVILLE && u <= 1e-12 * w) {  // (break / end rows stay on their knot)
                const long q = rows[i].span - p - 1;
                if (bc == PERIODIC || q >= 0) acc[S.basis_of(q)] += 0.0;
            }
        }
        for (auto &kv : acc)
            if (kv.second != 0.0 || P.dev_update) { P.A[i].col.push_back(kv.first); P.A[i].val.push_back(kv.second); }
        if (P.A[i].col.empty()) return {2, "empty collocation row"};
    }
    // candidate splits
    std::vector<std::pair<int, int>> cands;
    if (split_lo >= 0 || split_hi >= 0) {
        if (split_lo < 0 || split_hi < 0) return {1, "give both split_lo and split_hi, or neither"};
        if (bc == PERIODIC && split_lo != 0) return {1, "periodic split must have split_lo == 0"};
        cands.push_back({split_lo, split_hi});
    } else if (bc == PERIODIC) {
        int kl = 0, ku = 0;
        for (int i = 0; i < n; ++i)
            for (int c : P.A[i].col) {
                long o = lmod(c - i, n);
                if (o > n / 2) o -= n;
                kl = std::max<long>(kl, -o);
                ku = std::max<long>(ku, o);
            }
        for (int k = std::max(kl, ku); k <= std::min(n, KMAX_DELTA); ++k) cands.push_back({0, k});
    } else {
        // score candidates by (kernel band K, kl+ku, k)
        const int lo0 = P.nbc_lo, hi0 = P.nbc_hi;  // derivative rows always go to delta
        struct C { int K, bw, k, a, b; };
        std::vector<C> cs;
        for (int a = lo0; a <= lo0 + p + 1; ++a)
            for (int b = hi0; b <= hi0 + p + 1; ++b) {
                if (a + b > KMAX_DELTA || a + b >= n) continue;
                int kl = 0, ku = 0;
                for (int i = a; i < n - b; ++i)
                    for (int c : P.A[i].col)
                        if (c >= a && c < n - b) { kl = std::max(kl, i - c); ku = std::max(ku, c - i); }
                cs.push_back({std::max(1, std::max(kl, ku)), kl + ku, a + b, a, b});
            }
        std::sort(cs.begin(), cs.end(), [](const C &x, const C &y) {
            if (x.K != y.K) return x.K < y.K;
            if (x.bw != y.bw) return x.bw < y.bw;
            if (x.k != y.k) return x.k < y.k;
            return std::abs(x.a - x.b) < std::abs(y.a - y.b);
        });
        for (auto &c : cs) cands.push_back({c.a, c.b});
    }
    if (n <= KMAX_DELTA) cands.push_back({0, n});  // tiny: dense delta' only
    std::string why = "no admissible Schur split";
    int why_code = 2;
    std::mt19937_64 gen(12345);
    std::uniform_real_distribution<double> U(-1.0, 1.0);
    for (auto &c : cands) {
        SplitResult r = try_split(P, c.first, c.second);
        if (r.code) { why = r.msg; why_code = r.code; continue; }
        build_segplan(P, P.seg[0], 36);  // tile kernel fp64 / fp32 (instantiated lengths)
        build_segplan(P, P.seg[1], 72);
        {   // warp-per-RHS kernel: odd L (conflict-free smem transpose), S <= 32
            const int need = std::max(P.K, (P.nQ + 31) / 32);
            int Lpc = 0;
            for (int cand : {3, 5, 9, 17, 33, 63})  // instantiated in solve_kernels.cu
                if (cand >= need) { Lpc = cand; break; }
            if (Lpc) build_segplan(P, P.seg[2], Lpc);
            else P.seg[2] = SegPlan();
        }
        // self-check: residual of the equilibrated system with 4 random RHS
        const int nb = 4;
        std::vector<double> b((size_t)n * nb), x;
        for (auto &v : b) v = U(gen);
        x = b;
        plan_solve_cpu(P, x.data(), nb, 1, nb);
        double res = 0.0, bmax = 0.0;
        for (int rr = 0; rr < nb; ++rr)
            for (int i = 0; i < n; ++i) {
                double acc = 0.0;
                for (size_t e = 0; e < P.A[i].col.size(); ++e) acc += P.A[i].val[e] * x[(size_t)P.A[i].col[e] * nb + rr];
                double bi = b[(size_t)i * nb + rr] * P.rowscale[i];
                res = std::max(res, std::fabs(acc - bi));
                bmax = std::max(bmax, std::fabs(bi));
            }
        if (res <= 1e-13 * bmax) return {0, ""};
        why = "self-check residual too large for split";
        why_code = 2;
    }
    return {why_code, why};
}

}  // namespace sb
