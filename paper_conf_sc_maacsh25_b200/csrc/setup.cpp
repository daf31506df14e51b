// setup.cpp — host-side preconditioner construction for spcg_setup (Fig. 2,
// P:L306-339): input validation, wavefront-aware sparsification (Algorithm 2,
// P:L427-461), ILU(K) symbolic + numeric factorisation (§3.3) and
// wavefront levels (§2).
//
// Written independently of oracle/ (different algorithms, no shared code):
//   levels      Kahn frontier peeling        (oracle: longest-path DP)
//   drop order  stable LSD radix sort on the IEEE bits of |a_ij|  (oracle: qsort)
//   ILU(K)      fill-path BFS (Rose-Tarjan / Hysom-Pothen) per row, upper half,
//               lower half by transposition (oracle: row-merge with a linked list)
//   numeric     IKJ over level sets in parallel, windowed dense row workspace
// Compiled with -ffp-contract=off so the arithmetic matches the definitions.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <numeric>

#include "internal.h"

#ifdef _OPENMP
#include <omp.h>
#endif

namespace spcg {

static thread_local std::string g_err;
void set_error(const std::string& s) { g_err = s; }
const char* last_error_cstr() { return g_err.c_str(); }

double now_ms() {
    using namespace std::chrono;
    return duration<double, std::milli>(steady_clock::now().time_since_epoch()).count();
}

static inline uint64_t dbits(double v) { uint64_t b; std::memcpy(&b, &v, 8); return b; }

// ---------------------------------------------------------------- validation
spcg_status_t validate_and_mirror(const Csr& A, std::vector<int64_t>& pos_t) {
    const int64_t n = A.n;
    if (n <= 0) { set_error("n must be >= 1"); return SPCG_ERR_INVALID_ARG; }
    if ((int64_t)A.rp.size() != n + 1 || A.rp[0] != 0) { set_error("bad row_ptr"); return SPCG_ERR_BAD_MATRIX; }
    const int64_t nnz = A.rp[n];
    if (nnz >= (int64_t(1) << 31)) { set_error("nnz >= 2^31"); return SPCG_ERR_BAD_MATRIX; }
    std::vector<int64_t> cnt(n + 1, 0);
    for (int64_t i = 0; i < n; ++i) {
        if (A.rp[i + 1] < A.rp[i] || A.rp[i + 1] > nnz) { set_error("row_ptr not monotone"); return SPCG_ERR_BAD_MATRIX; }
        bool diag = false;
        int64_t prev = -1;
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q) {
            int64_t j = A.col[q];
            if (j < 0 || j >= n || j <= prev) { set_error("columns out of range, unsorted or duplicated in row " + std::to_string(i)); return SPCG_ERR_BAD_MATRIX; }
            prev = j;
            if (!std::isfinite(A.val[q])) { set_error("non-finite value in row " + std::to_string(i)); return SPCG_ERR_BAD_MATRIX; }
            if (j == i) {
                diag = true;
                if (!(A.val[q] > 0.0)) { set_error("non-positive diagonal at row " + std::to_string(i)); return SPCG_ERR_BAD_MATRIX; }
            }
            cnt[j + 1]++;
        }
        if (!diag) { set_error("missing diagonal at row " + std::to_string(i)); return SPCG_ERR_BAD_MATRIX; }
    }
    // transpose by counting sort; symmetric <=> transpose identical (pattern and bits)
    for (int64_t j = 0; j < n; ++j) cnt[j + 1] += cnt[j];
    for (int64_t j = 0; j <= n; ++j)
        if (cnt[j] != A.rp[j]) { set_error("pattern not symmetric"); return SPCG_ERR_BAD_MATRIX; }
    pos_t.assign(nnz, 0);
    std::vector<int64_t> next(cnt.begin(), cnt.end() - 1);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q) {
            int64_t j = A.col[q];
            int64_t tq = next[j]++;
            // position tq holds (j, i) in A iff A is symmetric
            if (A.col[tq] != i || dbits(A.val[tq]) != dbits(A.val[q])) {
                set_error("matrix not exactly symmetric at (" + std::to_string(i) + "," + std::to_string(j) + ")");
                return SPCG_ERR_BAD_MATRIX;
            }
            pos_t[q] = tq;
        }
    return SPCG_OK;
}

// ---------------------------------------------------------------- Kahn levels
int64_t kahn_levels(const Csr& M, bool lower, std::vector<int32_t>& lev) {
    const int64_t n = M.n;
    lev.assign(n, 0);
    std::vector<int32_t> indeg(n, 0);
    std::vector<int64_t> tp(n + 1, 0);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t q = M.rp[i]; q < M.rp[i + 1]; ++q) {
            int64_t j = M.col[q];
            if (lower ? (j < i) : (j > i)) { indeg[i]++; tp[j + 1]++; }
        }
    for (int64_t j = 0; j < n; ++j) tp[j + 1] += tp[j];
    std::vector<int32_t> dep(tp[n]);            // dependents of j
    {
        std::vector<int64_t> nx(tp.begin(), tp.end() - 1);
        for (int64_t i = 0; i < n; ++i)
            for (int64_t q = M.rp[i]; q < M.rp[i + 1]; ++q) {
                int64_t j = M.col[q];
                if (lower ? (j < i) : (j > i)) dep[nx[j]++] = (int32_t)i;
            }
    }
    std::vector<int32_t> front, nxt;
    for (int64_t i = 0; i < n; ++i) if (indeg[i] == 0) front.push_back((int32_t)i);
    int64_t level = 0, done = 0;
    while (!front.empty()) {
        nxt.clear();
        for (int32_t v : front) {
            lev[v] = (int32_t)level;
            for (int64_t q = tp[v]; q < tp[v + 1]; ++q)
                if (--indeg[dep[q]] == 0) nxt.push_back(dep[q]);
        }
        done += (int64_t)front.size();
        std::swap(front, nxt);
        ++level;
    }
    (void)done;
    return level;
}

// ---------------------------------------------------------------- Algorithm 2
// Stable LSD radix sort (11-bit digits) of candidate positions by the IEEE bits
// of |a| (non-negative doubles order like their bit patterns).  Input order is
// row-major, so ties stay in row-major order (reading A4).
static void radix_sort_by_mag(std::vector<uint64_t>& key, std::vector<int64_t>& idx) {
    const size_t m = key.size();
    std::vector<uint64_t> k2(m);
    std::vector<int64_t> i2(m);
    const int BITS = 11, R = 1 << BITS;
    std::vector<size_t> c(R + 1);
    for (int shift = 0; shift < 64; shift += BITS) {
        std::fill(c.begin(), c.end(), 0);
        bool trivial = true;
        uint64_t first = m ? ((key[0] >> shift) & (R - 1)) : 0;
        for (size_t t = 0; t < m; ++t) {
            uint64_t d = (key[t] >> shift) & (R - 1);
            c[d + 1]++;
            trivial &= (d == first);
        }
        if (trivial) continue;
        for (int d = 0; d < R; ++d) c[d + 1] += c[d];
        for (size_t t = 0; t < m; ++t) {
            size_t dst = c[(key[t] >> shift) & (R - 1)]++;
            k2[dst] = key[t]; i2[dst] = idx[t];
        }
        key.swap(k2); idx.swap(i2);
    }
}

// drop mask for ratio t: the first m entries of the sorted candidates plus mirrors
static Csr apply_drop(const Csr& A, const std::vector<int64_t>& pos_t, const std::vector<int64_t>& order,
                      int64_t m, std::vector<uint8_t>& drop) {
    drop.assign(A.nnz(), 0);
    for (int64_t t = 0; t < m; ++t) { drop[order[t]] = 1; drop[pos_t[order[t]]] = 1; }
    Csr H;
    H.n = A.n;
    H.rp.assign(A.n + 1, 0);
    H.col.reserve(A.nnz() - 2 * m);
    H.val.reserve(A.nnz() - 2 * m);
    for (int64_t i = 0; i < A.n; ++i) {
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q)
            if (!drop[q]) { H.col.push_back(A.col[q]); H.val.push_back(A.val[q]); }
        H.rp[i + 1] = (int64_t)H.col.size();
    }
    return H;
}

// Indicator of Alg. 2 lines 4-5: kappa ~ ||Ahat||_inf / min diag, ||Ahat^-1|| ~
// kappa / ||Ahat||_2, value ||Ahat^-1|| * ||S||; norms per reading A6, summed in
// row-major order.
// SPECTRAL reading (A6, SPCG_NORM_SPECTRAL): ||M||_2 by the power method — v_0 =
// (1..1)/sqrt(n), w = M v_k in CSR order, v_{k+1} = w / ||w||_2, 100 steps, the last
// ||w||_2 — with M = Ahat (keep = 1: entries not dropped) or S (keep = 0: the dropped
// ones) read straight from A and the mask (the same order as their compacted CSR).
static double norm_spec(const Csr& A, const std::vector<uint8_t>& drop, int keep) {
    const int64_t n = A.n;
    std::vector<double> v(n, 1.0 / std::sqrt((double)n)), w(n);
    double est = 0.0;
    for (int k = 0; k < 100; ++k) {
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) {
            double acc = 0.0;
            for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q)
                if ((drop[q] == 0) == (keep == 1)) acc += A.val[q] * v[A.col[q]];
            w[i] = acc;
        }
        double ss = 0.0;
        for (int64_t i = 0; i < n; ++i) ss += w[i] * w[i];
        est = std::sqrt(ss);
        if (est == 0.0) break;
        for (int64_t i = 0; i < n; ++i) v[i] = w[i] / est;
    }
    return est;
}

static double indicator(const Csr& A, const std::vector<uint8_t>& drop, int norm_reading) {
    double fro_h = 0.0, fro_s = 0.0, inf_h = 0.0, inf_s = 0.0, mind = INFINITY;
    for (int64_t i = 0; i < A.n; ++i) {
        double rh = 0.0, rs = 0.0;
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q) {
            double v = A.val[q];
            if (drop[q]) { fro_s += v * v; rs += std::fabs(v); }
            else {
                fro_h += v * v; rh += std::fabs(v);
                if (A.col[q] == i && v < mind) mind = v;
            }
        }
        if (rh > inf_h) inf_h = rh;
        if (rs > inf_s) inf_s = rs;
    }
    double kappa = inf_h / mind;
    double a2 = norm_reading == SPCG_NORM_INF ? inf_h
                : norm_reading == SPCG_NORM_SPECTRAL ? norm_spec(A, drop, 1) : std::sqrt(fro_h);
    double s = norm_reading == SPCG_NORM_INF ? inf_s
               : norm_reading == SPCG_NORM_SPECTRAL ? norm_spec(A, drop, 0) : std::sqrt(fro_s);
    double inv = kappa / a2;
    return inv * s;
}

spcg_status_t sparsify_select(const Csr& A, const std::vector<int64_t>& pos_t,
                              const spcg_drop_params_t& p, SparsifyResult& out) {
    std::vector<int32_t> lev;
    out.w_A = kahn_levels(A, true, lev);
    if (p.mode == SPCG_DROP_NONE) {
        out.Ahat = A;
        out.w_Ahat = out.w_A;
        out.chosen_pct = 0.0;
        return SPCG_OK;
    }
    // candidates: strictly lower entries, row-major; N_L = nnz(tril A) incl. diagonal (A1)
    std::vector<uint64_t> key;
    std::vector<int64_t> order;
    int64_t NL = 0;
    for (int64_t i = 0; i < A.n; ++i)
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q) {
            if (A.col[q] <= i) NL++;
            if (A.col[q] < i) { key.push_back(dbits(std::fabs(A.val[q]))); order.push_back(q); }
        }
    radix_sort_by_mag(key, order);
    const int64_t C = (int64_t)order.size();
    auto count = [&](double t) {
        int64_t m = (int64_t)std::floor(t * (double)NL / 100.0);   // A2
        return std::max<int64_t>(0, std::min(m, C));
    };
    std::vector<uint8_t> drop;
    if (p.mode == SPCG_DROP_FIXED) {
        int64_t m = count(p.fixed_pct);
        out.Ahat = apply_drop(A, pos_t, order, m, drop);
        out.chosen_pct = p.fixed_pct;
        out.m_t = m;
        out.w_Ahat = kahn_levels(out.Ahat, true, lev);
        return SPCG_OK;
    }
    if (p.n_ratios < 1 || p.n_ratios > 8) { set_error("n_ratios must be 1..8"); return SPCG_ERR_INVALID_ARG; }
    // Algorithm 2
    int nr = p.n_ratios;
    int chosen = -1;
    for (int r = 0; r < nr && chosen < 0; ++r) {
        double t = p.ratios_pct[r];
        int64_t m = count(t);
        Csr H = apply_drop(A, pos_t, order, m, drop);
        double ind = indicator(A, drop, p.norm_reading);
        out.tried_pct[r] = t; out.indicator[r] = ind; out.tried_w[r] = -1; out.reduction[r] = -1.0;
        out.n_tried = r + 1;
        bool last = (r == nr - 1);
        if (ind > p.tau) {                      // line 5
            if (last) { chosen = 0; break; }    // line 6: return A - S_first
            continue;                           // line 7
        }
        int64_t wt = kahn_levels(H, true, lev); // line 9
        double den = p.reduction_denominator == SPCG_DENOM_WAHAT ? (double)wt : (double)out.w_A;
        double red = 100.0 * (double)(out.w_A - wt) / den;    // Eq. 7 / line 10
        out.tried_w[r] = wt; out.reduction[r] = red;
        if (red >= p.omega_pct || last) {      // lines 10-11
            out.Ahat = std::move(H);
            out.chosen_pct = t; out.m_t = m; out.w_Ahat = wt;
            return SPCG_OK;
        }
    }
    if (chosen < 0) chosen = 0;                 // line 14
    int64_t m = count(p.ratios_pct[chosen]);
    out.Ahat = apply_drop(A, pos_t, order, m, drop);
    out.chosen_pct = p.ratios_pct[chosen];
    out.m_t = m;
    out.w_Ahat = kahn_levels(out.Ahat, true, lev);
    return SPCG_OK;
}

// ---------------------------------------------------------------- ILU(K) symbolic
// Fill-path theorem: (i,j) is in the ILU(K) pattern with level l iff the
// shortest path i -> j in G(Ahat) whose intermediate vertices are all numbered
// below min(i,j) has l+1 edges, l <= K (equivalent to the sum-rule level of
// fill).  For j > i the bound is i: a depth-limited BFS from i through vertices
// < i finds the upper half of row i.  The pattern is symmetric, so the lower
// half is the transpose.
spcg_status_t iluk_symbolic(const Csr& Ah, int K, Factors& F) {
    const int64_t n = Ah.n;
    std::vector<int64_t> urp(n + 1, 0);
    std::vector<int32_t> ucol;
    std::vector<int32_t> ulev;
    if (K == 0) {
        for (int64_t i = 0; i < n; ++i) {
            for (int64_t q = Ah.rp[i]; q < Ah.rp[i + 1]; ++q)
                if (Ah.col[q] >= i) { ucol.push_back(Ah.col[q]); ulev.push_back(0); }
            urp[i + 1] = (int64_t)ucol.size();
        }
    } else {
        int T = 1;
#ifdef _OPENMP
        T = omp_get_max_threads();
#endif
        std::vector<std::vector<int32_t>> tc(T), tl(T);
        std::vector<int64_t> rowlen(n, 0);
#pragma omp parallel num_threads(T)
        {
            int t = 0;
#ifdef _OPENMP
            t = omp_get_thread_num();
#endif
            int64_t lo = n * t / T, hi = n * (t + 1) / T;
            std::vector<int32_t> visit(n, -1), rec(n, -1);
            std::vector<int32_t> front, nxt;
            std::vector<std::pair<int32_t, int32_t>> found;
            for (int64_t i = lo; i < hi; ++i) {
                found.clear();
                front.assign(1, (int32_t)i);
                visit[i] = (int32_t)i;
                for (int d = 0; d <= K && !front.empty(); ++d) {
                    nxt.clear();
                    for (int32_t v : front)
                        for (int64_t q = Ah.rp[v]; q < Ah.rp[v + 1]; ++q) {
                            int32_t u = Ah.col[q];
                            if (u > i) {
                                if (rec[u] != (int32_t)i) { rec[u] = (int32_t)i; found.push_back({u, d}); }
                            } else if (u < i && visit[u] != (int32_t)i) {
                                visit[u] = (int32_t)i;
                                if (d + 1 <= K) nxt.push_back(u);
                            }
                        }
                    std::swap(front, nxt);
                }
                std::sort(found.begin(), found.end());
                tc[t].push_back((int32_t)i); tl[t].push_back(0);
                for (auto& f : found) { tc[t].push_back(f.first); tl[t].push_back(f.second); }
                rowlen[i] = 1 + (int64_t)found.size();
            }
        }
        for (int64_t i = 0; i < n; ++i) urp[i + 1] = urp[i] + rowlen[i];
        ucol.reserve(urp[n]); ulev.reserve(urp[n]);
        for (int t = 0; t < T; ++t) {
            ucol.insert(ucol.end(), tc[t].begin(), tc[t].end());
            ulev.insert(ulev.end(), tl[t].begin(), tl[t].end());
        }
    }
    // lower half = transpose of the strict upper half (levels are symmetric)
    std::vector<int64_t> lrp(n + 1, 0);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t q = urp[i] + 1; q < urp[i + 1]; ++q) lrp[ucol[q] + 1]++;
    for (int64_t i = 0; i < n; ++i) lrp[i + 1] += lrp[i];
    std::vector<int32_t> lcol(lrp[n]), llev(lrp[n]);
    {
        std::vector<int64_t> nx(lrp.begin(), lrp.end() - 1);
        for (int64_t i = 0; i < n; ++i)
            for (int64_t q = urp[i] + 1; q < urp[i + 1]; ++q) {
                int64_t dst = nx[ucol[q]]++;
                lcol[dst] = (int32_t)i; llev[dst] = ulev[q];
            }
    }
    F.L.n = n; F.L.rp = std::move(lrp); F.L.col.assign(lcol.begin(), lcol.end()); F.L.val.assign(F.L.col.size(), 0.0);
    F.U.n = n; F.U.rp = std::move(urp); F.U.col.assign(ucol.begin(), ucol.end()); F.U.val.assign(F.U.col.size(), 0.0);
    F.fill_level.resize(F.L.col.size() + F.U.col.size());
    int64_t o = 0;
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) F.fill_level[o++] = llev[q];
        for (int64_t q = F.U.rp[i]; q < F.U.rp[i + 1]; ++q) F.fill_level[o++] = ulev[q];
    }
    F.wL = kahn_levels(F.L, true, F.levL);
    F.wU = kahn_levels(F.U, false, F.levU);
    return SPCG_OK;
}

// ---------------------------------------------------------------- numeric ILU
// IKJ on the symbolic pattern, rows of one L-wavefront in
// parallel: row i only reads U rows k < i of its L pattern, all in earlier
// wavefronts.  Per row the update order (k ascending, j in U-row order) is the
// definition's, so the result does not depend on the thread count.
spcg_status_t ilu_numeric(const Csr& Ah, Factors& F) {
    const int64_t n = Ah.n;
    // level sets of L
    std::vector<int64_t> lp(F.wL + 1, 0);
    for (int64_t i = 0; i < n; ++i) lp[F.levL[i] + 1]++;
    for (int64_t l = 0; l < F.wL; ++l) lp[l + 1] += lp[l];
    std::vector<int32_t> lrows(n);
    {
        std::vector<int64_t> nx(lp.begin(), lp.end() - 1);
        for (int64_t i = 0; i < n; ++i) lrows[nx[F.levL[i]]++] = (int32_t)i;
    }
    // window = max column span of a factor row
    int64_t span = 1;
    for (int64_t i = 0; i < n; ++i) {
        int64_t lo = F.L.rp[i + 1] > F.L.rp[i] ? F.L.col[F.L.rp[i]] : i;
        int64_t hi = F.U.col[F.U.rp[i + 1] - 1];
        span = std::max(span, hi - lo + 1);
    }
    int64_t bad = INT64_MAX;
#pragma omp parallel
    {
        std::vector<double> wv(span);
        std::vector<int64_t> mark(span, -1);
        int64_t mybad = INT64_MAX;
        for (int64_t l = 0; l < F.wL; ++l) {
#pragma omp for schedule(dynamic, 64)
            for (int64_t t = lp[l]; t < lp[l + 1]; ++t) {
                const int64_t i = lrows[t];
                const int64_t base = F.L.rp[i + 1] > F.L.rp[i] ? F.L.col[F.L.rp[i]] : i;
                for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) { wv[F.L.col[q] - base] = 0.0; mark[F.L.col[q] - base] = i; }
                for (int64_t q = F.U.rp[i]; q < F.U.rp[i + 1]; ++q) { wv[F.U.col[q] - base] = 0.0; mark[F.U.col[q] - base] = i; }
                for (int64_t q = Ah.rp[i]; q < Ah.rp[i + 1]; ++q) wv[Ah.col[q] - base] = Ah.val[q];
                for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
                    const int64_t k = F.L.col[q];
                    const int64_t u0 = F.U.rp[k];
                    const double lik = wv[k - base] / F.U.val[u0];
                    wv[k - base] = lik;
                    for (int64_t r = u0 + 1; r < F.U.rp[k + 1]; ++r) {
                        const int64_t j = F.U.col[r];
                        const int64_t o = j - base;
                        if (o < span && mark[o] == i) wv[o] = wv[o] - lik * F.U.val[r];
                    }
                }
                for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) F.L.val[q] = wv[F.L.col[q] - base];
                for (int64_t q = F.U.rp[i]; q < F.U.rp[i + 1]; ++q) F.U.val[q] = wv[F.U.col[q] - base];
                const double d = F.U.val[F.U.rp[i]];
                if (d == 0.0 || !std::isfinite(d)) mybad = std::min(mybad, i);
            }
        }
#pragma omp critical
        bad = std::min(bad, mybad);
    }
    if (bad != INT64_MAX) {
        F.zero_pivot_row = bad;
        set_error("zero or non-finite pivot at row " + std::to_string(bad));
        return SPCG_ERR_ZERO_PIVOT;
    }
    return SPCG_OK;
}

}  // namespace spcg
