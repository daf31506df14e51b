// layout.cpp — device data layouts for the iterative phase.
//
// SpMV: SELL-32 of the ORIGINAL A in natural row order; inside a
// 32-row slice the k-th entries of the 32 rows are contiguous, so a warp reads
// 128 B of column indices and 256 B of values per step, fully coalesced.
//
// SpTRSV (the wavefront executor of §2): the same sliced layout,
// slices never straddle a wavefront.  Slice order and the dependency encoding
// depend on the executor:
//   LEVEL     slices ordered by wavefront (level sets of Fig. 1c); every
//             dependency read from the global vector after a grid barrier.
//   SYNCFREE  same order; every value published with a ready flag; no barriers.
//   CHUNKED   rows split into contiguous per-CTA parts; inside a part slices are
//             ordered by wavefront; a dependency on a row of the same part is a
//             shared-memory ring slot (when the ring cannot have overwritten it
//             by then), anything else goes through the row's ready flag.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <iterator>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <set>
#include <string>

#include "internal.h"

namespace spcg {

void build_spmv_layout(const Csr& A, SpmvLayout& out) {
    const int64_t n = A.n;
    const int32_t ns = (int32_t)((n + 31) / 32);
    out.nslices = ns;
    out.eoff.assign(ns + 1, 0);
    for (int32_t s = 0; s < ns; ++s) {
        int64_t w = 0;
        for (int64_t r = 32LL * s; r < std::min<int64_t>(n, 32LL * s + 32); ++r) w = std::max(w, A.rp[r + 1] - A.rp[r]);
        out.eoff[s + 1] = out.eoff[s] + w;
    }
    out.col.assign(out.eoff[ns] * 32, 0);          // (sequential builder: keeps the zero fill)
    out.val.assign(out.eoff[ns] * 32, 0.0);
    for (int32_t s = 0; s < ns; ++s)
        for (int l = 0; l < 32; ++l) {
            int64_t r = 32LL * s + l;
            int64_t w = out.eoff[s + 1] - out.eoff[s];
            for (int64_t k = 0; k < w; ++k) {
                int64_t e = (out.eoff[s] + k) * 32 + l;
                if (r < n && k < A.rp[r + 1] - A.rp[r]) {
                    out.col[e] = A.col[A.rp[r] + k];
                    out.val[e] = A.val[A.rp[r] + k];
                } else {
                    out.col[e] = (int32_t)(r < n ? r : 0);   // padding: harmless self gather
                    out.val[e] = 0.0;
                }
            }
        }
}

// one factor -> TriLayout
static void build_tri(const Csr& M, bool upper, const std::vector<int32_t>& lev, int64_t w,
                      int strategy, const std::vector<int64_t>& pb, int32_t ring, double wide_min, TriLayout& T) {
    const int64_t n = M.n;
    const int parts = (int)pb.size() - 1;
    auto dep_begin = [&](int64_t i) { return upper ? M.rp[i] + 1 : M.rp[i]; };   // U: skip diagonal
    auto dep_end = [&](int64_t i) { return M.rp[i + 1]; };

    // execution order: rows of each (part, level) group; parts = 1 for LEVEL/SYNCFREE
    std::vector<int32_t> order;
    order.reserve(n);
    std::vector<int32_t> grp_rows_ptr;   // group -> [start,end) in order
    grp_rows_ptr.push_back(0);
    T.part_gptr.assign(1, 0);
    std::vector<int32_t> step_of(n, 0);  // group index inside the part (chunked ring analysis)
    const int P = strategy == SPCG_SPTRSV_CHUNKED ? parts : 1;
    for (int c = 0; c < P; ++c) {
        int64_t lo = strategy == SPCG_SPTRSV_CHUNKED ? pb[c] : 0;
        int64_t hi = strategy == SPCG_SPTRSV_CHUNKED ? pb[c + 1] : n;
        // counting sort of rows [lo,hi) by level, ascending row inside a level
        int32_t lmin = INT32_MAX, lmax = -1;
        for (int64_t i = lo; i < hi; ++i) { lmin = std::min(lmin, lev[i]); lmax = std::max(lmax, lev[i]); }
        if (hi <= lo) { T.part_gptr.push_back((int32_t)(grp_rows_ptr.size() - 1)); continue; }
        std::vector<int64_t> cnt(lmax - lmin + 2, 0);
        for (int64_t i = lo; i < hi; ++i) cnt[lev[i] - lmin + 1]++;
        for (size_t l = 0; l + 1 < cnt.size(); ++l) cnt[l + 1] += cnt[l];
        size_t base = order.size();
        order.resize(base + (hi - lo));
        std::vector<int64_t> nx(cnt.begin(), cnt.end() - 1);
        for (int64_t i = lo; i < hi; ++i) order[base + nx[lev[i] - lmin]++] = (int32_t)i;
        int32_t local = 0;
        for (size_t l = 0; l + 1 < cnt.size(); ++l) {
            if (cnt[l + 1] == cnt[l]) continue;
            for (int64_t t = cnt[l]; t < cnt[l + 1]; ++t) step_of[order[base + t]] = local;
            grp_rows_ptr.push_back((int32_t)(base + cnt[l + 1]));
            ++local;
        }
        T.part_gptr.push_back((int32_t)(grp_rows_ptr.size() - 1));
    }
    T.ngroups = (int32_t)grp_rows_ptr.size() - 1;
    (void)w;

    // LEVEL + wide rows: warp-per-row CSR in execution order
    {
        int64_t deps = 0;
        for (int64_t i = 0; i < n; ++i) deps += dep_end(i) - dep_begin(i);
        // threshold on the mean dependencies per row (spcg_options_t.wide_min; 0 = SPCG_WCAP)
        const double wmin = wide_min > 0.0 ? wide_min : (double)SPCG_WCAP;
        T.wide = (strategy == SPCG_SPTRSV_LEVEL || strategy == SPCG_SPTRSV_SYNCFREE) && n > 0 &&
                 (double)deps / (double)n > wmin;
        if (T.wide) {
            T.wrow.assign(order.begin(), order.end());
            T.wgptr.assign(grp_rows_ptr.begin(), grp_rows_ptr.end());
            T.wptr.assign(n + 1, 0);
            for (int64_t t = 0; t < n; ++t) T.wptr[t + 1] = T.wptr[t] + (dep_end(order[t]) - dep_begin(order[t]));
            T.wcol.resize(T.wptr[n]);
            T.wval.resize(T.wptr[n]);
            if (upper) T.wdinv.resize(n);
            for (int64_t t = 0; t < n; ++t) {
                const int32_t r = order[t];
                int64_t e = T.wptr[t];
                for (int64_t q = dep_begin(r); q < dep_end(r); ++q, ++e) {
                    T.wcol[e] = M.col[q];
                    T.wval[e] = M.val[q];
                }
                if (upper) T.wdinv[t] = 1.0 / M.val[M.rp[r]];
            }
        }
    }

    // slices of <= 32 rows inside each group
    T.gptr.assign(1, 0);
    std::vector<int32_t> slice_start;    // index into order
    std::vector<int32_t> slice_cnt;
    for (int32_t g = 0; g < T.ngroups; ++g) {
        for (int32_t s = grp_rows_ptr[g]; s < grp_rows_ptr[g + 1]; s += 32) {
            slice_start.push_back(s);
            slice_cnt.push_back(std::min(32, grp_rows_ptr[g + 1] - s));
        }
        T.gptr.push_back((int32_t)slice_start.size());
    }
    const int32_t ns = (int32_t)slice_start.size();
    T.nslices = ns;
    T.eoff.assign(ns + 1, 0);
    T.rows.assign((size_t)ns * 32, -1);
    T.publish.assign((size_t)ns * 32, strategy == SPCG_SPTRSV_SYNCFREE ? 1 : 0);
    T.rlen.assign((size_t)ns * 32, 0);
    if (upper) T.dinv.assign((size_t)ns * 32, 0.0);
    std::vector<int64_t> slot_of(n, -1);
    for (int32_t s = 0; s < ns; ++s) {
        int64_t wmax = 0;
        for (int l = 0; l < slice_cnt[s]; ++l) {
            int32_t r = order[slice_start[s] + l];
            T.rows[(size_t)s * 32 + l] = r;
            slot_of[r] = (int64_t)s * 32 + l;
            wmax = std::max<int64_t>(wmax, dep_end(r) - dep_begin(r));
            T.rlen[(size_t)s * 32 + l] = (int32_t)(dep_end(r) - dep_begin(r));
            if (upper) T.dinv[(size_t)s * 32 + l] = 1.0 / M.val[M.rp[r]];
        }
        T.eoff[s + 1] = T.eoff[s] + wmax;
    }
    T.total_cols = T.eoff[ns];

    // chunked: next-writer analysis of the ring (slot = (row - part_begin) & (ring-1))
    std::vector<int32_t> part_of;
    std::vector<int32_t> next_writer;    // step at which the ring slot of row j is next written
    const int32_t INF = INT32_MAX;
    if (strategy == SPCG_SPTRSV_CHUNKED) {
        part_of.assign(n, 0);
        next_writer.assign(n, INF);
        for (int c = 0; c < parts; ++c) {
            for (int64_t i = pb[c]; i < pb[c + 1]; ++i) part_of[i] = c;
            const int64_t sz = pb[c + 1] - pb[c];
            if (sz <= ring) continue;        // no slot is shared inside this part
            std::vector<std::pair<int32_t, int32_t>> mem;
            for (int64_t cls = 0; cls < ring; ++cls) {
                mem.clear();
                for (int64_t j = pb[c] + cls; j < pb[c + 1]; j += ring) mem.push_back({step_of[j], (int32_t)j});
                if (mem.size() < 2) continue;
                std::sort(mem.begin(), mem.end());
                for (size_t a = 0; a < mem.size();) {
                    size_t b = a;
                    while (b < mem.size() && mem[b].first == mem[a].first) ++b;
                    int32_t nxt = (b - a > 1) ? mem[a].first : (b < mem.size() ? mem[b].first : INF);
                    for (size_t t = a; t < b; ++t) next_writer[mem[t].second] = nxt;
                    a = b;
                }
            }
        }
    }

    if (strategy == SPCG_SPTRSV_RESIDENT) {          // n <= SPCG_RESIDENT_MAX_N: 16-bit fields suffice
        T.rrec.assign((size_t)ns * 32 * SPCG_RREC_BYTES, 0);
        std::vector<int32_t> lev_of(ns, 0);
        for (int32_t g = 0; g < T.ngroups; ++g)
            for (int32_t s = T.gptr[g]; s < T.gptr[g + 1]; ++s) lev_of[s] = g;
        for (int32_t g = 0; g < T.ngroups; ++g)
            for (int32_t s = T.gptr[g]; s < T.gptr[g + 1]; ++s)
                for (int l = 0; l < 32; ++l) {
                    uint8_t* R = T.rrec.data() + ((size_t)s * 32 + l) * SPCG_RREC_BYTES;
                    const int32_t r = T.rows[(size_t)s * 32 + l];
                    const int32_t w0 = (r + 1) | (g << 16);
                    const int32_t len = r >= 0 ? (int32_t)(dep_end(r) - dep_begin(r)) : 0;
                    const int32_t nxt = s + SPCG_RES_WARPS < ns ? lev_of[s + SPCG_RES_WARPS] : 0xffff;
                    const int32_t w1 = len | (nxt << 16);
                    memcpy(R, &w0, 4);
                    memcpy(R + 4, &w1, 4);
                    for (int k = 0; k < SPCG_RREC_PF && k < len; ++k) {
                        const int32_t j = M.col[dep_begin(r) + k];
                        const double v = M.val[dep_begin(r) + k];
                        memcpy(R + 16 + 4 * k, &j, 4);
                        memcpy(R + 32 + 8 * k, &v, 8);
                    }
                    const double dv = (upper && r >= 0) ? 1.0 / M.val[M.rp[r]] : 0.0;
                    memcpy(R + 8, &dv, 8);
                }
    }

    const size_t ne = (size_t)T.total_cols * 32;
    T.src.assign(ne, 0);
    T.val.assign(ne, 0.0);
    for (int32_t s = 0; s < ns; ++s) {
        const int64_t wdt = T.eoff[s + 1] - T.eoff[s];
        for (int l = 0; l < 32; ++l) {
            int32_t r = T.rows[(size_t)s * 32 + l];
            int64_t len = r >= 0 ? dep_end(r) - dep_begin(r) : 0;
            for (int64_t k = 0; k < wdt; ++k) {
                size_t e = (size_t)(T.eoff[s] + k) * 32 + l;
                if (k >= len) {                  // padding: never read (k >= rlen)
                    T.val[e] = 0.0;
                    T.src[e] = 0;
                    continue;
                }
                int64_t q = dep_begin(r) + k;
                int32_t j = M.col[q];
                T.val[e] = M.val[q];
                if (strategy == SPCG_SPTRSV_CHUNKED) {
                    int c = part_of[r];
                    bool same = part_of[j] == c;
                    bool safe = same && next_writer[j] > step_of[r];
                    if (safe) {
                        T.src[e] = (int32_t)((j - pb[c]) & (ring - 1));
                    } else {
                        T.src[e] = -j - 1;
                        T.publish[slot_of[j]] = 1;
                    }
                } else {
                    T.src[e] = -j - 1;
                }
            }
        }
    }
}

// ---------------------------------------------------------------- chunked stream
// Partition of the rows over the CTAs (parts) for the chunked executor.
//
// Level-balanced affinity partition: wavefront by wavefront (levels of the L
// solve), every row goes to the part that owns most of its dependencies, but
// no part takes more than its equal share of that wavefront.  Every wavefront
// is therefore spread over all CTAs (parallelism), while dependency chains
// stay inside a CTA where possible (locality: the shared-memory ring instead of
// a cross-CTA flag).  Rows without dependencies are placed by their position
// inside the wavefront.  Needs no geometry.
struct Partition {
    int parts = 1;
    std::vector<int32_t> part_of;              // [n]
    std::vector<int32_t> lidx;                 // [n] index inside the part (ascending rows)
    std::vector<std::vector<int32_t>> rows;    // per part, ascending
};

static void partition_level_based(const Factors& F, int P, bool affinity, Partition& out) {
    const int64_t n = F.L.n;
    out.parts = P;
    out.part_of.assign(n, -1);
    std::vector<int64_t> lp(F.wL + 1, 0);
    for (int64_t i = 0; i < n; ++i) lp[F.levL[i] + 1]++;
    for (int64_t l = 0; l < F.wL; ++l) lp[l + 1] += lp[l];
    std::vector<int32_t> lrows(n);
    {
        std::vector<int64_t> nx(lp.begin(), lp.end() - 1);
        for (int64_t i = 0; i < n; ++i) lrows[nx[F.levL[i]]++] = (int32_t)i;
    }
    std::vector<int32_t> load(P, 0), cnt(P, 0), touched;
    std::vector<int32_t> deferred, target;
    for (int64_t l = 0; l < F.wL && !affinity; ++l) {   // position-in-wavefront variant
        // position-in-wavefront: the t-th of m rows (ascending) goes to part floor(t P / m)
        const int64_t m = lp[l + 1] - lp[l];
        for (int64_t t = lp[l]; t < lp[l + 1]; ++t) out.part_of[lrows[t]] = (int32_t)(((t - lp[l]) * P) / m);
    }
    for (int64_t l = 0; l < F.wL && affinity; ++l) {
        const int64_t m = lp[l + 1] - lp[l];
        const int32_t cap = (int32_t)((m + P - 1) / P);
        std::fill(load.begin(), load.end(), 0);
        deferred.clear();
        target.clear();
        for (int64_t t = lp[l]; t < lp[l + 1]; ++t) {
            const int32_t i = lrows[t];
            // part owning most dependencies (ties: the larger dependency row's part)
            int best = -1, bestc = 0;
            touched.clear();
            for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
                const int pj = out.part_of[F.L.col[q]];
                if (cnt[pj]++ == 0) touched.push_back(pj);
                if (cnt[pj] >= bestc) { bestc = cnt[pj]; best = pj; }
            }
            for (int pj : touched) cnt[pj] = 0;
            if (best >= 0 && load[best] < cap) {
                out.part_of[i] = best;
                load[best]++;
            } else {
                deferred.push_back(i);
                target.push_back(best >= 0 ? best : (int)(((t - lp[l]) * P) / m));
            }
        }
        // deferred rows: nearest part (by id) with spare capacity
        std::set<int> open;
        for (int p = 0; p < P; ++p) if (load[p] < cap) open.insert(p);
        for (size_t d = 0; d < deferred.size(); ++d) {
            auto it = open.lower_bound(target[d]);
            int p;
            if (it == open.end()) p = *open.rbegin();
            else if (it == open.begin()) p = *it;
            else { auto pr = std::prev(it); p = (*it - target[d] <= target[d] - *pr) ? *it : *pr; }
            out.part_of[deferred[d]] = p;
            if (++load[p] >= cap) open.erase(p);
        }
    }
    out.rows.assign(P, {});
    out.lidx.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int p = out.part_of[i];
        out.lidx[i] = (int32_t)out.rows[p].size();
        out.rows[p].push_back((int32_t)i);
    }
}

// Contiguous ranges of a row ordering, balanced by per-row work.
static void partition_contiguous(const Factors& F, int P, const std::vector<int32_t>& ord, Partition& out) {
    const int64_t n = F.L.n;
    out.parts = P;
    out.part_of.assign(n, 0);
    double tot = 0.0;
    for (int64_t i = 0; i < n; ++i) tot += 4.0 + (double)(F.L.rp[i + 1] - F.L.rp[i]) + (double)(F.U.rp[i + 1] - F.U.rp[i]);
    double acc = 0.0;
    for (int64_t t = 0; t < n; ++t) {
        const int32_t i = ord[t];
        const double wi = 4.0 + (double)(F.L.rp[i + 1] - F.L.rp[i]) + (double)(F.U.rp[i + 1] - F.U.rp[i]);
        out.part_of[i] = std::min(P - 1, (int)((acc + 0.5 * wi) * P / tot));
        acc += wi;
    }
    out.rows.assign(P, {});
    out.lidx.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int p = out.part_of[i];
        out.lidx[i] = (int32_t)out.rows[p].size();
        out.rows[p].push_back((int32_t)i);
    }
}

// Connected components of the dependency graph of L (undirected), packed onto
// the parts largest first (LPT by rows).  When sparsification decouples the
// matrix into independent blocks (the layered field: Algorithm 2 removes the
// weak couplings across the low-conductivity columns) this
// partition has no cross-CTA dependency at all: every wavefront chain stays in
// one CTA's shared-memory ring.  Returns the number of components.
static int64_t partition_components(const Factors& F, int P, Partition& out) {
    const int64_t n = F.L.n;
    std::vector<int32_t> par(n);
    for (int64_t i = 0; i < n; ++i) par[i] = (int32_t)i;
    auto find = [&](int32_t x) {
        while (par[x] != x) { par[x] = par[par[x]]; x = par[x]; }
        return x;
    };
    for (int64_t i = 0; i < n; ++i)
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
            const int32_t a = find((int32_t)i), b = find(F.L.col[q]);
            if (a != b) par[std::max(a, b)] = std::min(a, b);
        }
    std::vector<int32_t> comp(n), size_of;
    std::vector<int32_t> id(n, -1);
    for (int64_t i = 0; i < n; ++i) {
        const int32_t r = find((int32_t)i);
        if (id[r] < 0) { id[r] = (int32_t)size_of.size(); size_of.push_back(0); }
        comp[i] = id[r];
        size_of[id[r]]++;
    }
    const int64_t nc = (int64_t)size_of.size();
    std::vector<int32_t> order(nc);
    for (int64_t c = 0; c < nc; ++c) order[c] = (int32_t)c;
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return size_of[a] > size_of[b]; });
    std::vector<int64_t> load(P, 0);
    std::vector<int32_t> part_of_comp(nc, 0);
    for (int32_t c : order) {
        int best = 0;
        for (int p = 1; p < P; ++p) if (load[p] < load[best]) best = p;
        part_of_comp[c] = best;
        load[best] += size_of[c];
    }
    out.parts = P;
    out.part_of.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) out.part_of[i] = part_of_comp[comp[i]];
    out.rows.assign(P, {});
    out.lidx.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int p = out.part_of[i];
        out.lidx[i] = (int32_t)out.rows[p].size();
        out.rows[p].push_back((int32_t)i);
    }
    return nc;
}

// Executor model used to pick a partition: every part walks its wavefront groups
// in order, a slice of <= 32 rows costs t_rec, and a dependency produced by
// another part is usable H after it was produced.  Returns the modelled time of
// one forward solve (the backward solve mirrors it).
static double model_solve_time(const Factors& F, const Partition& PT, double t_rec, double t_ext, double H) {
    const int64_t n = F.L.n;
    std::vector<int64_t> lp(F.wL + 1, 0);
    for (int64_t i = 0; i < n; ++i) lp[F.levL[i] + 1]++;
    for (int64_t l = 0; l < F.wL; ++l) lp[l + 1] += lp[l];
    std::vector<int32_t> lrows(n);
    {
        std::vector<int64_t> nx(lp.begin(), lp.end() - 1);
        for (int64_t i = 0; i < n; ++i) lrows[nx[F.levL[i]]++] = (int32_t)i;
    }
    std::vector<double> fin(n, 0.0), clock(PT.parts, 0.0), ready(PT.parts, 0.0);
    std::vector<int32_t> cnt(PT.parts, 0), touched;
    std::vector<int32_t> ext(PT.parts, 0);
    for (int64_t l = 0; l < F.wL; ++l) {
        touched.clear();
        for (int64_t t = lp[l]; t < lp[l + 1]; ++t) {
            const int32_t i = lrows[t];
            const int p = PT.part_of[i];
            if (cnt[p]++ == 0) { touched.push_back(p); ready[p] = clock[p]; }
            bool e = false;
            for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
                const int32_t j = F.L.col[q];
                if (PT.part_of[j] != p) { ready[p] = std::max(ready[p], fin[j] + H); e = true; }
            }
            ext[p] += e;
        }
        for (int p : touched) {
            // cross-CTA terms cost extra: half of it once the record has any (poller handoff),
            // half in proportion to the rows that have them (fitted to the poisson3d 48^3 /
            // 64^3 / 102^3 measurements of strided, tiles and affinity)
            const double f = (double)ext[p] / (double)cnt[p];
            const double tr = ext[p] ? t_rec + 0.5 * (t_ext - t_rec) * (1.0 + f) : t_rec;
            clock[p] = ready[p] + tr * (double)((cnt[p] + 31) / 32);
            cnt[p] = 0;
            ext[p] = 0;
        }
        for (int64_t t = lp[l]; t < lp[l + 1]; ++t) fin[lrows[t]] = clock[PT.part_of[lrows[t]]];
    }
    return *std::max_element(clock.begin(), clock.end());
}

// most frequent strictly-lower offset i - j > 1 of L (the grid line length for stencils)
static int64_t dominant_stride(const Factors& F) {
    std::map<int64_t, int64_t> h;
    const int64_t n = F.L.n;
    const int64_t step = std::max<int64_t>(1, n / 20000);
    for (int64_t i = 0; i < n; i += step)
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
            const int64_t d = i - F.L.col[q];
            if (d > 1) h[d]++;
        }
    int64_t best = 0, bc = 0;
    for (auto& kv : h) if (kv.second > bc) { bc = kv.second; best = kv.first; }
    return best;
}

// 3-D natural-order grids (two strides s1 | s2 among L's offsets: x-lines of length
// s1, planes of s2 rows): whole x-lines stay in one part, the (y, z) plane of lines
// is tiled Ty x Tz <= P.  The x-chain then runs through the ring; only the tile
// faces exchange flags, and the cross-CTA pipeline is Ty + Tz hops deep instead of
// the P-long chain of a slab partition.  Returns false if no such strides exist.
static bool partition_tiles(const Factors& F, int P, Partition& out) {
    const int64_t n = F.L.n;
    std::map<int64_t, int64_t> h;
    const int64_t step = std::max<int64_t>(1, n / 20000);
    for (int64_t i = 0; i < n; i += step)
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
            const int64_t d = i - F.L.col[q];
            if (d > 1) h[d]++;
        }
    std::vector<std::pair<int64_t, int64_t>> byc;
    for (auto& kv : h) byc.push_back({-kv.second, kv.first});
    std::sort(byc.begin(), byc.end());
    if (byc.size() < 2) return false;
    int64_t s1 = byc[0].second, s2 = 0;
    for (size_t k = 1; k < byc.size() && k < 4; ++k)
        if (byc[k].second > s1 && byc[k].second % s1 == 0) { s2 = byc[k].second; break; }
    if (s2 == 0 || s1 < 2) {
        // the two leading offsets may come in the other order
        if (byc[1].second < s1 && s1 % byc[1].second == 0) { s2 = s1; s1 = byc[1].second; }
        else return false;
    }
    const int64_t NY = s2 / s1, NZ = (n + s2 - 1) / s2;
    if (NY < 2 || NZ < 2) return false;
    int Ty = std::max<int>(1, (int)std::lround(std::sqrt((double)P * (double)NY / (double)NZ)));
    Ty = (int)std::min<int64_t>(Ty, NY);
    int Tz = (int)std::min<int64_t>(std::max(1, P / Ty), NZ);
    // a tile must fit one 32-row record per wavefront (one row per x-line and level);
    // larger tiles split every wavefront into several records and lose to the slab
    // partitions (measured: 64^3 tiles 0.49 vs strided 0.54 ms/it; 102^3 1.48 vs 1.29)
    if ((double)NY * (double)NZ / ((double)Ty * (double)Tz) > 32.0) return false;
    out.parts = P;
    out.part_of.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int64_t y = (i / s1) % NY, z = i / s2;
        out.part_of[i] = (int32_t)(((z * Tz) / NZ) * Ty + (y * Ty) / NY);
    }
    out.rows.assign(P, {});
    out.lidx.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int p = out.part_of[i];
        out.lidx[i] = (int32_t)out.rows[p].size();
        out.rows[p].push_back((int32_t)i);
    }
    return true;
}

// Inspector: build candidate partitions and keep the one the model says is fastest.
static void partition_rows(const Factors& F, int P, int force_part, Partition& out, std::string* chosen) {
    const int64_t n = F.L.n;
    // microseconds per record without / with cross-CTA terms, handoff latency: measured on
    // B200 (tools/diag.py timelines)
    const double T_REC = 0.45, T_EXT = 0.8, H = 1.0;
    std::vector<std::pair<std::string, Partition>> cand;
    std::vector<int32_t> ord(n);
    for (int64_t i = 0; i < n; ++i) ord[i] = (int32_t)i;
    { Partition p; partition_contiguous(F, P, ord, p); cand.push_back({"contiguous", std::move(p)}); }
    const int64_t s = dominant_stride(F);
    if (s > 1 && s < n) {
        // rows ordered by (i mod s, i / s): contiguous ranges become strips across the stride
        std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return a % s < b % s; });
        Partition p;
        partition_contiguous(F, P, ord, p);
        cand.push_back({"strided", std::move(p)});
    }
    { Partition p; partition_level_based(F, P, true, p); cand.push_back({"affinity", std::move(p)}); }
    {
        Partition p;
        if (partition_components(F, P, p) >= P) cand.push_back({"components", std::move(p)});
    }
    {
        Partition p;
        if (partition_tiles(F, P, p)) cand.push_back({"tiles", std::move(p)});
    }
    static const char* kinds[] = {"contiguous", "strided", "affinity", "components", "tiles"};
    const char* force = (force_part >= 0 && force_part < 5) ? kinds[force_part] : nullptr;
    double best = 1e300;
    size_t bi = 0;
    bool forced = false;
    for (size_t c = 0; c < cand.size(); ++c) {
        // the model underrates the affinity partition (its rows' dependencies often go
        // through flags instead of the ring): measured 11 % slower than predicted relative
        // to strided on poisson3d 102^3, so it carries a 15 % penalty
        const double t = model_solve_time(F, cand[c].second, T_REC, T_EXT, H) * (cand[c].first == "affinity" ? 1.15 : 1.0);
        if (force && cand[c].first == force) { bi = c; forced = true; }
        if (!forced && t < best) { best = t; bi = c; }
    }
    out = std::move(cand[bi].second);
    if (chosen) *chosen = cand[bi].first;
}

// Ring-safety of intra-part dependencies for one factor (slot = lidx & (ring-1)):
// entry (i,j) may read j from the shared ring iff no other row of the part that
// maps to the same slot is written between j's step and i's step (inclusive).
static void ring_analysis(const Partition& PT, const std::vector<int32_t>& lev, int32_t ring,
                          std::vector<int32_t>& step_of, std::vector<int32_t>& next_writer) {
    const int64_t n = (int64_t)PT.part_of.size();
    step_of.assign(n, 0);
    next_writer.assign(n, INT32_MAX);
    std::vector<int32_t> lv;
    std::vector<std::pair<int32_t, int32_t>> mem;
    for (int c = 0; c < PT.parts; ++c) {
        const std::vector<int32_t>& R = PT.rows[c];
        lv.clear();
        for (int32_t i : R) lv.push_back(lev[i]);
        std::sort(lv.begin(), lv.end());
        lv.erase(std::unique(lv.begin(), lv.end()), lv.end());
        for (int32_t i : R) step_of[i] = (int32_t)(std::lower_bound(lv.begin(), lv.end(), lev[i]) - lv.begin());
        if ((int64_t)R.size() <= ring) continue;
        for (int64_t cls = 0; cls < ring; ++cls) {
            mem.clear();
            for (int64_t t = cls; t < (int64_t)R.size(); t += ring) mem.push_back({step_of[R[t]], R[t]});
            if (mem.size() < 2) continue;
            std::sort(mem.begin(), mem.end());
            for (size_t a = 0; a < mem.size();) {
                size_t b = a;
                while (b < mem.size() && mem[b].first == mem[a].first) ++b;
                const int32_t nxt = (b - a > 1) ? mem[a].first : (b < mem.size() ? mem[b].first : INT32_MAX);
                for (size_t t = a; t < b; ++t) next_writer[mem[t].second] = nxt;
                a = b;
            }
        }
    }
}

namespace {
struct StreamWriter {
    ChunkStream& S;
    int64_t cur = -1;       // current chunk index
    int32_t used = 0, nrec = 0;
    explicit StreamWriter(ChunkStream& s) : S(s) {}
    void new_chunk() {
        if (cur >= 0) finish();
        cur = (int64_t)(S.bytes.size() / SPCG_CHUNK_BYTES);
        S.bytes.resize(S.bytes.size() + SPCG_CHUNK_BYTES, 0);
        used = SPCG_CHUNK_HDR;
        nrec = 0;
    }
    void finish() {
        uint8_t* c = &S.bytes[cur * SPCG_CHUNK_BYTES];
        uint16_t nr = (uint16_t)nrec;
        uint32_t ub = (uint32_t)used;
        std::memcpy(c + 0, &nr, 2);
        std::memcpy(c + 4, &ub, 4);
        S.used_bytes += used;
        if ((int64_t)S.chunk_bytes.size() <= cur) S.chunk_bytes.resize(cur + 1, 16);
        S.chunk_bytes[cur] = ub;
    }
    uint8_t* alloc(int32_t bytes, uint8_t& side) {
        if (cur < 0 || used + bytes > SPCG_CHUNK_BYTES || nrec == SPCG_MAXREC) new_chunk();
        uint8_t* p = &S.bytes[cur * SPCG_CHUNK_BYTES + used];
        uint16_t off = (uint16_t)used;
        std::memcpy(&S.bytes[cur * SPCG_CHUNK_BYTES + 8 + 2 * nrec], &off, 2);   // record offset table
        used += bytes;
        side = (uint8_t)nrec++;
        S.records++;
        return p;
    }
};

template <class T>
void put(uint8_t* base, size_t off, T v) { std::memcpy(base + off, &v, sizeof(T)); }
}  // namespace

// one phase (L or U) of one part into the stream
static void emit_section(StreamWriter& W, const Csr& M, bool upper, const std::vector<int32_t>& lev,
                         const std::vector<int32_t>& prow, const Partition& PT, const std::vector<int32_t>& step_of,
                         const std::vector<int32_t>& next_writer, const std::vector<uint8_t>& publish, int32_t ring,
                         bool sync_first, int64_t& seq) {
    if (prow.empty()) return;
    auto dep_begin = [&](int64_t i) { return upper ? M.rp[i] + 1 : M.rp[i]; };
    // rows of the part grouped by level (ascending), rows ascending inside a level
    std::vector<int32_t> order(prow.begin(), prow.end());
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return lev[a] < lev[b]; });
    int prev_ns = -1;
    bool first_record = true;
    std::vector<int32_t> esrc[32];
    std::vector<double> evalv[32];
    int ne_tot[32];
    for (size_t g0 = 0; g0 < order.size();) {
        size_t g1 = g0;
        while (g1 < order.size() && lev[order[g1]] == lev[order[g0]]) ++g1;
        const int ns = (int)((g1 - g0 + 31) / 32);
        bool sync = (first_record && sync_first) || !(prev_ns == 1 && ns == 1);
        if (first_record && !sync_first) sync = false;
        for (int sl = 0; sl < ns; ++sl) {
            const size_t s0 = g0 + 32 * sl, s1 = std::min(g1, s0 + 32);
            const int m = (int)(s1 - s0);
            int wmax = 0;
            for (int l = 0; l < m; ++l) {
                const int32_t r = order[s0 + l];
                esrc[l].clear();
                evalv[l].clear();
                // mailbox entries first (CSR order), then ring entries (CSR order)
                for (int pass = 0; pass < 2; ++pass)
                    for (int64_t q = dep_begin(r); q < M.rp[r + 1]; ++q) {
                        const int32_t j = M.col[q];
                        const bool safe = PT.part_of[j] == PT.part_of[r] && next_writer[j] > step_of[r];
                        if ((pass == 0) == safe) continue;
                        esrc[l].push_back(safe ? (int32_t)(PT.lidx[j] & (ring - 1)) : -j - 1);
                        evalv[l].push_back(M.val[q]);
                    }
                ne_tot[l] = 0;
                for (int32_t sidx : esrc[l]) ne_tot[l] += sidx < 0;
                wmax = std::max<int>(wmax, (int)esrc[l].size());
            }
            const int warp = (int)(seq++ % SPCG_NSOLVER);   // slices of the part's stream, round-robin
            int k0 = 0;
            do {
                const int wp = std::min(SPCG_WCAP, wmax - k0);
                const bool firstp = (k0 == 0), lastp = (k0 + wp >= wmax);
                const int bytes = SPCG_REC_HDR + 384 * wp + ((upper && lastp) ? 256 : 0);
                uint8_t side = 0;
                uint8_t* rec = W.alloc(bytes, side);
                uint16_t flags = (firstp ? REC_FIRST : 0) | (lastp ? REC_LAST : 0) | (upper ? REC_UPPER : 0) |
                                 ((firstp && sl == 0 && sync) ? REC_SYNC : 0);
                uint32_t pub = 0, act = 0;
                bool any_ext = false;
                for (int l = 0; l < m; ++l) {
                    act |= 1u << l;
                    if (lastp && publish[order[s0 + l]]) pub |= 1u << l;
                    if (std::min<int>(wp, (int)esrc[l].size() - k0) > 0 && ne_tot[l] - k0 > 0) any_ext = true;
                }
                if (any_ext) flags |= REC_EXT;
                if (wp > SPCG_WP) flags |= REC_WIDE;
                // header: w, flags, warp, side, bytes, publish mask, active mask
                put<uint16_t>(rec, 0, (uint16_t)wp);
                put<uint16_t>(rec, 2, flags);
                put<uint8_t>(rec, 4, (uint8_t)warp);
                put<uint8_t>(rec, 5, side);
                put<uint16_t>(rec, 6, (uint16_t)bytes);
                put<uint32_t>(rec, 8, pub);
                put<uint32_t>(rec, 12, act);
                for (int l = 0; l < 32; ++l) {
                    const int32_t r = l < m ? order[s0 + l] : -1;
                    int len = 0, ne = 0;
                    uint32_t dst = 0;
                    if (l < m) {
                        len = std::max(0, std::min<int>(wp, (int)esrc[l].size() - k0));
                        ne = std::max(0, std::min<int>(len, ne_tot[l] - k0));
                        dst = (uint32_t)(PT.lidx[r] & (ring - 1));
                    }
                    // lane word: {row, meta = len | ne << 8 | publish << 16 | ring slot << 17}
                    const uint32_t meta = (uint32_t)len | ((uint32_t)ne << 8) | (((pub >> l) & 1u) << 16) | (dst << 17);
                    put<int32_t>(rec, 16 + 8 * l, r);
                    put<uint32_t>(rec, 20 + 8 * l, meta);
                    for (int k = 0; k < len; ++k) {
                        put<int32_t>(rec, SPCG_REC_HDR + 128 * k + 4 * l, esrc[l][k0 + k]);
                        put<double>(rec, SPCG_REC_HDR + 128 * wp + 256 * k + 8 * l, evalv[l][k0 + k]);
                    }
                    if (upper && lastp && l < m) put<double>(rec, SPCG_REC_HDR + 384 * wp + 8 * l, 1.0 / M.val[M.rp[r]]);
                }
                k0 += wp;
                first_record = false;
            } while (k0 < wmax);
        }
        prev_ns = ns;
        g0 = g1;
    }
}

static void build_chunk_stream(const Factors& F, const Partition& PT, int32_t ring, ChunkStream& S) {
    const int64_t n = F.L.n;
    const int parts = PT.parts;
    std::vector<int32_t> stepL, nwL, stepU, nwU;
    ring_analysis(PT, F.levL, ring, stepL, nwL);
    ring_analysis(PT, F.levU, ring, stepU, nwU);
    std::vector<uint8_t> pubL(n, 0), pubU(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
            const int32_t j = F.L.col[q];
            if (!(PT.part_of[j] == PT.part_of[i] && nwL[j] > stepL[i])) pubL[j] = 1;
        }
        for (int64_t q = F.U.rp[i] + 1; q < F.U.rp[i + 1]; ++q) {
            const int32_t j = F.U.col[q];
            if (!(PT.part_of[j] == PT.part_of[i] && nwU[j] > stepU[i])) pubU[j] = 1;
        }
    }
    S = ChunkStream();
    StreamWriter W(S);
    S.part_chunk.assign(parts + 1, 0);
    S.part_uchunk.assign(parts, 0);
    for (int c = 0; c < parts; ++c) {
        W.new_chunk();
        S.part_chunk[c] = (int32_t)W.cur;
        int64_t seq = 0;                     // slice sequence of this part (L then U section)
        emit_section(W, F.L, false, F.levL, PT.rows[c], PT, stepL, nwL, pubL, ring, false, seq);
        W.new_chunk();                     // U section starts on a chunk boundary
        S.part_uchunk[c] = (int32_t)W.cur;
        emit_section(W, F.U, true, F.levU, PT.rows[c], PT, stepU, nwU, pubU, ring, true, seq);
    }
    W.finish();
    S.part_chunk[parts] = (int32_t)(S.bytes.size() / SPCG_CHUNK_BYTES);
    S.chunk_bytes.resize(S.part_chunk[parts], 16);
}

void build_tri_layouts(const Factors& F, int strategy, int parts, int ring_max, double wide_min, int force_part,
                       Layouts& out) {
    const int64_t n = F.L.n;
    out.strategy = strategy;
    out.parts = parts;
    out.part_begin.assign(parts + 1, 0);
    if (strategy == SPCG_SPTRSV_CHUNKED) {
        Partition PT;
        partition_rows(F, parts, force_part, PT, &out.partition);
        // ring size: enough for the longest intra-part dependency distance in part-local
        // row numbering (slot = lidx & (ring - 1)), not the part size — a small ring leaves
        // shared memory to the L1 carve-out (layered 4096^2 SPCG: 8192 -> 64 entries).
        // Anything the ring cannot hold safely goes through the flags (ring analysis).
        int64_t maxdist = 1;
        for (const Csr* M : {&F.L, &F.U})
            for (int64_t i = 0; i < n; ++i)
                for (int64_t q = M->rp[i]; q < M->rp[i + 1]; ++q) {
                    const int32_t j = M->col[q];
                    if (j != i && PT.part_of[j] == PT.part_of[i])
                        maxdist = std::max<int64_t>(maxdist, std::llabs((int64_t)PT.lidx[i] - PT.lidx[j]));
                }
        // >= 16 entries: the ring occupies the front of dynamic shared memory and the
        // chunk slots behind it need 128-byte alignment (TMA destination, 16-byte header
        // loads); a 1- or 2-entry ring (n = 1) misaligned them (found by the n = 1 test)
        int32_t small = 16;
        while ((int64_t)small <= 2 * maxdist && small < ring_max) small <<= 1;
        // rows run in wavefront order, not in lidx order, so a short distance does not
        // make a small ring safe: keep it only if it sends no more dependencies through
        // the flags than the largest ring does (ring_analysis decides entry by entry)
        auto unsafe = [&](int32_t R) {
            int64_t cnt = 0;
            std::vector<int32_t> st, nw;
            for (int f = 0; f < 2; ++f) {
                const Csr& M = f ? F.U : F.L;
                ring_analysis(PT, f ? F.levU : F.levL, R, st, nw);
                for (int64_t i = 0; i < n; ++i)
                    for (int64_t q = M.rp[i]; q < M.rp[i + 1]; ++q) {
                        const int32_t j = M.col[q];
                        if (j != i && PT.part_of[j] == PT.part_of[i] && !(nw[j] > st[i])) ++cnt;
                    }
            }
            return cnt;
        };
        int32_t ring = ring_max;
        if (small < ring_max && unsafe(small) <= unsafe(ring_max)) ring = small;
        out.ring = ring;
        for (int c = 0; c < parts; ++c) out.part_begin[c + 1] = out.part_begin[c] + (int64_t)PT.rows[c].size();
        build_chunk_stream(F, PT, ring, out.S);
        return;
    }
    out.part_begin[parts] = n;
    out.ring = 0;
    const std::vector<int64_t> pb{0, n};
    build_tri(F.L, false, F.levL, F.wL, strategy, pb, out.ring, wide_min, out.L);
    build_tri(F.U, true, F.levU, F.wU, strategy, pb, out.ring, wide_min, out.U);
}

}  // namespace spcg
