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
    out.col.assign(out.eoff[ns] * 32, 0);
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
                      int strategy, const std::vector<int64_t>& pb, int32_t ring, TriLayout& T) {
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

void build_tri_layouts(const Factors& F, int strategy, int parts, int ring_max, Layouts& out) {
    const int64_t n = F.L.n;
    out.strategy = strategy;
    out.parts = parts;
    out.part_begin.assign(parts + 1, 0);
    if (strategy == SPCG_SPTRSV_CHUNKED) {
        // contiguous row ranges balanced by per-row work (rows + factor entries)
        std::vector<double> pre(n + 1, 0.0);
        for (int64_t i = 0; i < n; ++i)
            pre[i + 1] = pre[i] + 4.0 + (double)(F.L.rp[i + 1] - F.L.rp[i]) + (double)(F.U.rp[i + 1] - F.U.rp[i]);
        int64_t r = 0;
        for (int c = 1; c < parts; ++c) {
            double target = pre[n] * c / parts;
            while (r < n && pre[r] < target) ++r;
            out.part_begin[c] = r;
        }
        out.part_begin[parts] = n;
        int64_t maxsz = 0;
        for (int c = 0; c < parts; ++c) maxsz = std::max(maxsz, out.part_begin[c + 1] - out.part_begin[c]);
        int32_t ring = 1;
        while (ring < maxsz && ring < ring_max) ring <<= 1;
        out.ring = ring;
    } else {
        out.part_begin[parts] = n;
        out.ring = 0;
    }
    std::vector<int64_t> pb = strategy == SPCG_SPTRSV_CHUNKED ? out.part_begin : std::vector<int64_t>{0, n};
    build_tri(F.L, false, F.levL, F.wL, strategy, pb, out.ring, out.L);
    build_tri(F.U, true, F.levU, F.wU, strategy, pb, out.ring, out.U);
}

}  // namespace spcg
