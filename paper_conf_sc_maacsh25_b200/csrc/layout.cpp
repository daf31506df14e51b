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

// ---------------------------------------------------------------- chunked stream
// Ring-safety of intra-part dependencies for one factor (slot = (row - part_begin) & (ring-1)):
// entry (i,j) may read j from the shared ring iff no other row of the part that maps to the
// same slot is written between j's step and i's step (inclusive).
static void ring_analysis(const Csr& M, bool upper, const std::vector<int32_t>& lev, const std::vector<int64_t>& pb,
                          int32_t ring, std::vector<int32_t>& part_of, std::vector<int32_t>& step_of,
                          std::vector<int32_t>& next_writer) {
    const int64_t n = M.n;
    const int parts = (int)pb.size() - 1;
    (void)upper;
    part_of.assign(n, 0);
    step_of.assign(n, 0);
    next_writer.assign(n, INT32_MAX);
    for (int c = 0; c < parts; ++c) {
        int32_t lmin = INT32_MAX;
        for (int64_t i = pb[c]; i < pb[c + 1]; ++i) { part_of[i] = c; lmin = std::min(lmin, lev[i]); }
        // steps = dense rank of the levels present in the part
        std::vector<int32_t> lv;
        for (int64_t i = pb[c]; i < pb[c + 1]; ++i) lv.push_back(lev[i]);
        std::sort(lv.begin(), lv.end());
        lv.erase(std::unique(lv.begin(), lv.end()), lv.end());
        for (int64_t i = pb[c]; i < pb[c + 1]; ++i)
            step_of[i] = (int32_t)(std::lower_bound(lv.begin(), lv.end(), lev[i]) - lv.begin());
        const int64_t sz = pb[c + 1] - pb[c];
        if (sz <= ring) continue;
        std::vector<std::pair<int32_t, int32_t>> mem;
        for (int64_t cls = 0; cls < ring; ++cls) {
            mem.clear();
            for (int64_t j = pb[c] + cls; j < pb[c + 1]; j += ring) mem.push_back({step_of[j], (int32_t)j});
            if (mem.size() < 2) continue;
            std::sort(mem.begin(), mem.end());
            for (size_t a = 0; a < mem.size();) {
                size_t b = a;
                while (b < mem.size() && mem[b].first == mem[a].first) ++b;
                int32_t nxt = (b - a > 1) ? mem[a].first : (b < mem.size() ? mem[b].first : INT32_MAX);
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
        used = 16;
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
static void emit_section(StreamWriter& W, const Csr& M, bool upper, const std::vector<int32_t>& lev, int64_t lo,
                         int64_t hi, const std::vector<int32_t>& part_of, const std::vector<int32_t>& step_of,
                         const std::vector<int32_t>& next_writer, const std::vector<uint8_t>& publish, int64_t pbc,
                         int32_t ring, bool sync_first) {
    if (hi <= lo) return;
    auto dep_begin = [&](int64_t i) { return upper ? M.rp[i] + 1 : M.rp[i]; };
    // rows of the part grouped by level (ascending), rows ascending inside a level
    std::vector<int32_t> order;
    for (int64_t i = lo; i < hi; ++i) order.push_back((int32_t)i);
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
                        const bool safe = part_of[j] == part_of[r] && next_writer[j] > step_of[r];
                        if ((pass == 0) == safe) continue;
                        esrc[l].push_back(safe ? (int32_t)((j - pbc) & (ring - 1)) : -j - 1);
                        evalv[l].push_back(M.val[q]);
                    }
                ne_tot[l] = 0;
                for (int32_t sidx : esrc[l]) ne_tot[l] += sidx < 0;
                wmax = std::max<int>(wmax, (int)esrc[l].size());
            }
            const int warp = sl % SPCG_NSOLVER;
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
                    if (l < m) {
                        len = std::max(0, std::min<int>(wp, (int)esrc[l].size() - k0));
                        ne = std::max(0, std::min<int>(len, ne_tot[l] - k0));
                    }
                    // lane word: {row, meta = len | ne << 8 | publish << 16}
                    const uint32_t meta = (uint32_t)len | ((uint32_t)ne << 8) | (((pub >> l) & 1u) << 16);
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

static void build_chunk_stream(const Factors& F, const std::vector<int64_t>& pb, int32_t ring, ChunkStream& S) {
    const int64_t n = F.L.n;
    const int parts = (int)pb.size() - 1;
    std::vector<int32_t> partL, stepL, nwL, partU, stepU, nwU;
    ring_analysis(F.L, false, F.levL, pb, ring, partL, stepL, nwL);
    ring_analysis(F.U, true, F.levU, pb, ring, partU, stepU, nwU);
    std::vector<uint8_t> pubL(n, 0), pubU(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
            const int32_t j = F.L.col[q];
            if (!(partL[j] == partL[i] && nwL[j] > stepL[i])) pubL[j] = 1;
        }
        for (int64_t q = F.U.rp[i] + 1; q < F.U.rp[i + 1]; ++q) {
            const int32_t j = F.U.col[q];
            if (!(partU[j] == partU[i] && nwU[j] > stepU[i])) pubU[j] = 1;
        }
    }
    S = ChunkStream();
    StreamWriter W(S);
    S.part_chunk.assign(parts + 1, 0);
    S.part_uchunk.assign(parts, 0);
    for (int c = 0; c < parts; ++c) {
        W.new_chunk();
        S.part_chunk[c] = (int32_t)W.cur;
        emit_section(W, F.L, false, F.levL, pb[c], pb[c + 1], partL, stepL, nwL, pubL, pb[c], ring, false);
        W.new_chunk();                     // U section starts on a chunk boundary
        S.part_uchunk[c] = (int32_t)W.cur;
        emit_section(W, F.U, true, F.levU, pb[c], pb[c + 1], partU, stepU, nwU, pubU, pb[c], ring, true);
    }
    W.finish();
    S.part_chunk[parts] = (int32_t)(S.bytes.size() / SPCG_CHUNK_BYTES);
    S.chunk_bytes.resize(S.part_chunk[parts], 16);
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
    if (strategy == SPCG_SPTRSV_CHUNKED) {
        build_chunk_stream(F, pb, out.ring, out.S);
    } else {
        build_tri(F.L, false, F.levL, F.wL, strategy, pb, out.ring, out.L);
        build_tri(F.U, true, F.levU, F.wU, strategy, pb, out.ring, out.U);
    }
}

}  // namespace spcg
