// chain_layout.cpp — inspector of the warp-chain executor.
//
// The triangular solves of Algorithm 1 line 13 (forward/backward
// substitution P:L201-209) are executed wavefront by wavefront (the level sets of
// Fig. 1c/d).  Instead of a grid- or CTA-wide handoff per wavefront,
// rows are split into CHAINS that one warp walks alone: a step of a chain is <= 32
// rows of one level (one per lane), and a dependency produced by the same warp in
// its previous step is fetched with a register shuffle.  Only dependencies on other
// chains go through memory (ready flags, prefetched a chunk ahead).
//
// Partitions into chains (chosen in this order):
//   components  the dependency graph of L falls apart into connected components no
//               wider than 32 rows per level (the layered field after Algorithm 2
//               removes the weak couplings across its low-conductivity columns,
//               P:L463-469): components are skyline-packed onto the chains (each
//               keeps its own level structure, starting at whatever step its lanes
//               free up) — no dependency ever crosses a chain;
//   grid3d      a natural-order 3-D grid (two nested strides among L's offsets): the
//               (y, z) plane of x-lines is tiled Ty x Tz (<= 32 lines per chain);
//   grid2d      a natural-order 2-D grid (one dominant stride nx): 32-column blocks.
// Otherwise the executor does not apply (setup falls back to the others).
#include <algorithm>
#include <array>
#include <cmath>
#include <cstring>
#include <map>
#include <numeric>

#include "internal.h"

namespace spcg {

namespace {

struct ChainPart {
    std::vector<int32_t> chain_of;       // [n]
    std::vector<int64_t> key;            // [n] schedule key inside the chain (step order); empty = levL
    int32_t nchains = 0;
    std::string name;
};

int64_t find_root(std::vector<int32_t>& par, int32_t x) {
    while (par[x] != x) { par[x] = par[par[x]]; x = par[x]; }
    return x;
}

bool part_components(const Factors& F, int target_chains, ChainPart& out) {
    const int64_t n = F.L.n;
    std::vector<int32_t> par(n);
    std::iota(par.begin(), par.end(), 0);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) {
            const int32_t a = (int32_t)find_root(par, (int32_t)i), b = (int32_t)find_root(par, F.L.col[q]);
            if (a != b) par[std::max(a, b)] = std::min(a, b);
        }
    std::vector<int32_t> comp(n), id(n, -1);
    int32_t nc = 0;
    for (int64_t i = 0; i < n; ++i) {
        const int32_t r = (int32_t)find_root(par, (int32_t)i);
        if (id[r] < 0) id[r] = nc++;
        comp[i] = id[r];
    }
    // width of a component = max rows on one level; its levels form a contiguous range
    std::vector<int32_t> lmin(nc, INT32_MAX), lmax(nc, -1);
    for (int64_t i = 0; i < n; ++i) {
        lmin[comp[i]] = std::min(lmin[comp[i]], F.levL[i]);
        lmax[comp[i]] = std::max(lmax[comp[i]], F.levL[i]);
    }
    std::vector<int64_t> off(nc + 1, 0);
    for (int32_t c = 0; c < nc; ++c) off[c + 1] = off[c] + (lmax[c] - lmin[c] + 1);
    std::vector<int32_t> cnt(off[nc], 0), width(nc, 0), size(nc, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int32_t c = comp[i];
        const int32_t k = ++cnt[off[c] + F.levL[i] - lmin[c]];
        width[c] = std::max(width[c], k);
        size[c]++;
    }
    for (int32_t c = 0; c < nc; ++c)
        if (width[c] > 32) return false;
    // Components never depend on each other, so inside a chain each may start at any
    // step: skyline packing.  A component of width w (rows per level) and span h
    // (levels) takes w lanes of one chain for h consecutive steps, starting when its w
    // least-busy lanes are free; components go longest span first to the chain where
    // they finish earliest.  Rows per step never exceed 32 and each component keeps its
    // own level structure (a dependency stays one step back: a shuffle).
    int64_t area = 0, H = 0;
    for (int32_t c = 0; c < nc; ++c) {
        area += (int64_t)width[c] * (lmax[c] - lmin[c] + 1);
        H = std::max<int64_t>(H, lmax[c] - lmin[c] + 1);
    }
    int32_t NC = (int32_t)std::max<int64_t>(1, (area + 32 * H - 1) / (32 * H));
    NC = std::max<int32_t>(NC, std::min<int32_t>(target_chains, nc));
    std::vector<int32_t> order(nc);
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
        const int32_t ha = lmax[a] - lmin[a], hb = lmax[b] - lmin[b];
        return ha != hb ? ha > hb : width[a] > width[b];
    });
    std::vector<std::array<int64_t, 32>> fr(NC);      // per chain: lane free-from steps, ascending
    for (auto& f : fr) f.fill(0);
    std::vector<int32_t> chain_of_comp(nc, -1);
    std::vector<int64_t> start_of_comp(nc, 0), load(NC, 0);
    for (int32_t c : order) {
        const int w = width[c];
        const int64_t h = lmax[c] - lmin[c] + 1;
        int32_t best = 0;          // earliest finish; ties: the least loaded chain (rows)
        for (int32_t k = 1; k < NC; ++k)
            if (fr[k][w - 1] < fr[best][w - 1] || (fr[k][w - 1] == fr[best][w - 1] && load[k] < load[best])) best = k;
        load[best] += size[c];
        const int64_t start = fr[best][w - 1];
        for (int j = 0; j < w; ++j) fr[best][j] = start + h;
        std::sort(fr[best].begin(), fr[best].end());
        chain_of_comp[c] = best;
        start_of_comp[c] = start;
    }
    out.nchains = NC;
    out.chain_of.assign(n, 0);
    out.key.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        out.chain_of[i] = chain_of_comp[comp[i]];
        out.key[i] = start_of_comp[comp[i]] + (F.levL[i] - lmin[comp[i]]);
    }
    out.name = "components";
    return true;
}

// frequency of strictly-lower offsets i - j (sampled rows)
std::vector<std::pair<int64_t, int64_t>> offsets_by_count(const Factors& F) {
    std::map<int64_t, int64_t> h;
    const int64_t n = F.L.n;
    const int64_t step = std::max<int64_t>(1, n / 20000);
    for (int64_t i = 0; i < n; i += step)
        for (int64_t q = F.L.rp[i]; q < F.L.rp[i + 1]; ++q) h[i - F.L.col[q]]++;
    std::vector<std::pair<int64_t, int64_t>> v;
    for (auto& kv : h) v.push_back({kv.second, kv.first});
    std::sort(v.begin(), v.end(), [](auto& a, auto& b) { return a.first != b.first ? a.first > b.first : a.second < b.second; });
    return v;
}

bool part_grid3d(const Factors& F, ChainPart& out) {
    const int64_t n = F.L.n;
    auto v = offsets_by_count(F);
    // the x-line stride s1 and plane stride s2: the two most frequent offsets > 1 with s1 | s2
    int64_t s1 = 0, s2 = 0;
    std::vector<int64_t> big;
    for (auto& e : v)
        if (e.second > 1 && big.size() < 4) big.push_back(e.second);
    for (size_t a = 0; a < big.size() && !s2; ++a)
        for (size_t b = 0; b < big.size(); ++b)
            if (big[b] > big[a] && big[b] % big[a] == 0 && n % big[b] == 0) { s1 = big[a]; s2 = big[b]; break; }
    if (!s2) return false;
    const int64_t NY = s2 / s1, NZ = n / s2;
    if (NY < 2 || NZ < 2) return false;
    // tiles of Ty x Tz x-lines, Ty * Tz <= 32: fewest tile hops along the longest path
    int bestTy = 1, bestTz = 1;
    double best = 1e300;
    for (int Ty = 1; Ty <= 32; Ty *= 2) {
        const int Tz = 32 / Ty;
        const int ty = (int)std::min<int64_t>(Ty, NY), tz = (int)std::min<int64_t>(Tz, NZ);
        const double hops = std::ceil((double)NY / ty) + std::ceil((double)NZ / tz);
        const double cost = hops * 24.0 + ty + tz;      // a hop costs ~24 steps of pipeline lag
        if (cost < best) { best = cost; bestTy = ty; bestTz = tz; }
    }
    const int64_t ny_t = (NY + bestTy - 1) / bestTy;
    out.chain_of.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) {
        const int64_t y = (i / s1) % NY, z = i / s2;
        out.chain_of[i] = (int32_t)((z / bestTz) * ny_t + y / bestTy);
    }
    out.nchains = (int32_t)(ny_t * ((NZ + bestTz - 1) / bestTz));
    out.name = "grid3d";
    return true;
}

bool part_grid2d(const Factors& F, ChainPart& out) {
    const int64_t n = F.L.n;
    auto v = offsets_by_count(F);
    int64_t nx = 0;
    for (auto& e : v)
        if (e.second > 1) { nx = e.second; break; }
    if (nx < 2 || n % nx != 0 || n / nx < 2) return false;
    const int64_t nb = (nx + 31) / 32;
    out.chain_of.assign(n, 0);
    for (int64_t i = 0; i < n; ++i) out.chain_of[i] = (int32_t)((i % nx) / 32);
    out.nchains = (int32_t)nb;
    out.name = "grid2d";
    return true;
}

template <class T>
void put(fast_vector<uint8_t>& b, size_t off, T v) { std::memcpy(b.data() + off, &v, sizeof(T)); }

}  // namespace

bool build_chain_layout(const Csr& A, const Factors& F, int target_chains, bool f32, ChainLayout& out,
                        std::string* why) {
    const int64_t n = F.L.n;
    out = ChainLayout();
    // dependency columns per record
    int64_t wl = 0, wu = 0;
    for (int64_t i = 0; i < n; ++i) {
        wl = std::max<int64_t>(wl, F.L.rp[i + 1] - F.L.rp[i]);
        wu = std::max<int64_t>(wu, F.U.rp[i + 1] - F.U.rp[i] - 1);
    }
    if (wl > SPCG_CHAIN_WMAX || wu > SPCG_CHAIN_WMAX) {
        if (why) *why = "rows wider than SPCG_CHAIN_WMAX dependencies";
        return false;
    }
    ChainPart CP;
    if (!part_components(F, target_chains, CP) && !part_grid3d(F, CP) && !part_grid2d(F, CP)) {
        if (why) *why = "no chain partition (not decoupled, not a natural-order grid)";
        return false;
    }
    // chains: rows by (level, row); steps of <= 32 rows of one level
    std::vector<int64_t> cstart(CP.nchains + 1, 0);
    for (int64_t i = 0; i < n; ++i) cstart[CP.chain_of[i] + 1]++;
    for (int32_t c = 0; c < CP.nchains; ++c) cstart[c + 1] += cstart[c];
    std::vector<int32_t> rows(n);
    {
        std::vector<int64_t> nx(cstart.begin(), cstart.end() - 1);
        for (int64_t i = 0; i < n; ++i) rows[nx[CP.chain_of[i]]++] = (int32_t)i;
    }
    // drop empty chains (a tile of a ragged grid can be empty)
    std::vector<int32_t> remap(CP.nchains, -1);
    int32_t nch = 0;
    for (int32_t c = 0; c < CP.nchains; ++c)
        if (cstart[c + 1] > cstart[c]) remap[c] = nch++;
    std::vector<int64_t> step_of(n), lane_of(n);
    out.nchains = nch;
    out.chain_step.assign(nch + 1, 0);
    int64_t g = 0;
    // rows by schedule key (the wavefront level, or the packed component step), rows
    // ascending inside a key; a key with more than 32 rows spans several steps
    auto key = [&](int32_t x) -> int64_t { return CP.key.empty() ? (int64_t)F.levL[x] : CP.key[x]; };
#pragma omp parallel for schedule(dynamic, 1)
    for (int32_t c = 0; c < CP.nchains; ++c)
        std::stable_sort(rows.begin() + cstart[c], rows.begin() + cstart[c + 1],
                         [&](int32_t x, int32_t y) { return key(x) < key(y); });
    // steps of each chain (parallel over chains), their prefix, then the rows' steps/lanes
    std::vector<int64_t> csteps(CP.nchains, 0);
    auto walk = [&](int32_t c, int64_t g0, bool assign) {
        auto b = rows.begin() + cstart[c], e = rows.begin() + cstart[c + 1];
        int64_t gg = g0;
        for (auto it = b; it != e;) {
            auto jt = it;
            int lane = 0;
            while (jt != e && key(*jt) == key(*it) && lane < 32) {
                if (assign) {
                    step_of[*jt] = gg;
                    lane_of[*jt] = lane;
                }
                ++lane;
                ++jt;
            }
            ++gg;
            it = jt;
        }
        return gg - g0;
    };
#pragma omp parallel for schedule(dynamic, 1)
    for (int32_t c = 0; c < CP.nchains; ++c)
        if (remap[c] >= 0) csteps[c] = walk(c, 0, false);
    std::vector<int64_t> cfirst(CP.nchains, 0);
    for (int32_t c = 0; c < CP.nchains; ++c) {
        if (remap[c] < 0) continue;
        out.chain_step[remap[c]] = g;
        cfirst[c] = g;
        g += csteps[c];
    }
#pragma omp parallel for schedule(dynamic, 1)
    for (int32_t c = 0; c < CP.nchains; ++c)
        if (remap[c] >= 0) walk(c, cfirst[c], true);
    out.chain_step[nch] = g;
    out.nsteps = g;
    const int64_t npos = 32 * g;
    if (npos >= (1ll << 28)) {
        if (why) *why = "too many positions for the 28-bit tag payload";
        return false;
    }
    std::vector<int32_t> chain(n);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) chain[i] = remap[CP.chain_of[i]];
    out.perm.assign(npos, -1);
    out.iperm.assign(n, 0);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        const int64_t p = 32 * step_of[i] + lane_of[i];
        out.perm[p] = (int32_t)i;
        out.iperm[i] = (int32_t)p;
    }
    out.partition = CP.name;
    auto pow2 = [](int64_t w) { int64_t p = 1; while (p < w) p <<= 1; return (int32_t)p; };
    out.W_L = pow2(std::max<int64_t>(wl, 1));
    out.W_U = pow2(std::max<int64_t>(wu, 1));
    // NEXT-2: fp32 factor values (exactly representable after the setup's rounding) are
    // stored in 4 bytes when the records are narrow (the kernel's fp32 record variants)
    out.vb = (f32 && out.W_L <= 4 && out.W_U <= 4) ? 4 : 8;
    const int vrow = 128 + 32 * out.vb;   // bytes per entry column of a record: tags + values
    out.rec_L = vrow * out.W_L + 16;
    out.rec_U = vrow * out.W_U + 256 + 16;
    out.recL.resize((size_t)g * out.rec_L);         // uninitialised: zeroed below by step, in parallel
    out.recU.resize((size_t)g * out.rec_U);
#pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < g; ++s) {
        std::memset(out.recL.data() + (size_t)s * out.rec_L, 0, out.rec_L);
        std::memset(out.recU.data() + (size_t)s * out.rec_U, 0, out.rec_U);
    }
    out.chain_flags.assign(nch, 0u);

    // records: for each row, its dependencies in CSR order (the order of the definition)
    for (int upper = 0; upper < 2; ++upper) {
        const Csr& M = upper ? F.U : F.L;
        const int W = upper ? out.W_U : out.W_L;
        const int rb = upper ? out.rec_U : out.rec_L;
        fast_vector<uint8_t>& R = upper ? out.recU : out.recL;
        const size_t trailer = (size_t)vrow * W + (upper ? 256 : 0);
        int64_t n_prev = 0, n_hist = 0, n_glob = 0, n_ext = 0;
        bool bad = false;
#pragma omp parallel for schedule(dynamic, 1) reduction(+ : n_prev, n_hist, n_glob, n_ext) reduction(|| : bad)
        for (int32_t c = 0; c < nch; ++c) {
            const int64_t s0 = out.chain_step[c], s1 = out.chain_step[c + 1];
            for (int64_t s = s0; s < s1 && !bad; ++s) {
                uint32_t flags = 0;
                const size_t base = (size_t)s * rb;
                for (int l = 0; l < 32; ++l) {
                    const int32_t i = out.perm[32 * s + l];
                    if (i < 0) continue;
                    // pass step: L walks s0..s1-1, U walks s1-1..s0
                    const int64_t ps_i = upper ? (s1 - 1 - s) : (s - s0);
                    int k = 0, next = 0;
                    const int64_t q0 = upper ? M.rp[i] + 1 : M.rp[i];
                    for (int64_t q = q0; q < M.rp[i + 1]; ++q, ++k) {
                        const int32_t j = M.col[q];
                        const int64_t pj = out.iperm[j];
                        const int32_t cj = chain[j];
                        uint32_t tag;
                        if (cj == c) {
                            const int64_t sj = pj / 32;
                            const int64_t ps_j = upper ? (s1 - 1 - sj) : (sj - s0);
                            const int64_t d = ps_i - ps_j;
                            if (d < 1) { bad = true; break; }
                            if (d == 1) {
                                tag = ((uint32_t)CT_PREV << 29) | (uint32_t)(pj & 31);
                                n_prev++;
                            } else if (d < SPCG_CHAIN_HIST) {
                                tag = ((uint32_t)CT_HIST << 29) | (uint32_t)(pj & 31) | ((uint32_t)d << 5);
                                flags |= CS_SLOW;
                                __atomic_fetch_or(&out.chain_flags[c], (uint32_t)(upper ? CC_UHIST : CC_LHIST),
                                                  __ATOMIC_RELAXED);
                                n_hist++;
                            } else {
                                tag = ((uint32_t)CT_GLOB << 29) | (uint32_t)pj;
                                flags |= CS_SLOW;
                                __atomic_fetch_or(&out.chain_flags[c], (uint32_t)(upper ? CC_UGLOB : CC_LGLOB),
                                                  __ATOMIC_RELAXED);
                                n_glob++;
                            }
                        } else {
                            if (next < 2) {
                                tag = ((uint32_t)CT_EXT << 29) | ((uint32_t)next << 28) | (uint32_t)pj;
                                ++next;
                            } else {
                                tag = ((uint32_t)CT_EXTS << 29) | (uint32_t)pj;
                            }
                            flags |= CS_SLOW | CS_EXT;
                            __atomic_fetch_or(&out.chain_flags[c], (uint32_t)(upper ? CC_UEXT : CC_LEXT),
                                              __ATOMIC_RELAXED);
                            __atomic_fetch_or(&out.chain_flags[cj], (uint32_t)(upper ? CC_UPUB : CC_LPUB),
                                              __ATOMIC_RELAXED);
                            n_ext++;
                            // the producer publishes its value with a ready flag (its record's
                            // trailer: 4-byte aligned, possibly another chain's -> atomic OR)
                            const int64_t sj = pj / 32;
                            const size_t pb = (size_t)sj * rb + trailer;
                            __atomic_fetch_or((uint32_t*)(R.data() + pb), 1u << (pj & 31), __ATOMIC_RELAXED);
                        }
                        put<uint32_t>(R, base + 4 * ((size_t)W * l + k), tag);
                        if (out.vb == 4)
                            put<float>(R, base + (size_t)128 * W + 4 * ((size_t)W * l + k), (float)M.val[q]);
                        else
                            put<double>(R, base + (size_t)128 * W + 8 * ((size_t)W * l + k), M.val[q]);
                    }
                    if (upper) put<double>(R, base + (size_t)vrow * W + 8 * l, 1.0 / M.val[M.rp[i]]);
                }
                __atomic_fetch_or((uint32_t*)(R.data() + base + trailer + 4), flags, __ATOMIC_RELAXED);
            }
        }
        if (bad) {
            if (why) *why = "internal: dependency not earlier in its chain";
            return false;
        }
        out.prev_entries += n_prev;
        out.hist_entries += n_hist;
        out.glob_entries += n_glob;
        out.ext_entries += n_ext;
    }

    // SpMV: SELL-32 of the ORIGINAL A over positions, one slice per step;
    // columns are positions, entries of a row in CSR order
    // One width WA (the longest row of A) for every slice: slice s starts at entry column
    // s * WA, so a warp streams any range of slices with two bulk copies and needs no
    // offsets (stencil rows differ only at the boundary: little padding).
    SpmvLayout& S = out.A;
    S.nslices = (int32_t)g;
    int64_t WA = 1;
    for (int64_t i = 0; i < n; ++i) WA = std::max<int64_t>(WA, A.rp[i + 1] - A.rp[i]);
    out.WA = (int32_t)WA;
    S.eoff.assign(g + 1, 0);
    for (int64_t s = 0; s < g; ++s) S.eoff[s + 1] = S.eoff[s] + WA;
    S.col.resize(S.eoff[g] * 32);                    // every element is written below
    S.val.resize(S.eoff[g] * 32);
#pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < g; ++s)
        for (int l = 0; l < 32; ++l) {
            const int32_t i = out.perm[32 * s + l];
            const int64_t w = S.eoff[s + 1] - S.eoff[s];
            for (int64_t k = 0; k < w; ++k) {
                const int64_t e = (S.eoff[s] + k) * 32 + l;
                if (i >= 0 && k < A.rp[i + 1] - A.rp[i]) {
                    S.col[e] = out.iperm[A.col[A.rp[i] + k]];
                    S.val[e] = A.val[A.rp[i] + k];
                } else {
                    S.col[e] = (int32_t)(32 * s + l);     // padding: harmless self gather of a zero
                    S.val[e] = 0.0;
                }
            }
        }
    return true;
}

}  // namespace spcg

namespace spcg {

bool chain_smem_config(const ChainLayout& CL, int per_cta, ChainSmemCfg& out) {
    const size_t C = SPCG_CHAIN_C;
    const size_t step_bytes = std::max<size_t>((size_t)CL.rec_L + 4 * 256, (size_t)CL.rec_U + 2 * 256);
    const bool any_ext = CL.ext_entries > 0, any_hist = CL.hist_entries > 0;
    const size_t limit = SPCG_CHAIN_SMEM_LIMIT;
    const size_t stage = (C * step_bytes + 127) & ~(size_t)127;
    for (int NST = 16; NST >= 2; --NST) {
        size_t off = NST * stage;
        const size_t ext_off = off;
        if (any_ext) off += 2 * C * 2 * 32 * 16;
        const size_t hist_off = off;
        if (any_hist) off += (size_t)SPCG_CHAIN_HIST * 32 * 8;
        const size_t warp = (off + 127) & ~(size_t)127;
        if (warp * per_cta <= limit) {
            out.nst = NST;
            out.stage_bytes = (uint32_t)stage;
            out.warp_bytes = (uint32_t)warp;
            out.ext_off = (uint32_t)ext_off;
            out.hist_off = (uint32_t)hist_off;
            out.cta_bytes = warp * per_cta;
            // SpMV staging (the same shared memory, used between the triangular solves):
            // 8 warps x sp_nst stages of SPCG_SPMV_G slices of WA entry columns
            const size_t sp_stage = (size_t)SPCG_SPMV_G * CL.WA * 384;
            out.sp_nst = 0;
            out.sp_stage_bytes = (uint32_t)sp_stage;
            for (int sn = 3; sn >= 2; --sn)
                if (8 * sn * sp_stage <= limit) { out.sp_nst = sn; break; }
            out.cta_bytes = std::max(out.cta_bytes, 8 * (size_t)out.sp_nst * sp_stage);
            return true;
        }
    }
    return false;
}

}  // namespace spcg
