// gsetup.cu — NEXT-1: the setup of Fig. 2 on the
// GPU for ILU(0), as the paper's GPU pipeline does ("ILU(0) ... cuSPARSE", §3.3,
// P:L586-588; end-to-end comparison §4.3).  Every step runs in the
// kernels below; the host only walks Algorithm 2's branches (a few scalars per
// tried ratio) and receives the products:
//   validate        thread per row: sorted unique in-range columns, finite values,
//                   positive diagonal; exact symmetry by a binary search of the
//                   mirror (j,i) in row j (its position kept for the drop step)
//   levels          sync-free longest path (O2 / P:L263-283): a warp claims 32 rows
//                   in dependency order and loops until every lane's dependencies
//                   carry a level (warp-synchronous, so a lane waiting on a lane of
//                   its own warp never blocks it); integers, identical to the host's
//                   Kahn peeling
//   drop selection  radix SELECT of the m_t-th smallest key (bits of |a_ij|, row-
//                   major position) among the strictly-lower entries (reading A4:
//                   stable by |a|, ties row-major), eight 8-bit histogram passes, then
//                   the ties at the threshold ranked by a row scan; mirrors dropped
//                   with their entries (A3)
//   indicator       Alg. 2 lines 4-5: per-row sums in CSR order (the
//                   inf-norm, min diagonal: bit-exact), Frobenius sums per block in
//                   a fixed order (NOT the host's single row-major chain: equal up to
//                   rounding, DESIGN.md §2 reading A6g)
//   compaction      Ahat = A - S_t and the L / U split by row counts + scans
//   ILU(0) numeric  sync-free over rows (a row starts once the rows of its L pattern
//                   are final), IKJ per row in the definition's order with explicit
//                   round-to-nearest multiply / subtract / divide (no contraction):
//                   bit-exact with the host's level-parallel IKJ
// K > 0 (symbolic ILU(K) fill) stays on the host (setup.cpp).
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>

#include "internal.h"

namespace {

constexpr int GB = 256;                       // threads per block
constexpr long long G_SPIN_TIMEOUT = 8ll * 1000 * 1000 * 1000;

struct GErr {
    unsigned long long first_bad;             // (row << 4) | code, atomicMin
    int abort;
    int pad;
    unsigned long long bad_pivot;             // first zero / non-finite pivot row
    int max_level;
    int pad2;
};
enum { E_ROWPTR = 1, E_COL = 2, E_NONFINITE = 3, E_DIAG_NONPOS = 4, E_DIAG_MISSING = 5, E_PATTERN = 6,
       E_VALUE = 7 };

__device__ __forceinline__ uint64_t dbits(double v) { return (uint64_t)__double_as_longlong(v); }
__device__ __forceinline__ int ld_vol(const int* p) {
    int v;
    asm volatile("ld.volatile.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_vol(int* p, int v) {
    asm volatile("st.volatile.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_acq(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_rel(int* p, int v) {
    asm volatile("st.release.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ---------------------------------------------------------------- validation (O1)
__global__ void k_validate(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                           const double* __restrict__ val, int32_t* __restrict__ pos_t, GErr* err,
                           unsigned long long* counts /* [0] nnz(tril) incl. diag, [1] strictly lower */) {
    unsigned long long nl = 0, c = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t q0 = rp[i], q1 = rp[i + 1];
        const int64_t nnz = rp[n];
        unsigned code = 0;
        if (q1 < q0 || q0 < 0 || q1 > nnz) code = E_ROWPTR;      // never read outside col / val
        bool diag = false;
        int64_t prev = -1;
        for (int64_t q = q0; q < q1 && !code; ++q) {
            const int64_t j = col[q];
            if (j < 0 || j >= n || j <= prev) { code = E_COL; break; }
            prev = j;
            const double v = val[q];
            if (!isfinite(v)) { code = E_NONFINITE; break; }
            if (j == i) {
                diag = true;
                if (!(v > 0.0)) { code = E_DIAG_NONPOS; break; }
            }
            if (j <= i) ++nl;
            if (j < i) ++c;
        }
        if (!code && !diag) code = E_DIAG_MISSING;
        if (!code) {
            // mirror (j, i) of every entry: binary search in row j
            for (int64_t q = q0; q < q1; ++q) {
                const int64_t j = col[q];
                int64_t lo = rp[j], hi = rp[j + 1] - 1;
                if (hi < lo || lo < 0 || rp[j + 1] > nnz) { code = E_PATTERN; break; }
                int64_t found = -1;
                while (lo <= hi) {
                    const int64_t mid = (lo + hi) >> 1;
                    const int32_t cm = col[mid];
                    if (cm == i) { found = mid; break; }
                    if (cm < i) lo = mid + 1; else hi = mid - 1;
                }
                if (found < 0) { code = E_PATTERN; break; }
                if (dbits(val[found]) != dbits(val[q])) { code = E_VALUE; break; }
                pos_t[q] = (int32_t)found;
            }
        }
        if (code) atomicMin(&err->first_bad, ((unsigned long long)i << 4) | code);
    }
    // block totals (integer: order-free)
    __shared__ unsigned long long s0, s1;
    if (threadIdx.x == 0) { s0 = 0; s1 = 0; }
    __syncthreads();
    atomicAdd(&s0, nl);
    atomicAdd(&s1, c);
    __syncthreads();
    if (threadIdx.x == 0) {
        atomicAdd(counts + 0, s0);
        atomicAdd(counts + 1, s1);
    }
}

// ---------------------------------------------------------------- levels (O2)
// lev[i] = 1 + max{lev[j] : (i, j) a dependency}, max of nothing = -1 (levels from 0).
// lower: dependencies j < i, rows claimed ascending; upper: j > i, rows descending.
// drop (nullable): entries marked 1 are not part of the pattern (Ahat_t of Alg. 2
// line 9 without materialising it).  lev must be -1 on entry.
__global__ void k_levels(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                         const uint8_t* __restrict__ drop, int lower, int* lev, unsigned long long* counter,
                         GErr* err) {
    // A dependency inside the warp's own 32 rows (lane l on lane l-1: every natural-order
    // grid) is resolved through shared memory in rounds of __syncwarp, not by re-polling
    // global memory: a chain of 32 lanes costs 32 short rounds, not 32 L2 round trips.
    __shared__ int slv[GB / 32][32];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    int mymax = -1;
    for (;;) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(counter, 32ull);
        base = __shfl_sync(0xffffffffu, base, 0);
        if ((int64_t)base >= n) break;
        const int64_t t = (int64_t)base + lane;
        const int64_t i = lower ? t : n - 1 - t;
        // rows of this chunk: lower [base, base + 32), upper [n - base - 32, n - base)
        const int64_t lo = lower ? (int64_t)base : n - (int64_t)base - 32, hi = lo + 31;
        bool done = t >= n, ext_ok = done;
        int ext_max = -1, lvl = -1;
        slv[wib][lane] = -1;
        __syncwarp();
        const long long t0 = clock64();
        for (;;) {
            if (!ext_ok) {
                bool ok = true;
                int m = -1;
                for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
                    const int64_t j = col[q];
                    if ((lower ? j >= i : j <= i) || (drop && drop[q]) || (j >= lo && j <= hi)) continue;
                    const int v = ld_vol(lev + j);
                    if (v < 0) { ok = false; break; }
                    m = max(m, v);
                }
                if (ok) { ext_ok = true; ext_max = m; }
            }
            // internal rounds: a lane whose external part is known finishes once its
            // dependencies inside the chunk have (they are earlier lanes)
            for (int r = 0; r < 32; ++r) {
                bool progressed = false;
                if (ext_ok && !done) {
                    int m = ext_max;
                    bool ok = true;
                    for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
                        const int64_t j = col[q];
                        if ((lower ? j >= i : j <= i) || (drop && drop[q]) || j < lo || j > hi) continue;
                        const int v = *(volatile int*)&slv[wib][lower ? (int)(j - lo) : (int)(hi - j)];
                        if (v < 0) { ok = false; break; }
                        m = max(m, v);
                    }
                    if (ok) {
                        lvl = m + 1;
                        slv[wib][lane] = lvl;
                        st_vol(lev + i, lvl);
                        mymax = max(mymax, lvl);
                        done = true;
                        progressed = true;
                    }
                }
                __syncwarp();
                if (!__any_sync(0xffffffffu, progressed)) break;
            }
            if (__all_sync(0xffffffffu, done)) break;
            if (__any_sync(0xffffffffu, clock64() - t0 > G_SPIN_TIMEOUT || ld_vol(&err->abort) != 0)) {
                if (lane == 0) atomicExch(&err->abort, 1);
                return;
            }
        }
        __syncwarp();
    }
    for (int o = 16; o; o >>= 1) mymax = max(mymax, __shfl_xor_sync(0xffffffffu, mymax, o));
    if (lane == 0) atomicMax(&err->max_level, mymax);
}

// ---------------------------------------------------------------- drop selection (O3)
// key of a strictly-lower entry: IEEE bits of |a| (non-negative doubles order as their
// bits).  Pass: histogram of digit (key >> shift) & 255 over the candidates whose
// higher digits equal prefix.
__global__ void k_hist(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                       const double* __restrict__ val, int shift, uint64_t prefix, uint64_t pmask,
                       unsigned long long* hist) {
    __shared__ unsigned sh[256];
    for (int d = threadIdx.x; d < 256; d += blockDim.x) sh[d] = 0;
    __syncthreads();
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
            if (col[q] >= i) break;
            const uint64_t k = dbits(fabs(val[q]));
            if ((k & pmask) == prefix) atomicAdd(&sh[(k >> shift) & 255], 1u);
        }
    __syncthreads();
    for (int d = threadIdx.x; d < 256; d += blockDim.x)
        if (sh[d]) atomicAdd(hist + d, (unsigned long long)sh[d]);
}

// per-row count of candidates with key == T (for the rank of ties)
__global__ void k_count_eq(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                           const double* __restrict__ val, uint64_t T, int64_t* __restrict__ cnt) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = 0;
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
            if (col[q] >= i) break;
            c += dbits(fabs(val[q])) == T;
        }
        cnt[i] = c;
    }
}

// drop: key < T, or key == T with row-major rank < need; mirrors too
__global__ void k_mark(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                       const double* __restrict__ val, const int32_t* __restrict__ pos_t, uint64_t T, int64_t need,
                       const int64_t* __restrict__ eq_off, uint8_t* drop) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = eq_off ? eq_off[i] : 0;
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
            if (col[q] >= i) break;
            const uint64_t k = dbits(fabs(val[q]));
            bool d = k < T;
            if (k == T) d = (r++) < need;
            if (d) {
                drop[q] = 1;
                drop[pos_t[q]] = 1;
            }
        }
    }
}

// ---------------------------------------------------------------- indicator (O4)
struct IndPart {
    double fro_h, fro_s, inf_h, inf_s, mind;
};
__global__ void k_indicator(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                            const double* __restrict__ val, const uint8_t* __restrict__ drop, IndPart* part) {
    double fh = 0.0, fs = 0.0, ih = 0.0, is = 0.0, md = INFINITY;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double rh = 0.0, rs = 0.0, fh_r = 0.0, fs_r = 0.0;
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
            const double v = val[q];
            if (drop[q]) {
                fs_r = __dadd_rn(fs_r, __dmul_rn(v, v));
                rs = __dadd_rn(rs, fabs(v));
            } else {
                fh_r = __dadd_rn(fh_r, __dmul_rn(v, v));
                rh = __dadd_rn(rh, fabs(v));
                if (col[q] == i && v < md) md = v;
            }
        }
        fh = __dadd_rn(fh, fh_r);
        fs = __dadd_rn(fs, fs_r);
        ih = fmax(ih, rh);
        is = fmax(is, rs);
    }
    // block reduction in a fixed order (tree over threads), then one partial per block
    __shared__ double s[5][GB];
    s[0][threadIdx.x] = fh;
    s[1][threadIdx.x] = fs;
    s[2][threadIdx.x] = ih;
    s[3][threadIdx.x] = is;
    s[4][threadIdx.x] = md;
    __syncthreads();
    for (int o = blockDim.x / 2; o; o >>= 1) {
        if (threadIdx.x < o) {
            s[0][threadIdx.x] = __dadd_rn(s[0][threadIdx.x], s[0][threadIdx.x + o]);
            s[1][threadIdx.x] = __dadd_rn(s[1][threadIdx.x], s[1][threadIdx.x + o]);
            s[2][threadIdx.x] = fmax(s[2][threadIdx.x], s[2][threadIdx.x + o]);
            s[3][threadIdx.x] = fmax(s[3][threadIdx.x], s[3][threadIdx.x + o]);
            s[4][threadIdx.x] = fmin(s[4][threadIdx.x], s[4][threadIdx.x + o]);
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) part[blockIdx.x] = IndPart{s[0][0], s[1][0], s[2][0], s[3][0], s[4][0]};
}

// ---------------------------------------------------------------- scans and compaction
// per-row counts: mode 0 kept entries (drop may be null), 1 strictly lower, 2 upper incl. diagonal
__global__ void k_rowcount(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                           const uint8_t* __restrict__ drop, int mode, int64_t* __restrict__ cnt) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = 0;
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
            if (mode == 0) c += drop ? !drop[q] : 1;
            else if (mode == 1) c += col[q] < i;
            else c += col[q] >= i;
        }
        cnt[i] = c;
    }
}

// exclusive scan of int64 counts, three phases: block sums, scan of the block sums
// (one block, sequential per thread chunk), add back.  out[n] = total.
constexpr int SCAN_CHUNK = 4096;        // elements per block in phases 1 and 3
__global__ void k_scan_blocksum(int64_t n, const int64_t* __restrict__ in, int64_t* __restrict__ bsum) {
    const int64_t b0 = (int64_t)blockIdx.x * SCAN_CHUNK;
    int64_t s = 0;
    for (int64_t i = b0 + threadIdx.x; i < (n < b0 + SCAN_CHUNK ? n : b0 + SCAN_CHUNK); i += blockDim.x) s += in[i];
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    __shared__ int64_t w[GB / 32];
    if ((threadIdx.x & 31) == 0) w[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t t = 0;
        for (int k = 0; k < (int)(blockDim.x / 32); ++k) t += w[k];
        bsum[blockIdx.x] = t;
    }
}
__global__ void k_scan_top(int64_t nb, int64_t* bsum) {     // one thread: nb is n / 4096
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        int64_t run = 0;
        for (int64_t b = 0; b < nb; ++b) {
            const int64_t v = bsum[b];
            bsum[b] = run;
            run += v;
        }
        bsum[nb] = run;
    }
}
__global__ void k_scan_add(int64_t n, const int64_t* __restrict__ in, const int64_t* __restrict__ bsum,
                           int64_t* __restrict__ out) {
    // block-local exclusive scan of SCAN_CHUNK elements: each thread a contiguous run
    constexpr int PER = SCAN_CHUNK / GB;
    const int64_t b0 = (int64_t)blockIdx.x * SCAN_CHUNK;
    const int64_t s0 = b0 + (int64_t)threadIdx.x * PER;
    int64_t loc[PER];
    int64_t t = 0;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
        loc[k] = (s0 + k < n) ? in[s0 + k] : 0;
        t += loc[k];
    }
    // exclusive scan of the per-thread totals across the block
    __shared__ int64_t sh[GB];
    sh[threadIdx.x] = t;
    __syncthreads();
    for (int o = 1; o < GB; o <<= 1) {
        const int64_t v = threadIdx.x >= o ? sh[threadIdx.x - o] : 0;
        __syncthreads();
        sh[threadIdx.x] += v;
        __syncthreads();
    }
    int64_t run = bsum[blockIdx.x] + sh[threadIdx.x] - t;
#pragma unroll
    for (int k = 0; k < PER; ++k)
        if (s0 + k < n) {
            out[s0 + k] = run;
            run += loc[k];
        }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) out[n] = bsum[gridDim.x];
}

// copy the entries a row keeps (mode 0: not dropped; 1: strictly lower; 2: upper incl. diagonal)
__global__ void k_compact(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                          const double* __restrict__ val, const uint8_t* __restrict__ drop, int mode,
                          const int64_t* __restrict__ orp, int32_t* __restrict__ ocol, double* __restrict__ oval) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t o = orp[i];
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
            const bool keep = mode == 0 ? (drop ? !drop[q] : true) : (mode == 1 ? col[q] < i : col[q] >= i);
            if (keep) {
                ocol[o] = col[q];
                oval[o] = val[q];
                ++o;
            }
        }
    }
}

// ---------------------------------------------------------------- ILU(0) numeric (O7)
// In place on L / U initialised with Ahat's values.  Row i: for k in L(i) ascending,
// l_ik = a_ik / u_kk, then a_ij -= l_ik u_kj for j in U(k) \ {k} that lie in row i's
// pattern (merge walk: all three lists are sorted).  done[i] = 1 (release) once row i
// is final; a row starts when done[k] (acquire) for every k in L(i).
// Rows are taken in LEVEL order (order[]: the rows of level 0, then level 1, ...), so the
// 32 rows of a warp are independent or depend only on earlier levels: the dependency
// chain the rows wait on is the wavefront count of L (4110 on C4), not the natural order
// (where a warp's rows form one chain and each chunk waits for its left neighbour).
__global__ void k_ilu0(int64_t n, const int64_t* __restrict__ lrp, const int32_t* __restrict__ lcol,
                       double* lval, const int64_t* __restrict__ urp, const int32_t* __restrict__ ucol, double* uval,
                       const int32_t* __restrict__ order, int* done, unsigned long long* counter, GErr* err) {
    const int lane = threadIdx.x & 31;
    for (;;) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(counter, 32ull);
        base = __shfl_sync(0xffffffffu, base, 0);
        if ((int64_t)base >= n) break;
        const int64_t t = (int64_t)base + lane;
        const int64_t i = t < n ? (int64_t)order[t] : -1;
        bool fin = t >= n;
        const long long t0 = clock64();
        for (;;) {
            if (!fin) {
                bool ok = true;
                for (int64_t q = lrp[i]; q < lrp[i + 1]; ++q)
                    if (ld_acq(done + lcol[q]) == 0) { ok = false; break; }
                if (ok) {
                    const int64_t l0 = lrp[i], l1 = lrp[i + 1], u0i = urp[i], u1i = urp[i + 1];
                    for (int64_t q = l0; q < l1; ++q) {
                        const int64_t k = lcol[q];
                        const int64_t uk0 = urp[k], uk1 = urp[k + 1];
                        const double lik = __ddiv_rn(lval[q], __ldcg(uval + uk0));
                        lval[q] = lik;
                        int64_t pl = q + 1, pu = u0i;
                        for (int64_t rr = uk0 + 1; rr < uk1; ++rr) {
                            const int32_t j = __ldcg(ucol + rr);
                            const double ukj = __ldcg(uval + rr);
                            if (j < i) {
                                while (pl < l1 && lcol[pl] < j) ++pl;
                                if (pl < l1 && lcol[pl] == j) lval[pl] = __dsub_rn(lval[pl], __dmul_rn(lik, ukj));
                            } else {
                                while (pu < u1i && ucol[pu] < j) ++pu;
                                if (pu < u1i && ucol[pu] == j) uval[pu] = __dsub_rn(uval[pu], __dmul_rn(lik, ukj));
                            }
                        }
                    }
                    const double d = uval[u0i];
                    if (d == 0.0 || !isfinite(d)) atomicMin(&err->bad_pivot, (unsigned long long)i);
                    st_rel(done + i, 1);
                    fin = true;
                }
            }
            if (__all_sync(0xffffffffu, fin)) break;
            if (__any_sync(0xffffffffu, clock64() - t0 > G_SPIN_TIMEOUT || ld_vol(&err->abort) != 0)) {
                if (lane == 0) atomicExch(&err->abort, 1);
                return;
            }
        }
    }
}

// level-order permutation: count rows per level, scan, scatter (the order inside a level
// does not matter: its rows are independent)
__global__ void k_level_count(int64_t n, const int* __restrict__ lev, int64_t* cnt) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        atomicAdd((unsigned long long*)(cnt + lev[i]), 1ull);
}
__global__ void k_level_scatter(int64_t n, const int* __restrict__ lev, int64_t* cursor, int32_t* order) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        order[atomicAdd((unsigned long long*)(cursor + lev[i]), 1ull)] = (int32_t)i;
}

// ---------------------------------------------------------------- host-side compaction
// Ahat = the entries of A the mask keeps (row-major, CSR order: what k_compact wrote),
// L_s = its strictly-lower part, U = the rest (K = 0: no fill).  Rows in parallel.
void host_split(const spcg::Csr& A, const uint8_t* drop, spcg::Csr& H, spcg::Csr& L, spcg::Csr& U) {
    const int64_t n = A.n;
    H.n = L.n = U.n = n;
    H.rp.assign(n + 1, 0);
    L.rp.assign(n + 1, 0);
    U.rp.assign(n + 1, 0);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        int64_t h = 0, l = 0, u = 0;
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q) {
            if (drop && drop[q]) continue;
            ++h;
            if (A.col[q] < i) ++l; else ++u;
        }
        H.rp[i + 1] = h;
        L.rp[i + 1] = l;
        U.rp[i + 1] = u;
    }
    for (int64_t i = 0; i < n; ++i) {
        H.rp[i + 1] += H.rp[i];
        L.rp[i + 1] += L.rp[i];
        U.rp[i + 1] += U.rp[i];
    }
    H.col.resize(H.rp[n]);
    H.val.resize(H.rp[n]);
    L.col.resize(L.rp[n]);
    L.val.resize(L.rp[n]);
    U.col.resize(U.rp[n]);
    U.val.resize(U.rp[n]);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        int64_t h = H.rp[i], l = L.rp[i], u = U.rp[i];
        for (int64_t q = A.rp[i]; q < A.rp[i + 1]; ++q) {
            if (drop && drop[q]) continue;
            H.col[h] = A.col[q];
            H.val[h++] = A.val[q];
            if (A.col[q] < i) L.col[l++] = A.col[q];
            else U.col[u++] = A.col[q];
        }
    }
}

// ---------------------------------------------------------------- host driver
struct Pool {                 // device buffers of the setup, freed together
    DevAllocator alc;
    cudaStream_t s = nullptr;
    std::vector<std::pair<void*, size_t>> bufs;
    bool failed = false;
    template <class T>
    T* get(size_t count) {
        const size_t bytes = std::max<size_t>(count * sizeof(T), 16);
        void* p = nullptr;
        if (alc.alloc) p = alc.alloc(bytes, (void*)s, alc.ctx);
        else if (cudaMalloc(&p, bytes) != cudaSuccess) p = nullptr;
        if (!p) failed = true;
        else bufs.push_back({p, bytes});
        return (T*)p;
    }
    void release() {
        cudaStreamSynchronize(s);
        for (auto& b : bufs) {
            if (alc.free) alc.free(b.first, b.second, (void*)s, alc.ctx);
            else cudaFree(b.first);
        }
        bufs.clear();
    }
    ~Pool() { release(); }
};

#define GCK(x)                                                                         \
    do {                                                                               \
        cudaError_t e_ = (x);                                                          \
        if (e_ != cudaSuccess) {                                                       \
            spcg::set_error(std::string("gpu setup: ") + cudaGetErrorString(e_));     \
            return SPCG_ERR_CUDA;                                                      \
        }                                                                              \
    } while (0)

struct GCsr {                 // device CSR
    int64_t n = 0, nnz = 0;
    int64_t* rp = nullptr;
    int32_t* col = nullptr;
    double* val = nullptr;
};

struct Ctx {
    Pool pool;
    cudaStream_t s;
    int grid = 0;             // blocks for the row-parallel kernels
    int coop_grid = 0;        // co-resident blocks for the sync-free kernels
    GErr* err = nullptr;
    unsigned long long* cnt = nullptr;   // scratch counters [4]
    int64_t* tmp = nullptr;   // [n] counts
    int64_t* bsum = nullptr;  // scan block sums
};

spcg_status_t check_err(Ctx& C, GErr& h) {
    GCK(cudaMemcpyAsync(&h, C.err, sizeof(GErr), cudaMemcpyDeviceToHost, C.s));
    GCK(cudaStreamSynchronize(C.s));
    if (h.abort) {
        spcg::set_error("gpu setup: a sync-free kernel timed out (internal)");
        return SPCG_ERR_INTERNAL;
    }
    return SPCG_OK;
}

// exclusive scan of C.tmp[0..n) into out[0..n]
spcg_status_t scan(Ctx& C, int64_t n, int64_t* out) {
    const int64_t nb = (n + SCAN_CHUNK - 1) / SCAN_CHUNK;
    k_scan_blocksum<<<(unsigned)nb, GB, 0, C.s>>>(n, C.tmp, C.bsum);
    k_scan_top<<<1, 32, 0, C.s>>>(nb, C.bsum);
    k_scan_add<<<(unsigned)nb, GB, 0, C.s>>>(n, C.tmp, C.bsum, out);
    GCK(cudaGetLastError());
    return SPCG_OK;
}

// levels of M (lower / upper), optional drop mask; lev_out (device, n) or nullptr; returns w
spcg_status_t levels(Ctx& C, const GCsr& M, const uint8_t* drop, bool lower, int* lev, int64_t* w) {
    GCK(cudaMemsetAsync(lev, 0xff, sizeof(int) * M.n, C.s));
    GCK(cudaMemsetAsync(C.cnt, 0, 8, C.s));
    GCK(cudaMemsetAsync(&C.err->max_level, 0xff, 4, C.s));
    int64_t n = M.n;
    int lw = lower ? 1 : 0;
    void* args[] = {&n, (void*)&M.rp, (void*)&M.col, (void*)&drop, &lw, &lev, &C.cnt, &C.err};
    GCK(cudaLaunchCooperativeKernel((void*)k_levels, dim3(C.coop_grid), dim3(GB), args, 0, C.s));
    GErr h;
    spcg_status_t st = check_err(C, h);
    if (st != SPCG_OK) return st;
    *w = (int64_t)h.max_level + 1;
    return SPCG_OK;
}

// Host <-> device copies of pageable std::vector data through two pinned bounce
// buffers (a pageable cudaMemcpy runs at a few GB/s; this overlaps the host memcpy of
// one chunk with the DMA of the other).
constexpr size_t BOUNCE_MAX = 32u << 20;
struct Bounce {
    void* buf[2] = {nullptr, nullptr};
    cudaEvent_t ev[2] = {nullptr, nullptr};
    bool ok = false;
    size_t size = 0;            // bytes per buffer: the largest copy, at most BOUNCE_MAX
    explicit Bounce(size_t largest) {
        size = std::max<size_t>(4096, std::min(BOUNCE_MAX, largest));
        ok = cudaMallocHost(&buf[0], size) == cudaSuccess && cudaMallocHost(&buf[1], size) == cudaSuccess &&
             cudaEventCreateWithFlags(&ev[0], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&ev[1], cudaEventDisableTiming) == cudaSuccess;
    }
    ~Bounce() {
        for (int k = 0; k < 2; ++k) {
            if (ev[k]) cudaEventDestroy(ev[k]);
            if (buf[k]) cudaFreeHost(buf[k]);
        }
    }
};
spcg_status_t h2d(Ctx& C, Bounce& B, void* dst, const void* src, size_t bytes) {
    if (!B.ok) {
        GCK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, C.s));
        return SPCG_OK;
    }
    size_t off = 0;
    for (int k = 0; off < bytes; k ^= 1) {
        const size_t m = std::min(B.size, bytes - off);
        GCK(cudaEventSynchronize(B.ev[k]));                  // the DMA out of this buffer is done
        {
            char* bd = (char*)B.buf[k];
            const char* sp = (const char*)src + off;
            const int64_t nb = (int64_t)((m + (1u << 20) - 1) >> 20);
#pragma omp parallel for schedule(static)
            for (int64_t b = 0; b < nb; ++b) {
                const size_t o = (size_t)b << 20;
                std::memcpy(bd + o, sp + o, std::min<size_t>(1u << 20, m - o));
            }
        }
        GCK(cudaMemcpyAsync((char*)dst + off, B.buf[k], m, cudaMemcpyHostToDevice, C.s));
        GCK(cudaEventRecord(B.ev[k], C.s));
        off += m;
    }
    return SPCG_OK;
}
spcg_status_t d2h(Ctx& C, Bounce& B, void* dst, const void* src, size_t bytes) {
    if (!B.ok) {
        GCK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, C.s));
        GCK(cudaStreamSynchronize(C.s));
        return SPCG_OK;
    }
    // chunk j lands in buffer j & 1; it is drained while chunk j + 1 is in flight
    const size_t nch = (bytes + B.size - 1) / B.size;
    for (size_t j = 0; j < nch + 1; ++j) {
        if (j < nch) {
            const size_t off = j * B.size, m = std::min(B.size, bytes - off);
            GCK(cudaMemcpyAsync(B.buf[j & 1], (const char*)src + off, m, cudaMemcpyDeviceToHost, C.s));
            GCK(cudaEventRecord(B.ev[j & 1], C.s));
        }
        if (j > 0) {
            const size_t i = j - 1, off = i * B.size, m = std::min(B.size, bytes - off);
            GCK(cudaEventSynchronize(B.ev[i & 1]));
            char* dd = (char*)dst + off;
            const char* ss = (const char*)B.buf[i & 1];
            const int64_t nb = (int64_t)((m + (1u << 20) - 1) >> 20);
#pragma omp parallel for schedule(static)
            for (int64_t k = 0; k < nb; ++k) {
                const size_t o = (size_t)k << 20;
                std::memcpy(dd + o, ss + o, std::min<size_t>(1u << 20, m - o));
            }
        }
    }
    return SPCG_OK;
}


// compaction of A by a row predicate into a new device CSR
spcg_status_t compact(Ctx& C, const GCsr& A, const uint8_t* drop, int mode, GCsr& out) {
    out.n = A.n;
    k_rowcount<<<C.grid, GB, 0, C.s>>>(A.n, A.rp, A.col, drop, mode, C.tmp);
    out.rp = C.pool.get<int64_t>(A.n + 1);
    if (C.pool.failed) return SPCG_ERR_OOM;
    spcg_status_t st = scan(C, A.n, out.rp);
    if (st != SPCG_OK) return st;
    GCK(cudaMemcpyAsync(&out.nnz, out.rp + A.n, 8, cudaMemcpyDeviceToHost, C.s));
    GCK(cudaStreamSynchronize(C.s));
    out.col = C.pool.get<int32_t>(out.nnz);
    out.val = C.pool.get<double>(out.nnz);
    if (C.pool.failed) return SPCG_ERR_OOM;
    k_compact<<<C.grid, GB, 0, C.s>>>(A.n, A.rp, A.col, A.val, drop, mode, out.rp, out.col, out.val);
    GCK(cudaGetLastError());
    return SPCG_OK;
}

// the m smallest strictly-lower entries by (|a| bits, row-major position) and their
// mirrors -> drop (zeroed here)
spcg_status_t select_drop(Ctx& C, const GCsr& A, const int32_t* pos_t, int64_t m, uint8_t* drop) {
    GCK(cudaMemsetAsync(drop, 0, A.nnz, C.s));
    if (m <= 0) return SPCG_OK;
    uint64_t prefix = 0, pmask = 0;
    int64_t need = m;
    unsigned long long* hist = (unsigned long long*)C.bsum;   // 256 counters (bsum is larger)
    for (int shift = 56; shift >= 0; shift -= 8) {
        GCK(cudaMemsetAsync(hist, 0, 256 * 8, C.s));
        k_hist<<<C.grid, GB, 0, C.s>>>(A.n, A.rp, A.col, A.val, shift, prefix, pmask, hist);
        unsigned long long h[256];
        GCK(cudaMemcpyAsync(h, hist, sizeof h, cudaMemcpyDeviceToHost, C.s));
        GCK(cudaStreamSynchronize(C.s));
        int d = 0;
        for (; d < 256; ++d) {
            if ((int64_t)h[d] >= need) break;
            need -= (int64_t)h[d];
        }
        if (d == 256) {
            spcg::set_error("gpu setup: radix select out of range (internal)");
            return SPCG_ERR_INTERNAL;
        }
        prefix |= (uint64_t)d << shift;
        pmask |= (uint64_t)255 << shift;
    }
    // prefix = T, the key of the m-th smallest; need = how many entries with key T to take
    k_count_eq<<<C.grid, GB, 0, C.s>>>(A.n, A.rp, A.col, A.val, prefix, C.tmp);
    int64_t* eq_off = C.pool.get<int64_t>(A.n + 1);
    if (C.pool.failed) return SPCG_ERR_OOM;
    spcg_status_t st = scan(C, A.n, eq_off);
    if (st != SPCG_OK) return st;
    k_mark<<<C.grid, GB, 0, C.s>>>(A.n, A.rp, A.col, A.val, pos_t, prefix, need, eq_off, drop);
    GCK(cudaGetLastError());
    return SPCG_OK;
}

spcg_status_t indicator(Ctx& C, const GCsr& A, const uint8_t* drop, int norm_reading, double* ind) {
    IndPart* part = (IndPart*)C.bsum;       // C.grid partials (bsum holds >= grid * 5 doubles)
    k_indicator<<<C.grid, GB, 0, C.s>>>(A.n, A.rp, A.col, A.val, drop, part);
    std::vector<IndPart> h(C.grid);
    GCK(cudaMemcpyAsync(h.data(), part, sizeof(IndPart) * C.grid, cudaMemcpyDeviceToHost, C.s));
    GCK(cudaStreamSynchronize(C.s));
    double fh = 0.0, fs = 0.0, ih = 0.0, is = 0.0, md = INFINITY;
    for (const IndPart& p : h) {              // blocks in order
        fh += p.fro_h;
        fs += p.fro_s;
        ih = std::max(ih, p.inf_h);
        is = std::max(is, p.inf_s);
        md = std::min(md, p.mind);
    }
    const double kappa = ih / md;
    const double a2 = norm_reading == SPCG_NORM_INF ? ih : std::sqrt(fh);
    const double sn = norm_reading == SPCG_NORM_INF ? is : std::sqrt(fs);
    *ind = (kappa / a2) * sn;
    return SPCG_OK;
}

}  // namespace

namespace spcg {

spcg_status_t gpu_setup_k0(const Csr& Ain, const spcg_drop_params_t& p, int device, void* stream,
                           const ::DevAllocator& alc, SparsifyResult& sp, Factors& F, double* phase_ms) {
    const int64_t n = Ain.n;
    const int64_t nnz = Ain.nnz();
    if (n <= 0 || (int64_t)Ain.rp.size() != n + 1 || Ain.rp[0] != 0) {
        set_error("bad row_ptr");
        return SPCG_ERR_BAD_MATRIX;
    }
    if (nnz >= (int64_t(1) << 31)) {
        set_error("nnz >= 2^31");
        return SPCG_ERR_BAD_MATRIX;
    }
    GCK(cudaSetDevice(device));
    Ctx C;
    C.s = (cudaStream_t)stream;
    C.pool.s = C.s;
    C.pool.alc = alc;
    int sms = 0, per_sm = 0;
    GCK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    GCK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_levels, GB, 0));
    int per_sm2 = 0;
    GCK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm2, k_ilu0, GB, 0));
    C.coop_grid = sms * std::max(1, std::min(per_sm, per_sm2));
    C.grid = std::max<int>(1, (int)std::min<int64_t>((n + GB - 1) / GB, (int64_t)sms * 8));
    double t0 = now_ms();

    GCsr A;
    A.n = n;
    A.nnz = nnz;
    A.rp = C.pool.get<int64_t>(n + 1);
    A.col = C.pool.get<int32_t>(nnz);
    A.val = C.pool.get<double>(nnz);
    int32_t* pos_t = C.pool.get<int32_t>(nnz);
    uint8_t* drop = C.pool.get<uint8_t>(nnz);
    C.err = C.pool.get<GErr>(1);
    C.cnt = C.pool.get<unsigned long long>(4);
    C.tmp = C.pool.get<int64_t>(n + 1);
    const int64_t nb = (n + SCAN_CHUNK - 1) / SCAN_CHUNK;
    C.bsum = C.pool.get<int64_t>(std::max<int64_t>(nb + 1, std::max<int64_t>(512, 5 * (int64_t)C.grid)));
    int* lev = C.pool.get<int>(n);
    if (C.pool.failed) {
        set_error("gpu setup: device allocation failed");
        return SPCG_ERR_OOM;
    }
    Bounce B((size_t)8 * std::max<int64_t>(nnz, n + 1));
    spcg_status_t st;
    if ((st = h2d(C, B, A.rp, Ain.rp.data(), 8 * (n + 1))) != SPCG_OK) return st;
    if ((st = h2d(C, B, A.col, Ain.col.data(), 4 * nnz)) != SPCG_OK) return st;
    if ((st = h2d(C, B, A.val, Ain.val.data(), 8 * nnz)) != SPCG_OK) return st;
    {
        GErr e0{};
        e0.first_bad = ~0ull;
        e0.bad_pivot = ~0ull;
        e0.max_level = -1;
        GCK(cudaMemcpyAsync(C.err, &e0, sizeof e0, cudaMemcpyHostToDevice, C.s));
    }
    // ---- O1
    GCK(cudaMemsetAsync(C.cnt, 0, 32, C.s));
    k_validate<<<C.grid, GB, 0, C.s>>>(n, A.rp, A.col, A.val, pos_t, C.err, C.cnt);
    GCK(cudaGetLastError());
    unsigned long long counts[2];
    GCK(cudaMemcpyAsync(counts, C.cnt, 16, cudaMemcpyDeviceToHost, C.s));
    GErr he;
    st = check_err(C, he);
    if (st != SPCG_OK) return st;
    if (he.first_bad != ~0ull) {
        const int64_t row = (int64_t)(he.first_bad >> 4);
        static const char* what[] = {"", "row_ptr not monotone", "columns out of range, unsorted or duplicated",
                                     "non-finite value", "non-positive diagonal", "missing diagonal",
                                     "pattern not symmetric", "matrix not exactly symmetric"};
        set_error(std::string(what[he.first_bad & 15]) + " at row " + std::to_string(row));
        return SPCG_ERR_BAD_MATRIX;
    }
    const int64_t NL = (int64_t)counts[0], Ccand = (int64_t)counts[1];
    double t1 = now_ms();

    // ---- Algorithm 2: w_A, then the ratios
    st = levels(C, A, nullptr, true, lev, &sp.w_A);
    if (st != SPCG_OK) return st;
    auto count = [&](double t) {
        int64_t m = (int64_t)std::floor(t * (double)NL / 100.0);   // A2
        return std::max<int64_t>(0, std::min(m, Ccand));
    };
    double chosen_pct = 0.0;
    int64_t chosen_m = 0;
    bool have_drop = false;                   // drop holds the chosen ratio's mask
    if (p.mode == SPCG_DROP_NONE) {
        sp.w_Ahat = sp.w_A;
    } else if (p.mode == SPCG_DROP_FIXED) {
        chosen_pct = p.fixed_pct;
        chosen_m = count(p.fixed_pct);
        if ((st = select_drop(C, A, pos_t, chosen_m, drop)) != SPCG_OK) return st;
        have_drop = true;
        if ((st = levels(C, A, drop, true, lev, &sp.w_Ahat)) != SPCG_OK) return st;
    } else {
        if (p.n_ratios < 1 || p.n_ratios > 8) {
            set_error("n_ratios must be 1..8");
            return SPCG_ERR_INVALID_ARG;
        }
        const int nr = p.n_ratios;
        int chosen = -1;
        bool accepted = false;
        for (int r = 0; r < nr && chosen < 0; ++r) {
            const double t = p.ratios_pct[r];
            const int64_t m = count(t);
            if ((st = select_drop(C, A, pos_t, m, drop)) != SPCG_OK) return st;
            double ind;
            if ((st = indicator(C, A, drop, p.norm_reading, &ind)) != SPCG_OK) return st;
            sp.tried_pct[r] = t;
            sp.indicator[r] = ind;
            sp.tried_w[r] = -1;
            sp.reduction[r] = -1.0;
            sp.n_tried = r + 1;
            const bool last = r == nr - 1;
            if (ind > p.tau) {                       // line 5
                if (last) { chosen = 0; break; }     // line 6
                continue;                            // line 7
            }
            int64_t wt;
            if ((st = levels(C, A, drop, true, lev, &wt)) != SPCG_OK) return st;   // line 9
            const double den = p.reduction_denominator == SPCG_DENOM_WAHAT ? (double)wt : (double)sp.w_A;
            const double red = 100.0 * (double)(sp.w_A - wt) / den;               // Eq. 7 / line 10
            sp.tried_w[r] = wt;
            sp.reduction[r] = red;
            if (red >= p.omega_pct || last) {        // lines 10-11
                chosen = r;
                accepted = true;
                chosen_pct = t;
                chosen_m = m;
                sp.w_Ahat = wt;
                have_drop = true;
            }
        }
        if (!accepted) {                             // line 14: A - S_first
            chosen_pct = p.ratios_pct[0];
            chosen_m = count(chosen_pct);
            if ((st = select_drop(C, A, pos_t, chosen_m, drop)) != SPCG_OK) return st;
            have_drop = true;
            if ((st = levels(C, A, drop, true, lev, &sp.w_Ahat)) != SPCG_OK) return st;
        }
    }
    sp.chosen_pct = chosen_pct;
    sp.m_t = chosen_m;
    GCsr H;
    if ((st = compact(C, A, have_drop ? drop : nullptr, 0, H)) != SPCG_OK) return st;
    double t2 = now_ms();

    // ---- ILU(0): pattern of Ahat split into L_s and U (K = 0: no fill)
    GCsr Ld, Ud;
    if ((st = compact(C, H, nullptr, 1, Ld)) != SPCG_OK) return st;
    if ((st = compact(C, H, nullptr, 2, Ud)) != SPCG_OK) return st;
    double t3 = now_ms();
    // levels of the factors (O8); L's give the row order of the numeric factorisation
    F.levL.resize(n);
    F.levU.resize(n);
    // K = 0: the pattern of L_s is the strictly-lower part of Ahat, so L's levels are the
    // ones Algorithm 2 just computed for the chosen Ahat (still in lev): no second pass
    F.wL = sp.w_Ahat;
    {
        int32_t* order = C.pool.get<int32_t>(n);
        int* done = C.pool.get<int>(n);
        int64_t* lcnt = C.pool.get<int64_t>(F.wL + 1);
        if (C.pool.failed) return SPCG_ERR_OOM;
        GCK(cudaMemsetAsync(C.tmp, 0, sizeof(int64_t) * F.wL, C.s));
        k_level_count<<<C.grid, GB, 0, C.s>>>(n, lev, C.tmp);
        if ((st = scan(C, F.wL, lcnt)) != SPCG_OK) return st;
        k_level_scatter<<<C.grid, GB, 0, C.s>>>(n, lev, lcnt, order);
        GCK(cudaGetLastError());
        GCK(cudaMemsetAsync(done, 0, sizeof(int) * n, C.s));
        GCK(cudaMemsetAsync(C.cnt, 0, 8, C.s));
        int64_t nn = n;
        void* args[] = {&nn, &Ld.rp, &Ld.col, &Ld.val, &Ud.rp, &Ud.col, &Ud.val, &order, &done, &C.cnt, &C.err};
        GCK(cudaLaunchCooperativeKernel((void*)k_ilu0, dim3(C.coop_grid), dim3(GB), args, 0, C.s));
        if ((st = check_err(C, he)) != SPCG_OK) return st;
    }
    if ((st = d2h(C, B, F.levL.data(), lev, 4 * n)) != SPCG_OK) return st;
    if ((st = levels(C, Ud, nullptr, false, lev, &F.wU)) != SPCG_OK) return st;
    if ((st = d2h(C, B, F.levU.data(), lev, 4 * n)) != SPCG_OK) return st;
    double t4 = now_ms();
    // The host needs Ahat and the L / U patterns for the layout inspector: they follow from
    // A and the drop mask by the same row-major compaction the kernels did (so they are
    // identical), so only the mask and the factor VALUES cross the bus (C4: 84 MB + 0.63
    // GB instead of 1.9 GB of CSR arrays).
    {
        std::vector<uint8_t> dm;
        if (have_drop) {
            dm.resize(nnz);
            if ((st = d2h(C, B, dm.data(), drop, nnz)) != SPCG_OK) return st;
        }
        host_split(Ain, have_drop ? dm.data() : nullptr, sp.Ahat, F.L, F.U);
        if ((int64_t)F.L.col.size() != Ld.nnz || (int64_t)F.U.col.size() != Ud.nnz) {
            set_error("gpu setup: host / device compaction mismatch (internal)");
            return SPCG_ERR_INTERNAL;
        }
        if ((st = d2h(C, B, F.L.val.data(), Ld.val, 8 * (size_t)Ld.nnz)) != SPCG_OK) return st;
        if ((st = d2h(C, B, F.U.val.data(), Ud.val, 8 * (size_t)Ud.nnz)) != SPCG_OK) return st;
    }
    GCK(cudaStreamSynchronize(C.s));
    F.fill_level.assign(F.L.col.size() + F.U.col.size(), 0);
    double t5 = now_ms();
    if (he.bad_pivot != ~0ull) {
        F.zero_pivot_row = (int64_t)he.bad_pivot;
        set_error("zero or non-finite pivot at row " + std::to_string(F.zero_pivot_row));
        return SPCG_ERR_ZERO_PIVOT;
    }
    if (phase_ms) {
        phase_ms[0] = t1 - t0;      // upload of A + validation
        phase_ms[1] = t2 - t1;      // Algorithm 2 + Ahat
        phase_ms[2] = t3 - t2;      // L / U split
        phase_ms[3] = t4 - t3;      // ILU(0) numeric + factor levels
        phase_ms[4] = t5 - t4;      // download of Ahat, L, U
    }
    return SPCG_OK;
}

}  // namespace spcg
