// wchain_mrhs.cu — NEXT-4: M independent right-hand sides of one
// system solved together by the warp-chain executor.
//
// Algorithm 1 runs once per right-hand side — M independent PCG
// iterations, each with its own alpha, beta, rho and stopping test — but every
// stream of the iteration that does not depend on the right-hand side is read ONCE
// for all M: the SELL slices of A in the SpMV and the factor records (tags, values,
// 1/u_ii) in the triangular solves.  The vectors are interleaved, position-major
// (v[pos * M + m]), so a step's operand slice for all M is one contiguous
// 256 M-byte block (one TMA bulk copy) and a lane's M values are two 16-byte loads.
// In a chain step each lane carries M independent FMA chains through the same
// shuffles, so the wavefront latency that bounds a single solve (§5.5) is shared by
// M solves.  A right-hand side that has converged (or broken down) is frozen: alpha
// = beta = 0 keeps its x and r unchanged while the others continue.
// Scope: chain layouts whose every dependency is a shuffle (components / grid2d
// without cross-chain terms: the C4 layered field after Algorithm 2), chain warps
// without helpers, x0 = 0.
#include <cuda_runtime.h>

#include "internal.h"

using namespace spcg;

#include "dev_common.cuh"

namespace {

struct MArgs {
    int nrhs;                  // real right-hand sides (<= M; the rest are zero and frozen)
    const double* B;           // [nrhs][n] natural order (column-major n x nrhs)
    double* X;                 // [nrhs][n]
    double *r[2], *w[2], *p[2], *z[2], *y[2], *xp[2];   // halves h of the RHS: [npos * 2] position-major
    double* partials;          // [3 M][gridDim.x]
    double* out;               // [M][4]: k, ||r_k||^2, status, -
    int nst;                   // stages per chain warp
    unsigned stage_bytes;      // CC steps of records + operand slices
    unsigned warp_bytes;
};

constexpr int CC = SPCG_CHAIN_C;

__device__ __forceinline__ void ldm(const double* __restrict__ p, double* v, int M) {
    // M consecutive doubles (16-byte aligned for M >= 2)
    if (M == 1) {
        v[0] = *p;
    } else {
        for (int j = 0; j < M; j += 2) {
            const double2 a = *(const double2*)(p + j);
            v[j] = a.x;
            v[j + 1] = a.y;
        }
    }
}
__device__ __forceinline__ void stm(double* __restrict__ p, const double* v, int M) {
    if (M == 1) {
        *p = v[0];
    } else {
        for (int j = 0; j < M; j += 2) *(double2*)(p + j) = make_double2(v[j], v[j + 1]);
    }
}

// One chunk of CC (or cnt) steps of chain c for all M right-hand sides.
// L (KIND K_ITER): ops r, w, x, p: r_i = r - alpha w, x_i = x + alpha p (lines 11-12),
//   y_i = r_i - sum l_ik y_k, ||r||^2;  K_PRO: ops r (= b): y_i = r_i - ..., ||r||^2.
// U: ops y, r: z_i = (y_i - sum u_ik z_k) / u_ii, (r, z); K_PRO also p0 = z0.
template <int W, bool UPPER, int KIND, int M, int CNT>
__device__ __forceinline__ void mchunk(uint8_t* __restrict__ st, int cnt_rt, int64_t glo, double* __restrict__ out,
                                       double* __restrict__ Er, double* __restrict__ Exp, double* __restrict__ Ep,
                                       const double (&alpha)[M], double (&yprev)[M], double (&dot)[M]) {
    constexpr int RECB = 384 * W + (UPPER ? 256 : 0) + 16;
    const int lane = threadIdx.x & 31;
    const int cnt = CNT > 0 ? CNT : cnt_rt;
    const double* __restrict__ sv = (const double*)(st + (size_t)CC * RECB);   // operand slices, [v][CC][32][M]
    constexpr size_t VS = (size_t)CC * 32 * M;                                  // doubles per operand slice block
#pragma unroll(CNT > 0 ? CNT : 1)
    for (int t = 0; t < (CNT > 0 ? CNT : cnt); ++t) {
        const int i = UPPER ? cnt - 1 - t : t;
        const uint8_t* __restrict__ R = st + (size_t)i * RECB;
        const int64_t pos = 32 * (glo + i) + lane;
        uint32_t tg[W];
        double v[W];
#pragma unroll
        for (int k = 0; k < W; ++k) {
            tg[k] = *(const uint32_t*)(R + 4 * (W * lane + k));
            v[k] = *(const double*)(R + 128 * W + 8 * (W * lane + k));
        }
        const int o = (i * 32 + lane) * M;
        double acc[M], a0[M];
        ldm(sv + o, a0, M);
        if (!UPPER) {
            if (KIND == K_ITER) {
                double w0[M], x0[M], p0[M], xn[M];
                ldm(sv + VS + o, w0, M);
                ldm(sv + 2 * VS + o, x0, M);
                ldm(sv + 3 * VS + o, p0, M);
#pragma unroll
                for (int m = 0; m < M; ++m) {
                    acc[m] = a0[m] - alpha[m] * w0[m];
                    xn[m] = x0[m] + alpha[m] * p0[m];
                }
                stm(Er + pos * M, acc, M);
                stm(Exp + pos * M, xn, M);
            } else {
#pragma unroll
                for (int m = 0; m < M; ++m) acc[m] = a0[m];
            }
#pragma unroll
            for (int m = 0; m < M; ++m) dot[m] = fma(acc[m], acc[m], dot[m]);   // ||r||^2
        } else {
#pragma unroll
            for (int m = 0; m < M; ++m) acc[m] = a0[m];
        }
#pragma unroll
        for (int k = 0; k < W; ++k)
#pragma unroll
            for (int m = 0; m < M; ++m) {
                const double d = __shfl_sync(0xffffffffu, yprev[m], (int)(tg[k] & 31));
                acc[m] = fma(-v[k], d, acc[m]);
            }
        if (UPPER) {
            const double dinv = *(const double*)(R + 384 * W + 8 * lane);
            double rd[M];
            ldm(sv + VS + o, rd, M);
#pragma unroll
            for (int m = 0; m < M; ++m) {
                acc[m] *= dinv;
                dot[m] = fma(rd[m], acc[m], dot[m]);                                  // (r, z)
            }
            if (KIND == K_PRO) stm(Ep + pos * M, acc, M);                           // p0 = z0
        }
        stm(out + pos * M, acc, M);
#pragma unroll
        for (int m = 0; m < M; ++m) yprev[m] = acc[m];
    }
}

// one pass (L forward or U backward) of chain c for M right-hand sides
template <int W, bool UPPER, int KIND, int M>
__device__ __forceinline__ void mpass(const DevChain& D, const MArgs& R, uint8_t* stages, uint64_t* full, unsigned& cq,
                                      int c, const double* const* ops, int nv, double* out, double* Er, double* Exp,
                                      double* Ep, const double (&alpha)[M], double (&dot)[M], Scal* sc) {
    constexpr int RECB = 384 * W + (UPPER ? 256 : 0) + 16;
    const int lane = threadIdx.x & 31;
    const int64_t c0 = D.chain_step[c], c1 = D.chain_step[c + 1];
    const int nstp = (int)(c1 - c0);
    const int NST = R.nst;
    const uint8_t* recs = UPPER ? D.recU : D.recL;
    const int nch = (nstp + CC - 1) / CC;
    auto chunk_range = [&](int q, int64_t& glo, int& cnt) {
        cnt = min(CC, nstp - q * CC);
        glo = UPPER ? (c1 - (int64_t)q * CC - cnt) : (c0 + (int64_t)q * CC);
    };
    auto issue = [&](int q, unsigned slot) {
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        uint8_t* st = stages + (size_t)slot * R.stage_bytes;
        const unsigned rb = (unsigned)(cnt * RECB), vb = (unsigned)cnt * 256u * M;
        mbar_arrive_tx(&full[slot], rb + vb * nv);
        bulk_g2s(st, recs + (size_t)glo * RECB, rb, &full[slot]);
        for (int v = 0; v < nv; ++v)
            bulk_g2s(st + (size_t)CC * RECB + (size_t)v * CC * 256 * M, ops[v] + 32 * glo * M, vb, &full[slot]);
    };
    const unsigned sl0 = cq % (unsigned)NST, ph0 = (cq / (unsigned)NST) & 1u;
    if (lane == 0) {
        unsigned sl = sl0;
        for (int q = 0; q < min(NST, nch); ++q) {
            issue(q, sl);
            if (++sl == (unsigned)NST) sl = 0;
        }
    }
    double yprev[M];
#pragma unroll
    for (int m = 0; m < M; ++m) yprev[m] = 0.0;
    unsigned cs = sl0, cph = ph0;
    for (int q = 0; q < nch; ++q) {
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        if (!warp_ok(mbar_wait(&full[cs], cph, sc))) return;
        uint8_t* st = stages + (size_t)cs * R.stage_bytes;
        if (cnt == CC)
            mchunk<W, UPPER, KIND, M, CC>(st, cnt, glo, out, Er, Exp, Ep, alpha, yprev, dot);
        else
            mchunk<W, UPPER, KIND, M, 0>(st, cnt, glo, out, Er, Exp, Ep, alpha, yprev, dot);
        __syncwarp();
        if (lane == 0 && q + NST < nch) issue(q + NST, cs);
        if (++cs == (unsigned)NST) { cs = 0; cph ^= 1u; }
    }
    cq += (unsigned)nch;
}

template <bool UPPER, int KIND, int M>
__device__ __forceinline__ void mpass_any(const DevChain& D, const MArgs& R, uint8_t* stages, uint64_t* full,
                                          unsigned& cq, int c, const double* const* ops, int nv, double* out,
                                          double* Er, double* Exp, double* Ep, const double (&alpha)[M],
                                          double (&dot)[M], Scal* sc) {
    switch (UPPER ? D.W_U : D.W_L) {
        case 1: mpass<1, UPPER, KIND, M>(D, R, stages, full, cq, c, ops, nv, out, Er, Exp, Ep, alpha, dot, sc); break;
        case 2: mpass<2, UPPER, KIND, M>(D, R, stages, full, cq, c, ops, nv, out, Er, Exp, Ep, alpha, dot, sc); break;
        default: mpass<4, UPPER, KIND, M>(D, R, stages, full, cq, c, ops, nv, out, Er, Exp, Ep, alpha, dot, sc); break;
    }
}

// y = L^-1 r (with the fused updates of the kind) then z = U^-1 y.  The right-hand sides
// come in halves of two (position-major pairs): warp k walks chain blockIdx.x + (k mod
// per_cta) gridDim.x for half k / per_cta, so with M = 4 two warps walk each chain side
// by side, each carrying two FMA chains per step (the records are read by both, the
// second time from L2).  rr / rz: this thread's partial sums, zero for the other half.
template <int KIND, int M>
__device__ __noinline__ void mtri(const DevChain* Dp, const MArgs* Rp, uint8_t* dyn, uint64_t* bars, unsigned* cq,
                                  const double* alpha_in, double* rr, double* rz, Scal* sc) {
    constexpr int H = M / 2;
    const DevChain& D = *Dp;
    const MArgs& R = *Rp;
    const int warp = threadIdx.x >> 5;
    const int h = warp / D.per_cta, slot = warp % D.per_cta;
    const int c = blockIdx.x + slot * gridDim.x;
    if (h >= H || c >= D.nchains) return;
    uint8_t* stages = dyn + (size_t)warp * R.warp_bytes;
    uint64_t* full = bars + warp * 16;
    double alpha[2], a[2], b[2];
#pragma unroll
    for (int j = 0; j < 2; ++j) {
        alpha[j] = alpha_in[2 * h + j];
        a[j] = 0.0;
        b[j] = 0.0;
    }
    unsigned q = *cq;
    {
        const double* ops[4] = {R.r[h], R.w[h], R.xp[h], R.p[h]};
        mpass_any<false, KIND, 2>(D, R, stages, full, q, c, ops, KIND == K_ITER ? 4 : 1, R.y[h], R.r[h], R.xp[h],
                                  R.p[h], alpha, a, sc);
    }
    // the U pass reads y and r through TMA: order this warp's generic stores first
    asm volatile("fence.proxy.async.global;" ::: "memory");
    __syncwarp();
    {
        const double* ops[2] = {R.y[h], R.r[h]};
        mpass_any<true, KIND, 2>(D, R, stages, full, q, c, ops, 2, R.z[h], R.r[h], R.xp[h], R.p[h], alpha, b, sc);
    }
    *cq = q;
#pragma unroll
    for (int j = 0; j < 2; ++j) {
        rr[2 * h + j] += a[j];
        rz[2 * h + j] += b[j];
    }
}

// w = A p for M vectors (TMA-streamed slices of uniform width WA, gathers of the M values
// of a neighbour from the H = M / 2 position-major halves)
template <int WA, int M>
__device__ __forceinline__ void mspmv_stage(const int32_t* __restrict__ cs, const double* __restrict__ vs, int g,
                                            int64_t s, const MArgs& R, double (&pw)[M]) {
    constexpr int G = SPCG_SPMV_G, H = M / 2;
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int u = 0; u < G; ++u) {
        if (u >= g) break;
        double acc[M];
#pragma unroll
        for (int m = 0; m < M; ++m) acc[m] = 0.0;
        double gv[WA][M], vv[WA];
#pragma unroll
        for (int k = 0; k < WA; ++k) {
            const int c = cs[(u * WA + k) * 32 + lane];
            vv[k] = vs[(u * WA + k) * 32 + lane];
#pragma unroll
            for (int hh = 0; hh < H; ++hh) ldm(R.p[hh] + (int64_t)c * 2, gv[k] + 2 * hh, 2);
        }
#pragma unroll
        for (int k = 0; k < WA; ++k)
#pragma unroll
            for (int m = 0; m < M; ++m) acc[m] = fma(vv[k], gv[k][m], acc[m]);
        const int64_t row = (s + u) * 32 + lane;
        double pr[M];
#pragma unroll
        for (int hh = 0; hh < H; ++hh) {
            ldm(R.p[hh] + row * 2, pr + 2 * hh, 2);
            stm(R.w[hh] + row * 2, acc + 2 * hh, 2);
        }
#pragma unroll
        for (int m = 0; m < M; ++m) pw[m] = fma(pr[m], acc[m], pw[m]);
    }
}

template <int M>
__device__ void mspmv(const DevChain& D, const DevA& A, uint8_t* dyn, uint64_t* bars, unsigned& spq, const MArgs& R,
                      double (&pw)[M], Scal* sc) {
    constexpr int G = SPCG_SPMV_G;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t ns = A.nslices;
    const int64_t NW = (int64_t)gridDim.x * NWARP, gw = (int64_t)blockIdx.x * NWARP + warp;
    // groups of G slices dealt round-robin over the grid's warps (group gi = j NW + gw): the
    // positions of weak-coupling fragments cluster at the end of the layout, and contiguous
    // ranges left the warps that got them (far gathers) the last to reach the barrier
    const int64_t ngr = (ns + G - 1) / G;
    const int NS = D.sp_nst, WA = D.WA;
    uint8_t* ring = dyn + (size_t)warp * NS * D.sp_stage_bytes;
    uint64_t* bar = bars + warp * 4;
    const int nst = (int)(gw < ngr ? (ngr - gw + NW - 1) / NW : 0);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    auto issue = [&](int j) {
        const int slot = (spq + j) % NS;
        const int64_t s = ((int64_t)j * NW + gw) * G;
        const int g = (int)(ns - s < (int64_t)G ? ns - s : (int64_t)G);
        const unsigned cb = (unsigned)(g * WA * 128), vb = (unsigned)(g * WA * 256);
        uint8_t* st = ring + (size_t)slot * D.sp_stage_bytes;
        mbar_arrive_tx(&bar[slot], cb + vb);
        bulk_g2s(st, A.col + s * WA * 32, cb, &bar[slot]);
        bulk_g2s(st + (size_t)G * WA * 128, A.val + s * WA * 32, vb, &bar[slot]);
    };
    if (lane == 0)
        for (int j = 0; j < min(NS, nst); ++j) issue(j);
    for (int j = 0; j < nst; ++j) {
        const unsigned u = spq + j;
        if (!warp_ok(mbar_wait(&bar[u % NS], (u / NS) & 1, sc))) return;
        const uint8_t* st = ring + (size_t)(u % NS) * D.sp_stage_bytes;
        const int32_t* cs = (const int32_t*)st;
        const double* vs = (const double*)(st + (size_t)G * WA * 128);
        const int64_t s = ((int64_t)j * NW + gw) * G;
        const int g = (int)(ns - s < (int64_t)G ? ns - s : (int64_t)G);
        switch (WA) {
            case 3: mspmv_stage<3, M>(cs, vs, g, s, R, pw); break;
            case 4: mspmv_stage<4, M>(cs, vs, g, s, R, pw); break;
            case 5: mspmv_stage<5, M>(cs, vs, g, s, R, pw); break;
            case 6: mspmv_stage<6, M>(cs, vs, g, s, R, pw); break;
            case 7: mspmv_stage<7, M>(cs, vs, g, s, R, pw); break;
            default: mspmv_stage<8, M>(cs, vs, g, s, R, pw); break;
        }
        __syncwarp();
        if (lane == 0 && j + NS < nst) issue(j + NS);
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    spq += (unsigned)nst;
}

// per-CTA partials of 2 M sums (fixed order) -> partials[slot + m][blockIdx.x]
template <int M>
__device__ void mpartials(const double (&a)[M], const double (&b)[M], double* partials, int slot) {
    __shared__ double red[2 * 4][NWARP];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int m = 0; m < M; ++m) {
        const double x = warp_sum(a[m]), y = warp_sum(b[m]);
        if (lane == 0) {
            red[m][warp] = x;
            red[M + m][warp] = y;
        }
    }
    __syncthreads();
    if (warp == 0) {
#pragma unroll
        for (int j = 0; j < 2 * M; ++j) {
            double x = lane < NWARP ? red[j][lane] : 0.0;
            x = warp_sum(x);
            if (lane == 0) partials[(size_t)(slot + j) * gridDim.x + blockIdx.x] = x;
        }
    }
    __syncthreads();
}
template <int M>
__device__ void msums(const double* partials, int slot, int cnt, double* outv) {
    __shared__ double bc[2 * 4];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (warp == 0) {
        for (int j = 0; j < cnt; ++j) {
            double x = 0.0;
            for (int i = lane; i < (int)gridDim.x; i += 32) x += __ldcg(partials + (size_t)(slot + j) * gridDim.x + i);
            x = warp_sum(x);
            if (lane == 0) bc[j] = x;
        }
    }
    __syncthreads();
    for (int j = 0; j < cnt; ++j) outv[j] = bc[j];
    __syncthreads();
}

__device__ __forceinline__ void sync_tma(Scal* sc, unsigned& gen) {
    asm volatile("fence.proxy.async.global;" ::: "memory");
    grid_sync(sc, gen);
    asm volatile("fence.proxy.async.global;" ::: "memory");
}

template <int M>
__global__ void __launch_bounds__(BLOCK, 1) spcg_wchain_mrhs_kernel(Params P, MArgs R) {
    extern __shared__ __align__(128) uint8_t dynw[];
    __shared__ DevChain sD;
    __shared__ MArgs sR;
    __shared__ __align__(8) uint64_t bars[NWARP * 16];
    __shared__ __align__(8) uint64_t spbar[NWARP * 4];
    const DevChain& D = P.CH;
    if (threadIdx.x == 0) {
        sD = P.CH;
        sR = R;
        for (int i = 0; i < NWARP * 16; ++i) mbar_init(&bars[i], 1);
        for (int i = 0; i < NWARP * 4; ++i) mbar_init(&spbar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    unsigned gen = 0, cq = 0, spq = 0;
    const int64_t npos = D.npos, n = P.n;
    const int64_t stride = (int64_t)gridDim.x * BLOCK;
    // b to position order (r0 = b, x0 = 0: Alg. 1 lines 1-2)
    for (int64_t e = (int64_t)blockIdx.x * BLOCK + threadIdx.x; e < npos * M; e += stride) {
        const int64_t pos = e / M;
        const int m = (int)(e % M);
        const int32_t row = __ldg(D.perm + pos);
        const int64_t hi = pos * 2 + (m & 1);
        R.r[m >> 1][hi] = (row >= 0 && m < R.nrhs) ? R.B[(int64_t)m * n + row] : 0.0;
        R.xp[m >> 1][hi] = 0.0;
    }
    sync_tma(P.sc, gen);
    double alpha[M], rr_l[M], rz_l[M];
#pragma unroll
    for (int m = 0; m < M; ++m) { alpha[m] = 0.0; rr_l[m] = 0.0; rz_l[m] = 0.0; }
    mtri<K_PRO, M>(&sD, &sR, dynw, bars, &cq, alpha, rr_l, rz_l, P.sc);          // lines 3-4
    mpartials<M>(rz_l, rr_l, R.partials, 0);
    grid_sync(P.sc, gen);
    double sums[2 * 4];
    msums<M>(R.partials, 0, 2 * M, sums);
    double rho[M], rr[M];
    long long kconv[M];
    int st[M];
    bool frozen[M];
#pragma unroll
    for (int m = 0; m < M; ++m) {
        rho[m] = sums[m];
        rr[m] = sums[M + m];
        frozen[m] = m >= R.nrhs;
        kconv[m] = 0;
        st[m] = SPCG_OK;
    }
    long long k = 0;
    for (;;) {
        bool all = true;
#pragma unroll
        for (int m = 0; m < M; ++m) {
            if (!frozen[m] && (sqrt(rr[m]) < P.eps || rr[m] == 0.0)) {      // lines 6-7, per right-hand side
                frozen[m] = true;
                kconv[m] = k;
                st[m] = SPCG_OK;
            }
            all = all && frozen[m];
        }
        if (all) break;
        if (k == P.kmax) {                                                  // A14
#pragma unroll
            for (int m = 0; m < M; ++m)
                if (!frozen[m]) {
                    frozen[m] = true;
                    kconv[m] = k;
                    st[m] = P.eps > 0.0 ? SPCG_NOT_CONVERGED : SPCG_OK;
                }
            break;
        }
        if (__syncthreads_or(ld_volatile_int(&P.sc->abort))) break;
        // lines 9-10
        double pw[M], zero[M];
#pragma unroll
        for (int m = 0; m < M; ++m) { pw[m] = 0.0; zero[m] = 0.0; }
        mspmv<M>(sD, P.A, dynw, spbar, spq, sR, pw, P.sc);
        mpartials<M>(pw, zero, R.partials, 2 * M);
        sync_tma(P.sc, gen);
        msums<M>(R.partials, 2 * M, M, sums);
#pragma unroll
        for (int m = 0; m < M; ++m) {
            const double sigma = sums[m];
            if (frozen[m]) {
                alpha[m] = 0.0;
            } else if (!(sigma > 0.0) || !isfinite(sigma) || !isfinite(rho[m])) {
                frozen[m] = true;
                kconv[m] = k;
                st[m] = SPCG_ERR_BREAKDOWN;
                alpha[m] = 0.0;
            } else {
                alpha[m] = rho[m] / sigma;
            }
            rr_l[m] = 0.0;
            rz_l[m] = 0.0;
        }
        // lines 11-13 (+ ||r||^2, (r, z))
        mtri<K_ITER, M>(&sD, &sR, dynw, bars, &cq, alpha, rr_l, rz_l, P.sc);
        mpartials<M>(rz_l, rr_l, R.partials, 0);
        grid_sync(P.sc, gen);
        msums<M>(R.partials, 0, 2 * M, sums);
        // lines 14-15
        double beta[M];
#pragma unroll
        for (int m = 0; m < M; ++m) {
            beta[m] = frozen[m] ? 0.0 : sums[m] / rho[m];
            if (!frozen[m]) {
                rho[m] = sums[m];
                rr[m] = sums[M + m];
            }
        }
        // p = z + beta p, 16-byte accesses (a position's pair of a half), four in flight per thread
#pragma unroll
        for (int hh = 0; hh < M / 2; ++hh) {
            double2* __restrict__ p2 = (double2*)R.p[hh];
            const double2* __restrict__ z2 = (const double2*)R.z[hh];
            const double b0 = beta[2 * hh], b1 = beta[2 * hh + 1];
            for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < npos; i += 4 * stride) {
                double2 pv[4], zv[4];
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (i + u * stride < npos) {
                        pv[u] = p2[i + u * stride];
                        zv[u] = __ldcg(z2 + i + u * stride);
                    }
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (i + u * stride < npos)
                        p2[i + u * stride] = make_double2(fma(b0, pv[u].x, zv[u].x), fma(b1, pv[u].y, zv[u].y));
            }
        }
        sync_tma(P.sc, gen);
        ++k;
    }
    // x back to natural order
    for (int64_t e = (int64_t)blockIdx.x * BLOCK + threadIdx.x; e < npos * M; e += stride) {
        const int64_t pos = e / M;
        const int m = (int)(e % M);
        const int32_t row = __ldg(D.perm + pos);
        if (row >= 0 && m < R.nrhs) R.X[(int64_t)m * n + row] = R.xp[m >> 1][pos * 2 + (m & 1)];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
#pragma unroll
        for (int m = 0; m < M; ++m) {
            R.out[4 * m + 0] = (double)kconv[m];
            R.out[4 * m + 1] = rr[m];
            R.out[4 * m + 2] = (double)(ld_volatile_int(&P.sc->abort) ? SPCG_ERR_INTERNAL : st[m]);
        }
        P.sc->status = ld_volatile_int(&P.sc->abort) ? SPCG_ERR_INTERNAL : SPCG_OK;
    }
}

}  // namespace

// host hooks (kernels.cu owns the device handle)
void* spcg_wchain_mrhs_kernel_ptr(int M) {
    switch (M) {
        case 2: return (void*)spcg_wchain_mrhs_kernel<2>;
        case 4: return (void*)spcg_wchain_mrhs_kernel<4>;
        default: return nullptr;
    }
}
size_t spcg_mrhs_args_size() { return sizeof(MArgs); }
// fills an MArgs at dst (kernels.cu does not see the struct)
void spcg_mrhs_args_fill(void* dst, int nrhs, const double* B, double* X, double* const* vec, double* partials,
                         double* out, int nst, unsigned stage_bytes, unsigned warp_bytes) {
    // vec: 12 arrays, [vector][half] for r, w, p, z, y, xp
    MArgs* a = (MArgs*)dst;
    a->nrhs = nrhs;
    a->B = B;
    a->X = X;
    for (int h = 0; h < 2; ++h) {
        a->r[h] = vec[0 + h];
        a->w[h] = vec[2 + h];
        a->p[h] = vec[4 + h];
        a->z[h] = vec[6 + h];
        a->y[h] = vec[8 + h];
        a->xp[h] = vec[10 + h];
    }
    a->partials = partials;
    a->out = out;
    a->nst = nst;
    a->stage_bytes = stage_bytes;
    a->warp_bytes = warp_bytes;
}
