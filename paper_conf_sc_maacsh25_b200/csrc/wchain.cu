// wchain.cu — the warp-chain executor of the iterative phase.
//
// One persistent cooperative kernel runs Algorithm 1 on vectors kept
// in execution ("position") order for the whole solve: b is gathered and x
// scattered once per solve.  Per iteration:
//   w = A p (original A) + (p, w)          all warps, grid barrier, alpha
//   y = L^-1 r with the fused x / r update + ||r||^2   solver warps, one chain each
//   z = U^-1 y + (r, z)                                 same warps, chain in reverse
//   grid barrier, beta;  p = z + beta p;  grid barrier
// A chain is walked by ONE warp, a step (<= 32 rows of one wavefront level, one per
// lane) at a time.  A dependency produced by the same warp in its previous step is
// read from that lane's register with a shuffle — no memory access and no barrier
// on the chain; older own values come from a shared-memory ring, other chains'
// values from epoch-stamped ready flags prefetched with cp.async one chunk ahead.
// Records (tags, values, 1/u_ii) and the per-step operand slices of the position-
// ordered vectors stream into shared memory with TMA bulk copies (NST stages of C
// steps per solver warp), so the chain never waits on HBM.
#include <cuda_runtime.h>

#include <cstdio>

#include "internal.h"

using namespace spcg;

#include "dev_common.cuh"

namespace {


__device__ __forceinline__ void cpa16(void* sdst, const void* gsrc) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sdst)), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cpa_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cpa_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cpa_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }
// generic-proxy global writes -> later TMA (async-proxy) reads of the same data
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }

struct WarpSmem {
    uint64_t* full;        // [nst] mbarriers
    uint8_t* stages;       // nst x stage_bytes
    uint4* extq;           // [2][C][2][32] prefetched ready flags
    double* hist;          // [SPCG_CHAIN_HIST][32]
};

__device__ __forceinline__ WarpSmem warp_smem(const DevChain& D, uint8_t* dyn, int sw) {
    WarpSmem W;
    uint8_t* base = dyn + (size_t)sw * D.warp_bytes;
    W.full = (uint64_t*)base;
    W.stages = base + 128;
    W.extq = (uint4*)(base + D.ext_off);
    W.hist = (double*)(base + D.hist_off);
    return W;
}

// Operand vectors of a pass (position order); nv of them are staged per chunk.
struct PassOps {
    const double* v[4];
    int nv;
};

// One pass (L forward or U backward) of chain c by the calling warp.
//   L: KIND K_ITER: ops r, w, x, p -> r_i = r - alpha w, x_i = x + alpha p (Alg. 1 lines
//      11-12 fused), y_i = r_i - sum l_ij y_j, ||r||^2;  K_PRO: ops rsrc (b or b - A x0);
//      K_APPLY: ops in.
//   U: ops y [, rdot] -> z_i = (y_i - sum u_ij z_j) / u_ii, (rdot, z); K_PRO also p0 = z0.
// cq: chunks this warp consumed so far in the launch (mbarrier phase bookkeeping).
// Vectors and scalars a pass touches besides its operands (plain pointers: the
// kernel parameter block is never referenced from here, so nothing is copied to
// local memory).
struct PassEnv {
    double* r;
    double* p;
    double* xp;
    Scal* sc;
    int use_x0;
};

template <bool UPPER, int KIND>
__device__ __forceinline__ void chain_pass(const DevChain& D, const PassEnv& E, const WarpSmem& W, unsigned& cq, int c,
                                           const PassOps& ops, double* out, double alpha, double& acc_dot, uint4* mb,
                                           unsigned ep) {
    const int lane = threadIdx.x & 31;
    double* const Er = E.r;
    double* const Ep = E.p;
    double* const Exp = E.xp;
    const bool rsrc_is_r = ops.v[0] == Er;
    const int64_t s0 = D.chain_step[c], s1 = D.chain_step[c + 1];
    const int nst = (int)(s1 - s0);
    const int C = D.C, NST = D.nst;
    const int Wd = UPPER ? D.W_U : D.W_L;
    const int recb = UPPER ? D.rec_U : D.rec_L;
    const uint8_t* recs = UPPER ? D.recU : D.recL;
    const uint32_t cfl = D.chain_flags[c];
    const bool use_hist = cfl & (UPPER ? CC_UHIST : CC_LHIST);
    const bool use_ext = cfl & (UPPER ? CC_UEXT : CC_LEXT);
    const int nch = (nst + C - 1) / C;
    const size_t trailer = (size_t)384 * Wd + (UPPER ? 256 : 0);
    // global step range of chunk q (ascending inside the stage for both passes)
    auto chunk_range = [&](int q, int64_t& glo, int& cnt) {
        cnt = min(C, nst - q * C);
        glo = UPPER ? (s1 - (int64_t)q * C - cnt) : (s0 + (int64_t)q * C);
    };
    auto stage_of = [&](int q) { return W.stages + (size_t)((cq + q) % NST) * D.stage_bytes; };
    auto issue = [&](int q) {               // lane 0 only
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        const unsigned slot = (cq + q) % NST;
        uint8_t* st = stage_of(q);
        const unsigned rb = (unsigned)(cnt * recb), vb = (unsigned)cnt * 256u;
        mbar_arrive_tx(&W.full[slot], rb + vb * ops.nv);
        bulk_g2s(st, recs + (size_t)glo * recb, rb, &W.full[slot]);
        uint8_t* vdst = st + (size_t)C * recb;
        for (int v = 0; v < ops.nv; ++v)
            bulk_g2s(vdst + (size_t)v * C * 256, ops.v[v] + 32 * glo, vb, &W.full[slot]);
    };
    auto wait_chunk = [&](int q) -> bool {
        const unsigned u = cq + q;
        return warp_ok(mbar_wait(&W.full[u % NST], (u / NST) & 1, E.sc));
    };
    // ready flags of chunk q's cross-chain entries -> extq[q & 1] (one cp.async each)
    auto prefetch_ext = [&](int q) {
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        const uint8_t* st = stage_of(q);
        uint4* qb = W.extq + (size_t)(q & 1) * C * 64;
        for (int i = 0; i < cnt; ++i) {
            const uint8_t* R = st + (size_t)i * recb;
            if (!(*(const uint32_t*)(R + trailer + 4) & CS_EXT)) continue;
            const int t = UPPER ? cnt - 1 - i : i;          // pass-order index inside the chunk
            for (int k = 0; k < Wd; ++k) {
                const uint32_t tg = *(const uint32_t*)(R + 128 * k + 4 * lane);
                if ((tg >> 29) == CT_EXT)
                    cpa16(qb + ((size_t)t * 2 + ((tg >> 28) & 1)) * 32 + lane, mb + (tg & 0x0fffffffu));
            }
        }
    };

    if (lane == 0)
        for (int q = 0; q < min(NST, nch); ++q) issue(q);
    if (use_ext && nch > 0) {
        if (!wait_chunk(0)) return;
        prefetch_ext(0);
    }
    cpa_commit();
    double yprev = 0.0;
    double dot = acc_dot;
    int u = 0;                                              // pass step
    for (int q = 0; q < nch; ++q) {
        if (use_ext && q + 1 < nch) {
            if (!wait_chunk(q + 1)) return;
            prefetch_ext(q + 1);
        }
        cpa_commit();
        cpa_wait1();                                        // chunk q's flags landed
        if (!wait_chunk(q)) return;
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        const uint8_t* st = stage_of(q);
        const double* sv = (const double*)(st + (size_t)C * recb);
        const uint4* qb = W.extq + (size_t)(q & 1) * C * 64;
        for (int t = 0; t < cnt; ++t, ++u) {
            const int i = UPPER ? cnt - 1 - t : t;           // in-stage index (ascending g)
            const uint8_t* R = st + (size_t)i * recb;
            const int64_t pos = 32 * (glo + i) + lane;
            const uint32_t pubm = *(const uint32_t*)(R + trailer);
            const uint32_t fl = *(const uint32_t*)(R + trailer + 4);
            double acc, ri = 0.0, xn = 0.0, rdv = 0.0;
            if (!UPPER) {
                if (KIND == K_ITER) {
                    const double r0 = sv[i * 32 + lane], w0 = sv[C * 32 + i * 32 + lane];
                    const double x0 = sv[2 * C * 32 + i * 32 + lane], p0 = sv[3 * C * 32 + i * 32 + lane];
                    ri = r0 - alpha * w0;
                    xn = x0 + alpha * p0;
                } else {
                    ri = sv[i * 32 + lane];
                }
                acc = ri;
            } else {
                acc = sv[i * 32 + lane];
                if (ops.nv > 1) rdv = sv[C * 32 + i * 32 + lane];
            }
            if (!(fl & CS_SLOW)) {
                // every dependency is the previous step's value of some lane (or padding)
#pragma unroll
                for (int k = 0; k < SPCG_CHAIN_WMAX; ++k) {
                    if (k >= Wd) break;
                    const uint32_t tg = *(const uint32_t*)(R + 128 * k + 4 * lane);
                    const double v = *(const double*)(R + 128 * Wd + 256 * k + 8 * lane);
                    const double d = __shfl_sync(0xffffffffu, yprev, tg & 31);
                    acc = fma(-v, d, acc);
                }
            } else {
                for (int k = 0; k < Wd; ++k) {
                    const uint32_t tg = *(const uint32_t*)(R + 128 * k + 4 * lane);
                    const double v = *(const double*)(R + 128 * Wd + 256 * k + 8 * lane);
                    double d = __shfl_sync(0xffffffffu, yprev, tg & 31);
                    const uint32_t kind = tg >> 29;
                    if (kind == CT_HIST) {
                        d = W.hist[((u - (int)((tg >> 5) & 255)) & (SPCG_CHAIN_HIST - 1)) * 32 + (tg & 31)];
                    } else if (kind == CT_GLOB) {
                        d = __ldcg(out + (tg & 0x1fffffffu));
                    } else if (kind == CT_EXT) {
                        const uint4 f = qb[((size_t)t * 2 + ((tg >> 28) & 1)) * 32 + lane];
                        if (f.y == ep && f.w == ep) d = __longlong_as_double((long long)(((unsigned long long)f.z << 32) | f.x));
                        else d = ll_wait(mb + (tg & 0x0fffffffu), ep, E.sc);
                    } else if (kind == CT_EXTS) {
                        d = ll_wait(mb + (tg & 0x1fffffffu), ep, E.sc);
                    } else if (kind == CT_PAD) {
                        d = 0.0;
                    }
                    acc = fma(-v, d, acc);
                }
            }
            if (UPPER) {
                acc *= *(const double*)(R + 384 * Wd + 8 * lane);
                if (ops.nv > 1) dot = fma(rdv, acc, dot);           // (r, z)
                if (KIND == K_PRO) Ep[pos] = acc;                    // p0 = z0
            } else {
                dot = fma(ri, ri, dot);                              // ||r||^2
                if (KIND == K_ITER) {
                    Er[pos] = ri;
                    Exp[pos] = xn;
                } else if (KIND == K_PRO) {
                    if (!rsrc_is_r) Er[pos] = ri;
                    if (!E.use_x0) Exp[pos] = 0.0;
                }
            }
            out[pos] = acc;
            if ((pubm >> lane) & 1u) ll_store(mb + pos, acc, ep);
            if (use_hist) {
                W.hist[(u & (SPCG_CHAIN_HIST - 1)) * 32 + lane] = acc;
                __syncwarp();
            }
            yprev = acc;
        }
        __syncwarp();
        if (lane == 0 && q + NST < nch) issue(q + NST);
    }
    cpa_wait0();
    cq += (unsigned)nch;
    acc_dot = dot;
}

// z = U^-1 L^-1 r for every chain of this CTA (solver warps), the fused vector work
// of the kind; rr / rz: this thread's partial sums.  D: the chain layout, copied to
// shared memory by the kernel.
__device__ __noinline__ void tri_chains(const DevChain* Dp, PassEnv E, uint8_t* dyn, unsigned* cq, int kind,
                                        const double* rsrc, const double* w, double* y, double* z,
                                        const double* rdot, uint4* mbL, uint4* mbU, unsigned ep, double alpha,
                                        bool lower, bool upper, double* rr, double* rz) {
    const DevChain& D = *Dp;
    const int warp = threadIdx.x >> 5;
    const int c = blockIdx.x + warp * gridDim.x;
    if (warp >= D.per_cta || c >= D.nchains) return;
    const WarpSmem W = warp_smem(D, dyn, warp);
    unsigned q = *cq;
    double a = *rr, b = *rz;
    if (lower) {
        PassOps o{};
        if (kind == K_ITER) {
            o.v[0] = E.r; o.v[1] = w; o.v[2] = E.xp; o.v[3] = E.p; o.nv = 4;
            chain_pass<false, K_ITER>(D, E, W, q, c, o, y, alpha, a, mbL, ep);
        } else if (kind == K_PRO) {
            o.v[0] = rsrc; o.nv = 1;
            chain_pass<false, K_PRO>(D, E, W, q, c, o, y, 0.0, a, mbL, ep);
        } else {
            o.v[0] = rsrc; o.nv = 1;
            chain_pass<false, K_APPLY>(D, E, W, q, c, o, y, 0.0, a, mbL, ep);
        }
        // the U pass reads this warp's y (and r) through TMA: order the generic stores first
        fence_proxy_async_global();
        __syncwarp();
    }
    if (upper) {
        PassOps o{};
        o.v[0] = y;
        o.nv = 1;
        if (rdot) { o.v[1] = rdot; o.nv = 2; }
        if (kind == K_PRO) chain_pass<true, K_PRO>(D, E, W, q, c, o, z, 0.0, b, mbU, ep);
        else chain_pass<true, K_APPLY>(D, E, W, q, c, o, z, 0.0, b, mbU, ep);
    }
    *cq = q;
    *rr = a;
    *rz = b;
}

// position-order <-> natural-order copies
__device__ void gather(const Params& P, const double* nat, double* pos_out) {
    const int64_t stride = (int64_t)gridDim.x * BLOCK;
    for (int64_t p = (int64_t)blockIdx.x * BLOCK + threadIdx.x; p < P.CH.npos; p += stride) {
        const int32_t row = __ldg(P.CH.perm + p);
        pos_out[p] = row >= 0 ? nat[row] : 0.0;
    }
}
__device__ void scatter(const Params& P, const double* pos_in, double* nat) {
    const int64_t stride = (int64_t)gridDim.x * BLOCK;
    for (int64_t p = (int64_t)blockIdx.x * BLOCK + threadIdx.x; p < P.CH.npos; p += stride) {
        const int32_t row = __ldg(P.CH.perm + p);
        if (row >= 0) nat[row] = pos_in[p];
    }
}

// barrier after generic-proxy writes that TMA will read (both sides fence)
__device__ __forceinline__ void sync_for_tma(const Params& P, unsigned& gen) {
    fence_proxy_async_global();
    grid_sync(P.sc, gen);
    fence_proxy_async_global();
}

__global__ void __launch_bounds__(BLOCK, 1) spcg_wchain_kernel(Params P) {
    extern __shared__ __align__(128) uint8_t dynw[];
    __shared__ DevChain sD;
    const DevChain& D = P.CH;
    unsigned gen = 0;
    unsigned cq = 0;
    if (threadIdx.x == 0) {
        sD = P.CH;
        // mbarriers of every solver warp of this CTA
        for (int sw = 0; sw < D.per_cta; ++sw) {
            const WarpSmem W = warp_smem(D, dynw, sw);
            for (int s = 0; s < D.nst; ++s) mbar_init(&W.full[s], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const PassEnv E{P.r, P.p, D.xp, P.sc, P.use_x0};
    const int64_t npos = D.npos;

    if (P.mode != M_SOLVE) {
        double a = 0.0, b = 0.0;
        if (P.mode == M_SPMV) {
            gather(P, P.in, D.t1);
            grid_sync(P.sc, gen);
            phase_spmv(P.A, npos, D.t1, P.w, a);
            grid_sync(P.sc, gen);
            scatter(P, P.w, P.out);
        } else if (P.mode == M_LOWER) {
            gather(P, P.in, D.t1);
            sync_for_tma(P, gen);
            tri_chains(&sD, E, dynw, &cq, K_APPLY, D.t1, P.w, P.y, P.z, nullptr, P.mbL, P.mbU, P.epoch, 0.0, true, false,
                       &a, &b);
            grid_sync(P.sc, gen);
            scatter(P, P.y, P.out);
        } else if (P.mode == M_UPPER) {
            gather(P, P.in, P.y);
            if (P.aux) gather(P, P.aux, D.t1);
            sync_for_tma(P, gen);
            tri_chains(&sD, E, dynw, &cq, K_APPLY, nullptr, P.w, P.y, P.z, P.aux ? D.t1 : nullptr, P.mbL, P.mbU, P.epoch,
                       0.0, false, true, &a, &b);
            grid_sync(P.sc, gen);
            scatter(P, P.z, P.out);
        } else {
            gather(P, P.in, D.t1);
            sync_for_tma(P, gen);
            tri_chains(&sD, E, dynw, &cq, K_APPLY, D.t1, P.w, P.y, P.z, D.t1, P.mbL, P.mbU, P.epoch, 0.0, true, true, &a,
                       &b);
            grid_sync(P.sc, gen);
            scatter(P, P.z, P.out);
        }
        block_partials(a, b, P.partials, 0, 1);
        grid_sync(P.sc, gen);
        double sa, sb;
        global_sums(P.partials, 0, 1, sa, sb);
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            P.sc->out_scalar = P.mode == M_SPMV ? sa : sb;
            P.sc->rr = sa;
            P.sc->status = ld_volatile_int(&P.sc->abort) ? SPCG_ERR_INTERNAL : SPCG_OK;
        }
        return;
    }

    // ---------------- Alg. 1 lines 1-4 (b, x0 to position order first)
    gather(P, P.b, D.bp);
    if (P.use_x0) gather(P, P.x, D.xp);
    const double* r_src = D.bp;
    if (P.use_x0) {
        grid_sync(P.sc, gen);
        double dummy = 0.0;
        phase_spmv(P.A, npos, D.xp, P.w, dummy);
        grid_sync(P.sc, gen);
        const int64_t stride = (int64_t)gridDim.x * BLOCK;
        for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < npos; i += stride) P.r[i] = D.bp[i] - P.w[i];
        r_src = P.r;
    }
    sync_for_tma(P, gen);
    unsigned app = 0;
    double rr_l = 0.0, rz_l = 0.0;
    tri_chains(&sD, E, dynw, &cq, K_PRO, r_src, P.w, P.y, P.z, P.r, P.mbL, P.mbU, P.epoch + app, 0.0, true, true, &rr_l,
               &rz_l);
    ++app;
    block_partials(rz_l, rr_l, P.partials, 0, 1);
    grid_sync(P.sc, gen);
    double rho, rr;
    global_sums(P.partials, 0, 1, rho, rr);

    long long k = 0;
    int status = SPCG_OK;
    for (;;) {
        const double rn = sqrt(rr);
        if (blockIdx.x == 0 && threadIdx.x == 0 && P.rhist && k < P.rhist_cap) P.rhist[k] = rn;
        if (rn < P.eps || rr == 0.0) { status = SPCG_OK; break; }                       // lines 6-7
        if (k == P.kmax) { status = P.eps > 0.0 ? SPCG_NOT_CONVERGED : SPCG_OK; break; }  // A14
        if (__syncthreads_or(ld_volatile_int(&P.sc->abort))) { status = SPCG_ERR_INTERNAL; break; }
        // lines 9-10: w = A p, sigma = (p, w), alpha = rho / sigma
        double pw = 0.0;
        phase_spmv(P.A, npos, P.p, P.w, pw);
        block_partials(pw, 0.0, P.partials, 2, -1);
        sync_for_tma(P, gen);
        double sigma, unused;
        global_sums(P.partials, 2, -1, sigma, unused);
        if (!(sigma > 0.0) || !isfinite(sigma) || !isfinite(rho)) { status = SPCG_ERR_BREAKDOWN; break; }
        const double alpha = rho / sigma;
        // lines 11-13 (+ ||r||^2, (r, z))
        rr_l = 0.0;
        rz_l = 0.0;
        tri_chains(&sD, E, dynw, &cq, K_ITER, P.r, P.w, P.y, P.z, P.r, P.mbL, P.mbU, P.epoch + app, alpha, true, true,
                   &rr_l, &rz_l);
        ++app;
        block_partials(rz_l, rr_l, P.partials, 0, 1);
        grid_sync(P.sc, gen);
        double rho_new;
        global_sums(P.partials, 0, 1, rho_new, rr);
        // lines 14-15
        const double beta = rho_new / rho;
        rho = rho_new;
        const int64_t stride = (int64_t)gridDim.x * BLOCK;
        for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < npos; i += stride)
            P.p[i] = fma(beta, P.p[i], P.z[i]);
        sync_for_tma(P, gen);
        ++k;
    }
    // x back to natural order (every position written by this launch's own CTAs: no barrier
    // needed before, the last phase ended with one)
    scatter(P, D.xp, P.x);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        P.sc->k = k;
        P.sc->rr = rr;
        P.sc->rho = rho;
        P.sc->status = ld_volatile_int(&P.sc->abort) ? SPCG_ERR_INTERNAL : status;
    }
}

}  // namespace

// host-side hooks (kernels.cu owns the device handle)
void* spcg_wchain_kernel_ptr() { return (void*)spcg_wchain_kernel; }
