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
// named barrier for a chain warp and its helper (ids 1..4; 0 is __syncthreads)
__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

#ifndef SPCG_CHAIN_PROF
#define SPCG_CHAIN_PROF 0      // debug builds (tools/chain_prof.py): per-pass cycle counters, no cost otherwise
#endif
__device__ unsigned long long* g_chain_prof = nullptr;   // [24]: L at 0, U at 8 (chain_pass), phases at 16
__device__ __forceinline__ void prof_phase(int idx, long long& t) {
    if (SPCG_CHAIN_PROF && g_chain_prof && threadIdx.x == 0) {
        const long long now = clock64();
        atomicAdd(g_chain_prof + 16 + idx, (unsigned long long)(now - t));
        t = now;
    }
}

struct WarpSmem {
    uint64_t* full;        // [nst] mbarriers: TMA landed
    uint64_t* hand;        // [nst] mbarriers: handoff between the chain warp and its helper
    uint8_t* stages;       // nst x stage_bytes
    uint4* extq;           // [2][C][2][32] prefetched ready flags
    double* hist;          // [SPCG_CHAIN_HIST][32]
};

// per solver-warp slot: full[16] + hand[16] mbarriers, in static shared memory (the
// dynamic area is reused by the SpMV's TMA stages between the triangular solves)
__shared__ __align__(8) uint64_t s_chain_bar[NWARP][32];

__device__ __forceinline__ WarpSmem warp_smem(const DevChain& D, uint8_t* dyn, int sw) {
    WarpSmem W;
    uint8_t* base = dyn + (size_t)sw * D.warp_bytes;
    W.full = &s_chain_bar[sw][0];
    W.hand = &s_chain_bar[sw][16];
    W.stages = base;
    W.extq = (uint4*)(base + D.ext_off);
    W.hist = (double*)(base + D.hist_off);
    return W;
}

// Operand vectors of a pass (position order); nv of them are staged per chunk.
struct PassOps {
    const double* v[4];
    int nv;
};

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

constexpr int CC = SPCG_CHAIN_C;          // steps per stage

// lane-major record fields: W u32 tags / f64 values of this lane, vector shared loads
template <int W>
__device__ __forceinline__ void lds_tags(const uint8_t* __restrict__ p, uint32_t (&t)[W]) {
    if constexpr (W == 1) {
        t[0] = *(const uint32_t*)p;
    } else if constexpr (W == 2) {
        const uint2 a = *(const uint2*)p;
        t[0] = a.x;
        t[1] = a.y;
    } else {
#pragma unroll
        for (int j = 0; j < W; j += 4) {
            const uint4 a = *(const uint4*)(p + 4 * j);
            t[j] = a.x;
            t[j + 1] = a.y;
            t[j + 2] = a.z;
            t[j + 3] = a.w;
        }
    }
}
template <int W>
__device__ __forceinline__ void lds_vals(const uint8_t* __restrict__ p, double (&v)[W]) {
    if constexpr (W == 1) {
        v[0] = *(const double*)p;
    } else {
#pragma unroll
        for (int j = 0; j < W; j += 2) {
            const double2 a = *(const double2*)(p + 8 * j);
            v[j] = a.x;
            v[j + 1] = a.y;
        }
    }
}

// fp32 record values (NEXT-2): W floats of this lane, widened exactly to fp64
template <int W>
__device__ __forceinline__ void lds_vals_f32(const uint8_t* __restrict__ p, double (&v)[W]) {
    if constexpr (W == 1) {
        v[0] = (double)*(const float*)p;
    } else if constexpr (W == 2) {
        const float2 a = *(const float2*)p;
        v[0] = (double)a.x;
        v[1] = (double)a.y;
    } else {
#pragma unroll
        for (int j = 0; j < W; j += 4) {
            const float4 a = *(const float4*)(p + 4 * j);
            v[j] = (double)a.x;
            v[j + 1] = (double)a.y;
            v[j + 2] = (double)a.z;
            v[j + 3] = (double)a.w;
        }
    }
}

// What a GENERAL pass needs besides the shuffle path (HIST / GLOB / EXT entries,
// published values, the history ring).
struct GenCtx {
    double* hist;          // [SPCG_CHAIN_HIST][32]
    const uint4* qb;       // prefetched ready flags of this chunk: [CC][2][32]
    uint4* mb;             // this pass's ready flags (position order)
    Scal* sc;
    unsigned ep;
    bool use_hist;
};

// The steps of one staged chunk on the chain warp.  st: the stage (records, then the
// operand slices); glo: global step of in-stage index 0; u0: pass step of the chunk's
// first step.  A dependency's value comes from lane tag[k] of the previous step (a
// shuffle of the loop-carried yprev); GEN passes override the few other kinds.
// SPLIT: a helper warp does the vector work of the pass (the fused r/x update and
// ||r||^2 before the chain in L, which leaves r_i in the stage's first operand slice;
// the store of z, (r,z) and p0 after it in U, which reads z from that slice), so the
// chain warp's steps carry only the recurrence.  Pointers are restrict-qualified so
// later steps' shared-memory loads may be hoisted above this step's stores.
// L (KIND K_ITER): ops r, w, x, p: r_i = r - alpha w, x_i = x + alpha p (Alg. 1 lines
// 11-12 fused), y_i = r_i - sum_k l_ik y_k, ||r||^2;  K_PRO: ops rsrc; K_APPLY: ops in.
// U: ops y [, rdot]: z_i = (y_i - sum_k u_ik z_k) / u_ii, (rdot, z); K_PRO also p0 = z0.
template <int W, bool UPPER, int KIND, bool GEN, bool SPLIT, int CNT, int VB>
__device__ __forceinline__ void run_chunk(uint8_t* __restrict__ st, int cnt_rt, int64_t glo, int u0, int nv,
                                          bool rsrc_is_r, int use_x0, double* __restrict__ out,
                                          double* __restrict__ Er, double* __restrict__ Exp, double* __restrict__ Ep,
                                          double alpha, double& yprev, double& dot, const GenCtx& G) {
    constexpr int VROW = 128 + 32 * VB;                    // record bytes per entry column
    constexpr int RECB = VROW * W + (UPPER ? 256 : 0) + 16;
    constexpr size_t TRAILER = (size_t)VROW * W + (UPPER ? 256 : 0);
    const int lane = threadIdx.x & 31;
    const int cnt = CNT > 0 ? CNT : cnt_rt;
    double* __restrict__ sv = (double*)(st + (size_t)CC * RECB) + lane;
    const int64_t pbase = 32 * glo + lane;
#pragma unroll(CNT > 0 ? CNT : 1)
    for (int t = 0; t < (CNT > 0 ? CNT : cnt); ++t) {
        const int i = UPPER ? cnt - 1 - t : t;              // in-stage index (ascending global step)
        const uint8_t* __restrict__ R = st + (size_t)i * RECB;
        const int64_t pos = pbase + 32 * i;
        uint32_t tg[W];
        double v[W];
        lds_tags<W>(R + 4 * W * lane, tg);
        if constexpr (VB == 4) lds_vals_f32<W>(R + 128 * W + 4 * W * lane, v);
        else lds_vals<W>(R + 128 * W + 8 * W * lane, v);
        double acc, ri = 0.0, xn = 0.0, rdv = 0.0;
        if (!UPPER) {
            if (KIND == K_ITER && !SPLIT) {
                const double r0 = sv[i * 32], w0 = sv[CC * 32 + i * 32];
                const double x0 = sv[2 * CC * 32 + i * 32], p0 = sv[3 * CC * 32 + i * 32];
                ri = r0 - alpha * w0;
                xn = x0 + alpha * p0;
            } else {
                ri = sv[i * 32];
            }
            acc = ri;
        } else {
            acc = sv[i * 32];
            if (!SPLIT && nv > 1) rdv = sv[CC * 32 + i * 32];
        }
#pragma unroll
        for (int k = 0; k < W; ++k) {
            double d = __shfl_sync(0xffffffffu, yprev, (int)tg[k]);   // lane bits only (PREV)
            if (GEN && (tg[k] >> 29) != CT_PREV) {
                const uint32_t kind = tg[k] >> 29;
                if (kind == CT_HIST) {
                    d = G.hist[((u0 + t - (int)((tg[k] >> 5) & 255)) & (SPCG_CHAIN_HIST - 1)) * 32 + (tg[k] & 31)];
                } else if (kind == CT_GLOB) {
                    d = __ldcg(out + (tg[k] & 0x1fffffffu));
                } else if (kind == CT_EXT) {
                    const uint4 f = G.qb[((size_t)t * 2 + ((tg[k] >> 28) & 1)) * 32 + lane];
                    if (f.y == G.ep && f.w == G.ep)
                        d = __longlong_as_double((long long)(((unsigned long long)f.z << 32) | f.x));
                    else
                        d = ll_wait(G.mb + (tg[k] & 0x0fffffffu), G.ep, G.sc);
                } else {
                    d = ll_wait(G.mb + (tg[k] & 0x1fffffffu), G.ep, G.sc);
                }
            }
            acc = fma(-v[k], d, acc);
        }
        if (UPPER) {
            acc *= *(const double*)(R + VROW * W + 8 * lane);
            if (SPLIT) {
                sv[i * 32] = acc;                                  // z for the helper warp
                if (GEN) out[pos] = acc;                           // GLOB entries read z from global
            } else {
                if (nv > 1) dot = fma(rdv, acc, dot);              // (r, z)
                if (KIND == K_PRO) Ep[pos] = acc;                 // p0 = z0
                out[pos] = acc;
            }
        } else {
            if (!SPLIT) {
                dot = fma(ri, ri, dot);                           // ||r||^2
                if (KIND == K_ITER) {
                    Er[pos] = ri;
                    Exp[pos] = xn;
                } else if (KIND == K_PRO) {
                    if (!rsrc_is_r) Er[pos] = ri;
                    if (!use_x0) Exp[pos] = 0.0;
                }
            }
            out[pos] = acc;
        }
        if (GEN) {
            const uint32_t pubm = *(const uint32_t*)(R + TRAILER);
            if ((pubm >> lane) & 1u) ll_store(G.mb + pos, acc, G.ep);
            if (G.use_hist) {
                G.hist[((u0 + t) & (SPCG_CHAIN_HIST - 1)) * 32 + lane] = acc;
                __syncwarp();
            }
        }
        yprev = acc;
    }
}

// Helper-warp part of a chunk (SPLIT): L before the chain (r_i into the stage), U after
// it (z from the stage).
template <bool UPPER, int KIND>
__device__ __forceinline__ void help_chunk(uint8_t* __restrict__ st, int recb, int cnt, int64_t glo, int nv,
                                           bool rsrc_is_r, int use_x0, double* __restrict__ out,
                                           double* __restrict__ Er, double* __restrict__ Exp, double* __restrict__ Ep,
                                           double alpha, double& dot) {
    const int lane = threadIdx.x & 31;
    double* __restrict__ sv = (double*)(st + (size_t)CC * recb) + lane;
    const int64_t pbase = 32 * glo + lane;
    for (int i = 0; i < cnt; ++i) {
        const int64_t pos = pbase + 32 * i;
        if (!UPPER) {
            if (KIND == K_ITER) {
                const double r0 = sv[i * 32], w0 = sv[CC * 32 + i * 32];
                const double x0 = sv[2 * CC * 32 + i * 32], p0 = sv[3 * CC * 32 + i * 32];
                const double ri = r0 - alpha * w0;
                sv[i * 32] = ri;
                dot = fma(ri, ri, dot);                               // ||r||^2
                Er[pos] = ri;
                Exp[pos] = x0 + alpha * p0;
            } else {
                const double ri = sv[i * 32];
                dot = fma(ri, ri, dot);
                if (KIND == K_PRO) {
                    if (!rsrc_is_r) Er[pos] = ri;
                    if (!use_x0) Exp[pos] = 0.0;
                }
            }
        } else {
            const double z = sv[i * 32];
            if (nv > 1) dot = fma(sv[CC * 32 + i * 32], z, dot);      // (r, z)
            if (KIND == K_PRO) Ep[pos] = z;                          // p0 = z0
            out[pos] = z;
        }
    }
}

// One pass (L forward or U backward) of chain c: TMA-staged chunks of CC steps, NST
// stages in flight; cross-chain ready flags of chunk q+1 prefetched (cp.async) while
// chunk q runs.  ROLE 0: the chain warp alone; ROLE 1: the chain warp of a SPLIT pair;
// ROLE 2: its helper warp.  In a pair, the chain warp issues the first NST chunks, the
// last reader of a stage refills it (L: the chain warp, U: the helper), and hand[slot]
// carries the chunk from one to the other (L: helper -> chain, U: chain -> helper).
// cq: chunks consumed so far in the launch (mbarrier phase bookkeeping, identical in
// both warps of a pair).
template <int W, bool UPPER, int KIND, bool GEN, int ROLE, int VB>
__device__ __forceinline__ void chain_pass(const DevChain& D, const PassEnv& E, const WarpSmem& WS, unsigned& cq,
                                           int c, const PassOps& ops, double* out, double alpha, double& acc_dot,
                                           uint4* mb, unsigned ep) {
    constexpr int RECB = (128 + 32 * VB) * W + (UPPER ? 256 : 0) + 16;
    constexpr bool SPLIT = ROLE != 0;
    const int lane = threadIdx.x & 31;
    const int64_t s0 = D.chain_step[c], s1 = D.chain_step[c + 1];
    const int nst = (int)(s1 - s0);
    const int NST = D.nst;
    const uint8_t* recs = UPPER ? D.recU : D.recL;
    const uint32_t cfl = D.chain_flags[c];
    const bool use_ext = GEN && ROLE != 2 && (cfl & (UPPER ? CC_UEXT : CC_LEXT));
    const int nch = (nst + CC - 1) / CC;
    auto chunk_range = [&](int q, int64_t& glo, int& cnt) {
        cnt = min(CC, nst - q * CC);
        glo = UPPER ? (s1 - (int64_t)q * CC - cnt) : (s0 + (int64_t)q * CC);
    };
    // ring slots: chunk q of the pass sits in slot (cq + q) mod NST with mbarrier phase
    // ((cq + q) / NST) & 1; tracked incrementally (one division per pass, none per chunk)
    auto stage_at = [&](unsigned slot) { return WS.stages + (size_t)slot * D.stage_bytes; };
    auto next_slot = [&](unsigned& slot, unsigned& ph) {
        if (++slot == (unsigned)NST) { slot = 0; ph ^= 1u; }
    };
    auto issue = [&](int q, unsigned slot) {               // lane 0 only
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        uint8_t* st = stage_at(slot);
        const unsigned rb = (unsigned)(cnt * RECB), vb = (unsigned)cnt * 256u;
        mbar_arrive_tx(&WS.full[slot], rb + vb * ops.nv);
        bulk_g2s(st, recs + (size_t)glo * RECB, rb, &WS.full[slot]);
        uint8_t* vdst = st + (size_t)CC * RECB;
        for (int v = 0; v < ops.nv; ++v)
            bulk_g2s(vdst + (size_t)v * CC * 256, ops.v[v] + 32 * glo, vb, &WS.full[slot]);
    };
    auto wait_at = [&](uint64_t* bars, unsigned slot, unsigned ph) -> bool {
        return warp_ok(mbar_wait(&bars[slot], ph, E.sc));
    };
    // ready flags of chunk q's cross-chain entries -> extq[q & 1] (one cp.async each)
    auto prefetch_ext = [&](int q, unsigned slot) {
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        const uint8_t* st = stage_at(slot);
        uint4* qb = WS.extq + (size_t)(q & 1) * CC * 64;
        for (int i = 0; i < cnt; ++i) {
            const uint8_t* R = st + (size_t)i * RECB;
            const int t = UPPER ? cnt - 1 - i : i;          // pass-order index inside the chunk
            uint32_t tg[W];
            lds_tags<W>(R + 4 * W * lane, tg);
#pragma unroll
            for (int k = 0; k < W; ++k)
                if ((tg[k] >> 29) == CT_EXT)
                    cpa16(qb + ((size_t)t * 2 + ((tg[k] >> 28) & 1)) * 32 + lane, mb + (tg[k] & 0x0fffffffu));
        }
    };
    // Before a chunk runs, every prefetched flag that was still stale is polled again, all
    // of them together, until current: the chain then waits at most once per chunk (not
    // once per step), and the wait re-establishes a lag behind the producing chain of
    // about a chunk, so later prefetches find their values ready.
    auto settle_ext = [&](int q, unsigned slot) {
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        const uint8_t* st = stage_at(slot);
        uint4* qb = WS.extq + (size_t)(q & 1) * CC * 64;
        const long long t0 = clock64();
        for (;;) {
            bool stale = false;
            for (int i = 0; i < cnt; ++i) {
                const uint8_t* R = st + (size_t)i * RECB;
                const int t = UPPER ? cnt - 1 - i : i;
                uint32_t tg[W];
                lds_tags<W>(R + 4 * W * lane, tg);
#pragma unroll
                for (int k = 0; k < W; ++k)
                    if ((tg[k] >> 29) == CT_EXT) {
                        uint4* slotp = qb + ((size_t)t * 2 + ((tg[k] >> 28) & 1)) * 32 + lane;
                        uint4 f = *slotp;
                        if (f.y != ep || f.w != ep) {
                            asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                                         : "=r"(f.x), "=r"(f.y), "=r"(f.z), "=r"(f.w)
                                         : "l"(mb + (tg[k] & 0x0fffffffu))
                                         : "memory");
                            *slotp = f;
                            if (f.y != ep || f.w != ep) stale = true;
                        }
                    }
            }
            if (!__any_sync(0xffffffffu, stale)) break;
            if (__any_sync(0xffffffffu, ld_volatile_int(&E.sc->abort) != 0 || clock64() - t0 > SPIN_TIMEOUT_CYC)) {
                if (lane == 0) atomicExch(&E.sc->abort, 1);
                break;
            }
        }
    };
    const bool refill = ROLE == 0 || (ROLE == 1) == !UPPER;   // the last reader of a stage refills it

    long long t_pass = SPCG_CHAIN_PROF ? clock64() : 0, t_wait = 0, t_ext = 0;
    GenCtx G{WS.hist, WS.extq, mb, E.sc, ep, GEN && (cfl & (UPPER ? CC_UHIST : CC_LHIST)) != 0};
    const bool rsrc_is_r = ops.v[0] == E.r;
    const unsigned sl0 = cq % (unsigned)NST, ph0 = (cq / (unsigned)NST) & 1u;
    if (ROLE != 2 && lane == 0) {
        unsigned sl = sl0, ph = ph0;
        for (int q = 0; q < min(NST, nch); ++q) {
            issue(q, sl);
            next_slot(sl, ph);
        }
    }
    if (use_ext && nch > 0) {
        if (!wait_at(WS.full, sl0, ph0)) return;
        prefetch_ext(0, sl0);
    }
    if (GEN && ROLE != 2) cpa_commit();
    double yprev = 0.0;
    double dot = acc_dot;
    unsigned cs = sl0, cph = ph0;                        // slot / phase of chunk q
    for (int q = 0; q < nch; ++q) {
        int64_t glo;
        int cnt;
        chunk_range(q, glo, cnt);
        unsigned ns_ = cs, nph = cph;                    // slot / phase of chunk q + 1
        next_slot(ns_, nph);
        uint8_t* st = stage_at(cs);
        if (ROLE == 2) {
            // helper: L before the chain (wait for the data), U after it (wait for the chain)
            if (!wait_at(UPPER ? WS.hand : WS.full, cs, cph)) return;
            help_chunk<UPPER, KIND>(st, RECB, cnt, glo, ops.nv, rsrc_is_r, E.use_x0, out, E.r, E.xp, E.p, alpha, dot);
            __syncwarp();
            if (lane == 0) {
                if (!UPPER) mbar_arrive(&WS.hand[cs]);
                else if (q + NST < nch) issue(q + NST, cs);
            }
            cs = ns_;
            cph = nph;
            continue;
        }
        long long t0 = SPCG_CHAIN_PROF ? clock64() : 0;
        if (GEN) {
            if (use_ext && q + 1 < nch) {
                if (!wait_at(WS.full, ns_, nph)) return;
                prefetch_ext(q + 1, ns_);
            }
            cpa_commit();
            cpa_wait1();                                    // chunk q's flags landed
            G.qb = WS.extq + (size_t)(q & 1) * CC * 64;
            if (use_ext) settle_ext(q, cs);
        }
        if (SPCG_CHAIN_PROF) { t_ext += clock64() - t0; t0 = clock64(); }
        if (!wait_at(SPLIT && !UPPER ? WS.hand : WS.full, cs, cph)) return;
        if (SPCG_CHAIN_PROF) t_wait += clock64() - t0;
        // full chunks of narrow records run fully unrolled (immediate offsets, loads of
        // later steps hoisted); wide records and the ragged last chunk take the loop
        if (W <= 4 && cnt == CC)
            run_chunk<W, UPPER, KIND, GEN, SPLIT, (W <= 4 ? CC : 0), VB>(st, cnt, glo, q * CC, ops.nv, rsrc_is_r,
                                                                         E.use_x0, out, E.r, E.xp, E.p, alpha, yprev,
                                                                         dot, G);
        else
            run_chunk<W, UPPER, KIND, GEN, SPLIT, 0, VB>(st, cnt, glo, q * CC, ops.nv, rsrc_is_r, E.use_x0, out, E.r,
                                                         E.xp, E.p, alpha, yprev, dot, G);
        __syncwarp();
        if (lane == 0) {
            if (SPLIT && UPPER) mbar_arrive(&WS.hand[cs]);
            if (refill && q + NST < nch) issue(q + NST, cs);
        }
        cs = ns_;
        cph = nph;
    }
    if (GEN && ROLE != 2) cpa_wait0();
    cq += (unsigned)nch;
    acc_dot = dot;
    if (SPCG_CHAIN_PROF && ROLE != 2 && lane == 0 && g_chain_prof) {
        unsigned long long* g = g_chain_prof + (UPPER ? 8 : 0);
        atomicAdd(g + 0, (unsigned long long)(clock64() - t_pass));
        atomicAdd(g + 1, (unsigned long long)t_wait);
        atomicAdd(g + 2, (unsigned long long)t_ext);
        atomicAdd(g + 3, (unsigned long long)nst);
        atomicAdd(g + 4, (unsigned long long)nch);
        atomicAdd(g + 5, (unsigned long long)GEN);
        atomicAdd(g + 6, 1ull);
    }
}

// dispatch on the role, the record width (a power of two) and on whether the pass
// uses anything but shuffles
template <bool UPPER, int KIND>
__device__ __forceinline__ void chain_pass_any(const DevChain& D, const PassEnv& E, const WarpSmem& WS, unsigned& cq,
                                               int c, int role, const PassOps& ops, double* out, double alpha,
                                               double& acc_dot, uint4* mb, unsigned ep) {
    const uint32_t cfl = D.chain_flags[c];
    const bool gen = UPPER ? (cfl & (CC_UHIST | CC_UEXT | CC_UGLOB | CC_UPUB)) != 0
                           : (cfl & (CC_LHIST | CC_LEXT | CC_LGLOB | CC_LPUB)) != 0;
    const int W = UPPER ? D.W_U : D.W_L;
#define SPCG_CP(WW, GG, RR, VV) chain_pass<WW, UPPER, KIND, GG, RR, VV>(D, E, WS, cq, c, ops, out, alpha, acc_dot, mb, ep)
#define SPCG_CPW(GG, RR)                              \
    if (D.vb == 4) {                                  \
        switch (W) {                                  \
            case 1: SPCG_CP(1, GG, RR, 4); break;     \
            case 2: SPCG_CP(2, GG, RR, 4); break;     \
            default: SPCG_CP(4, GG, RR, 4); break;    \
        }                                             \
    } else {                                          \
        switch (W) {                                  \
            case 1: SPCG_CP(1, GG, RR, 8); break;     \
            case 2: SPCG_CP(2, GG, RR, 8); break;     \
            case 4: SPCG_CP(4, GG, RR, 8); break;     \
            case 8: SPCG_CP(8, GG, RR, 8); break;     \
            default: SPCG_CP(16, GG, RR, 8); break;   \
        }                                             \
    }
    if (role == 2) {      // the helper (the record width fixes the stage layout it reads)
        SPCG_CPW(false, 2)
    } else if (role == 1) {
        if (gen) { SPCG_CPW(true, 1) } else { SPCG_CPW(false, 1) }
    } else {
        if (gen) { SPCG_CPW(true, 0) } else { SPCG_CPW(false, 0) }
    }
#undef SPCG_CPW
#undef SPCG_CP
}

// z = U^-1 L^-1 r for every chain of this CTA, the fused vector work of the kind;
// rr / rz: this thread's partial sums.  Warps 0..per_cta-1 walk the chains; when the
// CTA has at most NWARP/2 chains, warp per_cta + i is the helper of chain warp i (the
// vector work off the chain).  Dp: the chain layout, copied to shared memory by the
// kernel.  One instantiation per kind (noinline: the kernel body stays small).
template <int KIND>
__device__ __noinline__ void tri_chains(const DevChain* Dp, PassEnv E, uint8_t* dyn, unsigned* cq,
                                        const double* rsrc, const double* w, double* y, double* z,
                                        const double* rdot, uint4* mbL, uint4* mbU, unsigned ep, double alpha,
                                        bool lower, bool upper, double* rr, double* rz) {
    const DevChain& D = *Dp;
    const int warp = threadIdx.x >> 5;
    const bool split = D.per_cta <= NWARP / 2;
    const int sw = (split && warp >= D.per_cta) ? warp - D.per_cta : warp;   // chain slot of this warp
    const int role = !split ? 0 : (warp < D.per_cta ? 1 : 2);
    const int c = blockIdx.x + sw * gridDim.x;
    if (sw >= D.per_cta || c >= D.nchains) return;
    const WarpSmem WS = warp_smem(D, dyn, sw);
    unsigned q = *cq;
    double a = *rr, b = *rz;
    if (lower) {
        PassOps o{};
        if (KIND == K_ITER) {
            o.v[0] = E.r; o.v[1] = w; o.v[2] = E.xp; o.v[3] = E.p; o.nv = 4;
        } else {
            o.v[0] = rsrc; o.nv = 1;
        }
        chain_pass_any<false, KIND>(D, E, WS, q, c, role, o, y, alpha, a, mbL, ep);
        // the U pass reads this chain's y (and r) through TMA: order the generic stores first
        fence_proxy_async_global();
        if (split) named_bar_sync(1 + sw, 64);     // the pair: both warps' L stores precede U's loads
        else __syncwarp();
    }
    if (upper) {
        PassOps o{};
        o.v[0] = y;
        o.nv = 1;
        if (rdot) { o.v[1] = rdot; o.nv = 2; }
        chain_pass_any<true, KIND == K_ITER ? K_APPLY : KIND>(D, E, WS, q, c, role, o, z, 0.0, b, mbU, ep);
    }
    *cq = q;
    *rr = a;
    *rz = b;
}

// w = A p over positions (SELL-32, one slice per step; padding rows have zero entries,
// so no row bound) and the partial (p, w).  A warp takes CSU consecutive slices and
// issues ALL their index/value loads (up to CSK entries per row) at once, then every
// gather, then the FMA chains (entries in CSR order, as the definition): two memory
// round trips per CSU slices; the next group's slice offsets are loaded one group ahead.
constexpr int CSU = 4, CSK = 8;
__device__ void chain_spmv(const DevA& A, const double* __restrict__ pin, double* __restrict__ wout, double& pw) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t ns = A.nslices;
    const int64_t stride = (int64_t)gridDim.x * NWARP * CSU;
    int64_t s0 = ((int64_t)blockIdx.x * NWARP + warp) * CSU;
    int64_t eo = (s0 < ns && lane <= CSU && s0 + lane <= ns) ? __ldg(A.eoff + s0 + lane) : 0;
    for (; s0 < ns; s0 += stride) {
        int64_t e[CSU];
        int wd[CSU];
        int wmax = 0;
#pragma unroll
        for (int u = 0; u < CSU; ++u) {
            e[u] = __shfl_sync(0xffffffffu, eo, u);
            const int64_t e1 = __shfl_sync(0xffffffffu, eo, u + 1);
            wd[u] = (s0 + u < ns) ? (int)(e1 - e[u]) : 0;
            wmax = max(wmax, wd[u]);
        }
        const int64_t sn = s0 + stride;                       // next group's offsets, one round trip ahead
        eo = (sn < ns && lane <= CSU && sn + lane <= ns) ? __ldg(A.eoff + sn + lane) : 0;
        double acc[CSU];
#pragma unroll
        for (int u = 0; u < CSU; ++u) acc[u] = 0.0;
        for (int kb = 0; kb < wmax; kb += CSK) {
            int c[CSU][CSK];
            double v[CSU][CSK], g[CSU][CSK];
#pragma unroll
            for (int u = 0; u < CSU; ++u)
#pragma unroll
                for (int k = 0; k < CSK; ++k) {
                    const bool on = kb + k < wd[u];
                    const int64_t idx = (e[u] + kb + k) * 32 + lane;
                    c[u][k] = on ? __ldg(A.col + idx) : 0;
                    v[u][k] = on ? __ldg(A.val + idx) : 0.0;
                }
#pragma unroll
            for (int u = 0; u < CSU; ++u)
#pragma unroll
                for (int k = 0; k < CSK; ++k) g[u][k] = (kb + k < wd[u]) ? pin[c[u][k]] : 0.0;
#pragma unroll
            for (int u = 0; u < CSU; ++u)
#pragma unroll
                for (int k = 0; k < CSK; ++k)
                    if (kb + k < wd[u]) acc[u] = fma(v[u][k], g[u][k], acc[u]);
        }
#pragma unroll
        for (int u = 0; u < CSU; ++u)
            if (s0 + u < ns) {
                const int64_t row = (s0 + u) * 32 + lane;
                wout[row] = acc[u];
                pw = fma(pin[row], acc[u], pw);
            }
    }
}

// The same SpMV with the matrix streamed by TMA (uniform slice width WA): warp gw of
// the grid takes the contiguous slice range [gw ns / NW, (gw+1) ns / NW); lane 0 keeps
// sp_nst stages of SPCG_SPMV_G slices (column indices, then values: two bulk copies)
// in flight in the warp's ring; the lanes gather p for every entry of a stage at once
// and accumulate in CSR order.  Only the gathers (L1/L2, neighbours in position order)
// remain on the warp's critical path.  spq: stages this warp consumed (mbarrier phases).
template <int WA>
__device__ __forceinline__ void spmv_tma_stage(const int32_t* __restrict__ cs, const double* __restrict__ vs,
                                               int g, int64_t s, const double* __restrict__ pin,
                                               double* __restrict__ wout, double& pw) {
    constexpr int G = SPCG_SPMV_G;
    const int lane = threadIdx.x & 31;
    double gv[G][WA], vv[G][WA];
#pragma unroll
    for (int u = 0; u < G; ++u)
#pragma unroll
        for (int k = 0; k < WA; ++k) {
            const int c = u < g ? cs[(u * WA + k) * 32 + lane] : 0;
            vv[u][k] = u < g ? vs[(u * WA + k) * 32 + lane] : 0.0;
            gv[u][k] = u < g ? pin[c] : 0.0;
        }
#pragma unroll
    for (int u = 0; u < G; ++u) {
        if (u >= g) break;
        double acc = 0.0;
#pragma unroll
        for (int k = 0; k < WA; ++k) acc = fma(vv[u][k], gv[u][k], acc);
        const int64_t row = (s + u) * 32 + lane;
        wout[row] = acc;
        pw = fma(pin[row], acc, pw);
    }
}

// Two stages at once: every gather of both is issued before the first is used (twice
// the loads in flight per warp: the SpMV is gather-latency bound); the
// values are re-read from shared memory at the FMA (registers for the gathers only).
// Same accumulation order as two calls of spmv_tma_stage: bitwise the same w and (p, w).
template <int WA>
__device__ __forceinline__ void spmv_tma_pair(const int32_t* __restrict__ cs0, const double* __restrict__ vs0, int g0,
                                              int64_t s0, const int32_t* __restrict__ cs1,
                                              const double* __restrict__ vs1, int g1, int64_t s1,
                                              const double* __restrict__ pin, double* __restrict__ wout, double& pw) {
    constexpr int G = SPCG_SPMV_G;
    const int lane = threadIdx.x & 31;
    double gv0[G][WA], gv1[G][WA];
#pragma unroll
    for (int u = 0; u < G; ++u)
#pragma unroll
        for (int k = 0; k < WA; ++k) {
            const int c0 = u < g0 ? cs0[(u * WA + k) * 32 + lane] : 0;
            const int c1 = u < g1 ? cs1[(u * WA + k) * 32 + lane] : 0;
            gv0[u][k] = u < g0 ? pin[c0] : 0.0;
            gv1[u][k] = u < g1 ? pin[c1] : 0.0;
        }
#pragma unroll
    for (int u = 0; u < G; ++u) {
        if (u >= g0) break;
        double acc = 0.0;
#pragma unroll
        for (int k = 0; k < WA; ++k) acc = fma(vs0[(u * WA + k) * 32 + lane], gv0[u][k], acc);
        const int64_t row = (s0 + u) * 32 + lane;
        wout[row] = acc;
        pw = fma(pin[row], acc, pw);
    }
#pragma unroll
    for (int u = 0; u < G; ++u) {
        if (u >= g1) break;
        double acc = 0.0;
#pragma unroll
        for (int k = 0; k < WA; ++k) acc = fma(vs1[(u * WA + k) * 32 + lane], gv1[u][k], acc);
        const int64_t row = (s1 + u) * 32 + lane;
        wout[row] = acc;
        pw = fma(pin[row], acc, pw);
    }
}

__device__ void chain_spmv_tma(const DevChain& D, const DevA& A, uint8_t* dyn, uint64_t* bars, unsigned& spq,
                               const double* __restrict__ pin, double* __restrict__ wout, double& pw, Scal* sc) {
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
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic reads of this smem done
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
    long long t_all = SPCG_CHAIN_PROF ? clock64() : 0, t_wait = 0;
    if (lane == 0)
        for (int j = 0; j < min(NS, nst); ++j) issue(j);
    for (int j = 0; j < nst;) {
        // narrow slices (WA <= 5: the registers of two stages' gathers fit) go two stages
        // at a time
        const bool two = WA <= 5 && j + 1 < nst;
        const unsigned u = spq + j;
        const long long tw = SPCG_CHAIN_PROF ? clock64() : 0;
        if (!warp_ok(mbar_wait(&bar[u % NS], (u / NS) & 1, sc))) return;
        if (two && !warp_ok(mbar_wait(&bar[(u + 1) % NS], ((u + 1) / NS) & 1, sc))) return;
        if (SPCG_CHAIN_PROF) t_wait += clock64() - tw;
        const uint8_t* st = ring + (size_t)(u % NS) * D.sp_stage_bytes;
        const int32_t* cs = (const int32_t*)st;
        const double* vs = (const double*)(st + (size_t)G * WA * 128);
        const int64_t s = ((int64_t)j * NW + gw) * G;
        const int g = (int)(ns - s < (int64_t)G ? ns - s : (int64_t)G);
        if (two) {
            const uint8_t* st1 = ring + (size_t)((u + 1) % NS) * D.sp_stage_bytes;
            const int32_t* cs1 = (const int32_t*)st1;
            const double* vs1 = (const double*)(st1 + (size_t)G * WA * 128);
            const int64_t s1 = ((int64_t)(j + 1) * NW + gw) * G;
            const int g1 = (int)(ns - s1 < (int64_t)G ? ns - s1 : (int64_t)G);
            switch (WA) {
                case 3: spmv_tma_pair<3>(cs, vs, g, s, cs1, vs1, g1, s1, pin, wout, pw); break;
                case 4: spmv_tma_pair<4>(cs, vs, g, s, cs1, vs1, g1, s1, pin, wout, pw); break;
                default: spmv_tma_pair<5>(cs, vs, g, s, cs1, vs1, g1, s1, pin, wout, pw); break;
            }
        } else {
            switch (WA) {
                case 3: spmv_tma_stage<3>(cs, vs, g, s, pin, wout, pw); break;
                case 4: spmv_tma_stage<4>(cs, vs, g, s, pin, wout, pw); break;
                case 5: spmv_tma_stage<5>(cs, vs, g, s, pin, wout, pw); break;
                case 6: spmv_tma_stage<6>(cs, vs, g, s, pin, wout, pw); break;
                case 7: spmv_tma_stage<7>(cs, vs, g, s, pin, wout, pw); break;
                default: spmv_tma_stage<8>(cs, vs, g, s, pin, wout, pw); break;
            }
        }
        __syncwarp();
        if (lane == 0) {
            if (j + NS < nst) issue(j + NS);
            if (two && j + 1 + NS < nst) issue(j + 1 + NS);
        }
        j += two ? 2 : 1;
    }
    spq += (unsigned)nst;
    if (SPCG_CHAIN_PROF && lane == 0 && g_chain_prof) {
        atomicAdd(g_chain_prof + 22, (unsigned long long)t_wait);
        atomicAdd(g_chain_prof + 23, (unsigned long long)(clock64() - t_all));
    }
}

// the SpMV of the iteration: TMA-streamed for uniform widths 3..8, the register path otherwise
__device__ __forceinline__ void chain_spmv_any(const DevChain& D, const DevA& A, uint8_t* dyn, uint64_t* bars,
                                               unsigned& spq, const double* pin, double* wout, double& pw, Scal* sc) {
    if (D.sp_nst >= 2 && D.WA >= 3 && D.WA <= 8) chain_spmv_tma(D, A, dyn, bars, spq, pin, wout, pw, sc);
    else chain_spmv(A, pin, wout, pw);
}

// p = z + beta p (Alg. 1 line 15) over positions: 16-byte accesses, four in flight per
// thread and array (npos is a multiple of 32)
__device__ void chain_pupdate(double* __restrict__ p, const double* __restrict__ z, double beta, int64_t npos) {
    const int64_t n2 = npos / 2;
    const int64_t stride = (int64_t)gridDim.x * BLOCK;
    double2* p2 = (double2*)p;
    const double2* z2 = (const double2*)z;
    for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < n2; i += 4 * stride) {
        double2 a[4], b[4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (i + u * stride < n2) {
                a[u] = p2[i + u * stride];
                b[u] = __ldcg(z2 + i + u * stride);
            }
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (i + u * stride < n2) p2[i + u * stride] = make_double2(fma(beta, a[u].x, b[u].x), fma(beta, a[u].y, b[u].y));
    }
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
    __shared__ __align__(8) uint64_t spbar[NWARP * 4];   // SpMV stage barriers, 4 per warp
    const DevChain& D = P.CH;
    unsigned gen = 0;
    unsigned cq = 0;
    if (threadIdx.x == 0) {
        sD = P.CH;
        // mbarriers of every solver warp of this CTA
        for (int sw = 0; sw < D.per_cta; ++sw) {
            const WarpSmem W = warp_smem(D, dynw, sw);
            for (int s = 0; s < D.nst; ++s) {
                mbar_init(&W.full[s], 1);
                mbar_init(&W.hand[s], 1);
            }
        }
        for (int i = 0; i < NWARP * 4; ++i) mbar_init(&spbar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const PassEnv E{P.r, P.p, D.xp, P.sc, P.use_x0};
    unsigned spq = 0;
    const int64_t npos = D.npos;

    if (P.mode != M_SOLVE) {
        double a = 0.0, b = 0.0;
        if (P.mode == M_SPMV) {
            gather(P, P.in, D.t1);
            grid_sync(P.sc, gen);
            chain_spmv_any(sD, P.A, dynw, spbar, spq, D.t1, P.w, a, P.sc);
            grid_sync(P.sc, gen);
            scatter(P, P.w, P.out);
        } else if (P.mode == M_LOWER) {
            gather(P, P.in, D.t1);
            sync_for_tma(P, gen);
            tri_chains<K_APPLY>(&sD, E, dynw, &cq, D.t1, P.w, P.y, P.z, nullptr, P.mbL, P.mbU, P.epoch, 0.0, true, false,
                       &a, &b);
            grid_sync(P.sc, gen);
            scatter(P, P.y, P.out);
        } else if (P.mode == M_UPPER) {
            gather(P, P.in, P.y);
            if (P.aux) gather(P, P.aux, D.t1);
            sync_for_tma(P, gen);
            tri_chains<K_APPLY>(&sD, E, dynw, &cq, nullptr, P.w, P.y, P.z, P.aux ? D.t1 : nullptr, P.mbL, P.mbU, P.epoch,
                       0.0, false, true, &a, &b);
            grid_sync(P.sc, gen);
            scatter(P, P.z, P.out);
        } else {
            gather(P, P.in, D.t1);
            sync_for_tma(P, gen);
            tri_chains<K_APPLY>(&sD, E, dynw, &cq, D.t1, P.w, P.y, P.z, D.t1, P.mbL, P.mbU, P.epoch, 0.0, true, true, &a,
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
        chain_spmv_any(sD, P.A, dynw, spbar, spq, D.xp, P.w, dummy, P.sc);
        grid_sync(P.sc, gen);
        const int64_t stride = (int64_t)gridDim.x * BLOCK;
        for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < npos; i += stride) P.r[i] = D.bp[i] - P.w[i];
        r_src = P.r;
    }
    sync_for_tma(P, gen);
    unsigned app = 0;
    double rr_l = 0.0, rz_l = 0.0;
    tri_chains<K_PRO>(&sD, E, dynw, &cq, r_src, P.w, P.y, P.z, P.r, P.mbL, P.mbU, P.epoch + app, 0.0, true, true, &rr_l,
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
        long long tph = SPCG_CHAIN_PROF ? clock64() : 0;
        double pw = 0.0;
        chain_spmv_any(sD, P.A, dynw, spbar, spq, P.p, P.w, pw, P.sc);
        prof_phase(0, tph);
        block_partials(pw, 0.0, P.partials, 2, -1);
        sync_for_tma(P, gen);
        prof_phase(1, tph);
        double sigma, unused;
        global_sums(P.partials, 2, -1, sigma, unused);
        if (!(sigma > 0.0) || !isfinite(sigma) || !isfinite(rho)) { status = SPCG_ERR_BREAKDOWN; break; }
        const double alpha = rho / sigma;
        // lines 11-13 (+ ||r||^2, (r, z))
        rr_l = 0.0;
        rz_l = 0.0;
        tri_chains<K_ITER>(&sD, E, dynw, &cq, P.r, P.w, P.y, P.z, P.r, P.mbL, P.mbU, P.epoch + app, alpha, true, true,
                   &rr_l, &rz_l);
        ++app;
        prof_phase(2, tph);
        block_partials(rz_l, rr_l, P.partials, 0, 1);
        grid_sync(P.sc, gen);
        prof_phase(3, tph);
        double rho_new;
        global_sums(P.partials, 0, 1, rho_new, rr);
        // lines 14-15
        const double beta = rho_new / rho;
        rho = rho_new;
        chain_pupdate(P.p, P.z, beta, npos);
        prof_phase(4, tph);
        sync_for_tma(P, gen);
        prof_phase(5, tph);
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

// debug (SPCG_CHAIN_PROF builds): first call installs the counters, later calls read and reset
extern "C" int spcg_dbg_chain_prof(unsigned long long* out) {
    static unsigned long long* d = nullptr;
    if (!d) {
        if (cudaMalloc(&d, 24 * 8) != cudaSuccess) return -1;
        cudaMemset(d, 0, 24 * 8);
        cudaMemcpyToSymbol(g_chain_prof, &d, sizeof(d));
        return 0;
    }
    cudaMemcpy(out, d, 24 * 8, cudaMemcpyDeviceToHost);
    cudaMemset(d, 0, 24 * 8);
    return 1;
}
