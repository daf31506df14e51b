// kernels.cu — the iterative phase of SPCG on sm_100a (B200).
//
// One persistent cooperative kernel runs the whole of Algorithm 1
// (P:L141-173): prologue (lines 1-4), then per iteration the stopping test
// (lines 5-8), w = A p with the ORIGINAL A (line 9) fused with
// (p,w), alpha (line 10), the x / r updates (lines 11-12) fused into the
// forward triangular solve together with ||r||^2, z = U^-1 L^-1 r (line 13,
// P:L198-209) with (r,z) fused into the backward solve, beta and the
// direction update (lines 14-15).  All scalars are computed on the device by
// every CTA from the same per-CTA partials in the same order, so they are
// bitwise identical everywhere and from run to run (deterministic k).
//
// Triangular solves are executed by one of three wavefront executors (§2,
// P:L263-283):
//   LEVEL     rows of one wavefront spread over all warps, a grid barrier
//             between wavefronts (the level-scheduled design of [36]);
//   SYNCFREE  rows in wavefront order, round-robin over all warps; every
//             value is published with an epoch-stamped ready flag and
//             consumers spin on the flags of their dependencies ([34, 41]);
//   CHUNKED   each CTA owns a contiguous block of rows and walks its own
//             wavefronts with CTA barriers; dependencies inside the block come
//             from a shared-memory ring, the others from ready flags.
// Ready flags use the "LL" layout {lo32, epoch, hi32, epoch} written and read
// as one 16-byte access: each 8-byte half is single-copy atomic, so a reader
// that sees both epochs current holds the whole value — no fence, no reset.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "internal.h"

using namespace spcg;

#include "dev_common.cuh"

namespace {

constexpr int SF_PF = 4;               // SYNCFREE: dependencies per row read in one batch
// One slice (<= 32 rows of one wavefront) of a triangular solve, thread per row.
// Lower (UPPER=false): y_i = r_i - sum_j l_ij y_j   (unit diagonal)
// Upper (UPPER=true):  z_i = (y_i - sum_j u_ij z_j) / u_ii
template <int STRAT, bool UPPER>
__device__ __forceinline__ void tri_slice(const Params& P, const DevTri& T, int64_t s, int kind,
                                          const double* in, double* out, const double* rdot,
                                          uint4* mb, unsigned ep, double alpha, double& acc_dot,
                                          double* ring, int64_t pb, int ringmask) {
    const int lane = threadIdx.x & 31;
    const int64_t slot = s * 32 + lane;
    const int row = __ldg(T.rows + slot);
    if (row >= 0) {
        const int len = __ldg(T.rlen + slot);
        const int64_t e0 = __ldg(T.eoff + s);
        const int32_t* sp = T.src + e0 * 32 + lane;
        const double* vp = T.val + e0 * 32 + lane;
        double acc;
        if (!UPPER) {
            double ri;
            if (kind == K_ITER) {                       // Alg. 1 lines 11-12 fused
                ri = P.r[row] - alpha * P.w[row];
                P.r[row] = ri;
                P.x[row] = P.x[row] + alpha * P.p[row];
            } else {
                ri = in[row];
                if (kind == K_PRO) {
                    if (in != P.r) P.r[row] = ri;
                    if (!P.use_x0) P.x[row] = 0.0;
                }
            }
            acc_dot = fma(ri, ri, acc_dot);            // ||r||^2
            acc = ri;
        } else {
            acc = in[row];
        }
        int k0 = 0;
        if (STRAT == ST_SYNCFREE) {
            // all (index, value) pairs of the row first, then every flag read in one batch:
            // one memory round trip per slice instead of one per dependency
            int sx[SF_PF];
            double vv[SF_PF];
            uint4 f[SF_PF];
#pragma unroll
            for (int k = 0; k < SF_PF; ++k) {
                sx[k] = k < len ? __ldg(sp + 32 * k) : -1;
                vv[k] = k < len ? __ldg(vp + 32 * k) : 0.0;
            }
#pragma unroll
            for (int k = 0; k < SF_PF; ++k)
                if (k < len) {
                    const uint4* a = mb + (-sx[k] - 1);
                    asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                                 : "=r"(f[k].x), "=r"(f[k].y), "=r"(f[k].z), "=r"(f[k].w)
                                 : "l"(a)
                                 : "memory");
                }
#pragma unroll
            for (int k = 0; k < SF_PF; ++k)
                if (k < len) {
                    const double d = (f[k].y == ep && f[k].w == ep)
                                         ? __longlong_as_double((long long)(((unsigned long long)f[k].z << 32) | f[k].x))
                                         : ll_wait(mb + (-sx[k] - 1), ep, P.sc);
                    acc = fma(-vv[k], d, acc);
                }
            k0 = SF_PF;
        }
        for (int k = k0; k < len; ++k) {
            const int sidx = __ldg(sp + 32 * k);
            const double v = __ldg(vp + 32 * k);
            double d;
            if (STRAT == ST_CHUNKED && sidx >= 0) d = ring[sidx];
            else if (STRAT == ST_LEVEL) d = out[-sidx - 1];
            else d = ll_wait(mb + (-sidx - 1), ep, P.sc);
            acc = fma(-v, d, acc);
        }
        if (UPPER) {
            acc *= __ldg(T.dinv + slot);
            if (rdot) acc_dot = fma(rdot[row], acc, acc_dot);   // (r, z)
            if (kind == K_PRO) P.p[row] = acc;                   // p_0 = z_0
        }
        out[row] = acc;
        if (STRAT == ST_CHUNKED) ring[(row - pb) & ringmask] = acc;
        if (STRAT != ST_LEVEL && __ldg(T.publish + slot)) ll_store(mb + row, acc, ep);
    }
    // Keep the warp in lockstep slice by slice: with independent thread scheduling,
    // lanes that finished (or padding lanes) could otherwise run ahead into the
    // warp's next slice and spin there on rows whose producers are the lanes
    // still in this slice — the spinners can starve them (observed deadlock).
    __syncwarp();
}

// LEVEL executor, wide rows (ILU(K) fill): one warp per row of the wavefront, the
// lanes stride the row's dependencies (coalesced CSR reads, 2 entries per lane
// prefetched before the previous wavefront's barrier completes), a fixed-order
// shuffle reduction, lane 0 finishes the row (fused x/r update and ||r||^2 for L;
// 1/u_ii, (r,z) and p0 for U).
constexpr int WPF = 2;                 // entries per lane prefetched across the barrier
template <bool UPPER>
__device__ void tri_level_wide(const Params& P, const DevTri& T, int kind, const double* in, double* out,
                               const double* rdot, double alpha, double& acc_dot, unsigned& gen) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t W = (int64_t)gridDim.x * NWARP;
    const int64_t gw = (int64_t)blockIdx.x * NWARP + warp;
    // prefetch state for the first position of this warp in level g
    int64_t q = -1, e0 = 0, e1 = 0;
    int row = -1;
    int cpf[WPF];
    double vpf[WPF];
    double r0 = 0.0, w0 = 0.0, x0 = 0.0, p0v = 0.0, a0 = 0.0, dv = 1.0;
    // the row's own operands (lane 0): none of them is written by this solve's
    // wavefronts, so they are loaded before the barrier that precedes their use
    auto own = [&]() {
        if (lane == 0) {
            if (!UPPER) {
                if (kind == K_ITER) { r0 = __ldcg(P.r + row); w0 = __ldcg(P.w + row); x0 = __ldcg(P.x + row); p0v = __ldcg(P.p + row); }
                else r0 = __ldcg(in + row);
            } else {
                r0 = __ldcg(in + row);
                if (rdot) a0 = __ldcg(rdot + row);
                dv = __ldg(T.wdinv + q);
            }
        }
    };
    auto prefetch = [&](int g) {
        const int64_t p0 = __ldg(T.wgptr + g), p1 = __ldg(T.wgptr + g + 1);
        q = p0 + gw < p1 ? p0 + gw : -1;
        if (q >= 0) {
            row = __ldg(T.wrow + q);
            e0 = __ldg(T.wptr + q);
            e1 = __ldg(T.wptr + q + 1);
#pragma unroll
            for (int u = 0; u < WPF; ++u) {
                const int64_t e = e0 + lane + 32 * u;
                cpf[u] = e < e1 ? __ldg(T.wcol + e) : -1;
                vpf[u] = e < e1 ? __ldg(T.wval + e) : 0.0;
            }
            own();
        }
    };
    if (T.ngroups > 0) prefetch(0);
    for (int g = 0; g < T.ngroups; ++g) {
        const int64_t p1 = __ldg(T.wgptr + g + 1);
        bool first = true;
        for (; q >= 0 && q < p1; q += W) {
            if (!first) {
                row = __ldg(T.wrow + q);
                e0 = __ldg(T.wptr + q);
                e1 = __ldg(T.wptr + q + 1);
#pragma unroll
                for (int u = 0; u < WPF; ++u) {
                    const int64_t e = e0 + lane + 32 * u;
                    cpf[u] = e < e1 ? __ldg(T.wcol + e) : -1;
                    vpf[u] = e < e1 ? __ldg(T.wval + e) : 0.0;
                }
                own();
            }
            first = false;
            double part = 0.0;
#pragma unroll
            for (int u = 0; u < WPF; ++u)
                if (cpf[u] >= 0) part = fma(vpf[u], __ldcg(out + cpf[u]), part);
            for (int64_t e = e0 + lane + 32 * WPF; e < e1; e += 32) part = fma(__ldg(T.wval + e), __ldcg(out + __ldg(T.wcol + e)), part);
            part = warp_sum(part);
            if (lane == 0) {
                double acc;
                if (!UPPER) {
                    double ri = r0;
                    if (kind == K_ITER) {
                        ri = r0 - alpha * w0;
                        P.r[row] = ri;
                        P.x[row] = x0 + alpha * p0v;
                    } else if (kind == K_PRO) {
                        if (in != P.r) P.r[row] = ri;
                        if (!P.use_x0) P.x[row] = 0.0;
                    }
                    acc_dot = fma(ri, ri, acc_dot);
                    acc = ri - part;
                } else {
                    acc = (r0 - part) * dv;
                    if (rdot) acc_dot = fma(a0, acc, acc_dot);
                    if (kind == K_PRO) P.p[row] = acc;
                }
                out[row] = acc;
            }
        }
        if (g + 1 < T.ngroups) prefetch(g + 1);     // independent of the barrier
        grid_sync(P.sc, gen);
    }
}

// SYNCFREE executor, wide rows: the warp-per-row CSR of tri_level_wide, but no
// barriers — rows in execution (level) order are dealt round-robin to all warps
// of the grid; each lane waits on the LL ready flags of its dependencies, the
// warp reduces, lane 0 publishes the row's value with its flag.  Deadlock-free
// because every dependency has a lower position and all warps are co-resident.
template <bool UPPER>
__device__ void tri_syncfree_wide(const Params& P, const DevTri& T, int kind, const double* in, double* out,
                                  const double* rdot, uint4* mb, unsigned ep, double alpha, double& acc_dot) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t W = (int64_t)gridDim.x * NWARP;
    // the warp's NEXT row (q + W) is loaded while it waits on the flags of the current
    // one: index/value pairs and the row's own operands do not depend on any flag
    struct RowOps {
        int row;
        int64_t e0, e1;
        int c[WPF];
        double v[WPF];
        double r0, w0, x0, p0v, a0, dv;
    };
    auto load = [&](int64_t q, RowOps& o) {
        o.row = __ldg(T.wrow + q);
        o.e0 = __ldg(T.wptr + q);
        o.e1 = __ldg(T.wptr + q + 1);
        o.r0 = o.w0 = o.x0 = o.p0v = o.a0 = 0.0;
        o.dv = 1.0;
        if (lane == 0) {
            if (!UPPER) {
                if (kind == K_ITER) {
                    o.r0 = __ldcg(P.r + o.row); o.w0 = __ldcg(P.w + o.row);
                    o.x0 = __ldcg(P.x + o.row); o.p0v = __ldcg(P.p + o.row);
                } else {
                    o.r0 = __ldcg(in + o.row);
                }
            } else {
                o.r0 = __ldcg(in + o.row);
                if (rdot) o.a0 = __ldcg(rdot + o.row);
                o.dv = __ldg(T.wdinv + q);
            }
        }
#pragma unroll
        for (int u = 0; u < WPF; ++u) {
            const int64_t e = o.e0 + lane + 32 * u;
            o.c[u] = e < o.e1 ? __ldg(T.wcol + e) : -1;
            o.v[u] = e < o.e1 ? __ldg(T.wval + e) : 0.0;
        }
    };
    RowOps nxt;
    int64_t q = (int64_t)blockIdx.x * NWARP + warp;
    if (q < P.n) load(q, nxt);
    for (; q < P.n; q += W) {
        const RowOps cur = nxt;
        if (q + W < P.n) load(q + W, nxt);
        const int row = cur.row;
        const int64_t e0 = cur.e0, e1 = cur.e1;
        const double r0 = cur.r0, w0 = cur.w0, x0 = cur.x0, p0v = cur.p0v, a0 = cur.a0, dv = cur.dv;
        double part = 0.0;
#pragma unroll
        for (int u = 0; u < WPF; ++u)
            if (cur.c[u] >= 0) part = fma(cur.v[u], ll_wait(mb + cur.c[u], ep, P.sc), part);
        for (int64_t e = e0 + lane + 32 * WPF; e < e1; e += 32)
            part = fma(__ldg(T.wval + e), ll_wait(mb + __ldg(T.wcol + e), ep, P.sc), part);
        part = warp_sum(part);
        if (lane == 0) {
            double acc;
            if (!UPPER) {
                double ri = r0;
                if (kind == K_ITER) {
                    ri = r0 - alpha * w0;
                    P.r[row] = ri;
                    P.x[row] = x0 + alpha * p0v;
                } else if (kind == K_PRO) {
                    if (in != P.r) P.r[row] = ri;
                    if (!P.use_x0) P.x[row] = 0.0;
                }
                acc_dot = fma(ri, ri, acc_dot);
                acc = ri - part;
            } else {
                acc = (r0 - part) * dv;
                if (rdot) acc_dot = fma(a0, acc, acc_dot);
                if (kind == K_PRO) P.p[row] = acc;
            }
            out[row] = acc;
            ll_store(mb + row, acc, ep);
        }
        __syncwarp();
    }
}

// RESIDENT executor's wavefront loop (one CTA; y/z and the fused operands in
// shared memory).  Slice s belongs to warp s % NWARP, so consecutive wavefronts
// (a single slice each on small 2-D grids) rotate over the warps.  A slice's
// static data is one fixed 64-byte record per lane (row, level, length, the
// first 4 dependency columns and values, 1/u_ii; layout.cpp), staged into a
// per-warp double buffer in shared memory with cp.async two slices ahead: the
// copies are asynchronous, so no warp stalls on a global load before a CTA
// barrier (every warp must arrive at every barrier, so one stalled warp delays
// the whole wavefront chain).  After a barrier only the staged-record read, the
// shared-memory gathers, the FMA chain (k ascending, as the definition) and the
// store remain.  The record's level tells a warp whether its next slice belongs
// to the current wavefront; no level pointer is read.
constexpr int RPF = SPCG_RREC_PF;
constexpr int RES_STAGE_BYTES = NWARP * 2 * 32 * SPCG_RREC_BYTES;   // 32 KB
__device__ __forceinline__ void cp_async16(void* sdst, const void* gsrc) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }

static_assert(NWARP >= SPCG_RES_WARPS, "the resident executor deals slices over 8 warps (layout.cpp records)");
template <bool UPPER>
__device__ void tri_resident(const Params& P, const DevTri& T, int kind, const double* in, double* out,
                             const double* rdot, double alpha, double& acc_dot, double* stage) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t ns = T.nslices;
    uint8_t* st = (uint8_t*)stage + (size_t)warp * 2 * 32 * SPCG_RREC_BYTES + lane * SPCG_RREC_BYTES;
    auto issue = [&](int64_t sl, int b) {
        if (sl < ns) {
            const uint8_t* g = T.rrec + (size_t)(sl * 32 + lane) * SPCG_RREC_BYTES;
            uint8_t* d = st + b * 32 * SPCG_RREC_BYTES;
#pragma unroll
            for (int q = 0; q < SPCG_RREC_BYTES / 16; ++q) cp_async16(d + 16 * q, g + 16 * q);
        }
        cp_async_commit();             // possibly empty: keeps the group count uniform
    };
    int64_t s = warp;
    int buf = 0;
    const bool owner = warp < SPCG_RES_WARPS;
    if (!owner) s = ns;
    issue(s, 0);
    issue(s + SPCG_RES_WARPS, 1);
    // level of my next slice: read once here, then carried in each record (the
    // owner of a wavefront goes from its store straight to the barrier)
    int gnext = 0xffff;
    if (s < ns) {
        cp_async_wait1();
        gnext = (*(const volatile int*)st) >> 16;
    }
    for (int g = 0; g < T.ngroups; ++g) {
        while (gnext == g) {           // warp-uniform
            cp_async_wait1();          // slice s landed (s + 8 may be in flight)
            const uint8_t* R = st + buf * 32 * SPCG_RREC_BYTES;
            const int w0 = *(const int*)R;
            const int w1 = *(const int*)(R + 4);
            gnext = w1 >> 16;
            const int row = (w0 & 0xffff) - 1;
            if (row >= 0) {
                const int len = w1 & 0xffff;
                const int4 cc = *(const int4*)(R + 16);
                const double2 v01 = *(const double2*)(R + 32);
                const double2 v23 = *(const double2*)(R + 48);
                const int c[RPF] = {cc.x, cc.y, cc.z, cc.w};
                const double v[RPF] = {v01.x, v01.y, v23.x, v23.y};
                double acc;
                if (!UPPER) {
                    double ri;
                    if (kind == K_ITER) {                       // Alg. 1 lines 11-12 fused
                        ri = P.r[row] - alpha * P.w[row];
                        P.r[row] = ri;
                        P.x[row] = P.x[row] + alpha * P.p[row];
                    } else {
                        ri = in[row];
                        if (kind == K_PRO) {
                            if (in != P.r) P.r[row] = ri;
                            if (!P.use_x0) P.x[row] = 0.0;
                        }
                    }
                    acc_dot = fma(ri, ri, acc_dot);            // ||r||^2
                    acc = ri;
                } else {
                    acc = in[row];
                }
                double d[RPF];
#pragma unroll
                for (int k = 0; k < RPF; ++k) d[k] = out[c[k]];
#pragma unroll
                for (int k = 0; k < RPF; ++k)
                    if (k < len) acc = fma(-v[k], d[k], acc);
                if (len > RPF) {
                    const int64_t e0 = __ldg(T.eoff + s);
                    for (int k = RPF; k < len; ++k)
                        acc = fma(-__ldg(T.val + (e0 + k) * 32 + lane), out[-__ldg(T.src + (e0 + k) * 32 + lane) - 1], acc);
                }
                if (UPPER) {
                    acc *= *(const double*)(R + 8);
                    if (rdot) acc_dot = fma(rdot[row], acc, acc_dot);   // (r, z)
                    if (kind == K_PRO) P.p[row] = acc;                   // p_0 = z_0
                }
                out[row] = acc;
            }
            issue(s + 2 * SPCG_RES_WARPS, buf);
            buf ^= 1;
            s += SPCG_RES_WARPS;
        }
        __syncthreads();
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
}

template <int STRAT, bool UPPER>
__device__ void tri_phase(const Params& P, const DevTri& T, int kind, const double* in, double* out,
                          const double* rdot, uint4* mb, unsigned ep, double alpha, double& acc_dot,
                          double* ring, unsigned& gen) {
    const int warp = threadIdx.x >> 5;
    if (STRAT == ST_RESIDENT) {
        tri_resident<UPPER>(P, T, kind, in, out, rdot, alpha, acc_dot, ring);
    } else if (STRAT == ST_LEVEL && T.wide) {
        tri_level_wide<UPPER>(P, T, kind, in, out, rdot, alpha, acc_dot, gen);
    } else if (STRAT == ST_SYNCFREE && T.wide) {
        tri_syncfree_wide<UPPER>(P, T, kind, in, out, rdot, mb, ep, alpha, acc_dot);
    } else if (STRAT == ST_LEVEL) {
        const int64_t W = (int64_t)gridDim.x * NWARP;
        const int64_t gw = (int64_t)blockIdx.x * NWARP + warp;
        for (int g = 0; g < T.ngroups; ++g) {
            const int64_t s0 = __ldg(T.gptr + g), s1 = __ldg(T.gptr + g + 1);
            for (int64_t s = s0 + gw; s < s1; s += W)
                tri_slice<STRAT, UPPER>(P, T, s, kind, in, out, rdot, mb, ep, alpha, acc_dot, ring, 0, 0);
            grid_sync(P.sc, gen);
        }
    } else if (STRAT == ST_SYNCFREE) {
        const int64_t W = (int64_t)gridDim.x * NWARP;
        for (int64_t s = (int64_t)blockIdx.x * NWARP + warp; s < T.nslices; s += W)
            tri_slice<STRAT, UPPER>(P, T, s, kind, in, out, rdot, mb, ep, alpha, acc_dot, ring, 0, 0);
    }
}

// ------------------------------------------------------------------ chunked pipeline
// Warp roles inside a CTA during a triangular-solve phase:
//   warp 0        producer: one lane streams the part's record chunks into the
//                 shared-memory ring with cp.async.bulk (TMA), mbarrier complete_tx
//   warps 1..2    pollers: a few records ahead of the solver, poll the ready flags
//                 of cross-CTA dependencies and leaves their partial sum in smem
//   warps 3..6    vector warps: per record, the dynamic per-row operands (fused
//                 x/r update and ||r||^2 for L; y_i and r_i for U)
//   warp 7        solver warp: the dependency chain, software-pipelined one record
//                 ahead so only ring gather -> FMA -> store sits on the critical path
constexpr int PRODUCER_WARP = 0;
constexpr int POLLER_WARP = 1;
#ifndef SPCG_NPOLL
#define SPCG_NPOLL (SPCG_BLOCK >= 256 && SPCG_NSOLVER_WARPS == 1 ? 2 : 1)
#endif
constexpr int NPOLL = SPCG_NPOLL;                 // poller warps (records alternate; 0: the solver polls)
constexpr int VEC_WARP0 = POLLER_WARP + NPOLL;
constexpr int NVEC = NWARP - 1 - NPOLL - SPCG_NSOLVER;   // 4 (8 warps, 1 solver) ...
static_assert(NVEC >= 1, "at least one vector warp");
constexpr int SOLVER_WARP0 = VEC_WARP0 + NVEC;
static_assert(SOLVER_WARP0 + SPCG_NSOLVER == NWARP, "warp roles must fill the CTA");
#ifndef SPCG_SOLVER_TREE
#define SPCG_SOLVER_TREE 0         // 1: fast-path row sum as two interleaved FMA chains (experiment)
#endif
#ifndef SPCG_SOLVER_UNROLL
#define SPCG_SOLVER_UNROLL 4       // record pairs per chunk unrolled in the solver (MAXREC / 2 = all)
#endif
#ifndef SPCG_PHASE_NOINLINE
#define SPCG_PHASE_NOINLINE 0      // 1: one shared copy of the chunked phase (smaller code, but Params then
                                   // live in local memory: 1.5x slower per iteration, measured)
#endif
constexpr int kSolverUnroll = SPCG_SOLVER_UNROLL;
#ifndef SPCG_POLL_AHEAD
#define SPCG_POLL_AHEAD 8
#endif
constexpr int POLL_AHEAD = SPCG_POLL_AHEAD;       // records
#ifndef SPCG_VGROUP
#define SPCG_VGROUP 4
#endif
constexpr int VGROUP = SPCG_VGROUP;               // chunks a vector warp serves per round
constexpr int VBATCH = 4;                         // records whose loads are in flight together
constexpr int VLIST = (VGROUP * SPCG_MAXREC + NVEC - 1) / NVEC;
static_assert(VGROUP >= 1 && VGROUP <= SPCG_NCHUNK, "vector group must fit the ring");
constexpr int SIDE_BYTES = 3 * 256 + 16;          // vec[32], aux[32], ext[32], ext mask
constexpr size_t CH_RING_BYTES = (size_t)SPCG_NCHUNK * SPCG_CHUNK_BYTES;
constexpr size_t CH_SIDE_BYTES = (size_t)SPCG_NCHUNK * SPCG_MAXREC * SIDE_BYTES;
constexpr size_t CH_BAR_BYTES = 512;
static_assert((3 * SPCG_NCHUNK + 1 + SPCG_NSOLVER + 1) <= 31 && 256 + 2 * NVEC * VLIST <= CH_BAR_BYTES,
              "barrier block layout");

__host__ __device__ constexpr size_t chunked_smem_bytes(int ring) {
    return (size_t)ring * 8 + CH_RING_BYTES + CH_SIDE_BYTES + CH_BAR_BYTES;
}

struct ChunkSmem {
    double* yring;
    uint8_t* chunks;
    uint8_t* side;
    uint64_t* full;        // [NCHUNK] TMA landed
    uint64_t* vfull;       // [NCHUNK] vector operands filled
    uint64_t* empty;       // [NCHUNK] solvers + poller done
    uint64_t* ldone;       // solvers finished the L section
    volatile long long* progress;   // [NSOLVER] record index each solver warp is at
    uint16_t* vlist;       // [NVEC][VLIST] per vector warp: (slot, record) of its records in a group
    volatile unsigned* chain;   // multi-solver: slices of this phase completed (ring accesses ordered by it)
};

struct PipeState {         // identical sequence in every role
    unsigned q;            // chunks consumed in this launch
    unsigned ldone_uses;
    long long rec;         // records walked in this launch
    long long k;           // iteration (debug timeline only)
};

__device__ ChunkSmem chunk_smem(double* dyn, int ring) {
    // the host guarantees ring >= 16 and a power of two (layout.cpp): chunks stay 128-byte aligned
    ChunkSmem S;
    uint8_t* base = (uint8_t*)dyn;
    S.yring = dyn;
    S.chunks = base + (size_t)ring * 8;
    S.side = S.chunks + CH_RING_BYTES;
    uint64_t* bars = (uint64_t*)(S.side + CH_SIDE_BYTES);
    S.full = bars;
    S.vfull = bars + SPCG_NCHUNK;
    S.empty = bars + 2 * SPCG_NCHUNK;
    S.ldone = bars + 3 * SPCG_NCHUNK;
    S.progress = (volatile long long*)(bars + 3 * SPCG_NCHUNK + 1);
    S.vlist = (uint16_t*)(bars + 32);
    S.chain = (volatile unsigned*)(bars + 31);
    return S;
}

__device__ void chunk_init(const ChunkSmem& S) {
    if (threadIdx.x == 0) {
        for (int i = 0; i < SPCG_NCHUNK; ++i) {
            mbar_init(&S.full[i], 1);
            mbar_init(&S.vfull[i], NVEC);
            mbar_init(&S.empty[i], SPCG_NSOLVER + NPOLL);
        }
        mbar_init(S.ldone, SPCG_NSOLVER);
        for (int i = 0; i < SPCG_NSOLVER; ++i) S.progress[i] = -1;
        *S.chain = 0u;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
}

// record view (byte layout written by layout.cpp emit_section):
//   [0,16)    header {u16 w, u16 flags, u8 warp, u8 side, u16 bytes, u32 publish, u32 active}
//   [16,272)  32 lane words {int32 row, u32 meta = len | ne << 8 | publish << 16}
//   [272, +128w) int32 src[w][32]; then f64 val[w][32]; then f64 dinv[32] (U, LAST)
struct Rec {
    const uint8_t* p;
    uint4 h;
    __device__ __forceinline__ explicit Rec(const uint8_t* q) : p(q), h(*(const uint4*)q) {}
    __device__ __forceinline__ int w() const { return (int)(h.x & 0xffffu); }
    __device__ __forceinline__ int flags() const { return (int)(h.x >> 16); }
    __device__ __forceinline__ int warp() const { return (int)(h.y & 0xffu); }
    __device__ __forceinline__ int bytes() const { return (int)(h.y >> 16); }
    __device__ __forceinline__ int2 lane(int l) const { return *(const int2*)(p + 16 + 8 * l); }
    __device__ __forceinline__ int row(int l) const { return *(const int*)(p + 16 + 8 * l); }
    __device__ __forceinline__ int src(int k, int l) const { return *(const int32_t*)(p + SPCG_REC_HDR + 128 * k + 4 * l); }
    __device__ __forceinline__ double val(int k, int l) const {
        return *(const double*)(p + SPCG_REC_HDR + 128 * w() + 256 * k + 8 * l);
    }
    __device__ __forceinline__ double dinv(int l) const { return *(const double*)(p + SPCG_REC_HDR + 384 * w() + 8 * l); }
};
__device__ __forceinline__ int meta_len(unsigned m) { return (int)(m & 0xffu); }
__device__ __forceinline__ int meta_ne(unsigned m) { return (int)((m >> 8) & 0xffu); }
__device__ __forceinline__ bool meta_pub(unsigned m) { return (m >> 16) & 1u; }
__device__ __forceinline__ double* side_vec(const ChunkSmem& S, int slot, int r) {
    return (double*)(S.side + ((size_t)slot * SPCG_MAXREC + r) * SIDE_BYTES);
}
__device__ __forceinline__ double* side_aux(const ChunkSmem& S, int slot, int r) { return side_vec(S, slot, r) + 32; }
__device__ __forceinline__ double* side_ext(const ChunkSmem& S, int slot, int r) { return side_vec(S, slot, r) + 64; }
__device__ __forceinline__ unsigned* side_mask(const ChunkSmem& S, int slot, int r) {
    return (unsigned*)(side_vec(S, slot, r) + 96);
}

// sum of the leading ne external terms v_k * y_k (k order), polling the flags in one batch
__device__ __forceinline__ bool ext_try(const Rec& R, int lane, int ne, const uint4* mb, unsigned ep, double& out) {
    double acc = 0.0;
    bool ok = true;
    for (int k0 = 0; k0 < ne; k0 += 4) {
        uint4 v[4];
#pragma unroll
        for (int t = 0; t < 4; ++t)
            if (k0 + t < ne) {
                const uint4* a = mb + (-R.src(k0 + t, lane) - 1);
                asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                             : "=r"(v[t].x), "=r"(v[t].y), "=r"(v[t].z), "=r"(v[t].w)
                             : "l"(a)
                             : "memory");
            }
#pragma unroll
        for (int t = 0; t < 4; ++t)
            if (k0 + t < ne) {
                if (v[t].y != ep || v[t].w != ep) ok = false;
                const double y = __longlong_as_double((long long)(((unsigned long long)v[t].z << 32) | v[t].x));
                acc = fma(R.val(k0 + t, lane), y, acc);
            }
    }
    out = acc;
    return ok;
}

__device__ __noinline__ double ext_wait(const Rec& R, int lane, int ne, const uint4* mb, unsigned ep, Scal* sc) {
    double acc;
    if (ext_try(R, lane, ne, mb, ep, acc)) return acc;
    acc = 0.0;
    for (int k = 0; k < ne; ++k) acc = fma(R.val(k, lane), ll_wait(mb + (-R.src(k, lane) - 1), ep, sc), acc);
    return acc;
}

// ring part of a record for a compile-time width W (warp-uniform dispatch keeps
// the instruction count proportional to the record's real width)
template <int W>
__device__ __forceinline__ double ring_terms(const uint8_t* p, int lane, int ne, int len, const double* yring,
                                             double acc) {
    const uint8_t* sp = p + SPCG_REC_HDR + 4 * lane;
    const uint8_t* vp = p + SPCG_REC_HDR + 128 * W + 8 * lane;
    int sidx[W > 0 ? W : 1];
    double v[W > 0 ? W : 1], d[W > 0 ? W : 1];
#pragma unroll
    for (int k = 0; k < W; ++k) {
        const bool on = k >= ne && k < len;
        sidx[k] = on ? *(const int*)(sp + 128 * k) : 0;
        v[k] = on ? *(const double*)(vp + 256 * k) : 0.0;
    }
#pragma unroll
    for (int k = 0; k < W; ++k) d[k] = yring[sidx[k]];
#pragma unroll
    for (int k = 0; k < W; ++k) acc = fma(-v[k], d[k], acc);   // v = 0 for masked-off k: acc unchanged
    return acc;
}

__device__ __forceinline__ double ring_terms_dispatch(int wd, const uint8_t* p, int lane, int ne, int len,
                                                      const double* yring, double acc) {
    switch (wd) {
        case 0: return acc;
        case 1: return ring_terms<1>(p, lane, ne, len, yring, acc);
        case 2: return ring_terms<2>(p, lane, ne, len, yring, acc);
        case 3: return ring_terms<3>(p, lane, ne, len, yring, acc);
        case 4: return ring_terms<4>(p, lane, ne, len, yring, acc);
        case 5: return ring_terms<5>(p, lane, ne, len, yring, acc);
        case 6: return ring_terms<6>(p, lane, ne, len, yring, acc);
        case 7: return ring_terms<7>(p, lane, ne, len, yring, acc);
        default: return ring_terms<8>(p, lane, ne, len, yring, acc);
    }
}

// ---- solver warp ------------------------------------------------------------
// A record's operands, loaded ahead of its computation (see solver_section).
constexpr int WP = SPCG_WP;
struct Prep {
    const uint8_t* p;
    int fl, wd, row, r;
    unsigned meta;
    int sidx[WP];
    double v[WP];
    double vec, dinv, aux;
};

struct SolveCtx {          // per-section constants of the solver warp
    double* yring;
    const ChunkSmem* S;
    double* out;
    const double* rdot;
    double* pvec;          // p (prologue: p0 = z0)
    const uint4* mb;
    Scal* sc;
    unsigned ep;
    int64_t pb;
    int mask;
};

template <bool UPPER>
__device__ __forceinline__ void prep_record(Prep& X, const ChunkSmem& S, const uint8_t* ch, int slot, int r, int lane) {
    X.r = r;
    X.p = ch + *(const uint16_t*)(ch + 8 + 2 * r);
    const uint4 h = *(const uint4*)X.p;
    X.fl = (int)(h.x >> 16);
    X.wd = (int)(h.x & 0xffffu);
    const int2 lw = *(const int2*)(X.p + 16 + 8 * lane);
    X.row = lw.x;
    X.meta = (unsigned)lw.y;
    const int len = meta_len(X.meta), ne = meta_ne(X.meta);
    const uint8_t* sp = X.p + SPCG_REC_HDR + 4 * lane;
    const uint8_t* vp = X.p + SPCG_REC_HDR + 128 * X.wd + 8 * lane;
    // ring entries in registers.  Only the warp-uniform width guards the loads: the
    // layout stores padding entries (k >= len, padding lanes) as (slot 0, 0.0), so
    // they add nothing; cross-CTA entries (k < ne, negative slots) exist only in
    // REC_EXT records, whose path masks them (solve_record).
    (void)len;
    (void)ne;
#pragma unroll
    for (int k = 0; k < WP; ++k) {
        const bool on = k < X.wd;
        X.sidx[k] = on ? *(const int*)(sp + 128 * k) : 0;
        X.v[k] = on ? *(const double*)(vp + 256 * k) : 0.0;
    }
    X.vec = side_vec(S, slot, r)[lane];
    if (UPPER) {
        const bool fast_last = (X.fl & (REC_LAST | REC_WIDE)) == REC_LAST;
        X.dinv = fast_last ? *(const double*)(X.p + SPCG_REC_HDR + 384 * X.wd + 8 * lane) : 1.0;
        X.aux = side_aux(S, slot, r)[lane];
    }
}

// row epilogue (Alg. 1 line 13 output + (r,z) + publication)
template <bool UPPER, bool PRO>
__device__ __forceinline__ void finish_row(const SolveCtx& C, int row, unsigned meta, double acc, double dinv,
                                           double ri, double& rz) {
    if (row >= 0) {
        if (UPPER) {
            acc *= dinv;
            rz = fma(ri, acc, rz);
            if (PRO) C.pvec[row] = acc;
        }
        C.yring[meta >> 17] = acc;                    // part-local ring slot
        C.out[row] = acc;
        if (meta_pub(meta)) ll_store((uint4*)C.mb + row, acc, C.ep);
    }
}

// general record: continuation of a row over several records, > WP entries, or
// cross-CTA dependencies the poller did not resolve (rare: kept out of line).
// Takes scalars only and returns {acc, rz} so no caller variable is address-taken.
template <bool UPPER, bool PRO>
__device__ __noinline__ double2 slow_record(const uint8_t* p, int fl, int wd, int row, unsigned meta, int r,
                                            double vec, double aux, double acc_carry, double rz, double* side_rec,
                                            double* yring, double* out, const double* rdot, double* pvec,
                                            const uint4* mb, Scal* sc, unsigned ep, int64_t pb, int mask) {
    const int lane = threadIdx.x & 31;
    const Rec R(p);
    const int len = meta_len(meta), ne = meta_ne(meta);
    double acc;
    if (fl & REC_FIRST) {
        double e = 0.0;
        if (row >= 0 && ne > 0) {
            const unsigned m = lds_acquire_u32((const unsigned*)(side_rec + 96));
            if (m & (1u << lane)) e = lds_volatile(side_rec + 64 + lane);
            else e = ext_wait(R, lane, ne, mb, ep, sc);
        }
        acc = vec - e;
    } else {
        acc = acc_carry;
        if (row >= 0 && ne > 0) acc -= ext_wait(R, lane, ne, mb, ep, sc);
    }
    if (row >= 0) acc = ring_terms_dispatch(wd, p, lane, ne, len, yring, acc);
    if ((fl & REC_LAST) && row >= 0) {
        double a = acc;
        if (UPPER) {
            a *= R.dinv(lane);
            const double ri = (fl & REC_FIRST) ? aux : (rdot ? __ldcg(rdot + row) : 0.0);
            rz = fma(ri, a, rz);
            if (PRO) pvec[row] = a;
        }
        yring[meta >> 17] = a;
        out[row] = a;
        if (meta_pub(meta)) ll_store((uint4*)mb + row, a, ep);
        acc = a;
    }
    return make_double2(acc, rz);
}

#ifndef SPCG_DEBUG_COUNTS
#define SPCG_DEBUG_COUNTS 0      // debug builds only (-DSPCG_DEBUG_COUNTS=1, tools/diag.py): no cost otherwise
#endif
__device__ unsigned long long* g_dbg_counts = nullptr;   // debug: [0] fast, [1] ext-fast, [2] slow
template <bool UPPER, bool PRO>
__device__ __forceinline__ void solve_record(const SolveCtx& C, const Prep& X, int slot, int lane, double& acc_carry,
                                             double& rz) {
    if ((X.fl & (REC_FIRST | REC_WIDE | REC_EXT)) == REC_FIRST) {
        // fast path: whole row in this record, <= WP ring entries, no cross-CTA term
        double d[WP];
#pragma unroll
        for (int k = 0; k < WP; ++k) d[k] = C.yring[X.sidx[k]];
        double acc;
        if (SPCG_SOLVER_TREE) {
            // two independent FMA chains then one add: depth 3 instead of WP = 4 on the
            // record-to-record dependency path (rounding order differs from the chain)
            double a0 = fma(-X.v[0], d[0], X.vec), a1 = -X.v[1] * d[1];
#pragma unroll
            for (int k = 2; k < WP; ++k) {
                if (k & 1) a1 = fma(-X.v[k], d[k], a1);
                else a0 = fma(-X.v[k], d[k], a0);
            }
            acc = a0 + a1;
        } else {
            acc = X.vec;
#pragma unroll
            for (int k = 0; k < WP; ++k) acc = fma(-X.v[k], d[k], acc);   // v = 0 off-entry
        }
        finish_row<UPPER, PRO>(C, X.row, X.meta, acc, X.dinv, X.aux, rz);
        acc_carry = acc;
    } else if ((X.fl & (REC_FIRST | REC_WIDE)) == REC_FIRST) {
        // cross-CTA terms: normally pre-resolved by the poller into the side slot
        const int ne = meta_ne(X.meta);
        const unsigned m = lds_acquire_u32(side_mask(*C.S, slot, X.r));
        const bool have = ne == 0 || (m >> lane) & 1u;
        const bool all_have = __all_sync(0xffffffffu, have);
        if (SPCG_DEBUG_COUNTS && g_dbg_counts && lane == 0) atomicAdd(g_dbg_counts + (all_have ? 1 : 2), 1ull);
        if (all_have) {
            double e = 0.0;
            if (ne > 0) e = lds_volatile(side_ext(*C.S, slot, X.r) + lane);
            double d[WP];
#pragma unroll
            for (int k = 0; k < WP; ++k) d[k] = C.yring[k < ne ? 0 : X.sidx[k]];
            double acc = X.vec - e;
#pragma unroll
            for (int k = 0; k < WP; ++k) acc = fma(k < ne ? 0.0 : -X.v[k], d[k], acc);
            finish_row<UPPER, PRO>(C, X.row, X.meta, acc, X.dinv, X.aux, rz);
            acc_carry = acc;
        } else {
            const double2 o = slow_record<UPPER, PRO>(X.p, X.fl, X.wd, X.row, X.meta, X.r, X.vec, X.aux, acc_carry, rz,
                                                      side_vec(*C.S, slot, X.r), C.yring, C.out, C.rdot, C.pvec, C.mb,
                                                      C.sc, C.ep, C.pb, C.mask);
            acc_carry = o.x;
            rz = o.y;
        }
    } else {
        if (SPCG_DEBUG_COUNTS && g_dbg_counts && lane == 0) atomicAdd(g_dbg_counts + 6, 1ull);
        const double2 o = slow_record<UPPER, PRO>(X.p, X.fl, X.wd, X.row, X.meta, X.r, X.vec, X.aux, acc_carry, rz,
                                                  side_vec(*C.S, slot, X.r), C.yring, C.out, C.rdot, C.pvec, C.mb,
                                                  C.sc, C.ep, C.pb, C.mask);
        acc_carry = o.x;
        rz = o.y;
    }
    __syncwarp();
}

// The solver warp over one section (all L or all U records of the part): per
// chunk, records are fully unrolled with a ping-pong prefetch so that record
// t+1's operands are in registers while record t computes; only ring gather ->
// FMA chain -> ring store remains on the dependency path.
template <bool UPPER, bool PRO>
__device__ __forceinline__ void solver_section(const SolveCtx& C, const ChunkSmem& S, unsigned q0, int ib, int ie,
                                               long long recn, double& rz, const Params& P, long long kk) {
    const int lane = threadIdx.x & 31;
    double acc_carry = 0.0;
    unsigned long long* dbg = SPCG_DEBUG_COUNTS ? g_dbg_counts : nullptr;   // debug: solver wait / busy cycles
    long long t_wait = 0, t_sec = dbg ? clock64() : 0, t_prep = 0, t_solve = 0, nchunks = 0;
    const long long recn0 = recn;
    for (int i = ib; i < ie; ++i) {
        const unsigned q = q0 + i;
        const int slot = q % SPCG_NCHUNK;
        const long long tw = dbg ? clock64() : 0;
        if (!warp_ok(mbar_wait(&S.vfull[slot], (q / SPCG_NCHUNK) & 1, C.sc))) return;
        if (dbg) t_wait += clock64() - tw;
        const uint8_t* ch = S.chunks + (size_t)slot * SPCG_CHUNK_BYTES;
        const int nrec = *(const uint16_t*)ch;
        // progress for the pollers, once per chunk (the first record the solver is on)
        if (lane == 0) S.progress[0] = recn;
        Prep A, B;
        if (nrec > 0) prep_record<UPPER>(A, S, ch, slot, 0, lane);
#pragma unroll kSolverUnroll
        for (int r = 0; r < SPCG_MAXREC; r += 2) {
            long long tp = dbg ? clock64() : 0;
            if (r + 1 < nrec) prep_record<UPPER>(B, S, ch, slot, r + 1, lane);
            if (dbg) { t_prep += clock64() - tp; tp = clock64(); }
            if (r < nrec) {
                solve_record<UPPER, PRO>(C, A, slot, lane, acc_carry, rz);
            }
            if (dbg) { t_solve += clock64() - tp; tp = clock64(); }
            if (r + 2 < nrec) prep_record<UPPER>(A, S, ch, slot, r + 2, lane);
            if (dbg) { t_prep += clock64() - tp; tp = clock64(); }
            if (r + 1 < nrec) {
                solve_record<UPPER, PRO>(C, B, slot, lane, acc_carry, rz);
            }
            if (dbg) t_solve += clock64() - tp;
        }
        recn += nrec;
        ++nchunks;
        __syncwarp();
        if (lane == 0) mbar_arrive(&S.empty[slot]);
    }
    if (dbg && lane == 0) {
        atomicAdd(dbg + 3, (unsigned long long)t_wait);
        atomicAdd(dbg + 4, (unsigned long long)(clock64() - t_sec));
        atomicAdd(dbg + 5, (unsigned long long)(recn - recn0));
        atomicAdd(dbg + 7, (unsigned long long)nchunks);
        atomicAdd(dbg + 8, (unsigned long long)t_prep);
        atomicAdd(dbg + 9, (unsigned long long)t_solve);
    }
}

// Several solver warps (SPCG_NSOLVER > 1): the slices of the part's stream are
// dealt round-robin to them (record header `warp`, layout.cpp); every solver warp
// walks all records to number the slices of this phase, prepares its own records
// ahead, then waits until the chain counter says every earlier slice is done,
// runs the record (ring gathers -> FMAs -> ring / global stores) and, after the
// slice's last record, publishes chain = slice + 1 (release fence, then a
// volatile store).  The ring is therefore read and written in exactly the
// sequential slice order the layout's ring analysis assumes, while each warp's
// instruction stream carries only 1/NSOLVER of the records.
__device__ __forceinline__ bool chain_wait(const ChunkSmem& S, unsigned s, Scal* sc) {
    const int lane = threadIdx.x & 31;
    unsigned it = 0;
    const long long t0 = clock64();
    for (;;) {
        const unsigned c = __shfl_sync(0xffffffffu, lane == 0 ? *S.chain : 0u, 0);
        if ((int)(c - s) >= 0) return true;
        if ((++it & 1023) == 0) {
            const bool late = __shfl_sync(0xffffffffu, clock64() - t0 > SPIN_TIMEOUT_CYC, 0);
            if (late && lane == 0) atomicExch(&sc->abort, 1);
            if (late || aborted(sc)) return false;
        }
    }
}

template <bool UPPER, bool PRO>
__device__ __noinline__ void solver_section_multi(const SolveCtx& C, const ChunkSmem& S, unsigned q0, int ib, int ie,
                                                  unsigned& lseq, double& rz, int sw, long long recn) {
    const int lane = threadIdx.x & 31;
    double acc_carry = 0.0;
    for (int i = ib; i < ie; ++i) {
        const unsigned q = q0 + i;
        const int slot = q % SPCG_NCHUNK;
        if (!warp_ok(mbar_wait(&S.vfull[slot], (q / SPCG_NCHUNK) & 1, C.sc))) return;
        const uint8_t* ch = S.chunks + (size_t)slot * SPCG_CHUNK_BYTES;
        const int nrec = *(const uint16_t*)ch;
        if (sw == 0 && lane == 0) S.progress[0] = recn;
        recn += nrec;
        for (int r = 0; r < nrec; ++r) {
            const uint8_t* p = ch + *(const uint16_t*)(ch + 8 + 2 * r);
            const int fl = (int)(*(const uint32_t*)p >> 16);
            const int owner = p[4];
            const unsigned sl = (fl & REC_FIRST) ? lseq++ : lseq - 1;   // slice of this record
            if (owner != sw) continue;
            Prep X;
            prep_record<UPPER>(X, S, ch, slot, r, lane);
            if ((fl & REC_FIRST) && !chain_wait(S, sl, C.sc)) return;
            if ((X.fl & (REC_FIRST | REC_LAST | REC_WIDE | REC_EXT)) == (REC_FIRST | REC_LAST)) {
                // fast path with the chain handoff before the global stores: ring store,
                // fence, counter, and only then out[] / p / the ready flag (a fence after
                // the global stores would wait for them)
                double d[WP];
#pragma unroll
                for (int k = 0; k < WP; ++k) d[k] = C.yring[X.sidx[k]];
                double acc = X.vec;
#pragma unroll
                for (int k = 0; k < WP; ++k) acc = fma(-X.v[k], d[k], acc);
                if (UPPER) acc *= X.dinv;
                if (X.row >= 0) C.yring[X.meta >> 17] = acc;
                fence_acq_rel_cta();
                __syncwarp();
                if (lane == 0) *S.chain = sl + 1;
                if (X.row >= 0) {
                    if (UPPER) {
                        rz = fma(X.aux, acc, rz);
                        if (PRO) C.pvec[X.row] = acc;
                    }
                    C.out[X.row] = acc;
                    if (meta_pub(X.meta)) ll_store((uint4*)C.mb + X.row, acc, C.ep);
                }
                acc_carry = acc;
                continue;
            }
            solve_record<UPPER, PRO>(C, X, slot, lane, acc_carry, rz);
            if (fl & REC_LAST) {
                fence_acq_rel_cta();            // this warp's ring stores before the counter
                __syncwarp();
                if (lane == 0) *S.chain = sl + 1;
            }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&S.empty[slot]);
    }
}

// One triangular-solve phase of a part: chunks [c0, c1) of its stream (L section,
// U section or both).  All threads of the CTA call it.
#if SPCG_PHASE_NOINLINE
__device__ __noinline__
#else
__device__ __forceinline__
#endif
void chunked_phase(const Params& P, const ChunkSmem& S, PipeState& st, int c0, int c1, int cu, int kind,
                              const double* rin, double* y, const double* yin, double* z, const double* rdot,
                              unsigned ep, double alpha, double& rr, double& rz, int64_t pb) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int mask = P.ring - 1;
    const unsigned q0 = st.q;
    const long long rec0 = st.rec;
    const int nch = c1 - c0;
    if (warp == PRODUCER_WARP) {
        // chunk sizes are read 32 at a time by the whole warp (one round trip), then
        // lane 0 issues the bulk copies as ring slots free up
        for (int b0 = 0; b0 < nch; b0 += 32) {
            const int cnt = min(32, nch - b0);
            unsigned my_bytes = 0;
            if (lane < cnt) my_bytes = __ldg(P.chunk_bytes + c0 + b0 + lane);
            bool ok = true;
            for (int t = 0; t < cnt && ok; ++t) {
                const unsigned bytes = __shfl_sync(0xffffffffu, my_bytes, t);
                if (lane == 0) {
                    const unsigned q = q0 + b0 + t, slot = q % SPCG_NCHUNK, use = q / SPCG_NCHUNK;
                    ok = mbar_wait(&S.empty[slot], (use & 1) ^ 1, P.sc);
                    if (ok) {
                    hbeat(P, 0, ((unsigned long long)(st.k + 1) << 40) | q);
                    mbar_arrive_tx(&S.full[slot], bytes);
                    bulk_g2s(S.chunks + (size_t)slot * SPCG_CHUNK_BYTES,
                             P.stream + (size_t)(c0 + b0 + t) * SPCG_CHUNK_BYTES, bytes, &S.full[slot]);
                    }
                }
                ok = __shfl_sync(0xffffffffu, ok, 0);
            }
            if (!ok) break;
        }
    } else if (warp >= VEC_WARP0 && warp < SOLVER_WARP0) {
        // Chunks are taken in groups of up to VGROUP (never straddling the L/U
        // boundary); this warp's records of the whole group are listed first and
        // then served VBATCH at a time with every global load of the batch issued
        // before the first use, so a group costs ~one memory latency instead of
        // one per chunk.  VGROUP <= SPCG_NCHUNK: the producer can fill the whole
        // group without any slot being released, so the wait cannot deadlock.
        const int v = warp - VEC_WARP0;
        bool waited_ldone = false;
        long long recn = rec0;
        uint16_t* mine = S.vlist + v * VLIST;
        for (int i0 = 0; i0 < nch;) {
            int i1 = min(nch, i0 + VGROUP);
            if (c0 + i0 < cu && c0 + i1 > cu) i1 = cu - c0;
            if (c0 + i0 >= cu && !waited_ldone && cu > c0) {   // y of the L section must be complete
                if (!warp_ok(mbar_wait(S.ldone, st.ldone_uses & 1, P.sc))) break;
                waited_ldone = true;
            }
            if (v == 0 && lane == 0) hbeat(P, 1, ((unsigned long long)(st.k + 1) << 40) | (q0 + i0));
            bool ok = true;
            for (int i = i0; i < i1 && ok; ++i) {
                const unsigned q = q0 + i;
                ok = mbar_wait(&S.full[q % SPCG_NCHUNK], (q / SPCG_NCHUNK) & 1, P.sc);
            }
            if (!warp_ok(ok)) break;
            // list: records are dealt to the vector warps by their global index
            int cnt = 0;
            for (int i = i0; i < i1; ++i) {
                const unsigned slot = (q0 + i) % SPCG_NCHUNK;
                const uint8_t* ch = S.chunks + (size_t)slot * SPCG_CHUNK_BYTES;
                const int nrec = *(const uint16_t*)ch;
                for (int r = 0; r < nrec; ++r, ++recn) {
                    if ((int)(recn % NVEC) != v) continue;
                    if (!(*(const uint16_t*)(ch + *(const uint16_t*)(ch + 8 + 2 * r) + 2) & REC_FIRST)) continue;
                    if (lane == 0) mine[cnt] = (uint16_t)(slot * SPCG_MAXREC + r);
                    ++cnt;
                }
            }
            __syncwarp();
            for (int b0 = 0; b0 < cnt; b0 += VBATCH) {
                int row[VBATCH], e[VBATCH], fl[VBATCH];
                double l0[VBATCH], l1[VBATCH], l2[VBATCH], l3[VBATCH];
#pragma unroll
                for (int j = 0; j < VBATCH; ++j) {
                    row[j] = -1;
                    fl[j] = 0;
                    e[j] = 0;
                    if (b0 + j < cnt) {
                        e[j] = mine[b0 + j];
                        const uint8_t* ch = S.chunks + (size_t)(e[j] / SPCG_MAXREC) * SPCG_CHUNK_BYTES;
                        const Rec R(ch + *(const uint16_t*)(ch + 8 + 2 * (e[j] % SPCG_MAXREC)));
                        fl[j] = R.flags();
                        row[j] = R.row(lane);
                    }
                }
#pragma unroll
                for (int j = 0; j < VBATCH; ++j) {      // every load of the batch before any use
                    l0[j] = l1[j] = l2[j] = l3[j] = 0.0;
                    if (row[j] >= 0) {
                        if (!(fl[j] & REC_UPPER)) {
                            if (kind == K_ITER) {
                                l0[j] = __ldcg(P.r + row[j]);
                                l1[j] = __ldcg(P.w + row[j]);
                                l2[j] = __ldcg(P.x + row[j]);
                                l3[j] = __ldcg(P.p + row[j]);
                            } else {
                                l0[j] = __ldcg(rin + row[j]);
                            }
                        } else {
                            l0[j] = __ldcg(yin + row[j]);
                            if (rdot) l1[j] = __ldcg(rdot + row[j]);
                        }
                    }
                }
#pragma unroll
                for (int j = 0; j < VBATCH; ++j) {
                    if (b0 + j >= cnt) continue;
                    const int slot = e[j] / SPCG_MAXREC, r = e[j] % SPCG_MAXREC;
                    if (row[j] >= 0) {
                        double* vec = side_vec(S, slot, r);
                        if (!(fl[j] & REC_UPPER)) {
                            double ri = l0[j];
                            if (kind == K_ITER) {
                                ri = l0[j] - alpha * l1[j];
                                P.r[row[j]] = ri;
                                P.x[row[j]] = l2[j] + alpha * l3[j];
                            } else if (kind == K_PRO) {
                                if (rin != P.r) P.r[row[j]] = ri;
                                if (!P.use_x0) P.x[row[j]] = 0.0;
                            }
                            rr = fma(ri, ri, rr);
                            vec[lane] = ri;
                        } else {
                            vec[lane] = l0[j];
                            side_aux(S, slot, r)[lane] = l1[j];
                        }
                    }
                    if (lane == 0) *side_mask(S, slot, r) = 0u;
                }
            }
            __syncwarp();
            if (lane == 0)
                for (int i = i0; i < i1; ++i) mbar_arrive(&S.vfull[(q0 + i) % SPCG_NCHUNK]);
            i0 = i1;
        }
    } else if (warp >= POLLER_WARP && warp < POLLER_WARP + NPOLL) {
        const int pw = warp - POLLER_WARP;
        long long recn = rec0;
        for (int i = 0; i < nch; ++i) {
            const unsigned q = q0 + i, slot = q % SPCG_NCHUNK, use = q / SPCG_NCHUNK;
            if (lane == 0 && pw == 0) hbeat(P, 2, ((unsigned long long)(st.k + 1) << 40) | q);
            if (!warp_ok(mbar_wait(&S.vfull[slot], use & 1, P.sc))) break;
            const uint8_t* ch = S.chunks + (size_t)slot * SPCG_CHUNK_BYTES;
            const int nrec = *(const uint16_t*)ch;
            for (int r = 0; r < nrec; ++r, ++recn) {
                const Rec R(ch + *(const uint16_t*)(ch + 8 + 2 * r));
                if (lane == 0 && pw == 0) hbeat(P, 3, ((unsigned long long)(st.k + 1) << 40) | (unsigned long long)recn);
                if ((int)(recn % (NPOLL > 0 ? NPOLL : 1)) != pw || !(R.flags() & REC_FIRST)) continue;
                const int2 lw = R.lane(lane);
                const int ne = lw.x >= 0 ? meta_ne((unsigned)lw.y) : 0;
                if (!__any_sync(0xffffffffu, ne > 0)) continue;
                const uint4* mb = (R.flags() & REC_UPPER) ? P.mbU : P.mbL;
                bool need = ne > 0;
                unsigned it = 0;
                const long long tp0 = clock64();
                for (;;) {                                     // warp-uniform control flow
                    __syncwarp();
                    const long long pmin = __shfl_sync(0xffffffffu, (long long)S.progress[0], 0);
                    if (lane == 0 && pw == 0) { hbeat(P, 6, (unsigned long long)pmin); hbeat(P, 7, it); }
                    if (pmin >= recn) break;                   // the solver is here: it polls itself
                    if (recn <= pmin + POLL_AHEAD) {           // close enough: values may be there
                        double e = 0.0;
                        const bool ok = need && ext_try(R, lane, ne, mb, ep, e);
                        __syncwarp();
                        if (ok) {
                            side_ext(S, slot, r)[lane] = e;
                            fence_acq_rel_cta();
                            atomicOr(side_mask(S, slot, r), 1u << lane);
                            need = false;
                        }
                        if (__ballot_sync(0xffffffffu, need) == 0u) break;
                    } else {
                        __nanosleep(64);
                    }
                    if ((++it & 255) == 0) {
                        const bool late = __shfl_sync(0xffffffffu, clock64() - tp0 > SPIN_TIMEOUT_CYC, 0);
                        if (late && lane == 0) atomicExch(&P.sc->abort, 1);
                        if (late || aborted(P.sc)) break;
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&S.empty[slot]);
        }
    } else {
        // ---------------- solver warp(s)
        const int ncL = (c0 < cu) ? min(cu, c1) - c0 : 0;       // chunks of the L section
        if (lane == 0) trace_mark(P, st.k, 8 + 4 * blockIdx.x + 0);
        SolveCtx C{S.yring, &S, y, nullptr, P.p, P.mbL, P.sc, ep, pb, mask};
        if (SPCG_NSOLVER > 1) {
            const int sw = warp - SOLVER_WARP0;
            unsigned lseq = 0;
            if (ncL > 0) {
                double dummy = 0.0;
                solver_section_multi<false, false>(C, S, q0, 0, ncL, lseq, dummy, sw, rec0);
                __syncwarp();
                if (lane == 0 && c1 > cu) mbar_arrive(S.ldone);
            }
            if (ncL < nch) {
                long long n = 0;
                for (int t = 0; t < ncL; ++t) n += *(const uint16_t*)(P.stream + (size_t)(c0 + t) * SPCG_CHUNK_BYTES);
                C.out = z;
                C.rdot = rdot;
                C.mb = P.mbU;
                if (kind == K_PRO) solver_section_multi<true, true>(C, S, q0, ncL, nch, lseq, rz, sw, rec0 + n);
                else solver_section_multi<true, false>(C, S, q0, ncL, nch, lseq, rz, sw, rec0 + n);
            }
        } else if (ncL > 0) {
            double dummy = 0.0;
            solver_section<false, false>(C, S, q0, 0, ncL, rec0, dummy, P, st.k);
            __syncwarp();
            if (lane == 0 && c1 > cu) {
                mbar_arrive(S.ldone);                              // y of the L section complete
                trace_mark(P, st.k, 8 + 4 * blockIdx.x + 1);
            }
        }
        if (SPCG_NSOLVER == 1 && ncL < nch) {
            long long n = 0;                                        // U records continue the numbering
            for (int t = 0; t < ncL; ++t) n += *(const uint16_t*)(P.stream + (size_t)(c0 + t) * SPCG_CHUNK_BYTES);
            C.out = z;
            C.rdot = rdot;
            C.mb = P.mbU;
            if (kind == K_PRO) solver_section<true, true>(C, S, q0, ncL, nch, rec0 + n, rz, P, st.k);
            else solver_section<true, false>(C, S, q0, ncL, nch, rec0 + n, rz, P, st.k);
        }
        if (lane == 0) trace_mark(P, st.k, 8 + 4 * blockIdx.x + 2);
    }
    // all roles walked the same chunk sequence
    st.q = q0 + nch;
    if (cu > c0 && c1 > cu) st.ldone_uses++;
    __syncthreads();
    // records count for the next phase (every role counts the same)
    if (threadIdx.x == 0) {
        long long n = 0;
        for (int i = 0; i < nch; ++i) n += *(const uint16_t*)(P.stream + (size_t)(c0 + i) * SPCG_CHUNK_BYTES);
        S.progress[SPCG_NSOLVER] = rec0 + n;
    }
    __syncthreads();
    st.rec = S.progress[SPCG_NSOLVER];
    if (threadIdx.x == 0) trace_mark(P, st.k, 8 + 4 * blockIdx.x + 3);
    if (threadIdx.x == 0) {
        for (int i = 0; i < SPCG_NSOLVER; ++i) S.progress[i] = st.rec - 1;
        *S.chain = 0u;                       // the next phase numbers its slices from 0
    }
    __syncthreads();
}

// M = I (K = -1): z = r with the fused update
__device__ void phase_identity(const Params& P, int kind, const double* in, double* out, const double* rdot,
                               double alpha, double& rr, double& rz) {
    const int64_t stride = (int64_t)gridDim.x * BLOCK;
    for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < P.n; i += stride) {
        double ri;
        if (kind == K_ITER) {
            ri = P.r[i] - alpha * P.w[i];
            P.r[i] = ri;
            P.x[i] = P.x[i] + alpha * P.p[i];
        } else {
            ri = in[i];
            if (kind == K_PRO) {
                if (in != P.r) P.r[i] = ri;
                if (!P.use_x0) P.x[i] = 0.0;
                P.p[i] = ri;
            }
        }
        out[i] = ri;
        rr = fma(ri, ri, rr);
        if (rdot) rz = fma(rdot[i], ri, rz);
    }
}

// p = z + beta p  (Alg. 1 line 15)
__device__ void phase_pupdate(const Params& P, double beta) {
    const int64_t stride = (int64_t)gridDim.x * BLOCK;
    for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < P.n; i += stride) P.p[i] = fma(beta, P.p[i], P.z[i]);
}

// Triangular solves of Alg. 1 line 13.  sec: 1 = forward (L) only, 2 = backward
// (U) only, 3 = both (z = U^-1 L^-1 r).  L reads rin, writes y; U reads yin, writes z.
template <int STRAT>
__device__ void tri_solve(const Params& P, int sec, int kind, const double* rin, double* y, const double* yin,
                          double* z, const double* rdot, unsigned ep, double alpha, double& rr, double& rz,
                          double* dyn, unsigned& gen, const ChunkSmem& CS, PipeState& ps) {
    if (P.identity) {
        if (sec == 2) phase_identity(P, K_APPLY, yin, z, rdot, 0.0, rr, rz);
        else phase_identity(P, kind, rin, sec == 1 ? y : z, sec == 3 ? rdot : nullptr, alpha, rr, rz);
        return;
    }
    if (STRAT == ST_CHUNKED) {
        const int c = blockIdx.x;
        const int cb = P.part_chunk[c], cu = P.part_uchunk[c], ce = P.part_chunk[c + 1];
        const int c0 = (sec & 1) ? cb : cu, c1 = (sec & 2) ? ce : cu;
        chunked_phase(P, CS, ps, c0, c1, cu, kind, rin, y, yin, z, rdot, ep, alpha, rr, rz, P.part_begin[c]);
        return;
    }
    if (sec & 1) tri_phase<STRAT, false>(P, P.L, kind, rin, y, nullptr, P.mbL, ep, alpha, rr, dyn, gen);
    if (STRAT == ST_SYNCFREE && sec == 3) grid_sync(P.sc, gen);   // r_i / y_i written by another warp
    if (sec & 2) tri_phase<STRAT, true>(P, P.U, kind, yin, z, rdot, P.mbU, ep, 0.0, rz, dyn, gen);
}

template <int STRAT>
__device__ __forceinline__ void pcg_body(const Params& P, double* dyn) {
    double* ring = dyn;
    unsigned gen = 0;
    if (threadIdx.x == 0) gen = ld_acquire_u32(&P.sc->bar_gen);
    ChunkSmem CS{};
    PipeState ps{0u, 0u, 0ll, -1ll};
    if (STRAT == ST_CHUNKED) {
        CS = chunk_smem(dyn, P.ring);
        for (int i = threadIdx.x; i < P.ring; i += BLOCK) ring[i] = 0.0;
        chunk_init(CS);
    }
    __syncthreads();
    unsigned app = 0;

    if (P.mode != M_SOLVE) {
        double a = 0.0, b = 0.0;
        if (P.mode == M_SPMV) {
            phase_spmv(P.A, P.n, P.in, P.out, a);
        } else if (P.mode == M_LOWER) {
            tri_solve<STRAT>(P, 1, K_APPLY, P.in, P.out, nullptr, nullptr, nullptr, P.epoch, 0.0, a, b, ring, gen, CS, ps);
        } else if (P.mode == M_UPPER) {
            tri_solve<STRAT>(P, 2, K_APPLY, nullptr, nullptr, P.in, P.out, P.aux, P.epoch, 0.0, a, b, ring, gen, CS, ps);
        } else {
            tri_solve<STRAT>(P, 3, K_APPLY, P.in, P.y, P.y, P.out, P.aux, P.epoch, 0.0, a, b, ring, gen, CS, ps);
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

    // ---------------- Alg. 1 lines 1-4: x0, r0 = b - A x0, z0 = M^-1 r0, p0 = z0
    const double* r_src = P.b;
    if (P.use_x0) {
        double dummy = 0.0;
        phase_spmv(P.A, P.n, P.x, P.w, dummy);
        grid_sync(P.sc, gen);
        const int64_t stride = (int64_t)gridDim.x * BLOCK;
        for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < P.n; i += stride) P.r[i] = P.b[i] - P.w[i];
        grid_sync(P.sc, gen);
        r_src = P.r;
    }
    double rr_l = 0.0, rz_l = 0.0;
    tri_solve<STRAT>(P, 3, K_PRO, r_src, P.y, P.y, P.z, P.r, P.epoch + app, 0.0, rr_l, rz_l, ring, gen, CS, ps);
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
        if (__syncthreads_or(ld_volatile_int(&P.sc->abort))) { status = SPCG_ERR_INTERNAL; break; }   // CTA-uniform
        ps.k = k;
        if (threadIdx.x == 0) hbeat(P, 5, (unsigned long long)k);
        if (blockIdx.x == 0 && threadIdx.x == 0) trace_mark(P, k, 0);
        // line 9-10: w = A p, sigma = (p, w), alpha = rho / sigma
        double pw = 0.0;
        phase_spmv(P.A, P.n, P.p, P.w, pw);
        block_partials(pw, 0.0, P.partials, 2, -1);
        grid_sync(P.sc, gen);
        double sigma, unused;
        global_sums(P.partials, 2, -1, sigma, unused);
        if (!(sigma > 0.0) || !isfinite(sigma) || !isfinite(rho)) { status = SPCG_ERR_BREAKDOWN; break; }
        const double alpha = rho / sigma;
        if (blockIdx.x == 0 && threadIdx.x == 0) trace_mark(P, k, 1);
        // lines 11-13 (+ ||r||^2, (r, z))
        rr_l = 0.0;
        rz_l = 0.0;
        tri_solve<STRAT>(P, 3, K_ITER, P.r, P.y, P.y, P.z, P.r, P.epoch + app, alpha, rr_l, rz_l, ring, gen, CS, ps);
        ++app;
        if (blockIdx.x == 0 && threadIdx.x == 0) trace_mark(P, k, 2);
        block_partials(rz_l, rr_l, P.partials, 0, 1);
        grid_sync(P.sc, gen);
        if (blockIdx.x == 0 && threadIdx.x == 0) trace_mark(P, k, 3);
        double rho_new;
        global_sums(P.partials, 0, 1, rho_new, rr);
        // lines 14-15
        const double beta = rho_new / rho;
        rho = rho_new;
        phase_pupdate(P, beta);
        grid_sync(P.sc, gen);
        if (blockIdx.x == 0 && threadIdx.x == 0) trace_mark(P, k, 4);
        ++k;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        P.sc->k = k;
        P.sc->rr = rr;
        P.sc->rho = rho;
        P.sc->status = ld_volatile_int(&P.sc->abort) ? SPCG_ERR_INTERNAL : status;
    }
}

template <int STRAT>
__global__ void __launch_bounds__(BLOCK, SPCG_CTAS_PER_SM) spcg_pcg_kernel(Params P) {
    extern __shared__ __align__(128) double dyn[];
    pcg_body<STRAT>(P, dyn);
}

// RESIDENT executor (small systems, n <= SPCG_RESIDENT_MAX_N): one CTA, every
// vector of Algorithm 1 (x, r, w, p, y, z) held in shared memory for the whole
// solve; the level-scheduled executor runs on them with CTA barriers between
// wavefronts (grid_sync is a __syncthreads for a one-CTA grid), so a wavefront
// handoff costs a CTA barrier (~15 ns) instead of a cross-CTA flag or a grid
// barrier (0.3-1.2 us).  The factors and A stream from L1/L2.
// b is read from global memory by the prologue; x is copied in (use_x0) and
// out at the end.  The single-operator modes run on the caller's global buffers.
__global__ void __launch_bounds__(BLOCK, 1) spcg_resident_kernel(Params P) {
    extern __shared__ __align__(128) double dyn[];
    if (P.mode != M_SOLVE) {
        pcg_body<ST_RESIDENT>(P, dyn);
        return;
    }
    const int64_t n = P.n;
    double* gx = P.x;
    Params Q = P;
    Q.x = dyn;
    Q.r = dyn + n;
    Q.w = dyn + 2 * n;
    Q.p = dyn + 3 * n;
    Q.y = dyn + 4 * n;
    Q.z = dyn + 5 * n;
    if (P.use_x0)
        for (int64_t i = threadIdx.x; i < n; i += BLOCK) Q.x[i] = gx[i];
    __syncthreads();
    pcg_body<ST_RESIDENT>(Q, dyn + 6 * n);
    __syncthreads();
    for (int64_t i = threadIdx.x; i < n; i += BLOCK) gx[i] = Q.x[i];
}

constexpr size_t resident_smem_bytes(int64_t n) { return (size_t)n * 6 * sizeof(double) + RES_STAGE_BYTES; }

// ------------------------------------------------------------------ host side
#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess) {                                                              \
            spcg::set_error(std::string(#call) + ": " + cudaGetErrorString(e_));              \
            return SPCG_ERR_CUDA;                                                             \
        }                                                                                     \
    } while (0)

}  // namespace

struct spcg_device_s {
    int device = 0;
    cudaStream_t stream = nullptr;
    int strategy = ST_CHUNKED;
    int parts = 1;
    size_t smem = 0;
    Params P{};
    DevAllocator A{};                                 // caller's allocator hooks (or cudaMalloc)
    std::vector<std::pair<void*, size_t>> allocs;
    size_t mb_bytes = 0;                              // bytes of each ready-flag array (mbL, mbU)
    int64_t glob_entries = 0;                         // wchain: own-chain dependencies read from global
    int64_t bytes = 0;
    unsigned epoch = 1;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    cudaEvent_t ev_bind = nullptr;   // spcg_dev_set_stream ordering
    unsigned long long* trace = nullptr;
    unsigned long long* hb = nullptr;
    // in-flight solve (spcg_dev_solve_begin .. _end)
    bool pending = false;
    double* pend_hist = nullptr;
    long long pend_cap = 0;
    double pend_eps = 0.0;
    void* sc_host = nullptr;       // pinned copy of the device scalars
    double* hist = nullptr;        // residual history buffer (grown on demand, reused)
    double* stage = nullptr;       // [2n] device copies of host b, x (SPCG_HOST_PTRS), allocated once
    long long hist_cap = 0;
    // setup-time upload: two pinned bounce buffers (the layouts are GBs of pageable
    // std::vector data; a pageable cudaMemcpy runs at a few GB/s), released after create
    void* ub[2] = {nullptr, nullptr};
    cudaEvent_t uev[2] = {nullptr, nullptr};
    // multi-RHS (NEXT-4, wchain_mrhs.cu): six position-major vectors of npos x mr_M, grown on demand
    int mr_M = 0;
    double* mr_vec[12] = {};       // [vector r, w, p, z, y, xp][half]
    double* mr_part = nullptr;
    double* mr_out = nullptr;
};

// debug: copy the heartbeat array while a kernel may still be running (own non-blocking stream)
extern "C" int spcg_dbg_heartbeats(void* handle_dev, unsigned long long* out, int n) {
    spcg_device_t* d = (spcg_device_t*)handle_dev;
    if (!d || !d->hb) return -1;
    int m = std::min(n, 8 * d->parts);
    for (int i = 0; i < m; ++i) out[i] = ((volatile unsigned long long*)d->hb)[i];
    return m;
}

// every device buffer of a handle: the caller's hooks (spcg_options_t.dev_alloc, e.g. the
// PyTorch caching allocator) or cudaMalloc; sizes rounded up to 256 B
static spcg_status_t dev_malloc(spcg_device_t* d, size_t b, void** out) {
    b = (std::max<size_t>(b, 16) + 255) & ~(size_t)255;
    void* p = nullptr;
    if (d->A.alloc) {
        p = d->A.alloc(b, (void*)d->stream, d->A.ctx);
        if (!p) { spcg::set_error("dev_alloc hook returned NULL"); return SPCG_ERR_OOM; }
    } else {
        cudaError_t e = cudaMalloc(&p, b);
        if (e != cudaSuccess) {
            spcg::set_error(std::string("cudaMalloc: ") + cudaGetErrorString(e));
            return e == cudaErrorMemoryAllocation ? SPCG_ERR_OOM : SPCG_ERR_CUDA;
        }
    }
    d->allocs.push_back({p, b});
    d->bytes += (int64_t)b;
    *out = p;
    return SPCG_OK;
}

static void dev_free(spcg_device_t* d, void* p) {
    for (size_t i = 0; i < d->allocs.size(); ++i)
        if (d->allocs[i].first == p) {
            if (d->A.free) d->A.free(p, d->allocs[i].second, (void*)d->stream, d->A.ctx);
            else cudaFree(p);
            d->bytes -= (int64_t)d->allocs[i].second;
            d->allocs.erase(d->allocs.begin() + i);
            return;
        }
}

constexpr size_t UP_BOUNCE = 32u << 20;
// large arrays through the pinned bounce buffers (chunk k: parallel memcpy into buffer
// k & 1 once its previous DMA is done, then an async copy on the handle's stream)
static spcg_status_t h2d_bounced(spcg_device_t* d, void* dst, const void* src, size_t bytes) {
    if (!d->ub[0]) {
        if (cudaMallocHost(&d->ub[0], UP_BOUNCE) != cudaSuccess || cudaMallocHost(&d->ub[1], UP_BOUNCE) != cudaSuccess ||
            cudaEventCreateWithFlags(&d->uev[0], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&d->uev[1], cudaEventDisableTiming) != cudaSuccess) {
            CK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, d->stream));   // no pinned memory: direct
            return SPCG_OK;
        }
    }
    size_t off = 0;
    for (int k = 0; off < bytes; k ^= 1) {
        const size_t m = std::min(UP_BOUNCE, bytes - off);
        CK(cudaEventSynchronize(d->uev[k]));
        char* bd = (char*)d->ub[k];
        const char* sp = (const char*)src + off;
        const int64_t nb = (int64_t)((m + (1u << 20) - 1) >> 20);
#pragma omp parallel for schedule(static)
        for (int64_t b = 0; b < nb; ++b) {
            const size_t o = (size_t)b << 20;
            std::memcpy(bd + o, sp + o, std::min<size_t>(1u << 20, m - o));
        }
        CK(cudaMemcpyAsync((char*)dst + off, bd, m, cudaMemcpyHostToDevice, d->stream));
        CK(cudaEventRecord(d->uev[k], d->stream));
        off += m;
    }
    return SPCG_OK;
}
static void release_bounce(spcg_device_t* d) {
    if (d->ub[0] || d->ub[1]) cudaStreamSynchronize(d->stream);
    for (int k = 0; k < 2; ++k) {
        if (d->uev[k]) cudaEventDestroy(d->uev[k]);
        if (d->ub[k]) cudaFreeHost(d->ub[k]);
        d->uev[k] = nullptr;
        d->ub[k] = nullptr;
    }
}

template <class T, class Al>
static spcg_status_t upload(spcg_device_t* d, const std::vector<T, Al>& v, const T** out) {
    void* p = nullptr;
    const size_t bytes = v.size() * sizeof(T);
    spcg_status_t s = dev_malloc(d, bytes, &p);
    if (s != SPCG_OK) return s;
    if (bytes >= (4u << 20)) {
        s = h2d_bounced(d, p, v.data(), bytes);
        if (s != SPCG_OK) return s;
    } else if (!v.empty()) {
        CK(cudaMemcpyAsync(p, v.data(), bytes, cudaMemcpyHostToDevice, d->stream));
    }
    *out = (const T*)p;
    return SPCG_OK;
}

static spcg_status_t alloc(spcg_device_t* d, size_t b, void** out) { return dev_malloc(d, b, out); }

#define UP(vec, dst)                                           \
    do {                                                       \
        spcg_status_t s_ = upload(d, vec, &(dst));             \
        if (s_ != SPCG_OK) { spcg_dev_destroy(d); return s_; } \
    } while (0)

static spcg_status_t upload_tri(spcg_device_t* d, const spcg::TriLayout& T, DevTri& D) {
    D.nslices = T.nslices;
    D.ngroups = T.ngroups;
    spcg_status_t s;
    if ((s = upload(d, T.eoff, &D.eoff))) return s;
    if ((s = upload(d, T.rows, &D.rows))) return s;
    if ((s = upload(d, T.publish, &D.publish))) return s;
    if ((s = upload(d, T.rlen, &D.rlen))) return s;
    if ((s = upload(d, T.src, &D.src))) return s;
    if ((s = upload(d, T.val, &D.val))) return s;
    if ((s = upload(d, T.dinv, &D.dinv))) return s;
    if ((s = upload(d, T.gptr, &D.gptr))) return s;
    if ((s = upload(d, T.part_gptr, &D.part_gptr))) return s;
    D.wide = T.wide ? 1 : 0;
    if ((s = upload(d, T.wrow, &D.wrow))) return s;
    if ((s = upload(d, T.wptr, &D.wptr))) return s;
    if ((s = upload(d, T.wcol, &D.wcol))) return s;
    if ((s = upload(d, T.wval, &D.wval))) return s;
    if ((s = upload(d, T.wdinv, &D.wdinv))) return s;
    if ((s = upload(d, T.wgptr, &D.wgptr))) return s;
    if ((s = upload(d, T.rrec, &D.rrec))) return s;
    return SPCG_OK;
}

// launch geometry the host setup must use (compile-time knobs of this build)
int spcg_dev_ctas_per_sm() { return SPCG_CTAS_PER_SM; }
int spcg_dev_ring_max() { return SPCG_RING_MAX; }

extern "C" int spcg_dev_sm_count(int device) {
    cudaDeviceProp prop;
    if (cudaSetDevice(device) != cudaSuccess) { spcg::set_error("cudaSetDevice failed"); return -1; }
    if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) { spcg::set_error("no device properties"); return -1; }
    if (prop.major < 10) { spcg::set_error("needs sm_100a (B200)"); return -1; }
    return prop.multiProcessorCount;
}

template <int STRAT>
static void* kernel_ptr() { return (void*)spcg_pcg_kernel<STRAT>; }

void* spcg_wchain_kernel_ptr();   // wchain.cu

static void* pick_kernel(int strategy) {
    switch (strategy) {
        case ST_WCHAIN: return spcg_wchain_kernel_ptr();
        case ST_RESIDENT: return (void*)spcg_resident_kernel;
        case ST_LEVEL: return kernel_ptr<ST_LEVEL>();
        case ST_SYNCFREE: return kernel_ptr<ST_SYNCFREE>();
        default: return kernel_ptr<ST_CHUNKED>();
    }
}

spcg_status_t spcg_dev_create(int device, void* stream, const spcg::Layouts& lay, int64_t n,
                              bool identity_precond, const DevAllocator& alc, spcg_device_t** out,
                              int64_t* bytes) {
    *out = nullptr;
    CK(cudaSetDevice(device));
    spcg_device_t* d = new spcg_device_t();
    d->device = device;
    d->stream = (cudaStream_t)stream;
    d->strategy = lay.strategy;
    d->parts = lay.parts;
    d->A = alc;
    Params& P = d->P;
    P.n = n;
    P.ring = lay.ring;
    P.identity = identity_precond ? 1 : 0;
    const bool wchain = lay.strategy == ST_WCHAIN;
    const spcg::SpmvLayout& AL = wchain ? lay.C.A : lay.A;
    // vectors of Algorithm 1: natural order, or execution (position) order for WCHAIN
    const int64_t nv = wchain ? 32 * lay.C.nsteps : n;
    d->mb_bytes = (size_t)nv * 16;
    P.A.nslices = AL.nslices;
    UP(AL.eoff, P.A.eoff);
    UP(AL.col, P.A.col);
    UP(AL.val, P.A.val);
    if (wchain) {
        const spcg::ChainLayout& CL = lay.C;
        DevChain& D = P.CH;
        D.nchains = CL.nchains;
        D.per_cta = (CL.nchains + lay.parts - 1) / lay.parts;
        D.W_L = CL.W_L;
        D.W_U = CL.W_U;
        D.rec_L = CL.rec_L;
        D.rec_U = CL.rec_U;
        D.vb = CL.vb;
        d->glob_entries = CL.glob_entries;
        D.nsteps = CL.nsteps;
        D.npos = nv;
        spcg::ChainSmemCfg cfg;
        if (D.per_cta > NWARP || !spcg::chain_smem_config(CL, D.per_cta, cfg)) {
            spcg::set_error("warp-chain layout: too many chains per CTA for shared memory");
            spcg_dev_destroy(d);
            return SPCG_ERR_INVALID_ARG;
        }
        D.nst = cfg.nst;
        D.stage_bytes = cfg.stage_bytes;
        D.warp_bytes = cfg.warp_bytes;
        D.ext_off = cfg.ext_off;
        D.hist_off = cfg.hist_off;
        D.WA = CL.WA;
        D.sp_nst = cfg.sp_nst;
        D.sp_stage_bytes = cfg.sp_stage_bytes;
        D.any_ext = CL.ext_entries > 0;
        D.any_hist = CL.hist_entries > 0;
        d->smem = cfg.cta_bytes;
        UP(CL.chain_step, D.chain_step);
        UP(CL.chain_flags, D.chain_flags);
        UP(CL.recL, D.recL);
        UP(CL.recU, D.recU);
        UP(CL.perm, D.perm);
    }
    if (upload_tri(d, lay.L, P.L) || upload_tri(d, lay.U, P.U)) { spcg_dev_destroy(d); return SPCG_ERR_CUDA; }
    UP(lay.part_begin, P.part_begin);
    UP(lay.S.bytes, P.stream);
    UP(lay.S.part_chunk, P.part_chunk);
    UP(lay.S.part_uchunk, P.part_uchunk);
    UP(lay.S.chunk_bytes, P.chunk_bytes);
    void* p;
    const size_t vb = (size_t)nv * sizeof(double);
#define AL(bytes_, dst, T)                                                  \
    do {                                                                    \
        if (alloc(d, bytes_, &p)) { spcg_dev_destroy(d); return SPCG_ERR_OOM; } \
        dst = (T)p;                                                         \
    } while (0)
    AL(vb, P.r, double*);
    AL(vb, P.w, double*);
    AL(vb, P.p, double*);
    AL(vb, P.z, double*);
    AL(vb, P.y, double*);
    if (wchain) {
        AL(vb, P.CH.xp, double*);
        AL(vb, P.CH.bp, double*);
        AL(vb, P.CH.t1, double*);
    }
    AL(d->mb_bytes, P.mbL, uint4*);
    AL(d->mb_bytes, P.mbU, uint4*);
    AL(sizeof(double) * 3 * (size_t)lay.parts, P.partials, double*);
    AL(sizeof(Scal), P.sc, Scal*);
#undef AL
    if (cudaMemsetAsync(P.mbL, 0xFF, d->mb_bytes, d->stream) != cudaSuccess ||
        cudaMemsetAsync(P.mbU, 0xFF, d->mb_bytes, d->stream) != cudaSuccess ||
        cudaMemsetAsync(P.sc, 0, sizeof(Scal), d->stream) != cudaSuccess) {
        spcg_dev_destroy(d);
        return SPCG_ERR_CUDA;
    }
    if (!wchain)
        d->smem = lay.strategy == ST_CHUNKED    ? chunked_smem_bytes(lay.ring)
                  : lay.strategy == ST_RESIDENT ? resident_smem_bytes(n)
                                                : 0;
    void* kfn = pick_kernel(d->strategy);
    // one attribute value for every handle: the largest ring (or resident system) any layout builds
    const int smem_max = lay.strategy == ST_CHUNKED    ? (int)chunked_smem_bytes(SPCG_RING_MAX)
                         : lay.strategy == ST_RESIDENT ? (int)resident_smem_bytes(SPCG_RESIDENT_MAX_N)
                         : wchain                      ? (int)spcg::SPCG_CHAIN_SMEM_LIMIT
                                                       : 0;
    if (cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_max) != cudaSuccess) {
        spcg::set_error("cannot reserve shared memory for the ring");
        spcg_dev_destroy(d);
        return SPCG_ERR_CUDA;
    }
    int nb = 0;
    int sms = spcg_dev_sm_count(device);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kfn, BLOCK, d->smem) != cudaSuccess || nb < 1 ||
        d->parts > nb * sms) {
        spcg::set_error("persistent grid does not fit co-resident");
        spcg_dev_destroy(d);
        return SPCG_ERR_CUDA;
    }
    if (getenv("SPCG_HB")) {
        void* hp = nullptr;
        if (cudaHostAlloc(&hp, sizeof(unsigned long long) * 8 * (size_t)lay.parts, cudaHostAllocMapped) == cudaSuccess) {
            memset(hp, 0, sizeof(unsigned long long) * 8 * (size_t)lay.parts);
            d->hb = (unsigned long long*)hp;                 // host view (zero-copy, readable any time)
            void* dp = nullptr;
            cudaHostGetDevicePointer(&dp, hp, 0);
            P.hb = (unsigned long long*)dp;
        }
    }
    if (getenv("SPCG_TRACE")) {
        void* tp = nullptr;
        if (alloc(d, sizeof(unsigned long long) * (8 + 4 * (size_t)lay.parts + 400), &tp) == SPCG_OK) {
            d->trace = (unsigned long long*)tp;
            P.trace = d->trace;
        }
    }
    if (cudaEventCreate(&d->ev0) != cudaSuccess || cudaEventCreate(&d->ev1) != cudaSuccess) {
        spcg_dev_destroy(d);
        return SPCG_ERR_CUDA;
    }
    if (cudaStreamSynchronize(d->stream) != cudaSuccess) { spcg_dev_destroy(d); return SPCG_ERR_CUDA; }
    release_bounce(d);
    *bytes = d->bytes;
    *out = d;
    return SPCG_OK;
}

void spcg_dev_destroy(spcg_device_t* d) {
    if (!d) return;
    cudaSetDevice(d->device);
    cudaStreamSynchronize(d->stream);
    if (d->sc_host) cudaFreeHost(d->sc_host);
    release_bounce(d);
    for (auto& a : d->allocs) {
        if (d->A.free) d->A.free(a.first, a.second, (void*)d->stream, d->A.ctx);
        else cudaFree(a.first);
    }
    d->allocs.clear();
    if (d->ev0) cudaEventDestroy(d->ev0);
    if (d->ev_bind) cudaEventDestroy(d->ev_bind);
    if (d->ev1) cudaEventDestroy(d->ev1);
    delete d;
}

static void report_abort(spcg_device_t* d, const Scal& sc) {
    char buf[256];
    long long a = sc.dbg_addr;
    long long lo = (long long)(size_t)d->P.mbL, uo = (long long)(size_t)d->P.mbU;
    long long nb = d->P.n * 16;
    const char* which = (a >= lo && a < lo + nb) ? "L" : (a >= uo && a < uo + nb) ? "U" : "barrier";
    long long row = which[0] == 'L' ? (a - lo) / 16 : which[0] == 'U' ? (a - uo) / 16 : -1;
    snprintf(buf, sizeof buf, "device spin timeout: waiting on %s flag of row %lld (epoch want %u seen %u)", which, row,
             sc.dbg_want, sc.dbg_seen);
    spcg::set_error(buf);
}

// Ready-flag epochs are 32-bit and advance by kmax + 3 per solve (kmax <= SPCG_KMAX_LIMIT).
// Before they could wrap, the flag arrays are re-initialised on the stream (0xFF..: the
// epoch 0xFFFFFFFF is never issued) and numbering restarts at 1, so a stale flag can
// never carry a current epoch.
static spcg_status_t reserve_epochs(spcg_device_t* d, unsigned long long need) {
    if ((unsigned long long)d->epoch + need < 0xFFFFFF00ull) return SPCG_OK;
    CK(cudaMemsetAsync(d->P.mbL, 0xFF, d->mb_bytes, d->stream));
    CK(cudaMemsetAsync(d->P.mbU, 0xFF, d->mb_bytes, d->stream));
    d->epoch = 1;
    return SPCG_OK;
}

static spcg_status_t launch(spcg_device_t* d, Params& P) {
    CK(cudaMemsetAsync(P.sc, 0, sizeof(Scal), d->stream));
    void* args[] = {&P};
    if (d->strategy == ST_RESIDENT)   // one CTA: no co-residency requirement
        CK(cudaLaunchKernel(pick_kernel(d->strategy), dim3(1), dim3(BLOCK), args, d->smem, d->stream));
    else
        CK(cudaLaunchCooperativeKernel(pick_kernel(d->strategy), dim3(d->parts), dim3(BLOCK), args, d->smem, d->stream));
    return SPCG_OK;
}

void* spcg_wchain_mrhs_kernel_ptr(int M);     // wchain_mrhs.cu
size_t spcg_mrhs_args_size();
void spcg_mrhs_args_fill(void* dst, int nrhs, const double* B, double* X, double* const* vec, double* partials,
                         double* out, int nst, unsigned stage_bytes, unsigned warp_bytes);

// NEXT-4: nrhs (1..4) right-hand sides of the handle's system together.
// B, X: device, column-major n x nrhs.  Requires the warp-chain executor with a chain
// layout of pure shuffles (no ring / global / flag dependencies), narrow fp64 records and
// the TMA SpMV.  Synchronous; out[m] = {k, ||r_k||^2, status}.
spcg_status_t spcg_dev_solve_multi(spcg_device_t* d, const double* B, double* X, int nrhs, double eps, int64_t kmax,
                                   double* out_host, double* ms) {
    if (d->pending) { spcg::set_error("a solve is already in flight on this handle"); return SPCG_ERR_INVALID_ARG; }
    const DevChain& D = d->P.CH;
    if (d->strategy != ST_WCHAIN || D.any_ext || D.any_hist || d->glob_entries || D.W_L > 4 || D.W_U > 4 ||
        D.vb != 8 || !(D.sp_nst >= 2 && D.WA >= 3 && D.WA <= 8)) {
        spcg::set_error("multi-RHS solve needs the warp-chain executor with shuffle-only chains, narrow fp64 "
                        "records and the TMA SpMV");
        return SPCG_ERR_INVALID_ARG;
    }
    if (nrhs < 1 || nrhs > 4) { spcg::set_error("nrhs must be 1..4 per call"); return SPCG_ERR_INVALID_ARG; }
    const int M = nrhs <= 2 ? 2 : 4;
    const int H = M / 2;                  // right-hand-side halves of two: one chain warp each
    if (H * D.per_cta > NWARP) { spcg::set_error("multi-RHS: too many chains per CTA"); return SPCG_ERR_INVALID_ARG; }
    CK(cudaSetDevice(d->device));
    // stage sizing per chain warp: CC steps of (record + operand slices of 2 x 256 bytes), L
    // needs 4 operands, U 2
    const size_t C = spcg::SPCG_CHAIN_C;
    const size_t stepL = (size_t)D.rec_L + 4 * 512, stepU = (size_t)D.rec_U + 2 * 512;
    const size_t stage = (C * std::max(stepL, stepU) + 127) & ~(size_t)127;
    int nst = (int)std::min<size_t>(16, spcg::SPCG_CHAIN_SMEM_LIMIT / ((size_t)H * D.per_cta * stage));
    if (nst < 2) { spcg::set_error("multi-RHS stages do not fit shared memory"); return SPCG_ERR_INVALID_ARG; }
    const size_t warp_bytes = stage * (size_t)nst;
    const size_t smem = std::max((size_t)H * D.per_cta * warp_bytes, (size_t)8 * D.sp_nst * D.sp_stage_bytes);
    if (M > d->mr_M) {
        CK(cudaStreamSynchronize(d->stream));
        for (auto& v : d->mr_vec)
            if (v) { dev_free(d, v); v = nullptr; }
        if (d->mr_part) { dev_free(d, d->mr_part); d->mr_part = nullptr; }
        if (d->mr_out) { dev_free(d, d->mr_out); d->mr_out = nullptr; }
        d->mr_M = 0;
        void* p;
        for (int k = 0; k < 12; ++k) {        // [vector][half]: r, w, p, z, y, xp
            double*& v = d->mr_vec[k];
            if ((k & 1) >= H) continue;
            spcg_status_t s = dev_malloc(d, sizeof(double) * (size_t)D.npos * 2, &p);
            if (s != SPCG_OK) return s;
            v = (double*)p;
        }
        spcg_status_t s = dev_malloc(d, sizeof(double) * 4 * (size_t)M * d->parts, &p);
        if (s != SPCG_OK) return s;
        d->mr_part = (double*)p;
        s = dev_malloc(d, sizeof(double) * 4 * (size_t)M, &p);
        if (s != SPCG_OK) return s;
        d->mr_out = (double*)p;
        d->mr_M = M;
    }
    void* kfn = spcg_wchain_mrhs_kernel_ptr(M);
    CK(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)spcg::SPCG_CHAIN_SMEM_LIMIT));
    Params P = d->P;
    P.mode = M_SOLVE;
    P.eps = eps;
    P.kmax = kmax;
    std::vector<uint8_t> margs(spcg_mrhs_args_size());
    spcg_mrhs_args_fill(margs.data(), nrhs, B, X, d->mr_vec, d->mr_part, d->mr_out, nst, (unsigned)stage,
                        (unsigned)warp_bytes);
    CK(cudaMemsetAsync(P.sc, 0, sizeof(Scal), d->stream));
    void* args[] = {&P, margs.data()};
    CK(cudaEventRecord(d->ev0, d->stream));
    CK(cudaLaunchCooperativeKernel(kfn, dim3(d->parts), dim3(BLOCK), args, smem, d->stream));
    CK(cudaEventRecord(d->ev1, d->stream));
    CK(cudaMemcpyAsync(out_host, d->mr_out, sizeof(double) * 4 * M, cudaMemcpyDeviceToHost, d->stream));
    Scal sc{};
    CK(cudaMemcpyAsync(&sc, P.sc, sizeof(Scal), cudaMemcpyDeviceToHost, d->stream));
    CK(cudaStreamSynchronize(d->stream));
    float t = 0.f;
    CK(cudaEventElapsedTime(&t, d->ev0, d->ev1));
    *ms = t;
    if (sc.status == SPCG_ERR_INTERNAL) {
        spcg::set_error("multi-RHS solve aborted by its watchdog (internal)");
        return SPCG_ERR_INTERNAL;
    }
    return SPCG_OK;
}

// Enqueue one solve on the handle's stream and return (asynchronous); the scalar
// block is copied into pinned host memory on the same stream.
spcg_status_t spcg_dev_solve_begin(spcg_device_t* d, const double* b, double* x, double eps, int64_t kmax,
                                   bool use_x0) {
    if (d->pending) { spcg::set_error("a solve is already in flight on this handle"); return SPCG_ERR_INVALID_ARG; }
    CK(cudaSetDevice(d->device));
    if (!d->sc_host) CK(cudaMallocHost(&d->sc_host, sizeof(Scal)));
    Params P = d->P;
    P.mode = M_SOLVE;
    P.b = b;
    P.x = x;
    P.eps = eps;
    P.kmax = kmax;
    P.use_x0 = use_x0 ? 1 : 0;
    {
        spcg_status_t es = reserve_epochs(d, (unsigned long long)kmax + 3ull);
        if (es != SPCG_OK) return es;
    }
    P.epoch = d->epoch;
    d->epoch += (unsigned)(kmax + 3);
    long long cap = std::min<long long>(kmax + 1, 1 << 20);
    if (cap > d->hist_cap) {                 // persistent: no allocation on the solve path
        if (d->hist) { CK(cudaStreamSynchronize(d->stream)); dev_free(d, d->hist); d->hist = nullptr; }
        d->hist_cap = std::max<long long>(cap, 1024);
        void* hp = nullptr;
        spcg_status_t hs = dev_malloc(d, sizeof(double) * d->hist_cap, &hp);
        if (hs != SPCG_OK) return hs;
        d->hist = (double*)hp;
    }
    double* dh = d->hist;
    P.rhist = dh;
    P.rhist_cap = cap;
    if (d->trace) CK(cudaMemsetAsync(d->trace, 0, sizeof(unsigned long long) * (8 + 4 * (size_t)d->parts + 400), d->stream));
    CK(cudaEventRecord(d->ev0, d->stream));
    spcg_status_t st = launch(d, P);
    if (st != SPCG_OK) return st;
    CK(cudaEventRecord(d->ev1, d->stream));
    CK(cudaMemcpyAsync(d->sc_host, P.sc, sizeof(Scal), cudaMemcpyDeviceToHost, d->stream));
    d->pending = true;
    d->pend_hist = dh;
    d->pend_cap = cap;
    d->pend_eps = eps;
    return SPCG_OK;
}

// Rebind the handle to another stream.  The new stream waits (on the device,
// through an event) for the work already queued on the old one, so it never
// overtakes it; the host does not block.
spcg_status_t spcg_dev_set_stream(spcg_device_t* d, void* stream) {
    if (d->pending) { spcg::set_error("cannot rebind the stream of a handle with a solve in flight"); return SPCG_ERR_INVALID_ARG; }
    if ((cudaStream_t)stream == d->stream) return SPCG_OK;
    CK(cudaSetDevice(d->device));
    if (!d->ev_bind) CK(cudaEventCreateWithFlags(&d->ev_bind, cudaEventDisableTiming));
    CK(cudaEventRecord(d->ev_bind, d->stream));
    CK(cudaStreamWaitEvent((cudaStream_t)stream, d->ev_bind, 0));
    d->stream = (cudaStream_t)stream;
    return SPCG_OK;
}

// Wait for the in-flight solve and fill info (and the residual history).
spcg_status_t spcg_dev_solve_end(spcg_device_t* d, spcg_solve_info_t* info, std::vector<double>* rhist) {
    if (!d->pending) { spcg::set_error("no solve in flight on this handle"); return SPCG_ERR_INVALID_ARG; }
    d->pending = false;
    CK(cudaSetDevice(d->device));
    CK(cudaStreamSynchronize(d->stream));
    const Scal sc = *(const Scal*)d->sc_host;
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, d->ev0, d->ev1));
    const long long cap = d->pend_cap;
    double* dh = d->pend_hist;
    long long kk = std::min<long long>(sc.k, cap - 1);
    if (rhist) {
        rhist->assign(kk + 1, 0.0);
        CK(cudaMemcpyAsync(rhist->data(), dh, sizeof(double) * (kk + 1), cudaMemcpyDeviceToHost, d->stream));
    }
    if (rhist) CK(cudaStreamSynchronize(d->stream));
    info->iterations = sc.k;
    info->rnorm = std::sqrt(sc.rr);
    info->status = sc.status;
    info->converged = (sc.status == SPCG_OK && d->pend_eps > 0.0) ? 1 : 0;
    info->iter_phase_ms = ms;
    if (sc.status == SPCG_ERR_INTERNAL) report_abort(d, sc);
    if (d->trace) {
        std::vector<unsigned long long> t(8 + 4 * (size_t)d->parts + 400);
        cudaMemcpy(t.data(), d->trace, t.size() * 8, cudaMemcpyDeviceToHost);
        if (FILE* f = fopen(getenv("SPCG_TRACE"), "a")) {
            fprintf(f, "trace parts=%d", d->parts);
            for (auto v : t) fprintf(f, " %llu", v);
            fprintf(f, "\n");
            fclose(f);
        }
    }
    return sc.status;
}

spcg_status_t spcg_dev_solve(spcg_device_t* d, const double* b, double* x, double eps, int64_t kmax, bool use_x0,
                             spcg_solve_info_t* info, std::vector<double>* rhist) {
    spcg_status_t st = spcg_dev_solve_begin(d, b, x, eps, kmax, use_x0);
    if (st != SPCG_OK) return st;
    return spcg_dev_solve_end(d, info, rhist);
}

spcg_status_t spcg_dev_apply(spcg_device_t* d, int op, const double* in, double* out, const double* aux,
                             double* scalar_out) {
    CK(cudaSetDevice(d->device));
    Params P = d->P;
    P.mode = op;
    P.in = in;
    P.out = out;
    P.aux = aux;
    {
        spcg_status_t es = reserve_epochs(d, 1ull);
        if (es != SPCG_OK) return es;
    }
    P.epoch = d->epoch;
    d->epoch += 1;
    P.rhist = nullptr;
    spcg_status_t st = launch(d, P);
    if (st != SPCG_OK) return st;
    Scal sc;
    CK(cudaMemcpyAsync(&sc, P.sc, sizeof(Scal), cudaMemcpyDeviceToHost, d->stream));
    CK(cudaStreamSynchronize(d->stream));
    if (scalar_out) *scalar_out = sc.out_scalar;
    if (sc.status == SPCG_ERR_INTERNAL) report_abort(d, sc);
    return sc.status;
}

// kind: 1 H2D, 2 D2H, -1 allocate (dst is void**), -2 free (dst is the pointer)
spcg_status_t spcg_dev_copy(spcg_device_t* d, void* dst, const void* src, size_t bytes, int kind) {
    CK(cudaSetDevice(d->device));
    if (kind == -1) {          // the handle's staging buffer for host b, x: [0, n) and [n, 2n)
        if (!d->stage) {
            void* sp = nullptr;
            spcg_status_t ss = dev_malloc(d, 2 * sizeof(double) * (size_t)d->P.n, &sp);
            if (ss != SPCG_OK) return ss;
            d->stage = (double*)sp;
        }
        *(double**)dst = d->stage;
        return SPCG_OK;
    }
    CK(cudaMemcpyAsync(dst, src, bytes, kind == 1 ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost, d->stream));
    CK(cudaStreamSynchronize(d->stream));
    return SPCG_OK;
}

// debug: slow-path counters (env SPCG_COUNT)
extern "C" int spcg_dbg_counts(unsigned long long* out) {
    static unsigned long long* d = nullptr;
    if (!d) {
        if (cudaMalloc(&d, 128) != cudaSuccess) return -1;
        cudaMemset(d, 0, 128);
        cudaMemcpyToSymbol(g_dbg_counts, &d, sizeof(d));
        return 0;
    }
    cudaMemcpy(out, d, 128, cudaMemcpyDeviceToHost);
    cudaMemset(d, 0, 128);
    return 1;
}
