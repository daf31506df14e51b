// dev_common.cuh — device-side structures and primitives shared by the executors
// (kernels.cu: level / sync-free / chunked / resident; wchain.cu: warp-chain).
// Each translation unit gets its own copy (anonymous namespace).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include "internal.h"

namespace {


#ifndef SPCG_BLOCK
#define SPCG_BLOCK 256            // threads per persistent CTA (128: 4-warp CTAs, two per SM)
#endif
constexpr int BLOCK = SPCG_BLOCK;
#ifndef SPCG_CTAS_PER_SM
#define SPCG_CTAS_PER_SM (SPCG_BLOCK == 128 ? 2 : 1)   // persistent CTAs per SM (independent chains per SM)
#endif
#ifndef SPCG_RING_MAX
#define SPCG_RING_MAX (SPCG_CTAS_PER_SM > 1 ? 4096 : 8192)   // shared-memory ring entries (power of two)
#endif
constexpr int NWARP = BLOCK / 32;
constexpr long long SPIN_TIMEOUT_CYC = 8ll * 1000 * 1000 * 1000;            // ~4 s of SM cycles: abort, never hang

enum { ST_LEVEL = SPCG_SPTRSV_LEVEL, ST_SYNCFREE = SPCG_SPTRSV_SYNCFREE, ST_CHUNKED = SPCG_SPTRSV_CHUNKED,
       ST_RESIDENT = SPCG_SPTRSV_RESIDENT, ST_WCHAIN = SPCG_SPTRSV_WCHAIN };
enum { K_APPLY = 0, K_PRO = 1, K_ITER = 2 };
enum { M_SOLVE = 0, M_SPMV = 1, M_LOWER = 2, M_UPPER = 3, M_PRECOND = 4 };

struct DevTri {
    int32_t nslices, ngroups;
    const int64_t* eoff;
    const int32_t* rows;
    const uint8_t* publish;
    const int32_t* rlen;
    const int32_t* src;
    const double* val;
    const double* dinv;
    const int32_t* gptr;
    const int32_t* part_gptr;
    int32_t wide;                  // LEVEL, wide rows: warp-per-row CSR below (layout.cpp)
    const int32_t* wrow;
    const int64_t* wptr;
    const int32_t* wcol;
    const double* wval;
    const double* wdinv;
    const int32_t* wgptr;
    const uint8_t* rrec;           // RESIDENT: 64-byte slot records (layout.cpp)
};

struct DevA {
    int32_t nslices;
    const int64_t* eoff;
    const int32_t* col;
    const double* val;
};

struct Scal {
    unsigned bar_count, bar_gen;
    int abort;
    int status;
    long long k;
    double rr, rho;
    double out_scalar;
    long long dbg_addr;       // first spin timeout: which flag slot, epochs seen/wanted
    unsigned dbg_want, dbg_seen;
};

// warp-chain executor (wchain.cu; layout: chain_layout.cpp, internal.h ChainLayout)
struct DevChain {
    int32_t nchains, per_cta;      // chains, solver warps per CTA (chain c -> CTA c % grid, warp c / grid)
    int32_t nst;                   // stages per solver warp (SPCG_CHAIN_C steps each)
    int32_t W_L, W_U, rec_L, rec_U;
    int32_t vb;                    // bytes per factor value in the records (8, or 4: fp32 factors)
    int32_t any_ext, any_hist;
    uint32_t stage_bytes, warp_bytes, ext_off, hist_off;
    int32_t WA, sp_nst;            // SpMV: uniform slice width, TMA stages per warp (0: register path)
    uint32_t sp_stage_bytes;
    int64_t nsteps, npos;
    const int64_t* chain_step;     // [nchains+1]
    const uint32_t* chain_flags;   // [nchains] CC_*
    const uint8_t* recL;
    const uint8_t* recU;
    const int32_t* perm;           // [npos] row at each position, -1 padding
    double* xp;                    // x in position order
    double* bp;                    // b (or the apply-mode input) in position order
    double* t1;                    // apply-mode temporary (position order)
};

struct Params {
    int64_t n;
    int ring;
    int identity;
    int mode;
    int use_x0;
    unsigned epoch;
    double eps;
    long long kmax;
    DevA A;
    DevTri L, U;
    const int64_t* part_begin;
    const uint8_t* stream;         // chunked executor: record stream (SPCG_CHUNK_BYTES per chunk)
    const int32_t* part_chunk;     // [parts+1]
    const int32_t* part_uchunk;    // [parts]
    const unsigned* chunk_bytes;   // used bytes of every chunk
    const double* b;
    double* x;
    double* r;
    double* w;
    double* p;
    double* z;
    double* y;
    const double* in;      // apply modes
    double* out;
    const double* aux;
    uint4* mbL;
    uint4* mbU;
    double* partials;      // [3][gridDim.x]
    Scal* sc;
    double* rhist;
    long long rhist_cap;
    unsigned long long* trace;     // debug timeline (env SPCG_TRACE), see trace_mark
    unsigned long long* hb;        // debug heartbeats [parts][8] (env SPCG_TRACE), see hbeat
    DevChain CH;
};
// heartbeat: role slot of this CTA <- (iteration << 40) | (phase step << 20) | value
__device__ __forceinline__ void hbeat(const Params& P, int role, unsigned long long v) {
    if (P.hb) *(volatile unsigned long long*)(P.hb + 8 * blockIdx.x + role) = v;
}

// Debug timeline: globaltimer stamps of iteration TRACE_IT.  [0..7] CTA 0 phase
// boundaries; [8 + 4c + e] per-CTA solver events (e: 0 first L record, 1 L done,
// 2 U done, 3 phase end).
constexpr int TRACE_IT = 2;
__device__ __forceinline__ void trace_max(const Params& P, long long k, int idx) {
    if (P.trace && k == TRACE_IT && blockIdx.x == 0 && idx < 400) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        atomicMax(P.trace + 8 + 4 * gridDim.x + idx, t);
    }
}
__device__ __forceinline__ void trace_x(const Params& P, long long k, int idx) {
    if (P.trace && k == TRACE_IT && blockIdx.x == 0 && idx < 400) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        P.trace[8 + 4 * gridDim.x + idx] = t;
    }
}
__device__ __forceinline__ void trace_mark(const Params& P, long long k, int idx) {
    if (P.trace && k == TRACE_IT) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        P.trace[idx] = t;
    }
}

// ------------------------------------------------------------------ primitives
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_volatile_int(const int* p) {
    int v;
    asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void ll_store(uint4* p, double v, unsigned ep) {
    unsigned long long b = (unsigned long long)__double_as_longlong(v);
    asm volatile("st.volatile.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"((unsigned)b), "r"(ep),
                 "r"((unsigned)(b >> 32)), "r"(ep)
                 : "memory");
}

__device__ __noinline__ double ll_wait_slow(const uint4* p, unsigned ep, Scal* sc) {
    const long long t0 = clock64();
    unsigned a, e1, c, e2;
    for (;;) {
        asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(a), "=r"(e1), "=r"(c), "=r"(e2)
                     : "l"(p)
                     : "memory");
        if (e1 == ep && e2 == ep) break;
        if (ld_volatile_int(&sc->abort)) return 0.0;
        if (clock64() - t0 > SPIN_TIMEOUT_CYC) {
            if (atomicExch(&sc->abort, 1) == 0) {
                sc->dbg_addr = (long long)(size_t)p;
                sc->dbg_want = ep;
                sc->dbg_seen = e1;
            }
            return 0.0;
        }
    }
    return __longlong_as_double((long long)(((unsigned long long)c << 32) | a));
}

__device__ __forceinline__ double ll_wait(const uint4* p, unsigned ep, Scal* sc) {
    unsigned a, e1, c, e2;
    asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(a), "=r"(e1), "=r"(c), "=r"(e2)
                 : "l"(p)
                 : "memory");
    if (e1 == ep && e2 == ep) return __longlong_as_double((long long)(((unsigned long long)c << 32) | a));
    return ll_wait_slow(p, ep, sc);
}

// grid-wide barrier (all CTAs co-resident: cooperative launch).  Monotonic
// arrival counter (zeroed per launch with the Scal block): CTA thread 0 adds 1
// with a release reduction (no round trip) and spins with acquire loads until
// the counter reaches gen x gridDim — one L2 hop less than counter + reset +
// generation flag (calibrated by spcg_calibrate, grid_sync_ns).
__device__ __forceinline__ void red_release_add(unsigned* p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void grid_sync(Scal* sc, unsigned& gen) {
    __syncthreads();
    if (gridDim.x > 1) {
        if (threadIdx.x == 0) {
            const unsigned target = (gen + 1) * gridDim.x;
            red_release_add(&sc->bar_count, 1u);
            const long long t0 = clock64();
            while ((int)(ld_acquire_u32(&sc->bar_count) - target) < 0) {
                if (ld_volatile_int(&sc->abort)) break;
                if (clock64() - t0 > SPIN_TIMEOUT_CYC) { atomicExch(&sc->abort, 1); break; }
            }
        }
        ++gen;
        __syncthreads();
    }
}

// per-CTA partial sums (fixed order) -> partials[slot][blockIdx.x]
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ void block_partials(double a, double b, double* partials, int slot_a, int slot_b) {
    __shared__ double red[2][NWARP];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    a = warp_sum(a);
    b = warp_sum(b);
    if (lane == 0) { red[0][warp] = a; red[1][warp] = b; }
    __syncthreads();
    if (warp == 0) {
        double x = lane < NWARP ? red[0][lane] : 0.0;
        double y = lane < NWARP ? red[1][lane] : 0.0;
        x = warp_sum(x);
        y = warp_sum(y);
        if (lane == 0) {
            if (slot_a >= 0) partials[slot_a * gridDim.x + blockIdx.x] = x;
            if (slot_b >= 0) partials[slot_b * gridDim.x + blockIdx.x] = y;
        }
    }
    __syncthreads();
}

// every CTA sums the G partials in the same order -> identical bits everywhere
__device__ void global_sums(const double* partials, int slot_a, int slot_b, double& a, double& b) {
    __shared__ double bc[2];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (warp == 0) {
        double x = 0.0, y = 0.0;
        for (int i = lane; i < (int)gridDim.x; i += 32) {
            x += __ldcg(partials + slot_a * gridDim.x + i);
            if (slot_b >= 0) y += __ldcg(partials + slot_b * gridDim.x + i);
        }
        x = warp_sum(x);
        y = warp_sum(y);
        if (lane == 0) { bc[0] = x; bc[1] = y; }
    }
    __syncthreads();
    a = bc[0];
    b = bc[1];
    __syncthreads();
}

// ------------------------------------------------------------------ phases
// w = A p (SELL-32, thread per row) and the partial (p, w).  A warp takes SU
// consecutive slices per step and issues all their index/value loads, then all
// gathers of p, then the FMA chains (k ascending per row, as the definition):
// SU x SK independent loads in flight instead of one dependent chain.
constexpr int SU = 4, SK = 4;
__device__ void phase_spmv(const DevA& A, int64_t nrows, const double* pin, double* wout, double& pw) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t ns = A.nslices;
    const int64_t stride = (int64_t)gridDim.x * NWARP * SU;
    for (int64_t s0 = ((int64_t)blockIdx.x * NWARP + warp) * SU; s0 < ns; s0 += stride) {
        const int64_t eo = (lane <= SU && s0 + lane <= ns) ? __ldg(A.eoff + s0 + lane) : 0;
        int64_t e[SU];
        int wd[SU];
        int wmax = 0;
#pragma unroll
        for (int u = 0; u < SU; ++u) {
            e[u] = __shfl_sync(0xffffffffu, eo, u);
            const int64_t e1 = __shfl_sync(0xffffffffu, eo, u + 1);
            wd[u] = (s0 + u < ns) ? (int)(e1 - e[u]) : 0;
            wmax = max(wmax, wd[u]);
        }
        double acc[SU];
#pragma unroll
        for (int u = 0; u < SU; ++u) acc[u] = 0.0;
        for (int kb = 0; kb < wmax; kb += SK) {
            int c[SU][SK];
            double v[SU][SK], g[SU][SK];
#pragma unroll
            for (int u = 0; u < SU; ++u)
#pragma unroll
                for (int k = 0; k < SK; ++k) {
                    const bool on = kb + k < wd[u];
                    const int64_t idx = (e[u] + kb + k) * 32 + lane;
                    c[u][k] = on ? __ldg(A.col + idx) : 0;
                    v[u][k] = on ? __ldg(A.val + idx) : 0.0;
                }
#pragma unroll
            for (int u = 0; u < SU; ++u)
#pragma unroll
                for (int k = 0; k < SK; ++k) g[u][k] = pin[c[u][k]];
#pragma unroll
            for (int u = 0; u < SU; ++u)
#pragma unroll
                for (int k = 0; k < SK; ++k)
                    if (kb + k < wd[u]) acc[u] = fma(v[u][k], g[u][k], acc[u]);
        }
#pragma unroll
        for (int u = 0; u < SU; ++u) {
            const int64_t row = (s0 + u) * 32 + lane;
            if (s0 + u < ns && row < nrows) {
                wout[row] = acc[u];
                pw = fma(pin[row], acc[u], pw);
            }
        }
    }
}


__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
#ifndef SPCG_MBAR_SUSPEND_NS
#define SPCG_MBAR_SUSPEND_NS 20000   // try_wait suspend-time hint (ns): the warp sleeps until the phase completes
#endif
__device__ __forceinline__ bool mbar_try(uint64_t* b, unsigned parity) {
    unsigned ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(b)), "r"(parity), "r"((unsigned)SPCG_MBAR_SUSPEND_NS)   // HW sleep until the phase completes
        : "memory");
    return ok != 0;
}
// returns false if the wait was abandoned because of an abort (callers make
// that warp-uniform before acting on it)
__device__ __noinline__ bool mbar_wait_slow(uint64_t* b, unsigned parity, Scal* sc) {
    const long long t0 = clock64();
    unsigned it = 0;
    while (!mbar_try(b, parity)) {
        if ((++it & 3) == 0) {
            if (ld_volatile_int(&sc->abort)) return false;
            if (clock64() - t0 > SPIN_TIMEOUT_CYC) { atomicExch(&sc->abort, 1); return false; }
        }
    }
    return true;
}
__device__ __forceinline__ bool mbar_wait(uint64_t* b, unsigned parity, Scal* sc) {
    return mbar_try(b, parity) || mbar_wait_slow(b, parity, sc);
}
__device__ __forceinline__ bool warp_ok(bool ok) { return __all_sync(0xffffffffu, ok); }
// Poller -> solver handoff of a resolved external sum through shared memory:
// the poller stores the value, fences (acq_rel, CTA scope: orders its two
// shared-memory stores without waiting for the SM's outstanding global
// stores, which membar.cta = fence.sc.cta would), then sets the mask bit; the
// solver reads the mask and then the value with volatile loads (kept in program
// order by the compiler; shared-memory accesses of one thread are performed
// in order).  No fence on the solver's critical path.
__device__ __forceinline__ void fence_acq_rel_cta() { asm volatile("fence.acq_rel.cta;" ::: "memory"); }
__device__ __forceinline__ double lds_volatile(const double* p) { return *(const volatile double*)p; }
// the solver's read of the poller's mask: an acquire load (CTA scope) pairs with the
// poller's fence.acq_rel + atomicOr, so the value load after it sees the value store
__device__ __forceinline__ unsigned lds_acquire_u32(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
    return v;
}
// After an abort the ring may hold stale chunks: roles must stop parsing them.
// Warp-collective code must take this decision warp-uniformly (a per-lane read
// of a racy flag lets lanes disagree; a divergent break then deadlocks the
// warp at its next __syncwarp / shuffle).
__device__ __forceinline__ bool aborted(Scal* sc) {
    return __any_sync(0xffffffffu, ld_volatile_int(&sc->abort) != 0);
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

}  // namespace
