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
#include <cstring>
#include <vector>

#include "internal.h"

namespace {

constexpr int BLOCK = 512;
constexpr int NWARP = BLOCK / 32;
constexpr unsigned long long SPIN_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;   // 20 s: abort, never hang

enum { ST_LEVEL = SPCG_SPTRSV_LEVEL, ST_SYNCFREE = SPCG_SPTRSV_SYNCFREE, ST_CHUNKED = SPCG_SPTRSV_CHUNKED };
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
};

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
    unsigned long long t0 = gtimer();
    unsigned a, e1, c, e2;
    for (;;) {
        asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(a), "=r"(e1), "=r"(c), "=r"(e2)
                     : "l"(p)
                     : "memory");
        if (e1 == ep && e2 == ep) break;
        if (ld_volatile_int(&sc->abort)) return 0.0;
        if (gtimer() - t0 > SPIN_TIMEOUT_NS) {
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

// grid-wide barrier (all CTAs co-resident: cooperative launch)
__device__ __forceinline__ void grid_sync(Scal* sc, unsigned& gen) {
    __syncthreads();
    if (gridDim.x > 1) {
        if (threadIdx.x == 0) {
            unsigned g = gen;
            __threadfence();
            unsigned prev = atomicAdd(&sc->bar_count, 1u);
            if (prev == gridDim.x - 1) {
                atomicExch(&sc->bar_count, 0u);
                __threadfence();
                st_release_u32(&sc->bar_gen, g + 1);
            } else {
                unsigned long long t0 = gtimer();
                while (ld_acquire_u32(&sc->bar_gen) == g) {
                    if (ld_volatile_int(&sc->abort)) break;
                    if (gtimer() - t0 > SPIN_TIMEOUT_NS) { atomicExch(&sc->abort, 1); break; }
                }
            }
            gen = g + 1;
        }
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
// w = A p (SELL-32, thread per row) and the partial (p, w)
__device__ void phase_spmv(const Params& P, const double* pin, double* wout, double& pw) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t W = (int64_t)gridDim.x * NWARP;
    for (int64_t s = (int64_t)blockIdx.x * NWARP + warp; s < P.A.nslices; s += W) {
        const int64_t e0 = P.A.eoff[s];
        const int wd = (int)(P.A.eoff[s + 1] - e0);
        const int32_t* cp = P.A.col + e0 * 32 + lane;
        const double* vp = P.A.val + e0 * 32 + lane;
        double acc = 0.0;
#pragma unroll 4
        for (int k = 0; k < wd; ++k) acc = fma(__ldg(vp + 32 * k), pin[__ldg(cp + 32 * k)], acc);
        const int64_t row = s * 32 + lane;
        if (row < P.n) {
            wout[row] = acc;
            pw = fma(pin[row], acc, pw);
        }
    }
}

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
        for (int k = 0; k < len; ++k) {
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

template <int STRAT, bool UPPER>
__device__ void tri_phase(const Params& P, const DevTri& T, int kind, const double* in, double* out,
                          const double* rdot, uint4* mb, unsigned ep, double alpha, double& acc_dot,
                          double* ring, unsigned& gen) {
    const int warp = threadIdx.x >> 5;
    if (STRAT == ST_LEVEL) {
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
    } else {
        const int c = blockIdx.x;
        const int64_t pb = P.part_begin[c];
        const int mask = P.ring - 1;
        const int g0 = __ldg(T.part_gptr + c), g1 = __ldg(T.part_gptr + c + 1);
        for (int g = g0; g < g1; ++g) {
            const int s0 = __ldg(T.gptr + g), s1 = __ldg(T.gptr + g + 1);
            for (int s = s0 + warp; s < s1; s += NWARP)
                tri_slice<STRAT, UPPER>(P, T, s, kind, in, out, rdot, mb, ep, alpha, acc_dot, ring, pb, mask);
            __syncthreads();
        }
    }
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

// z = M^-1 r : forward then backward solve (or identity)
template <int STRAT>
__device__ void precond(const Params& P, int kind, const double* rin, double* y, double* z, const double* rdot,
                        unsigned ep, double alpha, double& rr, double& rz, double* ring, unsigned& gen) {
    if (P.identity) {
        phase_identity(P, kind, rin, z, rdot, alpha, rr, rz);
        return;
    }
    tri_phase<STRAT, false>(P, P.L, kind, rin, y, nullptr, P.mbL, ep, alpha, rr, ring, gen);
    if (STRAT == ST_SYNCFREE) grid_sync(P.sc, gen);   // r_i / y_i written by another warp
    tri_phase<STRAT, true>(P, P.U, kind, y, z, rdot, P.mbU, ep, 0.0, rz, ring, gen);
}

template <int STRAT>
__global__ void __launch_bounds__(BLOCK, 1) spcg_pcg_kernel(Params P) {
    extern __shared__ double ring[];
    unsigned gen = 0;
    if (threadIdx.x == 0) gen = ld_acquire_u32(&P.sc->bar_gen);
    if (STRAT == ST_CHUNKED)
        for (int i = threadIdx.x; i < P.ring; i += BLOCK) ring[i] = 0.0;
    __syncthreads();
    unsigned app = 0;

    if (P.mode != M_SOLVE) {
        double a = 0.0, b = 0.0;
        if (P.mode == M_SPMV) {
            phase_spmv(P, P.in, P.out, a);
        } else if (P.mode == M_LOWER) {
            if (P.identity) phase_identity(P, K_APPLY, P.in, P.out, nullptr, 0.0, a, b);
            else tri_phase<STRAT, false>(P, P.L, K_APPLY, P.in, P.out, nullptr, P.mbL, P.epoch, 0.0, a, ring, gen);
        } else if (P.mode == M_UPPER) {
            if (P.identity) phase_identity(P, K_APPLY, P.in, P.out, P.aux, 0.0, a, b);
            else tri_phase<STRAT, true>(P, P.U, K_APPLY, P.in, P.out, P.aux, P.mbU, P.epoch, 0.0, b, ring, gen);
        } else {
            precond<STRAT>(P, K_APPLY, P.in, P.y, P.out, P.aux, P.epoch, 0.0, a, b, ring, gen);
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
        phase_spmv(P, P.x, P.w, dummy);
        grid_sync(P.sc, gen);
        const int64_t stride = (int64_t)gridDim.x * BLOCK;
        for (int64_t i = (int64_t)blockIdx.x * BLOCK + threadIdx.x; i < P.n; i += stride) P.r[i] = P.b[i] - P.w[i];
        grid_sync(P.sc, gen);
        r_src = P.r;
    }
    double rr_l = 0.0, rz_l = 0.0;
    precond<STRAT>(P, K_PRO, r_src, P.y, P.z, P.r, P.epoch + app, 0.0, rr_l, rz_l, ring, gen);
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
        if (ld_volatile_int(&P.sc->abort)) { status = SPCG_ERR_INTERNAL; break; }
        // line 9-10: w = A p, sigma = (p, w), alpha = rho / sigma
        double pw = 0.0;
        phase_spmv(P, P.p, P.w, pw);
        block_partials(pw, 0.0, P.partials, 2, -1);
        grid_sync(P.sc, gen);
        double sigma, unused;
        global_sums(P.partials, 2, -1, sigma, unused);
        if (!(sigma > 0.0) || !isfinite(sigma) || !isfinite(rho)) { status = SPCG_ERR_BREAKDOWN; break; }
        const double alpha = rho / sigma;
        // lines 11-13 (+ ||r||^2, (r, z))
        rr_l = 0.0;
        rz_l = 0.0;
        precond<STRAT>(P, K_ITER, P.r, P.y, P.z, P.r, P.epoch + app, alpha, rr_l, rz_l, ring, gen);
        ++app;
        block_partials(rz_l, rr_l, P.partials, 0, 1);
        grid_sync(P.sc, gen);
        double rho_new;
        global_sums(P.partials, 0, 1, rho_new, rr);
        // lines 14-15
        const double beta = rho_new / rho;
        rho = rho_new;
        phase_pupdate(P, beta);
        grid_sync(P.sc, gen);
        ++k;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        P.sc->k = k;
        P.sc->rr = rr;
        P.sc->rho = rho;
        P.sc->status = ld_volatile_int(&P.sc->abort) ? SPCG_ERR_INTERNAL : status;
    }
}

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
    std::vector<void*> allocs;
    int64_t bytes = 0;
    unsigned epoch = 1;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
};

template <class T>
static spcg_status_t upload(spcg_device_t* d, const std::vector<T>& v, const T** out) {
    void* p = nullptr;
    size_t b = std::max<size_t>(v.size() * sizeof(T), 16);
    CK(cudaMalloc(&p, b));
    d->allocs.push_back(p);
    d->bytes += (int64_t)b;
    if (!v.empty()) CK(cudaMemcpyAsync(p, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice, d->stream));
    *out = (const T*)p;
    return SPCG_OK;
}

static spcg_status_t alloc(spcg_device_t* d, size_t b, void** out) {
    void* p = nullptr;
    CK(cudaMalloc(&p, std::max<size_t>(b, 16)));
    d->allocs.push_back(p);
    d->bytes += (int64_t)b;
    *out = p;
    return SPCG_OK;
}

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
    return SPCG_OK;
}

extern "C" int spcg_dev_sm_count(int device) {
    cudaDeviceProp prop;
    if (cudaSetDevice(device) != cudaSuccess) { spcg::set_error("cudaSetDevice failed"); return -1; }
    if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) { spcg::set_error("no device properties"); return -1; }
    if (prop.major < 10) { spcg::set_error("needs sm_100a (B200)"); return -1; }
    return prop.multiProcessorCount;
}

template <int STRAT>
static void* kernel_ptr() { return (void*)spcg_pcg_kernel<STRAT>; }

static void* pick_kernel(int strategy) {
    switch (strategy) {
        case ST_LEVEL: return kernel_ptr<ST_LEVEL>();
        case ST_SYNCFREE: return kernel_ptr<ST_SYNCFREE>();
        default: return kernel_ptr<ST_CHUNKED>();
    }
}

spcg_status_t spcg_dev_create(int device, void* stream, const spcg::Layouts& lay, int64_t n,
                              bool identity_precond, spcg_device_t** out, int64_t* bytes) {
    *out = nullptr;
    CK(cudaSetDevice(device));
    spcg_device_t* d = new spcg_device_t();
    d->device = device;
    d->stream = (cudaStream_t)stream;
    d->strategy = lay.strategy;
    d->parts = lay.parts;
    Params& P = d->P;
    P.n = n;
    P.ring = lay.ring;
    P.identity = identity_precond ? 1 : 0;
    P.A.nslices = lay.A.nslices;
    UP(lay.A.eoff, P.A.eoff);
    UP(lay.A.col, P.A.col);
    UP(lay.A.val, P.A.val);
    if (upload_tri(d, lay.L, P.L) || upload_tri(d, lay.U, P.U)) { spcg_dev_destroy(d); return SPCG_ERR_CUDA; }
    UP(lay.part_begin, P.part_begin);
    void* p;
    const size_t vb = (size_t)n * sizeof(double);
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
    AL((size_t)n * 16, P.mbL, uint4*);
    AL((size_t)n * 16, P.mbU, uint4*);
    AL(sizeof(double) * 3 * (size_t)lay.parts, P.partials, double*);
    AL(sizeof(Scal), P.sc, Scal*);
#undef AL
    if (cudaMemsetAsync(P.mbL, 0xFF, (size_t)n * 16, d->stream) != cudaSuccess ||
        cudaMemsetAsync(P.mbU, 0xFF, (size_t)n * 16, d->stream) != cudaSuccess ||
        cudaMemsetAsync(P.sc, 0, sizeof(Scal), d->stream) != cudaSuccess) {
        spcg_dev_destroy(d);
        return SPCG_ERR_CUDA;
    }
    d->smem = lay.strategy == ST_CHUNKED ? (size_t)lay.ring * sizeof(double) : 0;
    void* kfn = pick_kernel(d->strategy);
    // one attribute value for every handle: the largest ring any layout builds (16384 entries)
    if (cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384 * (int)sizeof(double)) != cudaSuccess) {
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
    if (cudaEventCreate(&d->ev0) != cudaSuccess || cudaEventCreate(&d->ev1) != cudaSuccess) {
        spcg_dev_destroy(d);
        return SPCG_ERR_CUDA;
    }
    if (cudaStreamSynchronize(d->stream) != cudaSuccess) { spcg_dev_destroy(d); return SPCG_ERR_CUDA; }
    *bytes = d->bytes;
    *out = d;
    return SPCG_OK;
}

void spcg_dev_destroy(spcg_device_t* d) {
    if (!d) return;
    cudaSetDevice(d->device);
    cudaStreamSynchronize(d->stream);
    for (void* p : d->allocs) cudaFree(p);
    if (d->ev0) cudaEventDestroy(d->ev0);
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

static spcg_status_t launch(spcg_device_t* d, Params& P) {
    CK(cudaMemsetAsync(P.sc, 0, sizeof(Scal), d->stream));
    void* args[] = {&P};
    CK(cudaLaunchCooperativeKernel(pick_kernel(d->strategy), dim3(d->parts), dim3(BLOCK), args, d->smem, d->stream));
    return SPCG_OK;
}

spcg_status_t spcg_dev_solve(spcg_device_t* d, const double* b, double* x, double eps, int64_t kmax, bool use_x0,
                             spcg_solve_info_t* info, std::vector<double>* rhist) {
    CK(cudaSetDevice(d->device));
    Params P = d->P;
    P.mode = M_SOLVE;
    P.b = b;
    P.x = x;
    P.eps = eps;
    P.kmax = kmax;
    P.use_x0 = use_x0 ? 1 : 0;
    P.epoch = d->epoch;
    d->epoch += (unsigned)(kmax + 3);
    double* dh = nullptr;
    long long cap = std::min<long long>(kmax + 1, 1 << 20);
    CK(cudaMallocAsync((void**)&dh, sizeof(double) * cap, d->stream));
    P.rhist = dh;
    P.rhist_cap = cap;
    CK(cudaEventRecord(d->ev0, d->stream));
    spcg_status_t st = launch(d, P);
    if (st != SPCG_OK) { cudaFreeAsync(dh, d->stream); return st; }
    CK(cudaEventRecord(d->ev1, d->stream));
    Scal sc;
    CK(cudaMemcpyAsync(&sc, P.sc, sizeof(Scal), cudaMemcpyDeviceToHost, d->stream));
    CK(cudaStreamSynchronize(d->stream));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, d->ev0, d->ev1));
    long long kk = std::min<long long>(sc.k, cap - 1);
    if (rhist) {
        rhist->assign(kk + 1, 0.0);
        CK(cudaMemcpyAsync(rhist->data(), dh, sizeof(double) * (kk + 1), cudaMemcpyDeviceToHost, d->stream));
    }
    CK(cudaFreeAsync(dh, d->stream));
    CK(cudaStreamSynchronize(d->stream));
    info->iterations = sc.k;
    info->rnorm = std::sqrt(sc.rr);
    info->status = sc.status;
    info->converged = (sc.status == SPCG_OK && eps > 0.0) ? 1 : 0;
    info->iter_phase_ms = ms;
    if (sc.status == SPCG_ERR_INTERNAL) report_abort(d, sc);
    return sc.status;
}

spcg_status_t spcg_dev_apply(spcg_device_t* d, int op, const double* in, double* out, const double* aux,
                             double* scalar_out) {
    CK(cudaSetDevice(d->device));
    Params P = d->P;
    P.mode = op;
    P.in = in;
    P.out = out;
    P.aux = aux;
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
    if (kind == -1) {
        CK(cudaMallocAsync((void**)dst, bytes, d->stream));
        return SPCG_OK;
    }
    if (kind == -2) {
        CK(cudaFreeAsync(dst, d->stream));
        CK(cudaStreamSynchronize(d->stream));
        return SPCG_OK;
    }
    CK(cudaMemcpyAsync(dst, src, bytes, kind == 1 ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost, d->stream));
    CK(cudaStreamSynchronize(d->stream));
    return SPCG_OK;
}
