// calib.cu — chain-floor calibration (SURVEY.md §8(d) "Chain-floor calibration").
//
// A wavefront solve's critical path is (levels_L + levels_U) handoffs; its floor
// is that count times the cheapest handoff the executor uses.  These
// microbenchmarks measure the candidate handoffs on the box the bench runs on:
//   1. a grid-wide barrier with one CTA per SM (what LEVEL pays per wavefront),
//   2. kernel-to-kernel latency inside a CUDA graph (a launch per wavefront),
//   3. a release-store / acquire-spin flag handoff between two CTAs, split into
//      near (same die) and far (cross die) pairs (what SYNCFREE / CHUNKED pay
//      per cross-CTA dependency),
//   4. __syncthreads and a 2-CTA cluster barrier (intra-CTA / intra-cluster).
// All times come from %globaltimer (ns) on the device.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "internal.h"

namespace {

__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned ld_acq(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_rel(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// 1. grid barrier: the solver's scheme (monotonic arrival counter, release
//    reduction, acquire spin until gen x gridDim)
__global__ void k_gridsync(unsigned* bar, int iters, unsigned long long* out) {
    __syncthreads();
    const unsigned long long t0 = gtime();
    for (int it = 0; it < iters; ++it) {
        __syncthreads();
        if (threadIdx.x == 0) {
            const unsigned target = (unsigned)(it + 1) * gridDim.x;
            asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(bar), "r"(1u) : "memory");
            while ((int)(ld_acq(bar) - target) < 0) {
            }
        }
        __syncthreads();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = gtime() - t0;
}

// 2. empty kernel for the graph chain
__global__ void k_empty() {}

__device__ __forceinline__ unsigned ld_vol(const unsigned* p) {
    unsigned v;
    asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_vol(unsigned* p, unsigned v) {
    asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
template <bool RELAXED>
__device__ __forceinline__ unsigned ld_flag(const unsigned* p) { return RELAXED ? ld_vol(p) : ld_acq(p); }
template <bool RELAXED>
__device__ __forceinline__ void st_flag(unsigned* p, unsigned v) {
    if (RELAXED) st_vol(p, v);
    else st_rel(p, v);
}

// 3. ping-pong between CTA 0 and CTA j, j = 1..G-1 in turn.  RELAXED: volatile
// (relaxed) accesses with the value carrying its own validity, as the solver's
// LL flags do; otherwise release store / acquire load.
template <bool RELAXED>
__global__ void k_pingpong(unsigned* ping, unsigned* pong, unsigned* turn, int rounds, unsigned long long* rt_ns,
                           int* smid) {
    const int j = blockIdx.x;
    if (threadIdx.x != 0) return;
    int sm;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    smid[j] = sm;
    if (j == 0) {
        for (int p = 1; p < (int)gridDim.x; ++p) {
            st_rel(turn, (unsigned)p);
            // warm-up round trips, then the timed ones
            unsigned long long t0 = 0;
            for (int t = 1; t <= rounds + 8; ++t) {
                if (t == 9) t0 = gtime();
                st_flag<RELAXED>(ping + p, (unsigned)t);
                while (ld_flag<RELAXED>(pong + p) != (unsigned)t) {
                }
            }
            rt_ns[p] = gtime() - t0;
        }
        st_rel(turn, 0xffffffffu);
    } else {
        while (ld_acq(turn) != (unsigned)j) __nanosleep(256);
        for (int t = 1; t <= rounds + 8; ++t) {
            while (ld_flag<RELAXED>(ping + j) != (unsigned)t) {
            }
            st_flag<RELAXED>(pong + j, (unsigned)t);
        }
    }
}

// 4a. __syncthreads, 256 threads
__global__ void k_syncthreads(int iters, unsigned long long* out) {
    const unsigned long long t0 = gtime();
    for (int i = 0; i < iters; ++i) __syncthreads();
    if (threadIdx.x == 0) out[0] = gtime() - t0;
}

// 4b. cluster barrier, cluster of 2 CTAs
__global__ void k_clustersync(int iters, unsigned long long* out) {
    const unsigned long long t0 = gtime();
    for (int i = 0; i < iters; ++i) {
        asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = gtime() - t0;
}

double median(std::vector<double> v) {
    if (v.empty()) return 0.0;
    std::sort(v.begin(), v.end());
    return v[v.size() / 2];
}

// LL ready-flag stress (DESIGN.md §5.3 "Ready flags"): the executors publish a value
// as ONE 16-byte store {lo32, epoch, hi32, epoch} (dev_common.cuh ll_store) and accept
// it when a 16-byte volatile load sees both epochs current — correct only if each
// 8-byte half {lo32, epoch} / {hi32, epoch} is observed whole.  Producer CTAs rewrite
// every slot once per epoch with a value both of whose halves encode (epoch, slot);
// consumer CTAs poll slots at random the whole time.  torn = loads whose two epochs
// agree but whose value halves do not belong to that epoch (must be 0); mixed = loads
// whose two epochs differ (benign: the reader keeps spinning).
__device__ __forceinline__ unsigned ll_lo(unsigned e, unsigned s) { return (e * 0x9E3779B1u) ^ (s * 0x85EBCA77u); }
__device__ __forceinline__ unsigned ll_hi(unsigned e, unsigned s) { return ~(e * 0xC2B2AE3Du) ^ (s * 0x27D4EB2Fu); }

__global__ void k_llstress(uint4* slots, int nslots, int rounds, unsigned* done, unsigned long long* cnt) {
    const int nprod = (gridDim.x + 1) / 2;
    if ((blockIdx.x & 1) == 0) {
        const int p = blockIdx.x / 2;
        for (unsigned e = 1; e <= (unsigned)rounds; ++e)
            for (int s = p * blockDim.x + threadIdx.x; s < nslots; s += nprod * blockDim.x)
                asm volatile("st.volatile.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(slots + s),
                             "r"(ll_lo(e, (unsigned)s)), "r"(e), "r"(ll_hi(e, (unsigned)s)), "r"(e)
                             : "memory");
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(done, 1u);
        }
        return;
    }
    unsigned long long torn = 0, mixed = 0, ok = 0;
    unsigned x = 0x12345u + 7919u * (blockIdx.x * blockDim.x + threadIdx.x);
    for (int it = 0;; ++it) {
        if ((it & 255) == 0) {
            unsigned d;
            asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(d) : "l"(done) : "memory");
            if (d >= (unsigned)nprod) break;
        }
        x = x * 1664525u + 1013904223u;
        const unsigned s = (x >> 8) % (unsigned)nslots;
        unsigned a, e1, c, e2;
        asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(a), "=r"(e1), "=r"(c), "=r"(e2)
                     : "l"(slots + s)
                     : "memory");
        if (e1 != e2) ++mixed;
        else if (e1 != 0) {
            if (a != ll_lo(e1, s) || c != ll_hi(e1, s)) ++torn;
            else ++ok;
        }
    }
    atomicAdd(cnt + 0, torn);
    atomicAdd(cnt + 1, mixed);
    atomicAdd(cnt + 2, ok);
}

}  // namespace

#define CKC(x)                                                            \
    do {                                                                  \
        cudaError_t e_ = (x);                                             \
        if (e_ != cudaSuccess) {                                          \
            spcg::set_error(std::string(#x ": ") + cudaGetErrorString(e_)); \
            st = SPCG_ERR_CUDA;                                           \
            goto done;                                                    \
        }                                                                 \
    } while (0)

extern "C" spcg_status_t spcg_calibrate(int32_t device, spcg_calib_t* out) {
    if (!out) return SPCG_ERR_INVALID_ARG;
    *out = spcg_calib_t{};
    spcg_status_t st = SPCG_OK;
    int sms = 0, clk_khz = 0;
    unsigned* dbuf = nullptr;
    unsigned long long* dres = nullptr;
    int* dsm = nullptr;
    cudaStream_t s = nullptr;
    cudaGraph_t g = nullptr;
    cudaGraphExec_t ge = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    std::vector<unsigned long long> rt;
    std::vector<int> smid;
    float ms_a = 0.f, ms_b = 0.f;
    CKC(cudaSetDevice(device));
    CKC(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
    CKC(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, device));
    out->sms = sms;
    out->sm_clock_mhz = clk_khz / 1000.0;
    CKC(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    CKC(cudaEventCreate(&e0));
    CKC(cudaEventCreate(&e1));
    CKC(cudaMalloc(&dbuf, sizeof(unsigned) * (4 + 2 * 1024)));
    CKC(cudaMalloc(&dres, sizeof(unsigned long long) * 1024));
    CKC(cudaMalloc(&dsm, sizeof(int) * 1024));
    CKC(cudaMemsetAsync(dbuf, 0, sizeof(unsigned) * (4 + 2 * 1024), s));
    {   // 1. grid barrier, cooperative, one CTA of 256 threads per SM
        int iters = 4000;
        void* args[] = {&dbuf, &iters, &dres};
        CKC(cudaLaunchCooperativeKernel((void*)k_gridsync, dim3(sms), dim3(256), args, 0, s));   // warm-up
        CKC(cudaMemsetAsync(dbuf, 0, sizeof(unsigned) * 4, s));
        CKC(cudaLaunchCooperativeKernel((void*)k_gridsync, dim3(sms), dim3(256), args, 0, s));
        unsigned long long ns = 0;
        CKC(cudaMemcpyAsync(&ns, dres, 8, cudaMemcpyDeviceToHost, s));
        CKC(cudaStreamSynchronize(s));
        out->grid_sync_ns = (double)ns / iters;
    }
    {   // 2. graph of chained empty kernels: (T(200) - T(20)) / 180
        for (int pass = 0; pass < 2; ++pass) {
            const int nk = pass == 0 ? 20 : 200;
            CKC(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
            for (int i = 0; i < nk; ++i) k_empty<<<1, 32, 0, s>>>();
            CKC(cudaStreamEndCapture(s, &g));
            CKC(cudaGraphInstantiate(&ge, g, 0));
            CKC(cudaGraphLaunch(ge, s));
            CKC(cudaEventRecord(e0, s));
            for (int r = 0; r < 10; ++r) CKC(cudaGraphLaunch(ge, s));
            CKC(cudaEventRecord(e1, s));
            CKC(cudaEventSynchronize(e1));
            CKC(cudaEventElapsedTime(pass == 0 ? &ms_a : &ms_b, e0, e1));
            cudaGraphExecDestroy(ge);
            cudaGraphDestroy(g);
            ge = nullptr;
            g = nullptr;
        }
        out->graph_kernel_ns = (ms_b - ms_a) * 1e6 / 10.0 / 180.0;
    }
    for (int relaxed = 0; relaxed < 2; ++relaxed) {   // 3. flag ping-pong CTA 0 <-> CTA j
        int rounds = 200;
        unsigned* ping = dbuf + 4;
        unsigned* pong = dbuf + 4 + 1024;
        unsigned* turn = dbuf + 2;
        const int G = std::min(sms, 1024);
        CKC(cudaMemsetAsync(dbuf, 0, sizeof(unsigned) * (4 + 2 * 1024), s));
        void* args[] = {&ping, &pong, &turn, &rounds, &dres, &dsm};
        CKC(cudaLaunchCooperativeKernel(relaxed ? (void*)k_pingpong<true> : (void*)k_pingpong<false>, dim3(G), dim3(32),
                                        args, 0, s));
        rt.resize(G);
        smid.resize(G);
        CKC(cudaMemcpyAsync(rt.data(), dres, 8 * G, cudaMemcpyDeviceToHost, s));
        CKC(cudaMemcpyAsync(smid.data(), dsm, 4 * G, cudaMemcpyDeviceToHost, s));
        CKC(cudaStreamSynchronize(s));
        // one-way = round trip / 2; two populations (same die / cross die): split at the
        // largest gap of the sorted values
        std::vector<double> ow;
        for (int j = 1; j < G; ++j) ow.push_back((double)rt[j] / rounds / 2.0);
        std::sort(ow.begin(), ow.end());
        size_t cut = ow.size();
        double best = 0.0;
        for (size_t i = ow.size() / 4; i + 1 < ow.size() * 3 / 4 + 1 && i + 1 < ow.size(); ++i)
            if (ow[i + 1] - ow[i] > best) { best = ow[i + 1] - ow[i]; cut = i + 1; }
        std::vector<double> near(ow.begin(), ow.begin() + cut), far(ow.begin() + cut, ow.end());
        if (relaxed) {
            out->flag_relaxed_same_die_ns = median(near);
            out->flag_relaxed_cross_die_ns = far.empty() ? median(near) : median(far);
        } else {
            out->flag_same_die_ns = median(near);
            out->flag_cross_die_ns = far.empty() ? median(near) : median(far);
            out->flag_pairs_near = (int32_t)near.size();
        }
    }
    {   // 4a. __syncthreads
        int iters = 20000;
        k_syncthreads<<<1, 256, 0, s>>>(iters, dres);
        CKC(cudaGetLastError());
        unsigned long long ns = 0;
        CKC(cudaMemcpyAsync(&ns, dres, 8, cudaMemcpyDeviceToHost, s));
        CKC(cudaStreamSynchronize(s));
        out->syncthreads_ns = (double)ns / iters;
    }
    {   // 4b. cluster barrier (cluster of 2)
        int iters = 20000;
        cudaLaunchConfig_t cfg{};
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 2;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3(2);
        cfg.blockDim = dim3(256);
        cfg.stream = s;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        CKC(cudaLaunchKernelEx(&cfg, k_clustersync, iters, dres));
        unsigned long long ns = 0;
        CKC(cudaMemcpyAsync(&ns, dres, 8, cudaMemcpyDeviceToHost, s));
        CKC(cudaStreamSynchronize(s));
        out->cluster_sync_ns = (double)ns / iters;
    }
done:
    if (ge) cudaGraphExecDestroy(ge);
    if (g) cudaGraphDestroy(g);
    if (dbuf) cudaFree(dbuf);
    if (dres) cudaFree(dres);
    if (dsm) cudaFree(dsm);
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    if (s) cudaStreamDestroy(s);
    return st;
}

extern "C" spcg_status_t spcg_ll_stress(int32_t device, int32_t nslots, int32_t rounds, uint64_t* out) {
    if (!out || nslots <= 0 || rounds <= 0) {
        spcg::set_error("spcg_ll_stress: out == NULL or a non-positive size");
        return SPCG_ERR_INVALID_ARG;
    }
    if (cudaSetDevice(device) != cudaSuccess) {
        spcg::set_error("cudaSetDevice failed");
        return SPCG_ERR_CUDA;
    }
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    uint4* slots = nullptr;
    unsigned* done = nullptr;
    unsigned long long* cnt = nullptr;
    spcg_status_t st = SPCG_OK;
    int G = sms - (sms & 1);            // pairs of producer / consumer CTAs, all co-resident
    void* args[] = {&slots, &nslots, &rounds, &done, &cnt};
    if (cudaMalloc(&slots, sizeof(uint4) * (size_t)nslots) != cudaSuccess || cudaMalloc(&done, 4) != cudaSuccess ||
        cudaMalloc(&cnt, 24) != cudaSuccess) {
        st = SPCG_ERR_OOM;
        goto out_;
    }
    cudaMemset(slots, 0, sizeof(uint4) * (size_t)nslots);
    cudaMemset(done, 0, 4);
    cudaMemset(cnt, 0, 24);
    if (cudaLaunchCooperativeKernel((void*)k_llstress, dim3(G), dim3(256), args, 0, 0) != cudaSuccess ||
        cudaDeviceSynchronize() != cudaSuccess) {
        spcg::set_error(std::string("ll stress kernel: ") + cudaGetErrorString(cudaGetLastError()));
        st = SPCG_ERR_CUDA;
        goto out_;
    }
    {
        unsigned long long h[3];
        cudaMemcpy(h, cnt, 24, cudaMemcpyDeviceToHost);
        out[0] = h[0];
        out[1] = h[1];
        out[2] = h[2];
    }
out_:
    cudaFree(slots);
    cudaFree(done);
    cudaFree(cnt);
    return st;
}
