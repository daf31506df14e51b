// Latency microbenchmark (not part of the product): dependent chains of the
// warp-chain executor's critical-path operations, timed with clock64 by one warp.
#include <cstdio>
#include <cuda_runtime.h>
template <int MODE>
__global__ void k(double* out, long long* cyc, int n) {
    const int lane = threadIdx.x & 31;
    double y = lane * 0.001 + 1.0, v = 0.999, r = 0.5;
    float yf = lane * 0.001f + 1.0f;
    int yi = lane;
    const int src = (lane + 1) & 31;
    __syncwarp();
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < n; ++i) {
        if (MODE == 0) { double d = __shfl_sync(0xffffffffu, y, src); y = fma(-v, d, r); }
        if (MODE == 1) { y = fma(-v, y, r); }
        if (MODE == 2) { y = y + r; }
        if (MODE == 3) { yf = fmaf(-0.999f, yf, 0.5f); }
        if (MODE == 4) { yi = __shfl_sync(0xffffffffu, yi, src) + 1; }
        if (MODE == 5) { y = __shfl_sync(0xffffffffu, y, src) + 0.0; y = __longlong_as_double(__double_as_longlong(y) ^ 1); }
        if (MODE == 6) { yf = __shfl_sync(0xffffffffu, yf, src); yf = fmaf(-0.999f, yf, 0.5f); }
        if (MODE == 7) { y = y * v; }
        if (MODE == 8) { double d = __shfl_sync(0xffffffffu, y, src); double e = __shfl_sync(0xffffffffu, y, lane ^ 2); y = fma(-v, e, fma(-v, d, r)); }
        if (MODE == 9) { long long q = __double_as_longlong(y); int lo = __shfl_sync(0xffffffffu, (int)q, src); int hi = __shfl_sync(0xffffffffu, (int)(q >> 32), src); y = fma(-v, __hiloint2double(hi, lo), r); }
    }
    long long t1 = clock64();
    out[threadIdx.x] = y + yf + yi;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}
template <int M> void run(const char* name, double* o, long long* c) {
    long long h = 0;
    for (int rep = 0; rep < 3; ++rep) { k<M><<<1, 32>>>(o, c, 20000); cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost); }
    printf("%-34s %.1f cycles/iter\n", name, h / 20000.0);
}
int main() {
    double* o; long long* c; cudaMalloc(&o, 1024); cudaMalloc(&c, 8);
    run<0>("shfl64 -> dfma", o, c);
    run<1>("dfma chain", o, c);
    run<2>("dadd chain", o, c);
    run<3>("ffma chain", o, c);
    run<4>("shfl32 -> iadd", o, c);
    run<5>("shfl64 -> dadd -> lop", o, c);
    run<6>("shfl32 -> ffma", o, c);
    run<7>("dmul chain", o, c);
    run<8>("W2 step: 2 shfl64 -> 2 dfma", o, c);
    run<9>("manual lo/hi shfl -> dfma", o, c);
    return 0;
}
