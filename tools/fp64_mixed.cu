// scratch microbenchmark: can the FP64 DFMA pipe and the DMMA (mma.sync m8n8k4 f64) pipe
// issue concurrently on one SM?  Runs DFMA-only, DMMA-only, and a mixed kernel whose warps
// alternate between the two kinds (even warps DFMA, odd warps DMMA; and a per-warp
// interleaved form).  If the mixed kernel's combined flop rate exceeds the faster single
// pipe, the two pipes overlap.
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void dfma_body(double* out, int iters, double a, double b) {
    double x[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) x[q] = threadIdx.x + q;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j)
#pragma unroll
            for (int q = 0; q < 16; ++q) x[q] = fma(x[q], a, b);
    }
    double s = 0;
#pragma unroll
    for (int q = 0; q < 16; ++q) s += x[q];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__device__ __forceinline__ void dmma_body(double* out, int iters) {
    double a = threadIdx.x * 1e-3, b = threadIdx.x * 2e-3;
    double c[8][2];
#pragma unroll
    for (int q = 0; q < 8; ++q) { c[q][0] = 0; c[q][1] = 0; }
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int q = 0; q < 8; ++q)
                asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                             : "+d"(c[q][0]), "+d"(c[q][1]) : "d"(a), "d"(b));
    }
    double s = 0;
#pragma unroll
    for (int q = 0; q < 8; ++q) s += c[q][0] + c[q][1];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// per-thread flops: dfma 2*16*8*iters, dmma per warp 2*256*4*8*iters -> per thread 512*iters
__global__ void __launch_bounds__(512) k_dfma(double* o, int it, double a, double b) { dfma_body(o, it, a, b); }
__global__ void __launch_bounds__(512) k_dmma(double* o, int it) { dmma_body(o, it); }
__global__ void __launch_bounds__(512) k_mixed(double* o, int itf, int itm, double a, double b) {
    if ((threadIdx.x >> 5) & 1) dmma_body(o, itm); else dfma_body(o, itf, a, b);
}
// one warp does both: DMMA chain and DFMA chains interleaved in the same loop
__global__ void __launch_bounds__(512) k_inter(double* o, int it, double a, double b) {
    double x[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) x[q] = threadIdx.x + q;
    double ma = threadIdx.x * 1e-3, mb = threadIdx.x * 2e-3;
    double c[8][2];
#pragma unroll
    for (int q = 0; q < 8; ++q) { c[q][0] = 0; c[q][1] = 0; }
    for (int i = 0; i < it; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                             : "+d"(c[q][0]), "+d"(c[q][1]) : "d"(ma), "d"(mb));
#pragma unroll
                for (int w = 0; w < 16; ++w) x[w] = fma(x[w], a, b);
            }
        }
    }
    double s = 0;
#pragma unroll
    for (int q = 0; q < 16; ++q) s += x[q];
#pragma unroll
    for (int q = 0; q < 8; ++q) s += c[q][0] + c[q][1];
    o[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int blocks = sms * 4, threads = 512;
    double* o;
    cudaMalloc(&o, (size_t)blocks * threads * 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto timeit = [&](auto fn) {
        fn();
        cudaDeviceSynchronize();
        float best = 1e30f;
        for (int r = 0; r < 3; ++r) {
            cudaEventRecord(e0);
            fn();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        return best;
    };
    const int it = 4000;
    const double T = (double)blocks * threads;
    float ms = timeit([&] { k_dfma<<<blocks, threads>>>(o, it, 1.0000001, 1e-9); });
    double fdf = 2.0 * 16 * 8 * it * T;
    printf("dfma only : %.3f ms  %.2f TFLOP/s\n", ms, fdf / ms / 1e9);
    ms = timeit([&] { k_dmma<<<blocks, threads>>>(o, it); });
    double fmm = 512.0 * it * T;
    printf("dmma only : %.3f ms  %.2f TFLOP/s\n", ms, fmm / ms / 1e9);
    // mixed: half the warps each; iteration counts chosen so each half alone would take
    // about the same time at its own peak
    for (int itm : {it, it / 2}) {
        ms = timeit([&] { k_mixed<<<blocks, threads>>>(o, it, itm, 1.0000001, 1e-9); });
        double f = 0.5 * (2.0 * 16 * 8 * it * T) + 0.5 * (512.0 * itm * T);
        printf("mixed warps (dfma it %d, dmma it %d): %.3f ms  %.2f TFLOP/s combined\n", it, itm, ms, f / ms / 1e9);
    }
    ms = timeit([&] { k_inter<<<blocks, threads>>>(o, it, 1.0000001, 1e-9); });
    double fi = (2.0 * 16 * 32 * it + 512.0 * it) * T;
    printf("interleaved in-warp: %.3f ms  %.2f TFLOP/s combined (dfma share %.2f)\n", ms, fi / ms / 1e9,
           2.0 * 16 * 32 / (2.0 * 16 * 32 + 512.0));
    cudaError_t e = cudaGetLastError();
    printf("status: %s\n", cudaGetErrorString(e));
    return 0;
}
