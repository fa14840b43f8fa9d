// FP64 peak probes (measurement utility, not a method operation): the roofline
// denominators the bench reports for its FP64-bound kernels are measured live on the box
// with these, instead of a hard-coded number.
//   kind 0: DFMA  — 8 independent fma chains per thread (the spectral DFMA kernels' pipe)
//   kind 1: DMMA  — 8 independent mma.sync.m8n8k4.f64 chains per warp (the CCSD(T) and
//                   spectral tensor-core kernels' pipe)
// Grid: 8 CTAs x 512 threads per SM (enough warps to hide both pipes' latency).
#include "common.cuh"

namespace bc {

__global__ void __launch_bounds__(512) probe_dfma_kernel(double* out, int iters, double a, double b) {
    double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6,
           x7 = x0 + 7;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            x0 = fma(x0, a, b); x1 = fma(x1, a, b); x2 = fma(x2, a, b); x3 = fma(x3, a, b);
            x4 = fma(x4, a, b); x5 = fma(x5, a, b); x6 = fma(x6, a, b); x7 = fma(x7, a, b);
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

__global__ void __launch_bounds__(512) probe_dmma_kernel(double* out, int iters) {
    const double a = threadIdx.x * 1e-3, b = threadIdx.x * 2e-3;
    double c[8][2];
#pragma unroll
    for (int q = 0; q < 8; ++q) c[q][0] = c[q][1] = 0.0;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
            for (int q = 0; q < 8; ++q)
                asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                             : "+d"(c[q][0]), "+d"(c[q][1])
                             : "d"(a), "d"(b));
    }
    double s = 0.0;
#pragma unroll
    for (int q = 0; q < 8; ++q) s += c[q][0] + c[q][1];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int run_probe_fp64(int kind, int iters, double* scratch, double* flops, cudaStream_t s) {
    const int blocks = num_sms() * 8, threads = 512;
    if (kind == 0) {
        probe_dfma_kernel<<<blocks, threads, 0, s>>>(scratch, iters, 1.0000001, 1e-9);
        *flops = 2.0 * 8 * 16 * (double)iters * blocks * threads;
    } else {
        probe_dmma_kernel<<<blocks, threads, 0, s>>>(scratch, iters);
        *flops = 2.0 * 256 * 4 * 8 * (double)iters * blocks * (threads / 32);
    }
    return launch_status();
}

int probe_scratch_doubles() { return num_sms() * 8 * 512; }

}  // namespace bc
