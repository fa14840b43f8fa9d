// scratch microbenchmark: FP64 DFMA vs DMMA (mma.sync m8n8k4 f64) throughput, HBM copy
#include <cstdio>
#include <cuda_runtime.h>
__global__ void dfma_k(double* out, int iters, double a, double b) {
  double x0=threadIdx.x, x1=x0+1, x2=x0+2, x3=x0+3, x4=x0+4, x5=x0+5, x6=x0+6, x7=x0+7;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      x0 = fma(x0, a, b); x1 = fma(x1, a, b); x2 = fma(x2, a, b); x3 = fma(x3, a, b);
      x4 = fma(x4, a, b); x5 = fma(x5, a, b); x6 = fma(x6, a, b); x7 = fma(x7, a, b);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0+x1+x2+x3+x4+x5+x6+x7;
}
__global__ void dmma_k(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = threadIdx.x * 2e-3;
  double c[8][2];
  for (int q = 0; q < 8; ++q) { c[q][0] = 0; c[q][1] = 0; }
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
#pragma unroll
      for (int q = 0; q < 8; ++q)
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                     : "+d"(c[q][0]), "+d"(c[q][1]) : "d"(a), "d"(b));
    }
  }
  double s = 0; for (int q = 0; q < 8; ++q) s += c[q][0] + c[q][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void copy_k(const double2* __restrict__ a, double2* __restrict__ b, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x, st = (size_t)gridDim.x * blockDim.x;
  for (; i < n; i += st) b[i] = a[i];
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d clock(kHz) %d\n", sms, clk);
  double* out; cudaMalloc(&out, 1 << 26);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  for (int bpsm = 1; bpsm <= 8; bpsm *= 2) for (int thr : {256, 512}) {
    int blocks = sms * bpsm, iters = 2000;
    dfma_k<<<blocks, thr>>>(out, 10, 1.0000001, 1e-9);
    cudaEventRecord(e0); dfma_k<<<blocks, thr>>>(out, iters, 1.0000001, 1e-9); cudaEventRecord(e1);
    cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    double fl = 2.0 * 8 * 16 * (double)iters * blocks * thr;
    printf("DFMA blocks/SM %d thr %d: %.2f TFLOP/s\n", bpsm, thr, fl / ms / 1e9);
  }
  for (int bpsm = 1; bpsm <= 8; bpsm *= 2) for (int thr : {128, 256, 512}) {
    int blocks = sms * bpsm, iters = 500;
    dmma_k<<<blocks, thr>>>(out, 10);
    cudaEventRecord(e0); dmma_k<<<blocks, thr>>>(out, iters); cudaEventRecord(e1);
    cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    double fl = 2.0 * 256 * 4 * 8 * (double)iters * blocks * (thr / 32);
    printf("DMMA blocks/SM %d thr %d: %.2f TFLOP/s\n", bpsm, thr, fl / ms / 1e9);
  }
  size_t n = (size_t)1 << 28; // 2^28 double2 = 4 GiB
  double2 *a, *b; cudaMalloc(&a, n * 16); cudaMalloc(&b, n * 16);
  cudaMemset(a, 0, n * 16);
  for (int r = 0; r < 3; ++r) {
    cudaEventRecord(e0); copy_k<<<sms * 8, 512>>>(a, b, n); cudaEventRecord(e1);
    cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    printf("copy: %.1f GB/s\n", 2.0 * n * 16 / ms / 1e6);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
