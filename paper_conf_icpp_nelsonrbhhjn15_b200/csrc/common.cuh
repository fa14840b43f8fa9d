// libbarracuda internal helpers (sm_100a).  No method arithmetic lives here.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/barracuda.h"

namespace bc {

// thread-local status plumbing (api.cu)
void set_last_cuda_error(cudaError_t e);
void count_launch(int n = 1);
int num_sms();  // of the current device

// Launch attributes (cudaFuncSetAttribute, occupancy) are per device: caches keyed by the
// current device, so one process may call the library on several GPUs.
constexpr int BC_MAX_DEVICES = 64;
int current_device();
template <typename T>
struct PerDevice {
    T v[BC_MAX_DEVICES] = {};
    T& get() { return v[current_device()]; }
};

inline int launch_status() {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        set_last_cuda_error(e);
        return BC_ERR_CUDA;
    }
    count_launch();
    return BC_OK;
}

inline cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

// ---------------------------------------------------------------- fused check partials
// Kernels that fuse a check scalar write one fp64 partial per CTA to ws[8 + blockIdx.x]
// (at most CHECK_MAX_PARTIALS CTAs); run_check_finalize sums them in fixed order to ws[0].
constexpr int CHECK_MAX_PARTIALS = BC_CHECK_WS_DOUBLES - 8;
int run_check_finalize(int nparts, double* ws, cudaStream_t s);

// block-wide sum of v; thread 0 writes part[blockIdx.x]  (all threads must call)
__device__ __forceinline__ void block_partial(double v, double* part) {
    __shared__ double red[32];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    __syncthreads();
    if (l == 0) red[w] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        double s = 0.0;
        for (int i = 0; i < (int)((blockDim.x + 31) >> 5); ++i) s += red[i];
        part[blockIdx.x] = s;
    }
}

// ---------------------------------------------------------------- cp.async (LDGSTS)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cp_async_16(void* dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(smem_u32(dst)), "l"(src));
}
__device__ __forceinline__ void cp_async_8(void* dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(smem_u32(dst)), "l"(src));
}
__device__ __forceinline__ void cp_async_4(void* dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(smem_u32(dst)), "l"(src));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait_n() {  // at most N of this thread's groups pending
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N));
}

template <typename T>
__device__ __forceinline__ void cp_async_elem(T* dst, const T* src) {
    if constexpr (sizeof(T) == 8)
        cp_async_8(dst, src);
    else
        cp_async_4(dst, src);
}

// streaming global store (written once, not re-read by this kernel)
__device__ __forceinline__ void st_cs(double* p, double v) {
    asm volatile("st.global.cs.f64 [%0], %1;\n" ::"l"(p), "d"(v));
}
__device__ __forceinline__ void st_cs(float* p, float v) {
    asm volatile("st.global.cs.f32 [%0], %1;\n" ::"l"(p), "f"(v));
}

// ---------------------------------------------------------------- mbarriers, bulk copies
__device__ __forceinline__ void mbar_init(uint32_t bar, int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, int bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, int parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}\n" ::"r"(bar), "r"(parity) : "memory");
}
// non-blocking: has the phase with parity `parity` of the mbarrier completed?
__device__ __forceinline__ bool mbar_test(uint32_t bar, int parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void named_bar_sync(int id, int n) {
    asm volatile("bar.sync %0, %1;\n" ::"r"(id), "r"(n) : "memory");
}

// Consumer warp releases a ring slot it has finished reading.  The slot's next contents
// are written by TMA, i.e. by the ASYNC proxy, while the consumers read it with ordinary
// ld.shared (the GENERIC proxy); the mbarrier release/acquire pair orders the two only
// after a proxy fence: without `fence.proxy.async`, ptxas issues the arrive while the
// stage's last ld.shared are still in flight and the producer's refill can overwrite a
// fragment before it is read (measured: 183 of 200 repeat runs of the tile-16 fused
// kernel corrupted 128-1648 t3 values, one warp m-tile each; with the fence 0 of 200 —
// DESIGN.md §4.2).  Every lane fences its own reads, then lane 0 arrives for the warp.
__device__ __forceinline__ void release_slot(uint32_t bar_empty_slot, int lane) {
    asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
    __syncwarp();
    if (lane == 0) mbar_arrive(bar_empty_slot);
}

// 1-D bulk copy global -> shared (TMA engine, async proxy), completion counted on `bar`:
// dst and src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
// 1-D bulk copy shared -> global (async proxy, bulk async-group of the issuing thread):
// dst and src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_store(void* dst, uint32_t src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;\n" ::"l"(dst), "r"(src), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;\n" ::: "memory"); }
// at most N of this thread's bulk groups still reading their shared-memory source
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;\n" ::"n"(N) : "memory");
}
// at most N of this thread's bulk groups not yet complete (writes performed)
template <int N>
__device__ __forceinline__ void bulk_wait() {
    asm volatile("cp.async.bulk.wait_group %0;\n" ::"n"(N) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
}

template <typename T>
struct Pair;
template <>
struct Pair<double> {
    using type = double2;
};
template <>
struct Pair<float> {
    using type = float2;
};

}  // namespace bc
