// libbarracuda internal helpers (sm_100a).  No method arithmetic lives here.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/barracuda.h"

namespace bc {

// thread-local status plumbing (api.cu)
void set_last_cuda_error(cudaError_t e);
void count_launch(int n = 1);
int num_sms();

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
