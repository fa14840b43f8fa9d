// Check scalars (R18) and the device side of the counter-based input generator.
#include "common.cuh"

namespace bc {

constexpr int RED_NT = 256;
constexpr int RED_MAX_BLOCKS = BC_CHECK_WS_DOUBLES - 8;

__device__ __forceinline__ double block_sum(double v, double* sh) {
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    const int w = threadIdx.x / 32, l = threadIdx.x % 32;
    if (l == 0) sh[w] = v;
    __syncthreads();
    double s = 0.0;
    if (threadIdx.x == 0)
        for (int i = 0; i < RED_NT / 32; ++i) s += sh[i];
    return s;  // valid on thread 0
}

__global__ void __launch_bounds__(RED_NT) sumsq_partial(int64_t n, const double* __restrict__ x,
                                                       double* __restrict__ part) {
    __shared__ double sh[RED_NT / 32];
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)RED_NT + threadIdx.x; i < n; i += (int64_t)gridDim.x * RED_NT) {
        const double v = __ldcs(x + i);
        s = fma(v, v, s);
    }
    s = block_sum(s, sh);
    if (threadIdx.x == 0) part[blockIdx.x] = s;
}

__global__ void __launch_bounds__(RED_NT) finalize(int nb, const double* __restrict__ part, double* __restrict__ out) {
    __shared__ double sh[RED_NT / 32];
    double s = 0.0;
    for (int i = threadIdx.x; i < nb; i += RED_NT) s += part[i];
    s = block_sum(s, sh);
    if (threadIdx.x == 0) *out = s;
}

struct EnergyDims {
    int h1, h2, h3, p4, p5, p6;
};

// canonical t3 order (h3,h2,h1,p6,p5,p4), Fortran (h3 fastest) = [particle plane][hole index]
// Blocks stride over particle planes; the hole part of the denominator, (e3+e2)+e1, is
// tabulated once per block in shared memory (when it fits), so the per-element work is
// ((dh - f6) - f5) - f4: the oracle's summation order.
constexpr int EN_TAB = 4096;
__global__ void __launch_bounds__(RED_NT) energy_partial(EnergyDims d, const double* __restrict__ t3,
                                                        const double* __restrict__ eh, const double* __restrict__ ep,
                                                        double* __restrict__ part) {
    __shared__ double sh[RED_NT / 32];
    __shared__ double dh[EN_TAB];
    const int nh = d.h1 * d.h2 * d.h3;
    const int np = d.p4 * d.p5 * d.p6;
    const double* e1 = eh;
    const double* e2 = eh + d.h1;
    const double* e3 = eh + d.h1 + d.h2;
    const double* f4 = ep;
    const double* f5 = ep + d.p4;
    const double* f6 = ep + d.p4 + d.p5;
    const bool tab = nh <= EN_TAB;
    if (tab)
        for (int i = threadIdx.x; i < nh; i += RED_NT) {
            const int h3 = i % d.h3, h2 = (i / d.h3) % d.h2, h1 = i / (d.h3 * d.h2);
            dh[i] = (e3[h3] + e2[h2]) + e1[h1];
        }
    __syncthreads();
    double s = 0.0;
    for (int pl = blockIdx.x; pl < np; pl += gridDim.x) {
        const int p6 = pl % d.p6, p5 = (pl / d.p6) % d.p5, p4 = pl / (d.p6 * d.p5);
        const double a6 = f6[p6], a5 = f5[p5], a4 = f4[p4];
        const double* row = t3 + (int64_t)pl * nh;
        int i = threadIdx.x;
        if (tab) {
            // EN_UNR independent loads in flight per thread before the dependent divisions:
            // one load per iteration left the pass latency-bound (≈0.3 of HBM at tile 16).
            constexpr int EN_UNR = 8;
            for (; i + (EN_UNR - 1) * RED_NT < nh; i += EN_UNR * RED_NT) {
                double t[EN_UNR];
#pragma unroll
                for (int u = 0; u < EN_UNR; ++u) t[u] = __ldcs(row + i + u * RED_NT);
#pragma unroll
                for (int u = 0; u < EN_UNR; ++u) {
                    const double den = ((dh[i + u * RED_NT] - a6) - a5) - a4;
                    s += t[u] * t[u] / den;
                }
            }
        }
        for (; i < nh; i += RED_NT) {
            double h;
            if (tab) {
                h = dh[i];
            } else {
                const int h3 = i % d.h3, h2 = (i / d.h3) % d.h2, h1 = i / (d.h3 * d.h2);
                h = (e3[h3] + e2[h2]) + e1[h1];
            }
            const double den = ((h - a6) - a5) - a4;
            const double t = __ldcs(row + i);
            s += t * t / den;
        }
    }
    s = block_sum(s, sh);
    if (threadIdx.x == 0) part[blockIdx.x] = s;
}

static int red_blocks(int64_t n) {
    int64_t b = (n + RED_NT * 8 - 1) / (RED_NT * 8);
    int64_t cap = (int64_t)num_sms() * 4;
    if (cap > RED_MAX_BLOCKS) cap = RED_MAX_BLOCKS;
    if (b > cap) b = cap;
    return b < 1 ? 1 : (int)b;
}

int run_check_finalize(int nparts, double* ws, cudaStream_t s) {
    finalize<<<1, RED_NT, 0, s>>>(nparts, ws + 8, ws);
    return launch_status();
}

int run_sumsq(int64_t n, const double* x, double* ws, cudaStream_t s) {
    const int nb = red_blocks(n);
    sumsq_partial<<<nb, RED_NT, 0, s>>>(n, x, ws + 8);
    int st = launch_status();
    if (st) return st;
    finalize<<<1, RED_NT, 0, s>>>(nb, ws + 8, ws);
    return launch_status();
}

int run_energy(const int* ext7, const double* t3, const double* eh, const double* ep, double* ws, cudaStream_t s) {
    EnergyDims d{ext7[0], ext7[1], ext7[2], ext7[3], ext7[4], ext7[5]};
    const int np = d.p4 * d.p5 * d.p6;
    int nb = red_blocks((int64_t)np * RED_NT * 8);
    if (nb > np) nb = np;
    energy_partial<<<nb, RED_NT, 0, s>>>(d, t3, eh, ep, ws + 8);
    int st = launch_status();
    if (st) return st;
    finalize<<<1, RED_NT, 0, s>>>(nb, ws + 8, ws);
    return launch_status();
}

// ---------------------------------------------------------------- input generator
__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

template <typename T>
__global__ void fill_kernel(int kind, uint64_t base, int64_t n, double lo, double hi, T* __restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const uint64_t z = splitmix64(base + (uint64_t)i);
        double x;
        if (kind == 1) {
            x = (double)(z >> 61) - 4.0;
        } else {
            const double u = (double)(z >> 11) * 0x1.0p-53;
            // explicit _rn ops: no FMA contraction, bit-identical to the numpy generator
            x = (kind == 0) ? __dadd_rn(__dmul_rn(u, 2.0), -1.0) : __dadd_rn(lo, __dmul_rn(__dadd_rn(hi, -lo), u));
        }
        out[i] = (T)x;
    }
}

template <typename T>
int run_fill(int kind, uint64_t seed, uint64_t tid, uint64_t offset, int64_t n, double lo, double hi, T* out,
             cudaStream_t s) {
    const uint64_t base = seed + (tid << 40) + offset;
    int64_t blocks = (n + 255) / 256;
    const int64_t cap = (int64_t)num_sms() * 16;
    if (blocks > cap) blocks = cap;
    fill_kernel<T><<<(unsigned)blocks, 256, 0, s>>>(kind, base, n, lo, hi, out);
    return launch_status();
}
template int run_fill<double>(int, uint64_t, uint64_t, uint64_t, int64_t, double, double, double*, cudaStream_t);
template int run_fill<float>(int, uint64_t, uint64_t, uint64_t, int64_t, double, double, float*, cudaStream_t);

}  // namespace bc
