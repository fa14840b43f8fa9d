// Spectral family on the FP64 tensor cores (DMMA, mma.sync.m8n8k4.f64), sm_100a.
//
// Why: the DFMA kernels in spectral.cu are bound by the shared-memory
// pipe — a broadcast operator read costs full-warp wavefronts, ~1 wavefront per DFMA.
// Here each contraction stage of an element is a small GEMM
//     Y[k][line] = sum_n M[k][n] X[n][line]        (k, n < P1 padded to KP = 8 or 16)
// with the operator M held in REGISTERS as DMMA A-fragments for the whole kernel, and
// X streamed from shared memory as B-fragments: one 8-byte read per lane feeds MF DMMAs
// (MF*256 FMAs per warp).  Shared-memory layout: rows padded to RS (= 4 or 12 mod 16)
// and planes to PS (= 4 or 12 mod 16), which makes the B-fragment reads (4 contracted
// values x 8 lines per instruction) bank-conflict free along every axis.
//
// Stages run in place (a fragment's 8 lines are read by one warp before it writes them,
// mma.sync being warp-synchronous), and the LAST stage contracts the fastest axis so
// that C-fragment stores to global memory are 64-byte contiguous runs.  The sum
// factorisation commutes, so sumfact3d runs C (axis 0) -> B (axis 1) -> A (axis 2):
// same result as the paper's order up to rounding (bitwise on integer data).
#include "common.cuh"

namespace bc {

__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

template <int P1, int NA>
struct MG {
    static constexpr int KP = P1 <= 8 ? 8 : 16;  // padded operator size
    static constexpr int MF = KP / 8;            // m-fragments (output rows / 8)
    static constexpr int KS = KP / 4;            // k-steps of 4
    static constexpr int RS = P1 <= 4 ? 4 : (P1 <= 12 ? 12 : 20);               // row stride
    static constexpr int PS = (NA == 1) ? RS * P1 : P1 * RS + ((P1 % 2) ? 0 : 4);  // plane stride
    static constexpr int ES0 = (NA == 1) ? P1 * RS : P1 * PS;
    static constexpr int ES = (ES0 + 1) & ~1;    // element stride (16-byte multiple)
    static constexpr int NPTS = NA * P1 * P1;
    static constexpr int LPE = NA * P1;          // lines per element along any axis
};

// Line geometry: line l of element e (l < LPE); base offset and contracted-index stride.
template <int P1, int NA, int AXIS>
struct ML {
    using G = MG<P1, NA>;
    static constexpr int STRIDE = AXIS == 2 ? 1 : (AXIS == 1 ? G::RS : G::PS);
    __device__ __forceinline__ static int base(int e, int l) {
        const int x = l / P1, y = l - (l / P1) * P1;
        if constexpr (AXIS == 2) return e * G::ES + x * G::PS + y * G::RS;   // (a, b): rows
        else if constexpr (AXIS == 1) return e * G::ES + x * G::PS + y;       // (a, c)
        else return e * G::ES + x * G::RS + y;                                // (b, c)
    }
    // global element-relative offset of output k of line l (2-D: x = 0 plane)
    __device__ __forceinline__ static int gofs(int l, int k) {
        const int x = l / P1, y = l - (l / P1) * P1;
        if constexpr (AXIS == 2) return (x * P1 + y) * P1 + k;
        else if constexpr (AXIS == 1) return (x * P1 + k) * P1 + y;
        else return (k * P1 + x) * P1 + y;
    }
};

// A-fragments of operator M (row-major P1 x P1, y_k = sum_n M[k][n] x_n), zero padded.
// TRANSPOSE: use M^T.
template <int P1, bool TRANSPOSE = false>
__device__ __forceinline__ void load_afrag(double (&a)[MG<P1, 1>::MF][MG<P1, 1>::KS], const double* __restrict__ Mat) {
    using G = MG<P1, 1>;
    const int lane = threadIdx.x & 31, gq = lane >> 2, tq = lane & 3;
#pragma unroll
    for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
        for (int ks = 0; ks < G::KS; ++ks) {
            const int k = mf * 8 + gq, n = ks * 4 + tq;
            a[mf][ks] = (k < P1 && n < P1) ? __ldg(Mat + (TRANSPOSE ? n * P1 + k : k * P1 + n)) : 0.0;
        }
}

// One stage over `ne` elements of `buf`: every line of every element along AXIS.
// out(e, l, k, v) consumes the outputs (in place or to global).
template <int P1, int NA, int AXIS, int NW, typename Out>
__device__ __forceinline__ void mma_stage(const double* buf, const double (&a)[MG<P1, 1>::MF][MG<P1, 1>::KS],
                                          int ne, Out out) {
    using G = MG<P1, NA>;
    using L = ML<P1, NA, AXIS>;
    constexpr int MF = G::MF, KS = G::KS;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, gq = lane >> 2, tq = lane & 3;
    const int total = ne * G::LPE;
    const int nfrag = (total + 7) >> 3;
    // two fragments per iteration: 2*MF independent accumulator chains
    for (int f0 = warp * 2; f0 < nfrag; f0 += NW * 2) {
        double c[2][MF][2];
        int bofs[2];
#pragma unroll
        for (int t = 0; t < 2; ++t) {
            int l = (f0 + t) * 8 + gq;
            l = l < total ? l : total - 1;  // clamp: finite data, result discarded
            const int e = l / G::LPE;
            bofs[t] = L::base(e, l - e * G::LPE);
#pragma unroll
            for (int mf = 0; mf < MF; ++mf) c[t][mf][0] = c[t][mf][1] = 0.0;
        }
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
            int n = ks * 4 + tq;
            n = n < P1 ? n : P1 - 1;  // padded k: zero operator column, finite data
            double b[2];
#pragma unroll
            for (int t = 0; t < 2; ++t) b[t] = buf[bofs[t] + n * L::STRIDE];
#pragma unroll
            for (int t = 0; t < 2; ++t)
#pragma unroll
                for (int mf = 0; mf < MF; ++mf) dmma(c[t][mf][0], c[t][mf][1], a[mf][ks], b[t]);
        }
        // the C fragments below are written (in place) to lines that OTHER lanes of this
        // warp read as B fragments above: order those reads before these writes explicitly
        // (the mma.sync data dependence already does in practice, but carries no memory-
        // model ordering; racecheck flagged it)
        __syncwarp();
#pragma unroll
        for (int t = 0; t < 2; ++t)
#pragma unroll
            for (int j = 0; j < 2; ++j) {
                const int l = (f0 + t) * 8 + 2 * tq + j;
                if (l < total) {
                    const int e = l / G::LPE, ll = l - e * G::LPE;
#pragma unroll
                    for (int mf = 0; mf < MF; ++mf) {
                        const int k = mf * 8 + gq;
                        if (k < P1) out(e, ll, k, c[t][mf][j]);
                    }
                }
            }
    }
}

// Stage `ne` contiguous elements from global into the padded layout (cp.async, 8 B).
template <int P1, int NA, int NT>
__device__ __forceinline__ void mma_load_group(double* dst, const double* __restrict__ src, int ne) {
    using G = MG<P1, NA>;
    const int total = ne * G::NPTS;
    for (int f = threadIdx.x; f < total; f += NT) {
        const int e = f / G::NPTS;
        const int r = f - e * G::NPTS;
        const int row = r / P1, c = r - (r / P1) * P1;
        const int a = row / P1, b = row - (row / P1) * P1;
        const int so = (NA == 1) ? e * G::ES + row * G::RS + c : e * G::ES + a * G::PS + b * G::RS + c;
        cp_async_8(dst + so, src + f);
    }
}

template <int P1, int NA>
struct MCfg {
    using G = MG<P1, NA>;
    static constexpr int NW = 8, NT = NW * 32;
    // elements per group: ~24 KiB per buffer (3-D p=12: 1 element of 27 KiB), 2 buffers
    static constexpr int E0 = (24 * 1024) / (G::ES * 8);
    static constexpr int E = E0 < 1 ? 1 : E0;
    static constexpr size_t SMEM = (size_t)2 * E * G::ES * 8;
};

// Group loop with one-group-ahead prefetch; body(in, e0, ne).
template <int P1, int NA, typename Body>
__device__ __forceinline__ void mma_group_loop(int64_t N, const double* __restrict__ src, double* buf0, Body body) {
    using C = MCfg<P1, NA>;
    using G = MG<P1, NA>;
    constexpr int E = C::E;
    const int64_t ngroups = (N + E - 1) / E;
    int64_t g = blockIdx.x;
    if (g < ngroups) mma_load_group<P1, NA, C::NT>(buf0, src + g * E * G::NPTS, (int)(N - g * E < E ? N - g * E : E));
    cp_async_commit();
    int cur = 0;
    for (; g < ngroups; g += gridDim.x) {
        const int64_t e0 = g * E;
        const int ne = (int)(N - e0 < E ? N - e0 : E);
        cp_async_wait_all();
        __syncthreads();
        double* in = buf0 + cur * E * G::ES;
        const int64_t gn = g + gridDim.x;
        if (gn < ngroups)
            mma_load_group<P1, NA, C::NT>(buf0 + (cur ^ 1) * E * G::ES, src + gn * E * G::NPTS,
                                          (int)(N - gn * E < E ? N - gn * E : E));
        cp_async_commit();
        body(in, e0, ne);
        cur ^= 1;
    }
}

// ------------------------------------------------------------------ sumfact3d
//   C along axis 0 (l), B along axis 1 (m), A along axis 2 (n) -> V (coalesced stores)
template <int P1>
__global__ void __launch_bounds__(MCfg<P1, P1>::NT) sumfact3d_mma_kernel(int64_t N, const double* __restrict__ A,
                                                                       const double* __restrict__ B,
                                                                       const double* __restrict__ C,
                                                                       const double* __restrict__ U,
                                                                       double* __restrict__ V,
                                                                       double* __restrict__ ws) {
    using G = MG<P1, P1>;
    constexpr int NW = MCfg<P1, P1>::NW;
    extern __shared__ __align__(16) double smd[];
    double aA[G::MF][G::KS], aB[G::MF][G::KS], aC[G::MF][G::KS];
    double sq = 0.0;
    load_afrag<P1>(aA, A);
    load_afrag<P1>(aB, B);
    load_afrag<P1>(aC, C);
    mma_group_loop<P1, P1>(N, U, smd, [&](double* in, int64_t e0, int ne) {
        mma_stage<P1, P1, 0, NW>(in, aC, ne, [&](int e, int l, int k, double v) {
            in[ML<P1, P1, 0>::base(e, l) + k * G::PS] = v;
        });
        __syncthreads();
        mma_stage<P1, P1, 1, NW>(in, aB, ne, [&](int e, int l, int k, double v) {
            in[ML<P1, P1, 1>::base(e, l) + k * G::RS] = v;
        });
        __syncthreads();
        double* Vg = V + e0 * G::NPTS;
        mma_stage<P1, P1, 2, NW>(in, aA, ne, [&](int e, int l, int k, double v) {
            st_cs(Vg + e * G::NPTS + ML<P1, P1, 2>::gofs(l, k), v);
            sq = fma(v, v, sq);
        });
    });
    if (ws != nullptr) block_partial(sq, ws + 8);
}

// ------------------------------------------------------------------ sumfact2d
//   B along axis "0" (l, columns), then A along the fastest axis (m) -> V
template <int P1>
__global__ void __launch_bounds__(MCfg<P1, 1>::NT) sumfact2d_mma_kernel(int64_t N, const double* __restrict__ A,
                                                                      const double* __restrict__ B,
                                                                      const double* __restrict__ U,
                                                                      double* __restrict__ V) {
    using G = MG<P1, 1>;
    constexpr int NW = MCfg<P1, 1>::NW;
    extern __shared__ __align__(16) double smd[];
    double aA[G::MF][G::KS], aB[G::MF][G::KS];
    load_afrag<P1>(aA, A);
    load_afrag<P1>(aB, B);
    mma_group_loop<P1, 1>(N, U, smd, [&](double* in, int64_t e0, int ne) {
        // 2-D element [a][c]: "axis 1" lines = columns c (contract a, stride RS)
        mma_stage<P1, 1, 1, NW>(in, aB, ne, [&](int e, int l, int k, double v) {
            in[ML<P1, 1, 1>::base(e, l) + k * G::RS] = v;
        });
        __syncthreads();
        double* Vg = V + e0 * G::NPTS;
        mma_stage<P1, 1, 2, NW>(in, aA, ne, [&](int e, int l, int k, double v) {
            st_cs(Vg + e * G::NPTS + ML<P1, 1, 2>::gofs(l, k), v);
        });
    });
}

// ------------------------------------------------------------------ local_grad3
//   ut (axis 0), us (axis 1), ur (axis 2) of U[k][j][i], all stored from fragments
template <int P1>
__global__ void __launch_bounds__(MCfg<P1, P1>::NT) local_grad3_mma_kernel(int64_t N, const double* __restrict__ D,
                                                                         const double* __restrict__ U,
                                                                         double* __restrict__ ur,
                                                                         double* __restrict__ us,
                                                                         double* __restrict__ ut) {
    using G = MG<P1, P1>;
    constexpr int NW = MCfg<P1, P1>::NW;
    extern __shared__ __align__(16) double smd[];
    double aD[G::MF][G::KS];
    load_afrag<P1>(aD, D);
    mma_group_loop<P1, P1>(N, U, smd, [&](double* in, int64_t e0, int ne) {
        const int64_t gb = e0 * G::NPTS;
        mma_stage<P1, P1, 0, NW>(in, aD, ne, [&](int e, int l, int k, double v) {
            st_cs(ut + gb + e * G::NPTS + ML<P1, P1, 0>::gofs(l, k), v);
        });
        mma_stage<P1, P1, 1, NW>(in, aD, ne, [&](int e, int l, int k, double v) {
            st_cs(us + gb + e * G::NPTS + ML<P1, P1, 1>::gofs(l, k), v);
        });
        mma_stage<P1, P1, 2, NW>(in, aD, ne, [&](int e, int l, int k, double v) {
            st_cs(ur + gb + e * G::NPTS + ML<P1, P1, 2>::gofs(l, k), v);
        });
    });
}

// ------------------------------------------------------------------ host
template <typename K>
static int mma_grid(K kernel, size_t smem, int nt, int64_t ngroups, int* occ) {
    if (*occ == 0) {
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int o = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kernel, nt, smem);
        *occ = o < 1 ? 1 : o;
    }
    const int64_t cap = (int64_t)num_sms() * *occ;
    return (int)(ngroups < cap ? ngroups : cap);
}

template <int P1>
static int launch_sf3d_mma(int64_t N, const double* A, const double* B, const double* C, const double* U, double* V,
                           double* ws, cudaStream_t s) {
    using CF = MCfg<P1, P1>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    int grid = mma_grid(sumfact3d_mma_kernel<P1>, CF::SMEM, CF::NT, (N + CF::E - 1) / CF::E, &occ);
    if (ws && grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
    sumfact3d_mma_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, A, B, C, U, V, ws);
    const int st = launch_status();
    if (st || !ws) return st;
    return run_check_finalize(grid, ws, s);
}
template <int P1>
static int launch_sf2d_mma(int64_t N, const double* A, const double* B, const double* U, double* V, cudaStream_t s) {
    using CF = MCfg<P1, 1>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int grid = mma_grid(sumfact2d_mma_kernel<P1>, CF::SMEM, CF::NT, (N + CF::E - 1) / CF::E, &occ);
    sumfact2d_mma_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, A, B, U, V);
    return launch_status();
}
template <int P1>
static int launch_lg3_mma(int64_t N, const double* D, const double* U, double* ur, double* us, double* ut,
                          cudaStream_t s) {
    using CF = MCfg<P1, P1>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int grid = mma_grid(local_grad3_mma_kernel<P1>, CF::SMEM, CF::NT, (N + CF::E - 1) / CF::E, &occ);
    local_grad3_mma_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, D, U, ur, us, ut);
    return launch_status();
}

// Dispatch table (measured on B200, tools/sweep_spectral.py; profiles/sweep_spectral_r01.jsonl):
// the tensor-core kernels win where padding P1 -> KP wastes little (P1 = 8, 15, 16: e.g.
// p = 15 sumfact3d 0.58 vs 0.39, sumfact2d 0.84 vs 0.50 of HBM peak) and lose at P1 = 13
// (37% padding waste; local_grad3 0.44 vs 0.71).  Returns 1 (not covered) otherwise; the
// caller then uses the DFMA kernels of spectral.cu.
#define BC_MMA_SWITCH(P1VAR, CALL) \
    switch (P1VAR) {               \
        case 8: return CALL(8);    \
        case 15: return CALL(15);  \
        case 16: return CALL(16);  \
        default: return 1;  /* not covered */ \
    }

int run_sumfact3d_mma(int64_t N, int p, const double* A, const double* B, const double* C, const double* U, double* V,
                      double* ws, cudaStream_t s) {
#define CALL(P) launch_sf3d_mma<P>(N, A, B, C, U, V, ws, s)
    BC_MMA_SWITCH(p + 1, CALL)
#undef CALL
}
int run_sumfact2d_mma(int64_t N, int p, const double* A, const double* B, const double* U, double* V, cudaStream_t s) {
#define CALL(P) launch_sf2d_mma<P>(N, A, B, U, V, s)
    BC_MMA_SWITCH(p + 1, CALL)
#undef CALL
}
int run_local_grad3_mma(int64_t N, int p, const double* D, const double* U, double* ur, double* us, double* ut,
                        cudaStream_t s) {
#define CALL(P) launch_lg3_mma<P>(N, D, U, ur, us, ut, s)
    BC_MMA_SWITCH(p + 1, CALL)
#undef CALL
}

}  // namespace bc
