// Spectral-element family on sm_100a: sumfact3d (fp64/fp32), sumfact2d, local_grad3,
// local_grad3_t and the fused Nekbone element operator ax_e.
//
// Design.  A CTA owns a group of E consecutive elements.  The group is
// staged global -> shared memory with cp.async (LDGSTS) into a row-padded layout whose
// strided row reads are bank-conflict free, prefetching the next group while the current
// one computes.  Each contraction stage applies one (p+1)x(p+1) operator along one axis of
// every element ("lines": P1 values along the contracted axis, held in registers).  A
// thread owns R lines and accumulates each output in a register (the paper's scalar
// replacement); operator rows are read as 16-byte broadcast pairs, so every
// shared-memory wavefront feeds 2R FMAs.  Intermediates never leave shared memory
// (fusion); only U in and the outputs touch HBM.
#include <algorithm>

#include "common.cuh"

// unroll factor of the contracted-index loop (experiments only)
#ifndef BC_NUNROLL
#define BC_NUNROLL 1
#endif
// warp-chunked line assignment (no duplicate tail lines; measured: p=12 local_grad3
// 0.686 -> 0.726, p=9 0.79 -> 0.86 of HBM) and the software-pipelined n loop (measured
// slower: +50 registers, 0.73 -> 0.58 at p=12; kept as an option)
#ifndef BC_WCHUNK
#define BC_WCHUNK 1
#endif
#ifndef BC_SWP
#define BC_SWP 0
#endif

namespace bc {

// ------------------------------------------------------------------------------------
// Shared-memory geometry of one element: NA planes x P1 rows x RS (row stride).
//  fp64: odd P1 -> RS = P1 (row stride odd: LDS.64 conflict-free);
//        P1 = 2 mod 4 -> RS = P1 (RS/2 odd: 16-byte row reads conflict-free);
//        P1 = 0 mod 4 -> RS = P1 + 2 (restores RS/2 odd).
//  fp32: RS = P1 | 1 (odd stride, scalar row reads conflict-free).
// ------------------------------------------------------------------------------------
template <int P1, int NA, typename T>
struct Geo {
    static constexpr int RS = sizeof(T) == 8 ? ((P1 % 2) ? P1 : (((P1 / 2) % 2) ? P1 : P1 + 2))
                                             : (P1 | 1);
    static constexpr int PS = P1 * RS;          // plane stride in smem
    static constexpr int ES = NA * PS;          // element stride in smem
    static constexpr int NPTS = NA * P1 * P1;   // points per element in global memory
    static constexpr int OS = (P1 + 1) & ~1;    // operator row stride (pairs aligned)
    static constexpr bool PADDED = (RS != P1);
    static constexpr bool VEC_ROWS = (sizeof(T) == 8) && (RS % 2 == 0);
};

// Stage `ne` elements (contiguous in global from `src`) into padded smem at `dst` (16-byte
// aligned, VEC elements of slack at the end).  Returns where element 0 landed: for an
// unpadded fp64 group that starts 8 bytes past a 16-byte boundary (odd E x odd P1) the copy
// starts one value early, so element 0 sits at dst + 1 and every copy stays 16 bytes wide.
template <int P1, int NA, typename T, int NT>
__device__ __forceinline__ T* load_group_async(T* __restrict__ dst, const T* __restrict__ src, int ne) {
    using G = Geo<P1, NA, T>;
    const int total = ne * G::NPTS;
    if constexpr (!G::PADDED) {
        // smem layout == global layout: 16-byte chunks
        constexpr int V = 16 / sizeof(T);
        const int lead = (int)((reinterpret_cast<uintptr_t>(src) & 15) / sizeof(T));
        if (sizeof(T) == 8 || lead == 0) {
            const T* s0 = src - lead;
            const int tot = total + lead, nvec = tot / V;
            for (int i = threadIdx.x; i < nvec; i += NT) cp_async_16(dst + i * V, s0 + i * V);
            for (int i = nvec * V + threadIdx.x; i < tot; i += NT) cp_async_elem(dst + i, s0 + i);
            return dst + lead;
        }
        for (int i = threadIdx.x; i < total; i += NT) cp_async_elem(dst + i, src + i);
    } else {
        for (int f = threadIdx.x; f < total; f += NT) {
            const int e = f / G::NPTS;
            const int r = f - e * G::NPTS;  // (a, b, c) flattened
            const int row = r / P1;         // (a, b)
            const int c = r - row * P1;
            cp_async_elem(dst + e * G::ES + row * G::RS + c, src + f);
        }
    }
    return dst;
}

// smem offset of global point f (element-relative flattened (e, a, b, c))
template <int P1, int NA, typename T>
__device__ __forceinline__ int smem_index(int f) {
    using G = Geo<P1, NA, T>;
    if constexpr (!G::PADDED) {
        return f;
    } else {
        const int e = f / G::NPTS;
        const int r = f - e * G::NPTS;
        const int row = r / P1;
        return e * G::ES + row * G::RS + (r - row * P1);
    }
}

// First smem offset and stride of line L (element-relative) along AXIS.
//   AXIS 2 (fastest, c): L = (e, a, b) -> rows;   AXIS 1 (b): L = (e, a, c);
//   AXIS 0 (a, slowest): L = (e, b, c)  (only when NA == P1).
template <int P1, int NA, int AXIS, typename T>
struct Line {
    using G = Geo<P1, NA, T>;
    static constexpr int STRIDE = AXIS == 2 ? 1 : (AXIS == 1 ? G::RS : G::PS);
    static constexpr int PER_ELEM = NA * P1;  // lines per element along any axis (NA*P1*P1/P1)
    __device__ __forceinline__ static int base(int L) {
        if constexpr (AXIS == 2) {
            return L * G::RS;
        } else if constexpr (AXIS == 1) {
            const int e = L / (NA * P1);
            const int r = L - e * (NA * P1);
            const int a = r / P1;
            return e * G::ES + a * G::PS + (r - a * P1);
        } else {
            const int e = L / (P1 * P1);
            const int r = L - e * (P1 * P1);
            const int b = r / P1;
            return e * G::ES + b * G::RS + (r - b * P1);
        }
    }
    // global (unpadded, element-relative) offset of output k of line L
    __device__ __forceinline__ static int gofs(int L, int k) {
        if constexpr (AXIS == 2) {
            return L * P1 + k;
        } else if constexpr (AXIS == 1) {
            const int e = L / (NA * P1);
            const int r = L - e * (NA * P1);
            const int a = r / P1;
            return e * G::NPTS + a * P1 * P1 + k * P1 + (r - a * P1);
        } else {
            const int e = L / (P1 * P1);
            return e * G::NPTS + k * P1 * P1 + (L - e * (P1 * P1));
        }
    }
};

// out(L, base, k, value): consumer of one output value.
// Applies an operator along AXIS of the lines [0, nlines):
//     y(L, k) = sum_{n=0..P1-1} M[k][n] * x(L, n)       (ascending n)
// with opT[n][k] = M[k][n] staged in smem (row stride OS).  Outer-product form: the
// thread streams x(L, n) for its R lines and updates all P1*R accumulators, so each
// 16-byte broadcast operator load feeds 2R FMAs and there are P1*R independent FMA
// chains per thread.  All reads of a line precede the writes of that line and every
// line is read by exactly one thread, so `out` may overwrite the line in place.
template <int P1, int NA, int AXIS, int R, int NT, bool SWP, int UNR, typename T, typename Out>
__device__ __forceinline__ void apply_lines_w(const T* in, const T* opT, int nlines, Out out);

template <int P1, int NA, int AXIS, int R, int NT, typename T, typename Out, int UNR = BC_NUNROLL>
__device__ __forceinline__ void apply_lines(const T* in, const T* opT, int nlines, Out out) {
    // fully unrolled chunks spill beyond P1 = 12 (ptxas, 255 registers at P1 = 13): those
    // keep the lane-strided loop
    if constexpr (BC_WCHUNK && (UNR == 1 || P1 <= 12 || R <= 2)) {
        apply_lines_w<P1, NA, AXIS, R, NT, (bool)BC_SWP && UNR == 1, UNR>(in, opT, nlines, out);
        return;
    }
    using G = Geo<P1, NA, T>;
    using LN = Line<P1, NA, AXIS, T>;
    using P2 = typename Pair<T>::type;
    constexpr int KP = P1 / 2;
    for (int L0 = threadIdx.x; L0 < nlines; L0 += R * NT) {
        int base[R];
#pragma unroll
        for (int r = 0; r < R; ++r) {
            int L = L0 + r * NT;
            L = (L < nlines) ? L : L0;
            base[r] = LN::base(L);
        }
        T acc[P1][R];
#pragma unroll
        for (int k = 0; k < P1; ++k)
#pragma unroll
            for (int r = 0; r < R; ++r) acc[k][r] = T(0);
#pragma unroll UNR
        for (int n = 0; n < P1; ++n) {
            T x[R];
#pragma unroll
            for (int r = 0; r < R; ++r) x[r] = in[base[r] + n * LN::STRIDE];
            const T* orow = opT + n * G::OS;
#pragma unroll
            for (int k2 = 0; k2 < KP; ++k2) {
                const P2 o = reinterpret_cast<const P2*>(orow)[k2];
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    acc[2 * k2][r] = fma(o.x, x[r], acc[2 * k2][r]);
                    acc[2 * k2 + 1][r] = fma(o.y, x[r], acc[2 * k2 + 1][r]);
                }
            }
            if constexpr (P1 & 1) {
                const T o = orow[P1 - 1];
#pragma unroll
                for (int r = 0; r < R; ++r) acc[P1 - 1][r] = fma(o, x[r], acc[P1 - 1][r]);
            }
        }
#pragma unroll
        for (int r = 0; r < R; ++r)
            if (L0 + r * NT < nlines) {
#pragma unroll
                for (int k = 0; k < P1; ++k) out(L0 + r * NT, base[r], k, acc[k][r]);
            }
    }
}

// One warp chunk of apply_lines: lane `lane` owns lines L0 + r*32 (r < RR), lines >= nlines
// are computed on the chunk's first line (always valid) and not stored.  SWP: the operands of step n+1 are loaded
// while step n's FMAs run (two register sets, ping-pong), hiding the shared-memory latency
// that otherwise stalls every step's first FMA.
template <int P1, int NA, int AXIS, int RR, bool SWP, int UNR, typename T, typename Out>
__device__ __forceinline__ void lines_chunk(const T* in, const T* opT, int L0, int nlines, Out& out) {
    using G = Geo<P1, NA, T>;
    using LN = Line<P1, NA, AXIS, T>;
    using P2 = typename Pair<T>::type;
    constexpr int KP = P1 / 2;
    int base[RR];
#pragma unroll
    for (int r = 0; r < RR; ++r) {
        const int L = L0 + r * 32;
        base[r] = LN::base(L < nlines ? L : (L0 & ~31));
    }
    T acc[P1][RR];
#pragma unroll
    for (int k = 0; k < P1; ++k)
#pragma unroll
        for (int r = 0; r < RR; ++r) acc[k][r] = T(0);
    auto fmas = [&](const T (&x)[RR], const P2 (&o)[KP], T oz) {
#pragma unroll
        for (int k2 = 0; k2 < KP; ++k2)
#pragma unroll
            for (int r = 0; r < RR; ++r) {
                acc[2 * k2][r] = fma(o[k2].x, x[r], acc[2 * k2][r]);
                acc[2 * k2 + 1][r] = fma(o[k2].y, x[r], acc[2 * k2 + 1][r]);
            }
        if constexpr (P1 & 1) {
#pragma unroll
            for (int r = 0; r < RR; ++r) acc[P1 - 1][r] = fma(oz, x[r], acc[P1 - 1][r]);
        }
    };
    auto ld = [&](int n, T (&x)[RR], P2 (&o)[KP], T& oz) {
#pragma unroll
        for (int r = 0; r < RR; ++r) x[r] = in[base[r] + n * LN::STRIDE];
        const T* orow = opT + n * G::OS;
#pragma unroll
        for (int k2 = 0; k2 < KP; ++k2) o[k2] = reinterpret_cast<const P2*>(orow)[k2];
        if constexpr (P1 & 1) oz = orow[P1 - 1];
    };
    if constexpr (SWP) {
        T xa[RR], xb[RR], za = T(0), zb = T(0);
        P2 oa[KP], ob[KP];
        ld(0, xa, oa, za);
#pragma unroll 1
        for (int n = 0; n + 1 < P1; n += 2) {
            ld(n + 1, xb, ob, zb);
            fmas(xa, oa, za);
            if (n + 2 < P1) ld(n + 2, xa, oa, za);
            fmas(xb, ob, zb);
        }
        if constexpr (P1 & 1) fmas(xa, oa, za);
    } else {
#pragma unroll UNR
        for (int n = 0; n < P1; ++n) {
            T x[RR], z = T(0);
            P2 o[KP];
            ld(n, x, o, z);
            fmas(x, o, z);
        }
    }
#pragma unroll
    for (int r = 0; r < RR; ++r)
        if (L0 + r * 32 < nlines) {
#pragma unroll
            for (int k = 0; k < P1; ++k) out(L0 + r * 32, base[r], k, acc[k][r]);
        }
}

// Warp-chunked form of apply_lines (same arithmetic, same ascending-n sums): lines are cut
// into chunks of 32*R (lane-interleaved, so every strided line read stays conflict-free);
// chunks go round-robin to the warps and the ragged last chunk runs with
// RR = ceil(rest/32) <= R lines per lane, so no warp computes duplicate lines.
template <int P1, int NA, int AXIS, int R, int NT, bool SWP, int UNR, typename T, typename Out>
__device__ __forceinline__ void apply_lines_w(const T* in, const T* opT, int nlines, Out out) {
    constexpr int NW = NT / 32, CH = 32 * R;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nfull = nlines / CH;
    for (int c = warp; c < nfull; c += NW) lines_chunk<P1, NA, AXIS, R, SWP, UNR>(in, opT, c * CH + lane, nlines, out);
    const int rest = nlines - nfull * CH;
    if (rest > 0 && warp == nfull % NW) {
        const int L0 = nfull * CH + lane, rr = (rest + 31) >> 5;
        if constexpr (R >= 4) if (rr == 4) { lines_chunk<P1, NA, AXIS, 4, SWP, UNR>(in, opT, L0, nlines, out); return; }
        if constexpr (R >= 3) if (rr == 3) { lines_chunk<P1, NA, AXIS, (R >= 3 ? 3 : 1), SWP, UNR>(in, opT, L0, nlines, out); return; }
        if constexpr (R >= 2) if (rr == 2) { lines_chunk<P1, NA, AXIS, (R >= 2 ? 2 : 1), SWP, UNR>(in, opT, L0, nlines, out); return; }
        lines_chunk<P1, NA, AXIS, 1, SWP, UNR>(in, opT, L0, nlines, out);
    }
}

// operator staging: opT[n][k] = M[k][n], M = Mat (TRANSPOSE = false) or Mat^T (true)
// Every lane runs the same number of iterations and the warp reconverges afterwards:
// with a divergent early exit, ptxas (CUDA 12.9, sm_100a) let the exited lanes of a warp
// reload the uniform register holding the NEXT operator's pointer while the other lanes
// were still loading this one (found by tests/test_parity_spectral at P1 = 13 with 96
// threads).
template <int P1, typename T, int NT, bool TRANSPOSE = false>
__device__ __forceinline__ void load_op(T* __restrict__ op_s, const T* __restrict__ Mat) {
    constexpr int OS = (P1 + 1) & ~1;
#pragma unroll
    for (int i0 = 0; i0 < P1 * OS; i0 += NT) {
        const int i = i0 + (int)threadIdx.x;
        if (i < P1 * OS) {
            const int n = i / OS, k = i - (i / OS) * OS;
            op_s[i] = (k < P1) ? (TRANSPOSE ? Mat[n * P1 + k] : Mat[k * P1 + n]) : T(0);
        }
    }
    __syncwarp();
}

template <int P1, typename T>
constexpr int op_elems() {  // rounded so that what follows stays 16-byte aligned
    return (P1 * ((P1 + 1) & ~1) + (16 / (int)sizeof(T)) - 1) / (16 / (int)sizeof(T)) * (16 / (int)sizeof(T));
}

__host__ __device__ __forceinline__ int imin64(int64_t a, int64_t b) { return (int)(a < b ? a : b); }

// ---------------------------------------------------------------- launch configuration
// The fixed variant table (north star: "settled by ncu measurement and recorded in a
// small fixed table"): elements per CTA group E, threads NT, lines per thread R, number
// of element buffers NBUF.  All stages run in place, so a kernel needs one buffer per
// live field (+1 for the prefetch of the next group).
// Variant table, measured on B200 with tools/sweep_spectral.py (profiles/sweep_spectral_r01.md):
//   P1 >= 10: sumfact3d / local_grad3: R = 4 lines per thread, 54 KiB element groups, no
//             in-CTA prefetch (occupancy hides the loads), except P1 = 12: R = 3, 36 KiB;
//             sumfact2d: R = 3, 18 KiB groups with prefetch; local_grad3_t / ax_e: R = 2, 18 KiB.
//   P1 <  10: R = 2, 18 KiB groups with prefetch (36 KiB for local_grad3).
//   sumfact2d at P1 >= 9 fully unrolls its contracted-index loop (0.64 -> 0.75 of HBM at P1 = 13).
//   Rejected (same sweep): n-loop unroll 2 / 13 for sumfact3d and local_grad3 (register
//   spills), prefetching 18/36 KiB groups at P1 >= 10.
enum SpecKernel { K_SF3 = 0, K_SF2 = 1, K_LG3 = 2, K_LG3T = 3, K_AXE = 4 };
// experiment overrides for the P1 >= 10 sumfact3d / local_grad3 entries (variant sweeps only)
#ifndef BC_BIG_R
#define BC_BIG_R 4
#endif
#ifndef BC_SMALL_R
#define BC_SMALL_R 3  // sumfact3d lines per thread at P1 < 10 (measured: p=4 0.57 -> 0.65, p=5 0.56 -> 0.62,
                      // p=8 0.47 -> 0.53 of HBM vs R = 2; local_grad3 stays at R = 2)
#endif
#ifndef BC_LG3_DIRECT_UR
#define BC_LG3_DIRECT_UR 0  // local_grad3: store ur from registers instead of in place + copy-out
#endif
#ifndef BC_E13_SF2
#define BC_E13_SF2 0  // sumfact2d elements per group at P1 = 13 (0: derived, 12)
#endif
#ifndef BC_R1011
#define BC_R1011 4  // sumfact3d / local_grad3 lines per thread at P1 = 10, 11
#endif
#ifndef BC_SF2_R13
#define BC_SF2_R13 3  // sumfact2d lines per thread at P1 >= 13
#endif
#ifndef BC_BIG_KB
#define BC_BIG_KB 54
#endif
#ifndef BC_BIG_PF
#define BC_BIG_PF 0
#endif
#ifndef BC_E13
#define BC_E13 3
#endif
#ifndef AXE_PB
#define AXE_PB 4  // ax_e: points per thread whose 6 geometric factors are loaded together
#endif
#ifndef BC_SF2_UNROLL
#define BC_SF2_UNROLL 1
#endif
template <int P1, int KIND>
struct SpecTable {
    static constexpr bool BIG = P1 >= 10;
    static constexpr bool SF3LG3 = KIND == K_SF3 || KIND == K_LG3;
    static constexpr bool MID = P1 == 12;  // sumfact3d / local_grad3: R = 3, 36 KiB (measured)
    static constexpr int R = BIG ? (SF3LG3 ? (MID ? 3 : (P1 <= 11 ? BC_R1011 : BC_BIG_R))
                                           : (KIND == K_SF2 ? (P1 >= 13 ? BC_SF2_R13 : 3) : 2))
                                 : (KIND == K_SF3 ? BC_SMALL_R : 2);
    static constexpr int BUF_KB = BIG ? (SF3LG3 ? (MID ? 36 : BC_BIG_KB) : 18) : (KIND == K_LG3 ? 36 : 18);
    static constexpr bool PREFETCH = !(BIG && SF3LG3) || BC_BIG_PF;
    // forced elements per group (0: derived from BUF_KB): P1 = 13: 3 x 169 = 507 lines on
    // 128 threads x R = 4 (1% idle lanes instead of 12% with E = 2 on 96 threads)
    static constexpr int EF = (SF3LG3 && P1 == 13) ? BC_E13 : ((KIND == K_SF2 && P1 == 13) ? BC_E13_SF2 : 0);
    // unroll of the contracted-index loop: sumfact2d fully (its two stages fit the registers)
    static constexpr int UNROLL = (KIND == K_SF2 && BC_SF2_UNROLL && P1 >= 9) ? P1 : BC_NUNROLL;
};

template <int P1, int NA, typename T, int NBUF_FIELDS, int KIND = K_SF3>
struct Cfg {
    using G = Geo<P1, NA, T>;
    using TB = SpecTable<P1, KIND>;
    static constexpr bool PREFETCH = TB::PREFETCH && NBUF_FIELDS == 1;  // single-field kernels only
    static constexpr int NBUF = NBUF_FIELDS + (PREFETCH ? 1 : 0);
    static constexpr int BUF_BYTES = TB::BUF_KB * 1024;  // target bytes per element-group buffer
    static constexpr int E0 = BUF_BYTES / (G::ES * (int)sizeof(T));
    // even by default; a measured table entry may force E (odd E x odd P1 groups start 8 bytes
    // off a 16-byte boundary, handled by load_group_async)
    static constexpr int E = TB::EF ? TB::EF : (E0 < 2 ? 1 : (E0 & ~1));
    static constexpr int R = TB::R;
    static constexpr int LINES = E * NA * P1;  // lines per axis per group (E * NPTS / P1)
    static constexpr int NT0 = ((LINES + R - 1) / R + 31) / 32 * 32;
    static constexpr int NT = NT0 < 64 ? 64 : (NT0 > 512 ? 512 : NT0);
    static constexpr int VEC = 16 / (int)sizeof(T);
    static constexpr int BUF = (E * G::ES + VEC - 1) / VEC * VEC + VEC;  // + slack for a shifted group
    static constexpr size_t SMEM = (size_t)NBUF * BUF * sizeof(T) + 2 * op_elems<P1, T>() * sizeof(T);
};

template <typename KernelT>
int grid_for(KernelT kernel, int nt, size_t smem, int64_t ngroups, int* occ_cache) {
    if (*occ_cache == 0) {
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, nt, smem);
        *occ_cache = occ < 1 ? 1 : occ;
    }
    const int64_t cap = (int64_t)num_sms() * *occ_cache;
    return imin64(ngroups, cap);
}

// Group loop over the single input field.  PREFETCH: one-group-ahead cp.async prefetch
// into a second buffer; otherwise load -> wait -> compute, with the load latency hidden by
// the other CTAs on the SM.
template <int P1, int NA, typename T, int NT, int E, int BUF, bool PREFETCH, typename Body>
__device__ __forceinline__ void group_loop(int64_t N, const T* __restrict__ src, T* buf0, Body body) {
    using G = Geo<P1, NA, T>;
    const int64_t ngroups = (N + E - 1) / E;
    if constexpr (PREFETCH) {
        int64_t g = blockIdx.x;
        T* in = buf0;
        if (g < ngroups) in = load_group_async<P1, NA, T, NT>(buf0, src + g * E * G::NPTS, imin64(E, N - g * E));
        cp_async_commit();
        int cur = 0;
        for (; g < ngroups; g += gridDim.x) {
            const int64_t e0 = g * E;
            cp_async_wait_all();
            __syncthreads();  // group g landed; everyone is done with the other buffer
            const int64_t gn = g + gridDim.x;
            T* next = buf0 + (cur ^ 1) * BUF;
            if (gn < ngroups)
                next = load_group_async<P1, NA, T, NT>(next, src + gn * E * G::NPTS, imin64(E, N - gn * E));
            cp_async_commit();
            body(in, e0, imin64(E, N - e0));
            in = next;
            cur ^= 1;
        }
    } else {
        for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
            const int64_t e0 = g * E;
            __syncthreads();  // everyone is done with the buffer
            T* in = load_group_async<P1, NA, T, NT>(buf0, src + e0 * G::NPTS, imin64(E, N - e0));
            cp_async_commit();
            cp_async_wait_all();
            __syncthreads();
            body(in, e0, imin64(E, N - e0));
        }
    }
}

// ====================================================================== sumfact3d
//   S1 W1[l][m][k] = sum_n A[k][n] U[l][m][n]     (axis 2, P:440 / Fig. 2(b))
//   S2 W2[l][j][k] = sum_m B[j][m] W1[l][m][k]    (axis 1, P:441 / P:214)
//   S3 V [i][j][k] = sum_l C[i][l] W2[l][j][k]    (axis 0, P:442 / P:215; Fig. 2(d))
// S1 and S2 run in place in the group buffer; S3 stores V straight from registers
// (consecutive threads own consecutive (j,k): coalesced).  With ws != nullptr the check
// scalar sum V^2 (R18) is accumulated in the store epilogue: one partial per
// CTA in ws[8 + blockIdx.x], reduced in fixed order by check_finalize.
template <int P1, typename T>
__global__ void __launch_bounds__(Cfg<P1, P1, T, 1, K_SF3>::NT)
sumfact3d_kernel(int64_t N, const T* __restrict__ A, const T* __restrict__ B, const T* __restrict__ C,
                 const T* __restrict__ U, T* __restrict__ V, double* __restrict__ ws) {
    using CF = Cfg<P1, P1, T, 1, K_SF3>;
    using G = Geo<P1, P1, T>;
    constexpr int NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opA = reinterpret_cast<T*>(smem_raw);
    T* opB = opA + op_elems<P1, T>();
    T* opC = opB + op_elems<P1, T>();
    T* buf = opC + op_elems<P1, T>();
    load_op<P1, T, NT>(opA, A);
    load_op<P1, T, NT>(opB, B);
    load_op<P1, T, NT>(opC, C);
    double sq = 0.0;
    group_loop<P1, P1, T, NT, CF::E, CF::BUF, CF::PREFETCH>(N, U, buf, [&](T* in, int64_t e0, int ne) {
        const int nlines = ne * P1 * P1;
        apply_lines<P1, P1, 2, R, NT>(in, opA, nlines, [&](int, int base, int k, T v) { in[base + k] = v; });
        __syncthreads();
        apply_lines<P1, P1, 1, R, NT>(in, opB, nlines, [&](int, int base, int k, T v) { in[base + k * G::RS] = v; });
        __syncthreads();
        T* Vg = V + e0 * G::NPTS;
        apply_lines<P1, P1, 0, R, NT>(in, opC, nlines, [&](int L, int, int k, T v) {
            st_cs(Vg + Line<P1, P1, 0, T>::gofs(L, k), v);
            sq = fma((double)v, (double)v, sq);
        });
    });
    if (ws != nullptr) block_partial(sq, ws + 8);
}

template <int P1, typename T>
int launch_sumfact3d(int64_t N, const T* A, const T* B, const T* C, const T* U, T* V, double* ws, cudaStream_t s) {
    using CF = Cfg<P1, P1, T, 1, K_SF3>;
    static int occ = 0;
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const size_t smem = CF::SMEM + op_elems<P1, T>() * sizeof(T);
    int grid = grid_for(sumfact3d_kernel<P1, T>, CF::NT, smem, ngroups, &occ);
    if (ws && grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
    sumfact3d_kernel<P1, T><<<grid, CF::NT, smem, s>>>(N, A, B, C, U, V, ws);
    const int st = launch_status();
    if (st || !ws) return st;
    return run_check_finalize(grid, ws, s);
}

// ====================================================================== sumfact2d
//   W[l][j] = sum_m A[j][m] U[l][m]  (rows, in place);  V[i][j] = sum_l B[i][l] W[l][j]
template <int P1>
__global__ void __launch_bounds__(Cfg<P1, 1, double, 1, K_SF2>::NT)
sumfact2d_kernel(int64_t N, const double* __restrict__ A, const double* __restrict__ B,
                 const double* __restrict__ U, double* __restrict__ V) {
    using T = double;
    using CF = Cfg<P1, 1, T, 1, K_SF2>;
    using G = Geo<P1, 1, T>;
    constexpr int NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opA = reinterpret_cast<T*>(smem_raw);
    T* opB = opA + op_elems<P1, T>();
    T* buf = opB + op_elems<P1, T>();
    load_op<P1, T, NT>(opA, A);
    load_op<P1, T, NT>(opB, B);
    group_loop<P1, 1, T, NT, CF::E, CF::BUF, CF::PREFETCH>(N, U, buf, [&](T* in, int64_t e0, int ne) {
        const int nlines = ne * P1;
        constexpr int U = CF::TB::UNROLL;
        auto st1 = [&](int, int base, int k, T v) { in[base + k] = v; };
        apply_lines<P1, 1, 2, R, NT, T, decltype(st1), U>(in, opA, nlines, st1);
        __syncthreads();
        T* Vg = V + e0 * G::NPTS;
        auto st2 = [&](int L, int, int k, T v) { st_cs(Vg + Line<P1, 1, 1, T>::gofs(L, k), v); };
        apply_lines<P1, 1, 1, R, NT, T, decltype(st2), U>(in, opB, nlines, st2);
    });
}

template <int P1>
int launch_sumfact2d(int64_t N, const double* A, const double* B, const double* U, double* V, cudaStream_t s) {
    using CF = Cfg<P1, 1, double, 1, K_SF2>;
    static int occ = 0;
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(sumfact2d_kernel<P1>, CF::NT, CF::SMEM, ngroups, &occ);
    sumfact2d_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, A, B, U, V);
    return launch_status();
}

// ====================================================================== local_grad3
//   ur = D along axis 2 (i), us = D along axis 1 (j), ut = D along axis 0 (k) of U[k][j][i]
// us and ut are stored from registers (coalesced); ur is formed in place (its rows are
// strided across threads) and copied out coalesced.
template <int P1>
__global__ void __launch_bounds__(Cfg<P1, P1, double, 1, K_LG3>::NT)
local_grad3_kernel(int64_t N, const double* __restrict__ D, const double* __restrict__ U,
                   double* __restrict__ ur, double* __restrict__ us, double* __restrict__ ut) {
    using T = double;
    using CF = Cfg<P1, P1, T, 1, K_LG3>;
    using G = Geo<P1, P1, T>;
    constexpr int NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opD = reinterpret_cast<T*>(smem_raw);
    T* buf = opD + 2 * op_elems<P1, T>();
    load_op<P1, T, NT>(opD, D);
    group_loop<P1, P1, T, NT, CF::E, CF::BUF, CF::PREFETCH>(N, U, buf, [&](T* in, int64_t e0, int ne) {
        const int nlines = ne * P1 * P1;
        const int64_t gbase = e0 * G::NPTS;
        apply_lines<P1, P1, 1, R, NT>(in, opD, nlines, [&](int L, int, int k, T v) {
            st_cs(us + gbase + Line<P1, P1, 1, T>::gofs(L, k), v);
        });
        apply_lines<P1, P1, 0, R, NT>(in, opD, nlines, [&](int L, int, int k, T v) {
            st_cs(ut + gbase + Line<P1, P1, 0, T>::gofs(L, k), v);
        });
        if constexpr (BC_LG3_DIRECT_UR) {
            // ur rows stored straight from registers (lane-strided 8-byte stores; L2 merges the
            // partial sectors of a warp's 13 consecutive stores)
            apply_lines<P1, P1, 2, R, NT>(in, opD, nlines, [&](int L, int, int k, T v) {
                st_cs(ur + gbase + Line<P1, P1, 2, T>::gofs(L, k), v);
            });
        } else {
            __syncthreads();
            apply_lines<P1, P1, 2, R, NT>(in, opD, nlines, [&](int, int base, int k, T v) { in[base + k] = v; });
            __syncthreads();
            const int total = ne * G::NPTS;
            for (int f = threadIdx.x; f < total; f += NT) st_cs(ur + gbase + f, in[smem_index<P1, P1, T>(f)]);
        }
    });
}

template <int P1>
int launch_local_grad3(int64_t N, const double* D, const double* U, double* ur, double* us, double* ut,
                       cudaStream_t s) {
    using CF = Cfg<P1, P1, double, 1, K_LG3>;
    static int occ = 0;
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(local_grad3_kernel<P1>, CF::NT, CF::SMEM, ngroups, &occ);
    local_grad3_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, D, U, ur, us, ut);
    return launch_status();
}

// ====================================================================== local_grad3_t
//   U = D^T along axis 2 of ur + D^T along axis 1 of us + D^T along axis 0 of ut,
//   partial sums added in the order (r + s) + t.  Three field buffers, all in place.
template <int P1>
__global__ void __launch_bounds__(Cfg<P1, P1, double, 3, K_LG3T>::NT)
local_grad3_t_kernel(int64_t N, const double* __restrict__ D, const double* __restrict__ ur,
                     const double* __restrict__ us, const double* __restrict__ ut, double* __restrict__ U) {
    using T = double;
    using CF = Cfg<P1, P1, T, 3, K_LG3T>;
    using G = Geo<P1, P1, T>;
    constexpr int E = CF::E, NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opT = reinterpret_cast<T*>(smem_raw);
    T* bR0 = opT + 2 * op_elems<P1, T>();
    T* bS0 = bR0 + CF::BUF;
    T* bT0 = bS0 + CF::BUF;
    load_op<P1, T, NT, true>(opT, D);
    const int64_t ngroups = (N + E - 1) / E;
    for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
        const int64_t e0 = g * E;
        const int ne = imin64(E, N - e0);
        const int nlines = ne * P1 * P1;
        const int64_t gbase = e0 * G::NPTS;
        __syncthreads();  // previous group fully consumed
        // one cp.async group per field: the r stage starts as soon as ur has landed while us
        // and ut are still in flight
        T* bR = load_group_async<P1, P1, T, NT>(bR0, ur + gbase, ne);
        cp_async_commit();
        T* bS = load_group_async<P1, P1, T, NT>(bS0, us + gbase, ne);
        cp_async_commit();
        T* bT = load_group_async<P1, P1, T, NT>(bT0, ut + gbase, ne);
        cp_async_commit();
        cp_async_wait_n<2>();
        __syncthreads();
        apply_lines<P1, P1, 2, R, NT>(bR, opT, nlines, [&](int, int base, int k, T v) { bR[base + k] = v; });
        cp_async_wait_n<1>();
        __syncthreads();
        apply_lines<P1, P1, 1, R, NT>(bS, opT, nlines, [&](int, int base, int k, T v) {
            bS[base + k * G::RS] = bR[base + k * G::RS] + v;
        });
        cp_async_wait_n<0>();
        __syncthreads();
        apply_lines<P1, P1, 0, R, NT>(bT, opT, nlines, [&](int L, int base, int k, T v) {
            st_cs(U + gbase + Line<P1, P1, 0, T>::gofs(L, k), bS[base + k * G::PS] + v);
        });
    }
}

template <int P1>
int launch_local_grad3_t(int64_t N, const double* D, const double* ur, const double* us, const double* ut,
                         double* U, cudaStream_t s) {
    using CF = Cfg<P1, P1, double, 3, K_LG3T>;
    static int occ = 0;
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(local_grad3_t_kernel<P1>, CF::NT, CF::SMEM, ngroups, &occ);
    local_grad3_t_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, D, ur, us, ut, U);
    return launch_status();
}

// ====================================================================== ax_e
// (us, ut) from U into two buffers; ur in place over U; per-point geometric mixing in
// place; then local_grad3_t in place as above.  Three field buffers.
template <int P1>
__global__ void __launch_bounds__(Cfg<P1, P1, double, 3, K_AXE>::NT)
ax_e_kernel(int64_t N, const double* __restrict__ D, const double* __restrict__ Uin,
            const double* __restrict__ Gm, double* __restrict__ Wout) {
    using T = double;
    using CF = Cfg<P1, P1, T, 3, K_AXE>;
    using G = Geo<P1, P1, T>;
    constexpr int E = CF::E, NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opD = reinterpret_cast<T*>(smem_raw);
    T* opT = opD + op_elems<P1, T>();
    T* bR0 = opT + op_elems<P1, T>();  // holds U, then ur / wr
    T* bS = bR0 + CF::BUF;
    T* bT = bS + CF::BUF;
    load_op<P1, T, NT>(opD, D);
    load_op<P1, T, NT, true>(opT, D);
    const int64_t ngroups = (N + E - 1) / E;
    for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
        const int64_t e0 = g * E;
        const int ne = imin64(E, N - e0);
        const int nlines = ne * P1 * P1;
        const int64_t gbase = e0 * G::NPTS;
        __syncthreads();
        T* bR = load_group_async<P1, P1, T, NT>(bR0, Uin + gbase, ne);
        cp_async_commit();
        cp_async_wait_all();
        __syncthreads();
        apply_lines<P1, P1, 1, R, NT>(bR, opD, nlines, [&](int, int base, int k, T v) { bS[base + k * G::RS] = v; });
        apply_lines<P1, P1, 0, R, NT>(bR, opD, nlines, [&](int, int base, int k, T v) { bT[base + k * G::PS] = v; });
        __syncthreads();
        apply_lines<P1, P1, 2, R, NT>(bR, opD, nlines, [&](int, int base, int k, T v) { bR[base + k] = v; });
        __syncthreads();
        const int total = ne * G::NPTS;
        // G[e][c][q]: AXE_PB points per thread per batch, all 6*AXE_PB loads issued before use
        constexpr int PB = AXE_PB;
        for (int f0 = threadIdx.x; f0 < total; f0 += PB * NT) {
            T gv[PB][6];
#pragma unroll
            for (int b = 0; b < PB; ++b) {
                const int f = f0 + b * NT;
                const int fc = f < total ? f : f0;
                const int e = fc / G::NPTS;
                const T* gp = Gm + (e0 + e) * 6 * (int64_t)G::NPTS + (fc - e * G::NPTS);
#pragma unroll
                for (int c = 0; c < 6; ++c) gv[b][c] = __ldcs(gp + c * G::NPTS);
            }
#pragma unroll
            for (int b = 0; b < PB; ++b) {
                const int f = f0 + b * NT;
                if (f < total) {
                    const int si = smem_index<P1, P1, T>(f);
                    const T r = bR[si], s = bS[si], t = bT[si];
                    bR[si] = (gv[b][0] * r + gv[b][1] * s) + gv[b][2] * t;
                    bS[si] = (gv[b][1] * r + gv[b][3] * s) + gv[b][4] * t;
                    bT[si] = (gv[b][2] * r + gv[b][4] * s) + gv[b][5] * t;
                }
            }
        }
        __syncthreads();
        apply_lines<P1, P1, 2, R, NT>(bR, opT, nlines, [&](int, int base, int k, T v) { bR[base + k] = v; });
        __syncthreads();
        apply_lines<P1, P1, 1, R, NT>(bS, opT, nlines, [&](int, int base, int k, T v) {
            bS[base + k * G::RS] = bR[base + k * G::RS] + v;
        });
        __syncthreads();
        apply_lines<P1, P1, 0, R, NT>(bT, opT, nlines, [&](int L, int base, int k, T v) {
            st_cs(Wout + gbase + Line<P1, P1, 0, T>::gofs(L, k), bS[base + k * G::PS] + v);
        });
    }
}

template <int P1>
int launch_ax_e(int64_t N, const double* D, const double* U, const double* Gm, double* W, cudaStream_t s) {
    using CF = Cfg<P1, P1, double, 3, K_AXE>;
    static int occ = 0;
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(ax_e_kernel<P1>, CF::NT, CF::SMEM, ngroups, &occ);
    ax_e_kernel<P1><<<grid, CF::NT, CF::SMEM, s>>>(N, D, U, Gm, W);
    return launch_status();
}

// ---------------------------------------------------------------- P1 dispatch
#define BC_P1_SWITCH(P1VAR, CALL)   \
    switch (P1VAR) {                \
        case 2: return CALL(2);     \
        case 3: return CALL(3);     \
        case 4: return CALL(4);     \
        case 5: return CALL(5);     \
        case 6: return CALL(6);     \
        case 7: return CALL(7);     \
        case 8: return CALL(8);     \
        case 9: return CALL(9);     \
        case 10: return CALL(10);   \
        case 11: return CALL(11);   \
        case 12: return CALL(12);   \
        case 13: return CALL(13);   \
        case 14: return CALL(14);   \
        case 15: return CALL(15);   \
        case 16: return CALL(16);   \
        default: return BC_ERR_UNSUPPORTED; \
    }

int run_sumfact3d(int64_t N, int p, const double* A, const double* B, const double* C, const double* U,
                  double* V, double* ws, cudaStream_t s) {
#define CALL(P) launch_sumfact3d<P, double>(N, A, B, C, U, V, ws, s)
    BC_P1_SWITCH(p + 1, CALL)
#undef CALL
}
int run_sumfact3d_f32(int64_t N, int p, const float* A, const float* B, const float* C, const float* U,
                      float* V, cudaStream_t s) {
#define CALL(P) launch_sumfact3d<P, float>(N, A, B, C, U, V, nullptr, s)
    BC_P1_SWITCH(p + 1, CALL)
#undef CALL
}
int run_sumfact2d(int64_t N, int p, const double* A, const double* B, const double* U, double* V,
                  cudaStream_t s) {
#define CALL(P) launch_sumfact2d<P>(N, A, B, U, V, s)
    BC_P1_SWITCH(p + 1, CALL)
#undef CALL
}
int run_local_grad3(int64_t N, int p, const double* D, const double* U, double* ur, double* us, double* ut,
                    cudaStream_t s) {
#define CALL(P) launch_local_grad3<P>(N, D, U, ur, us, ut, s)
    BC_P1_SWITCH(p + 1, CALL)
#undef CALL
}
int run_local_grad3_t(int64_t N, int p, const double* D, const double* ur, const double* us,
                      const double* ut, double* U, cudaStream_t s) {
#define CALL(P) launch_local_grad3_t<P>(N, D, ur, us, ut, U, s)
    BC_P1_SWITCH(p + 1, CALL)
#undef CALL
}
int run_ax_e(int64_t N, int p, const double* D, const double* U, const double* Gm, double* W, cudaStream_t s) {
#define CALL(P) launch_ax_e<P>(N, D, U, Gm, W, s)
    BC_P1_SWITCH(p + 1, CALL)
#undef CALL
}

}  // namespace bc
