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
//
// For odd P1 (smem layout == HBM layout) and batches of >= 128 elements the production
// kernels are the warp-specialised TMA element rings further down (sumfact_tma_kernel,
// local_grad3_tma_kernel, local_grad3_t_tma_kernel): a loader warp streams items of E
// elements into an NB-slot ring with 1-D bulk copies, consumer groups run the same stages
// (chunk_c) on their slot behind named barriers, and local_grad3's ur leaves through a
// storer warp's bulk stores.
#include <algorithm>
#include <mutex>
#include <type_traits>

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
    // lanes of a ragged chunk read (and discard) the chunk's first line, which lane 0
    // overwrites in place below: order every lane's reads before the writes
    __syncwarp();
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
#ifndef BC_CST_R
#define BC_CST_R 0  // lines per thread of the constant-bank-operator kernels (0: as the smem ones)
#endif
#ifndef BC_CST_R_SF3
#define BC_CST_R_SF3 0  // sumfact3d lines per thread with constant-bank operators (0: table)
#endif
#ifndef BC_CST_NUNROLL
#define BC_CST_NUNROLL 2  // unroll of the constant-operator stages' n loop (measured: 2 >= 1)
#endif
#ifndef BC_CST_PF_SF3
#define BC_CST_PF_SF3 0  // sumfact3d with constant-bank operators: prefetch the next group
#endif
#ifndef BC_CST_PF
#define BC_CST_PF -1  // constant-bank-operator kernels: -1 = prefetch as the smem table, 0/1 = off/on
#endif
#ifndef BC_CST_E
#define BC_CST_E 0  // constant-bank-operator kernels at P1 >= 10: elements per group (0: as the smem table)
#endif
#ifndef BC_CST_REGS
#define BC_CST_REGS 0  // register cap of the constant-bank-operator kernels (0: none)
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
    // lines per thread with constant-bank operators (tools/sweep_spectral.py, DESIGN.md
    // §4.1): 4, except sumfact2d at P1 >= 12 (3) and the 3-field kernels (2)
    static constexpr int RC = BC_CST_R ? BC_CST_R
                                       : ((KIND == K_SF3 && BC_CST_R_SF3) ? BC_CST_R_SF3
                                       : (KIND == K_SF2 && P1 >= 12) ? 3 : (KIND == K_LG3T || KIND == K_AXE ? 2 : 4));
    // unroll of the contracted-index loop: sumfact2d fully (its two stages fit the registers)
    static constexpr int UNROLL = (KIND == K_SF2 && BC_SF2_UNROLL && P1 >= 9) ? P1 : BC_NUNROLL;
};

template <int P1, int NA, typename T, int NBUF_FIELDS, int KIND = K_SF3, bool CST = false>
struct Cfg {
    using G = Geo<P1, NA, T>;
    using TB = SpecTable<P1, KIND>;
    static constexpr bool PREFETCH = ((CST && KIND == K_SF3 && BC_CST_PF_SF3) ? true
                                      : ((CST && BC_CST_PF >= 0) ? (bool)BC_CST_PF : TB::PREFETCH)) &&
                                     NBUF_FIELDS == 1;  // single-field kernels only
    static constexpr int NBUF = NBUF_FIELDS + (PREFETCH ? 1 : 0);
    static constexpr int BUF_BYTES = TB::BUF_KB * 1024;  // target bytes per element-group buffer
    static constexpr int E0 = BUF_BYTES / (G::ES * (int)sizeof(T));
    // even by default; a measured table entry may force E (odd E x odd P1 groups start 8 bytes
    // off a 16-byte boundary, handled by load_group_async)
    // (measured with constant-bank operators: local_grad3 at P1 = 13 with 4-element groups,
    // 0.805 -> 0.822 of HBM; sumfact3d keeps 3)
    static constexpr int E = (CST && BC_CST_E && P1 >= 10) ? BC_CST_E
                           : (CST && KIND == K_LG3 && P1 == 13) ? 4
                           : (TB::EF ? TB::EF : (E0 < 2 ? 1 : (E0 & ~1)));
    static constexpr int R = CST ? TB::RC : TB::R;
    static constexpr int LINES = E * NA * P1;  // lines per axis per group (E * NPTS / P1)
    static constexpr int NT0 = ((LINES + R - 1) / R + 31) / 32 * 32;
    static constexpr int NT = NT0 < 64 ? 64 : (NT0 > 512 ? 512 : NT0);
    static constexpr int VEC = 16 / (int)sizeof(T);
    static constexpr int BUF = (E * G::ES + VEC - 1) / VEC * VEC + VEC;  // + slack for a shifted group
    static constexpr size_t SMEM = (size_t)NBUF * BUF * sizeof(T) + 2 * op_elems<P1, T>() * sizeof(T);
    // CTAs per SM requested from ptxas (__launch_bounds__): with constant-bank operators
    // a register cap makes ptxas re-load operators (LDCU) instead of parking them in
    // registers across the group loop
    static constexpr int MINB = (CST && BC_CST_REGS) ? (65536 / (NT * BC_CST_REGS) > 0 ? 65536 / (NT * BC_CST_REGS) : 1) : 1;
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

// ---------------------------------------------------------------- constant-bank operators
// For batches of at least OPS_CONST_MIN_N elements the (p+1)x(p+1) operators are staged
// into the constant bank (c_ops, row-major M[k][n] = cop[k * P1 + n]) by a stream-ordered
// device-to-device copy ahead of the launch, and the DFMAs read them as uniform-register
// operands: a warp-wide 16-byte broadcast read from shared memory costs the same 4
// wavefronts as a full 512-byte read, so with shared-memory operators the SMEM pipe,
// not the FP64 pipe, bounded these kernels (~1 wavefront per DFMA).
// OPS_SLOTS slots are reused round robin; a call waits (cudaStreamWaitEvent) for the last
// kernel that read its slot, so concurrent calls on different streams stay correct.  The
// slot is a template parameter of the kernels: the operator offsets must be immediates.
// Small batches keep the shared-memory operators (no extra copy latency).
constexpr int OPS_SLOTS = 2, OPS_PER_SLOT = 3, OPS_STRIDE = 256;  // 2 x 3 x 16 x 16 doubles = 12 KiB
#ifndef BC_OPS_CONST_MIN_N
#define BC_OPS_CONST_MIN_N 128
#endif
constexpr int64_t OPS_CONST_MIN_N = BC_OPS_CONST_MIN_N;
__constant__ double c_ops[OPS_SLOTS][OPS_PER_SLOT][OPS_STRIDE];

int op_slot_acquire(cudaStream_t s, const double* const* ops, int nops, int P1, int* slot);  // below
void op_slot_release(cudaStream_t s, int slot);

// One warp chunk (lane owns lines L0 + 32 r, r < RR) of a stage with operator OPI of
// slot CS from the constant bank: y(L, k) = sum_n M[k][n] x(L, n), ascending n (the same
// fma sequence as lines_chunk).  The operator reads are constant-bank loads that ptxas
// turns into LDCUs into uniform registers feeding the DFMAs.  __noinline__: inlined into
// the group loop, ptxas hoisted all P1^2 operator values out of the loop into regular
// registers (255 registers + spills at P1 = 13); as a call, each chunk re-reads them.
// Inside the call n is warp-uniform, so with the n loop rolled (BC_CST_NUNROLL) the reads
// are LDCUs with a uniform-register index (~1 KB of code per stage instead of ~16 KB
// fully unrolled: the unrolled stages missed the instruction cache, 17% of stalls).
// Output modes (k = output index along AXIS, line offset base):
//   OUT_SMEM        dst[base + k*STRIDE] = y           (dst == in: in place; every read of a
//                   line precedes its writes, and a line belongs to one lane)
//   OUT_SMEM_ADD    dst[base + k*STRIDE] = add[base + k*STRIDE] + y
//   OUT_GLOBAL      gdst[gofs(L, k)] = y               (streaming; SQ: returns sum y^2)
//   OUT_GLOBAL_ADD  gdst[gofs(L, k)] = add[base + k*STRIDE] + y
// TRANS: the operator is applied transposed, M[k][n] = cop[n*P1 + k] (local_grad3_t, ax_e).
enum { OUT_SMEM = 0, OUT_GLOBAL = 1, OUT_SMEM_ADD = 2, OUT_GLOBAL_ADD = 3 };
template <int P1, int NA, int AXIS, int RR, int CS, int OPI, int OMODE, bool SQ, bool TRANS, int NUNR = BC_CST_NUNROLL>
__device__ __noinline__ double chunk_c(const double* in, double* dst, const double* add, double* __restrict__ gdst,
                                       int L0, int nlines) {
    using LN = Line<P1, NA, AXIS, double>;
    int base[RR];
#pragma unroll
    for (int r = 0; r < RR; ++r) {
        const int L = L0 + r * 32;
        base[r] = LN::base(L < nlines ? L : (L0 & ~31));
    }
    double acc[P1][RR];
#pragma unroll
    for (int k = 0; k < P1; ++k)
#pragma unroll
        for (int r = 0; r < RR; ++r) acc[k][r] = 0.0;
    // x(L, n+1) is loaded while step n's FMAs run
    double x[RR];
#pragma unroll
    for (int r = 0; r < RR; ++r) x[r] = in[base[r]];
#pragma unroll NUNR
    for (int n = 0; n < P1; ++n) {
        double xn[RR];
        const int nn = n + 1 < P1 ? n + 1 : n;
#pragma unroll
        for (int r = 0; r < RR; ++r) xn[r] = in[base[r] + nn * LN::STRIDE];
#pragma unroll
        for (int k = 0; k < P1; ++k) {
            const double o = TRANS ? c_ops[CS][OPI][n * P1 + k] : c_ops[CS][OPI][k * P1 + n];
#pragma unroll
            for (int r = 0; r < RR; ++r) acc[k][r] = fma(o, x[r], acc[k][r]);
        }
#pragma unroll
        for (int r = 0; r < RR; ++r) x[r] = xn[r];
    }
    __syncwarp();  // dummy reads of ragged lanes (the chunk's first line) precede the in-place writes
    double sq[RR];  // one partial per line: independent chains instead of one serial chain
#pragma unroll
    for (int r = 0; r < RR; ++r) {
        sq[r] = 0.0;
        if (L0 + r * 32 < nlines) {
#pragma unroll
            for (int k = 0; k < P1; ++k) {
                const int so = base[r] + k * LN::STRIDE;
                if constexpr (OMODE == OUT_SMEM) {
                    dst[so] = acc[k][r];
                } else if constexpr (OMODE == OUT_SMEM_ADD) {
                    dst[so] = add[so] + acc[k][r];
                } else {
                    const double v = (OMODE == OUT_GLOBAL_ADD) ? add[so] + acc[k][r] : acc[k][r];
                    st_cs(gdst + LN::gofs(L0 + r * 32, k), v);
                    if constexpr (SQ) sq[r] = fma(v, v, sq[r]);
                }
            }
        }
    }
    double t = 0.0;
#pragma unroll
    for (int r = 0; r < RR; ++r) t += sq[r];
    return t;
}

// apply_lines with operator OPI of constant slot CS (same warp-chunked line assignment as
// apply_lines_w): reads `in`, writes per OMODE; returns this thread's sum of squares of
// its outputs (SQ) or 0.
// apply_lines_gc: the same over NW warps of which this is warp `warp` (a consumer group of
// a warp-specialised kernel); apply_lines_c: all NT threads of the CTA.
template <int P1, int NA, int AXIS, int R, int NW, int CS, int OPI, int OMODE, bool SQ = false, bool TRANS = false,
          int NUNR = BC_CST_NUNROLL>
__device__ __forceinline__ double apply_lines_gc(int warp, const double* in, double* dst, const double* add,
                                                 double* gdst, int nlines) {
    constexpr int CH = 32 * R;
    const int lane = threadIdx.x & 31;
    const int nfull = nlines / CH;
    double sq = 0.0;
    for (int c = warp; c < nfull; c += NW)
        sq += chunk_c<P1, NA, AXIS, R, CS, OPI, OMODE, SQ, TRANS, NUNR>(in, dst, add, gdst, c * CH + lane, nlines);
    const int rest = nlines - nfull * CH;
    if (rest > 0 && warp == nfull % NW) {
        const int L0 = nfull * CH + lane, rr = (rest + 31) >> 5;
        if constexpr (R >= 4) if (rr == 4) return sq + chunk_c<P1, NA, AXIS, 4, CS, OPI, OMODE, SQ, TRANS, NUNR>(in, dst, add, gdst, L0, nlines);
        if constexpr (R >= 3) if (rr == 3) return sq + chunk_c<P1, NA, AXIS, (R >= 3 ? 3 : 1), CS, OPI, OMODE, SQ, TRANS, NUNR>(in, dst, add, gdst, L0, nlines);
        if constexpr (R >= 2) if (rr == 2) return sq + chunk_c<P1, NA, AXIS, (R >= 2 ? 2 : 1), CS, OPI, OMODE, SQ, TRANS, NUNR>(in, dst, add, gdst, L0, nlines);
        sq += chunk_c<P1, NA, AXIS, 1, CS, OPI, OMODE, SQ, TRANS, NUNR>(in, dst, add, gdst, L0, nlines);
    }
    return sq;
}

template <int P1, int NA, int AXIS, int R, int NT, int CS, int OPI, int OMODE, bool SQ = false, bool TRANS = false>
__device__ __forceinline__ double apply_lines_c(const double* in, double* dst, const double* add, double* gdst,
                                                int nlines) {
    return apply_lines_gc<P1, NA, AXIS, R, NT / 32, CS, OPI, OMODE, SQ, TRANS>(threadIdx.x >> 5, in, dst, add, gdst,
                                                                               nlines);
}

// ====================================================================== sumfact3d
//   S1 W1[l][m][k] = sum_n A[k][n] U[l][m][n]     (axis 2, P:440 / Fig. 2(b))
//   S2 W2[l][j][k] = sum_m B[j][m] W1[l][m][k]    (axis 1, P:441 / P:214)
//   S3 V [i][j][k] = sum_l C[i][l] W2[l][j][k]    (axis 0, P:442 / P:215; Fig. 2(d))
// S1 and S2 run in place in the group buffer; S3 stores V straight from registers
// (consecutive threads own consecutive (j,k): coalesced).  With ws != nullptr the check
// scalar sum V^2 (R18) is accumulated in the store epilogue: one partial per
// CTA in ws[8 + blockIdx.x], reduced in fixed order by check_finalize.
template <int P1, typename T, int CS>
__global__ void __launch_bounds__(Cfg<P1, P1, T, 1, K_SF3, (CS >= 0)>::NT, Cfg<P1, P1, T, 1, K_SF3, (CS >= 0)>::MINB)
sumfact3d_kernel(int64_t N, const T* __restrict__ A, const T* __restrict__ B, const T* __restrict__ C,
                 const T* __restrict__ U, T* __restrict__ V, double* __restrict__ ws) {
    constexpr bool CST = CS >= 0;
    using CF = Cfg<P1, P1, T, 1, K_SF3, CST>;
    using G = Geo<P1, P1, T>;
    constexpr int NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opA = reinterpret_cast<T*>(smem_raw);
    T* opB = opA + op_elems<P1, T>();
    T* opC = opB + op_elems<P1, T>();
    T* buf = opC + op_elems<P1, T>();
    if constexpr (!CST) {
        load_op<P1, T, NT>(opA, A);
        load_op<P1, T, NT>(opB, B);
        load_op<P1, T, NT>(opC, C);
    }
    double sq = 0.0;
    group_loop<P1, P1, T, NT, CF::E, CF::BUF, CF::PREFETCH>(N, U, buf, [&](T* in, int64_t e0, int ne) {
        const int nlines = ne * P1 * P1;
        auto s1 = [&](int, int base, int k, T v) { in[base + k] = v; };
        auto s2 = [&](int, int base, int k, T v) { in[base + k * G::RS] = v; };
        T* Vg = V + e0 * G::NPTS;
        auto s3 = [&](int L, int, int k, T v) {
            st_cs(Vg + Line<P1, P1, 0, T>::gofs(L, k), v);
            sq = fma((double)v, (double)v, sq);
        };
        if constexpr (CST) {
            constexpr int C = CST ? CS : 0;
            apply_lines_c<P1, P1, 2, R, NT, C, 0, OUT_SMEM>(in, in, nullptr, nullptr, nlines);
            __syncthreads();
            apply_lines_c<P1, P1, 1, R, NT, C, 1, OUT_SMEM>(in, in, nullptr, nullptr, nlines);
            __syncthreads();
            sq += apply_lines_c<P1, P1, 0, R, NT, C, 2, OUT_GLOBAL, true>(in, nullptr, nullptr, Vg, nlines);
        } else {
            apply_lines<P1, P1, 2, R, NT>(in, opA, nlines, s1);
            __syncthreads();
            apply_lines<P1, P1, 1, R, NT>(in, opB, nlines, s2);
            __syncthreads();
            apply_lines<P1, P1, 0, R, NT>(in, opC, nlines, s3);
        }
    });
    if (ws != nullptr) block_partial(sq, ws + 8);
}

template <int P1, typename T, int CS>
int launch_sumfact3d_k(int64_t N, const T* A, const T* B, const T* C, const T* U, T* V, double* ws, cudaStream_t s) {
    using CF = Cfg<P1, P1, T, 1, K_SF3, (CS >= 0)>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const size_t smem = CF::SMEM + op_elems<P1, T>() * sizeof(T);
    int grid = grid_for(sumfact3d_kernel<P1, T, CS>, CF::NT, smem, ngroups, &occ);
    if (ws && grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
    sumfact3d_kernel<P1, T, CS><<<grid, CF::NT, smem, s>>>(N, A, B, C, U, V, ws);
    const int st = launch_status();
    if (CS >= 0) op_slot_release(s, CS);
    if (st || !ws) return st;
    return run_check_finalize(grid, ws, s);
}

// ------------------------------------------------------------ sumfact3d, TMA element ring
// Warp-specialised persistent form of sumfact3d_kernel for odd P1 (smem layout == global
// layout, no row padding), constant-bank operators.  One CTA per SM:
//   * a loader warp streams items (E consecutive elements, E*P1^3*8 bytes, a multiple of 16
//     for even E) into an NB-slot shared-memory ring with 1-D bulk copies (TMA engine,
//     cp.async.bulk ... mbarrier::complete_tx), full/empty mbarrier pair per slot;
//   * NG consumer groups of NWG warps each take items round robin (item j -> group j % NG)
//     and run S1 -> S2 -> S3 on their slot exactly as sumfact3d_kernel does (S1/S2 in place,
//     S3 stored from registers, coalesced), separated by the group's named barrier, then
//     release the slot (generic->async proxy fence, one arrive per warp).
// The loads of the next NB - NG items are in flight while the groups compute, so no warp
// waits for its element data (the unbuffered kernel's 18% long-scoreboard stall), and a
// group's stage barriers stall only that group.
#ifndef BC_T3_E
#define BC_T3_E 2
#endif
#ifndef BC_T3_NB
#define BC_T3_NB 5
#endif
#ifndef BC_T3_NG
#define BC_T3_NG 3
#endif
#ifndef BC_T3_NWG
#define BC_T3_NWG 4
#endif
#ifndef BC_T3_R
#define BC_T3_R 3
#endif
#ifndef BC_T2_NUNR
#define BC_T2_NUNR BC_CST_NUNROLL  // n-loop unroll of the 2-D ring's stages
#endif
#ifndef BC_T3_NUNR
#define BC_T3_NUNR 4  // n-loop unroll of the 3-D ring's stages (P1 <= 5: full; measured)
#endif
#ifndef BC_T3S_NB
#define BC_T3S_NB 10
#endif
#ifndef BC_T3S_NG
#define BC_T3S_NG 6
#endif
#ifndef BC_T3S_R
#define BC_T3S_R 4
#endif
// Ring geometry: items of E elements of NPTS values, NB slots, NG x NWG consumer warps plus
// XW service warps (loader; storer).
template <int NPTS_, int E_, int NB_, int NG_, int NWG_, int R_, int XW, int NF_ = 1>
struct Ring {
    static constexpr int E = E_, NB = NB_, NG = NG_, NWG = NWG_, R = R_, NPTS = NPTS_, NF = NF_;
    // doubles per field of a slot: an item may start 8 bytes past a 16-byte boundary (odd
    // E x odd NPTS); its copy then starts one value early and may end one value late
    // (16-byte aligned, multiple-of-16 bulk copies), so a field holds E * NPTS + 2 values.
    // A slot holds NF fields (local_grad3_t: ur, us, ut).
    static constexpr int SUB = (E * NPTS + 2 + 1) & ~1;
    static constexpr int SLOT = NF * SUB;
    static constexpr int NT = 32 * (NG * NWG + XW);
    static constexpr size_t SMEM = (size_t)NB * SLOT * 8 + 3 * NB * 8;
    static constexpr bool FITS = SMEM <= 227 * 1024;
    static_assert(NB > NG, "ring_wait_full needs more slots than consumer groups");
};
// 2-D (sumfact2d) ring: items of E2 elements of P1^2 values
#ifndef BC_T2_E
#define BC_T2_E 0  // 0: as many elements as fill the group's 32 NWG R lanes' lines
#endif
#ifndef BC_T2_NB
#define BC_T2_NB 10
#endif
#ifndef BC_T2_NG
#define BC_T2_NG 6
#endif
#ifndef BC_T2_NWG
#define BC_T2_NWG 2
#endif
#ifndef BC_T2_R
#define BC_T2_R 3
#endif
template <int P1, int NA = P1>
using TmaSf3 = typename std::conditional<
    NA == 1, Ring<P1 * P1, (BC_T2_E ? BC_T2_E : 32 * BC_T2_NWG * BC_T2_R / P1), BC_T2_NB, BC_T2_NG, BC_T2_NWG, BC_T2_R, 1>,
    typename std::conditional<
        P1 == 13, Ring<P1 * P1 * P1, BC_T3_E, BC_T3_NB, BC_T3_NG, BC_T3_NWG, BC_T3_R, 1>,
        // other odd P1: items of max(1, 192 / P1^2) elements on 2-warp groups
        Ring<P1 * P1 * P1, (64 * BC_T3S_R / (P1 * P1) > 1 ? 64 * BC_T3S_R / (P1 * P1) : 1), BC_T3S_NB, BC_T3S_NG, 2,
             BC_T3S_R, 1>>::type>::type;

// item j of this CTA: elements [e0, e0 + ne); its first value sits at slot + item_lead
__device__ __forceinline__ int item_lead(const double* p) { return (int)((reinterpret_cast<uintptr_t>(p) >> 3) & 1); }

// Loader (one thread): items j = 0 .. nitems-1 of this CTA into slot j % NB.  Copies
// [src - lead, src - lead + 16 nv) with nv 16-byte units covering the item; where that
// would read past the field's end (the last item only), the final value is copied by a
// plain load/store instead, ordered before the consumers' reads by the release of
// expect_tx.  A slot is refilled after its empty barrier's previous phase completed.
template <class RG, int NL = RG::NF>
__device__ __forceinline__ void ring_loader(int64_t N, const double* __restrict__ U, double* slots, uint32_t full0,
                                            uint32_t empty0, int64_t nitems, const double* __restrict__ U1 = nullptr,
                                            const double* __restrict__ U2 = nullptr) {
    const double* F[3] = {U, U1, U2};
    for (int64_t j = 0; j < nitems; ++j) {
        const int b = (int)(j % RG::NB);
        const int64_t use = j / RG::NB;
        if (use > 0) mbar_wait(empty0 + 8 * b, (int)((use - 1) & 1));
        const int64_t e0 = (blockIdx.x + j * gridDim.x) * RG::E;
        const int ne = (int)imin64(RG::E, N - e0);
        int nv[NL], bytes = 0;
#pragma unroll
        for (int f = 0; f < NL; ++f) {
            const double* src = F[f] + e0 * RG::NPTS;
            const int lead = item_lead(src);
            const int tot = lead + ne * RG::NPTS;
            nv[f] = (tot + 1) >> 1;
            if ((tot & 1) && e0 + ne == N) {
                nv[f] = tot >> 1;
                slots[(size_t)b * RG::SLOT + f * RG::SUB + tot - 1] = src[tot - 1 - lead];
            }
            bytes += nv[f] * 16;
        }
        mbar_expect_tx(full0 + 8 * b, bytes);
#pragma unroll
        for (int f = 0; f < NL; ++f) {
            const double* src = F[f] + e0 * RG::NPTS;
            bulk_load(smem_u32(slots + (size_t)b * RG::SLOT + f * RG::SUB), src - item_lead(src),
                      (uint32_t)nv[f] * 16u, full0 + 8 * b);
        }
    }
}

// Consumer wait for item j (slot b = j % NB, use u = j / NB).  A parity wait is exact only
// while the barrier is at most one phase behind the awaited one, and with NG groups sharing
// the ring a group can reach use u of a slot whose use u-1 (another group's item, its bulk
// copy still in flight: copies complete out of order) has not completed yet -- the parity
// of phase u would then read as complete and the group would compute on the previous
// item's bytes.  So for u >= 1 the consumer first waits for the release of use u-1 (empty
// phase u-1, which implies full phase u-1 completed), then for full phase u.  The empty
// wait itself cannot alias: this group consumed item j - NG > j - NB, so the loader had
// passed its wait for empty phase u-2.  (Found as intermittent 'unspecified launch failure'
// at large N: the mis-synchronised group's release over-arrived the empty barrier and the
// ring's transaction accounting broke.)
template <int NB>
__device__ __forceinline__ void ring_wait_full(uint32_t full0, uint32_t empty0, int b, int64_t j) {
    const int64_t use = j / NB;
    if (use > 0) mbar_wait(empty0 + 8 * b, (int)((use - 1) & 1));
    mbar_wait(full0 + 8 * b, (int)(use & 1));
}

// NA = P1: sumfact3d (S1, S2 in place, S3 to V);  NA = 1: sumfact2d (W in place, V = B W).
template <int P1, int NA, int CS>
__global__ void __launch_bounds__(TmaSf3<P1, NA>::NT, 1)
sumfact_tma_kernel(int64_t N, const double* __restrict__ U, double* __restrict__ V, double* __restrict__ ws) {
    using TC = TmaSf3<P1, NA>;
    constexpr int E = TC::E, NB = TC::NB, NG = TC::NG, NWG = TC::NWG, NPTS = TC::NPTS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    double* slots = reinterpret_cast<double*>(smem_raw);
    const uint32_t full0 = smem_u32(smem_raw + (size_t)NB * TC::SLOT * 8), empty0 = full0 + 8 * NB;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(full0 + 8 * b, 1);
            mbar_init(empty0 + 8 * b, NWG);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t ngroups = (N + E - 1) / E;
    const int64_t nitems = ngroups > blockIdx.x ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    double sq = 0.0;
    if (warp == NG * NWG) {
        if (lane == 0) ring_loader<TC>(N, U, slots, full0, empty0, nitems);
    } else {
        constexpr int C = CS;
        const int grp = warp / NWG, wg = warp - grp * NWG;
        for (int64_t j = grp; j < nitems; j += NG) {
            const int b = (int)(j % NB);
            ring_wait_full<NB>(full0, empty0, b, j);
            const int64_t e0 = (blockIdx.x + j * gridDim.x) * E;
            const int nlines = (int)imin64(E, N - e0) * NA * P1;
            double* in = slots + (size_t)b * TC::SLOT + item_lead(U + e0 * NPTS);
            constexpr int U = NA == 1 ? BC_T2_NUNR : (P1 <= 5 ? P1 : BC_T3_NUNR);
            apply_lines_gc<P1, NA, 2, TC::R, NWG, C, 0, OUT_SMEM, false, false, U>(wg, in, in, nullptr, nullptr, nlines);
            named_bar_sync(1 + grp, NWG * 32);
            if constexpr (NA == 1) {
                apply_lines_gc<P1, 1, 1, TC::R, NWG, C, 1, OUT_GLOBAL, false, false, U>(wg, in, nullptr, nullptr,
                                                                                       V + e0 * NPTS, nlines);
            } else {
                apply_lines_gc<P1, P1, 1, TC::R, NWG, C, 1, OUT_SMEM, false, false, U>(wg, in, in, nullptr, nullptr,
                                                                                      nlines);
                named_bar_sync(1 + grp, NWG * 32);
                sq += apply_lines_gc<P1, P1, 0, TC::R, NWG, C, 2, OUT_GLOBAL, true, false, U>(wg, in, nullptr, nullptr,
                                                                                             V + e0 * NPTS, nlines);
            }
            release_slot(empty0 + 8 * b, lane);
        }
    }
    if (NA != 1 && ws != nullptr) block_partial(sq, ws + 8);
}

// Odd P1 >= BC_T3_MIN_P1 with constant-bank operators and 16-byte aligned U: the TMA ring
// kernel (measured: DESIGN.md §4.1); BC_SF3_TMA=0 in the environment selects the
// unbuffered kernel for A/B measurements (read once).
#ifndef BC_T3_MIN_P1
#define BC_T3_MIN_P1 5
#endif
#ifndef BC_T2_MIN_P1
#define BC_T2_MIN_P1 5
#endif
static bool sf2_tma_enabled() {
    static const bool on = [] {
        const char* v = getenv("BC_SF2_TMA");
        return !(v && v[0] == '0');
    }();
    return on;
}
static bool sf3_tma_enabled() {
    static const bool on = [] {
        const char* v = getenv("BC_SF3_TMA");
        return !(v && v[0] == '0');
    }();
    return on;
}

template <int P1, int NA, int CS>
int launch_sumfact_tma(int64_t N, const double* U, double* V, double* ws, cudaStream_t s) {
    using TC = TmaSf3<P1, NA>;
    static PerDevice<int> attr_dev;
    int& attr = attr_dev.get();
    if (!attr) {
        cudaFuncSetAttribute(sumfact_tma_kernel<P1, NA, CS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)TC::SMEM);
        attr = 1;
    }
    const int64_t ngroups = (N + TC::E - 1) / TC::E;
    int grid = (int)imin64(ngroups, num_sms());
    if (ws && grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
    sumfact_tma_kernel<P1, NA, CS><<<grid, TC::NT, TC::SMEM, s>>>(N, U, V, ws);
    const int st = launch_status();
    op_slot_release(s, CS);
    if (st || !ws) return st;
    return run_check_finalize(grid, ws, s);
}

template <int P1, typename T>
int launch_sumfact3d(int64_t N, const T* A, const T* B, const T* C, const T* U, T* V, double* ws, cudaStream_t s) {
    if constexpr (sizeof(T) == 8) {
        if (N >= OPS_CONST_MIN_N) {
            const double* ops[3] = {A, B, C};
            int slot, st;
            if ((st = op_slot_acquire(s, ops, 3, P1, &slot))) return st;
            if constexpr (P1 % 2 == 1 && TmaSf3<P1>::FITS && P1 >= BC_T3_MIN_P1) {
                if (sf3_tma_enabled() && (reinterpret_cast<uintptr_t>(U) & 15) == 0)
                    return slot == 0 ? launch_sumfact_tma<P1, P1, 0>(N, U, V, ws, s)
                                     : launch_sumfact_tma<P1, P1, 1>(N, U, V, ws, s);
            }
            return slot == 0 ? launch_sumfact3d_k<P1, T, 0>(N, A, B, C, U, V, ws, s)
                             : launch_sumfact3d_k<P1, T, 1>(N, A, B, C, U, V, ws, s);
        }
    }
    return launch_sumfact3d_k<P1, T, -1>(N, A, B, C, U, V, ws, s);
}

// ====================================================================== sumfact2d
//   W[l][j] = sum_m A[j][m] U[l][m]  (rows, in place);  V[i][j] = sum_l B[i][l] W[l][j]
template <int P1, int CS>
__global__ void __launch_bounds__(Cfg<P1, 1, double, 1, K_SF2, (CS >= 0)>::NT, Cfg<P1, 1, double, 1, K_SF2, (CS >= 0)>::MINB)
sumfact2d_kernel(int64_t N, const double* __restrict__ A, const double* __restrict__ B,
                 const double* __restrict__ U, double* __restrict__ V) {
    using T = double;
    constexpr bool CST = CS >= 0;
    using CF = Cfg<P1, 1, T, 1, K_SF2, CST>;
    using G = Geo<P1, 1, T>;
    constexpr int NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opA = reinterpret_cast<T*>(smem_raw);
    T* opB = opA + op_elems<P1, T>();
    T* buf = opB + op_elems<P1, T>();
    if constexpr (!CST) {
        load_op<P1, T, NT>(opA, A);
        load_op<P1, T, NT>(opB, B);
    }
    group_loop<P1, 1, T, NT, CF::E, CF::BUF, CF::PREFETCH>(N, U, buf, [&](T* in, int64_t e0, int ne) {
        const int nlines = ne * P1;
        constexpr int U = CF::TB::UNROLL;
        auto st1 = [&](int, int base, int k, T v) { in[base + k] = v; };
        T* Vg = V + e0 * G::NPTS;
        auto st2 = [&](int L, int, int k, T v) { st_cs(Vg + Line<P1, 1, 1, T>::gofs(L, k), v); };
        if constexpr (CST) {
            constexpr int C = CST ? CS : 0;
            apply_lines_c<P1, 1, 2, R, NT, C, 0, OUT_SMEM>(in, in, nullptr, nullptr, nlines);
            __syncthreads();
            apply_lines_c<P1, 1, 1, R, NT, C, 1, OUT_GLOBAL>(in, nullptr, nullptr, Vg, nlines);
        } else {
            apply_lines<P1, 1, 2, R, NT, T, decltype(st1), U>(in, opA, nlines, st1);
            __syncthreads();
            apply_lines<P1, 1, 1, R, NT, T, decltype(st2), U>(in, opB, nlines, st2);
        }
    });
}

template <int P1, int CS>
int launch_sumfact2d_k(int64_t N, const double* A, const double* B, const double* U, double* V, cudaStream_t s) {
    using CF = Cfg<P1, 1, double, 1, K_SF2, (CS >= 0)>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(sumfact2d_kernel<P1, CS>, CF::NT, CF::SMEM, ngroups, &occ);
    sumfact2d_kernel<P1, CS><<<grid, CF::NT, CF::SMEM, s>>>(N, A, B, U, V);
    const int st = launch_status();
    if (CS >= 0) op_slot_release(s, CS);
    return st;
}

template <int P1>
int launch_sumfact2d(int64_t N, const double* A, const double* B, const double* U, double* V, cudaStream_t s) {
    if (N >= OPS_CONST_MIN_N) {
        const double* ops[2] = {A, B};
        int slot, st;
        if ((st = op_slot_acquire(s, ops, 2, P1, &slot))) return st;
        if constexpr (P1 % 2 == 1 && TmaSf3<P1, 1>::FITS && P1 >= BC_T2_MIN_P1) {
            if (sf2_tma_enabled() && (reinterpret_cast<uintptr_t>(U) & 15) == 0)
                return slot == 0 ? launch_sumfact_tma<P1, 1, 0>(N, U, V, nullptr, s)
                                 : launch_sumfact_tma<P1, 1, 1>(N, U, V, nullptr, s);
        }
        return slot == 0 ? launch_sumfact2d_k<P1, 0>(N, A, B, U, V, s) : launch_sumfact2d_k<P1, 1>(N, A, B, U, V, s);
    }
    return launch_sumfact2d_k<P1, -1>(N, A, B, U, V, s);
}

// ====================================================================== local_grad3
//   ur = D along axis 2 (i), us = D along axis 1 (j), ut = D along axis 0 (k) of U[k][j][i]
// us and ut are stored from registers (coalesced); ur is formed in place (its rows are
// strided across threads) and copied out coalesced.
template <int P1, int CS>
__global__ void __launch_bounds__(Cfg<P1, P1, double, 1, K_LG3, (CS >= 0)>::NT, Cfg<P1, P1, double, 1, K_LG3, (CS >= 0)>::MINB)
local_grad3_kernel(int64_t N, const double* __restrict__ D, const double* __restrict__ U,
                   double* __restrict__ ur, double* __restrict__ us, double* __restrict__ ut) {
    using T = double;
    constexpr bool CST = CS >= 0;
    using CF = Cfg<P1, P1, T, 1, K_LG3, CST>;
    using G = Geo<P1, P1, T>;
    constexpr int NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opD = reinterpret_cast<T*>(smem_raw);
    T* buf = opD + 2 * op_elems<P1, T>();
    if constexpr (!CST) load_op<P1, T, NT>(opD, D);
    // one stage: the operator along AXIS of the group's lines, from smem or the constant bank
    group_loop<P1, P1, T, NT, CF::E, CF::BUF, CF::PREFETCH>(N, U, buf, [&](T* in, int64_t e0, int ne) {
        const int nlines = ne * P1 * P1;
        const int64_t gbase = e0 * G::NPTS;
        if constexpr (CST) {
            constexpr int C = CST ? CS : 0;
            apply_lines_c<P1, P1, 1, R, NT, C, 0, OUT_GLOBAL>(in, nullptr, nullptr, us + gbase, nlines);
            apply_lines_c<P1, P1, 0, R, NT, C, 0, OUT_GLOBAL>(in, nullptr, nullptr, ut + gbase, nlines);
            __syncthreads();
            apply_lines_c<P1, P1, 2, R, NT, C, 0, OUT_SMEM>(in, in, nullptr, nullptr, nlines);
        } else {
            apply_lines<P1, P1, 1, R, NT>(in, opD, nlines, [&](int L, int, int k, T v) {
                st_cs(us + gbase + Line<P1, P1, 1, T>::gofs(L, k), v);
            });
            apply_lines<P1, P1, 0, R, NT>(in, opD, nlines, [&](int L, int, int k, T v) {
                st_cs(ut + gbase + Line<P1, P1, 0, T>::gofs(L, k), v);
            });
            __syncthreads();
            apply_lines<P1, P1, 2, R, NT>(in, opD, nlines, [&](int, int base, int k, T v) { in[base + k] = v; });
        }
        __syncthreads();
        const int total = ne * G::NPTS;
        for (int f = threadIdx.x; f < total; f += NT) st_cs(ur + gbase + f, in[smem_index<P1, P1, T>(f)]);
    });
}

// ------------------------------------------------------------ local_grad3, TMA element ring
// Warp-specialised persistent form of local_grad3_kernel (odd P1, constant-bank D), the
// same ring as sumfact_tma_kernel plus a storer warp:
//   consumers (group of NWG warps per item): us and ut stored from registers (coalesced),
//     group barrier, ur formed in place in the slot, generic->async proxy fence, one
//     `done` arrive per warp;
//   storer (one thread): per item in order, waits `done`, writes ur with a 1-D bulk copy
//     shared -> global (the values outside its 16-byte aligned interior by plain stores),
//     and releases the previous item's slot once that copy has finished reading it.
// The loader and the storer run asynchronously to the consumers, so the consumers neither
// wait for element data nor issue the ur copy-out (the unbuffered kernel's 24%
// long-scoreboard and 19% barrier stalls).
#ifndef BC_L3_E
#define BC_L3_E 0  // 0: max(1, elements whose lines fill the group's 32 NWG R lanes)
#endif
#ifndef BC_L3_NB
#define BC_L3_NB 10
#endif
#ifndef BC_L3_NG
#define BC_L3_NG 5
#endif
#ifndef BC_L3_NWG
#define BC_L3_NWG 2
#endif
#ifndef BC_L3_R
#define BC_L3_R 3
#endif
#ifndef BC_L3_NUNR
#define BC_L3_NUNR 1
#endif
#ifndef BC_L3_POLL
#define BC_L3_POLL 1  // storer polls the slots (out-of-order items) instead of waiting in item order
#endif
template <int P1>
using TmaLg3 = Ring<P1 * P1 * P1,
                    (BC_L3_E ? BC_L3_E : (32 * BC_L3_NWG * BC_L3_R / (P1 * P1) > 1 ? 32 * BC_L3_NWG * BC_L3_R / (P1 * P1) : 1)),
                    BC_L3_NB, BC_L3_NG, BC_L3_NWG, BC_L3_R, 2>;

template <int P1, int CS>
__global__ void __launch_bounds__(TmaLg3<P1>::NT, 1)
local_grad3_tma_kernel(int64_t N, const double* __restrict__ U, double* __restrict__ ur, double* __restrict__ us,
                       double* __restrict__ ut) {
    using TC = TmaLg3<P1>;
    constexpr int E = TC::E, NB = TC::NB, NG = TC::NG, NWG = TC::NWG, NPTS = TC::NPTS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    double* slots = reinterpret_cast<double*>(smem_raw);
    const uint32_t full0 = smem_u32(smem_raw + (size_t)NB * TC::SLOT * 8), empty0 = full0 + 8 * NB,
                   done0 = empty0 + 8 * NB;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(full0 + 8 * b, 1);
            mbar_init(empty0 + 8 * b, 1);
            mbar_init(done0 + 8 * b, NWG);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t ngroups = (N + E - 1) / E;
    const int64_t nitems = ngroups > blockIdx.x ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    if (warp == NG * NWG) {
        if (lane == 0) ring_loader<TC>(N, U, slots, full0, empty0, nitems);
    } else if (warp == NG * NWG + 1) {
        if (lane == 0) {
            // store item j (slot b) once its `done` phase completed, then release the slot as
            // soon as the bulk copy has read it
            auto store_item = [&](int64_t j, int b) {
                const int64_t e0 = (blockIdx.x + j * gridDim.x) * E;
                const int n = (int)imin64(E, N - e0) * NPTS;
                const int h = item_lead(U + e0 * NPTS);  // == item_lead(ur + e0 * NPTS)
                const double* in = slots + (size_t)b * TC::SLOT + h;
                double* dst = ur + e0 * NPTS;
                const int m = (n - h) & ~1;  // values in the 16-byte aligned interior [h, h + m)
                if (h) dst[0] = in[0];
                if (h + m < n) dst[n - 1] = in[n - 1];
                if (m) bulk_store(dst + h, smem_u32(in + h), (uint32_t)m * 8u);
                bulk_commit();
                bulk_wait_read<0>();
                fence_proxy_async();
                mbar_arrive(empty0 + 8 * b);
            };
            if constexpr (BC_L3_POLL) {
                // slots are polled round robin (non-blocking test_wait), so an item finished
                // by a fast group is stored and its slot released without waiting for an
                // earlier item of a slower group (slot b holds items b, b + NB, ... in order,
                // and its `done` barrier cannot run a phase ahead: the next phase needs this
                // release)
                int use[NB];
#pragma unroll
                for (int b = 0; b < NB; ++b) use[b] = 0;
                int64_t left = nitems;
                while (left > 0) {
#pragma unroll
                    for (int b = 0; b < NB; ++b) {
                        const int64_t j = b + (int64_t)NB * use[b];
                        if (j < nitems && mbar_test(done0 + 8 * b, use[b] & 1)) {
                            store_item(j, b);
                            ++use[b];
                            --left;
                        }
                    }
                }
            } else {
                for (int64_t j = 0; j < nitems; ++j) {
                    const int b = (int)(j % NB);
                    mbar_wait(done0 + 8 * b, (int)((j / NB) & 1));
                    store_item(j, b);
                }
            }
            bulk_wait<0>();
        }
    } else {
        constexpr int C = CS;
        const int grp = warp / NWG, wg = warp - grp * NWG;
        for (int64_t j = grp; j < nitems; j += NG) {
            const int b = (int)(j % NB);
            ring_wait_full<NB>(full0, empty0, b, j);
            const int64_t e0 = (blockIdx.x + j * gridDim.x) * E, gbase = e0 * NPTS;
            const int nlines = (int)imin64(E, N - e0) * P1 * P1;
            double* in = slots + (size_t)b * TC::SLOT + item_lead(U + gbase);
            constexpr int U = BC_L3_NUNR;
            apply_lines_gc<P1, P1, 1, TC::R, NWG, C, 0, OUT_GLOBAL, false, false, U>(wg, in, nullptr, nullptr,
                                                                                   us + gbase, nlines);
            apply_lines_gc<P1, P1, 0, TC::R, NWG, C, 0, OUT_GLOBAL, false, false, U>(wg, in, nullptr, nullptr,
                                                                                   ut + gbase, nlines);
            named_bar_sync(1 + grp, NWG * 32);  // every read of the item precedes ur's in-place writes
            apply_lines_gc<P1, P1, 2, TC::R, NWG, C, 0, OUT_SMEM, false, false, U>(wg, in, in, nullptr, nullptr, nlines);
            fence_proxy_async();  // ur (generic writes) is read next by the storer's bulk copy
            __syncwarp();
            if (lane == 0) mbar_arrive(done0 + 8 * b);
        }
    }
}

#ifndef BC_L3_MIN_P1
#define BC_L3_MIN_P1 5
#endif
static bool lg3_tma_enabled() {
    static const bool on = [] {
        const char* v = getenv("BC_LG3_TMA");
        return !(v && v[0] == '0');
    }();
    return on;
}

template <int P1, int CS>
int launch_local_grad3_tma(int64_t N, const double* U, double* ur, double* us, double* ut, cudaStream_t s) {
    using TC = TmaLg3<P1>;
    static PerDevice<int> attr_dev;
    int& attr = attr_dev.get();
    if (!attr) {
        cudaFuncSetAttribute(local_grad3_tma_kernel<P1, CS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)TC::SMEM);
        attr = 1;
    }
    const int grid = (int)imin64((N + TC::E - 1) / TC::E, num_sms());
    local_grad3_tma_kernel<P1, CS><<<grid, TC::NT, TC::SMEM, s>>>(N, U, ur, us, ut);
    const int st = launch_status();
    op_slot_release(s, CS);
    return st;
}

template <int P1, int CS>
int launch_local_grad3_k(int64_t N, const double* D, const double* U, double* ur, double* us, double* ut,
                         cudaStream_t s) {
    using CF = Cfg<P1, P1, double, 1, K_LG3, (CS >= 0)>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(local_grad3_kernel<P1, CS>, CF::NT, CF::SMEM, ngroups, &occ);
    local_grad3_kernel<P1, CS><<<grid, CF::NT, CF::SMEM, s>>>(N, D, U, ur, us, ut);
    const int st = launch_status();
    if (CS >= 0) op_slot_release(s, CS);
    return st;
}

template <int P1>
int launch_local_grad3(int64_t N, const double* D, const double* U, double* ur, double* us, double* ut,
                       cudaStream_t s) {
    if (N >= OPS_CONST_MIN_N) {
        int slot, st;
        if ((st = op_slot_acquire(s, &D, 1, P1, &slot))) return st;
        // odd P1 (unpadded smem layout) except 11, where a one-element item's 121 lines fill
        // 121 of a group's 192 lanes (measured: ring 0.74 vs unbuffered 0.86 of HBM)
        if constexpr (P1 % 2 == 1 && TmaLg3<P1>::FITS && P1 >= BC_L3_MIN_P1 && P1 != 11) {
            if (lg3_tma_enabled() && ((reinterpret_cast<uintptr_t>(U) | reinterpret_cast<uintptr_t>(ur)) & 15) == 0)
                return slot == 0 ? launch_local_grad3_tma<P1, 0>(N, U, ur, us, ut, s)
                                 : launch_local_grad3_tma<P1, 1>(N, U, ur, us, ut, s);
        }
        return slot == 0 ? launch_local_grad3_k<P1, 0>(N, D, U, ur, us, ut, s)
                         : launch_local_grad3_k<P1, 1>(N, D, U, ur, us, ut, s);
    }
    return launch_local_grad3_k<P1, -1>(N, D, U, ur, us, ut, s);
}

// ====================================================================== local_grad3_t
//   U = D^T along axis 2 of ur + D^T along axis 1 of us + D^T along axis 0 of ut,
//   partial sums added in the order (r + s) + t.  Three field buffers, all in place.
template <int P1, int CS>
__global__ void __launch_bounds__(Cfg<P1, P1, double, 3, K_LG3T, (CS >= 0)>::NT)
local_grad3_t_kernel(int64_t N, const double* __restrict__ D, const double* __restrict__ ur,
                     const double* __restrict__ us, const double* __restrict__ ut, double* __restrict__ U) {
    using T = double;
    constexpr bool CST = CS >= 0;
    constexpr int C = CST ? CS : 0;
    using CF = Cfg<P1, P1, T, 3, K_LG3T, CST>;
    using G = Geo<P1, P1, T>;
    constexpr int E = CF::E, NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opT = reinterpret_cast<T*>(smem_raw);
    T* bR0 = opT + 2 * op_elems<P1, T>();
    T* bS0 = bR0 + CF::BUF;
    T* bT0 = bS0 + CF::BUF;
    if constexpr (!CST) load_op<P1, T, NT, true>(opT, D);
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
        if constexpr (CST)
            apply_lines_c<P1, P1, 2, R, NT, C, 0, OUT_SMEM, false, true>(bR, bR, nullptr, nullptr, nlines);
        else
            apply_lines<P1, P1, 2, R, NT>(bR, opT, nlines, [&](int, int base, int k, T v) { bR[base + k] = v; });
        cp_async_wait_n<1>();
        __syncthreads();
        if constexpr (CST)
            apply_lines_c<P1, P1, 1, R, NT, C, 0, OUT_SMEM_ADD, false, true>(bS, bS, bR, nullptr, nlines);
        else
            apply_lines<P1, P1, 1, R, NT>(bS, opT, nlines, [&](int, int base, int k, T v) {
                bS[base + k * G::RS] = bR[base + k * G::RS] + v;
            });
        cp_async_wait_n<0>();
        __syncthreads();
        if constexpr (CST)
            apply_lines_c<P1, P1, 0, R, NT, C, 0, OUT_GLOBAL_ADD, false, true>(bT, nullptr, bS, U + gbase, nlines);
        else
            apply_lines<P1, P1, 0, R, NT>(bT, opT, nlines, [&](int L, int base, int k, T v) {
                st_cs(U + gbase + Line<P1, P1, 0, T>::gofs(L, k), bS[base + k * G::PS] + v);
            });
    }
}

// ------------------------------------------------------------ local_grad3_t, TMA element ring
// The ring of local_grad3 with three input fields per item (ur, us, ut in one slot, one
// full barrier for the three bulk copies): r stage in place on ur, group barrier, s stage
// into us adding ur, group barrier, t stage to U (global, coalesced) adding us; the same
// (r + s) + t order as local_grad3_t_kernel.  Items of one element (3 x 17.6 KB at P1 = 13).
#ifndef BC_LT_NB
#define BC_LT_NB 4
#endif
#ifndef BC_LT_NG
#define BC_LT_NG 3
#endif
#ifndef BC_LT_NWG
#define BC_LT_NWG 3
#endif
#ifndef BC_LT_R
#define BC_LT_R 3
#endif
#ifndef BC_LT_NUNR
#define BC_LT_NUNR BC_CST_NUNROLL  // n-loop unroll of the local_grad3_t ring's stages
#endif
#ifndef BC_LT13_NUNR
#define BC_LT13_NUNR 4  // ... at P1 = 13 (measured: 0.82-0.84 -> 0.85-0.86 of HBM; 4 is worse at p=4/8)
#endif
#ifndef BC_LT13_R
#define BC_LT13_R 2  // P1 = 13: 169 lines on 3 warps x 64 lanes (R = 3 leaves one warp idle)
#endif
template <int P1, int LR = (P1 == 13 ? BC_LT13_R : BC_LT_R)>
using TmaLgT = Ring<P1 * P1 * P1,
                    (32 * BC_LT_NWG * LR / (P1 * P1) > 1 ? 32 * BC_LT_NWG * LR / (P1 * P1) : 1),
                    BC_LT_NB, BC_LT_NG, BC_LT_NWG, LR, 1, 3>;

template <int P1, int CS>
__global__ void __launch_bounds__(TmaLgT<P1>::NT, 1)
local_grad3_t_tma_kernel(int64_t N, const double* __restrict__ ur, const double* __restrict__ us,
                         const double* __restrict__ ut, double* __restrict__ U) {
    using TC = TmaLgT<P1>;
    constexpr int E = TC::E, NB = TC::NB, NG = TC::NG, NWG = TC::NWG, NPTS = TC::NPTS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    double* slots = reinterpret_cast<double*>(smem_raw);
    const uint32_t full0 = smem_u32(smem_raw + (size_t)NB * TC::SLOT * 8), empty0 = full0 + 8 * NB;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(full0 + 8 * b, 1);
            mbar_init(empty0 + 8 * b, NWG);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t ngroups = (N + E - 1) / E;
    const int64_t nitems = ngroups > blockIdx.x ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    if (warp == NG * NWG) {
        if (lane == 0) ring_loader<TC>(N, ur, slots, full0, empty0, nitems, us, ut);
    } else {
        constexpr int C = CS;
        const int grp = warp / NWG, wg = warp - grp * NWG;
        for (int64_t j = grp; j < nitems; j += NG) {
            const int b = (int)(j % NB);
            ring_wait_full<NB>(full0, empty0, b, j);
            const int64_t e0 = (blockIdx.x + j * gridDim.x) * E, gbase = e0 * NPTS;
            const int nlines = (int)imin64(E, N - e0) * P1 * P1;
            double* slot = slots + (size_t)b * TC::SLOT;
            double* bR = slot + item_lead(ur + gbase);
            double* bS = slot + TC::SUB + item_lead(us + gbase);
            double* bT = slot + 2 * TC::SUB + item_lead(ut + gbase);
            constexpr int UN = P1 == 13 ? BC_LT13_NUNR : BC_LT_NUNR;
            apply_lines_gc<P1, P1, 2, TC::R, NWG, C, 0, OUT_SMEM, false, true, UN>(wg, bR, bR, nullptr, nullptr, nlines);
            named_bar_sync(1 + grp, NWG * 32);
            apply_lines_gc<P1, P1, 1, TC::R, NWG, C, 0, OUT_SMEM_ADD, false, true, UN>(wg, bS, bS, bR, nullptr, nlines);
            named_bar_sync(1 + grp, NWG * 32);
            apply_lines_gc<P1, P1, 0, TC::R, NWG, C, 0, OUT_GLOBAL_ADD, false, true, UN>(wg, bT, nullptr, bS, U + gbase,
                                                                                         nlines);
            release_slot(empty0 + 8 * b, lane);
        }
    }
}

#ifndef BC_LT_MIN_P1
#define BC_LT_MIN_P1 5
#endif
static bool lg3t_tma_enabled() {
    static const bool on = [] {
        const char* v = getenv("BC_LG3T_TMA");
        return !(v && v[0] == '0');
    }();
    return on;
}

template <int P1, int CS>
int launch_local_grad3_t_tma(int64_t N, const double* ur, const double* us, const double* ut, double* U,
                             cudaStream_t s) {
    using TC = TmaLgT<P1>;
    static PerDevice<int> attr_dev;
    int& attr = attr_dev.get();
    if (!attr) {
        cudaFuncSetAttribute(local_grad3_t_tma_kernel<P1, CS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)TC::SMEM);
        attr = 1;
    }
    const int grid = (int)imin64((N + TC::E - 1) / TC::E, num_sms());
    local_grad3_t_tma_kernel<P1, CS><<<grid, TC::NT, TC::SMEM, s>>>(N, ur, us, ut, U);
    const int st = launch_status();
    op_slot_release(s, CS);
    return st;
}

template <int P1, int CS>
int launch_local_grad3_t_k(int64_t N, const double* D, const double* ur, const double* us, const double* ut,
                           double* U, cudaStream_t s) {
    using CF = Cfg<P1, P1, double, 3, K_LG3T, (CS >= 0)>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(local_grad3_t_kernel<P1, CS>, CF::NT, CF::SMEM, ngroups, &occ);
    local_grad3_t_kernel<P1, CS><<<grid, CF::NT, CF::SMEM, s>>>(N, D, ur, us, ut, U);
    const int st = launch_status();
    if (CS >= 0) op_slot_release(s, CS);
    return st;
}

template <int P1>
int launch_local_grad3_t(int64_t N, const double* D, const double* ur, const double* us, const double* ut,
                         double* U, cudaStream_t s) {
    if (N >= OPS_CONST_MIN_N) {
        int slot, st;
        if ((st = op_slot_acquire(s, &D, 1, P1, &slot))) return st;
        if constexpr (P1 % 2 == 1 && TmaLgT<P1>::FITS && P1 >= BC_LT_MIN_P1) {
            if (lg3t_tma_enabled() &&
                ((reinterpret_cast<uintptr_t>(ur) | reinterpret_cast<uintptr_t>(us) | reinterpret_cast<uintptr_t>(ut)) &
                 15) == 0)
                return slot == 0 ? launch_local_grad3_t_tma<P1, 0>(N, ur, us, ut, U, s)
                                 : launch_local_grad3_t_tma<P1, 1>(N, ur, us, ut, U, s);
        }
        return slot == 0 ? launch_local_grad3_t_k<P1, 0>(N, D, ur, us, ut, U, s)
                         : launch_local_grad3_t_k<P1, 1>(N, D, ur, us, ut, U, s);
    }
    return launch_local_grad3_t_k<P1, -1>(N, D, ur, us, ut, U, s);
}

// ====================================================================== ax_e
// (us, ut) from U into two buffers; ur in place over U; per-point geometric mixing in
// place; then local_grad3_t in place as above.  Three field buffers.
template <int P1, int CS>
__global__ void __launch_bounds__(Cfg<P1, P1, double, 3, K_AXE, (CS >= 0)>::NT)
ax_e_kernel(int64_t N, const double* __restrict__ D, const double* __restrict__ Uin,
            const double* __restrict__ Gm, double* __restrict__ Wout) {
    using T = double;
    constexpr bool CST = CS >= 0;
    constexpr int C = CST ? CS : 0;
    using CF = Cfg<P1, P1, T, 3, K_AXE, CST>;
    using G = Geo<P1, P1, T>;
    constexpr int E = CF::E, NT = CF::NT, R = CF::R;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* opD = reinterpret_cast<T*>(smem_raw);
    T* opT = opD + op_elems<P1, T>();
    T* bR0 = opT + op_elems<P1, T>();  // holds U, then ur / wr
    T* bS = bR0 + CF::BUF;
    T* bT = bS + CF::BUF;
    if constexpr (!CST) {
        load_op<P1, T, NT>(opD, D);
        load_op<P1, T, NT, true>(opT, D);
    }
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
        if constexpr (CST) {
            apply_lines_c<P1, P1, 1, R, NT, C, 0, OUT_SMEM>(bR, bS, nullptr, nullptr, nlines);
            apply_lines_c<P1, P1, 0, R, NT, C, 0, OUT_SMEM>(bR, bT, nullptr, nullptr, nlines);
            __syncthreads();
            apply_lines_c<P1, P1, 2, R, NT, C, 0, OUT_SMEM>(bR, bR, nullptr, nullptr, nlines);
        } else {
            apply_lines<P1, P1, 1, R, NT>(bR, opD, nlines, [&](int, int base, int k, T v) { bS[base + k * G::RS] = v; });
            apply_lines<P1, P1, 0, R, NT>(bR, opD, nlines, [&](int, int base, int k, T v) { bT[base + k * G::PS] = v; });
            __syncthreads();
            apply_lines<P1, P1, 2, R, NT>(bR, opD, nlines, [&](int, int base, int k, T v) { bR[base + k] = v; });
        }
        __syncthreads();
        const int total = ne * G::NPTS;
        // G[e][c][q]: AXE_PB points per thread per batch, all 6*AXE_PB loads issued before use
        constexpr int PB = P1 == 9 ? 8 : AXE_PB;  // measured: P1 = 9 0.57 -> 0.73 with 8; 8 is slower at 5 and 13
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
        if constexpr (CST) {
            apply_lines_c<P1, P1, 2, R, NT, C, 0, OUT_SMEM, false, true>(bR, bR, nullptr, nullptr, nlines);
            __syncthreads();
            apply_lines_c<P1, P1, 1, R, NT, C, 0, OUT_SMEM_ADD, false, true>(bS, bS, bR, nullptr, nlines);
            __syncthreads();
            apply_lines_c<P1, P1, 0, R, NT, C, 0, OUT_GLOBAL_ADD, false, true>(bT, nullptr, bS, Wout + gbase, nlines);
        } else {
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
}

template <int P1, int CS>
int launch_ax_e_k(int64_t N, const double* D, const double* U, const double* Gm, double* W, cudaStream_t s) {
    using CF = Cfg<P1, P1, double, 3, K_AXE, (CS >= 0)>;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    const int64_t ngroups = (N + CF::E - 1) / CF::E;
    const int grid = grid_for(ax_e_kernel<P1, CS>, CF::NT, CF::SMEM, ngroups, &occ);
    ax_e_kernel<P1, CS><<<grid, CF::NT, CF::SMEM, s>>>(N, D, U, Gm, W);
    const int st = launch_status();
    if (CS >= 0) op_slot_release(s, CS);
    return st;
}

template <int P1>
int launch_ax_e(int64_t N, const double* D, const double* U, const double* Gm, double* W, cudaStream_t s) {
    if (N >= OPS_CONST_MIN_N) {
        int slot, st;
        if ((st = op_slot_acquire(s, &D, 1, P1, &slot))) return st;
        return slot == 0 ? launch_ax_e_k<P1, 0>(N, D, U, Gm, W, s) : launch_ax_e_k<P1, 1>(N, D, U, Gm, W, s);
    }
    return launch_ax_e_k<P1, -1>(N, D, U, Gm, W, s);
}

// ---------------------------------------------------------------- constant-bank slots (host)
// One mutex serialises slot hand-out, the operator copies, the launch and the event record,
// so a slot's event always marks the last kernel that read it.  Per device: the symbol's
// backing address and one event per slot.  While `s` is being captured into a CUDA graph
// the cross-call wait/record is skipped (stream order inside the graph still holds; a
// replayed graph must not run concurrently with other spectral calls on the device).
namespace {
constexpr int MAX_DEV = 64;
struct DevSlots {
    double* base = nullptr;
    int next = 0;
    cudaEvent_t ev[OPS_SLOTS] = {};
    bool recorded[OPS_SLOTS] = {};
};
std::mutex g_ops_mu;
DevSlots g_ops[MAX_DEV];
thread_local bool g_ops_capturing = false;
}  // namespace

int op_slot_acquire(cudaStream_t s, const double* const* ops, int nops, int P1, int* slot) {
    g_ops_mu.lock();
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e == cudaSuccess && (dev < 0 || dev >= MAX_DEV)) e = cudaErrorInvalidDevice;
    DevSlots* d = e == cudaSuccess ? &g_ops[dev] : nullptr;
    if (e == cudaSuccess && !d->base) e = cudaGetSymbolAddress(reinterpret_cast<void**>(&d->base), c_ops);
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if (e == cudaSuccess) e = cudaStreamIsCapturing(s, &cap);
    g_ops_capturing = cap != cudaStreamCaptureStatusNone;
    if (e == cudaSuccess) {
        *slot = d->next;
        d->next = (d->next + 1) % OPS_SLOTS;
        if (!g_ops_capturing && d->recorded[*slot]) e = cudaStreamWaitEvent(s, d->ev[*slot], 0);
    }
    for (int i = 0; i < nops && e == cudaSuccess; ++i)
        e = cudaMemcpyAsync(d->base + ((size_t)*slot * OPS_PER_SLOT + i) * OPS_STRIDE, ops[i],
                            (size_t)P1 * P1 * sizeof(double), cudaMemcpyDeviceToDevice, s);
    if (e != cudaSuccess) {
        set_last_cuda_error(e);
        g_ops_mu.unlock();
        return BC_ERR_CUDA;
    }
    return BC_OK;  // lock held until op_slot_release
}

void op_slot_release(cudaStream_t s, int slot) {
    int dev = 0;
    if (!g_ops_capturing && cudaGetDevice(&dev) == cudaSuccess) {
        DevSlots& d = g_ops[dev];
        if (!d.ev[slot]) cudaEventCreateWithFlags(&d.ev[slot], cudaEventDisableTiming);
        if (d.ev[slot] && cudaEventRecord(d.ev[slot], s) == cudaSuccess) d.recorded[slot] = true;
    }
    g_ops_mu.unlock();
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
