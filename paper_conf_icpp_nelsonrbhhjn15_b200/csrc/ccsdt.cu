// CCSD(T) triples family on sm_100a: NWChem sd_t_d1 / sd_t_d2 / sd_t_s1, all 9 variants,
// single-variant and fused.
//
// Design.  The t3 block is cut into work units = (a cube of side BS in the
// three HOLE storage positions q1..q3) x (one value of the three PARTICLE positions
// q4..q6).  A CTA owns one unit and keeps its BS^3 t3 values as an fp64 accumulator in
// shared memory, so t3 is read and written exactly once per launch whatever the number of
// variants (the fused form reads/writes it once for up to 9 variants).
//
// For one variant the unit is a small GEMM in name space:
//   d1/s1:  X[(h3,h2), h1] = sum_k v2[h3,h2,p6,k] * t2[k,p4,p5,h1]
//   d2   :  X[(h1,h2), h3] = sum_k t2[k,p4,h1,h2] * v2[k,h3,p6,p5]
// (s1 is the K = 1 outer product v2[h3,h2,p6,p5] * t1[p4,h1]).  The "strided" operand
// covers a PAIR of hole names (BS^2 values), the "broadcast" operand the third (BS).  A
// cube in q-space is a cube in name space for every hole permutation, so the GEMM shape
// is the same for all variants.  Operand slices for (variant, k-chunk) stages are staged
// in shared memory by cp.async (zero-filled at block edges) one stage ahead of the
// compute.  Each thread accumulates a TS x TB register tile over k (scalar replacement,
// P:553-558): TS strided values at lane stride (conflict-free scalar reads) times TB
// broadcast values (16-byte reads); the variant's sign flips the broadcast values' sign
// bit.  Variants sharing a hole permutation ("class") accumulate into the same
// registers; a class is flushed into the shared accumulator cube at its permuted
// positions.  The cube has odd strides (1, BS+1, (BS+1)^2) on every axis, so the flush is
// bank-conflict free for any permutation.  The (h1,h2,h3) <-> storage-position maps are
// derived here from the generating rule of DESIGN.md R12 (not copied from the oracle).
//
// Kernels (dispatch in run_ccsdt / run_ccsdt_triples_energy):
//   ccsdt_kernel<FAM,BS>        DFMA cube kernel, any shape (fallback)
//   ccsdt_tma_kernel<FAM>       16-cube DMMA, warp-specialised TMA ring (fused, tile 16)
//   ccsdt_tma24_kernel<FAM>     exact 24-cube version (tile 24, fused and single variant)
//   ccsdt_svs_kernel<FAM,H>     one d1/d2 variant, t3 streamed through registers (16^3 holes)
//   ccsdt_s1h_kernel<H> / ccsdt_s1_stream_kernel<RUN>   s1 streams (equal 16/24 holes / any)
//   ccsdt_triples_energy_kernel / ccsdt_triples24_kernel  f4: 27 variants + energy (16- / 24-cube)
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstdlib>
#include <cstring>

#include "common.cuh"

namespace bc {

enum Family { FAM_D1 = 1, FAM_D2 = 2, FAM_S1 = 3 };
enum NameId { N_H1 = 0, N_H2 = 1, N_H3 = 2, N_P4 = 3, N_P5 = 4, N_P6 = 5, N_K = 6 };

struct VariantInfo {
    int order[6];  // storage position q -> name id (q = 0 fastest)
    int sign;
};

// Generating rule (R12): with i = (v-1) % 3 and j = (v-1) / 3,
//   d1, s1 holes : h1 at 0-based position 2-i, (h3, h2) keep their order
//   d2 holes     : h3 at position {0,2,1}[i], (h2, h1) keep their order
//   d1 particles : p6 at position {0,2,1}[j], (p5, p4) keep their order
//   d2, s1 part. : p4 at position 2-j,       (p6, p5) keep their order
//   sign         : -(hole parity)(particle parity) for d1/d2, + for s1, parities taken
//                  against (h3,h2,h1) and (p6,p5,p4).
static void place(int* out3, int moving, int pos, int a, int b) {
    int rest[2] = {a, b}, r = 0;
    for (int q = 0; q < 3; ++q) out3[q] = (q == pos) ? moving : rest[r++];
}
static int parity3(const int* s, const int* ref) {
    int idx[3];
    for (int q = 0; q < 3; ++q)
        for (int t = 0; t < 3; ++t)
            if (s[q] == ref[t]) idx[q] = t;
    int inv = 0;
    for (int a = 0; a < 3; ++a)
        for (int b = a + 1; b < 3; ++b) inv += idx[a] > idx[b];
    return (inv & 1) ? -1 : 1;
}
VariantInfo variant_info(int fam, int v) {
    VariantInfo vi;
    const int i = (v - 1) % 3, j = (v - 1) / 3;
    static const int p021[3] = {0, 2, 1};
    if (fam == FAM_D2)
        place(vi.order, N_H3, p021[i], N_H2, N_H1);
    else
        place(vi.order, N_H1, 2 - i, N_H3, N_H2);
    if (fam == FAM_D1)
        place(vi.order + 3, N_P6, p021[j], N_P5, N_P4);
    else
        place(vi.order + 3, N_P4, 2 - j, N_P6, N_P5);
    const int href[3] = {N_H3, N_H2, N_H1}, pref[3] = {N_P6, N_P5, N_P4};
    const int par = parity3(vi.order, href) * parity3(vi.order + 3, pref);
    vi.sign = (fam == FAM_S1) ? par : -par;
    return vi;
}

struct CcsdtParams {
    double* t3;
    const double* opA[9];  // t2 (d1, d2) or t1 (s1), per variant entry
    const double* opB[9];  // v2, per variant entry
    double sign[9];
    uint32_t smask[9];  // sign as the high-word sign-bit mask (0 or 0x80000000)
    int ppos[9][3];   // per entry: storage position (3..5) of p4, p5, p6
    int ecls[9];      // per entry: class slot
    int hpos[3][3];   // per class slot: storage position (0..2) of h1, h2, h3
    int nentry, ncls;
    int ext[7];       // named extents h1 h2 h3 p4 p5 p6 k
    int qe[6];        // storage-position extents
    int ncube[3];     // cubes along q1, q2, q3
    // optional energy check fused into the 16-cube TMA kernel's store pass (canonical
    // storage only): ews[blockIdx.x] = sum over the stored t3 of t^2 / den (bc_check_energy)
    const double* eps_h;
    const double* eps_p;
    double* ews;
};

// Per cube side BS: register tile TS (strided operand, one value per lane-stride) x TB
// (broadcast operand, 16-byte smem reads), k chunk KC.
template <int BS>
struct CcTile;
template <>
struct CcTile<16> { static constexpr int TS = 4, TB = 8; };
template <>
struct CcTile<12> { static constexpr int TS = 4, TB = 4; };
template <>
struct CcTile<8> { static constexpr int TS = 2, TB = 4; };

template <int BS>
struct CcGeo {
    static constexpr int TS = CcTile<BS>::TS, TB = CcTile<BS>::TB;
    static constexpr int SD = BS * BS;            // strided dim: a PAIR of hole names
    static constexpr int BD = BS;                 // broadcast dim: the third hole name
    static constexpr int MS = SD / TS;            // lanes along the strided dim
    static constexpr int NB = BD / TB;
    static constexpr int TILES = MS * NB;
    static constexpr int NT = (TILES + 31) / 32 * 32;
    static constexpr int KC = (BS >= 16) ? 8 : 16;  // k chunk per pipeline stage
    static constexpr int SS = SD + 1;             // odd row stride: conflict-free both ways
    static constexpr int SB = BD + 2;             // even row stride: 16-byte rows
    static constexpr int CST = BS + 1;            // accumulator cube strides 1, CST, CST^2 (all odd)
    static constexpr int ACC = BS * CST * CST;
    static constexpr int STAGE = KC * SS + KC * SB;  // even (KC even): stage bases stay 16-byte aligned
    static constexpr size_t SMEM = (size_t)(ACC + (ACC & 1) + 2 * STAGE + 2) * sizeof(double);
};

__device__ __forceinline__ void cp_async_8_zfill(void* dst, const void* src, bool valid) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(smem_u32(dst)), "l"(src),
                 "r"(valid ? 8 : 0));
}

// cp.async ordered after the preceding shared-memory reads of the same thread (the
// store-then-reseed of a cube position: the "memory" clobber keeps the compiler from
// moving the read of the old value past the copy that overwrites it)
__device__ __forceinline__ void cp_async_8_after_read(void* dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}

__device__ __forceinline__ double flip_sign(double x, uint32_t mask_hi) {
    return __hiloint2double(__double2hiint(x) ^ (int)mask_hi, __double2loint(x));
}

template <int FAM, int BS>
__global__ void __launch_bounds__(CcGeo<BS>::NT) ccsdt_kernel(const CcsdtParams P) {
    using CG = CcGeo<BS>;
    constexpr int NT = CG::NT, KC = CG::KC, TS = CG::TS, TB = CG::TB, MS = CG::MS;
    constexpr int SD = CG::SD, BD = CG::BD, SS = CG::SS, SB = CG::SB, CST = CG::CST;
    extern __shared__ __align__(16) double sm[];
    double* acc_s = sm;
    double* stage0 = sm + ((CG::ACC + 1) & ~1);

    // ---- unit decode: cube (o, len) in the hole positions, plane qv in the particle ones
    const int ncubes = P.ncube[0] * P.ncube[1] * P.ncube[2];
    const int cube = blockIdx.x % ncubes;
    const int plane = blockIdx.x / ncubes;
    int o[3], len[3];
    o[0] = (cube % P.ncube[0]) * BS;
    o[1] = ((cube / P.ncube[0]) % P.ncube[1]) * BS;
    o[2] = (cube / (P.ncube[0] * P.ncube[1])) * BS;
    for (int q = 0; q < 3; ++q) len[q] = min(BS, P.qe[q] - o[q]);
    int qv[3];
    qv[0] = plane % P.qe[3];
    qv[1] = (plane / P.qe[3]) % P.qe[4];
    qv[2] = plane / (P.qe[3] * P.qe[4]);

    for (int i = threadIdx.x; i < CG::ACC; i += NT) acc_s[i] = 0.0;

    const int H1 = P.ext[N_H1], H2 = P.ext[N_H2], H3 = P.ext[N_H3];
    const int P4 = P.ext[N_P4], P5 = P.ext[N_P5], P6 = P.ext[N_P6];
    const int K = (FAM == FAM_S1) ? 1 : P.ext[N_K];
    const int nchunk = (K + KC - 1) / KC;
    const int nstage = P.nentry * nchunk;

    // stage (entry e, chunk c) -> smem buffer b: strided operand Ss[kk][sd], broadcast Bb[kk][bd]
    auto issue = [&](int st, int b) {
        const int e = st / nchunk, k0 = (st - e * nchunk) * KC;
        const int kc = min(KC, K - k0);
        double* Ss = stage0 + b * CG::STAGE;
        double* Bb = Ss + KC * SS;
        const int c = P.ecls[e];
        const int hp1 = P.hpos[c][0], hp2 = P.hpos[c][1], hp3 = P.hpos[c][2];
        const int O1 = o[hp1], O2 = o[hp2], O3 = o[hp3];
        const int L1 = len[hp1], L2 = len[hp2], L3 = len[hp3];
        const int p4 = qv[P.ppos[e][0] - 3], p5 = qv[P.ppos[e][1] - 3], p6 = qv[P.ppos[e][2] - 3];
        const double* __restrict__ tA = P.opA[e];
        const double* __restrict__ vB = P.opB[e];
        if constexpr (FAM == FAM_D1 || FAM == FAM_S1) {
            // Ss[kk][i3 + BS*i2] = v2[h3,h2,p6,k] (d1) | v2[h3,h2,p6,p5] (s1): contiguous along h3
            for (int x = threadIdx.x; x < KC * SD; x += NT) {
                const int kk = x / SD, sd = x - kk * SD;
                const int i2 = sd / BS, i3 = sd - i2 * BS;
                const bool ok = kk < kc && i3 < L3 && i2 < L2;
                const int last = (FAM == FAM_S1) ? p5 : (k0 + kk);
                const double* src = vB + (ok ? (O3 + i3) + (int64_t)H3 * ((O2 + i2) + (int64_t)H2 * (p6 + (int64_t)P6 * last)) : 0);
                cp_async_8_zfill(Ss + kk * SS + sd, src, ok);
            }
            // Bb[kk][i1] = t2[k,p4,p5,h1] (d1) | t1[p4,h1] (s1): contiguous along k
            for (int x = threadIdx.x; x < KC * BD; x += NT) {
                const int i1 = x / KC, kk = x - i1 * KC;
                const bool ok = kk < kc && i1 < L1;
                int64_t off = 0;
                if (ok) {
                    if constexpr (FAM == FAM_S1)
                        off = p4 + (int64_t)P4 * (O1 + i1);
                    else
                        off = (k0 + kk) + (int64_t)K * (p4 + (int64_t)P4 * (p5 + (int64_t)P5 * (O1 + i1)));
                }
                cp_async_8_zfill(Bb + kk * SB + i1, tA + off, ok);
            }
        } else {
            // Ss[kk][i1 + BS*i2] = t2[k,p4,h1,h2]: contiguous along k
            for (int x = threadIdx.x; x < KC * SD; x += NT) {
                const int sd = x / KC, kk = x - sd * KC;
                const int i2 = sd / BS, i1 = sd - i2 * BS;
                const bool ok = kk < kc && i1 < L1 && i2 < L2;
                const double* src = tA + (ok ? (k0 + kk) + (int64_t)K * (p4 + (int64_t)P4 * ((O1 + i1) + (int64_t)H1 * (O2 + i2))) : 0);
                cp_async_8_zfill(Ss + kk * SS + sd, src, ok);
            }
            // Bb[kk][i3] = v2[k,h3,p6,p5]: contiguous along k
            for (int x = threadIdx.x; x < KC * BD; x += NT) {
                const int i3 = x / KC, kk = x - i3 * KC;
                const bool ok = kk < kc && i3 < L3;
                const double* src = vB + (ok ? (k0 + kk) + (int64_t)K * ((O3 + i3) + (int64_t)H3 * (p6 + (int64_t)P6 * p5)) : 0);
                cp_async_8_zfill(Bb + kk * SB + i3, src, ok);
            }
        }
    };

    const int tid = threadIdx.x;
    const bool has_tile = tid < CG::TILES;
    const int ms = tid % MS, nb = tid / MS;

    double acc[TS][TB];
#pragma unroll
    for (int a = 0; a < TS; ++a)
#pragma unroll
        for (int b = 0; b < TB; ++b) acc[a][b] = 0.0;

    if (nstage > 0) issue(0, 0);
    cp_async_commit();
    for (int st = 0; st < nstage; ++st) {
        cp_async_wait_all();
        __syncthreads();
        if (st + 1 < nstage) issue(st + 1, (st + 1) & 1);
        cp_async_commit();
        const int e = st / nchunk, k0 = (st - e * nchunk) * KC;
        const int kc = min(KC, K - k0);
        const double* Ss = stage0 + (st & 1) * CG::STAGE;
        const double* Bb = Ss + KC * SS;
        const uint32_t smask = P.sign[e] < 0 ? 0x80000000u : 0u;
        if (has_tile) {
#pragma unroll 4
            for (int kk = 0; kk < kc; ++kk) {
                double sv[TS], bv[TB];
#pragma unroll
                for (int a = 0; a < TS; ++a) sv[a] = Ss[kk * SS + ms + MS * a];
#pragma unroll
                for (int b = 0; b < TB; b += 2) {
                    const double2 t = *reinterpret_cast<const double2*>(Bb + kk * SB + TB * nb + b);
                    bv[b] = flip_sign(t.x, smask);
                    bv[b + 1] = flip_sign(t.y, smask);
                }
#pragma unroll
                for (int a = 0; a < TS; ++a)
#pragma unroll
                    for (int b = 0; b < TB; ++b) acc[a][b] = fma(sv[a], bv[b], acc[a][b]);
            }
        }
        // last chunk of the last entry of a class: flush the class into the cube
        const bool last_chunk = (k0 + KC >= K);
        const bool class_end = last_chunk && (e + 1 == P.nentry || P.ecls[e + 1] != P.ecls[e]);
        if (class_end) {
            if (has_tile) {
                const int c = P.ecls[e];
                const int strq[3] = {1, CST, CST * CST};
                const int s1 = strq[P.hpos[c][0]], s2 = strq[P.hpos[c][1]], s3 = strq[P.hpos[c][2]];
#pragma unroll
                for (int a = 0; a < TS; ++a) {
                    const int sd = ms + MS * a;
                    const int hi = sd / BS, lo = sd - hi * BS;
                    // d1/s1: strided = (i3 = lo, i2 = hi), broadcast = i1;  d2: strided = (i1 = lo, i2 = hi), broadcast = i3
                    const int base = (FAM == FAM_D2) ? (lo * s1 + hi * s2) : (lo * s3 + hi * s2);
                    const int sb = (FAM == FAM_D2) ? s3 : s1;
#pragma unroll
                    for (int b = 0; b < TB; ++b) {
                        acc_s[base + (TB * nb + b) * sb] += acc[a][b];
                        acc[a][b] = 0.0;
                    }
                }
            }
        }
    }
    __syncthreads();
    // ---- t3 += accumulator (read and written once, coalesced along q1)
    const int64_t pbase = (int64_t)P.qe[0] * P.qe[1] * P.qe[2] *
                          (qv[0] + (int64_t)P.qe[3] * (qv[1] + (int64_t)P.qe[4] * qv[2]));
    const int nvol = len[0] * len[1] * len[2];
    for (int i = tid; i < nvol; i += NT) {
        const int q0 = i % len[0], r = i / len[0];
        const int q1 = r % len[1], q2 = r / len[1];
        double* p = P.t3 + pbase + (o[0] + q0) + (int64_t)P.qe[0] * ((o[1] + q1) + (int64_t)P.qe[1] * (o[2] + q2));
        *p += acc_s[q0 + CST * (q1 + CST * q2)];
    }
}

// FP64 tensor-core MMA (no tcgen05 f64 kind exists; DMMA reaches the full FP64 rate with
// 1/8 of DFMA's instruction count, profiles/fp64_peak_r01.txt)
__device__ __forceinline__ void dmma_8x8x4(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

// ==================================================================================
// Blackwell-native path (BS = 16, d1/d2): persistent, warp-specialised kernel.
//   warp 8 (producer): one lane drives the Tensor Memory Accelerator —
//     cp.async.bulk.tensor copies of each (variant, k-chunk) operand slice straight from
//     the 4-D t2 / v2 tensors into a 4-deep shared-memory ring, with hardware swizzling
//     (bank-conflict-free fragment reads) and out-of-bounds zero fill (ragged blocks),
//     completion tracked by full/empty mbarriers — no per-thread staging code at all.
//   warps 0-7 (consumers): FP64 DMMA m8n8k4 on the staged slices, accumulating per hole
//     permutation class in registers, flushed into the unit's t3 cube in shared memory.
// Each CTA loops over units (a 16^3 hole cube x one particle plane); the unit's t3 values
// seed the cube (read once, cp.async) and the cube is stored once.
// Operand layouts in one stage (KC = 8 k values):
//   d1: A = v2[h3, O2+i2, p6, k]: 8 copies (h2 pairs) of [k][h2'][h3] (128 B rows, 128B
//       swizzle; the swizzle row 2k + h2' differs for the 4 k of a fragment)
//       B = t2[k, p4, p5, h1]: [h1][k] (64 B rows, 64B swizzle)
//   d2: A = t2[k, p4, h1, h2]: [h2][h1][k] (64 B rows, 64B swizzle)
//       B = v2[k, h3, p6, p5]: [h3][k] (64 B rows, 64B swizzle)
// 64B-swizzled fragment rows are permuted ({0,1,4,5,2,3,6,7}) so that each half-warp
// touches 16 distinct banks.
// ==================================================================================
struct TmaMaps {
    CUtensorMap a[9];  // d1: v2_v (h3,h2,p6,k) | d2: t2_v (k,p4,h1,h2)
    CUtensorMap b[9];  // d1: t2_v (k,p4,p5,h1) | d2: v2_v (k,h3,p6,p5)
};

#ifndef BC_TC16_SINGLE_NS1
#define BC_TC16_SINGLE_NS1 1
#endif
#ifndef BC_TC16_KC
#define BC_TC16_KC 16
#endif
#ifndef BC_EXP16_NOFLUSH
#define BC_EXP16_NOFLUSH 0  // timing experiments only: skip the class flushes of the 16-cube kernel
#endif
#ifndef BC_EXP16_NOTMA
#define BC_EXP16_NOTMA 0  // timing experiments only: no operand copies (the ring still cycles)
#endif
#ifndef BC_EXP16_NOSTORE
#define BC_EXP16_NOSTORE 0  // timing experiments only: skip the store / re-seed of the 16-cube kernel
#endif
#ifndef BC_FLUSH_ALWAYS_BAR
#define BC_FLUSH_ALWAYS_BAR 0  // consumer barrier before every class flush (else only where needed)
#endif
#ifndef BC_TC16_NS
#define BC_TC16_NS 0  // ring depth of the fused tile-16 kernel (0: 2 at KC = 16, 4 at KC = 8)
#endif
#ifndef BC_TC16_MINB
#define BC_TC16_MINB 2  // CTAs per SM of the fused tile-16 kernel
#endif
struct TmaGeo {
    // two CTAs per SM (measured better than one CTA with a deeper ring).  KC = 8: 64 B
    // operand rows (64B swizzle), 4-deep ring;  KC = 16: 128 B rows (128B swizzle, half the
    // TMA rows per byte), 2-deep ring
    static constexpr int BS = 16, KC = BC_TC16_KC, NS = BC_TC16_NS ? BC_TC16_NS : (KC == 16 ? 2 : 4), NCW = 8,
                         NT = (NCW + 1) * 32;
    static constexpr int A_BYTES = 16 * 16 * KC * 8;  // 16 | 32 KiB
    static constexpr int B_BYTES = 16 * KC * 8;       // 1 | 2 KiB
    static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;  // multiple of 1 KiB
    static constexpr int ROW = KC * 8;                // operand row bytes (k innermost)
    static constexpr int CST = BS + 1;
    static constexpr int ACC = BS * CST * CST;          // doubles
    static constexpr size_t SMEM = 1024 + (size_t)NS * STAGE_BYTES + ACC * 8 + 2 * NS * 8;
};

__device__ __forceinline__ void tma_load_4d(uint32_t dst, const CUtensorMap* map, int c0, int c1, int c2, int c3,
                                            uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];\n"
        ::"r"(dst), "l"(map), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(bar) : "memory");
}
// fragment loads as volatile asm: kept in program order relative to the (volatile) DMMAs,
// so a stage's fragments are all loaded into distinct registers before its first DMMA
// (plain loads let ptxas reuse one register per fragment and expose the LDS latency
// between DMMAs)
__device__ __forceinline__ double lds64(const void* p) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];\n" : "=d"(v) : "r"(smem_u32(p)));
    return v;
}

// 64B-swizzle fragment row permutation (see header)
__device__ __forceinline__ int perm64(int g) { return (g & 1) + 4 * ((g >> 1) & 1) + 2 * (g >> 2); }
// byte offset of element (row, col) in 64-byte rows under the 64B swizzle
__device__ __forceinline__ uint32_t swz64(uint32_t row, uint32_t col) {
    const uint32_t off = row * 64 + col * 8;
    return off ^ (((off >> 7) & 3) << 4);
}
// 16-cube kernels: k-innermost operand rows of TmaGeo::ROW bytes, swizzled (64B | 128B);
// fragment row permutation so a half-warp's 4 rows x 4 k hit 16 distinct banks, and an
// 8-row step (+8 ROW bytes) leaves the XOR pattern unchanged
__device__ __forceinline__ int permK(int g) {
    return TmaGeo::KC == 16 ? 2 * (g & 3) + (g >> 2) : perm64(g);
}
__device__ __forceinline__ uint32_t swzK(uint32_t row, uint32_t col) {
    if (TmaGeo::KC == 16) {
        const uint32_t off = row * 128 + col * 8;
        return off ^ ((row & 7) << 4);
    }
    return swz64(row, col);
}

// ---- per-family pieces shared by the TMA kernels ----------------------------------
// d1's A slice v2[h3, h2, p6, k] (k outermost in global memory): 1 = one TMA box
// {16, 16, 1, 8} -> [k][h2][h3] (4-way conflicted fragment reads, 2 boxes per stage);
// 0 = 8 boxes {16, 2, 1, 8} with 128B swizzle (conflict-free reads, 9 boxes per stage).
// The TMA unit costs ~70 clk per box + ~3.3 clk per box row (measured).
#ifndef BC_TC16_ONEBOX
#define BC_TC16_ONEBOX 0
#endif
// producer: issue the TMA copies of one (entry e, k chunk k0) stage into slot buffers A/B
template <int FE>
__device__ __forceinline__ void tma_issue_stage(const CUtensorMap* ma, const CUtensorMap* mb, uint32_t A, uint32_t B,
                                                uint32_t full, int lane, int O1, int O2, int O3, int p4, int p5,
                                                int p6, int k0) {
    if constexpr (FE == FAM_D1 && BC_TC16_ONEBOX) {
        if (lane == 0) tma_load_4d(A, ma, O3, O2, p6, k0, full);
        if (lane == 1) tma_load_4d(B, mb, k0, p4, p5, O1, full);
    } else if constexpr (FE == FAM_D1) {
        if (lane == 0) {  // one issuing lane measured faster than spreading the copies
#pragma unroll 1
            for (int j = 0; j < 8; ++j) tma_load_4d(A + j * (TmaGeo::A_BYTES / 8), ma, O3, O2 + 2 * j, p6, k0, full);
            tma_load_4d(B, mb, k0, p4, p5, O1, full);
        }
    } else {
        if (lane == 0) tma_load_4d(A, ma, k0, p4, O1, O2, full);
        if (lane == 1) tma_load_4d(B, mb, k0, O3, p6, p5, full);
    }
}

// consumer: one KC = 8 stage of DMMA for this warp's 32 pairs x 16 thirds (k beyond the
// tensor extent arrives zero-filled by TMA)
template <int FE>
__device__ __forceinline__ void tma_consume_stage(const unsigned char* A, const unsigned char* B, uint32_t smask,
                                                      double (&c)[4][2][2], int warp, int gq, int tq) {
    double bfa[TmaGeo::KC / 4][2], afa[TmaGeo::KC / 4][4];
    // an 8-row step of a 64B-swizzled operand is +512 B with the same XOR pattern, so the
    // n-/m-tiles are immediate offsets from one base per k-step
#pragma unroll
    for (int ks = 0; ks < TmaGeo::KC / 4; ++ks) {
        const unsigned char* Bk = B + swzK(permK(gq), ks * 4 + tq);
#pragma unroll
        for (int ni = 0; ni < 2; ++ni) bfa[ks][ni] = lds64(Bk + ni * 8 * TmaGeo::ROW);
    }
#pragma unroll
    for (int ks = 0; ks < TmaGeo::KC / 4; ++ks) {
        const int kk = ks * 4 + tq;
        const unsigned char* Ak = (FE == FAM_D1) ? A + (kk * 256 + 32 * warp + gq) * 8
                                                 : A + 32 * warp * TmaGeo::ROW + swzK(permK(gq), kk);
#pragma unroll
        for (int mi = 0; mi < 4; ++mi) {
            uint32_t off;
            if constexpr (FE == FAM_D1 && BC_TC16_ONEBOX) {
                // one box [k][h2][h3]: pair (h3, h2) = (8 (mi & 1) + gq, 2 warp + (mi >> 1))
                afa[ks][mi] = lds64(Ak + ((mi >> 1) * 16 + 8 * (mi & 1)) * 8);
                continue;
            } else if constexpr (FE == FAM_D2) {
                afa[ks][mi] = lds64(Ak + mi * 8 * TmaGeo::ROW);
                continue;
            } else if constexpr (FE == FAM_D1) {
                // copy j = warp holds h2 = O2 + 2 warp + {0,1}: rows r = 2 kk + (mi >> 1)
                const int i3 = 8 * (mi & 1) + gq;
                const int r = 2 * kk + (mi >> 1);
                off = warp * (TmaGeo::A_BYTES / 8) + r * 128 + ((((i3 >> 1) ^ r) & 7) << 4) + ((i3 & 1) << 3);
            } else {
                off = swzK(32 * warp + 8 * mi + permK(gq), kk);
            }
            afa[ks][mi] = lds64(A + off);
        }
    }
#pragma unroll
    for (int ks = 0; ks < TmaGeo::KC / 4; ++ks)
#pragma unroll
        for (int ni = 0; ni < 2; ++ni) bfa[ks][ni] = flip_sign(bfa[ks][ni], smask);
#pragma unroll
    for (int ks = 0; ks < TmaGeo::KC / 4; ++ks)
#pragma unroll
        for (int mi = 0; mi < 4; ++mi)
#pragma unroll
            for (int ni = 0; ni < 2; ++ni) dmma_8x8x4(c[mi][ni][0], c[mi][ni][1], afa[ks][mi], bfa[ks][ni]);
}

// consumer: add a class's register tile into the accumulator cube at its permuted
// positions (hp = storage positions of h1, h2, h3) and clear the registers
template <int FE, bool STORE = false>
__device__ __forceinline__ void tma_flush_class(double* acc_s, double (&c)[4][2][2], const int* hp, int warp, int gq,
                                                int tq) {
    constexpr int CST = TmaGeo::CST;
    const int s1 = hp[0] == 0 ? 1 : (hp[0] == 1 ? CST : CST * CST);
    const int s2 = hp[1] == 0 ? 1 : (hp[1] == 1 ? CST : CST * CST);
    const int s3 = hp[2] == 0 ? 1 : (hp[2] == 1 ? CST : CST * CST);
    // The 16 positions a thread updates are distinct, but the compiler cannot prove it and
    // serialised the read-modify-writes (LDS -> DADD -> STS -> next LDS: ~16 dependent
    // round trips per flush).  All reads are issued first, then the adds and stores.
    int pos[4][2][2];
#pragma unroll
    for (int mi = 0; mi < 4; ++mi) {
        int hi, lo;  // strided pair (lo = fast name, hi = h2)
        if constexpr (FE == FAM_D1) {
            hi = 2 * warp + (mi >> 1);
            lo = 8 * (mi & 1) + gq;
        } else {
            const int sidx = 32 * warp + 8 * mi + permK(gq);
            hi = sidx >> 4;
            lo = sidx & 15;
        }
        const int rowoff = (FE == FAM_D2) ? (lo * s1 + hi * s2) : (lo * s3 + hi * s2);
        const int sb = (FE == FAM_D2) ? s3 : s1;
#pragma unroll
        for (int ni = 0; ni < 2; ++ni)
#pragma unroll
            for (int j = 0; j < 2; ++j) pos[mi][ni][j] = rowoff + (ni * 8 + permK(2 * tq + j)) * sb;
    }
    // STORE: the unit's first class writes the cube (every position, out-of-range ones as
    // zeros from the zero-filled operands) instead of read-modify-writing a zeroed cube
    double old[4][2][2];
#pragma unroll
    for (int mi = 0; mi < 4; ++mi)
#pragma unroll
        for (int ni = 0; ni < 2; ++ni)
#pragma unroll
            for (int j = 0; j < 2; ++j) old[mi][ni][j] = STORE ? 0.0 : acc_s[pos[mi][ni][j]];
#pragma unroll
    for (int mi = 0; mi < 4; ++mi)
#pragma unroll
        for (int ni = 0; ni < 2; ++ni)
#pragma unroll
            for (int j = 0; j < 2; ++j) {
                acc_s[pos[mi][ni][j]] = old[mi][ni][j] + c[mi][ni][j];
                c[mi][ni][j] = 0.0;
            }
}

// NSR: ring depth.  Single-variant launches (one stage per unit at tile 16) use NSR = 1
// and 3 CTAs/SM: more units (t3 seeds) in flight for the HBM-bound case.
// Unit index u = cube + ncubes * plane as six mixed-radix digits (cube coordinates along
// the three hole positions, plane coordinates along the three particle positions), so a
// persistent CTA advances u by gridDim.x with carries instead of six runtime divisions.
struct UnitDigits {
    int d[6];
};
__device__ __forceinline__ UnitDigits unit_digits(int u, const int (&r)[6]) {  // divisions: once per CTA
    UnitDigits x;
#pragma unroll
    for (int i = 0; i < 6; ++i) {
        const int q = u / r[i];
        x.d[i] = u - q * r[i];
        u = q;
    }
    return x;
}
__device__ __forceinline__ void unit_add(UnitDigits& x, const UnitDigits& s, const int (&r)[6]) {
    int carry = 0;
#pragma unroll
    for (int i = 0; i < 6; ++i) {
        const int v = x.d[i] + s.d[i] + carry;
        carry = v >= r[i];
        x.d[i] = carry ? v - r[i] : v;
    }
}
// EN: the fused energy check (a separate instantiation: the energy code in the store pass
// slowed the plain kernel by 4-5% even when disabled at run time)
template <int FAM, int NSR = TmaGeo::NS, int MINB = BC_TC16_MINB, bool EN = false>
__global__ void __launch_bounds__(TmaGeo::NT, MINB) ccsdt_tma_kernel(const __grid_constant__ CcsdtParams P,
                                                                     const __grid_constant__ TmaMaps M, int units) {
    using TG = TmaGeo;
    constexpr int BS = TG::BS, KC = TG::KC, NS = NSR, CST = TG::CST;
    extern __shared__ unsigned char smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023) & ~1023u;
    unsigned char* gbase = smem_raw + (base - raw);
    const uint32_t st_u32 = base;                                   // stage ring
    double* acc_s = reinterpret_cast<double*>(gbase + NS * TG::STAGE_BYTES);
    const uint32_t bar_full = base + NS * TG::STAGE_BYTES + TG::ACC * 8;
    const uint32_t bar_empty = bar_full + NS * 8;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) {
            mbar_init(bar_full + 8 * i, 1);
            mbar_init(bar_empty + 8 * i, TG::NCW);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();

    const int K = P.ext[N_K];
    const int nchunk = (K + KC - 1) / KC;
    const int nstage = P.nentry * nchunk;

    int rad[6] = {P.ncube[0], P.ncube[1], P.ncube[2], P.qe[3], P.qe[4], P.qe[5]};
    const UnitDigits ustep = unit_digits(gridDim.x, rad);
    auto decode_d = [&](const UnitDigits& x, int* o, int* len, int* qv) {
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            o[q] = x.d[q] * BS;
            len[q] = min(BS, P.qe[q] - o[q]);
            qv[q] = x.d[3 + q];
        }
    };

    if (warp == TG::NCW) {
        // ================================ producer: lane 0 arms the stage, lanes issue copies
        int g = 0;
        UnitDigits ud = unit_digits(blockIdx.x, rad);
        for (int u = blockIdx.x; u < units; u += gridDim.x, unit_add(ud, ustep, rad)) {
            int o[3], len[3], qv[3];
            decode_d(ud, o, len, qv);
            int e = 0, kc_i = 0;
            for (int st = 0; st < nstage; ++st, ++g) {
                const int slot = g % NS;
                const uint32_t full = bar_full + 8 * slot;
                if (lane == 0) {
                    mbar_wait(bar_empty + 8 * slot, ((g / NS) & 1) ^ 1);
                    if (BC_EXP16_NOTMA)  // timing experiment only (stale operands)
                        mbar_arrive(full);
                    else
                        mbar_expect_tx(full, TG::STAGE_BYTES);
                }
                __syncwarp();
                if (BC_EXP16_NOTMA) continue;
                const int k0 = kc_i * KC;
                if (++kc_i == nchunk) kc_i = 0;
                const int e_cur = e;
                if (kc_i == 0) ++e;
                const int c = P.ecls[e_cur];
                auto opos = [&](int pos) { return pos == 0 ? o[0] : (pos == 1 ? o[1] : o[2]); };
                const int O1 = opos(P.hpos[c][0]), O2 = opos(P.hpos[c][1]), O3 = opos(P.hpos[c][2]);
                auto pick = [&](int pos) { return pos == 3 ? qv[0] : (pos == 4 ? qv[1] : qv[2]); };
                const int p4 = pick(P.ppos[e_cur][0]), p5 = pick(P.ppos[e_cur][1]), p6 = pick(P.ppos[e_cur][2]);
                const uint32_t A = st_u32 + slot * TG::STAGE_BYTES;
                tma_issue_stage<FAM>(&M.a[e_cur], &M.b[e_cur], A, A + TG::A_BYTES, full, lane, O1, O2, O3, p4, p5, p6,
                                     k0);
            }
        }
        return;
    }

    // ==================================== consumers (warps 0..7)
    const int gq = lane >> 2, tq = lane & 3;
    const int tid = threadIdx.x;  // < 256
    // t3 of the unit -> cube (cp.async, one group).  Full 16^3 cubes: thread t owns
    // (q0, q1) = (t & 15, t >> 4) for every q2 — a constant stride per copy.
    const int Q0 = P.qe[0], Q01 = P.qe[0] * P.qe[1];
    auto seed = [&](const int* o, const int* len, int64_t pbase, double* cube) {
        if (len[0] == BS && len[1] == BS && len[2] == BS) {
            const int q0 = tid & 15, q1 = tid >> 4;
            const double* src = P.t3 + pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)P.qe[1] * o[2]);
            double* dst = cube + q0 + CST * q1;
#pragma unroll
            for (int q2 = 0; q2 < BS; ++q2) cp_async_8(dst + CST * CST * q2, src + (int64_t)Q01 * q2);
        } else {
            const int nvol = len[0] * len[1] * len[2];
            for (int i = tid; i < nvol; i += 256) {
                const int q0 = i % len[0], r = i / len[0];
                const int q1 = r % len[1], q2 = r / len[1];
                cp_async_8(cube + q0 + CST * (q1 + CST * q2),
                           P.t3 + pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)P.qe[1] * (o[2] + q2)));
            }
        }
    };
    const bool full_cubes = P.qe[0] % BS == 0 && P.qe[1] % BS == 0 && P.qe[2] % BS == 0;
    double energy = 0.0;  // fused energy check (P.ews; the launcher passes it for full cubes only)
    int g = 0;
    UnitDigits ud = unit_digits(blockIdx.x, rad);
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
        int o[3], len[3], qv[3];
        decode_d(ud, o, len, qv);
        unit_add(ud, ustep, rad);  // ud: the CTA's next unit (u + gridDim.x)
        const int64_t pbase = (int64_t)P.qe[0] * P.qe[1] * P.qe[2] *
                              (qv[0] + (int64_t)P.qe[3] * (qv[1] + (int64_t)P.qe[4] * qv[2]));
        const int nvol = len[0] * len[1] * len[2];
        // all cubes full: thread t owns positions (t & 15, t >> 4, *) in every unit, so the
        // previous unit's store and this unit's seed were issued together at its end (no
        // barrier); otherwise barrier, then seed
        if (!full_cubes) {
            named_bar_sync(1, 256);  // the previous unit's store from the cube is complete
            seed(o, len, pbase, acc_s);  // lands while the first stages compute
        } else if (u == (int)blockIdx.x) {
            seed(o, len, pbase, acc_s);
        }
        cp_async_commit();
        bool seeded = false;


        double c[4][2][2];
#pragma unroll
        for (int mi = 0; mi < 4; ++mi)
#pragma unroll
            for (int ni = 0; ni < 2; ++ni) c[mi][ni][0] = c[mi][ni][1] = 0.0;

        // per-entry values cached in registers (dynamic-index constant-bank loads every stage
        // showed up as long-scoreboard stalls)
        int e = 0, kc_i = 0, cls_stages = 0;
        uint32_t smask = P.smask[0];
        bool class_end = (P.nentry == 1) || (P.ecls[1] != P.ecls[0]);
        for (int st = 0; st < nstage; ++st, ++g) {
            ++cls_stages;
            const int slot = g % NS;
            mbar_wait(bar_full + 8 * slot, (g / NS) & 1);
            const unsigned char* A = gbase + slot * TG::STAGE_BYTES;
            const unsigned char* B = A + TG::A_BYTES;
            tma_consume_stage<FAM>(A, B, smask, c, warp, gq, tq);
            release_slot(bar_empty + 8 * slot, lane);
            const bool last_chunk = (++kc_i == nchunk);
            const int e_cur = e;
            if (last_chunk) {
                kc_i = 0;
                ++e;
            }
            if (last_chunk && class_end) {
                // consumer warps only meet at unit boundaries, so without this barrier a fast
                // warp could flush the next class onto positions a slow warp is still
                // read-modify-writing for this one (and the seed must have landed).  Not
                // needed after the first flush when the class spans more than NS stages: the
                // producer refills a slot only after all consumers released it, so the
                // fastest warp is at most NS stages ahead of the slowest.
                const bool need_bar = BC_FLUSH_ALWAYS_BAR || !seeded || cls_stages <= NS;
                if (!seeded) cp_async_wait_n<0>();
                seeded = true;
                if (need_bar) named_bar_sync(1, 256);
                cls_stages = 0;
                if (BC_EXP16_NOFLUSH) {  // timing experiment only (wrong results)
#pragma unroll
                    for (int mi = 0; mi < 4; ++mi)
#pragma unroll
                        for (int ni = 0; ni < 2; ++ni)
                            if (c[mi][ni][0] == 1.2345) acc_s[mi] = c[mi][ni][1];
                } else {
                    tma_flush_class<FAM>(acc_s, c, P.hpos[P.ecls[e_cur]], warp, gq, tq);
                }
            }
            if (last_chunk && e < P.nentry) {
                smask = P.smask[e];
                class_end = (e + 1 == P.nentry) || (P.ecls[e + 1] != P.ecls[e]);
            }
        }
        if (!seeded) {
            cp_async_wait_n<0>();
            seeded = true;
        }
        named_bar_sync(1, 256);  // all flushes into / reads of this cube are done
        if (BC_EXP16_NOSTORE) {  // timing experiment only (wrong results)
        } else if (full_cubes) {
            // store this unit and seed the CTA's next unit, position by position (same owner)
            const int q0 = tid & 15, q1 = tid >> 4;
            double* dstg = P.t3 + pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)P.qe[1] * o[2]);
            double* srcs = acc_s + q0 + CST * q1;
            // fused energy check (canonical storage: q = h3, h2, h1, p6, p5, p4), the order
            // of additions of bc_check_energy's denominator
            double dh = 0.0, dp = 0.0;
            const double* eh1 = P.eps_h;
            double dp5 = 0.0, dp4 = 0.0;
            if constexpr (EN) {
                dh = P.eps_h[P.ext[N_H1] + P.ext[N_H2] + o[0] + q0] + P.eps_h[P.ext[N_H1] + o[1] + q1];
                dp = P.eps_p[P.ext[N_P4] + P.ext[N_P5] + qv[0]];
                dp5 = P.eps_p[P.ext[N_P4] + qv[1]];
                dp4 = P.eps_p[qv[2]];
            }
            // t^2 / den with a hardware reciprocal estimate refined by two Newton steps
            // (relative error ~1 ulp; the DDIV sequence in the unit epilogue cost more than
            // the separate energy pass it replaces)
            auto en = [&](double t, int q2) {
                if constexpr (EN) {
                    const double den = (((dh + eh1[o[2] + q2]) - dp) - dp5) - dp4;
                    double r;
                    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(den));
                    r = fma(r, fma(-den, r, 1.0), r);
                    r = fma(r, fma(-den, r, 1.0), r);
                    energy = fma(t * t, r, energy);
                }
            };
            const int un = u + gridDim.x;
            if (un < units) {
                int on[3], lenn[3], qvn[3];
                decode_d(ud, on, lenn, qvn);
                const int64_t pbn = (int64_t)P.qe[0] * P.qe[1] * P.qe[2] *
                                    (qvn[0] + (int64_t)P.qe[3] * (qvn[1] + (int64_t)P.qe[4] * qvn[2]));
                const double* srcg = P.t3 + pbn + (on[0] + q0) + (int64_t)Q0 * ((on[1] + q1) + (int64_t)P.qe[1] * on[2]);
#pragma unroll
                for (int q2 = 0; q2 < BS; ++q2) {
                    const double t = srcs[CST * CST * q2];
                    dstg[(int64_t)Q01 * q2] = t;
                    cp_async_8_after_read(srcs + CST * CST * q2, srcg + (int64_t)Q01 * q2);
                    en(t, q2);
                }
                cp_async_commit();
            } else {
#pragma unroll
                for (int q2 = 0; q2 < BS; ++q2) {
                    const double t = srcs[CST * CST * q2];
                    dstg[(int64_t)Q01 * q2] = t;
                    en(t, q2);
                }
            }
        } else if (len[0] == BS && len[1] == BS && len[2] == BS) {
            const int q0 = tid & 15, q1 = tid >> 4;
            double* dstg = P.t3 + pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)P.qe[1] * o[2]);
            const double* srcs = acc_s + q0 + CST * q1;
#pragma unroll
            for (int q2 = 0; q2 < BS; ++q2) dstg[(int64_t)Q01 * q2] = srcs[CST * CST * q2];
        } else {
            for (int i = tid; i < nvol; i += 256) {
                const int q0 = i % len[0], r = i / len[0];
                const int q1 = r % len[1], q2 = r / len[1];
                P.t3[pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)P.qe[1] * (o[2] + q2))] =
                    acc_s[q0 + CST * (q1 + CST * q2)];
            }
        }
    }
    cp_async_wait_all();
    if constexpr (EN) {  // consumer-only block reduction (the producer warp has left)
        __shared__ double red[TG::NCW];
        for (int off = 16; off > 0; off >>= 1) energy += __shfl_xor_sync(0xffffffffu, energy, off);
        if (lane == 0) red[warp] = energy;
        named_bar_sync(1, 256);
        if (tid == 0) {
            double sum = 0.0;
            for (int w = 0; w < TG::NCW; ++w) sum += red[w];
            P.ews[blockIdx.x] = sum;
        }
    }
}

// ---- host: tensor maps (driver entry point, no -lcuda)
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {  // process-wide driver entry point
    static const PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
        return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    }();
    return fn;
}

static bool encode_4d_sw(CUtensorMap* m, const double* ptr, const int* dims, const int* box, CUtensorMapSwizzle sw) {
    auto enc = get_encode();
    if (!enc) return false;
    cuuint64_t gdim[4], gstr[3];
    cuuint32_t bdim[4], estr[4] = {1, 1, 1, 1};
    cuuint64_t st = 8;
    for (int i = 0; i < 4; ++i) {
        gdim[i] = (cuuint64_t)dims[i];
        bdim[i] = (cuuint32_t)box[i];
        if (i > 0) gstr[i - 1] = st;
        st *= (cuuint64_t)dims[i];
    }
    const CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, const_cast<double*>(ptr), gdim, gstr, bdim, estr,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

static bool encode_4d(CUtensorMap* m, const double* ptr, const int* dims, const int* box, bool swz128) {
    return encode_4d_sw(m, ptr, dims, box, swz128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B);
}

// d1 A (v2) tensor map of the 16-cube kernels (see BC_TC16_ONEBOX)
static bool encode_d1_a16(CUtensorMap* m, const double* v2, const int* dims) {
    const int one[4] = {16, 16, 1, TmaGeo::KC}, eight[4] = {16, 2, 1, TmaGeo::KC};
    return BC_TC16_ONEBOX ? encode_4d_sw(m, v2, dims, one, CU_TENSOR_MAP_SWIZZLE_NONE)
                          : encode_4d_sw(m, v2, dims, eight, CU_TENSOR_MAP_SWIZZLE_128B);
}

// returns 1 when the TMA path is unavailable (caller falls back)
template <int FAM>
static int launch_ccsdt_tma(const CcsdtParams& P, cudaStream_t s) {
    TmaMaps M;
    memset(&M, 0, sizeof(M));
    const int H1 = P.ext[N_H1], H2 = P.ext[N_H2], H3 = P.ext[N_H3];
    const int P4 = P.ext[N_P4], P5 = P.ext[N_P5], P6 = P.ext[N_P6], K = P.ext[N_K];
    for (int e = 0; e < P.nentry; ++e) {
        bool ok;
        if (FAM == FAM_D1) {
            const int da[4] = {H3, H2, P6, K};
            const int db[4] = {K, P4, P5, H1}, bb[4] = {TmaGeo::KC, 1, 1, 16};
            ok = encode_d1_a16(&M.a[e], P.opB[e], da) && encode_4d(&M.b[e], P.opA[e], db, bb, TmaGeo::KC == 16);
        } else {
            const int da[4] = {K, P4, H1, H2}, ba[4] = {TmaGeo::KC, 1, 16, 16};
            const int db[4] = {K, H3, P6, P5}, bb[4] = {TmaGeo::KC, 16, 1, 1};
            ok = encode_4d(&M.a[e], P.opA[e], da, ba, TmaGeo::KC == 16) &&
                 encode_4d(&M.b[e], P.opB[e], db, bb, TmaGeo::KC == 16);
        }
        if (!ok) return 1;
    }
    const int64_t units = (int64_t)P.ncube[0] * P.ncube[1] * P.ncube[2] * P.qe[3] * P.qe[4] * P.qe[5];
    if (units == 0) return P.ews ? run_check_finalize(0, P.ews - 8, s) : BC_OK;
    auto go = [&](auto kern, size_t smem, int* occ) {
        if (*occ == 0) {
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, TmaGeo::NT, smem);
            if (*occ < 1) *occ = 1;
        }
        const int64_t cap = (int64_t)num_sms() * *occ;
        int grid = (int)(units < cap ? units : cap);
        if (P.ews && grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
        kern<<<grid, TmaGeo::NT, smem, s>>>(P, M, (int)units);
        const int st = launch_status();
        if (st || !P.ews) return st;
        return run_check_finalize(grid, P.ews - 8, s);  // ews = ws + 8: partials -> ws[0]
    };
    const size_t smem1 = 1024 + (size_t)TmaGeo::STAGE_BYTES + TmaGeo::ACC * 8 + 2 * 8;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    static PerDevice<int> occ1_dev;
    int& occ1 = occ1_dev.get();
    if (P.nentry == 1 && BC_TC16_SINGLE_NS1 && !P.ews) return go(ccsdt_tma_kernel<FAM, 1, 3>, smem1, &occ1);
    if (P.ews) {
        static PerDevice<int> occe_dev;
        return go(ccsdt_tma_kernel<FAM, TmaGeo::NS, BC_TC16_MINB, true>, TmaGeo::SMEM, &occe_dev.get());
    }
    return go(ccsdt_tma_kernel<FAM>, TmaGeo::SMEM, &occ);
}

// ==================================================================================
// Tile-24 path (hole extents in (16, 24], d1/d2): the same warp-specialised TMA/DMMA
// scheme on a 24-cube, so a tile-24 block is 24^3 particle planes of one exact cube each
// (a 16-cube covers 24 as 16 + 8 and computes 2.37x the useful volume).  One CTA per SM:
// a (1, 25, 601)-strided fp64 cube (115 KB) + a 3-deep ring of KC = 8 stages (37.5 KiB).
// 8 consumer warps + 1 producer (at most 3 warps per SM sub-partition: 168 registers, so
// a stage's 24 fragments stay in distinct registers next to 54 accumulators); warp w owns
// the hole pairs with h2 in {3w, 3w+1, 3w+2}: 9 m-tiles x 3 n-tiles of the third hole.
// Measured on B200 (profiles/): the TMA unit costs ~70 clk per box + ~3.3 clk per box
// row, so a stage is two boxes with long rows.  Stage layouts:
//   d2 A = t2[k, p4, h1, h2]: box {8, 1, 24, 24} -> [h2][h1][k] (64 B rows, 64B swizzle);
//        m-tile mt = 9w + mi: rows 8 mt + perm64(gq), (h1, h2) = (8 (mt % 3) + perm64(gq), mt / 3)
//   d1 A = v2[h3, h2, p6, k] (k outermost in global memory): box {24, 24, 1, 8} ->
//        [k][h2][h3] (192 B rows; the 4 k of a fragment share a bank: 4-way conflicted
//        reads, measured faster than 36 conflict-free 64B-swizzled boxes);
//        m-tile (h3, h2) = (8 (mi % 3) + gq, 3w + mi / 3)
//   B    = t2[k, p4, p5, h1] (d1) | v2[k, h3, p6, p5] (d2): box -> [third][k] (64B swizzle)
// ==================================================================================
#ifndef BC_EXP_NOSEED
#define BC_EXP_NOSEED 0  // timing experiments only: skip the t3 seed/store
#endif
#ifndef BC_EXP_NOFLUSH
#define BC_EXP_NOFLUSH 0  // timing experiments only: skip the class flushes
#endif
struct Tma24Geo {
    static constexpr int BS = 24, KC = 8, NS = 3, NCW = 8, NT = (NCW + 1) * 32, NCT = NCW * 32;
    static constexpr int A_BYTES = 576 * KC * 8;          // 36 KiB
    static constexpr int B_BYTES = BS * KC * 8;           // 1.5 KiB
    static constexpr int STAGE_BYTES = A_BYTES + B_BYTES; // 38400 = 75 * 512 (64B-swizzle alignment)
    static constexpr int C1 = 25, C2 = 601;               // cube strides of q1, q2 (q0: 1)
    static constexpr int ACC = (BS - 1) * (1 + C1 + C2) + 2;  // doubles (even)
    static constexpr size_t SMEM = 1024 + (size_t)NS * STAGE_BYTES + (size_t)ACC * 8 + 2 * NS * 8;
};

template <int FAM>
__global__ void __launch_bounds__(Tma24Geo::NT, 1) ccsdt_tma24_kernel(const __grid_constant__ CcsdtParams P,
                                                                      const __grid_constant__ TmaMaps M, int units) {
    using TG = Tma24Geo;
    constexpr int BS = TG::BS, KC = TG::KC, NS = TG::NS, NCT = TG::NCT;
    extern __shared__ unsigned char smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023) & ~1023u;
    unsigned char* gbase = smem_raw + (base - raw);
    double* acc_s = reinterpret_cast<double*>(gbase + NS * TG::STAGE_BYTES);
    const uint32_t bar_full = base + NS * TG::STAGE_BYTES + TG::ACC * 8;
    const uint32_t bar_empty = bar_full + NS * 8;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) {
            mbar_init(bar_full + 8 * i, 1);
            mbar_init(bar_empty + 8 * i, TG::NCW);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();

    const int ncubes = P.ncube[0] * P.ncube[1] * P.ncube[2];
    const int K = P.ext[N_K];
    const int nchunk = (K + KC - 1) / KC;
    const int nstage = P.nentry * nchunk;
    auto decode = [&](int u, int* o, int* len, int* qv) {
        const int cube = u % ncubes, plane = u / ncubes;
        o[0] = (cube % P.ncube[0]) * BS;
        o[1] = ((cube / P.ncube[0]) % P.ncube[1]) * BS;
        o[2] = (cube / (P.ncube[0] * P.ncube[1])) * BS;
        for (int q = 0; q < 3; ++q) len[q] = min(BS, P.qe[q] - o[q]);
        qv[0] = plane % P.qe[3];
        qv[1] = (plane / P.qe[3]) % P.qe[4];
        qv[2] = plane / (P.qe[3] * P.qe[4]);
    };

    if (warp == TG::NCW) {
        // ================================ producer: lane 0 arms the stage, lanes 0/1 issue A/B
        int g = 0;
        for (int u = blockIdx.x; u < units; u += gridDim.x) {
            int o[3], len[3], qv[3];
            decode(u, o, len, qv);
            for (int st = 0; st < nstage; ++st, ++g) {
                const int slot = g % NS;
                const uint32_t full = bar_full + 8 * slot;
                if (lane == 0) {
                    mbar_wait(bar_empty + 8 * slot, ((g / NS) & 1) ^ 1);
                    mbar_expect_tx(full, TG::STAGE_BYTES);
                }
                __syncwarp();
                const int e = st / nchunk, k0 = (st - e * nchunk) * KC;
                const int c = P.ecls[e];
                const int O1 = o[P.hpos[c][0]], O2 = o[P.hpos[c][1]], O3 = o[P.hpos[c][2]];
                auto pick = [&](int pos) { return pos == 3 ? qv[0] : (pos == 4 ? qv[1] : qv[2]); };
                const int p4 = pick(P.ppos[e][0]), p5 = pick(P.ppos[e][1]), p6 = pick(P.ppos[e][2]);
                const uint32_t A = base + slot * TG::STAGE_BYTES;
                const uint32_t B = A + TG::A_BYTES;
                if constexpr (FAM == FAM_D1) {
                    if (lane == 0) tma_load_4d(A, &M.a[e], O3, O2, p6, k0, full);
                    if (lane == 1) tma_load_4d(B, &M.b[e], k0, p4, p5, O1, full);
                } else {
                    if (lane == 0) tma_load_4d(A, &M.a[e], k0, p4, O1, O2, full);
                    if (lane == 1) tma_load_4d(B, &M.b[e], k0, O3, p6, p5, full);
                }
            }
        }
        return;
    }

    // ==================================== consumers (warps 0..7)
    const int gq = lane >> 2, tq = lane & 3;
    const int tid = threadIdx.x;  // < NCT
    const int Q0 = P.qe[0], Q1 = P.qe[1];
    // full 24-cubes of a block whose hole extents are 24: the unit's t3 values are one
    // contiguous run, and thread t owns q0 = t % 24 (NCT = 256: q0 advances by 16 per copy)
    const bool dense = (P.qe[0] == BS && P.qe[1] == BS && P.qe[2] == BS);
    int g = 0;
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
        int o[3], len[3], qv[3];
        decode(u, o, len, qv);
        const int64_t pbase = (int64_t)P.qe[0] * P.qe[1] * P.qe[2] *
                              (qv[0] + (int64_t)P.qe[3] * (qv[1] + (int64_t)P.qe[4] * qv[2]));
        const int nvol = len[0] * len[1] * len[2];
        // Dense blocks: thread t owns cube positions i = t + NCT j in every unit, so the
        // previous unit's store and this unit's seed (issued together at the end of the
        // previous unit, below) need no barrier between them; only the CTA's first unit
        // seeds here.  Ragged cubes: barrier, then seed.
        if (BC_EXP_NOSEED) {
        } else if (dense) {
            if (u == (int)blockIdx.x) {
                const double* src = P.t3 + pbase;
#pragma unroll 6
                for (int i = tid; i < BS * BS * BS; i += NCT) {
                    const int r = i / BS, q0 = i - r * BS;  // constant divisor: multiply-shift
                    const int q2 = r / BS, q1 = r - q2 * BS;
                    cp_async_8(acc_s + q0 + TG::C1 * q1 + TG::C2 * q2, src + i);
                }
            }
        } else {
            named_bar_sync(1, NCT);  // the previous unit's store from the cube is complete
            for (int i = tid; i < nvol; i += NCT) {
                const int q0 = i % len[0], r = i / len[0];
                const int q1 = r % len[1], q2 = r / len[1];
                cp_async_8(acc_s + q0 + TG::C1 * q1 + TG::C2 * q2,
                           P.t3 + pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)Q1 * (o[2] + q2)));
            }
        }
        cp_async_commit();
        bool seeded = false;

        double c[9][3][2];
#pragma unroll
        for (int mi = 0; mi < 9; ++mi)
#pragma unroll
            for (int ni = 0; ni < 3; ++ni) c[mi][ni][0] = c[mi][ni][1] = 0.0;

        int e = 0, kc_i = 0, cls_stages = 0;
        uint32_t smask = P.smask[0];
        bool class_end = (P.nentry == 1) || (P.ecls[1] != P.ecls[0]);
        for (int st = 0; st < nstage; ++st, ++g) {
            ++cls_stages;
            const int slot = g % NS;
            mbar_wait(bar_full + 8 * slot, (g / NS) & 1);
            const unsigned char* A = gbase + slot * TG::STAGE_BYTES;
            const unsigned char* B = A + TG::A_BYTES;
            double bf[KC / 4][3], af[KC / 4][9];
            // one base address per k-step; the m-/n-tiles are immediate offsets (an 8-row
            // step of a 64B-swizzled operand is 512 B and leaves the XOR pattern unchanged)
#pragma unroll
            for (int ks = 0; ks < KC / 4; ++ks) {
                const unsigned char* Bk = B + swz64(perm64(gq), 4 * ks + tq);
                const unsigned char* Ak = (FAM == FAM_D1) ? A + ((4 * ks + tq) * 576 + 72 * warp + gq) * 8
                                                          : A + 9 * warp * 512 + swz64(perm64(gq), 4 * ks + tq);
#pragma unroll
                for (int ni = 0; ni < 3; ++ni) bf[ks][ni] = lds64(Bk + ni * 512);
#pragma unroll
                for (int mi = 0; mi < 9; ++mi)
                    af[ks][mi] = lds64(Ak + ((FAM == FAM_D1) ? ((mi / 3) * 24 + 8 * (mi % 3)) * 8 : mi * 512));
            }
#pragma unroll
            for (int ks = 0; ks < KC / 4; ++ks)
#pragma unroll
                for (int ni = 0; ni < 3; ++ni) bf[ks][ni] = flip_sign(bf[ks][ni], smask);
#pragma unroll
            for (int ks = 0; ks < KC / 4; ++ks)
#pragma unroll
                for (int mi = 0; mi < 9; ++mi)
#pragma unroll
                    for (int ni = 0; ni < 3; ++ni) dmma_8x8x4(c[mi][ni][0], c[mi][ni][1], af[ks][mi], bf[ks][ni]);
            release_slot(bar_empty + 8 * slot, lane);
            const bool last_chunk = (++kc_i == nchunk);
            const int e_cur = e;
            if (last_chunk) {
                kc_i = 0;
                ++e;
            }
            if (last_chunk && class_end) {
                // CTA-wide barrier before a flush: always before the first (the seed copies of
                // all threads have landed); before later ones only when the class that just
                // ends here spans <= NS stages.  Otherwise no warp can reach this flush while
                // another is still flushing the previous class: the producer refills a slot
                // only after all consumers released it, so the fastest warp is at most NS
                // stages ahead of the slowest.
                const bool need_bar = BC_FLUSH_ALWAYS_BAR || !seeded || cls_stages <= NS;
                if (!seeded) cp_async_wait_n<0>();
                seeded = true;
                if (need_bar) named_bar_sync(1, NCT);
                cls_stages = 0;
                if (BC_EXP_NOFLUSH) {
#pragma unroll
                    for (int mi = 0; mi < 9; ++mi)
#pragma unroll
                        for (int ni = 0; ni < 3; ++ni) if (c[mi][ni][0] == 1.2345) acc_s[mi] = c[mi][ni][1];
                } else {
                const int* hp = P.hpos[P.ecls[e_cur]];
                const int s1 = hp[0] == 0 ? 1 : (hp[0] == 1 ? TG::C1 : TG::C2);
                const int s2 = hp[1] == 0 ? 1 : (hp[1] == 1 ? TG::C1 : TG::C2);
                const int s3 = hp[2] == 0 ? 1 : (hp[2] == 1 ? TG::C1 : TG::C2);
                const int slo = (FAM == FAM_D1) ? s3 : s1;  // lo = h3 (d1) | h1 (d2)
                const int sth = (FAM == FAM_D1) ? s1 : s3;  // third = h1 (d1) | h3 (d2)
#pragma unroll
                for (int mi = 0; mi < 9; ++mi) {
                    const int h2 = 3 * warp + mi / 3;
                    const int lo = 8 * (mi % 3) + ((FAM == FAM_D1) ? gq : perm64(gq));
                    double* row = acc_s + lo * slo + h2 * s2;
                    double old[3][2];  // reads first (positions are distinct; see tma_flush_class)
#pragma unroll
                    for (int ni = 0; ni < 3; ++ni)
#pragma unroll
                        for (int j = 0; j < 2; ++j) old[ni][j] = row[(8 * ni + perm64(2 * tq + j)) * sth];
#pragma unroll
                    for (int ni = 0; ni < 3; ++ni)
#pragma unroll
                        for (int j = 0; j < 2; ++j) {
                            row[(8 * ni + perm64(2 * tq + j)) * sth] = old[ni][j] + c[mi][ni][j];
                            c[mi][ni][j] = 0.0;
                        }
                }
                }
            }
            if (last_chunk && e < P.nentry) {
                smask = P.smask[e];
                class_end = (e + 1 == P.nentry) || (P.ecls[e + 1] != P.ecls[e]);
            }
        }
        if (!seeded) cp_async_wait_n<0>();
        named_bar_sync(1, NCT);  // all flushes into this cube are done
        if (BC_EXP_NOSEED) {
        } else if (dense) {
            // store this unit and seed the CTA's next unit position by position (same owner)
            double* dst = P.t3 + pbase;
            const int un = u + gridDim.x;
            const double* src = P.t3 + (int64_t)BS * BS * BS * (un < units ? un : u);
            const bool next = un < units;
#pragma unroll 6
            for (int i = tid; i < BS * BS * BS; i += NCT) {
                const int r = i / BS, q0 = i - r * BS;
                const int q2 = r / BS, q1 = r - q2 * BS;
                double* x = acc_s + q0 + TG::C1 * q1 + TG::C2 * q2;
                dst[i] = *x;
                if (next) cp_async_8_after_read(x, src + i);
            }
            cp_async_commit();
        } else {
            for (int i = tid; i < nvol; i += NCT) {
                const int q0 = i % len[0], r = i / len[0];
                const int q1 = r % len[1], q2 = r / len[1];
                P.t3[pbase + (o[0] + q0) + (int64_t)Q0 * ((o[1] + q1) + (int64_t)Q1 * (o[2] + q2))] =
                    acc_s[q0 + TG::C1 * q1 + TG::C2 * q2];
            }
        }
    }
    cp_async_wait_all();
}


// returns 1 when the TMA path is unavailable (caller falls back)
template <int FAM>
static int launch_ccsdt_tma24(const CcsdtParams& P, cudaStream_t s) {
    TmaMaps M;
    memset(&M, 0, sizeof(M));
    const int H1 = P.ext[N_H1], H2 = P.ext[N_H2], H3 = P.ext[N_H3];
    const int P4 = P.ext[N_P4], P5 = P.ext[N_P5], P6 = P.ext[N_P6], K = P.ext[N_K];
    constexpr int KC = Tma24Geo::KC;
    for (int e = 0; e < P.nentry; ++e) {
        bool ok;
        if (FAM == FAM_D1) {
            const int da[4] = {H3, H2, P6, K}, ba[4] = {24, 24, 1, KC};
            const int db[4] = {K, P4, P5, H1}, bb[4] = {KC, 1, 1, 24};
            ok = encode_4d_sw(&M.a[e], P.opB[e], da, ba, CU_TENSOR_MAP_SWIZZLE_NONE) &&
                 encode_4d_sw(&M.b[e], P.opA[e], db, bb, CU_TENSOR_MAP_SWIZZLE_64B);
        } else {
            const int da[4] = {K, P4, H1, H2}, ba[4] = {KC, 1, 24, 24};
            const int db[4] = {K, H3, P6, P5}, bb[4] = {KC, 24, 1, 1};
            ok = encode_4d_sw(&M.a[e], P.opA[e], da, ba, CU_TENSOR_MAP_SWIZZLE_64B) &&
                 encode_4d_sw(&M.b[e], P.opB[e], db, bb, CU_TENSOR_MAP_SWIZZLE_64B);
        }
        if (!ok) return 1;
    }
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    if (occ == 0) {
        cudaFuncSetAttribute(ccsdt_tma24_kernel<FAM>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Tma24Geo::SMEM);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ccsdt_tma24_kernel<FAM>, Tma24Geo::NT, Tma24Geo::SMEM);
        if (occ < 1) occ = 1;
    }
    const int64_t units = (int64_t)P.ncube[0] * P.ncube[1] * P.ncube[2] * P.qe[3] * P.qe[4] * P.qe[5];
    if (units == 0) return BC_OK;
    const int64_t cap = (int64_t)num_sms() * occ;
    const int grid = (int)(units < cap ? units : cap);
    ccsdt_tma24_kernel<FAM><<<grid, Tma24Geo::NT, Tma24Geo::SMEM, s>>>(P, M, (int)units);
    return launch_status();
}

// ==================================================================================
// f4: all 27 triples variants of one tile block — d1 and d2 (18 entries)
// on the tensor cores through the same TMA ring, s1 as rank-1 updates of the cube — into
// a shared-memory-resident t3 that never touches HBM, followed by the energy epilogue
// E += t3^2 / (eh3 + eh2 + eh1 - ep6 - ep5 - ep4) over the canonical (h3,h2,h1,p6,p5,p4)
// positions (the check of R18, here the consumer of t3).  One partial per CTA in
// ws[8 + blockIdx.x], fixed-order finalize.  Equal hole extents and equal particle
// extents (the tile case) so all variants share one t3 geometry.
// ==================================================================================
constexpr int TRIP_MAXE = 18;
struct TripParams {
    int nentry;
    int efam[TRIP_MAXE], ecls[TRIP_MAXE];
    uint32_t smask[TRIP_MAXE];
    int ppos[TRIP_MAXE][3];
    int hpos[6][3];
    int ns1;
    const double* s1t1[9];
    const double* s1v2[9];
    double s1sign[9];
    int s1hpos[9][3], s1ppos[9][3];
    int ext[7], qe[6], ncube[3];
    const double* eps_h;
    const double* eps_p;
    double* ws;
};
struct TripMaps {
    CUtensorMap a[TRIP_MAXE];
    CUtensorMap b[TRIP_MAXE];
};

#ifndef BC_F4_STORE_FIRST
#define BC_F4_STORE_FIRST 1  // f4 16-cube: the first class stores into the cube (no zeroing pass)
#endif
#ifndef BC_F4_MINB
#define BC_F4_MINB 2  // CTAs per SM of the 16-cube f4 kernel (1: ptxas took 130 registers)
#endif
__global__ void __launch_bounds__(TmaGeo::NT, BC_F4_MINB) ccsdt_triples_energy_kernel(const __grid_constant__ TripParams P,
                                                                          const __grid_constant__ TripMaps M,
                                                                          int units) {
    using TG = TmaGeo;
    constexpr int BS = TG::BS, KC = TG::KC, NS = TG::NS, CST = TG::CST;
    extern __shared__ unsigned char smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023) & ~1023u;
    unsigned char* gbase = smem_raw + (base - raw);
    double* acc_s = reinterpret_cast<double*>(gbase + NS * TG::STAGE_BYTES);
    const uint32_t bar_full = base + NS * TG::STAGE_BYTES + TG::ACC * 8;
    const uint32_t bar_empty = bar_full + NS * 8;
    __shared__ double red[8];
    __shared__ __align__(16) double s1v[2][256], s1t[2][16];  // s1 slices, double-buffered
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) {
            mbar_init(bar_full + 8 * i, 1);
            mbar_init(bar_empty + 8 * i, TG::NCW);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();
    const int ncubes = P.ncube[0] * P.ncube[1] * P.ncube[2];
    const int K = P.ext[N_K];
    const int nchunk = (K + KC - 1) / KC;
    const int nstage = P.nentry * nchunk;
    auto decode = [&](int u, int* o, int* len, int* qv) {
        const int cube = u % ncubes, plane = u / ncubes;
        o[0] = (cube % P.ncube[0]) * BS;
        o[1] = ((cube / P.ncube[0]) % P.ncube[1]) * BS;
        o[2] = (cube / (P.ncube[0] * P.ncube[1])) * BS;
        for (int q = 0; q < 3; ++q) len[q] = min(BS, P.qe[q] - o[q]);
        qv[0] = plane % P.qe[3];
        qv[1] = (plane / P.qe[3]) % P.qe[4];
        qv[2] = plane / (P.qe[3] * P.qe[4]);
    };
    auto pick = [](const int* qv, int pos) { return pos == 3 ? qv[0] : (pos == 4 ? qv[1] : qv[2]); };

    if (warp == TG::NCW) {
        int g = 0;
        for (int u = blockIdx.x; u < units; u += gridDim.x) {
            int o[3], len[3], qv[3];
            decode(u, o, len, qv);
            for (int st = 0; st < nstage; ++st, ++g) {
                const int slot = g % NS;
                const uint32_t full = bar_full + 8 * slot;
                if (lane == 0) {
                    mbar_wait(bar_empty + 8 * slot, ((g / NS) & 1) ^ 1);
                    mbar_expect_tx(full, TG::STAGE_BYTES);
                }
                __syncwarp();
                const int e = st / nchunk, k0 = (st - e * nchunk) * KC;
                const int c = P.ecls[e];
                const int O1 = o[P.hpos[c][0]], O2 = o[P.hpos[c][1]], O3 = o[P.hpos[c][2]];
                const int p4 = pick(qv, P.ppos[e][0]), p5 = pick(qv, P.ppos[e][1]), p6 = pick(qv, P.ppos[e][2]);
                const uint32_t A = base + slot * TG::STAGE_BYTES;
                if (P.efam[e] == FAM_D1)
                    tma_issue_stage<FAM_D1>(&M.a[e], &M.b[e], A, A + TG::A_BYTES, full, lane, O1, O2, O3, p4, p5, p6, k0);
                else
                    tma_issue_stage<FAM_D2>(&M.a[e], &M.b[e], A, A + TG::A_BYTES, full, lane, O1, O2, O3, p4, p5, p6, k0);
            }
        }
        return;
    }

    const int gq = lane >> 2, tq = lane & 3;
    const int tid = threadIdx.x;
    const int H1 = P.ext[N_H1], H2 = P.ext[N_H2], H3 = P.ext[N_H3];
    const int P4 = P.ext[N_P4], P5 = P.ext[N_P5], P6 = P.ext[N_P6];
    const double* eh1 = P.eps_h;
    const double* eh2 = P.eps_h + H1;
    const double* eh3 = P.eps_h + H1 + H2;
    const double* ep4 = P.eps_p;
    const double* ep5 = P.eps_p + P4;
    const double* ep6 = P.eps_p + P4 + P5;
    double energy = 0.0;
    int g = 0;
    const int q0 = tid & 15, q1 = tid >> 4;
    // s1 slice of variant v for the unit (o, qv) into buffer b: s1v[b][i2*16 + i3] =
    // v2[O3+i3, O2+i2, p6, p5], s1t[b][i1] = t1[p4, O1+i1] (zero-filled outside the block;
    // the sign is applied at use)
    auto s1_issue = [&](int v, int b, const int* o, const int* qv) {
        const int O1 = o[P.s1hpos[v][0]], O2 = o[P.s1hpos[v][1]], O3 = o[P.s1hpos[v][2]];
        const int p4 = pick(qv, P.s1ppos[v][0]), p5 = pick(qv, P.s1ppos[v][1]), p6 = pick(qv, P.s1ppos[v][2]);
        const int i3 = tid & 15, i2 = tid >> 4;
        const bool ok = O3 + i3 < H3 && O2 + i2 < H2;
        cp_async_8_zfill(&s1v[b][tid],
                         P.s1v2[v] + (ok ? (O3 + i3) + (int64_t)H3 * ((O2 + i2) + (int64_t)H2 * (p6 + (int64_t)P6 * p5)) : 0),
                         ok);
        if (tid < 16) {
            const bool okt = O1 + tid < H1;
            cp_async_8_zfill(&s1t[b][tid], P.s1t1[v] + (okt ? p4 + (int64_t)P4 * (O1 + tid) : 0), okt);
        }
    };
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
        int o[3], len[3], qv[3];
        decode(u, o, len, qv);
        named_bar_sync(1, 256);  // previous unit's epilogue done with the cube and the s1 buffers
        // the first two s1 slices land while the d1/d2 stages run
        for (int v = 0; v < 2; ++v) {
            if (v < P.ns1) s1_issue(v, v, o, qv);
            cp_async_commit();
        }
        if (nstage == 0 || !BC_F4_STORE_FIRST) {  // no d1/d2 class (s1 only): a zero cube
            for (int i = tid; i < BS * CST * CST; i += 256) acc_s[i] = 0.0;
            named_bar_sync(1, 256);
        }
        bool first_flush = BC_F4_STORE_FIRST;
        double c[4][2][2];
#pragma unroll
        for (int mi = 0; mi < 4; ++mi)
#pragma unroll
            for (int ni = 0; ni < 2; ++ni) c[mi][ni][0] = c[mi][ni][1] = 0.0;
        int cls_stages = 0;
        for (int st = 0; st < nstage; ++st, ++g) {
            ++cls_stages;
            const int slot = g % NS;
            mbar_wait(bar_full + 8 * slot, (g / NS) & 1);
            const unsigned char* A = gbase + slot * TG::STAGE_BYTES;
            const unsigned char* B = A + TG::A_BYTES;
            const int e = st / nchunk, k0 = (st - e * nchunk) * KC;
            const bool d1 = P.efam[e] == FAM_D1;
            if (d1) tma_consume_stage<FAM_D1>(A, B, P.smask[e], c, warp, gq, tq);
            else tma_consume_stage<FAM_D2>(A, B, P.smask[e], c, warp, gq, tq);
            release_slot(bar_empty + 8 * slot, lane);
            if (k0 + KC >= K && (e + 1 == P.nentry || P.ecls[e + 1] != P.ecls[e])) {
                // no two classes flush concurrently: the cube was zeroed behind a barrier, and
                // a class spanning more than NS stages cannot overlap the previous class's
                // flush (the producer refills a slot only after every consumer released it,
                // so the fastest warp is at most NS stages ahead; as in ccsdt_tma_kernel)
                if (BC_FLUSH_ALWAYS_BAR || cls_stages <= NS) named_bar_sync(1, 256);
                cls_stages = 0;
                const int* hp = P.hpos[P.ecls[e]];
                if (first_flush) {  // the unit-start barrier ordered the previous unit's reads
                    if (d1) tma_flush_class<FAM_D1, true>(acc_s, c, hp, warp, gq, tq);
                    else tma_flush_class<FAM_D2, true>(acc_s, c, hp, warp, gq, tq);
                    first_flush = false;
                } else {
                    if (d1) tma_flush_class<FAM_D1>(acc_s, c, hp, warp, gq, tq);
                    else tma_flush_class<FAM_D2>(acc_s, c, hp, warp, gq, tq);
                }
            }
        }
        // s1 rank-1 updates t3 += s t1[p4,h1] v2[h3,h2,p6,p5], accumulated in registers for
        // this thread's positions (q0, q1, *) and folded into the energy epilogue (t3 is
        // never stored, so the cube is not updated)
        double s1acc[BS];
#pragma unroll
        for (int q2 = 0; q2 < BS; ++q2) s1acc[q2] = 0.0;
        for (int v = 0; v < P.ns1; ++v) {
            const int b = v & 1;
            cp_async_wait_n<1>();    // this thread's copies of slice v landed (v+1 may be in flight)
            named_bar_sync(1, 256);  // everyone's copies of slice v landed
            const int hp1 = P.s1hpos[v][0], hp2 = P.s1hpos[v][1], hp3 = P.s1hpos[v][2];
            const double sgn = P.s1sign[v];
            const double* sv = s1v[b];
            const double* stt = s1t[b];
#pragma unroll
            for (int q2 = 0; q2 < BS; ++q2) {
                const int i1 = hp1 == 0 ? q0 : (hp1 == 1 ? q1 : q2);
                const int i2 = hp2 == 0 ? q0 : (hp2 == 1 ? q1 : q2);
                const int i3 = hp3 == 0 ? q0 : (hp3 == 1 ? q1 : q2);
                s1acc[q2] = fma(sgn * stt[i1], sv[i2 * 16 + i3], s1acc[q2]);
            }
            named_bar_sync(1, 256);  // slice v consumed: its buffer takes slice v+2
            if (v + 2 < P.ns1) s1_issue(v + 2, b, o, qv);
            cp_async_commit();
        }
        cp_async_wait_n<0>();
        named_bar_sync(1, 256);  // all d1/d2 classes flushed
        // energy of every cube position this thread owns (canonical (h3,h2,h1,p6,p5,p4))
#pragma unroll
        for (int q2 = 0; q2 < BS; ++q2) {
            if (q0 >= len[0] || q1 >= len[1] || q2 >= len[2]) continue;
            const double t = acc_s[q0 + CST * (q1 + CST * q2)] + s1acc[q2];
            const double den = ((((eh3[o[0] + q0] + eh2[o[1] + q1]) + eh1[o[2] + q2]) - ep6[qv[0]]) - ep5[qv[1]]) -
                               ep4[qv[2]];
            energy += t * t / den;
        }
    }
    // consumer-only block reduction (the producer warp has left)
    for (int off = 16; off > 0; off >>= 1) energy += __shfl_xor_sync(0xffffffffu, energy, off);
    if (lane == 0) red[warp] = energy;
    named_bar_sync(1, 256);
    if (tid == 0) {
        double sum = 0.0;
        for (int w = 0; w < TG::NCW; ++w) sum += red[w];
        P.ws[8 + blockIdx.x] = sum;
    }
}

// ---- f4 on exact 24-cubes (hole extents 24, the tile-24 block): the tile-24 DMMA scheme of
// ccsdt_tma24_kernel with d1 and d2 entries mixed in one TMA ring (2 stages, so that the
// 24-cube, the ring and the double-buffered s1 slices fit one SM), the cube zeroed per unit
// instead of seeded, s1 applied to the cube, and the energy epilogue instead of the store.
// (The 16-cube f4 kernel covers 24 as 16 + 8: 2.37x the useful volume.)
struct Trip24Geo {
    static constexpr int BS = 24, KC = 8, NS = 2, NCW = 8, NT = (NCW + 1) * 32, NCT = NCW * 32;
    static constexpr int STAGE_BYTES = Tma24Geo::STAGE_BYTES, A_BYTES = Tma24Geo::A_BYTES;
    static constexpr int C1 = Tma24Geo::C1, C2 = Tma24Geo::C2, ACC = Tma24Geo::ACC;
    static constexpr size_t SMEM = 1024 + (size_t)NS * STAGE_BYTES + (size_t)ACC * 8 + 2 * NS * 8;
};

// consumer: one KC = 8 stage of the 24-cube DMMA for family FE (see ccsdt_tma24_kernel)
template <int FE>
__device__ __forceinline__ void t24_consume(const unsigned char* A, const unsigned char* B, uint32_t smask,
                                            double (&c)[9][3][2], int warp, int gq, int tq) {
    constexpr int KC = Trip24Geo::KC;
    double bf[KC / 4][3], af[KC / 4][9];
#pragma unroll
    for (int ks = 0; ks < KC / 4; ++ks) {
        const unsigned char* Bk = B + swz64(perm64(gq), 4 * ks + tq);
        const unsigned char* Ak = (FE == FAM_D1) ? A + ((4 * ks + tq) * 576 + 72 * warp + gq) * 8
                                                 : A + 9 * warp * 512 + swz64(perm64(gq), 4 * ks + tq);
#pragma unroll
        for (int ni = 0; ni < 3; ++ni) bf[ks][ni] = lds64(Bk + ni * 512);
#pragma unroll
        for (int mi = 0; mi < 9; ++mi)
            af[ks][mi] = lds64(Ak + ((FE == FAM_D1) ? ((mi / 3) * 24 + 8 * (mi % 3)) * 8 : mi * 512));
    }
#pragma unroll
    for (int ks = 0; ks < KC / 4; ++ks)
#pragma unroll
        for (int ni = 0; ni < 3; ++ni) bf[ks][ni] = flip_sign(bf[ks][ni], smask);
#pragma unroll
    for (int ks = 0; ks < KC / 4; ++ks)
#pragma unroll
        for (int mi = 0; mi < 9; ++mi)
#pragma unroll
            for (int ni = 0; ni < 3; ++ni) dmma_8x8x4(c[mi][ni][0], c[mi][ni][1], af[ks][mi], bf[ks][ni]);
}

// consumer: add a class's register tile into the 24-cube at its permuted positions, clear it
template <int FE>
__device__ __forceinline__ void t24_flush(double* acc_s, double (&c)[9][3][2], const int* hp, int warp, int gq,
                                          int tq) {
    constexpr int C1 = Trip24Geo::C1, C2 = Trip24Geo::C2;
    const int s1 = hp[0] == 0 ? 1 : (hp[0] == 1 ? C1 : C2);
    const int s2 = hp[1] == 0 ? 1 : (hp[1] == 1 ? C1 : C2);
    const int s3 = hp[2] == 0 ? 1 : (hp[2] == 1 ? C1 : C2);
    const int slo = (FE == FAM_D1) ? s3 : s1;
    const int sth = (FE == FAM_D1) ? s1 : s3;
#pragma unroll
    for (int mi = 0; mi < 9; ++mi) {
        const int h2 = 3 * warp + mi / 3;
        const int lo = 8 * (mi % 3) + ((FE == FAM_D1) ? gq : perm64(gq));
        double* row = acc_s + lo * slo + h2 * s2;
        double old[3][2];  // reads first (positions are distinct; see tma_flush_class)
#pragma unroll
        for (int ni = 0; ni < 3; ++ni)
#pragma unroll
            for (int j = 0; j < 2; ++j) old[ni][j] = row[(8 * ni + perm64(2 * tq + j)) * sth];
#pragma unroll
        for (int ni = 0; ni < 3; ++ni)
#pragma unroll
            for (int j = 0; j < 2; ++j) {
                row[(8 * ni + perm64(2 * tq + j)) * sth] = old[ni][j] + c[mi][ni][j];
                c[mi][ni][j] = 0.0;
            }
    }
}

__global__ void __launch_bounds__(Trip24Geo::NT, 1) ccsdt_triples24_kernel(const __grid_constant__ TripParams P,
                                                                          const __grid_constant__ TripMaps M,
                                                                          int units) {
    using TG = Trip24Geo;
    constexpr int BS = TG::BS, KC = TG::KC, NS = TG::NS, NCT = TG::NCT, C1 = TG::C1, C2 = TG::C2;
    extern __shared__ unsigned char smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023) & ~1023u;
    unsigned char* gbase = smem_raw + (base - raw);
    double* acc_s = reinterpret_cast<double*>(gbase + NS * TG::STAGE_BYTES);
    const uint32_t bar_full = base + NS * TG::STAGE_BYTES + TG::ACC * 8;
    const uint32_t bar_empty = bar_full + NS * 8;
    __shared__ double red[8];
    __shared__ __align__(16) double s1v[2][576], s1t[2][24];  // s1 slices, double-buffered
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) {
            mbar_init(bar_full + 8 * i, 1);
            mbar_init(bar_empty + 8 * i, TG::NCW);
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();
    const int K = P.ext[N_K];
    const int nchunk = (K + KC - 1) / KC;
    const int nstage = P.nentry * nchunk;
    auto decode = [&](int plane, int* qv) {  // one exact cube per particle plane
        qv[0] = plane % P.qe[3];
        qv[1] = (plane / P.qe[3]) % P.qe[4];
        qv[2] = plane / (P.qe[3] * P.qe[4]);
    };
    auto pick = [](const int* qv, int pos) { return pos == 3 ? qv[0] : (pos == 4 ? qv[1] : qv[2]); };

    if (warp == TG::NCW) {
        int g = 0;
        for (int u = blockIdx.x; u < units; u += gridDim.x) {
            int qv[3];
            decode(u, qv);
            for (int st = 0; st < nstage; ++st, ++g) {
                const int slot = g % NS;
                const uint32_t full = bar_full + 8 * slot;
                if (lane == 0) {
                    mbar_wait(bar_empty + 8 * slot, ((g / NS) & 1) ^ 1);
                    mbar_expect_tx(full, TG::STAGE_BYTES);
                }
                __syncwarp();
                const int e = st / nchunk, k0 = (st - e * nchunk) * KC;
                const int p4 = pick(qv, P.ppos[e][0]), p5 = pick(qv, P.ppos[e][1]), p6 = pick(qv, P.ppos[e][2]);
                const uint32_t A = base + slot * TG::STAGE_BYTES;
                const uint32_t B = A + TG::A_BYTES;
                if (P.efam[e] == FAM_D1) {  // one cube: every hole offset is 0
                    if (lane == 0) tma_load_4d(A, &M.a[e], 0, 0, p6, k0, full);
                    if (lane == 1) tma_load_4d(B, &M.b[e], k0, p4, p5, 0, full);
                } else {
                    if (lane == 0) tma_load_4d(A, &M.a[e], k0, p4, 0, 0, full);
                    if (lane == 1) tma_load_4d(B, &M.b[e], k0, 0, p6, p5, full);
                }
            }
        }
        return;
    }

    // ==================================== consumers (warps 0..7)
    const int gq = lane >> 2, tq = lane & 3;
    const int tid = threadIdx.x;
    const int P4 = P.ext[N_P4], P6 = P.ext[N_P6];
    const double* eh1 = P.eps_h;
    const double* eh2 = P.eps_h + BS;
    const double* eh3 = P.eps_h + 2 * BS;
    const double* ep4 = P.eps_p;
    const double* ep5 = P.eps_p + P4;
    const double* ep6 = P.eps_p + 2 * P4;
    auto s1_issue = [&](int v, int b, const int* qv) {
        const int p4 = pick(qv, P.s1ppos[v][0]), p5 = pick(qv, P.s1ppos[v][1]), p6 = pick(qv, P.s1ppos[v][2]);
        const double* src = P.s1v2[v] + (int64_t)BS * BS * (p6 + (int64_t)P6 * p5);  // [h3 + 24 h2]
        for (int i = tid; i < 288; i += NCT) cp_async_16(&s1v[b][2 * i], src + 2 * i);
        if (tid < BS) cp_async_8(&s1t[b][tid], P.s1t1[v] + p4 + (int64_t)P4 * tid);
    };
    double energy = 0.0;
    int g = 0;
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
        int qv[3];
        decode(u, qv);
        named_bar_sync(1, NCT);  // previous unit's epilogue done with the cube and s1 buffers
        for (int v = 0; v < 2; ++v) {
            if (v < P.ns1) s1_issue(v, v, qv);
            cp_async_commit();
        }
        for (int i = tid; i < TG::ACC; i += NCT) acc_s[i] = 0.0;
        named_bar_sync(1, NCT);
        double c[9][3][2];
#pragma unroll
        for (int mi = 0; mi < 9; ++mi)
#pragma unroll
            for (int ni = 0; ni < 3; ++ni) c[mi][ni][0] = c[mi][ni][1] = 0.0;
        int e = 0, kc_i = 0, cls_stages = 0;
        for (int st = 0; st < nstage; ++st, ++g) {
            ++cls_stages;
            const int slot = g % NS;
            mbar_wait(bar_full + 8 * slot, (g / NS) & 1);
            const unsigned char* A = gbase + slot * TG::STAGE_BYTES;
            const unsigned char* B = A + TG::A_BYTES;
            const bool d1 = P.efam[e] == FAM_D1;
            if (d1) t24_consume<FAM_D1>(A, B, P.smask[e], c, warp, gq, tq);
            else t24_consume<FAM_D2>(A, B, P.smask[e], c, warp, gq, tq);
            release_slot(bar_empty + 8 * slot, lane);
            const bool last_chunk = (++kc_i == nchunk);
            const int e_cur = e;
            if (last_chunk) {
                kc_i = 0;
                ++e;
            }
            const bool class_end = last_chunk && (e == P.nentry || P.ecls[e] != P.ecls[e_cur]);
            if (class_end) {
                // as in ccsdt_tma24_kernel: a barrier only when the ending class spans <= NS
                // stages (otherwise no warp can be flushing the previous class)
                if (cls_stages <= NS) named_bar_sync(1, NCT);
                cls_stages = 0;
                if (d1) t24_flush<FAM_D1>(acc_s, c, P.hpos[P.ecls[e_cur]], warp, gq, tq);
                else t24_flush<FAM_D2>(acc_s, c, P.hpos[P.ecls[e_cur]], warp, gq, tq);
            }
        }
        // s1 rank-1 updates into the cube, one variant at a time (slices double-buffered)
        for (int v = 0; v < P.ns1; ++v) {
            const int b = v & 1;
            cp_async_wait_n<1>();
            named_bar_sync(1, NCT);  // slice v landed; all d1/d2 flushes are done
            const int hp1 = P.s1hpos[v][0], hp2 = P.s1hpos[v][1], hp3 = P.s1hpos[v][2];
            const double sgn = P.s1sign[v];
            // (q0, q1) rows of 24 q2 values: the name-to-coordinate selects are per row, the
            // q2 steps are strides
            for (int i = tid; i < BS * BS; i += NCT) {
                const int q1 = i / BS, q0 = i - q1 * BS;
                // name index = a + b q2 for each of h1, h2, h3
                const int a1 = hp1 == 0 ? q0 : (hp1 == 1 ? q1 : 0), b1 = hp1 == 2;
                const int a2 = hp2 == 0 ? q0 : (hp2 == 1 ? q1 : 0), b2 = hp2 == 2;
                const int a3 = hp3 == 0 ? q0 : (hp3 == 1 ? q1 : 0), b3 = hp3 == 2;
                const double* tp = s1t[b] + a1;
                const double* vp = s1v[b] + a2 * BS + a3;
                const int dt = b1, dv = b2 * BS + b3;
                double* xp = acc_s + q0 + C1 * q1;
#pragma unroll 8
                for (int q2 = 0; q2 < BS; ++q2) xp[C2 * q2] = fma(sgn * tp[dt * q2], vp[dv * q2], xp[C2 * q2]);
            }
            named_bar_sync(1, NCT);  // slice v consumed: its buffer takes slice v+2
            if (v + 2 < P.ns1) s1_issue(v + 2, b, qv);
            cp_async_commit();
        }
        cp_async_wait_n<0>();
        named_bar_sync(1, NCT);  // all updates of the cube are done
        // energy over the canonical (h3,h2,h1,p6,p5,p4) positions: (q0,q1,q2) = (h3,h2,h1)
        const double e6 = ep6[qv[0]], e5 = ep5[qv[1]], e4 = ep4[qv[2]];
        for (int i = tid; i < BS * BS; i += NCT) {
            const int q1 = i / BS, q0 = i - q1 * BS;
            const double h32 = eh3[q0] + eh2[q1];
            const double* xp = acc_s + q0 + C1 * q1;
#pragma unroll 4
            for (int q2 = 0; q2 < BS; ++q2) {
                const double t = xp[C2 * q2];
                const double den = (((h32 + eh1[q2]) - e6) - e5) - e4;
                energy += t * t / den;
            }
        }
    }
    for (int off = 16; off > 0; off >>= 1) energy += __shfl_xor_sync(0xffffffffu, energy, off);
    if (lane == 0) red[warp] = energy;
    named_bar_sync(1, NCT);
    if (tid == 0) {
        double sum = 0.0;
        for (int w = 0; w < TG::NCW; ++w) sum += red[w];
        P.ws[8 + blockIdx.x] = sum;
    }
}


// Host: d1/d2 entries grouped by class (d1 classes 0-2, d2 classes 3-5), s1 list.
int run_ccsdt_triples_energy(const int* ext7, const double* const* t1, const double* const* v2s1,
                             const double* const* t2d1, const double* const* v2d1, const double* const* t2d2,
                             const double* const* v2d2, const double* eps_h, const double* eps_p, double* ws,
                             cudaStream_t s) {
    TripParams P;
    memset(&P, 0, sizeof(P));
    TripMaps M;
    memset(&M, 0, sizeof(M));
    for (int q = 0; q < 7; ++q) P.ext[q] = ext7[q];
    const int H = ext7[N_H1], PP = ext7[N_P4], K = ext7[N_K];
    for (int q = 0; q < 3; ++q) P.qe[q] = H;
    for (int q = 3; q < 6; ++q) P.qe[q] = PP;
    for (int q = 0; q < 3; ++q) P.ncube[q] = (H + 15) / 16;
    // exact 24-cubes (tile 24): the 24-cube kernel (BC_NO_TRIP24: the 16-cube one)
    const bool c24 = H == 24 && K % 2 == 0;
    P.eps_h = eps_h;
    P.eps_p = eps_p;
    P.ws = ws;
    int n = 0, ncls = 0;
    const double* const* tA[2] = {t2d1, t2d2};
    const double* const* vB[2] = {v2d1, v2d2};
    for (int f = 0; f < 2; ++f) {
        const int fam = f == 0 ? FAM_D1 : FAM_D2;
        for (int cls = 0; cls < 3; ++cls) {
            bool any = false;
            for (int v = 1; v <= 9; ++v) {
                if ((v - 1) % 3 != cls || !tA[f][v - 1]) continue;
                const VariantInfo vi = variant_info(fam, v);
                if (!any) {
                    for (int q = 0; q < 3; ++q) P.hpos[ncls][vi.order[q]] = q;
                    any = true;
                }
                for (int q = 3; q < 6; ++q) P.ppos[n][vi.order[q] - 3] = q;
                P.efam[n] = fam;
                P.ecls[n] = ncls;
                P.smask[n] = vi.sign < 0 ? 0x80000000u : 0u;
                bool ok;
                if (c24) {  // the tile-24 boxes of ccsdt_tma24_kernel
                    constexpr int KC24 = Trip24Geo::KC;
                    if (fam == FAM_D1) {
                        const int da[4] = {H, H, PP, K}, ba[4] = {24, 24, 1, KC24};
                        const int db[4] = {K, PP, PP, H}, bb[4] = {KC24, 1, 1, 24};
                        ok = encode_4d_sw(&M.a[n], vB[f][v - 1], da, ba, CU_TENSOR_MAP_SWIZZLE_NONE) &&
                             encode_4d_sw(&M.b[n], tA[f][v - 1], db, bb, CU_TENSOR_MAP_SWIZZLE_64B);
                    } else {
                        const int da[4] = {K, PP, H, H}, ba[4] = {KC24, 1, 24, 24};
                        const int db[4] = {K, H, PP, PP}, bb[4] = {KC24, 24, 1, 1};
                        ok = encode_4d_sw(&M.a[n], tA[f][v - 1], da, ba, CU_TENSOR_MAP_SWIZZLE_64B) &&
                             encode_4d_sw(&M.b[n], vB[f][v - 1], db, bb, CU_TENSOR_MAP_SWIZZLE_64B);
                    }
                } else if (fam == FAM_D1) {
                    const int da[4] = {H, H, PP, K};
                    const int db[4] = {K, PP, PP, H}, bb[4] = {TmaGeo::KC, 1, 1, 16};
                    ok = encode_d1_a16(&M.a[n], vB[f][v - 1], da) &&
                         encode_4d(&M.b[n], tA[f][v - 1], db, bb, TmaGeo::KC == 16);
                } else {
                    const int da[4] = {K, PP, H, H}, ba[4] = {TmaGeo::KC, 1, 16, 16};
                    const int db[4] = {K, H, PP, PP}, bb[4] = {TmaGeo::KC, 16, 1, 1};
                    ok = encode_4d(&M.a[n], tA[f][v - 1], da, ba, TmaGeo::KC == 16) &&
                         encode_4d(&M.b[n], vB[f][v - 1], db, bb, TmaGeo::KC == 16);
                }
                if (!ok) return BC_ERR_UNSUPPORTED;
                ++n;
            }
            if (any) ++ncls;
        }
    }
    P.nentry = n;
    int ns = 0;
    for (int v = 1; v <= 9; ++v) {
        if (!t1[v - 1]) continue;
        const VariantInfo vi = variant_info(FAM_S1, v);
        for (int q = 0; q < 3; ++q) P.s1hpos[ns][vi.order[q]] = q;
        for (int q = 3; q < 6; ++q) P.s1ppos[ns][vi.order[q] - 3] = q;
        P.s1sign[ns] = vi.sign;
        P.s1t1[ns] = t1[v - 1];
        P.s1v2[ns] = v2s1[v - 1];
        ++ns;
    }
    P.ns1 = ns;
    if (c24) {
        static PerDevice<int> occ24_dev;
        int& occ24 = occ24_dev.get();
        if (occ24 == 0) {
            cudaFuncSetAttribute(ccsdt_triples24_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Trip24Geo::SMEM);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ24, ccsdt_triples24_kernel, Trip24Geo::NT, Trip24Geo::SMEM);
            if (occ24 < 1) occ24 = 1;
        }
        const int units24 = PP * PP * PP;
        int grid = num_sms() * occ24;
        if (grid > units24) grid = units24;
        if (grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
        ccsdt_triples24_kernel<<<grid, Trip24Geo::NT, Trip24Geo::SMEM, s>>>(P, M, units24);
        const int st = launch_status();
        if (st) return st;
        return run_check_finalize(grid, ws, s);
    }
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    if (occ == 0) {
        cudaFuncSetAttribute(ccsdt_triples_energy_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TmaGeo::SMEM);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ccsdt_triples_energy_kernel, TmaGeo::NT, TmaGeo::SMEM);
        if (occ < 1) occ = 1;
    }
    const int units = P.ncube[0] * P.ncube[1] * P.ncube[2] * PP * PP * PP;
    int grid = num_sms() * occ;
    if (grid > units) grid = units;
    if (grid > CHECK_MAX_PARTIALS) grid = CHECK_MAX_PARTIALS;
    ccsdt_triples_energy_kernel<<<grid, TmaGeo::NT, TmaGeo::SMEM, s>>>(P, M, units);
    const int st = launch_status();
    if (st) return st;
    return run_check_finalize(grid, ws, s);
}

// ==================================================================================
// s1 streaming path (single or fused variants sharing one t3 geometry).  s1 has no
// contracted index: t3[sigma_v] += s_v t1[p4,h1] v2[h3,h2,p6,p5] is a rank-1 update per
// particle plane, so the kernel is a pure t3 read-modify-write stream (AI 2 flop / 16 B per
// variant).  A CTA owns whole particle planes (the hole volume of a plane is contiguous in
// t3 for every storage order, since the holes are the three fastest positions): it stages
// the plane's per-entry factors in shared memory — Vs_e[h2][h3] = s_e v2_e[h3,h2,p6,p5]
// (row stride H3+1: conflict-free whichever hole name runs along the lanes) and
// Ts_e[h1] = t1_e[p4,h1] — then streams the plane's t3 values with all of a thread's
// loads in flight at once.  Per element and entry: 2 shared loads and one FMA; the hole
// names of an element are linear forms of its storage coordinates, one per class.
// ==================================================================================
constexpr int S1S_NT = 256, S1S_U = 4;  // threads, runs in flight per thread
#ifndef BC_S1_MINB
#define BC_S1_MINB 2  // measured: 2 CTAs/SM (128 registers) beat 1 (156), 3 (79) and 4 (64)
#endif

// RUN consecutive storage-position-0 values per thread (16-byte accesses when RUN = 4).
// Shared layout per class c (CS doubles): V_c[pair][m] (pair = h2 (H3+1) + h3) then
// T_c[h1][m], m = the entry's rank inside its class, so one address per class serves its
// (up to 3) entries through immediate offsets.
template <int RUN>
__global__ void __launch_bounds__(S1S_NT, BC_S1_MINB) ccsdt_s1_stream_kernel(const __grid_constant__ CcsdtParams P,
                                                                 int nplanes) {
    extern __shared__ __align__(16) double s1sm[];
    const int H1 = P.ext[N_H1], H2 = P.ext[N_H2], H3 = P.ext[N_H3];
    const int P4 = P.ext[N_P4], P6 = P.ext[N_P6];
    const int VS = H2 * (H3 + 1), CS = 3 * (VS + H1);
    const int BUFD = P.ncls * CS;
    const int Q0 = P.qe[0], Q1 = P.qe[1], Q2 = P.qe[2];
    const int nh = Q0 * Q1 * Q2, R0 = Q0 / RUN, nruns = nh / RUN;
    const int tid = threadIdx.x;
    int n0 = 0, n1 = 0, n2 = 0;
    for (int e = 0; e < P.nentry; ++e) {
        const int c = P.ecls[e];
        n0 += c == 0;
        n1 += c == 1;
        n2 += c == 2;
    }
    const int cb[3] = {0, n0, n0 + n1}, cnt[3] = {n0, n1, n2};
    int av[3][3], at[3][3];
#pragma unroll
    for (int c = 0; c < 3; ++c)
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            const bool ok = c < P.ncls;
            at[c][q] = (ok && P.hpos[c][0] == q) ? 1 : 0;                                            // h1
            av[c][q] = (ok && P.hpos[c][1] == q) ? H3 + 1 : ((ok && P.hpos[c][2] == q) ? 1 : 0);  // h2, h3
        }
    auto pvals = [&](int plane, int e, int& p4, int& p5, int& p6) {
        const int qv0 = plane % P.qe[3], qv1 = (plane / P.qe[3]) % P.qe[4], qv2 = plane / (P.qe[3] * P.qe[4]);
        auto pick = [&](int pos) { return pos == 3 ? qv0 : (pos == 4 ? qv1 : qv2); };
        p4 = pick(P.ppos[e][0]);
        p5 = pick(P.ppos[e][1]);
        p6 = pick(P.ppos[e][2]);
    };
    // V factors of a plane: cp.async into buffer b.  The plane's particle values are decoded
    // once; this thread's first (h2, h3) is hoisted (one element per entry when H2 H3 <= NT).
    const int vh2 = tid / (H3 > 0 ? H3 : 1), vh3 = tid - vh2 * H3;
    auto stage_v = [&](int plane, int b) {
        double* buf = s1sm + b * BUFD;
        const int qv0 = plane % P.qe[3], qv1 = (plane / P.qe[3]) % P.qe[4], qv2 = plane / (P.qe[3] * P.qe[4]);
        auto pick = [&](int pos) { return pos == 3 ? qv0 : (pos == 4 ? qv1 : qv2); };
        for (int e = 0; e < P.nentry; ++e) {
            const int p5 = pick(P.ppos[e][1]), p6 = pick(P.ppos[e][2]);
            const int c = P.ecls[e], m = e - (c == 0 ? 0 : (c == 1 ? n0 : n0 + n1));
            const double* v2 = P.opB[e] + (int64_t)H3 * H2 * (p6 + (int64_t)P6 * p5);
            double* dst = buf + c * CS + m;
            if (tid < H2 * H3) cp_async_8(dst + 3 * (vh2 * (H3 + 1) + vh3), v2 + tid);
            for (int i = tid + S1S_NT; i < H2 * H3; i += S1S_NT) {
                const int h2 = i / H3, h3 = i - h2 * H3;
                cp_async_8(dst + 3 * (h2 * (H3 + 1) + h3), v2 + i);
            }
        }
    };
    // T factors (sign folded): thread t < nentry*H1 owns one value; loaded one plane ahead
    const int te = tid / (H1 > 0 ? H1 : 1), th1 = tid - te * H1;
    const bool towner = te < P.nentry;
    const int tc = towner ? P.ecls[te] : 0;
    const int tdst = tc * CS + 3 * VS + 3 * th1 + (te - (tc == 0 ? 0 : (tc == 1 ? n0 : n0 + n1)));
    const double tsg = towner ? P.sign[te] : 0.0;
    auto load_t = [&](int plane) {
        if (!towner) return 0.0;
        int p4, p5, p6;
        pvals(plane, te, p4, p5, p6);
        return __ldg(P.opA[te] + p4 + (int64_t)P4 * th1);
    };
    const bool t_fast = P.nentry * H1 <= S1S_NT;
    auto stage_t_slow = [&](int plane, int b) {  // more T values than threads
        double* buf = s1sm + b * BUFD;
        for (int i = tid; i < P.nentry * H1; i += S1S_NT) {
            const int e = i / H1, h1 = i - e * H1;
            int p4, p5, p6;
            pvals(plane, e, p4, p5, p6);
            const int c = P.ecls[e], m = e - (c == 0 ? 0 : (c == 1 ? n0 : n0 + n1));
            buf[c * CS + 3 * VS + 3 * h1 + m] = P.sign[e] * __ldg(P.opA[e] + p4 + (int64_t)P4 * h1);
        }
    };
    // this thread's run coordinates at run index tid, and the step for += S1S_NT runs
    const int iq0 = tid % R0, iq1 = (tid / R0) % Q1, iq2 = tid / (R0 * Q1);
    const int d0 = S1S_NT % R0, d1 = (S1S_NT / R0) % Q1, d2 = S1S_NT / (R0 * Q1);

    int it = 0;
    if ((int)blockIdx.x < nplanes) {
        stage_v(blockIdx.x, 0);
        if (t_fast) {
            if (towner) s1sm[tdst] = tsg * load_t(blockIdx.x);
        } else {
            stage_t_slow(blockIdx.x, 0);
        }
    }
    cp_async_commit();
    for (int plane = blockIdx.x; plane < nplanes; plane += gridDim.x, ++it) {
        cp_async_wait_all();
        __syncthreads();  // this plane's factors are in place; the other buffer is free
        const int nxt = plane + gridDim.x;
        double tnext = 0.0;
        if (nxt < nplanes) {
            stage_v(nxt, (it + 1) & 1);
            if (t_fast) tnext = load_t(nxt);
            else stage_t_slow(nxt, (it + 1) & 1);
        }
        cp_async_commit();
        const double* buf = s1sm + (it & 1) * BUFD;
        double* t3p = P.t3 + (int64_t)nh * plane;
        int q0 = iq0, q1 = iq1, q2 = iq2;
        for (int r0 = 0; r0 < nruns; r0 += S1S_NT * S1S_U) {
            double x[S1S_U][RUN];
#pragma unroll
            for (int u = 0; u < S1S_U; ++u) {
                const int r = r0 + u * S1S_NT + tid;
                if (r < nruns) {
                    if constexpr (RUN == 4) {
                        const double2 a = __ldcs(reinterpret_cast<const double2*>(t3p) + 2 * r);
                        const double2 b = __ldcs(reinterpret_cast<const double2*>(t3p) + 2 * r + 1);
                        x[u][0] = a.x; x[u][1] = a.y; x[u][2] = b.x; x[u][3] = b.y;
                    } else {
                        x[u][0] = __ldcs(t3p + r);
                    }
                } else {
#pragma unroll
                    for (int k = 0; k < RUN; ++k) x[u][k] = 0.0;
                }
            }
            // per run and class: offsets of the V row and the T entry (this run's first element)
            int vo[S1S_U][3], to[S1S_U][3];
#pragma unroll
            for (int u = 0; u < S1S_U; ++u) {
                const int qq0 = q0 * RUN;
                const bool ok = r0 + u * S1S_NT + tid < nruns;  // past the end: read in-range, discard
#pragma unroll
                for (int c = 0; c < 3; ++c) {
                    vo[u][c] = ok ? c * CS + 3 * (qq0 * av[c][0] + q1 * av[c][1] + q2 * av[c][2]) : 0;
                    to[u][c] = ok ? c * CS + 3 * (VS + qq0 * at[c][0] + q1 * at[c][1] + q2 * at[c][2]) : 0;
                }
                q0 += d0;
                const int c0 = q0 >= R0;
                q0 -= c0 ? R0 : 0;
                q1 += d1 + c0;
                const int c1 = q1 >= Q1;
                q1 -= c1 ? Q1 : 0;
                q2 += d2 + c1;
            }
            // entries outermost: 4 runs x RUN independent accumulation chains per entry
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                if (c < P.ncls) {
                    const int dv = 3 * av[c][0], dt = 3 * at[c][0];
#pragma unroll
                    for (int m = 0; m < 3; ++m) {
                        if (m < cnt[c]) {
#pragma unroll
                            for (int u = 0; u < S1S_U; ++u)
#pragma unroll
                                for (int k = 0; k < RUN; ++k)
                                    x[u][k] = fma(buf[to[u][c] + k * dt + m], buf[vo[u][c] + k * dv + m], x[u][k]);
                        }
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < S1S_U; ++u) {
                const int r = r0 + u * S1S_NT + tid;
                if (r < nruns) {
                    if constexpr (RUN == 4) {
                        __stcs(reinterpret_cast<double2*>(t3p) + 2 * r, make_double2(x[u][0], x[u][1]));
                        __stcs(reinterpret_cast<double2*>(t3p) + 2 * r + 1, make_double2(x[u][2], x[u][3]));
                    } else {
                        __stcs(t3p + r, x[u][0]);
                    }
                }
            }
        }
        if (t_fast && towner && nxt < nplanes) s1sm[((it + 1) & 1) * BUFD + tdst] = tsg * tnext;
    }
}

// Equal hole extents H (16, 24): the same stream with every shape constant compile-time.
// Per entry e (a compile-time slot): V_e [h2][h3] (row stride H+2: conflict-free 16-byte
// reads) and T_e [h1] at fixed offsets, so every shared read is one base register plus an
// immediate.  For s1 the name at storage position 0 is h3 or h1 (h2 always follows h3), so
// along a run either V (4 contiguous values, T broadcast) or T (V broadcast) varies.
template <int H>
__global__ void __launch_bounds__(S1S_NT, 2) ccsdt_s1h_kernel(const __grid_constant__ CcsdtParams P, int nplanes) {
    constexpr int RS = H + 2, VS = H * RS, ES = VS + H, BUFD = 9 * ES;
    constexpr int NV = H * H * H, R0 = H / 4, NRUN = NV / 4;
    constexpr int NB = (NRUN + S1S_NT * S1S_U - 1) / (S1S_NT * S1S_U);  // run batches per plane
    extern __shared__ __align__(16) double s1sm[];
    const int P4 = P.ext[N_P4], P6 = P.ext[N_P6];
    const int tid = threadIdx.x;
    const int ne = P.nentry;
    // per class: V offset = qq0*av0 + q1*av1 + q2*av2, T offset = ... ; q0 is h3 (kind 0) or h1 (kind 1)
    int av[3][3], at[3][3];
    bool q0h1[3];
#pragma unroll
    for (int c = 0; c < 3; ++c) {
        const bool ok = c < P.ncls;
        q0h1[c] = ok && P.hpos[c][0] == 0;
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            at[c][q] = (ok && P.hpos[c][0] == q) ? 1 : 0;
            av[c][q] = (ok && P.hpos[c][1] == q) ? RS : ((ok && P.hpos[c][2] == q) ? 1 : 0);
        }
    }
    auto stage_v = [&](int plane, int b) {
        const int qv0 = plane % P.qe[3], qv1 = (plane / P.qe[3]) % P.qe[4], qv2 = plane / (P.qe[3] * P.qe[4]);
        auto pick = [&](int pos) { return pos == 3 ? qv0 : (pos == 4 ? qv1 : qv2); };
        double* buf = s1sm + b * BUFD;
#pragma unroll
        for (int e = 0; e < 9; ++e) {
            if (e < ne) {
                const double* v2 = P.opB[e] + (int64_t)H * H * (pick(P.ppos[e][2]) + (int64_t)P6 * pick(P.ppos[e][1]));
#pragma unroll
                for (int i0 = 0; i0 < VS / 2; i0 += S1S_NT) {  // 16-byte chunks of the H x H slice
                    const int i = i0 + tid;
                    if (i < H * H / 2) {
                        const int row = i / (H / 2), col = 2 * (i - row * (H / 2));
                        cp_async_16(buf + e * ES + row * RS + col, v2 + row * H + col);
                    }
                }
            }
        }
    };
    // T (sign folded): thread t < ne*H owns T_e[h1], loaded one plane ahead into a register
    const int te = tid / H, th1 = tid - te * H;
    const bool towner = te < ne;
    const double tsg = towner ? P.sign[te] : 0.0;
    auto load_t = [&](int plane) {
        if (!towner) return 0.0;
        const int qv0 = plane % P.qe[3], qv1 = (plane / P.qe[3]) % P.qe[4], qv2 = plane / (P.qe[3] * P.qe[4]);
        const int pos = P.ppos[te][0];
        const int p4 = pos == 3 ? qv0 : (pos == 4 ? qv1 : qv2);
        return __ldg(P.opA[te] + p4 + (int64_t)P4 * th1);
    };
    const int tdst = te * ES + VS + th1;
    int it = 0;
    if ((int)blockIdx.x < nplanes) {
        stage_v(blockIdx.x, 0);
        if (towner) s1sm[tdst] = tsg * load_t(blockIdx.x);
    }
    cp_async_commit();
    for (int plane = blockIdx.x; plane < nplanes; plane += gridDim.x, ++it) {
        cp_async_wait_all();
        __syncthreads();  // this plane's factors are in place; the other buffer is free
        const int nxt = plane + gridDim.x;
        double tnext = 0.0;
        if (nxt < nplanes) {
            stage_v(nxt, (it + 1) & 1);
            tnext = load_t(nxt);
        }
        cp_async_commit();
        const double* buf = s1sm + (it & 1) * BUFD;
        double* t3p = P.t3 + (int64_t)NV * plane;
#pragma unroll 1
        for (int bt = 0; bt < NB; ++bt) {
            double x[S1S_U][4];
            int vo[S1S_U][3], to[S1S_U][3];
            bool ok[S1S_U];
#pragma unroll
            for (int u = 0; u < S1S_U; ++u) {
                const int r = (bt * S1S_U + u) * S1S_NT + tid;
                ok[u] = r < NRUN;
                const int rr = ok[u] ? r : 0;
                const int qq0 = 4 * (rr % R0), q1 = (rr / R0) % H, q2 = rr / (R0 * H);
                if (ok[u]) {
                    const double2 a = __ldcs(reinterpret_cast<const double2*>(t3p) + 2 * r);
                    const double2 b = __ldcs(reinterpret_cast<const double2*>(t3p) + 2 * r + 1);
                    x[u][0] = a.x; x[u][1] = a.y; x[u][2] = b.x; x[u][3] = b.y;
                } else {
                    x[u][0] = x[u][1] = x[u][2] = x[u][3] = 0.0;
                }
#pragma unroll
                for (int c = 0; c < 3; ++c) {
                    vo[u][c] = qq0 * av[c][0] + q1 * av[c][1] + q2 * av[c][2];
                    to[u][c] = VS + qq0 * at[c][0] + q1 * at[c][1] + q2 * at[c][2];
                }
            }
#pragma unroll
            for (int e = 0; e < 9; ++e) {
                if (e < ne) {
                    const int c = P.ecls[e];
                    const double* eb = buf + e * ES;
                    const bool kind_h1 = c == 0 ? q0h1[0] : (c == 1 ? q0h1[1] : q0h1[2]);
                    if (kind_h1) {  // run along h1: T varies, V broadcast
#pragma unroll
                        for (int u = 0; u < S1S_U; ++u) {
                            const int voff = c == 0 ? vo[u][0] : (c == 1 ? vo[u][1] : vo[u][2]);
                            const int toff = c == 0 ? to[u][0] : (c == 1 ? to[u][1] : to[u][2]);
                            const double v = eb[voff];
                            const double2 t01 = *reinterpret_cast<const double2*>(eb + toff);
                            const double2 t23 = *reinterpret_cast<const double2*>(eb + toff + 2);
                            x[u][0] = fma(t01.x, v, x[u][0]);
                            x[u][1] = fma(t01.y, v, x[u][1]);
                            x[u][2] = fma(t23.x, v, x[u][2]);
                            x[u][3] = fma(t23.y, v, x[u][3]);
                        }
                    } else {  // run along h3: V varies, T broadcast
#pragma unroll
                        for (int u = 0; u < S1S_U; ++u) {
                            const int voff = c == 0 ? vo[u][0] : (c == 1 ? vo[u][1] : vo[u][2]);
                            const int toff = c == 0 ? to[u][0] : (c == 1 ? to[u][1] : to[u][2]);
                            const double t = eb[toff];
                            const double2 v01 = *reinterpret_cast<const double2*>(eb + voff);
                            const double2 v23 = *reinterpret_cast<const double2*>(eb + voff + 2);
                            x[u][0] = fma(t, v01.x, x[u][0]);
                            x[u][1] = fma(t, v01.y, x[u][1]);
                            x[u][2] = fma(t, v23.x, x[u][2]);
                            x[u][3] = fma(t, v23.y, x[u][3]);
                        }
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < S1S_U; ++u) {
                const int r = (bt * S1S_U + u) * S1S_NT + tid;
                if (ok[u]) {
                    __stcs(reinterpret_cast<double2*>(t3p) + 2 * r, make_double2(x[u][0], x[u][1]));
                    __stcs(reinterpret_cast<double2*>(t3p) + 2 * r + 1, make_double2(x[u][2], x[u][3]));
                }
            }
        }
        if (towner && nxt < nplanes) s1sm[((it + 1) & 1) * BUFD + tdst] = tsg * tnext;
    }
}

template <int H>
static int launch_ccsdt_s1h(const CcsdtParams& P, cudaStream_t s) {
    constexpr size_t smem = 2 * 9 * (size_t)(H * (H + 2) + H) * 8;
    const int nplanes = P.qe[3] * P.qe[4] * P.qe[5];
    if (nplanes == 0) return BC_OK;
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    if (occ == 0) {
        cudaFuncSetAttribute(ccsdt_s1h_kernel<H>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ccsdt_s1h_kernel<H>, S1S_NT, smem);
        if (occ < 1) occ = 1;
    }
    const int64_t cap = (int64_t)num_sms() * occ;
    const int grid = (int)(nplanes < cap ? nplanes : cap);
    ccsdt_s1h_kernel<H><<<grid, S1S_NT, smem, s>>>(P, nplanes);
    return launch_status();
}

static int launch_ccsdt_s1_stream(const CcsdtParams& P, cudaStream_t s) {
    const int H = P.ext[N_H1];
    if (H == P.ext[N_H2] && H == P.ext[N_H3]) {
        if (H == 16) return launch_ccsdt_s1h<16>(P, s);
        if (H == 24) return launch_ccsdt_s1h<24>(P, s);
    }
    const size_t smem = 2 * ((size_t)P.ncls * 3 * (P.ext[N_H2] * (P.ext[N_H3] + 1) + P.ext[N_H1])) * 8;
    if (smem > 200 * 1024) return 1;
    const int nplanes = P.qe[3] * P.qe[4] * P.qe[5];
    if (nplanes == 0 || P.qe[0] * P.qe[1] * P.qe[2] == 0) return BC_OK;
    const bool run4 = P.qe[0] % 4 == 0;
    auto go = [&](auto kern, size_t* last_smem, int* occ) {
        if (smem != *last_smem) {
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, S1S_NT, smem);
            if (*occ < 1) *occ = 1;
            *last_smem = smem;
        }
        const int64_t cap = (int64_t)num_sms() * *occ;
        const int grid = (int)(nplanes < cap ? nplanes : cap);
        kern<<<grid, S1S_NT, smem, s>>>(P, nplanes);
        return launch_status();
    };
    static PerDevice<size_t> ls4_dev;
    size_t& ls4 = ls4_dev.get();
    static PerDevice<size_t> ls1_dev;
    size_t& ls1 = ls1_dev.get();
    static PerDevice<int> occ4_dev;
    int& occ4 = occ4_dev.get();
    static PerDevice<int> occ1_dev;
    int& occ1 = occ1_dev.get();
    return run4 ? go(ccsdt_s1_stream_kernel<4>, &ls4, &occ4) : go(ccsdt_s1_stream_kernel<1>, &ls1, &occ1);
}

// ==================================================================================
// Single-variant d1/d2 streaming path (hole extents 16^3, one variant per call: the
// HBM-bound configs 3/4 per-variant rows).  One variant touches each t3 value once, so
// the kernel streams t3 planes (the 16^3 hole volume of one particle triple is 32 KB
// contiguous in every storage order) through registers: the thread's 16 t3 values are
// the initial values of its 4 x 4 DFMA accumulator tile, t3 += sum_k A B is accumulated in
// place and stored — no shared-memory cube, no flush.  The next plane's t3 values and B
// slice are in flight while the current plane computes.
//   GEMM per plane: X[(f, x), y] = sum_k A[k][f][x] B[k][y]
//     d1: f = h2, x = h3, y = h1;  A = s v2[h3,h2,p6,k] (per p6),  B = t2[k,p4,p5,h1]
//     d2: f = h1, x = h2, y = h3;  A = s t2[k,p4,h1,h2] (per p4),  B = v2[k,h3,p6,p5]
// Storage position 0 is always x or y (d1: h3 or h1; d2: h3 or h2), so a thread's 4 x 4
// tile is 4 rows of 4 contiguous t3 values (two 16-byte accesses each) and 4 lanes cover a
// 128-byte run.  Planes are visited with the A name slowest, so A (sign folded) is staged
// once per CTA or twice.
// ==================================================================================
constexpr int SV_NT = 256, SV_RS = 18, SV_PS = 16 * SV_RS + 2;  // A row / k-plane strides (doubles)

__device__ __forceinline__ double2 ld_cs2(const double* p) { return __ldcs(reinterpret_cast<const double2*>(p)); }
__device__ __forceinline__ void st_cs2(double* p, double a, double b) {
    __stcs(reinterpret_cast<double2*>(p), make_double2(a, b));
}

#ifndef BC_SVS_MINB
#define BC_SVS_MINB 2
#endif
#ifndef BC_SVS_PF
#define BC_SVS_PF 1  // next unit's t3 tile prefetched into registers
#endif
// Geometry per hole extent H: a unit is (particle plane, range of NF values of f); thread
// tiles are 4 x 4 over (x, y), so a unit has (H/4)^2 NF tiles = NT threads.
template <int H>
struct SvGeo {
    static constexpr int NB = H / 4;               // tile blocks per hole axis
    static constexpr int NF = H == 16 ? 16 : 4;    // f values per unit
    static constexpr int NT = NB * NB * NF;        // 256 | 144
    static constexpr int MINB = H == 16 ? BC_SVS_MINB : 3;  // CTAs per SM (128 registers at 2)
    static constexpr int NFR = H / NF;             // units per plane: 1 | 6
    static constexpr int RS = H + 2;               // A row stride (doubles, even)
    static constexpr int PS = NF * RS + 2;         // A k-plane stride
};

template <int FAM, int H>
__global__ void __launch_bounds__(SvGeo<H>::NT, SvGeo<H>::MINB) ccsdt_svs_kernel(const __grid_constant__ CcsdtParams P, int nunits) {
    using G = SvGeo<H>;
    constexpr int NB = G::NB, NF = G::NF, NT = G::NT, RS = G::RS, PS = G::PS, NFR = G::NFR;
    extern __shared__ __align__(16) double svsm[];
    const int K = P.ext[N_K];
    double* As = svsm;                 // [k][fl][x]
    double* Bs = As + K * PS;          // 2 buffers of [k][y]
    const int tid = threadIdx.x;
    const int bq = tid % NB, bo = (tid / NB) % NB, fl = tid / (NB * NB);
    const int* hp = P.hpos[0];         // storage positions of h1, h2, h3
    const int posX = (FAM == FAM_D1) ? hp[2] : hp[1];
    const int posY = (FAM == FAM_D1) ? hp[0] : hp[2];
    const int posF = (FAM == FAM_D1) ? hp[1] : hp[0];
    const bool xfast = posX == 0;      // else posY == 0
    const int bx = xfast ? bq : bo, by = xfast ? bo : bq;
    auto hstride = [](int pos) { return pos == 0 ? 1 : (pos == 1 ? H : H * H); };
    const int sX = hstride(posX), sY = hstride(posY), sF = hstride(posF);
    const int rstride = xfast ? sY : sX;
    const int tbase = 4 * bx * sX + 4 * by * sY + fl * sF;
    const int P4 = P.ext[N_P4], P5 = P.ext[N_P5], P6 = P.ext[N_P6];
    const int PO1 = (FAM == FAM_D1) ? P5 : P6, PO2 = (FAM == FAM_D1) ? P4 : P5;
    constexpr int64_t HV = (int64_t)H * H * H;
    auto qstride = [&](int pos) {
        return pos == 3 ? HV : (pos == 4 ? HV * P.qe[3] : HV * P.qe[3] * P.qe[4]);
    };
    const int64_t sp4 = qstride(P.ppos[0][0]), sp5 = qstride(P.ppos[0][1]), sp6 = qstride(P.ppos[0][2]);
    const double sg = P.sign[0];
    const double* __restrict__ opA = P.opA[0];  // t2
    const double* __restrict__ opB = P.opB[0];  // v2
    const int lo = (int)((int64_t)nunits * blockIdx.x / gridDim.x);
    const int hi = (int)((int64_t)nunits * (blockIdx.x + 1) / gridDim.x);
    // unit u -> (akey = a * NFR + fr, o1, o2), a = the A name (d1 p6, d2 p4) slowest; decoded
    // once per CTA and then advanced by carries (no divisions per unit)
    struct UnitId { int akey, o1, o2; };
    auto decode = [&](int u) {
        UnitId id;
        id.akey = u / (PO1 * PO2);
        const int r = u - id.akey * (PO1 * PO2);
        id.o1 = r / PO2;
        id.o2 = r - id.o1 * PO2;
        return id;
    };
    auto advance = [&](UnitId id) {
        if (++id.o2 == PO2) {
            id.o2 = 0;
            if (++id.o1 == PO1) {
                id.o1 = 0;
                ++id.akey;
            }
        }
        return id;
    };
    auto unit_ptr = [&](const UnitId& id) {
        const int a = id.akey / NFR, fr = id.akey - a * NFR;  // NFR is a compile-time constant
        const int p4 = (FAM == FAM_D1) ? id.o2 : a, p5 = (FAM == FAM_D1) ? id.o1 : id.o2;
        const int p6 = (FAM == FAM_D1) ? a : id.o1;
        return P.t3 + p4 * sp4 + p5 * sp5 + p6 * sp6 + fr * NF * sF + tbase;
    };
    // B copies: element i = tid + m NT of [y][k] -> (y, k), first and step precomputed
    const int by0 = tid / K, bk0 = tid - (tid / K) * K, bdy = NT / K, bdk = NT - (NT / K) * K;
    auto issue_B = [&](const UnitId& id, double* dst) {  // B[k][y]
        const double* src = (FAM == FAM_D1) ? opA + (int64_t)K * (id.o2 + (int64_t)P4 * id.o1)       // t2[k,p4,p5,h1]
                                            : opB + (int64_t)K * H * (id.o1 + (int64_t)P6 * id.o2);  // v2[k,h3,p6,p5]
        const int stride_y = (FAM == FAM_D1) ? K * P4 * P5 : K;
        int y = by0, k = bk0;
        for (int i = tid; i < H * K; i += NT) {
            cp_async_8(dst + k * H + y, src + (int64_t)stride_y * y + k);
            k += bdk;
            if (k >= K) {
                k -= K;
                ++y;
            }
            y += bdy;
        }
    };
    auto load_tile = [&](const double* p, double (&x)[4][4]) {
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            const double2 u = ld_cs2(p + r * rstride), w = ld_cs2(p + r * rstride + 2);
            x[r][0] = u.x; x[r][1] = u.y; x[r][2] = w.x; x[r][3] = w.y;
        }
    };
    if (lo >= hi) return;
    double x[4][4];  // [row][c]: xfast -> (y = row, x = c), else (x = row, y = c)
    UnitId cur = decode(lo);
    load_tile(unit_ptr(cur), x);
    issue_B(cur, Bs);
    cp_async_commit();
    int curA = -1;
    for (int u = lo; u < hi; ++u) {
        const int akey = cur.akey;
        const UnitId nxt = advance(cur);
        if (akey != curA) {  // stage A (sign folded) for (a, f range): once or twice per CTA
            __syncthreads();
            const int a = akey / NFR, f0 = (akey - a * NFR) * NF;
            if (FAM == FAM_D1) {  // As[k][fl][h3] = v2[h3, f0+fl, p6, k]: 16-byte copies
                const double* src = opB + (int64_t)H * (f0 + (int64_t)H * a);
                for (int i = tid; i < K * NF * (H / 2); i += NT) {
                    const int k = i / (NF * (H / 2)), r = i - k * (NF * (H / 2));
                    const int f = r / (H / 2), c = 2 * (r - f * (H / 2));
                    cp_async_16(As + k * PS + f * RS + c, src + (int64_t)H * H * P6 * k + (int64_t)H * f + c);
                }
            } else {  // As[k][fl][h2] = t2[k, p4, f0+fl, h2]
                const double* src = opA + (int64_t)K * (a + (int64_t)P4 * f0);
                for (int i = tid; i < K * NF * H; i += NT) {
                    const int r = i / K, k = i - r * K;  // r = fl + NF * h2
                    const int f = r % NF, x2 = r / NF;
                    cp_async_8(As + k * PS + f * RS + x2, src + (int64_t)K * P4 * (f + (int64_t)H * x2) + k);
                }
            }
            cp_async_commit();
            if (sg < 0.0) {  // fold the variant's sign into A once (exact)
                cp_async_wait_all();
                __syncthreads();
                for (int i = tid; i < K * NF * H; i += NT) {
                    const int k = i / (NF * H), r = i - k * (NF * H);
                    double& v = As[k * PS + (r / H) * RS + (r % H)];
                    v = -v;
                }
            }
            curA = akey;
        }
        cp_async_wait_all();
        __syncthreads();  // B(u) landed, A staged, the other B buffer is free
        const double* Bc = Bs + ((u - lo) & 1) * H * K;
        if (u + 1 < hi) issue_B(nxt, Bs + ((u + 1 - lo) & 1) * H * K);
        cp_async_commit();
        if (!BC_SVS_PF && u != lo) load_tile(unit_ptr(cur), x);
        double acc[4][4];
#pragma unroll
        for (int r = 0; r < 4; ++r)
#pragma unroll
            for (int c = 0; c < 4; ++c) acc[r][c] = x[r][c];
        double* tp = unit_ptr(cur);
        if (BC_SVS_PF && u + 1 < hi) load_tile(unit_ptr(nxt), x);
        const double* Ap = As + fl * RS + 4 * bx;
        const double* Bp = Bc + 4 * by;
#pragma unroll 4
        for (int k = 0; k < K; ++k) {
            const double2 a01 = *reinterpret_cast<const double2*>(Ap + k * PS);
            const double2 a23 = *reinterpret_cast<const double2*>(Ap + k * PS + 2);
            const double2 b01 = *reinterpret_cast<const double2*>(Bp + k * H);
            const double2 b23 = *reinterpret_cast<const double2*>(Bp + k * H + 2);
            const double av[4] = {a01.x, a01.y, a23.x, a23.y}, bv[4] = {b01.x, b01.y, b23.x, b23.y};
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
                for (int jj = 0; jj < 4; ++jj) {
                    // xfast: row = y (jj), element = x (i); else row = x (i), element = y (jj)
                    double& t = xfast ? acc[jj][i] : acc[i][jj];
                    t = fma(av[i], bv[jj], t);
                }
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            st_cs2(tp + r * rstride, acc[r][0], acc[r][1]);
            st_cs2(tp + r * rstride + 2, acc[r][2], acc[r][3]);
        }
        cur = nxt;
    }
}

template <int FAM, int H>
static int launch_ccsdt_svs(const CcsdtParams& P, cudaStream_t s) {
    using G = SvGeo<H>;
    const int K = P.ext[N_K];
    const size_t smem = ((size_t)K * G::PS + 2 * (size_t)H * K) * 8;
    const int nunits = P.qe[3] * P.qe[4] * P.qe[5] * G::NFR;
    if (nunits == 0) return BC_OK;
    static PerDevice<size_t> last_smem_dev;
    size_t& last_smem = last_smem_dev.get();
    static PerDevice<int> occ_dev;
    int& occ = occ_dev.get();
    if (smem != last_smem) {
        cudaFuncSetAttribute(ccsdt_svs_kernel<FAM, H>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ccsdt_svs_kernel<FAM, H>, G::NT, smem);
        if (occ < 1) occ = 1;
        last_smem = smem;
    }
    const int64_t cap = (int64_t)num_sms() * occ;
    const int grid = (int)(nunits < cap ? nunits : cap);
    ccsdt_svs_kernel<FAM, H><<<grid, G::NT, smem, s>>>(P, nunits);
    return launch_status();
}

// ------------------------------------------------------------------------------------ host
static int choose_bs(const int* qe) {
    // smallest padded volume over the three hole positions; ties -> larger cube
    int best = 16;
    long best_vol = -1;
    for (int bs : {16, 12, 8}) {
        long vol = 1;
        for (int q = 0; q < 3; ++q) vol *= (long)((qe[q] + bs - 1) / bs) * bs;
        if (best_vol < 0 || vol < best_vol) {
            best_vol = vol;
            best = bs;
        }
    }
    return best;
}

template <int FAM, int BS>
static int launch_ccsdt_bs(const CcsdtParams& P, cudaStream_t s) {
    using TT = CcGeo<BS>;
    static PerDevice<bool> init_dev;
    bool& init = init_dev.get();
    if (!init) {
        cudaFuncSetAttribute(ccsdt_kernel<FAM, BS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TT::SMEM);
        init = true;
    }
    const int64_t units = (int64_t)P.ncube[0] * P.ncube[1] * P.ncube[2] * P.qe[3] * P.qe[4] * P.qe[5];
    if (units == 0) return BC_OK;
    ccsdt_kernel<FAM, BS><<<(unsigned)units, TT::NT, TT::SMEM, s>>>(P);
    return launch_status();
}

// Launch variants listed in `vs` (ascending), all sharing one t3 geometry.
int run_energy(const int* ext7, const double* t3, const double* eh, const double* ep, double* ws, cudaStream_t s);
static int run_ccsdt_impl(int fam, const int* ext7, double* t3, const int* vs, int nv, const double* const* opA,
                          const double* const* opB, const double* eps_h, const double* eps_p, double* ws,
                          bool* fused_energy, cudaStream_t s);

// t3 += the listed variants; with ws != nullptr also ws[0] = the energy check of the updated
// t3 (bc_check_energy), fused into the 16-cube TMA kernel's store pass where that kernel
// runs on full cubes, else a separate pass after the update.
int run_ccsdt(int fam, const int* ext7, double* t3, const int* vs, int nv, const double* const* opA,
              const double* const* opB, cudaStream_t s, const double* eps_h, const double* eps_p, double* ws) {
    bool fused = false;
    const int st = run_ccsdt_impl(fam, ext7, t3, vs, nv, opA, opB, eps_h, eps_p, ws, &fused, s);
    if (st || !ws || fused) return st;
    return run_energy(ext7, t3, eps_h, eps_p, ws, s);
}

static int run_ccsdt_impl(int fam, const int* ext7, double* t3, const int* vs, int nv, const double* const* opA,
                          const double* const* opB, const double* eps_h, const double* eps_p, double* ws,
                          bool* fused_energy, cudaStream_t s) {
    CcsdtParams P{};
    P.t3 = t3;
    for (int q = 0; q < 7; ++q) P.ext[q] = ext7[q];
    const VariantInfo v0 = variant_info(fam, vs[0]);
    for (int q = 0; q < 6; ++q) P.qe[q] = ext7[v0.order[q]];
    // group entries by hole permutation class (class = (v-1) % 3), ascending v inside
    int n = 0, ncls = 0;
    for (int cls = 0; cls < 3; ++cls) {
        bool any = false;
        for (int t = 0; t < nv; ++t) {
            const int v = vs[t];
            if ((v - 1) % 3 != cls) continue;
            const VariantInfo vi = variant_info(fam, v);
            if (!any) {
                for (int q = 0; q < 3; ++q) P.hpos[ncls][vi.order[q]] = q;  // name (h1,h2,h3 = 0,1,2) -> position
                any = true;
            }
            for (int q = 3; q < 6; ++q) P.ppos[n][vi.order[q] - 3] = q;
            P.sign[n] = vi.sign;
            P.smask[n] = vi.sign < 0 ? 0x80000000u : 0u;
            P.ecls[n] = ncls;
            P.opA[n] = opA[t];
            P.opB[n] = opB[t];
            ++n;
        }
        if (any) ++ncls;
    }
    P.nentry = n;
    P.ncls = ncls;
    if (fam == FAM_S1) {
        const int st = launch_ccsdt_s1_stream(P, s);
        if (st != 1) return st;  // 1: factors exceed shared memory (cube kernel below)
    }
    // one d1/d2 variant on 16^3 hole volumes: t3 streamed through registers (HBM-bound)
    if (n == 1 && fam != FAM_S1 && ext7[N_H1] == 16 && ext7[N_H2] == 16 && ext7[N_H3] == 16 && ext7[N_K] <= 32)
        return fam == FAM_D1 ? launch_ccsdt_svs<FAM_D1, 16>(P, s) : launch_ccsdt_svs<FAM_D2, 16>(P, s);
    // tensor-core path: 16-cubes with 16-byte-aligned operand rows (even k, even h3 for d1).
    // It also takes hole extents the 16-cube does not divide (e.g. tile 24 = 16 + 8, ragged
    // cubes zero-filled by TMA): measured 2x faster than the 12-cube DFMA kernel at tile 24.
    const bool tc_shape = (fam != FAM_S1) && (ext7[N_K] % 2 == 0) && (fam != FAM_D1 || ext7[N_H3] % 2 == 0) &&
                          P.qe[0] >= 12 && P.qe[1] >= 12 && P.qe[2] >= 12;
    // 24-cube TMA path when its padded hole volume is smaller than the 16-cube's (tile 24)
    if (tc_shape) {
        long v16 = 1, v24 = 1;
        for (int q = 0; q < 3; ++q) {
            v16 *= (long)((P.qe[q] + 15) / 16) * 16;
            v24 *= (long)((P.qe[q] + 23) / 24) * 24;
        }
        if (v24 < v16) {
            for (int q = 0; q < 3; ++q) P.ncube[q] = (P.qe[q] + 23) / 24;
            const int st = (fam == FAM_D1) ? launch_ccsdt_tma24<FAM_D1>(P, s) : launch_ccsdt_tma24<FAM_D2>(P, s);
            if (st != 1) return st;
        }
    }
    // 16-cube TMA kernel; if the driver cannot encode tensor maps (returns 1), the DFMA
    // cube kernel below takes the shape
    const int bs = tc_shape ? 16 : choose_bs(P.qe);
    for (int q = 0; q < 3; ++q) P.ncube[q] = (P.qe[q] + bs - 1) / bs;
    if (tc_shape) {
        // the energy check rides along when every cube is full (its store pass covers t3)
        const bool fuse = ws && P.qe[0] % 16 == 0 && P.qe[1] % 16 == 0 && P.qe[2] % 16 == 0 &&
                          ext7[N_H1] == ext7[N_H2] && ext7[N_H2] == ext7[N_H3] && ext7[N_P4] == ext7[N_P5] &&
                          ext7[N_P5] == ext7[N_P6];
        if (fuse) {
            P.eps_h = eps_h;
            P.eps_p = eps_p;
            P.ews = ws + 8;
        }
        const int st = (fam == FAM_D1) ? launch_ccsdt_tma<FAM_D1>(P, s) : launch_ccsdt_tma<FAM_D2>(P, s);
        if (st != 1) {
            *fused_energy = fuse;
            return st;
        }
        P.eps_h = P.eps_p = nullptr;
        P.ews = nullptr;
    }
#define LAUNCH(F)                                                          \
    if (bs == 16) return launch_ccsdt_bs<F, 16>(P, s);                      \
    if (bs == 12) return launch_ccsdt_bs<F, 12>(P, s);                      \
    return launch_ccsdt_bs<F, 8>(P, s);
    if (fam == FAM_D1) { LAUNCH(FAM_D1) }
    if (fam == FAM_D2) { LAUNCH(FAM_D2) }
    LAUNCH(FAM_S1)
#undef LAUNCH
}

}  // namespace bc
