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
//   d1/s1:  X[(h3,h2), h1] = sum_k v2[h3,h2,p6,k] * t2[k,p4,p5,h1]     (M = BS^2, N = BS)
//   d2   :  X[h3, (h1,h2)] = sum_k v2[k,h3,p6,p5] * t2[k,p4,h1,h2]     (M = BS,   N = BS^2)
// (s1 is the K = 1 outer product t1[p4,h1] * v2[h3,h2,p6,p5]).  A cube in q-space is a
// cube in name space for every hole permutation, so the GEMM shape is the same for all
// variants.  Operand slices are staged in shared memory (zero-padded at block edges,
// sign folded into the N operand), each thread accumulates a 4x4 register tile over k
// (scalar replacement), and variants sharing a hole permutation ("class")
// accumulate into the same registers; a class is flushed into the shared accumulator at
// its permuted positions.  The (h1,h2,h3) <-> storage-position maps are derived here from
// the generating rule of DESIGN.md R12 (not copied from the oracle's table).
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
    int ppos[9][3];   // per entry: storage position (3..5) of p4, p5, p6
    int ecls[9];      // per entry: class slot
    int hpos[3][3];   // per class slot: storage position (0..2) of h1, h2, h3
    int nentry, ncls;
    int ext[7];       // named extents h1 h2 h3 p4 p5 p6 k
    int qe[6];        // storage-position extents
    int ncube[3];     // cubes along q1, q2, q3
};

template <int BS>
struct CcTile {
    static constexpr int TILES = BS * BS * BS / 16;          // 4x4 register tiles
    static constexpr int NT = (TILES + 31) / 32 * 32;
    static constexpr int KC = 16;                            // k chunk
    static constexpr int MN2 = BS * BS + 2;                  // padded smem row (x doubles)
    static constexpr int MN1 = BS + 2;
    static constexpr size_t SMEM = (size_t)(BS * BS * BS + KC * MN2 + KC * MN2) * sizeof(double);
};

template <int FAM, int BS>
__global__ void __launch_bounds__(CcTile<BS>::NT) ccsdt_kernel(const CcsdtParams P) {
    using TT = CcTile<BS>;
    constexpr int NT = TT::NT, KC = TT::KC;
    constexpr int M = (FAM == FAM_D2) ? BS : BS * BS;   // v2 side
    constexpr int N = (FAM == FAM_D2) ? BS * BS : BS;   // t2 / t1 side
    constexpr int SA = M + 2, SB = N + 2;                // smem row strides (16B-aligned rows)
    constexpr int MT = M / 4;
    extern __shared__ __align__(16) double sm[];
    double* acc_s = sm;                  // BS^3 accumulator, index q0 + BS*(q1 + BS*q2)
    double* As = acc_s + BS * BS * BS;   // [KC][SA]
    double* Bs = As + KC * SA;           // [KC][SB]

    // ---- unit decode
    const int ncubes = P.ncube[0] * P.ncube[1] * P.ncube[2];
    const int cube = blockIdx.x % ncubes;
    const int plane = blockIdx.x / ncubes;
    int o[3], len[3];
    {
        const int c0 = cube % P.ncube[0];
        const int c1 = (cube / P.ncube[0]) % P.ncube[1];
        const int c2 = cube / (P.ncube[0] * P.ncube[1]);
        o[0] = c0 * BS;
        o[1] = c1 * BS;
        o[2] = c2 * BS;
        for (int q = 0; q < 3; ++q) len[q] = min(BS, P.qe[q] - o[q]);
    }
    int qv[3];
    qv[0] = plane % P.qe[3];
    qv[1] = (plane / P.qe[3]) % P.qe[4];
    qv[2] = plane / (P.qe[3] * P.qe[4]);

    for (int i = threadIdx.x; i < BS * BS * BS; i += NT) acc_s[i] = 0.0;

    const int H1 = P.ext[N_H1], H2 = P.ext[N_H2], H3 = P.ext[N_H3];
    const int P4 = P.ext[N_P4], P5 = P.ext[N_P5], P6 = P.ext[N_P6];
    const int K = (FAM == FAM_S1) ? 1 : P.ext[N_K];

    const int tt = threadIdx.x;
    const bool has_tile = tt < TT::TILES;
    const int mt = tt % MT, nt = tt / MT;

    int entry = 0;
    for (int c = 0; c < P.ncls; ++c) {
        // name-space origin / length of the cube for this class's hole permutation
        const int hp1 = P.hpos[c][0], hp2 = P.hpos[c][1], hp3 = P.hpos[c][2];
        const int O1 = o[hp1], O2 = o[hp2], O3 = o[hp3];
        const int L1 = len[hp1], L2 = len[hp2], L3 = len[hp3];
        double acc[4][4];
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int b = 0; b < 4; ++b) acc[a][b] = 0.0;

        for (; entry < P.nentry && P.ecls[entry] == c; ++entry) {
            const double* __restrict__ tA = P.opA[entry];
            const double* __restrict__ vB = P.opB[entry];
            const double sg = P.sign[entry];
            const int p4 = qv[P.ppos[entry][0] - 3];
            const int p5 = qv[P.ppos[entry][1] - 3];
            const int p6 = qv[P.ppos[entry][2] - 3];
            for (int k0 = 0; k0 < K; k0 += KC) {
                const int kc = min(KC, K - k0);
                __syncthreads();
                // ---- stage the v2 slice (M side) and the t2/t1 slice (N side, signed)
                if constexpr (FAM == FAM_D1 || FAM == FAM_S1) {
                    // As[kk][i3 + BS*i2] = v2[h3, h2, p6, k]   (d1)  |  v2[h3, h2, p6, p5] (s1)
                    for (int x = threadIdx.x; x < KC * M; x += NT) {
                        const int kk = x / M, m = x - kk * M;
                        const int i2 = m / BS, i3 = m - i2 * BS;
                        double v = 0.0;
                        if (kk < kc && i3 < L3 && i2 < L2) {
                            const int last = (FAM == FAM_S1) ? p5 : (k0 + kk);
                            v = __ldg(vB + (O3 + i3) + (int64_t)H3 * ((O2 + i2) + (int64_t)H2 * (p6 + (int64_t)P6 * last)));
                        }
                        As[kk * SA + m] = v;
                    }
                    // Bs[kk][i1] = s * t2[k, p4, p5, h1]  (d1)  |  s * t1[p4, h1] (s1)
                    for (int x = threadIdx.x; x < KC * N; x += NT) {
                        const int i1 = x / KC, kk = x - i1 * KC;
                        double v = 0.0;
                        if (kk < kc && i1 < L1) {
                            if constexpr (FAM == FAM_S1)
                                v = sg * __ldg(tA + p4 + (int64_t)P4 * (O1 + i1));
                            else
                                v = sg * __ldg(tA + (k0 + kk) + (int64_t)K * (p4 + (int64_t)P4 * (p5 + (int64_t)P5 * (O1 + i1))));
                        }
                        Bs[kk * SB + i1] = v;
                    }
                } else {
                    // As[kk][i3] = v2[k, h3, p6, p5]
                    for (int x = threadIdx.x; x < KC * M; x += NT) {
                        const int i3 = x / KC, kk = x - i3 * KC;
                        double v = 0.0;
                        if (kk < kc && i3 < L3)
                            v = __ldg(vB + (k0 + kk) + (int64_t)K * ((O3 + i3) + (int64_t)H3 * (p6 + (int64_t)P6 * p5)));
                        As[kk * SA + i3] = v;
                    }
                    // Bs[kk][i1 + BS*i2] = s * t2[k, p4, h1, h2]
                    for (int x = threadIdx.x; x < KC * N; x += NT) {
                        const int n = x / KC, kk = x - n * KC;
                        const int i2 = n / BS, i1 = n - i2 * BS;
                        double v = 0.0;
                        if (kk < kc && i1 < L1 && i2 < L2)
                            v = sg * __ldg(tA + (k0 + kk) + (int64_t)K * (p4 + (int64_t)P4 * ((O1 + i1) + (int64_t)H1 * (O2 + i2))));
                        Bs[kk * SB + n] = v;
                    }
                }
                __syncthreads();
                if (has_tile) {
                    for (int kk = 0; kk < kc; ++kk) {
                        const double2 a01 = *reinterpret_cast<const double2*>(As + kk * SA + 4 * mt);
                        const double2 a23 = *reinterpret_cast<const double2*>(As + kk * SA + 4 * mt + 2);
                        const double2 b01 = *reinterpret_cast<const double2*>(Bs + kk * SB + 4 * nt);
                        const double2 b23 = *reinterpret_cast<const double2*>(Bs + kk * SB + 4 * nt + 2);
                        const double av[4] = {a01.x, a01.y, a23.x, a23.y};
                        const double bv[4] = {b01.x, b01.y, b23.x, b23.y};
#pragma unroll
                        for (int a = 0; a < 4; ++a)
#pragma unroll
                            for (int b = 0; b < 4; ++b) acc[a][b] = fma(av[a], bv[b], acc[a][b]);
                    }
                }
            }
        }
        // ---- flush this class into the cube accumulator at its permuted positions
        if (has_tile) {
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int b = 0; b < 4; ++b) {
                    const int m = 4 * mt + a, n = 4 * nt + b;
                    int i1, i2, i3;
                    if constexpr (FAM == FAM_D2) {
                        i3 = m;
                        i2 = n / BS;
                        i1 = n - i2 * BS;
                    } else {
                        i2 = m / BS;
                        i3 = m - i2 * BS;
                        i1 = n;
                    }
                    if (i1 < L1 && i2 < L2 && i3 < L3) {
                        int ql[3];
                        ql[hp1] = i1;
                        ql[hp2] = i2;
                        ql[hp3] = i3;
                        acc_s[ql[0] + BS * (ql[1] + BS * ql[2])] += acc[a][b];
                    }
                }
        }
    }
    __syncthreads();
    // ---- t3 += accumulator (read and written once)
    const int64_t pbase = (int64_t)P.qe[0] * P.qe[1] * P.qe[2] *
                          (qv[0] + (int64_t)P.qe[3] * (qv[1] + (int64_t)P.qe[4] * qv[2]));
    for (int i = threadIdx.x; i < BS * BS * BS; i += NT) {
        const int q0 = i % BS, q1 = (i / BS) % BS, q2 = i / (BS * BS);
        if (q0 < len[0] && q1 < len[1] && q2 < len[2]) {
            double* p = P.t3 + pbase + (o[0] + q0) + (int64_t)P.qe[0] * ((o[1] + q1) + (int64_t)P.qe[1] * (o[2] + q2));
            *p += acc_s[i];
        }
    }
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
    using TT = CcTile<BS>;
    static bool init = false;
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
int run_ccsdt(int fam, const int* ext7, double* t3, const int* vs, int nv, const double* const* opA,
              const double* const* opB, cudaStream_t s) {
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
            P.ecls[n] = ncls;
            P.opA[n] = opA[t];
            P.opB[n] = opB[t];
            ++n;
        }
        if (any) ++ncls;
    }
    P.nentry = n;
    P.ncls = ncls;
    const int bs = choose_bs(P.qe);
    for (int q = 0; q < 3; ++q) P.ncube[q] = (P.qe[q] + bs - 1) / bs;
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
