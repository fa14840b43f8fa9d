/*
 * libbarracuda — B200-native (sm_100a) batched small tensor contractions.
 *
 * The data-parallel hot path of Nelson et al., "Generating Efficient Tensor Contractions
 * for GPUs" (ICPP 2015): thousands of identically-sized small tensors contracted
 * independently per spectral element or per CCSD(T) tile.
 * Citations "P:<lines>" are PAPER.md line numbers; "R<n>" are the readings listed in
 * DESIGN.md §3 (where the paper is silent, garbled or ambiguous).
 *
 * CONVENTIONS (every entry point)
 *  - All tensor pointers are DEVICE pointers owned by the caller.  The library never
 *    allocates, frees or synchronises; every call is asynchronous on `stream`
 *    (a cudaStream_t passed as void*; NULL = legacy default stream) and returns after
 *    the launch.  Host-side structs (bc_tile_dims, pointer arrays) are read during the
 *    call only.
 *  - fp64 unless the name ends in _f32.  Spectral tensors are row-major (last index
 *    fastest), elements contiguous (R5).  CCSD(T) tensors are
 *    Fortran order (first index fastest), as in the NWChem kernels [7] (R12).
 *  - Return value: BC_OK or a negative bc_status.  Validation is synchronous:
 *      BC_ERR_ARG          N < 0, p not in [1,15], variant not in [1,9], extent <= 0,
 *                          NULL pointer with non-zero work
 *      BC_ERR_UNSUPPORTED  size beyond the compiled maximum (p > 15, extent > 64)
 *      BC_ERR_ALIGN        a pointer not 16-byte aligned (8-byte for _f32)
 *      BC_ERR_ALIAS        an output overlapping an input (in-place is not supported, R20)
 *      BC_ERR_CUDA         a CUDA launch error; bc_last_cuda_error() returns its code
 *    Nothing is launched when an error is returned.  N == 0 is a no-op returning BC_OK.
 *  - Thread safety: no global mutable state except a once-initialised device-attribute
 *    cache and a thread-local last-CUDA-error slot.  Safe to call concurrently on
 *    different streams.
 *  - Results are deterministic: each output is computed by one thread in a fixed
 *    summation order that does not depend on N, the grid, or the shard (R15).
 */
#ifndef BARRACUDA_H
#define BARRACUDA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    BC_OK = 0,
    BC_ERR_ARG = -1,
    BC_ERR_ALIGN = -2,
    BC_ERR_ALIAS = -3,
    BC_ERR_UNSUPPORTED = -4,
    BC_ERR_CUDA = -5
} bc_status;

#define BC_MAX_P 15          /* spectral order p in [1, 15]  =>  P1 = p + 1 in [2, 16] */
#define BC_MAX_TILE_EXTENT 64 /* CCSD(T) extents in [1, 64] */
#define BC_CHECK_WS_DOUBLES 1024 /* workspace size (doubles) for bc_check_* */

/* ===================================================================== spectral family */

/* 3-D sum-factorised contraction, Eq. (1) (Fig. 2(a)) in the
 * BASELINE form (R1):
 *     V[e][i][j][k] = sum_{l,m,n=0..p} A[k][n] * B[j][m] * C[i][l] * U[e][l][m][n]
 * for e in [0, N).  A, B, C: (p+1)x(p+1) row-major, shared by all elements (R6).
 * U, V: N x (p+1)^3, row-major per element, elements contiguous.  V is OVERWRITTEN (R3).
 * Evaluated factored and fused: S1 contracts n, S2 m, S3 l, with the
 * intermediates kept in shared memory (R4).  The paper's own index placement is
 * paper(A,B,C,U) = bc_sumfact3d(A^T, B^T, C^T, reverse_axes(U)). */
int bc_sumfact3d(int64_t N, int p, const double* A, const double* B, const double* C,
                 const double* U, double* V, void* stream);
/* Same, plus the check scalar ws[0] = sum over all V of V^2 (R18), accumulated in the
 * kernel's store epilogue instead of re-reading V (ws: device workspace of
 * >= BC_CHECK_WS_DOUBLES doubles, deterministic fixed-order reduction). */
int bc_sumfact3d_check(int64_t N, int p, const double* A, const double* B, const double* C,
                       const double* U, double* V, double* ws, void* stream);
/* Same in fp32 (R16). */
int bc_sumfact3d_f32(int64_t N, int p, const float* A, const float* B, const float* C,
                     const float* U, float* V, void* stream);

/* 2-D form (R2):  V[e][i][j] = sum_{l,m} B[i][l] * A[j][m] * U[e][l][m]
 * (V = B U A^T per element).  U, V: N x (p+1)^2 row-major.  V is OVERWRITTEN. */
int bc_sumfact2d(int64_t N, int p, const double* A, const double* B, const double* U,
                 double* V, void* stream);

/* Nekbone local_grad3 (Table I).  U[e][k][j][i] with i fastest (Nekbone
 * u(i,j,k), R5); D is (p+1)x(p+1) row-major (the GLL derivative matrix in Nekbone, R11):
 *     ur[e][k][j][i] = sum_l D[i][l] U[e][k][j][l]
 *     us[e][k][j][i] = sum_l D[j][l] U[e][k][l][i]
 *     ut[e][k][j][i] = sum_l D[k][l] U[e][l][j][i]
 * ur, us, ut OVERWRITTEN; they must not overlap U or each other. */
int bc_local_grad3(int64_t N, int p, const double* D, const double* U, double* ur,
                   double* us, double* ut, void* stream);

/* Nekbone local_grad3_t (Table I): the transpose, summed:
 *     U[e][k][j][i] = sum_l D[l][i] ur[e][k][j][l] + sum_l D[l][j] us[e][k][l][i]
 *                   + sum_l D[l][k] ut[e][l][j][i]                      (OVERWRITE U) */
int bc_local_grad3_t(int64_t N, int p, const double* D, const double* ur, const double* us,
                     const double* ut, double* U, void* stream);

/* Nekbone element operator ax_e (R22):
 *     (ur,us,ut) = local_grad3(D,U);  (wr,ws,wt) = G (ur,us,ut) per point;
 *     W = local_grad3_t(D, wr, ws, wt)
 * G: N x 6 x (p+1)^3 holding g0..g5 of the symmetric 3x3 metric per point:
 *     wr = g0 ur + g1 us + g2 ut;  ws = g1 ur + g3 us + g4 ut;  wt = g2 ur + g4 us + g5 ut.
 * W OVERWRITTEN. */
int bc_ax_e(int64_t N, int p, const double* D, const double* U, const double* G, double* W,
            void* stream);

/* ===================================================================== CCSD(T) family */

/* Named extents of one tile block.  k is the contracted extent (h7 for d1, p7 for d2;
 * ignored by s1). */
typedef struct {
    int h1, h2, h3, p4, p5, p6, k;
} bc_tile_dims;

/* NWChem TCE triples kernels [7] (Table I), variant
 * v in 1..9.  t3 is ACCUMULATED (R3):
 *   d1: t3[sigma_v(h3,h2,h1,p6,p5,p4)] += s_v * sum_h7 t2[h7,p4,p5,h1] * v2[h3,h2,p6,h7]
 *   d2: t3[sigma_v(h3,h2,h1,p6,p5,p4)] += s_v * sum_p7 t2[p7,p4,h1,h2] * v2[p7,h3,p6,p5]
 *   s1: t3[sigma_v(h3,h2,h1,p6,p5,p4)] += s_v * t1[p4,h1] * v2[h3,h2,p6,p5]
 * where sigma_v is the variant's t3 storage order and s_v its sign (R12:
 * d1 hole h1 at storage position 3,2,1 and particle p6 at 1,3,2, hole permutation
 * cycling fastest in v; d2 hole h3 at 1,3,2 and particle p4 at 3,2,1; s1 hole as d1,
 * particle as d2; s_v = -(hole parity)(particle parity) for d1/d2, + for s1).
 * All tensors Fortran order; a storage position takes the extent of the name held
 * there.  t3 must not overlap t2/v2 (BC_ERR_ALIAS). */
int bc_ccsdt_d1(int variant, const bc_tile_dims* d, double* t3, const double* t2,
                const double* v2, void* stream);
int bc_ccsdt_d2(int variant, const bc_tile_dims* d, double* t3, const double* t2,
                const double* v2, void* stream);
int bc_ccsdt_s1(int variant, const bc_tile_dims* d, double* t3, const double* t1,
                const double* v2, void* stream);

/* Fused variants: t3 += sum_{v : t2[v-1] != NULL} contribution_v(t2[v-1],
 * v2[v-1]), t3 read and written once.  t2/v2 are HOST arrays of 9 DEVICE pointers;
 * a NULL t2[v-1] skips variant v.  Equal to the ascending sequence of single-variant
 * calls up to rounding.  When the hole extents or the particle extents are not all
 * equal the variants' t3 geometries differ and the call issues the per-variant
 * kernels in ascending v instead (same result). */
int bc_ccsdt_d1_fused(const bc_tile_dims* d, double* t3, const double* const t2[9],
                      const double* const v2[9], void* stream);
int bc_ccsdt_d2_fused(const bc_tile_dims* d, double* t3, const double* const t2[9],
                      const double* const v2[9], void* stream);
int bc_ccsdt_s1_fused(const bc_tile_dims* d, double* t3, const double* const t1[9],
                      const double* const v2[9], void* stream);

/* A fused family update followed by its check scalar (R18: the "CCSD(T) energy-style sum"
 * the north star names for the checks; P:705-712 usage): family 1 = d1, 2 = d2, 3 = s1;
 * a/b as bc_ccsdt_{d1,d2,s1}_fused.  After t3 += the listed variants,
 *     ws[0] = E = bc_check_energy(d, t3, eps_h, eps_p) of the UPDATED t3
 * (same definition and layouts; equal up to the order of the fp64 sum).  Where the 16-cube
 * tensor-core kernel runs on full cubes (hole extents multiples of 16, equal hole and
 * equal particle extents) the energy is accumulated in that kernel's t3 store pass (t3 is
 * not read again); otherwise the update and a separate energy pass run back to back.
 * ws: device, >= BC_CHECK_WS_DOUBLES doubles, not overlapping t3. */
int bc_ccsdt_fused_energy(int family, const bc_tile_dims* d, double* t3, const double* const a[9],
                          const double* const b[9], const double* eps_h, const double* eps_p,
                          double* ws, void* stream);

/* All 27 triples variants of one tile block fused, t3 never stored (
 * P:705-712 "representative of what executes at the socket level"):
 *     t3 = sum_v s1_v + sum_v d1_v + sum_v d2_v        (from zero, R3/R12/R23)
 *     ws[0] = E = sum over t3 (canonical order) of t3^2 / (eh3+eh2+eh1-ep6-ep5-ep4)
 * i.e. bc_check_energy of the t3 that the 27 per-variant calls would build on a zeroed
 * buffer.  Host arrays of 9 device pointers per list; NULL skips a variant.
 * Requires h1 = h2 = h3 (even, >= 12), p4 = p5 = p6 and even k (the tile case);
 * otherwise BC_ERR_UNSUPPORTED.  ws: >= BC_CHECK_WS_DOUBLES doubles. */
int bc_ccsdt_triples_energy(const bc_tile_dims* d, const double* const t1[9],
                            const double* const v2s1[9], const double* const t2d1[9],
                            const double* const v2d1[9], const double* const t2d2[9],
                            const double* const v2d2[9], const double* eps_h,
                            const double* eps_p, double* ws, void* stream);

/* North-star convenience form ("trip counts of 16 iterations in each dimension"):
 * all seven extents equal to `tile`. */
int bc_ccsdt_d1_tile(int variant, int tile, double* t3, const double* t2, const double* v2,
                     void* stream);
int bc_ccsdt_d2_tile(int variant, int tile, double* t3, const double* t2, const double* v2,
                     void* stream);

/* ===================================================================== checks (R18) */

/* ws[0] = sum_i x[i]^2 (fp64, fixed reduction tree: deterministic).  ws: device
 * workspace of >= BC_CHECK_WS_DOUBLES doubles; the result is left in ws[0]. */
int bc_check_sumsq(int64_t n, const double* x, double* ws, void* stream);

/* ws[0] = E = sum t3[x]^2 / (eh3[h3]+eh2[h2]+eh1[h1]-ep6[p6]-ep5[p5]-ep4[p4]) over t3 in
 * the canonical order (h3,h2,h1,p6,p5,p4), Fortran.  eps_h = [eh1 | eh2 | eh3]
 * (h1+h2+h3 values), eps_p = [ep4 | ep5 | ep6] (device arrays). */
int bc_check_energy(const bc_tile_dims* d, const double* t3, const double* eps_h,
                    const double* eps_p, double* ws, void* stream);

/* ===================================================================== synthetic inputs */

/* Counter-based input generator (same definition as synthetic/__init__.py):
 *   z = splitmix64(seed + (tensor_id << 40) + offset + i),  i in [0, n)
 *   kind 0: x = ((z >> 11) * 2^-53) * 2 - 1      kind 1: x = (z >> 61) - 4
 *   kind 2: x = lo + (hi - lo) * ((z >> 11) * 2^-53)
 * out[i] = x (fp64) or (float)x (_f32). */
int bc_fill(int kind, uint64_t seed, uint64_t tensor_id, uint64_t offset, int64_t n,
            double lo, double hi, double* out, void* stream);
int bc_fill_f32(int kind, uint64_t seed, uint64_t tensor_id, uint64_t offset, int64_t n,
                double lo, double hi, float* out, void* stream);

/* ===================================================================== measurement */

/* FP64 peak probe (a measurement utility, not a method operation): launches a kernel of
 * independent FP64 chains so the bench can time the FP64 roofline denominators live
 * (DESIGN.md §4): kind 0 = DFMA (fma.rn.f64), kind 1 = DMMA (mma.sync.m8n8k4.f64).
 * iters in [1, 2^20] scales the work; *flops (HOST pointer) receives the number of
 * floating-point operations the launch performs (the caller times it with CUDA events).
 * scratch: device, >= bc_probe_scratch_doubles() doubles (receives the chain results). */
int bc_probe_fp64(int kind, int iters, double* scratch, int64_t scratch_doubles, double* flops,
                  void* stream);
int64_t bc_probe_scratch_doubles(void);

/* ===================================================================== misc */

const char* bc_status_string(int status);
/* cudaError_t code behind the last BC_ERR_CUDA returned on this host thread. */
int bc_last_cuda_error(void);
/* (major << 16) | minor */
int bc_version(void);
/* Number of kernels this library has launched on this host thread (for the bench's
 * gpu_launches count); bc_reset_launch_count() zeroes it. */
int64_t bc_launch_count(void);
void bc_reset_launch_count(void);

#ifdef __cplusplus
}
#endif

#endif /* BARRACUDA_H */
