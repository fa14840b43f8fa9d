/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU definitions of every operation on the hot path of
 * Nelson et al., "Generating Efficient Tensor Contractions for GPUs" (ICPP 2015), as
 * restated in SURVEY.md §8(c).  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_icpp_nelsonrbhhjn15_b200/) never links, imports or calls it, and the
 * two share no code, headers, tables or constant generators.
 *
 * Arithmetic: IEEE fp64, compiled -O2 -ffp-contract=off (no FMA contraction, no
 * fast-math), summation in ascending index order.  OpenMP parallelises only over
 * independent elements / output tiles, never inside a sum, so the result does not
 * depend on the thread count.
 *
 * "P:<lines>" = /root/reference/PAPER.md line numbers.
 *
 * Parity pins (tests/test_oracle_*.py, -m "not gpu"):
 *   sumfact3d_def  : numpy.kron form (C (x) B (x) A) vec(U); identity/permutation
 *                    operators (bitwise); separable U (closed form); paper-form
 *                    relabelling + transcription of Fig. 2(c)/(d) (bitwise, integers)
 *   sumfact3d      : == sumfact3d_def bitwise on integer data; all of the above
 *   sumfact2d(_def): numpy matmul B U A^T; paper 2-D form P:82-91 relabelled (bitwise)
 *   local_grad3    : D = I copies (bitwise); == sumfact3d with identity factors;
 *                    exact GLL differentiation of polynomials of degree <= p
 *   local_grad3_t  : adjoint identity <Lg3 u, w> = <u, Lg3t w> ; D = I sums
 *   ccsdt_d1/d2    : reshaped numpy.matmul GEMM, unequal extents, bitwise on integers;
 *                    one-hot bookkeeping; sign = antisymmetriser parity
 *   ccsdt_s1       : brute-force outer product; one-hot bookkeeping
 *   sumsq / energy : math.fsum / brute force on small inputs
 */
#include <math.h>
#include <stdint.h>
#include <string.h>

#define EXPORT __attribute__((visibility("default")))

/* ------------------------------------------------------------------------------------
 * Spectral family.  Row-major, elements contiguous, last index fastest (P:201, 241-242,
 * 521 "access: linearize", "assuming row-major layout").  P1 = p + 1 points per axis
 * (sums run 0..p).
 * ---------------------------------------------------------------------------------- */

/* sumfact3d, Level 0 (the definition).  BASELINE.json north_star form
 *   V[e][i][j][k] = sum_{l,m,n} A[k][n] * B[j][m] * C[i][l] * U[e][l][m][n]
 * which is Eq. (1) (Fig. 2(a)) after the relabelling of
 * DESIGN.md reading R1.  The 6-deep loop is the paper's naive nest.
 * Product evaluated ((A*B)*C)*U, sum in (l, m, n) lexicographic order.  O(P1^6). */
EXPORT void oracle_sumfact3d_def(int64_t N, int p, const double* A, const double* B,
                                 const double* C, const double* U, double* V) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1 * P1;
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < N; ++e) {
        const double* u = U + e * S;
        double* v = V + e * S;
        for (int i = 0; i < P1; ++i)
            for (int j = 0; j < P1; ++j)
                for (int k = 0; k < P1; ++k) {
                    double acc = 0.0;
                    for (int l = 0; l < P1; ++l)
                        for (int m = 0; m < P1; ++m)
                            for (int n = 0; n < P1; ++n)
                                acc += A[k * P1 + n] * B[j * P1 + m] * C[i * P1 + l] *
                                       u[(l * P1 + m) * P1 + n];
                    v[(i * P1 + j) * P1 + k] = acc;
                }
    }
}

/* sumfact3d, Level 1 (sum factorisation; OCTOPI output P:439-459 and TCR
 * input Fig. 2(b): contract U's fastest index first).  Three passes:
 *   S1  W1[l][m][k] = sum_n A[k][n] U[l][m][n]
 *   S2  W2[l][j][k] = sum_m B[j][m] W1[l][m][k]
 *   S3  V [i][j][k] = sum_l C[i][l] W2[l][j][k]        (overwrite: reading R3)
 * Ascending-index summation, per-element scratch.  O(P1^4) per element. */
EXPORT void oracle_sumfact3d(int64_t N, int p, const double* A, const double* B,
                             const double* C, const double* U, double* V) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1 * P1;
#pragma omp parallel
    {
        double W1[16 * 16 * 16], W2[16 * 16 * 16];
#pragma omp for schedule(static)
        for (int64_t e = 0; e < N; ++e) {
            const double* u = U + e * S;
            double* v = V + e * S;
            for (int l = 0; l < P1; ++l)
                for (int m = 0; m < P1; ++m)
                    for (int k = 0; k < P1; ++k) {
                        double acc = 0.0;
                        for (int n = 0; n < P1; ++n) acc += A[k * P1 + n] * u[(l * P1 + m) * P1 + n];
                        W1[(l * P1 + m) * P1 + k] = acc;
                    }
            for (int l = 0; l < P1; ++l)
                for (int j = 0; j < P1; ++j)
                    for (int k = 0; k < P1; ++k) {
                        double acc = 0.0;
                        for (int m = 0; m < P1; ++m) acc += B[j * P1 + m] * W1[(l * P1 + m) * P1 + k];
                        W2[(l * P1 + j) * P1 + k] = acc;
                    }
            for (int i = 0; i < P1; ++i)
                for (int j = 0; j < P1; ++j)
                    for (int k = 0; k < P1; ++k) {
                        double acc = 0.0;
                        for (int l = 0; l < P1; ++l) acc += C[i * P1 + l] * W2[(l * P1 + j) * P1 + k];
                        v[(i * P1 + j) * P1 + k] = acc;
                    }
        }
    }
}

/* sumfact2d, Level 0.  2-D contraction of P:82-91 in the repo's form (reading R2):
 *   V[e][i][j] = sum_{l,m} B[i][l] * A[j][m] * U[e][l][m]          (V = B U A^T) */
EXPORT void oracle_sumfact2d_def(int64_t N, int p, const double* A, const double* B,
                                 const double* U, double* V) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1;
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < N; ++e) {
        const double* u = U + e * S;
        double* v = V + e * S;
        for (int i = 0; i < P1; ++i)
            for (int j = 0; j < P1; ++j) {
                double acc = 0.0;
                for (int l = 0; l < P1; ++l)
                    for (int m = 0; m < P1; ++m) acc += B[i * P1 + l] * A[j * P1 + m] * u[l * P1 + m];
                v[i * P1 + j] = acc;
            }
    }
}

/* sumfact2d, Level 1 ("compute W_il = B_ik U_kl followed by V_ij = A_lj W_il",
 * in the repo's form):  W[l][j] = sum_m A[j][m] U[l][m];  V[i][j] = sum_l B[i][l] W[l][j]. */
EXPORT void oracle_sumfact2d(int64_t N, int p, const double* A, const double* B,
                             const double* U, double* V) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1;
#pragma omp parallel
    {
        double W[16 * 16];
#pragma omp for schedule(static)
        for (int64_t e = 0; e < N; ++e) {
            const double* u = U + e * S;
            double* v = V + e * S;
            for (int l = 0; l < P1; ++l)
                for (int j = 0; j < P1; ++j) {
                    double acc = 0.0;
                    for (int m = 0; m < P1; ++m) acc += A[j * P1 + m] * u[l * P1 + m];
                    W[l * P1 + j] = acc;
                }
            for (int i = 0; i < P1; ++i)
                for (int j = 0; j < P1; ++j) {
                    double acc = 0.0;
                    for (int l = 0; l < P1; ++l) acc += B[i * P1 + l] * W[l * P1 + j];
                    v[i * P1 + j] = acc;
                }
        }
    }
}

/* local_grad3 (Table I P:667 "local grad3 from Nekbone"; Nekbone [11,30]).
 * Nekbone stores u(i,j,k) with i fastest, i.e. C order U[e][k][j][i] (reading R5).
 *   ur[k][j][i] = sum_l D[i][l] U[k][j][l]
 *   us[k][j][i] = sum_l D[j][l] U[k][l][i]
 *   ut[k][j][i] = sum_l D[k][l] U[l][j][i]                           (overwrite) */
EXPORT void oracle_local_grad3(int64_t N, int p, const double* D, const double* U,
                               double* ur, double* us, double* ut) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1 * P1;
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < N; ++e) {
        const double* u = U + e * S;
        for (int k = 0; k < P1; ++k)
            for (int j = 0; j < P1; ++j)
                for (int i = 0; i < P1; ++i) {
                    double ar = 0.0, as = 0.0, at = 0.0;
                    for (int l = 0; l < P1; ++l) ar += D[i * P1 + l] * u[(k * P1 + j) * P1 + l];
                    for (int l = 0; l < P1; ++l) as += D[j * P1 + l] * u[(k * P1 + l) * P1 + i];
                    for (int l = 0; l < P1; ++l) at += D[k * P1 + l] * u[(l * P1 + j) * P1 + i];
                    const int64_t o = e * S + (k * P1 + j) * P1 + i;
                    ur[o] = ar;
                    us[o] = as;
                    ut[o] = at;
                }
    }
}

/* local_grad3_t (Table I P:668 "local grad3t from Nekbone"): the
 * transpose of local_grad3 applied to (ur, us, ut), summed:
 *   u[k][j][i] = sum_l D[l][i] ur[k][j][l] + sum_l D[l][j] us[k][l][i]
 *              + sum_l D[l][k] ut[l][j][i]                                (overwrite)
 * The three partial sums are formed separately and added in the order r, s, t. */
EXPORT void oracle_local_grad3_t(int64_t N, int p, const double* D, const double* ur,
                                 const double* us, const double* ut, double* U) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1 * P1;
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < N; ++e) {
        const double* r = ur + e * S;
        const double* s = us + e * S;
        const double* t = ut + e * S;
        for (int k = 0; k < P1; ++k)
            for (int j = 0; j < P1; ++j)
                for (int i = 0; i < P1; ++i) {
                    double ar = 0.0, as = 0.0, at = 0.0;
                    for (int l = 0; l < P1; ++l) ar += D[l * P1 + i] * r[(k * P1 + j) * P1 + l];
                    for (int l = 0; l < P1; ++l) as += D[l * P1 + j] * s[(k * P1 + l) * P1 + i];
                    for (int l = 0; l < P1; ++l) at += D[l * P1 + k] * t[(l * P1 + j) * P1 + i];
                    U[e * S + (k * P1 + j) * P1 + i] = (ar + as) + at;
                }
    }
}

/* Nekbone element operator ax_e ("jointly optimizing
 * lgrad3, lgrad3t and adjacent code" P:1208-1211):
 *   (ur,us,ut) = local_grad3(D, U);
 *   wr = g0 ur + g1 us + g2 ut;  ws = g1 ur + g3 us + g4 ut;  wt = g2 ur + g4 us + g5 ut
 *   W  = local_grad3_t(D, wr, ws, wt)
 * G[e][6][P1^3] holds the six symmetric geometric factors per point (reading R22). */
EXPORT void oracle_ax_e(int64_t N, int p, const double* D, const double* U, const double* G,
                        double* W) {
    const int P1 = p + 1;
    const int64_t S = (int64_t)P1 * P1 * P1;
#pragma omp parallel
    {
        double r[4096], s[4096], t[4096], wr[4096], ws[4096], wt[4096];
#pragma omp for schedule(static)
        for (int64_t e = 0; e < N; ++e) {
            oracle_local_grad3(1, p, D, U + e * S, r, s, t);
            const double* g = G + e * 6 * S;
            for (int64_t q = 0; q < S; ++q) {
                wr[q] = (g[0 * S + q] * r[q] + g[1 * S + q] * s[q]) + g[2 * S + q] * t[q];
                ws[q] = (g[1 * S + q] * r[q] + g[3 * S + q] * s[q]) + g[4 * S + q] * t[q];
                wt[q] = (g[2 * S + q] * r[q] + g[4 * S + q] * s[q]) + g[5 * S + q] * t[q];
            }
            oracle_local_grad3_t(1, p, D, wr, ws, wt, W + e * S);
        }
    }
}

/* ------------------------------------------------------------------------------------
 * CCSD(T) triples, NWChem loop-driven kernels [7].
 * Fortran column-major: first-listed index fastest.  Extents are given per NAME
 * (h1,h2,h3,p4,p5,p6,k); a position takes the extent of the name stored there.
 *   d1:  t3[sigma_v(h3,h2,h1,p6,p5,p4)] += s_v * sum_h7 t2[h7,p4,p5,h1] * v2[h3,h2,p6,h7]
 *   d2:  t3[sigma_v(h3,h2,h1,p6,p5,p4)] += s_v * sum_p7 t2[p7,p4,h1,h2] * v2[p7,h3,p6,p5]
 *   s1:  t3[sigma_v(h3,h2,h1,p6,p5,p4)] += s_v * t1[p4,h1] * v2[h3,h2,p6,p5]
 * Storage orders and signs: the table of DESIGN.md reading R12,
 * written out literally below, one string per NWChem subroutine.
 * ---------------------------------------------------------------------------------- */

/* name ids */
enum { H1 = 0, H2 = 1, H3 = 2, P4 = 3, P5 = 4, P6 = 5, KK = 6 };

typedef struct { int order[6]; int sign; } t3_variant;

/* sd_t_d1_1 .. sd_t_d1_9: triplesx(<order>) (+|-)= t2sub(h7,p4,p5,h1)*v2sub(h3,h2,p6,h7) */
static const t3_variant D1[9] = {
    {{H3, H2, H1, P6, P5, P4}, -1},  /* d1_1 */
    {{H3, H1, H2, P6, P5, P4}, +1},  /* d1_2 */
    {{H1, H3, H2, P6, P5, P4}, -1},  /* d1_3 */
    {{H3, H2, H1, P5, P4, P6}, -1},  /* d1_4 */
    {{H3, H1, H2, P5, P4, P6}, +1},  /* d1_5 */
    {{H1, H3, H2, P5, P4, P6}, -1},  /* d1_6 */
    {{H3, H2, H1, P5, P6, P4}, +1},  /* d1_7 */
    {{H3, H1, H2, P5, P6, P4}, -1},  /* d1_8 */
    {{H1, H3, H2, P5, P6, P4}, +1},  /* d1_9 */
};
/* sd_t_d2_1 .. sd_t_d2_9: triplesx(<order>) (+|-)= t2sub(p7,p4,h1,h2)*v2sub(p7,h3,p6,p5) */
static const t3_variant D2[9] = {
    {{H3, H2, H1, P6, P5, P4}, -1},  /* d2_1 */
    {{H2, H1, H3, P6, P5, P4}, -1},  /* d2_2 */
    {{H2, H3, H1, P6, P5, P4}, +1},  /* d2_3 */
    {{H3, H2, H1, P6, P4, P5}, +1},  /* d2_4 */
    {{H2, H1, H3, P6, P4, P5}, +1},  /* d2_5 */
    {{H2, H3, H1, P6, P4, P5}, -1},  /* d2_6 */
    {{H3, H2, H1, P4, P6, P5}, -1},  /* d2_7 */
    {{H2, H1, H3, P4, P6, P5}, -1},  /* d2_8 */
    {{H2, H3, H1, P4, P6, P5}, +1},  /* d2_9 */
};
/* sd_t_s1_1 .. sd_t_s1_9: triplesx(<order>) (+|-)= t1sub(p4,h1)*v2sub(h3,h2,p6,p5) */
static const t3_variant S1[9] = {
    {{H3, H2, H1, P6, P5, P4}, +1},  /* s1_1 */
    {{H3, H1, H2, P6, P5, P4}, -1},  /* s1_2 */
    {{H1, H3, H2, P6, P5, P4}, +1},  /* s1_3 */
    {{H3, H2, H1, P6, P4, P5}, -1},  /* s1_4 */
    {{H3, H1, H2, P6, P4, P5}, +1},  /* s1_5 */
    {{H1, H3, H2, P6, P4, P5}, -1},  /* s1_6 */
    {{H3, H2, H1, P4, P6, P5}, +1},  /* s1_7 */
    {{H3, H1, H2, P4, P6, P5}, -1},  /* s1_8 */
    {{H1, H3, H2, P4, P6, P5}, +1},  /* s1_9 */
};

/* Fortran offset of a named index tuple stored in `order` (first = fastest). */
static int64_t t3_offset(const int order[6], const int idx[7], const int ext[7]) {
    int64_t off = 0;
    for (int q = 5; q >= 0; --q) off = off * ext[order[q]] + idx[order[q]];
    return off;
}

/* ext[7] = {h1d, h2d, h3d, p4d, p5d, p6d, kd}.  7-deep loop, contracted index innermost,
 * one t3 element per (p4,p5,p6,h1,h2,h3) updated once with the full sum. */
EXPORT void oracle_ccsdt_d1(int variant, const int* ext, double* t3, const double* t2,
                            const double* v2) {
    const t3_variant* tv = &D1[variant - 1];
    const int h1d = ext[H1], h2d = ext[H2], h3d = ext[H3], p4d = ext[P4], p5d = ext[P5],
              p6d = ext[P6], h7d = ext[KK];
#pragma omp parallel for collapse(2) schedule(static)
    for (int p4 = 0; p4 < p4d; ++p4)
        for (int p5 = 0; p5 < p5d; ++p5)
            for (int p6 = 0; p6 < p6d; ++p6)
                for (int h1 = 0; h1 < h1d; ++h1)
                    for (int h2 = 0; h2 < h2d; ++h2)
                        for (int h3 = 0; h3 < h3d; ++h3) {
                            double acc = 0.0;
                            for (int h7 = 0; h7 < h7d; ++h7) {
                                const double a = t2[h7 + (int64_t)h7d * (p4 + (int64_t)p4d * (p5 + (int64_t)p5d * h1))];
                                const double b = v2[h3 + (int64_t)h3d * (h2 + (int64_t)h2d * (p6 + (int64_t)p6d * h7))];
                                acc += a * b;
                            }
                            const int idx[7] = {h1, h2, h3, p4, p5, p6, 0};
                            t3[t3_offset(tv->order, idx, ext)] += tv->sign * acc;
                        }
}

EXPORT void oracle_ccsdt_d2(int variant, const int* ext, double* t3, const double* t2,
                            const double* v2) {
    const t3_variant* tv = &D2[variant - 1];
    const int h1d = ext[H1], h2d = ext[H2], h3d = ext[H3], p4d = ext[P4], p5d = ext[P5],
              p6d = ext[P6], p7d = ext[KK];
#pragma omp parallel for collapse(2) schedule(static)
    for (int p4 = 0; p4 < p4d; ++p4)
        for (int p5 = 0; p5 < p5d; ++p5)
            for (int p6 = 0; p6 < p6d; ++p6)
                for (int h1 = 0; h1 < h1d; ++h1)
                    for (int h2 = 0; h2 < h2d; ++h2)
                        for (int h3 = 0; h3 < h3d; ++h3) {
                            double acc = 0.0;
                            for (int p7 = 0; p7 < p7d; ++p7) {
                                const double a = t2[p7 + (int64_t)p7d * (p4 + (int64_t)p4d * (h1 + (int64_t)h1d * h2))];
                                const double b = v2[p7 + (int64_t)p7d * (h3 + (int64_t)h3d * (p6 + (int64_t)p6d * p5))];
                                acc += a * b;
                            }
                            const int idx[7] = {h1, h2, h3, p4, p5, p6, 0};
                            t3[t3_offset(tv->order, idx, ext)] += tv->sign * acc;
                        }
}

EXPORT void oracle_ccsdt_s1(int variant, const int* ext, double* t3, const double* t1,
                            const double* v2) {
    const t3_variant* tv = &S1[variant - 1];
    const int h1d = ext[H1], h2d = ext[H2], h3d = ext[H3], p4d = ext[P4], p5d = ext[P5],
              p6d = ext[P6];
#pragma omp parallel for collapse(2) schedule(static)
    for (int p4 = 0; p4 < p4d; ++p4)
        for (int p5 = 0; p5 < p5d; ++p5)
            for (int p6 = 0; p6 < p6d; ++p6)
                for (int h1 = 0; h1 < h1d; ++h1)
                    for (int h2 = 0; h2 < h2d; ++h2)
                        for (int h3 = 0; h3 < h3d; ++h3) {
                            const double a = t1[p4 + (int64_t)p4d * h1];
                            const double b = v2[h3 + (int64_t)h3d * (h2 + (int64_t)h2d * (p6 + (int64_t)p6d * p5))];
                            const int idx[7] = {h1, h2, h3, p4, p5, p6, 0};
                            t3[t3_offset(tv->order, idx, ext)] += tv->sign * (a * b);
                        }
}

/* Storage order and sign of a variant, for tests (family 1 = d1, 2 = d2, 3 = s1). */
EXPORT int oracle_ccsdt_variant(int family, int variant, int* order6) {
    const t3_variant* t = (family == 1 ? D1 : family == 2 ? D2 : S1) + (variant - 1);
    for (int q = 0; q < 6; ++q) order6[q] = t->order[q];
    return t->sign;
}

/* ------------------------------------------------------------------------------------
 * Check scalars (SURVEY §8(c) reading R18).  Plain sequential sums, ascending index.
 * ---------------------------------------------------------------------------------- */
EXPORT double oracle_sumsq(int64_t n, const double* x) {
    double s = 0.0;
    for (int64_t i = 0; i < n; ++i) s += x[i] * x[i];
    return s;
}

/* E = sum over t3 (canonical order h3,h2,h1,p6,p5,p4, Fortran) of t3^2 / denom,
 * denom = eps_h3[h3] + eps_h2[h2] + eps_h1[h1] - eps_p6[p6] - eps_p5[p5] - eps_p4[p4].
 * eps_h = [eps_h1 (h1d) | eps_h2 (h2d) | eps_h3 (h3d)], eps_p = [eps_p4 | eps_p5 | eps_p6]. */
EXPORT double oracle_energy(const int* ext, const double* t3, const double* eps_h,
                            const double* eps_p) {
    const int h1d = ext[H1], h2d = ext[H2], h3d = ext[H3], p4d = ext[P4], p5d = ext[P5],
              p6d = ext[P6];
    const double* e1 = eps_h;
    const double* e2 = eps_h + h1d;
    const double* e3 = eps_h + h1d + h2d;
    const double* f4 = eps_p;
    const double* f5 = eps_p + p4d;
    const double* f6 = eps_p + p4d + p5d;
    double E = 0.0;
    int64_t x = 0;
    for (int p4 = 0; p4 < p4d; ++p4)
        for (int p5 = 0; p5 < p5d; ++p5)
            for (int p6 = 0; p6 < p6d; ++p6)
                for (int h1 = 0; h1 < h1d; ++h1)
                    for (int h2 = 0; h2 < h2d; ++h2)
                        for (int h3 = 0; h3 < h3d; ++h3, ++x) {
                            const double den = ((((e3[h3] + e2[h2]) + e1[h1]) - f6[p6]) - f5[p5]) - f4[p4];
                            E += t3[x] * t3[x] / den;
                        }
    return E;
}
