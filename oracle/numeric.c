/*
 * numeric.c -- the CPU ORACLE's dense steps of the factor-update (F-U) call,
 * in plain C with OpenMP on loops only.  No BLAS/LAPACK: results stay
 * independent of any vendor library.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle/__init__.py): called by oracle/numeric.py,
 * which only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may import.  Shares no code with the product.
 *
 * What it computes, in the paper's order [PAPER.md L27 Sec. II-A, Fig. 1 L33-65]
 * on one dense frontal matrix F (f x f, column-major, leading dimension ld,
 * lower triangle valid), k pivot columns, m = f - k:
 *   potrf:  F[0:k,0:k] = L1 L1^T              (textbook column algorithm)
 *   trsm:   L2 = F[k:f,0:k] L1^{-T}           (substitution, column by column)
 *   syrk:   U  = F[k:f,k:f] - L2 L2^T          (lower triangle incl. diagonal)
 * plus the extend-add F[map[i], map[j]] += U_c[i, j] (i >= j) and the two
 * supernodal triangular solves of PAPER.md L7.
 *
 * "Loops may be cache-blocked and OpenMP-parallel":
 * each step is the textbook loop nest with its loops tiled -- the blocked
 * potrf is the column algorithm on a 64-column diagonal block followed by the
 * same trsm/syrk arithmetic on the rest of L1; the only building block is
 * C[i][j] -= sum_p A[i][p] * B[j][p] (gemm_nt below), a register-tiled triple
 * loop.  Every sum is over exactly the products the definition names; only
 * the order of those additions differs from the unblocked loops (rounding).
 * Division and sqrt are the correctly rounded IEEE operations (reading C9).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define IDX(i, j, ld) ((int64_t)(i) + (int64_t)(j) * (int64_t)(ld))

/* ------------------------------------------------------------------------
 * gemm_nt: C[i][j] -= sum_{p<K} A[i][p] * B[j][p], 0 <= i < M, 0 <= j < N,
 * and with lower != 0 only the entries with i >= j.  All matrices are
 * column-major.  Tiling: C in MC x NC tiles (one OpenMP task each); the inner
 * dimension in KC chunks; inside a tile an MR x NR block of C lives in
 * registers while p runs over the chunk (so each chunk's products are summed
 * into a local accumulator from 0, then subtracted from C).  The operands of a
 * chunk are first copied ("packed") into contiguous buffers so that the inner
 * loop reads them sequentially -- a copy, no arithmetic.
 * ---------------------------------------------------------------------- */
enum { MR = 8, NR = 4, MC = 128, NC = 128, KC = 256 };

typedef double v4d __attribute__((vector_size(32)));

/* The MR x NR register block: acc[r][c] = sum_p a[p][r] * b[p][c]. */
static void micro_kernel(int64_t kc, const double *a, const double *b, double acc[MR * NR]) {
    v4d c00 = {0}, c01 = {0}, c02 = {0}, c03 = {0};   /* rows 0-3, columns 0..3 */
    v4d c10 = {0}, c11 = {0}, c12 = {0}, c13 = {0};   /* rows 4-7 */
    for (int64_t p = 0; p < kc; p++) {
        v4d a0, a1;
        memcpy(&a0, a + p * MR, sizeof a0);
        memcpy(&a1, a + p * MR + 4, sizeof a1);
        const double *bp = b + p * NR;
        c00 += a0 * bp[0]; c10 += a1 * bp[0];
        c01 += a0 * bp[1]; c11 += a1 * bp[1];
        c02 += a0 * bp[2]; c12 += a1 * bp[2];
        c03 += a0 * bp[3]; c13 += a1 * bp[3];
    }
    v4d cols0[NR] = {c00, c01, c02, c03}, cols1[NR] = {c10, c11, c12, c13};
    for (int c = 0; c < NR; c++)
        for (int r = 0; r < 4; r++) {
            acc[r + c * MR] = cols0[c][r];
            acc[4 + r + c * MR] = cols1[c][r];
        }
}

/* Copy rows [i0, i0+mc) x columns [p0, p0+kc) of column-major X into panels of
 * R rows: dst[(i / R) * kc * R + p * R + i % R]; rows past mc are zero. */
static void pack(const double *X, int64_t ldx, int64_t i0, int64_t mc, int64_t p0, int64_t kc, int R,
                 double *dst) {
    for (int64_t ib = 0; ib < mc; ib += R) {
        double *d = dst + (ib / R) * kc * R;
        const int64_t rr = mc - ib < R ? mc - ib : R;
        for (int64_t p = 0; p < kc; p++) {
            const double *src = X + IDX(i0 + ib, p0 + p, ldx);
            int64_t r = 0;
            for (; r < rr; r++) d[p * R + r] = src[r];
            for (; r < R; r++) d[p * R + r] = 0.0;
        }
    }
}

static void gemm_nt(double *C, int64_t ldc, const double *A, int64_t lda, const double *B, int64_t ldb, int64_t M,
                    int64_t N, int64_t K, int lower) {
    if (M <= 0 || N <= 0 || K <= 0) return;
    const int64_t tm = (M + MC - 1) / MC, tn = (N + NC - 1) / NC;
#pragma omp parallel if (tm * tn > 1)
    {
        double *pa = (double *)aligned_alloc(64, sizeof(double) * MC * KC);
        double *pb = (double *)aligned_alloc(64, sizeof(double) * NC * KC);
#pragma omp for schedule(dynamic, 1) collapse(2)
        for (int64_t ti = 0; ti < tm; ti++)
            for (int64_t tj = 0; tj < tn; tj++) {
                const int64_t i0 = ti * MC, j0 = tj * NC;
                const int64_t mc = M - i0 < MC ? M - i0 : MC, nc = N - j0 < NC ? N - j0 : NC;
                if (lower && i0 + mc <= j0) continue;          /* tile wholly above the diagonal */
                for (int64_t p0 = 0; p0 < K; p0 += KC) {
                    const int64_t kc = K - p0 < KC ? K - p0 : KC;
                    pack(A, lda, i0, mc, p0, kc, MR, pa);
                    pack(B, ldb, j0, nc, p0, kc, NR, pb);
                    for (int64_t jb = 0; jb < nc; jb += NR)
                        for (int64_t ib = 0; ib < mc; ib += MR) {
                            if (lower && i0 + ib + MR <= j0 + jb) continue;
                            double acc[MR * NR];
                            micro_kernel(kc, pa + (ib / MR) * kc * MR, pb + (jb / NR) * kc * NR, acc);
                            for (int c = 0; c < NR && jb + c < nc; c++)
                                for (int r = 0; r < MR && ib + r < mc; r++) {
                                    const int64_t i = i0 + ib + r, j = j0 + jb + c;
                                    if (lower && i < j) continue;
                                    C[IDX(i, j, ldc)] -= acc[r + c * MR];
                                }
                        }
                }
            }
        free(pa);
        free(pb);
    }
}

/* ------------------------------------------------------------------------
 * Column algorithm on a small diagonal block T (n x n, ld), in place:
 * for j: L_jj = sqrt(T_jj); L_ij = T_ij / L_jj (i > j);
 *        T_ab -= L_aj L_bj for j < b <= a   (right-looking, "textbook").
 * Returns 0, or 1 + the first column whose pivot is <= 0 or NaN (reading C8).
 * ---------------------------------------------------------------------- */
static int64_t potrf_column(double *T, int64_t ld, int64_t n) {
    for (int64_t j = 0; j < n; j++) {
        const double d = T[IDX(j, j, ld)];
        if (!(d > 0.0)) return j + 1;
        const double l = sqrt(d);
        T[IDX(j, j, ld)] = l;
        for (int64_t i = j + 1; i < n; i++) T[IDX(i, j, ld)] /= l;
        for (int64_t b = j + 1; b < n; b++) {
            const double lbj = T[IDX(b, j, ld)];
            for (int64_t a = b; a < n; a++) T[IDX(a, b, ld)] -= T[IDX(a, j, ld)] * lbj;
        }
    }
    return 0;
}

/* X (rows x n, ldx) <- X L^{-T}, L = lower n x n (ldl): for each row x,
 * x_j = (x_j - sum_{p<j} x_p L_jp) / L_jj, by columns (right-looking), rows in
 * parallel. */
static void trsm_column(double *X, int64_t ldx, int64_t rows, const double *L, int64_t ldl, int64_t n) {
    const int64_t RB = 256;
#pragma omp parallel for schedule(static) if (rows > RB)
    for (int64_t r0 = 0; r0 < rows; r0 += RB) {
        const int64_t r1 = r0 + RB < rows ? r0 + RB : rows;
        for (int64_t j = 0; j < n; j++) {
            const double ljj = L[IDX(j, j, ldl)];
            double *xj = X + IDX(0, j, ldx);
            for (int64_t i = r0; i < r1; i++) xj[i] /= ljj;
            for (int64_t b = j + 1; b < n; b++) {
                const double lbj = L[IDX(b, j, ldl)];
                double *xb = X + IDX(0, b, ldx);
                for (int64_t i = r0; i < r1; i++) xb[i] -= xj[i] * lbj;
            }
        }
    }
}

enum { NB = 64 };   /* diagonal block width of the blocked potrf / trsm */

/* potrf on the k x k block (blocked right-looking: column algorithm on each
 * NB-wide diagonal block, trsm of the rows below it inside L1, syrk of the
 * rest of L1).  Returns 0 or 1 + failing column. */
static int64_t potrf_blocked(double *F, int64_t ld, int64_t k) {
    for (int64_t j0 = 0; j0 < k; j0 += NB) {
        const int64_t jb = k - j0 < NB ? k - j0 : NB;
        double *D = F + IDX(j0, j0, ld);
        const int64_t info = potrf_column(D, ld, jb);
        if (info) return j0 + info;
        const int64_t rest = k - j0 - jb;
        if (rest > 0) {
            double *P = F + IDX(j0 + jb, j0, ld);             /* rows below the block */
            trsm_column(P, ld, rest, D, ld, jb);
            gemm_nt(F + IDX(j0 + jb, j0 + jb, ld), ld, P, ld, P, ld, rest, rest, jb, 1);
        }
    }
    return 0;
}

/* trsm L2 = F21 L1^{-T} (m x k), blocked over NB-column blocks of L1: block J
 * first subtracts the already-solved columns 0..J-1 (X[:,J] -= X[:,0:J0] L1[J,0:J0]^T),
 * then solves with the diagonal block by substitution. */
static void trsm_blocked(double *X, int64_t ldx, int64_t m, const double *L1, int64_t ldl, int64_t k) {
    for (int64_t j0 = 0; j0 < k; j0 += NB) {
        const int64_t jb = k - j0 < NB ? k - j0 : NB;
        if (j0 > 0) gemm_nt(X + IDX(0, j0, ldx), ldx, X, ldx, L1 + IDX(j0, 0, ldl), ldl, m, jb, j0, 0);
        trsm_column(X + IDX(0, j0, ldx), ldx, m, L1 + IDX(j0, j0, ldl), ldl, jb);
    }
}

/* One F-U call on the dense front F (f x f, ld): potrf, trsm, syrk in place.
 * On return F[:, 0:k] holds [L1; L2] (upper triangle of L1 untouched) and
 * F[k:f, k:f] (lower) holds U.  Returns 0, or 1 + the first failing column. */
int64_t oracle_front_fu(double *F, int64_t ld, int64_t f, int64_t k) {
    const int64_t m = f - k;
    const int64_t info = potrf_blocked(F, ld, k);                        /* potrf */
    if (info) return info;
    if (m > 0) {
        trsm_blocked(F + IDX(k, 0, ld), ld, m, F, ld, k);                 /* trsm  */
        gemm_nt(F + IDX(k, k, ld), ld, F + IDX(k, 0, ld), ld, F + IDX(k, 0, ld), ld, m, m, k, 1); /* syrk */
    }
    return 0;
}

/* Extend-add: F[map[i], map[j]] += U[i, j] for i >= j, U m x m
 * column-major (ldu), map ascending positions in the parent's row list. */
void oracle_extend_add(double *F, int64_t ld, const double *U, int64_t ldu, int64_t m, const int64_t *map) {
#pragma omp parallel for schedule(dynamic, 16) if (m > 256)
    for (int64_t j = 0; j < m; j++) {
        double *Fc = F + IDX(0, map[j], ld);
        const double *Uc = U + IDX(0, j, ldu);
        for (int64_t i = j; i < m; i++) Fc[map[i]] += Uc[i];
    }
}

/* Supernodal forward step (L y = b): with the panel P = [L1; L2]
 * (f x k, ldp), y1 <- L1^{-1} y1 (forward substitution), y2 <- y2 - L2 y1. */
void oracle_panel_forward(const double *P, int64_t ldp, int64_t f, int64_t k, double *y1, double *y2) {
    for (int64_t j = 0; j < k; j++) {
        y1[j] /= P[IDX(j, j, ldp)];
        for (int64_t i = j + 1; i < k; i++) y1[i] -= P[IDX(i, j, ldp)] * y1[j];
    }
    for (int64_t j = 0; j < k; j++)
        for (int64_t i = k; i < f; i++) y2[i - k] -= P[IDX(i, j, ldp)] * y1[j];
}

/* Supernodal backward step (L^T x = y): y1 <- L1^{-T} (y1 - L2^T y2). */
void oracle_panel_backward(const double *P, int64_t ldp, int64_t f, int64_t k, double *y1, const double *y2) {
    for (int64_t j = 0; j < k; j++) {
        double s = 0.0;
        for (int64_t i = k; i < f; i++) s += P[IDX(i, j, ldp)] * y2[i - k];
        y1[j] -= s;
    }
    for (int64_t j = k - 1; j >= 0; j--) {
        double s = y1[j];
        for (int64_t i = j + 1; i < k; i++) s -= P[IDX(i, j, ldp)] * y1[i];
        y1[j] = s / P[IDX(j, j, ldp)];
    }
}

/* ------------------------------------------------------------------------
 * Higher-precision REFEREE (reading C11): the plain unblocked column algorithm
 * of potrf_column above in long double (x87 extended, 64-bit significand) on a
 * whole dense n x n matrix (column-major), used only to judge how close the
 * fp64 oracle and the GPU factor are to the exact L on elasticity fronts.
 * ---------------------------------------------------------------------- */
int64_t oracle_dense_potrf_ld(long double *T, int64_t n) {
    for (int64_t j = 0; j < n; j++) {
        const long double d = T[IDX(j, j, n)];
        if (!(d > 0.0L)) return j + 1;
        const long double l = sqrtl(d);
        T[IDX(j, j, n)] = l;
        for (int64_t i = j + 1; i < n; i++) T[IDX(i, j, n)] /= l;
#pragma omp parallel for schedule(dynamic, 8)
        for (int64_t b = j + 1; b < n; b++) {
            const long double lbj = T[IDX(b, j, n)];
            if (lbj == 0.0L) continue;
            for (int64_t a = b; a < n; a++) T[IDX(a, b, n)] -= T[IDX(a, j, n)] * lbj;
        }
    }
    return 0;
}
