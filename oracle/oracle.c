/*
 * oracle/oracle.c -- plain, slow, obviously-correct CPU oracle for the xk hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or call this library.  The product path
 * (paper_conf_sc_gautierl21_b200/) never links, imports or executes anything here, and
 * this file shares no code, header, table or helper with it.
 *
 * What it computes: the BLAS level-3 operations in their textbook definition.  The paper
 * states that XKBlas' tiled algorithms "have the same behavior of those from PLASMA or
 * Chameleon" (§III) and refers to the BLAS standard [1] for the
 * operations themselves.  The definitions written out below follow
 * SURVEY.md §8(c) "Numerical oracle":
 *
 *   DGEMM  : C <- alpha*op(A)*op(B) + beta*C,  s_ij = sum_l op(A)_il*op(B)_lj as a
 *            sequential l-loop (no FMA contraction: built with -ffp-contract=off),
 *            then C_ij = alpha*s_ij + beta*C_ij.
 *   DSYRK  : C <- alpha*A*A^T + beta*C (N) / alpha*A^T*A + beta*C (T), uplo triangle only.
 *   DSYR2K : C <- alpha*A*B^T + alpha*B*A^T + beta*C (N) / A^T*B + B^T*A (T), uplo only.
 *   DSYMM  : C <- alpha*sym(A)*B + beta*C (L) / alpha*B*sym(A) + beta*C (R).
 *   DTRMM  : B <- alpha*op(tri(A))*B (L) / alpha*B*op(tri(A)) (R).
 *   DTRSM  : solve op(tri(A))*X = alpha*B (L) / X*op(tri(A)) = alpha*B (R), B <- X,
 *            by forward/back substitution in the natural order.
 *
 * BLAS "not referenced" rules: beta==0 -> C is not read; alpha==0 ->
 * A and B are not read; only the uplo triangle of A (SYMM/TRMM/TRSM) and of C
 * (SYRK/SYR2K) is touched; diag=='U' -> the diagonal of A is not read.
 * Argument errors return -i (i = position of the first invalid argument, numbered like
 * the reference BLAS XERBLA), success returns 0; the oracle never aborts.
 *
 * Parallelism: OpenMP over output columns (rows for right-side TRMM/TRSM), each output
 * element computed by one thread in a fixed order -> bitwise deterministic at any
 * thread count.
 *
 * Pins (tests/test_oracle_*.py, run with -m "not gpu"): exact-rational brute force on
 * tiny integer matrices (Python fractions), closed forms (identity, diagonal 2^p
 * scaling, rank-1 SYRK, bidiagonal TRSM with known inverse, TRSM->TRMM round trip),
 * scipy/OpenBLAS cross-checks within the north_star bound, NaN-poisoning invariants,
 * hand-worked golden fixtures under tests/golden/.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <ctype.h>

typedef int64_t i64;

/* column-major element (i,j) of an array with leading dimension ld */
#define EL(P, i, j, ld) ((P)[(i64)(i) + (i64)(j) * (i64)(ld)])

static int is_trans(char t) { t = (char)toupper((unsigned char)t); return t == 'T' || t == 'C'; }
static int ok_trans(char t) { t = (char)toupper((unsigned char)t); return t == 'N' || t == 'T' || t == 'C'; }
static int ok_uplo(char u) { u = (char)toupper((unsigned char)u); return u == 'L' || u == 'U'; }
static int ok_side(char s) { s = (char)toupper((unsigned char)s); return s == 'L' || s == 'R'; }
static int ok_diag(char d) { d = (char)toupper((unsigned char)d); return d == 'N' || d == 'U'; }
static int is_lower(char u) { return toupper((unsigned char)u) == 'L'; }
static i64 imax(i64 a, i64 b) { return a > b ? a : b; }

/* ------------------------------------------------------------------ DGEMM */
/* op(A)_il: A is m x k (N) or k x m stored (T). */
static double opA_el(int ta, const double *A, i64 lda, i64 i, i64 l)
{
    return ta ? EL(A, l, i, lda) : EL(A, i, l, lda);
}
/* op(B)_lj: B is k x n (N) or n x k stored (T). */
static double opB_el(int tb, const double *B, i64 ldb, i64 l, i64 j)
{
    return tb ? EL(B, j, l, ldb) : EL(B, l, j, ldb);
}

int oracle_dgemm(char transA, char transB, i64 m, i64 n, i64 k, double alpha,
                 const double *A, i64 lda, const double *B, i64 ldb,
                 double beta, double *C, i64 ldc)
{
    if (!ok_trans(transA)) return -1;
    if (!ok_trans(transB)) return -2;
    if (m < 0) return -3;
    if (n < 0) return -4;
    if (k < 0) return -5;
    int ta = is_trans(transA), tb = is_trans(transB);
    i64 nrowa = ta ? k : m, nrowb = tb ? n : k;
    if (lda < imax(1, nrowa)) return -8;
    if (ldb < imax(1, nrowb)) return -10;
    if (ldc < imax(1, m)) return -13;
    if (m == 0 || n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return 0;

#pragma omp parallel for schedule(static)
    for (i64 j = 0; j < n; ++j) {
        for (i64 i = 0; i < m; ++i) {
            double c;
            if (alpha == 0.0) {
                c = (beta == 0.0) ? 0.0 : beta * EL(C, i, j, ldc);
            } else {
                double s = 0.0;
                for (i64 l = 0; l < k; ++l)
                    s += opA_el(ta, A, lda, i, l) * opB_el(tb, B, ldb, l, j);
                c = (beta == 0.0) ? alpha * s : alpha * s + beta * EL(C, i, j, ldc);
            }
            EL(C, i, j, ldc) = c;
        }
    }
    return 0;
}

/* ------------------------------------------------------------------ DSYRK */
static int in_tri(int lower, i64 i, i64 j) { return lower ? (i >= j) : (i <= j); }

int oracle_dsyrk(char uplo, char trans, i64 n, i64 k, double alpha,
                 const double *A, i64 lda, double beta, double *C, i64 ldc)
{
    if (!ok_uplo(uplo)) return -1;
    if (!ok_trans(trans)) return -2;
    if (n < 0) return -3;
    if (k < 0) return -4;
    int tr = is_trans(trans);
    if (lda < imax(1, tr ? k : n)) return -7;
    if (ldc < imax(1, n)) return -10;
    if (n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return 0;
    int lower = is_lower(uplo);
#pragma omp parallel for schedule(dynamic, 4)
    for (i64 j = 0; j < n; ++j) {
        for (i64 i = 0; i < n; ++i) {
            if (!in_tri(lower, i, j)) continue;
            double c;
            if (alpha == 0.0) {
                c = (beta == 0.0) ? 0.0 : beta * EL(C, i, j, ldc);
            } else {
                double s = 0.0;
                /* op(A) is n x k: A (N) or A^T (T); C = op(A) op(A)^T */
                for (i64 l = 0; l < k; ++l)
                    s += opA_el(tr, A, lda, i, l) * opA_el(tr, A, lda, j, l);
                c = (beta == 0.0) ? alpha * s : alpha * s + beta * EL(C, i, j, ldc);
            }
            EL(C, i, j, ldc) = c;
        }
    }
    return 0;
}

/* ----------------------------------------------------------------- DSYR2K */
int oracle_dsyr2k(char uplo, char trans, i64 n, i64 k, double alpha,
                  const double *A, i64 lda, const double *B, i64 ldb,
                  double beta, double *C, i64 ldc)
{
    if (!ok_uplo(uplo)) return -1;
    if (!ok_trans(trans)) return -2;
    if (n < 0) return -3;
    if (k < 0) return -4;
    int tr = is_trans(trans);
    i64 nrow = tr ? k : n;
    if (lda < imax(1, nrow)) return -7;
    if (ldb < imax(1, nrow)) return -9;
    if (ldc < imax(1, n)) return -12;
    if (n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return 0;
    int lower = is_lower(uplo);
#pragma omp parallel for schedule(dynamic, 4)
    for (i64 j = 0; j < n; ++j) {
        for (i64 i = 0; i < n; ++i) {
            if (!in_tri(lower, i, j)) continue;
            double c;
            if (alpha == 0.0) {
                c = (beta == 0.0) ? 0.0 : beta * EL(C, i, j, ldc);
            } else {
                double s = 0.0;
                /* (op(A) op(B)^T + op(B) op(A)^T)_ij, op(X) = X (N) or X^T (T), n x k */
                for (i64 l = 0; l < k; ++l)
                    s += opA_el(tr, A, lda, i, l) * opA_el(tr, B, ldb, j, l)
                       + opA_el(tr, B, ldb, i, l) * opA_el(tr, A, lda, j, l);
                c = (beta == 0.0) ? alpha * s : alpha * s + beta * EL(C, i, j, ldc);
            }
            EL(C, i, j, ldc) = c;
        }
    }
    return 0;
}

/* ------------------------------------------------------------------ DSYMM */
/* sym(A)_il read from the uplo triangle only. */
static double sym_el(int lower, const double *A, i64 lda, i64 i, i64 l)
{
    if (in_tri(lower, i, l)) return EL(A, i, l, lda);
    return EL(A, l, i, lda);
}

int oracle_dsymm(char side, char uplo, i64 m, i64 n, double alpha,
                 const double *A, i64 lda, const double *B, i64 ldb,
                 double beta, double *C, i64 ldc)
{
    if (!ok_side(side)) return -1;
    if (!ok_uplo(uplo)) return -2;
    if (m < 0) return -3;
    if (n < 0) return -4;
    int left = toupper((unsigned char)side) == 'L';
    i64 ka = left ? m : n;
    if (lda < imax(1, ka)) return -7;
    if (ldb < imax(1, m)) return -9;
    if (ldc < imax(1, m)) return -12;
    if (m == 0 || n == 0 || (alpha == 0.0 && beta == 1.0)) return 0;
    int lower = is_lower(uplo);
#pragma omp parallel for schedule(static)
    for (i64 j = 0; j < n; ++j) {
        for (i64 i = 0; i < m; ++i) {
            double c;
            if (alpha == 0.0) {
                c = (beta == 0.0) ? 0.0 : beta * EL(C, i, j, ldc);
            } else {
                double s = 0.0;
                if (left)
                    for (i64 l = 0; l < m; ++l) s += sym_el(lower, A, lda, i, l) * EL(B, l, j, ldb);
                else
                    for (i64 l = 0; l < n; ++l) s += EL(B, i, l, ldb) * sym_el(lower, A, lda, l, j);
                c = (beta == 0.0) ? alpha * s : alpha * s + beta * EL(C, i, j, ldc);
            }
            EL(C, i, j, ldc) = c;
        }
    }
    return 0;
}

/* ------------------------------------------------------------ DTRMM/DTRSM */
/* op(tri(A))_il with A triangular (uplo), diag 'U' = implicit unit diagonal (not read). */
static double tri_op_el(int lower, int trans, int unit, const double *A, i64 lda, i64 i, i64 l)
{
    i64 r = trans ? l : i, c = trans ? i : l; /* stored coordinates */
    if (r == c) return unit ? 1.0 : EL(A, r, c, lda);
    if (!in_tri(lower, r, c)) return 0.0;
    return EL(A, r, c, lda);
}

static int check_tr(char side, char uplo, char transA, char diag, i64 m, i64 n, i64 lda, i64 ldb)
{
    if (!ok_side(side)) return -1;
    if (!ok_uplo(uplo)) return -2;
    if (!ok_trans(transA)) return -3;
    if (!ok_diag(diag)) return -4;
    if (m < 0) return -5;
    if (n < 0) return -6;
    i64 ka = toupper((unsigned char)side) == 'L' ? m : n;
    if (lda < imax(1, ka)) return -9;
    if (ldb < imax(1, m)) return -11;
    return 0;
}

int oracle_dtrmm(char side, char uplo, char transA, char diag, i64 m, i64 n, double alpha,
                 const double *A, i64 lda, double *B, i64 ldb)
{
    int info = check_tr(side, uplo, transA, diag, m, n, lda, ldb);
    if (info) return info;
    if (m == 0 || n == 0) return 0;
    int left = toupper((unsigned char)side) == 'L', lower = is_lower(uplo);
    int tr = is_trans(transA), unit = toupper((unsigned char)diag) == 'U';
    if (alpha == 0.0) {
        for (i64 j = 0; j < n; ++j)
            for (i64 i = 0; i < m; ++i) EL(B, i, j, ldb) = 0.0;
        return 0;
    }
    double *X = (double *)malloc(sizeof(double) * (size_t)(m * n));
    if (!X) return 1;
#pragma omp parallel for schedule(static)
    for (i64 j = 0; j < n; ++j) {
        for (i64 i = 0; i < m; ++i) {
            double s = 0.0;
            if (left) /* (op(A) B)_ij, op(A) m x m */
                for (i64 l = 0; l < m; ++l) s += tri_op_el(lower, tr, unit, A, lda, i, l) * EL(B, l, j, ldb);
            else /* (B op(A))_ij, op(A) n x n */
                for (i64 l = 0; l < n; ++l) s += EL(B, i, l, ldb) * tri_op_el(lower, tr, unit, A, lda, l, j);
            X[i + j * m] = alpha * s;
        }
    }
    for (i64 j = 0; j < n; ++j)
        for (i64 i = 0; i < m; ++i) EL(B, i, j, ldb) = X[i + j * m];
    free(X);
    return 0;
}

int oracle_dtrsm(char side, char uplo, char transA, char diag, i64 m, i64 n, double alpha,
                 const double *A, i64 lda, double *B, i64 ldb)
{
    int info = check_tr(side, uplo, transA, diag, m, n, lda, ldb);
    if (info) return info;
    if (m == 0 || n == 0) return 0;
    int left = toupper((unsigned char)side) == 'L', lower = is_lower(uplo);
    int tr = is_trans(transA), unit = toupper((unsigned char)diag) == 'U';
    if (alpha == 0.0) {
        for (i64 j = 0; j < n; ++j)
            for (i64 i = 0; i < m; ++i) EL(B, i, j, ldb) = 0.0;
        return 0;
    }
    /* op(tri(A)) is lower triangular iff (lower && !trans) || (!lower && trans). */
    int op_lower = lower != tr;
    if (left) {
        /* op(A) X = alpha B, column by column */
#pragma omp parallel for schedule(static)
        for (i64 j = 0; j < n; ++j) {
            if (op_lower) { /* forward substitution, i = 0 .. m-1 */
                for (i64 i = 0; i < m; ++i) {
                    double s = alpha * EL(B, i, j, ldb);
                    for (i64 l = 0; l < i; ++l) s -= tri_op_el(lower, tr, unit, A, lda, i, l) * EL(B, l, j, ldb);
                    EL(B, i, j, ldb) = unit ? s : s / tri_op_el(lower, tr, 0, A, lda, i, i);
                }
            } else { /* back substitution, i = m-1 .. 0 */
                for (i64 i = m - 1; i >= 0; --i) {
                    double s = alpha * EL(B, i, j, ldb);
                    for (i64 l = i + 1; l < m; ++l) s -= tri_op_el(lower, tr, unit, A, lda, i, l) * EL(B, l, j, ldb);
                    EL(B, i, j, ldb) = unit ? s : s / tri_op_el(lower, tr, 0, A, lda, i, i);
                }
            }
        }
    } else {
        /* X op(A) = alpha B, row by row: x_i. op(A) = alpha b_i. */
#pragma omp parallel for schedule(static)
        for (i64 i = 0; i < m; ++i) {
            if (!op_lower) { /* op(A) upper: forward in j */
                for (i64 j = 0; j < n; ++j) {
                    double s = alpha * EL(B, i, j, ldb);
                    for (i64 l = 0; l < j; ++l) s -= EL(B, i, l, ldb) * tri_op_el(lower, tr, unit, A, lda, l, j);
                    EL(B, i, j, ldb) = unit ? s : s / tri_op_el(lower, tr, 0, A, lda, j, j);
                }
            } else { /* op(A) lower: backward in j */
                for (i64 j = n - 1; j >= 0; --j) {
                    double s = alpha * EL(B, i, j, ldb);
                    for (i64 l = j + 1; l < n; ++l) s -= EL(B, i, l, ldb) * tri_op_el(lower, tr, unit, A, lda, l, j);
                    EL(B, i, j, ldb) = unit ? s : s / tri_op_el(lower, tr, 0, A, lda, j, j);
                }
            }
        }
    }
    return 0;
}

/* --------------------------------------------- sampled DGEMM entries (large-N parity) */
/* C_ref(i_s, j_s) for a list of sampled coordinates: the same dot loop as oracle_dgemm,
 * evaluated only where asked.  c0 holds the original C entries (ignored if beta == 0). */
int oracle_dgemm_sampled(char transA, char transB, i64 k, double alpha,
                         const double *A, i64 lda, const double *B, i64 ldb, double beta,
                         const double *c0, const i64 *ii, const i64 *jj, i64 ns, double *out)
{
    int ta = is_trans(transA), tb = is_trans(transB);
#pragma omp parallel for schedule(static)
    for (i64 q = 0; q < ns; ++q) {
        i64 i = ii[q], j = jj[q];
        double c;
        if (alpha == 0.0) {
            c = (beta == 0.0) ? 0.0 : beta * c0[q];
        } else {
            double s = 0.0;
            for (i64 l = 0; l < k; ++l) s += opA_el(ta, A, lda, i, l) * opB_el(tb, B, ldb, l, j);
            c = (beta == 0.0) ? alpha * s : alpha * s + beta * c0[q];
        }
        out[q] = c;
    }
    return 0;
}

int oracle_num_threads(void)
{
#ifdef _OPENMP
    extern int omp_get_max_threads(void);
    return omp_get_max_threads();
#else
    return 1;
#endif
}
