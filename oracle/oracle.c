/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of the six fp32 Level-3
 * BLAS routines whose GPU derivation is the subject of Cui, Wang, Xue, Yang,
 * Feng, "Automatic Library Generation for BLAS3 on GPUs" (IPDPS 2011),
 * /root/reference/PAPER.md (cited as P:<line>).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (its cpu_baseline leg and
 * `--impl reference` arm) may load this library.  The product path
 * (paper_conf_ipps_cuiwxyf11_b200/) never calls it; the two share no code.
 *
 * Conventions
 *   - Matrices are column-major "to be consistent with BLAS3":
 *     X(i,j) = X[i + j*ldx].  The paper's [i][j] subscripts are mathematical
 *     indices (reading Q6).
 *   - Inputs are fp32 (the paper evaluates single precision); every
 *     product of two fp32 numbers is exact in fp64 and all accumulation is in
 *     fp64, so the oracle's own error is ~K * 2^-53 (negligible).
 *   - Outputs are fp64 so the comparison is never polluted by a final
 *     rounding to fp32.
 *   - The paper defers argument semantics to BLAS3; the
 *     meaning of side/uplo/trans/diag/alpha/beta below is the reference-BLAS
 *     one.  Readings taken where the paper is silent are listed in DESIGN.md
 *     (Q3 alpha/diag in TRSM, Q7 symmetric storage by selection, Q8 blank
 *     triangle never read, Q10 TRMM in place, Q11 beta=0, Q12 alpha=0,
 *     Q13 trans='C').
 *   - Sampling: every routine computes only the output columns listed in
 *     `sel` (all columns when sel == NULL), except STRSM side='R', whose
 *     output rows are the independent unit and are listed instead.  Output t
 *     of `sel` is written to out[(.) + t*ldo].  Columns (rows) are
 *     independent, so a sampled column is exactly the full result's column.
 *
 * Loop order is j-l-i (axpy; contiguous inner loop, SURVEY EXP-2).  OpenMP
 * runs independent output columns (or rows) on separate threads; it does not
 * reorder any column's arithmetic.
 */
#include <stddef.h>
#include <stdint.h>
#include <stdlib.h>
#include <ctype.h>

#define EL(X, ld, i, j) ((X)[(int64_t)(i) + (int64_t)(j) * (int64_t)(ld)])

static int up(char c) { return toupper((unsigned char)c); }

/* op(X)(i,l) for a general matrix: transa in {N,T,C}; 'C' == 'T' for real
 * data (reading Q13). */
static double opget(const float *X, int64_t ld, int trans, int64_t i, int64_t l)
{
    return trans ? (double)EL(X, ld, l, i) : (double)EL(X, ld, i, l);
}

static int64_t selected(const int64_t *sel, int64_t t) { return sel ? sel[t] : t; }

/* -------------------------------------------------------------------------
 * SGEMM  C <- alpha*op(A)*op(B) + beta*C
 * The paper's GEMM-NN loop nest C[i][j] += A[i][k]*B[k][j] and its
 * GEMM-TN variant C[i][j] += A[k][i]*B[k][j], with BLAS scaling.
 * m x k = op(A), k x n = op(B), m x n = C.
 * ------------------------------------------------------------------------- */
void oracle_sgemm(char transa, char transb, int64_t m, int64_t n, int64_t k,
                  double alpha, const float *A, int64_t lda,
                  const float *B, int64_t ldb, double beta,
                  const float *C, int64_t ldc,
                  double *out, int64_t ldo, const int64_t *sel, int64_t nsel)
{
    int ta = up(transa) != 'N', tb = up(transb) != 'N';
    int64_t ncols = sel ? nsel : n;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t t = 0; t < ncols; ++t) {
        int64_t j = selected(sel, t);
        double *o = out + t * ldo;
        for (int64_t i = 0; i < m; ++i) o[i] = 0.0;
        if (alpha != 0.0) {                       /* alpha = 0: A, B not read (Q12) */
            for (int64_t l = 0; l < k; ++l) {
                double b = opget(B, ldb, tb, l, j);
                for (int64_t i = 0; i < m; ++i) o[i] += opget(A, lda, ta, i, l) * b;
            }
        }
        for (int64_t i = 0; i < m; ++i)
            o[i] = alpha * o[i] + (beta == 0.0 ? 0.0 : beta * (double)EL(C, ldc, i, j)); /* Q11 */
    }
}

/* -------------------------------------------------------------------------
 * SSYMM  side=L: C <- alpha*A*B + beta*C ; side=R: C <- alpha*B*A + beta*C
 * A is symmetric with only the `uplo` triangle stored (the "real area";
 * the "shadow area" is derived from it).  The shadow is obtained
 * by SELECTION Asym(i,l) = A(max,min) (lower) / A(min,max) (upper), never by
 * the addition src + src^T - diag(src) of P:95, which is only valid when the
 * unreferenced triangle holds zeros (reading Q7).
 * ------------------------------------------------------------------------- */
static double symget(const float *A, int64_t lda, int lower, int64_t i, int64_t l)
{
    int64_t hi = i > l ? i : l, lo = i > l ? l : i;
    return lower ? (double)EL(A, lda, hi, lo) : (double)EL(A, lda, lo, hi);
}

void oracle_ssymm(char side, char uplo, int64_t m, int64_t n, double alpha,
                  const float *A, int64_t lda, const float *B, int64_t ldb,
                  double beta, const float *C, int64_t ldc,
                  double *out, int64_t ldo, const int64_t *sel, int64_t nsel)
{
    int left = up(side) == 'L', lower = up(uplo) == 'L';
    int64_t ncols = sel ? nsel : n;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t t = 0; t < ncols; ++t) {
        int64_t j = selected(sel, t);
        double *o = out + t * ldo;
        for (int64_t i = 0; i < m; ++i) o[i] = 0.0;
        if (alpha != 0.0) {
            if (left) {                 /* C(:,j) = sum_l Asym(:,l) B(l,j) */
                for (int64_t l = 0; l < m; ++l) {
                    double b = EL(B, ldb, l, j);
                    for (int64_t i = 0; i < m; ++i) o[i] += symget(A, lda, lower, i, l) * b;
                }
            } else {                    /* C(:,j) = sum_l B(:,l) Asym(l,j) */
                for (int64_t l = 0; l < n; ++l) {
                    double a = symget(A, lda, lower, l, j);
                    for (int64_t i = 0; i < m; ++i) o[i] += (double)EL(B, ldb, i, l) * a;
                }
            }
        }
        for (int64_t i = 0; i < m; ++i)
            o[i] = alpha * o[i] + (beta == 0.0 ? 0.0 : beta * (double)EL(C, ldc, i, j));
    }
}

/* -------------------------------------------------------------------------
 * SSYRK  trans=N: C <- alpha*A*A^T + beta*C  (A n x k)
 *        trans=T: C <- alpha*A^T*A + beta*C  (A k x n)
 * Only the `uplo` triangle of C is referenced; the other triangle is copied
 * through unchanged so callers can check it is bit-identical.
 * ------------------------------------------------------------------------- */
void oracle_ssyrk(char uplo, char trans, int64_t n, int64_t k, double alpha,
                  const float *A, int64_t lda, double beta,
                  const float *C, int64_t ldc,
                  double *out, int64_t ldo, const int64_t *sel, int64_t nsel)
{
    int lower = up(uplo) == 'L', ta = up(trans) != 'N';
    int64_t ncols = sel ? nsel : n;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t t = 0; t < ncols; ++t) {
        int64_t j = selected(sel, t);
        int64_t i0 = lower ? j : 0, i1 = lower ? n : j + 1;   /* triangle rows of column j */
        double *o = out + t * ldo;
        for (int64_t i = 0; i < n; ++i) o[i] = (double)EL(C, ldc, i, j);  /* untouched part */
        for (int64_t i = i0; i < i1; ++i) o[i] = 0.0;
        if (alpha != 0.0) {
            for (int64_t l = 0; l < k; ++l) {
                double b = opget(A, lda, ta, j, l);            /* op(A)(j,l) */
                for (int64_t i = i0; i < i1; ++i) o[i] += opget(A, lda, ta, i, l) * b;
            }
        }
        for (int64_t i = i0; i < i1; ++i)
            o[i] = alpha * o[i] + (beta == 0.0 ? 0.0 : beta * (double)EL(C, ldc, i, j));
    }
}

/* -------------------------------------------------------------------------
 * SSYR2K trans=N: C <- alpha*(A*B^T + B*A^T) + beta*C  (A, B n x k)
 *        trans=T: C <- alpha*(A^T*B + B^T*A) + beta*C  (A, B k x n)
 * ------------------------------------------------------------------------- */
void oracle_ssyr2k(char uplo, char trans, int64_t n, int64_t k, double alpha,
                   const float *A, int64_t lda, const float *B, int64_t ldb,
                   double beta, const float *C, int64_t ldc,
                   double *out, int64_t ldo, const int64_t *sel, int64_t nsel)
{
    int lower = up(uplo) == 'L', ta = up(trans) != 'N';
    int64_t ncols = sel ? nsel : n;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t t = 0; t < ncols; ++t) {
        int64_t j = selected(sel, t);
        int64_t i0 = lower ? j : 0, i1 = lower ? n : j + 1;
        double *o = out + t * ldo;
        for (int64_t i = 0; i < n; ++i) o[i] = (double)EL(C, ldc, i, j);
        for (int64_t i = i0; i < i1; ++i) o[i] = 0.0;
        if (alpha != 0.0) {
            for (int64_t l = 0; l < k; ++l) {
                double bj = opget(B, ldb, ta, j, l), aj = opget(A, lda, ta, j, l);
                for (int64_t i = i0; i < i1; ++i)
                    o[i] += opget(A, lda, ta, i, l) * bj + opget(B, ldb, ta, i, l) * aj;
            }
        }
        for (int64_t i = i0; i < i1; ++i)
            o[i] = alpha * o[i] + (beta == 0.0 ? 0.0 : beta * (double)EL(C, ldc, i, j));
    }
}

/* -------------------------------------------------------------------------
 * Triangular operand.  Atri(i,l): the stored value strictly inside the
 * `uplo` triangle, 1 on the diagonal when diag='U' (stored value not read),
 * A(i,i) when diag='N', and 0 outside ("blank area"; never read,
 * reading Q8).  op(T)(i,l) = Atri(i,l) (transa=N) or Atri(l,i).
 * `tri_nz` says whether op(T)(i,l) lies in the nonzero region so that the
 * loops below never touch (and never multiply) blank entries.
 * ------------------------------------------------------------------------- */
static int tri_nz(int lower, int ta, int64_t i, int64_t l)
{
    int64_t r = ta ? l : i, c = ta ? i : l;        /* stored coordinates */
    return lower ? r >= c : r <= c;
}

static double triget(const float *A, int64_t lda, int lower, int ta, int unit,
                     int64_t i, int64_t l)
{
    int64_t r = ta ? l : i, c = ta ? i : l;
    if (r == c) return unit ? 1.0 : (double)EL(A, lda, r, r);
    if (lower ? r > c : r < c) return (double)EL(A, lda, r, c);
    return 0.0;
}

/* STRMM side=L: B <- alpha*op(T)*B ; side=R: B <- alpha*B*op(T).
 * BLAS overwrites B in place (reading Q10); the oracle reads the original B
 * and writes `out`, i.e. it is the definition, not an in-place schedule.  The
 * paper's TRMM-LL-N loop is C[i][j] += A[i][k]*B[k][j], k <= i. */
void oracle_strmm(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                  double alpha, const float *A, int64_t lda, const float *B, int64_t ldb,
                  double *out, int64_t ldo, const int64_t *sel, int64_t nsel)
{
    int left = up(side) == 'L', lower = up(uplo) == 'L';
    int ta = up(transa) != 'N', unit = up(diag) == 'U';
    int64_t ncols = sel ? nsel : n;
#pragma omp parallel for schedule(dynamic, 1)
    for (int64_t t = 0; t < ncols; ++t) {
        int64_t j = selected(sel, t);
        double *o = out + t * ldo;
        for (int64_t i = 0; i < m; ++i) o[i] = 0.0;
        if (alpha != 0.0) {
            if (left) {                 /* o = sum_l op(T)(:,l) B(l,j) */
                for (int64_t l = 0; l < m; ++l) {
                    double b = EL(B, ldb, l, j);
                    for (int64_t i = 0; i < m; ++i)
                        if (tri_nz(lower, ta, i, l))
                            o[i] += triget(A, lda, lower, ta, unit, i, l) * b;
                }
            } else {                    /* o = sum_l B(:,l) op(T)(l,j) */
                for (int64_t l = 0; l < n; ++l) {
                    if (!tri_nz(lower, ta, l, j)) continue;
                    double a = triget(A, lda, lower, ta, unit, l, j);
                    for (int64_t i = 0; i < m; ++i) o[i] += (double)EL(B, ldb, i, l) * a;
                }
            }
        }
        for (int64_t i = 0; i < m; ++i) o[i] *= alpha;
    }
}

/* STRSM side=L: solve op(T)*X = alpha*B ; side=R: solve X*op(T) = alpha*B.
 * X overwrites B in BLAS; here X goes to `out`.  Plain substitution in fp64:
 * the dependence B[i] <- B[k], k < i of the paper's solver loop (P:227-234,
 * TRSM-LL-N in Fig. 14, which is the unit-diagonal alpha=1 case,
 * reading Q3).  op(T) lower-triangular -> forward, else backward.
 * side=L: sel lists columns of X (out is m x nsel).
 * side=R: sel lists ROWS of X; out is laid out nsel x n with leading
 *         dimension ldo (row t of the sample in out[t + j*ldo]). */
void oracle_strsm(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                  double alpha, const float *A, int64_t lda, const float *B, int64_t ldb,
                  double *out, int64_t ldo, const int64_t *sel, int64_t nsel)
{
    int left = up(side) == 'L', lower = up(uplo) == 'L';
    int ta = up(transa) != 'N', unit = up(diag) == 'U';
    if (left) {
        int forward = lower != ta;          /* op(T) lower-triangular */
        int64_t ncols = sel ? nsel : n;
#pragma omp parallel for schedule(dynamic, 1)
        for (int64_t t = 0; t < ncols; ++t) {
            int64_t j = selected(sel, t);
            double *x = out + t * ldo;
            for (int64_t i = 0; i < m; ++i) x[i] = alpha * (double)EL(B, ldb, i, j);
            if (alpha == 0.0) continue;
            for (int64_t s = 0; s < m; ++s) {
                int64_t i = forward ? s : m - 1 - s;
                double acc = x[i];
                for (int64_t q = 0; q < s; ++q) {      /* already-solved unknowns */
                    int64_t l = forward ? q : m - 1 - q;
                    acc -= triget(A, lda, lower, ta, unit, i, l) * x[l];
                }
                x[i] = unit ? acc : acc / triget(A, lda, lower, ta, unit, i, i);
            }
        }
    } else {
        int forward = lower == ta;          /* op(T) upper-triangular */
        int64_t nrows = sel ? nsel : m;
#pragma omp parallel for schedule(dynamic, 1)
        for (int64_t t = 0; t < nrows; ++t) {
            int64_t i = selected(sel, t);
            for (int64_t j = 0; j < n; ++j) out[t + j * ldo] = alpha * (double)EL(B, ldb, i, j);
            if (alpha == 0.0) continue;
            for (int64_t s = 0; s < n; ++s) {
                int64_t j = forward ? s : n - 1 - s;
                double acc = out[t + j * ldo];
                for (int64_t q = 0; q < s; ++q) {
                    int64_t l = forward ? q : n - 1 - q;
                    acc -= out[t + l * ldo] * triget(A, lda, lower, ta, unit, l, j);
                }
                out[t + j * ldo] = unit ? acc : acc / triget(A, lda, lower, ta, unit, j, j);
            }
        }
    }
}

/* Number of OpenMP threads the oracle will use (reported as `cores`). */
int oracle_num_threads(void)
{
#ifdef _OPENMP
    extern int omp_get_max_threads(void);
    return omp_get_max_threads();
#else
    return 1;
#endif
}
