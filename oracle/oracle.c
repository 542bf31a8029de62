/*
 * oracle.c -- plain, slow, obviously-correct CPU reference for irrLU.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_sc_abdelfattahgbtld22_b200/csrc); neither includes the other.
 *
 * Built with:  gcc -O2 -ffp-contract=off -fno-fast-math -fopenmp -shared -fPIC
 * (no FMA contraction, no flush-to-zero: every a - b*c is a separate multiply
 * and subtract, IEEE round-to-nearest-even).
 *
 * What it computes (citations are /root/reference/PAPER.md lines):
 *  - oracle_getrf: LU with partial pivoting, P*L*U = A (L106 §III-B), as the
 *    plain column-by-column definition (LAPACK dgetf2 semantics).  The paper's
 *    blocked right-looking algorithm (L106, Fig. 1) reaches the same result in
 *    exact arithmetic; readings Q3 (idamax tie -> smallest row), Q5 (exact zero
 *    pivot: info = first step, no swap, no scaling, continue), Q6 (true IEEE
 *    division) of SURVEY.md §8(c) are applied.
 *  - oracle_getrf_partial: the per-front steps of L95-L97 (§III-A):
 *        P L U <- LU(F11)              (pivoting restricted to F11, L99)
 *        F12   <- U^-1 L^-1 P^T F12
 *        F22   <- F22 - F21 F12        (F21 untouched)
 *  - oracle_gemm / oracle_trsm / oracle_laswp: the building blocks of
 *    §IV-C (L171-173), §IV-D (L175-182) and §IV-F (L188-195) as their plain
 *    BLAS/LAPACK definitions.
 *  - oracle_getrs: the solve with the factors (LAPACK dgetrs steps), the
 *    GETRS composition the paper benchmarks irrTRSM against (L96, L215).
 *  - oracle_extend_add: the extend-add of a child's Schur complement into
 *    its parent front (L99 §III-A: "the Schur complement F_{r:22} is added
 *    into the parent frontal matrix ... this requires a scatter operation"),
 *    as its plain definition Fp[rel_i, rel_j] += F22[i, j].
 *  - oracle_backward_error: ||PA - LU||_F / (||A||_F * k * eps) (north_star;
 *    SURVEY reading Q11), accumulated in long double.
 *  - oracle_getrf_partial_lapack: the LAPACK-style variant of the partial
 *    front factorization (reading Q8's alternative; the
 *    solver's factors L21 = F21 U^-1, U12 = L^-1 P^T F12, L96-97), written
 *    out as its steps: GEPP of F11, swaps on F12, forward substitution on
 *    F12, row-by-row substitution x U = f on F21, F22 - L21 U12.
 *  - oracle_zgetrf / oracle_zbackward_error: LU with partial pivoting of a
 *    COMPLEX matrix (the solver's A in C^{N x N}, L71 §III-A; SURVEY §8(f)
 *    NEXT 3) with LAPACK zgetf2 semantics (reading Q20 in DESIGN.md): pivot =
 *    the smallest row maximising |Re| + |Im| (izamax), the textbook complex
 *    division (a+bi)/(c+di) = ((ac+bd) + (bc-ad)i) / (c^2+d^2), complex
 *    multiply (ac-bd) + (ad+bc)i, interleaved (re, im) column-major storage.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <float.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define A_(i, j) A[(size_t)(i) + (size_t)(j) * (size_t)ld]

static int imin(int a, int b) { return a < b ? a : b; }
static int imax(int a, int b) { return a > b ? a : b; }

/* ---------------------------------------------------------------------------
 * GEPP, one matrix.  P:L106 §III-B; SURVEY §8(c) "Plain definition".
 * min_sep (may be NULL): rho = min over steps of |best| / |second best|
 * among the pivot candidates, +inf if never defined.
 * Returns 0, or -(argument position) for a bad m / n / ld.
 * ------------------------------------------------------------------------- */
int oracle_getrf(int m, int n, double *A, int ld, int *ipiv, int *info, double *min_sep)
{
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (ld < imax(1, m)) return -4;
    *info = 0;
    double sep = INFINITY;
    const int K = imin(m, n);
    for (int k = 0; k < K; ++k) {
        /* 1. p = smallest index i >= k maximising |a_ik| */
        int p = k;
        double best = fabs(A_(k, k)), second = -1.0;
        for (int i = k + 1; i < m; ++i) {
            double v = fabs(A_(i, k));
            if (v > best) { second = best; best = v; p = i; }
            else if (v > second) second = v;
        }
        if (best > 0.0 && second > 0.0) {
            double r = best / second;
            if (r < sep) sep = r;
        }
        /* 2. record the pivot (1-based) */
        ipiv[k] = p + 1;
        /* 3. swap + scale, or flag the first exact zero pivot */
        if (A_(p, k) != 0.0) {
            if (p != k)
                for (int j = 0; j < n; ++j) { double t = A_(k, j); A_(k, j) = A_(p, j); A_(p, j) = t; }
            const double piv = A_(k, k);
            for (int i = k + 1; i < m; ++i) A_(i, k) = A_(i, k) / piv;
        } else if (*info == 0) {
            *info = k + 1;
        }
        /* 4. rank-1 update of the trailing matrix */
        for (int j = k + 1; j < n; ++j) {
            const double akj = A_(k, j);
            for (int i = k + 1; i < m; ++i) A_(i, j) = A_(i, j) - A_(i, k) * akj;
        }
    }
    if (min_sep) *min_sep = sep;
    return 0;
}

/* flops of one matrix, for largest-first scheduling only */
static double work_of(int m, int n) { double a = m, b = n; return a * b * (a < b ? a : b); }

static int cmp_desc(const void *x, const void *y)
{
    const double *a = (const double *)x, *b = (const double *)y;
    return (a[0] < b[0]) - (a[0] > b[0]);
}

static int *largest_first(int batch, const int *m, const int *n)
{
    double *w = (double *)malloc(sizeof(double) * 2 * (size_t)(batch > 0 ? batch : 1));
    int *order = (int *)malloc(sizeof(int) * (size_t)(batch > 0 ? batch : 1));
    for (int i = 0; i < batch; ++i) { w[2 * i] = work_of(m[i], n[i]); w[2 * i + 1] = i; }
    qsort(w, (size_t)batch, 2 * sizeof(double), cmp_desc);
    for (int i = 0; i < batch; ++i) order[i] = (int)w[2 * i + 1];
    free(w);
    return order;
}

/* Batched GEPP: OpenMP over matrices, largest first.  info[i] < 0 marks a bad
 * argument (matrix skipped).  min_sep may be NULL.  nthreads <= 0: default. */
int oracle_getrf_batch(int batch, const int *m, const int *n, double *const *A, const int *ld,
                       int *const *ipiv, int *info, double *min_sep, int nthreads)
{
    if (batch < 0) return -1;
    int *order = largest_first(batch, m, n);
#ifdef _OPENMP
    if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
    for (int t = 0; t < batch; ++t) {
        int i = order[t];
        double s;
        int r = oracle_getrf(m[i], n[i], A[i], ld[i], ipiv[i], &info[i], &s);
        if (r < 0) { info[i] = r; s = INFINITY; }
        if (min_sep) min_sep[i] = s;
    }
    free(order);
    (void)nthreads;
    return 0;
}

/* ---------------------------------------------------------------------------
 * Partial front factorization, P:L95-L99 taken literally.
 * ------------------------------------------------------------------------- */
int oracle_getrf_partial(int n1, int n2, double *F11, int ld11, double *F12, int ld12,
                         const double *F21, int ld21, double *F22, int ld22, int *ipiv, int *info)
{
    if (n1 < 0) return -1;
    if (n2 < 0) return -2;
    if (ld11 < imax(1, n1)) return -4;
    if (ld12 < imax(1, n1)) return -6;
    if (ld21 < imax(1, n2)) return -8;
    if (ld22 < imax(1, n2)) return -10;
    /* step 1: P L U <- LU(F11), pivot search over F11's n1 rows only */
    int r = oracle_getrf(n1, n1, F11, ld11, ipiv, info, NULL);
    if (r < 0) return r;
#define F11_(i, j) F11[(size_t)(i) + (size_t)(j) * ld11]
#define F12_(i, j) F12[(size_t)(i) + (size_t)(j) * ld12]
#define F21_(i, j) F21[(size_t)(i) + (size_t)(j) * ld21]
#define F22_(i, j) F22[(size_t)(i) + (size_t)(j) * ld22]
    /* step 2: P^T F12 -- apply the swaps k = 0..n1-1 in order */
    for (int k = 0; k < n1; ++k) {
        int p = ipiv[k] - 1;
        if (p != k)
            for (int c = 0; c < n2; ++c) { double t = F12_(k, c); F12_(k, c) = F12_(p, c); F12_(p, c) = t; }
    }
    /* The dot products of steps 3-5 run along ROWS of F11 and F21; they read
     * them from row-major copies (T11[i][j] = F11(i, j), T21[i][k] = F21(i, k)),
     * which changes only where the same values are read from: every sum has
     * the same terms in the same order. */
    double *T11 = (double *)malloc(sizeof(double) * (size_t)(n1 > 0 ? n1 : 1) * (size_t)(n1 > 0 ? n1 : 1));
    double *T21 = (double *)malloc(sizeof(double) * (size_t)(n1 > 0 ? n1 : 1) * (size_t)(n2 > 0 ? n2 : 1));
    for (int j = 0; j < n1; ++j)
        for (int i = 0; i < n1; ++i) T11[(size_t)i * n1 + j] = F11_(i, j);
    for (int k = 0; k < n1; ++k)
        for (int i = 0; i < n2; ++i) T21[(size_t)i * n1 + k] = F21_(i, k);
    for (int c = 0; c < n2; ++c) {
        /* step 3: L^-1 (unit lower): row i -= sum_{j<i} l_ij row j */
        for (int i = 0; i < n1; ++i) {
            double s = 0.0;
            for (int j = 0; j < i; ++j) s = s + T11[(size_t)i * n1 + j] * F12_(j, c);
            F12_(i, c) = F12_(i, c) - s;
        }
        /* step 4: U^-1: row i = (row i - sum_{j>i} u_ij row j) / u_ii */
        for (int i = n1 - 1; i >= 0; --i) {
            double s = 0.0;
            for (int j = i + 1; j < n1; ++j) s = s + T11[(size_t)i * n1 + j] * F12_(j, c);
            F12_(i, c) = (F12_(i, c) - s) / F11_(i, i);
        }
    }
    /* step 5: F22 <- F22 - F21 F12, plain triple loop, k ascending */
    for (int j = 0; j < n2; ++j)
        for (int i = 0; i < n2; ++i) {
            double s = 0.0;
            for (int k = 0; k < n1; ++k) s = s + T21[(size_t)i * n1 + k] * F12_(k, j);
            F22_(i, j) = F22_(i, j) - s;
        }
    free(T11);
    free(T21);
#undef F11_
#undef F12_
#undef F21_
#undef F22_
    return 0;
}

int oracle_getrf_partial_batch(int batch, const int *n1, const int *n2,
                               double *const *F11, const int *ld11, double *const *F12, const int *ld12,
                               const double *const *F21, const int *ld21, double *const *F22, const int *ld22,
                               int *const *ipiv, int *info, int nthreads)
{
    if (batch < 0) return -1;
    int *nf = (int *)malloc(sizeof(int) * (size_t)(batch > 0 ? batch : 1));
    for (int i = 0; i < batch; ++i) nf[i] = n1[i] + n2[i];
    int *order = largest_first(batch, nf, nf);
    free(nf);
#ifdef _OPENMP
    if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
    for (int t = 0; t < batch; ++t) {
        int i = order[t];
        int r = oracle_getrf_partial(n1[i], n2[i], F11[i], ld11[i], F12[i], ld12[i], F21[i], ld21[i],
                                     F22[i], ld22[i], ipiv[i], &info[i]);
        if (r < 0) info[i] = r;
    }
    free(order);
    (void)nthreads;
    return 0;
}

/* ---------------------------------------------------------------------------
 * Building blocks, plain definitions.
 * trans: 0 = N, 1 = T.  side: 0 = left, 1 = right.  uplo: 0 = lower, 1 = upper.
 * diag: 0 = non-unit, 1 = unit.
 * ------------------------------------------------------------------------- */

/* C <- alpha op(A) op(B) + beta C (BLAS dgemm; beta == 0 does not read C). */
void oracle_gemm(int ta, int tb, int m, int n, int k, double alpha,
                 const double *A, int lda, const double *B, int ldb,
                 double beta, double *C, int ldc)
{
    for (int j = 0; j < n; ++j)
        for (int i = 0; i < m; ++i) {
            double s = 0.0;
            for (int l = 0; l < k; ++l) {
                double a = ta ? A[l + (size_t)i * lda] : A[i + (size_t)l * lda];
                double b = tb ? B[j + (size_t)l * ldb] : B[l + (size_t)j * ldb];
                s = s + a * b;
            }
            double *c = &C[i + (size_t)j * ldc];
            *c = (beta == 0.0) ? alpha * s : alpha * s + beta * *c;
        }
}

/* Solve op(T) X = alpha B (side = left, T is m x m) or X op(T) = alpha B
 * (side = right, T is n x n); B is m x n, overwritten by X (BLAS dtrsm).
 * op(T) is materialised as a dense triangle M, then plain substitution. */
void oracle_trsm(int side, int uplo, int trans, int diag, int m, int n, double alpha,
                 const double *T, int ldt, double *B, int ldb)
{
    const int kt = side ? n : m;
    double *M = (double *)calloc((size_t)kt * (size_t)(kt > 0 ? kt : 1), sizeof(double));
    for (int j = 0; j < kt; ++j)
        for (int i = 0; i < kt; ++i) {
            int in_tri = uplo ? (i <= j) : (i >= j);
            double t = in_tri ? T[i + (size_t)j * ldt] : 0.0;
            if (i == j && diag) t = 1.0;
            if (trans) M[j + (size_t)i * kt] = t; else M[i + (size_t)j * kt] = t;
        }
    /* effective triangle of M = op(T) */
    const int m_lower = trans ? uplo : !uplo;
    double *x = (double *)malloc(sizeof(double) * (size_t)(kt > 0 ? kt : 1));
    const int nrhs = side ? m : n;
    for (int r = 0; r < nrhs; ++r) {
        /* left: solve M x = alpha b, b = column r.  right: x^T M = alpha b^T,
           i.e. M^T x = alpha b with b = row r; M^T is lower iff M is upper. */
        for (int i = 0; i < kt; ++i)
            x[i] = alpha * (side ? B[r + (size_t)i * ldb] : B[i + (size_t)r * ldb]);
        int fwd = side ? !m_lower : m_lower;
#define S_(i, j) (side ? M[(j) + (size_t)(i) * kt] : M[(i) + (size_t)(j) * kt])
        if (fwd) {
            for (int i = 0; i < kt; ++i) {
                double s = 0.0;
                for (int j = 0; j < i; ++j) s = s + S_(i, j) * x[j];
                x[i] = (x[i] - s) / S_(i, i);
            }
        } else {
            for (int i = kt - 1; i >= 0; --i) {
                double s = 0.0;
                for (int j = i + 1; j < kt; ++j) s = s + S_(i, j) * x[j];
                x[i] = (x[i] - s) / S_(i, i);
            }
        }
#undef S_
        for (int i = 0; i < kt; ++i) {
            if (side) B[r + (size_t)i * ldb] = x[i]; else B[i + (size_t)r * ldb] = x[i];
        }
    }
    free(x);
    free(M);
}

/* Row interchanges (LAPACK dlaswp, incx = 1): for k = k1..k2-1 (0-based),
 * swap row k with row ipiv[k]-1 across the n columns.  P:L190. */
void oracle_laswp(int n, double *A, int lda, int k1, int k2, const int *ipiv)
{
    for (int k = k1; k < k2; ++k) {
        int p = ipiv[k] - 1;
        if (p != k)
            for (int j = 0; j < n; ++j) {
                double t = A[k + (size_t)j * lda];
                A[k + (size_t)j * lda] = A[p + (size_t)j * lda];
                A[p + (size_t)j * lda] = t;
            }
    }
}

/* ---------------------------------------------------------------------------
 * GETRS with the factors of oracle_getrf (the paper's
 * GETRS = LASWP + TRSM(L, unit) + TRSM(U)): B <- U^-1 L^-1 P^T B
 * for an n x n L\U and n x nrhs B, as the plain steps of LAPACK dgetrs:
 *   1. apply the swaps k = 0..n-1 in order to the rows of B;
 *   2. forward substitution with the unit L: row i -= sum_{j<i} l_ij row j;
 *   3. back substitution with U: row i = (row i - sum_{j>i} u_ij row j) / u_ii.
 * Returns 0, or -(argument position) for a bad n / nrhs / ld.
 * ------------------------------------------------------------------------- */
int oracle_getrs(int n, int nrhs, const double *LU, int ld, const int *ipiv, double *B, int ldb)
{
    if (n < 0) return -1;
    if (nrhs < 0) return -2;
    if (ld < imax(1, n)) return -4;
    if (ldb < imax(1, n)) return -7;
#define LU_(i, j) LU[(size_t)(i) + (size_t)(j) * ld]
#define B_(i, j) B[(size_t)(i) + (size_t)(j) * ldb]
    for (int k = 0; k < n; ++k) {
        int p = ipiv[k] - 1;
        if (p != k)
            for (int c = 0; c < nrhs; ++c) { double t = B_(k, c); B_(k, c) = B_(p, c); B_(p, c) = t; }
    }
    for (int c = 0; c < nrhs; ++c) {
        for (int i = 0; i < n; ++i) {
            double s = 0.0;
            for (int j = 0; j < i; ++j) s = s + LU_(i, j) * B_(j, c);
            B_(i, c) = B_(i, c) - s;
        }
        for (int i = n - 1; i >= 0; --i) {
            double s = 0.0;
            for (int j = i + 1; j < n; ++j) s = s + LU_(i, j) * B_(j, c);
            B_(i, c) = (B_(i, c) - s) / LU_(i, i);
        }
    }
#undef LU_
#undef B_
    return 0;
}

/* ---------------------------------------------------------------------------
 * Extend-add: the child's n2 x n2 Schur
 * complement F22 is scattered into its parent front Fp (np x np) through the
 * index map rel (0-based parent row / column of each child row / column):
 *     Fp[rel[i], rel[j]] = Fp[rel[i], rel[j]] + F22[i, j]   for all i, j < n2.
 * Returns 0, or -(argument position) for a bad n2 / ld22 / rel entry / np /
 * ldp (then Fp is untouched).  Several children of one parent are applied by
 * calling this once per child, in the caller's order.
 * ------------------------------------------------------------------------- */
int oracle_extend_add(int n2, const double *F22, int ld22, const int *rel, int np, double *Fp, int ldp)
{
    if (n2 < 0) return -1;
    if (ld22 < imax(1, n2)) return -3;
    if (np < 0) return -5;
    if (ldp < imax(1, np)) return -7;
    for (int i = 0; i < n2; ++i)
        if (rel[i] < 0 || rel[i] >= np) return -4;
    for (int j = 0; j < n2; ++j)
        for (int i = 0; i < n2; ++i)
            Fp[(size_t)rel[i] + (size_t)rel[j] * ldp] = Fp[(size_t)rel[i] + (size_t)rel[j] * ldp] +
                                                        F22[(size_t)i + (size_t)j * ld22];
    return 0;
}

/* ||PA - LU||_F / (||A||_F * max(1, min(m,n)) * eps)  (north_star).
 * PA = the recorded swaps applied in order to a copy of A0.  L = unit lower
 * trapezoid of LU (m x k), U = upper trapezoid (k x n).  long double sums.
 * ||A|| = 0: returns 0 if LU reproduces PA exactly, +inf otherwise. */
double oracle_backward_error(int m, int n, const double *A0, int lda0, const double *LU, int ld,
                             const int *ipiv)
{
    const int K = imin(m, n);
    long double *PA = (long double *)malloc(sizeof(long double) * (size_t)(m > 0 ? m : 1) * (size_t)(n > 0 ? n : 1));
    for (int j = 0; j < n; ++j)
        for (int i = 0; i < m; ++i) PA[i + (size_t)j * m] = A0[i + (size_t)j * lda0];
    for (int k = 0; k < K; ++k) {
        int p = ipiv[k] - 1;
        if (p != k)
            for (int j = 0; j < n; ++j) {
                long double t = PA[k + (size_t)j * m];
                PA[k + (size_t)j * m] = PA[p + (size_t)j * m];
                PA[p + (size_t)j * m] = t;
            }
    }
    /* the rows of L copied row-major once, so that both operands of the dot
     * products below are read contiguously (same terms, same order) */
    double *Lr = (double *)malloc(sizeof(double) * (size_t)(m > 0 ? m : 1) * (size_t)(K > 0 ? K : 1));
    for (int i = 0; i < m; ++i)
        for (int l = 0; l < imin(i, K); ++l) Lr[(size_t)i * K + l] = LU[i + (size_t)l * ld];
    long double rn = 0.0L, an = 0.0L;
    for (int j = 0; j < n; ++j)
        for (int i = 0; i < m; ++i) {
            long double s = 0.0L;
            int lim = imin(imin(i, j), K - 1);
            const double *li = Lr + (size_t)i * K;
            const double *uj = LU + (size_t)j * ld;
            for (int l = 0; l <= lim; ++l) {
                long double lv = (l == i) ? 1.0L : (long double)li[l];
                s += lv * (long double)uj[l];
            }
            long double d = PA[i + (size_t)j * m] - s;
            rn += d * d;
            long double a = A0[i + (size_t)j * lda0];
            an += a * a;
        }
    free(PA);
    free(Lr);
    if (an == 0.0L) return rn == 0.0L ? 0.0 : INFINITY;
    return (double)(sqrtl(rn) / (sqrtl(an) * (long double)imax(1, K) * (long double)DBL_EPSILON));
}

/* ---------------------------------------------------------------------------
 * LAPACK-style partial front (reading Q8's
 * alternative): F11 -> L\U (pivots within F11), F12 -> U12 = L^-1 P^T F12,
 * F21 -> L21 = F21 U^-1, F22 -> F22 - L21 U12.  In exact arithmetic the same
 * Schur complement as oracle_getrf_partial.
 * ------------------------------------------------------------------------- */
int oracle_getrf_partial_lapack(int n1, int n2, double *F11, int ld11, double *F12, int ld12,
                                double *F21, int ld21, double *F22, int ld22, int *ipiv, int *info)
{
    if (n1 < 0) return -1;
    if (n2 < 0) return -2;
    if (ld11 < imax(1, n1)) return -4;
    if (ld12 < imax(1, n1)) return -6;
    if (ld21 < imax(1, n2)) return -8;
    if (ld22 < imax(1, n2)) return -10;
    /* step 1: P L U <- LU(F11), pivot search over F11's n1 rows only */
    int r = oracle_getrf(n1, n1, F11, ld11, ipiv, info, NULL);
    if (r < 0) return r;
#define F11_(i, j) F11[(size_t)(i) + (size_t)(j) * ld11]
#define F12_(i, j) F12[(size_t)(i) + (size_t)(j) * ld12]
#define F21_(i, j) F21[(size_t)(i) + (size_t)(j) * ld21]
#define F22_(i, j) F22[(size_t)(i) + (size_t)(j) * ld22]
    /* step 2: P^T F12 -- the swaps k = 0..n1-1 in order */
    for (int k = 0; k < n1; ++k) {
        int p = ipiv[k] - 1;
        if (p != k)
            for (int c = 0; c < n2; ++c) { double t = F12_(k, c); F12_(k, c) = F12_(p, c); F12_(p, c) = t; }
    }
    /* step 3: U12 = L^-1 F12 (unit lower): row i -= sum_{j<i} l_ij row j */
    for (int c = 0; c < n2; ++c)
        for (int i = 0; i < n1; ++i) {
            double s = 0.0;
            for (int j = 0; j < i; ++j) s = s + F11_(i, j) * F12_(j, c);
            F12_(i, c) = F12_(i, c) - s;
        }
    /* step 4: L21 = F21 U^-1: each row x of F21 solves x U = f,
     * x_j = (f_j - sum_{k<j} x_k u_kj) / u_jj, j ascending */
    for (int i = 0; i < n2; ++i)
        for (int j = 0; j < n1; ++j) {
            double s = 0.0;
            for (int k = 0; k < j; ++k) s = s + F21_(i, k) * F11_(k, j);
            F21_(i, j) = (F21_(i, j) - s) / F11_(j, j);
        }
    /* step 5: F22 <- F22 - L21 U12, plain triple loop, k ascending */
    for (int j = 0; j < n2; ++j)
        for (int i = 0; i < n2; ++i) {
            double s = 0.0;
            for (int k = 0; k < n1; ++k) s = s + F21_(i, k) * F12_(k, j);
            F22_(i, j) = F22_(i, j) - s;
        }
#undef F11_
#undef F12_
#undef F21_
#undef F22_
    return 0;
}

/* ---------------------------------------------------------------------------
 * Complex LU with partial pivoting (the solver's
 * A in C^{N x N}).  Storage: column-major, element (i, j) at A[2 (i + j ld)]
 * (re) and A[2 (i + j ld) + 1] (im) -- C99 / std::complex<double> layout.
 * LAPACK zgetf2 semantics (DESIGN reading Q20): k = 0..min(m,n)-1:
 *   1. p = smallest i >= k maximising cabs1(a_ik) = |Re| + |Im| (izamax);
 *   2. ipiv[k] = p + 1;
 *   3. if a_pk != 0: swap rows k, p across all n columns; a_ik <- a_ik / a_kk
 *      for i > k (textbook complex division); else info <- k + 1 (first);
 *   4. a_ij <- a_ij - a_ik a_kj for i, j > k (complex multiply, then subtract).
 * min_sep: rho = min over steps of cabs1(best) / cabs1(second best) (Q13).
 * ------------------------------------------------------------------------- */
static double cabs1(double re, double im) { return fabs(re) + fabs(im); }

int oracle_zgetrf(int m, int n, double *A, int ld, int *ipiv, int *info, double *min_sep)
{
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (ld < imax(1, m)) return -4;
    *info = 0;
    double sep = INFINITY;
#define RE(i, j) A[2 * ((size_t)(i) + (size_t)(j) * (size_t)ld)]
#define IM(i, j) A[2 * ((size_t)(i) + (size_t)(j) * (size_t)ld) + 1]
    const int K = imin(m, n);
    for (int k = 0; k < K; ++k) {
        int p = k;
        double best = cabs1(RE(k, k), IM(k, k)), second = -1.0;
        for (int i = k + 1; i < m; ++i) {
            double v = cabs1(RE(i, k), IM(i, k));
            if (v > best) { second = best; best = v; p = i; }
            else if (v > second) second = v;
        }
        if (best > 0.0 && second > 0.0) {
            double r = best / second;
            if (r < sep) sep = r;
        }
        ipiv[k] = p + 1;
        if (RE(p, k) != 0.0 || IM(p, k) != 0.0) {
            if (p != k)
                for (int j = 0; j < n; ++j) {
                    double tr = RE(k, j), ti = IM(k, j);
                    RE(k, j) = RE(p, j); IM(k, j) = IM(p, j);
                    RE(p, j) = tr; IM(p, j) = ti;
                }
            const double c = RE(k, k), d = IM(k, k);
            const double den = c * c + d * d;
            for (int i = k + 1; i < m; ++i) {
                const double a = RE(i, k), b = IM(i, k);
                RE(i, k) = (a * c + b * d) / den;
                IM(i, k) = (b * c - a * d) / den;
            }
        } else if (*info == 0) {
            *info = k + 1;
        }
        for (int j = k + 1; j < n; ++j) {
            const double ur = RE(k, j), ui = IM(k, j);
            for (int i = k + 1; i < m; ++i) {
                const double lr = RE(i, k), li = IM(i, k);
                const double pr = lr * ur - li * ui, pi = lr * ui + li * ur;
                RE(i, j) = RE(i, j) - pr;
                IM(i, j) = IM(i, j) - pi;
            }
        }
    }
#undef RE
#undef IM
    if (min_sep) *min_sep = sep;
    return 0;
}

/* ||PA - LU||_F / (||A||_F * max(1, min(m,n)) * eps) for complex factors
 * (Q11 with the complex Frobenius norm), long double accumulation. */
double oracle_zbackward_error(int m, int n, const double *A0, int lda0, const double *LU, int ld,
                              const int *ipiv)
{
    const int K = imin(m, n);
    const size_t mm = (size_t)(m > 0 ? m : 1), nn = (size_t)(n > 0 ? n : 1);
    long double *PR = (long double *)malloc(sizeof(long double) * mm * nn);
    long double *PI = (long double *)malloc(sizeof(long double) * mm * nn);
    for (int j = 0; j < n; ++j)
        for (int i = 0; i < m; ++i) {
            PR[i + (size_t)j * m] = A0[2 * (i + (size_t)j * lda0)];
            PI[i + (size_t)j * m] = A0[2 * (i + (size_t)j * lda0) + 1];
        }
    for (int k = 0; k < K; ++k) {
        int p = ipiv[k] - 1;
        if (p != k)
            for (int j = 0; j < n; ++j) {
                long double t = PR[k + (size_t)j * m]; PR[k + (size_t)j * m] = PR[p + (size_t)j * m]; PR[p + (size_t)j * m] = t;
                t = PI[k + (size_t)j * m]; PI[k + (size_t)j * m] = PI[p + (size_t)j * m]; PI[p + (size_t)j * m] = t;
            }
    }
    long double rn = 0.0L, an = 0.0L;
    for (int j = 0; j < n; ++j)
        for (int i = 0; i < m; ++i) {
            long double sr = 0.0L, si = 0.0L;
            int lim = imin(imin(i, j), K - 1);
            for (int l = 0; l <= lim; ++l) {
                long double lr = (l == i) ? 1.0L : (long double)LU[2 * (i + (size_t)l * ld)];
                long double li = (l == i) ? 0.0L : (long double)LU[2 * (i + (size_t)l * ld) + 1];
                long double ur = (long double)LU[2 * (l + (size_t)j * ld)];
                long double ui = (long double)LU[2 * (l + (size_t)j * ld) + 1];
                sr += lr * ur - li * ui;
                si += lr * ui + li * ur;
            }
            long double dr = PR[i + (size_t)j * m] - sr, di = PI[i + (size_t)j * m] - si;
            rn += dr * dr + di * di;
            long double ar = A0[2 * (i + (size_t)j * lda0)], ai = A0[2 * (i + (size_t)j * lda0) + 1];
            an += ar * ar + ai * ai;
        }
    free(PR);
    free(PI);
    if (an == 0.0L) return rn == 0.0L ? 0.0 : INFINITY;
    return (double)(sqrtl(rn) / (sqrtl(an) * (long double)imax(1, K) * (long double)DBL_EPSILON));
}

int oracle_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
