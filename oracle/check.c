/*
 * check.c -- batched parity checker (TEST INFRASTRUCTURE ONLY, built into
 * liboracle.so next to oracle.c; same rules: only tests/, smoke() and the
 * bench's cpu legs load it; it shares nothing with the CUDA path).
 *
 * It adds NO arithmetic of the method: every reference result comes from the
 * oracle functions of oracle.c (oracle_getrf, oracle_getrf_partial,
 * oracle_backward_error), called on copies of the original inputs.  What is
 * here is the comparison of a GPU result against them, per matrix, written
 * out as numbers so the pass / fail rules stay in Python (tests/parity.py,
 * north_star tolerances).  It exists so that EVERY
 * matrix of a full config (10^6 matrices for C1-big) can be checked without
 * a Python object per matrix.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <float.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int oracle_getrf(int m, int n, double *A, int ld, int *ipiv, int *info, double *min_sep);
int oracle_getrf_partial(int n1, int n2, double *F11, int ld11, double *F12, int ld12,
                         const double *F21, int ld21, double *F22, int ld22, int *ipiv, int *info);
double oracle_backward_error(int m, int n, const double *A0, int lda0, const double *LU, int ld,
                             const int *ipiv);

/* fields of one getrf result record (doubles) */
enum {
    CK_INFO_O = 0,   /* oracle info */
    CK_IPIV_EQ,      /* 1: GPU ipiv == oracle ipiv */
    CK_FIRST_DIFF,   /* first step whose pivot differs, -1 if none */
    CK_BE,           /* backward error of the GPU factors (Q11) */
    CK_DL,           /* max|L - L_o| / max|L_o|  (NaN unless ipiv agrees) */
    CK_DU,           /* max|U - U_o| / max|U_o| */
    CK_RHO,          /* oracle min_sep (Q13) */
    CK_LMAX,         /* max |l_ij| of the GPU's strict lower L (G8: <= 1, i.e. the GPU's
                        pivot is the column maximum in its own arithmetic) */
    CK_EXACT,        /* 1: LU, ipiv, info all bitwise equal to the oracle */
    CK_NF
};

static int imin_(int a, int b) { return a < b ? a : b; }

static double *dup_matrix(int m, int n, const double *A, int lda)
{
    const int ldc = m > 0 ? m : 1;
    double *C = (double *)malloc(sizeof(double) * (size_t)ldc * (size_t)(n > 0 ? n : 1));
    for (int j = 0; j < n; ++j) memcpy(C + (size_t)j * ldc, A + (size_t)j * lda, sizeof(double) * (size_t)m);
    return C;
}

/* One matrix: GPU (LU, ld, ipiv, info) against oracle_getrf of A0. */
static void check_one(int m, int n, const double *A0, int ld0, const double *LU, int ld, const int *ipiv,
                      int info, double *out)
{
    const int K = imin_(m, n);
    for (int f = 0; f < CK_NF; ++f) out[f] = 0.0;
    double *LUo = dup_matrix(m, n, A0, ld0);
    int *ipo = (int *)malloc(sizeof(int) * (size_t)(K > 0 ? K : 1));
    int info_o = 0;
    double rho = INFINITY;
    oracle_getrf(m, n, LUo, m > 0 ? m : 1, ipo, &info_o, &rho);
    const int ldo = m > 0 ? m : 1;
    int first = -1;
    for (int k = 0; k < K; ++k)
        if (ipiv[k] != ipo[k]) { first = k; break; }
    out[CK_INFO_O] = info_o;
    out[CK_IPIV_EQ] = first < 0;
    out[CK_FIRST_DIFF] = first;
    out[CK_RHO] = rho;
    out[CK_BE] = K > 0 ? oracle_backward_error(m, n, A0, ld0, LU, ld, ipiv) : 0.0;
    double lmax = 0.0, dl = 0.0, du = 0.0, sl = 0.0, su = 0.0;
    int exact = first < 0 && info == info_o;
    for (int j = 0; j < n; ++j)
        for (int i = 0; i < m; ++i) {
            const double g = LU[i + (size_t)j * ld], o = LUo[i + (size_t)j * ldo];
            if (g != o && !(g != g && o != o)) exact = 0;
            if (i > j && j < K) {              /* strict lower: L */
                if (fabs(g) > lmax || g != g) lmax = (g != g) ? INFINITY : fabs(g);
                if (fabs(g - o) > dl) dl = fabs(g - o);
                if (fabs(o) > sl) sl = fabs(o);
            } else if (i < K) {                /* upper: U */
                if (fabs(g - o) > du) du = fabs(g - o);
                if (fabs(o) > su) su = fabs(o);
            }
        }
    out[CK_LMAX] = lmax;
    out[CK_EXACT] = exact;
    if (first < 0) {
        out[CK_DL] = sl > 0 ? dl / sl : dl;
        out[CK_DU] = su > 0 ? du / su : du;
    } else {
        out[CK_DL] = NAN;
        out[CK_DU] = NAN;
    }
    free(LUo);
    free(ipo);
}

static double work_of_(int m, int n) { double a = m, b = n; return a * b * (a < b ? a : b); }

static int cmp_desc_(const void *x, const void *y)
{
    const double *a = (const double *)x, *b = (const double *)y;
    return (a[0] < b[0]) - (a[0] > b[0]);
}

static int *order_desc(int batch, const int *m, const int *n)
{
    double *w = (double *)malloc(sizeof(double) * 2 * (size_t)(batch > 0 ? batch : 1));
    int *order = (int *)malloc(sizeof(int) * (size_t)(batch > 0 ? batch : 1));
    for (int i = 0; i < batch; ++i) { w[2 * i] = work_of_(m[i], n[i]); w[2 * i + 1] = i; }
    qsort(w, (size_t)batch, 2 * sizeof(double), cmp_desc_);
    for (int i = 0; i < batch; ++i) order[i] = (int)w[2 * i + 1];
    free(w);
    return order;
}

/* out[i * CK_NF + field]; matrices with info[i] < 0 (rejected by the GPU) are
 * not compared (out = NaN).  OpenMP over matrices, largest first. */
int check_getrf_batch(int batch, const int *m, const int *n, const double *const *A0, const int *ld0,
                      const double *const *LU, const int *ld, const int *const *ipiv, const int *info,
                      double *out, int nthreads)
{
    int *order = order_desc(batch, m, n);
#ifdef _OPENMP
    if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
    for (int t = 0; t < batch; ++t) {
        const int i = order[t];
        double *o = out + (size_t)i * CK_NF;
        if (info[i] < 0) {
            for (int f = 0; f < CK_NF; ++f) o[f] = NAN;
            continue;
        }
        check_one(m[i], n[i], A0[i], ld0[i], LU[i], ld[i], ipiv[i], info[i], o);
    }
    free(order);
    (void)nthreads;
    return CK_NF;
}

/* fields of one partial-front record: the getrf fields of F11, then */
enum {
    CP_F21_SAME = CK_NF, /* 1: F21 bitwise untouched */
    CP_D12,              /* max|F12 - F12_o| / max|F12_o| (NaN unless ipiv agrees) */
    CP_D22,              /* max|F22 - F22_o| / sigma, sigma = max(|F22_in| + |F21| |F12_o|) (Q12) */
    CP_EXACT,            /* 1: F11, F12, F22, ipiv, info bitwise equal to the oracle */
    CP_NF
};

/* Front i is one nf x nf column-major block (ld) with nf = n1 + n2:
 * F11 = [0, n1)^2, F12 = rows [0, n1) x cols [n1, nf), F21, F22 likewise.
 * F0: the original fronts, F: the GPU results. */
int check_partial_batch(int batch, const int *n1, const int *n2, const double *const *F0, const int *ld0,
                        const double *const *F, const int *ld, const int *const *ipiv, const int *info,
                        double *out, int nthreads)
{
    int *nf = (int *)malloc(sizeof(int) * (size_t)(batch > 0 ? batch : 1));
    for (int i = 0; i < batch; ++i) nf[i] = n1[i] + n2[i];
    int *order = order_desc(batch, nf, nf);
    free(nf);
#ifdef _OPENMP
    if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
    for (int t = 0; t < batch; ++t) {
        const int i = order[t];
        double *o = out + (size_t)i * CP_NF;
        if (info[i] < 0) {
            for (int f = 0; f < CP_NF; ++f) o[f] = NAN;
            continue;
        }
        const int a = n1[i], b = n2[i], N = a + b, l0 = ld0[i], l = ld[i];
        const double *A = F0[i], *G = F[i];
        /* the oracle on copies of the four blocks */
        double *o11 = dup_matrix(a, a, A, l0);
        double *o12 = dup_matrix(a, b, A + (size_t)a * l0, l0);
        double *o21 = dup_matrix(b, a, A + a, l0);
        double *o22 = dup_matrix(b, b, A + a + (size_t)a * l0, l0);
        int *ipo = (int *)malloc(sizeof(int) * (size_t)(a > 0 ? a : 1));
        int info_o = 0;
        const int la = a > 0 ? a : 1, lb = b > 0 ? b : 1;
        oracle_getrf_partial(a, b, o11, la, o12, la, o21, lb, o22, lb, ipo, &info_o);
        /* F11: the getrf record against the original F11 */
        check_one(a, a, A, l0, G, l, ipiv[i], info[i], o);
        const int eq = o[CK_IPIV_EQ] != 0.0;
        int same21 = 1, exact = (int)o[CK_EXACT];
        for (int j = 0; j < a; ++j)
            for (int r = 0; r < b; ++r)
                if (G[a + r + (size_t)j * l] != A[a + r + (size_t)j * l0]) same21 = 0;
        double d12 = 0.0, s12 = 0.0;
        for (int j = 0; j < b; ++j)
            for (int r = 0; r < a; ++r) {
                const double g = G[r + (size_t)(a + j) * l], x = o12[r + (size_t)j * la];
                if (g != x) exact = 0;
                if (fabs(g - x) > d12) d12 = fabs(g - x);
                if (fabs(x) > s12) s12 = fabs(x);
            }
        /* sigma = max_ij (|F22_in| + |F21| |F12_o|)_ij: |F21| transposed once so
         * the dot products run along contiguous memory */
        double *t21 = (double *)malloc(sizeof(double) * (size_t)(a > 0 ? a : 1) * (size_t)lb);
        for (int k = 0; k < a; ++k)
            for (int r = 0; r < b; ++r) t21[k + (size_t)r * a] = fabs(A[a + r + (size_t)k * l0]);
        double d22 = 0.0, sigma = 0.0;
        for (int j = 0; j < b; ++j)
            for (int r = 0; r < b; ++r) {
                const double g = G[a + r + (size_t)(a + j) * l], x = o22[r + (size_t)j * lb];
                if (g != x) exact = 0;
                if (fabs(g - x) > d22) d22 = fabs(g - x);
                double s = fabs(A[a + r + (size_t)(a + j) * l0]);
                const double *tr = t21 + (size_t)r * a, *xc = o12 + (size_t)j * la;
                for (int k = 0; k < a; ++k) s += tr[k] * fabs(xc[k]);
                if (s > sigma) sigma = s;
            }
        free(t21);
        o[CP_F21_SAME] = same21;
        o[CP_D12] = eq ? (s12 > 0 ? d12 / s12 : d12) : NAN;
        o[CP_D22] = eq ? (sigma > 0 ? d22 / sigma : d22) : NAN;
        o[CP_EXACT] = exact && same21 && eq && info[i] == info_o;
        (void)N;
        free(o11); free(o12); free(o21); free(o22); free(ipo);
    }
    free(order);
    (void)nthreads;
    return CP_NF;
}
