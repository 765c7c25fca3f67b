/*
 * oracle.c — CPU ORACLE for vbatched DPOTRF and the vbatched BLAS it uses.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (paper_conf_ipps_abdelfattahhtd16_b200/, libvbatched.so) never calls it, and this file
 * shares no code, header, table or helper with the CUDA path.
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -fopenmp -shared -fPIC (no FMA contraction,
 * no reassociation: every sum below is evaluated in the order written).
 *
 * What is computed (citations are /root/reference/PAPER.md line numbers):
 *  - oracle_dpotrf_lower: the Cholesky factor A = L L^T of one SPD matrix (Fig. 1,
 *    PAPER.md:187-212, "xPOTRF(A(i)) -> L_i L_i^T"; potf2 = LAPACK [7], PAPER.md:358,
 *    2338-2342). Written as the textbook unblocked Cholesky-Crout recurrence
 *        l_jj = sqrt(a_jj - sum_{k<j} l_jk^2),   l_ij = (a_ij - sum_{k<j} l_ik l_jk) / l_jj,
 *    k ascending, with LAPACK DPOTRF error reporting (SURVEY.md §8(c) readings #2, #3):
 *    info = j+1 (1-based) at the first pivot that is not > 0 (NaN counts as failure); the
 *    failing pivot value is stored at (j,j) and the routine stops. Pinned by
 *    tests/test_oracle.py (closed forms, exact integer families, MKL, exact rationals).
 *  - oracle_spotrf_lower: the same recurrence in IEEE single precision (float arithmetic,
 *    sqrtf correctly rounded, no contraction) — the FP32 problem of SURVEY.md §8(f) NEXT-3
 *    (the paper's SP runs; LAPACK SPOTRF).
 *  - oracle_dpotrf_batch: the vbatched problem (§III-A: each matrix has
 *    its own size and leading dimension) = the single-matrix oracle applied to each matrix;
 *    OpenMP dynamic over matrices (one core per matrix, the paper's CPU scheme,
 *    PAPER.md:1705-1713).
 *  - oracle_dgemm / oracle_dsyrk / oracle_dtrsm: the BLAS definitions of the separated
 *    kernels (§III-E: potf2, trsm, gemm, syrk), as plain loops.
 *  - oracle_backward_error: ||A - L L^T||_F / (n ||A||_F eps) in long double
 *    (BASELINE.json north_star gate; SURVEY.md §8(c) reading #13, eps = 2^-53).
 *  - oracle_dgetrf: LU with partial pivoting, A = P L U (the extension to LU the paper names
 *    as future work, §V, and PAPER.md:740-744, §III-E; SURVEY.md §8(f)
 *    NEXT-4). Written as the textbook unblocked right-looking elimination with LAPACK DGETF2
 *    conventions: pivot = first row of maximal |a_ik| (IDAMAX), row swap, l_ik = a_ik / u_kk
 *    (IEEE division), rank-1 update a_ij -= l_ik u_kj in k order; a zero pivot records
 *    info = k+1 (first only) and elimination continues (nothing to scale: the column is zero).
 *  - oracle_getrf_backward_error: ||P A - L U||_F / (max(m,n) ||A||_F eps), long double.
 *  - oracle_zpotrf_lower / oracle_cpotrf_lower: the complex Hermitian problem A = L L^H (the
 *    paper's "supports complex precisions", §IV-A; LAPACK ZPOTRF/CPOTRF;
 *    SURVEY.md §8(f) NEXT-3). The same Crout recurrence with conjugates,
 *        l_jj = sqrt(Re a_jj - sum_{k<j} |l_jk|^2),  l_ij = (a_ij - sum_{k<j} l_ik conj(l_jk)) / l_jj,
 *    complex arithmetic written out in real operations (no C99 complex), k ascending; the
 *    imaginary part of the diagonal is ignored and stored as 0 (LAPACK). Interleaved storage
 *    (re, im) per element, column-major. Double (Z) and single (C) precision.
 *  - oracle_zpotrf_backward_error: ||A - L L^H||_F / (n ||A||_F eps), long double, eps = 2^-53.
 *  - oracle_dgeqrf: Householder QR, A = Q R (the QR extension named as future work,
 *    PAPER.md:2279-2285, §V), textbook unblocked form with LAPACK
 *    DGEQR2 / DLARFG conventions: for column k, alpha = a_kk, xnorm = ||a_(k+1:m, k)||_2 (plain
 *    sum of squares, k ascending), beta = -sign(alpha) sqrt(alpha^2 + xnorm^2), tau = (beta -
 *    alpha) / beta, v = a_(k+1:m, k) / (alpha - beta) (IEEE division), a_kk = beta; then
 *    H_k = I - tau v v^T (v_0 = 1) applied to columns k+1..n-1: w = v^T a_j, a_j -= tau w v.
 *    xnorm == 0 gives tau = 0 (H = I). R on and above the diagonal, v below it.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define IDX(i, j, ld) ((size_t)(j) * (size_t)(ld) + (size_t)(i))

/* Unblocked Cholesky-Crout on the lower triangle of column-major a (n x n, leading dim lda).
 * The lower triangle is copied to a row-major work array w (storage only: the arithmetic is
 * the recurrence above, element by element, in the order written), factored, copied back.
 * The strict upper triangle of a is never read or written. Returns LAPACK info. */
int oracle_dpotrf_lower(int n, double* a, int lda) {
  if (n <= 0) return 0;
  double* w = (double*)malloc(sizeof(double) * (size_t)n * (size_t)n);
  if (!w) return -1000;
  for (int i = 0; i < n; ++i)
    for (int j = 0; j <= i; ++j) w[(size_t)i * n + j] = a[IDX(i, j, lda)];
  int info = 0;
  int done = n; /* number of columns fully computed */
  for (int j = 0; j < n; ++j) {
    const double* lj = w + (size_t)j * n;
    double s = w[(size_t)j * n + j];
    for (int k = 0; k < j; ++k) s = s - lj[k] * lj[k];
    if (!(s > 0.0)) { /* NaN or non-positive pivot: leading minor of order j+1 not PD */
      w[(size_t)j * n + j] = s;
      info = j + 1;
      done = j;
      break;
    }
    const double ljj = sqrt(s);
    w[(size_t)j * n + j] = ljj;
    for (int i = j + 1; i < n; ++i) {
      const double* li = w + (size_t)i * n;
      double t = li[j];
      for (int k = 0; k < j; ++k) t = t - li[k] * lj[k];
      w[(size_t)i * n + j] = t / ljj;
    }
  }
  /* Copy back: computed columns (all rows), plus the failing pivot. Columns after a
   * failure are left as they were in a (LAPACK stops there). */
  for (int j = 0; j < done; ++j)
    for (int i = j; i < n; ++i) a[IDX(i, j, lda)] = w[(size_t)i * n + j];
  if (info > 0) a[IDX(info - 1, info - 1, lda)] = w[(size_t)(info - 1) * n + (info - 1)];
  free(w);
  return info;
}

/* oracle_dpotrf_lower in IEEE single precision (same order of operations). */
int oracle_spotrf_lower(int n, float* a, int lda) {
  if (n <= 0) return 0;
  float* w = (float*)malloc(sizeof(float) * (size_t)n * (size_t)n);
  if (!w) return -1000;
  for (int i = 0; i < n; ++i)
    for (int j = 0; j <= i; ++j) w[(size_t)i * n + j] = a[IDX(i, j, lda)];
  int info = 0;
  int done = n;
  for (int j = 0; j < n; ++j) {
    const float* lj = w + (size_t)j * n;
    float s = w[(size_t)j * n + j];
    for (int k = 0; k < j; ++k) s = s - lj[k] * lj[k];
    if (!(s > 0.0f)) {
      w[(size_t)j * n + j] = s;
      info = j + 1;
      done = j;
      break;
    }
    const float ljj = sqrtf(s);
    w[(size_t)j * n + j] = ljj;
    for (int i = j + 1; i < n; ++i) {
      const float* li = w + (size_t)i * n;
      float t = li[j];
      for (int k = 0; k < j; ++k) t = t - li[k] * lj[k];
      w[(size_t)i * n + j] = t / ljj;
    }
  }
  for (int j = 0; j < done; ++j)
    for (int i = j; i < n; ++i) a[IDX(i, j, lda)] = w[(size_t)i * n + j];
  if (info > 0) a[IDX(info - 1, info - 1, lda)] = w[(size_t)(info - 1) * n + (info - 1)];
  free(w);
  return info;
}

/* The vbatched problem: matrix b is n[b] x n[b] at A[b] with leading dim lda[b]. */
void oracle_dpotrf_batch(int batch, const int* n, double* const* A, const int* lda, int* info,
                         int nthreads) {
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
  for (int b = 0; b < batch; ++b) info[b] = oracle_dpotrf_lower(n[b], A[b], lda[b]);
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* op(X)(i,j) for trans in {'N','T'} (also 'C' == 'T' for real data). */
static double opel(char t, const double* X, int ld, int i, int j) {
  return (t == 'N' || t == 'n') ? X[IDX(i, j, ld)] : X[IDX(j, i, ld)];
}

/* C = alpha op(A) op(B) + beta C, C m x n, op(A) m x k, op(B) k x n (BLAS DGEMM). */
void oracle_dgemm(char ta, char tb, int m, int n, int k, double alpha, const double* A, int lda,
                  const double* B, int ldb, double beta, double* C, int ldc) {
  for (int j = 0; j < n; ++j)
    for (int i = 0; i < m; ++i) {
      double s = 0.0;
      for (int p = 0; p < k; ++p) s = s + opel(ta, A, lda, i, p) * opel(tb, B, ldb, p, j);
      double c = (beta == 0.0) ? 0.0 : beta * C[IDX(i, j, ldc)];
      C[IDX(i, j, ldc)] = alpha * s + c;
    }
}

/* C = alpha op(A) op(A)^T + beta C on the `uplo` triangle of the n x n C (BLAS DSYRK):
 * trans 'N': A is n x k, op(A) op(A)^T = A A^T; trans 'T': A is k x n, = A^T A. */
void oracle_dsyrk(char uplo, char trans, int n, int k, double alpha, const double* A, int lda,
                  double beta, double* C, int ldc) {
  const int lower = (uplo == 'L' || uplo == 'l');
  const int notr = (trans == 'N' || trans == 'n');
  for (int j = 0; j < n; ++j)
    for (int i = 0; i < n; ++i) {
      if (lower ? (i < j) : (i > j)) continue;
      double s = 0.0;
      for (int p = 0; p < k; ++p) {
        double x = notr ? A[IDX(i, p, lda)] : A[IDX(p, i, lda)];
        double y = notr ? A[IDX(j, p, lda)] : A[IDX(p, j, lda)];
        s = s + x * y;
      }
      double c = (beta == 0.0) ? 0.0 : beta * C[IDX(i, j, ldc)];
      C[IDX(i, j, ldc)] = alpha * s + c;
    }
}

/* Triangular solve (BLAS DTRSM), B is m x n, overwritten by X:
 *   side 'L': op(A) X = alpha B   (A m x m);   side 'R': X op(A) = alpha B   (A n x n).
 * A is `uplo`-triangular ('L'/'U'), op = transA ('N'/'T'), diag 'U' = unit diagonal.
 * Plain substitution on the explicit triangular matrix T = op(A) (entries outside the
 * triangle of A are never read). */
void oracle_dtrsm(char side, char uplo, char transA, char diag, int m, int n, double alpha,
                  const double* A, int lda, double* B, int ldb) {
  const int left = (side == 'L' || side == 'l');
  const int lower = (uplo == 'L' || uplo == 'l');
  const int notr = (transA == 'N' || transA == 'n');
  const int unit = (diag == 'U' || diag == 'u');
  const int na = left ? m : n;
  /* T(i,j) = op(A)(i,j) restricted to A's triangle; T is lower iff (lower xor trans). */
  double* T = (double*)calloc((size_t)(na > 0 ? na : 1) * (size_t)(na > 0 ? na : 1), sizeof(double));
  for (int j = 0; j < na; ++j)
    for (int i = 0; i < na; ++i) {
      int ai = notr ? i : j, aj = notr ? j : i; /* element of A that is T(i,j) */
      int in_tri = lower ? (ai >= aj) : (ai <= aj);
      double v = in_tri ? A[IDX(ai, aj, lda)] : 0.0;
      if (ai == aj && unit) v = 1.0;
      T[(size_t)j * na + i] = v;
    }
  const int tlower = lower ^ (!notr);
  if (left) { /* T X = alpha B, column by column of B */
    for (int c = 0; c < n; ++c) {
      double* x = B + (size_t)c * ldb;
      for (int i = 0; i < m; ++i) x[i] = alpha * x[i];
      if (tlower) {
        for (int i = 0; i < m; ++i) {
          double s = x[i];
          for (int p = 0; p < i; ++p) s = s - T[(size_t)p * na + i] * x[p];
          x[i] = s / T[(size_t)i * na + i];
        }
      } else {
        for (int i = m - 1; i >= 0; --i) {
          double s = x[i];
          for (int p = i + 1; p < m; ++p) s = s - T[(size_t)p * na + i] * x[p];
          x[i] = s / T[(size_t)i * na + i];
        }
      }
    }
  } else { /* X T = alpha B, row by row of B: x T = b  <=>  T^T x^T = b^T */
    double* x = (double*)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    for (int r = 0; r < m; ++r) {
      for (int j = 0; j < n; ++j) x[j] = alpha * B[IDX(r, j, ldb)];
      if (tlower) { /* x_j = (b_j - sum_{p>j} x_p T(p,j)) / T(j,j), j descending */
        for (int j = n - 1; j >= 0; --j) {
          double s = x[j];
          for (int p = j + 1; p < n; ++p) s = s - x[p] * T[(size_t)j * na + p];
          x[j] = s / T[(size_t)j * na + j];
        }
      } else { /* upper T: j ascending */
        for (int j = 0; j < n; ++j) {
          double s = x[j];
          for (int p = 0; p < j; ++p) s = s - x[p] * T[(size_t)j * na + p];
          x[j] = s / T[(size_t)j * na + j];
        }
      }
      for (int j = 0; j < n; ++j) B[IDX(r, j, ldb)] = x[j];
    }
    free(x);
  }
  free(T);
}

/* Backward error ||A - L L^T||_F / (nb ||A||_F eps), eps = 2^-53, in long double.
 * A = full symmetric matrix rebuilt from the lower triangle of A0; L = lower triangle of Lf
 * (upper part taken as zero). nb = n if info == 0 else info-1 (leading block only,
 * SURVEY.md §8(c) readings #3, #13). Returns 0 for nb == 0. */
double oracle_backward_error(int n, const double* A0, int lda0, const double* Lf, int ldl,
                             int info) {
  int nb = info > 0 ? info - 1 : n;
  if (nb <= 0) return 0.0;
  long double num = 0.0L, den = 0.0L;
  for (int j = 0; j < nb; ++j)
    for (int i = 0; i < nb; ++i) {
      long double aij = (i >= j) ? (long double)A0[IDX(i, j, lda0)] : (long double)A0[IDX(j, i, lda0)];
      long double s = 0.0L;
      int kmax = i < j ? i : j;
      for (int k = 0; k <= kmax; ++k)
        s += (long double)Lf[IDX(i, k, ldl)] * (long double)Lf[IDX(j, k, ldl)];
      long double d = aij - s;
      num += d * d;
      den += aij * aij;
    }
  if (den == 0.0L) return num == 0.0L ? 0.0 : INFINITY;
  const long double eps = ldexpl(1.0L, -53);
  return (double)(sqrtl(num) / ((long double)nb * sqrtl(den) * eps));
}

/* Batched backward error (OpenMP over matrices). */
void oracle_backward_error_batch(int batch, const int* n, double* const* A0, const int* lda0,
                                 double* const* Lf, const int* ldl, const int* info, double* out,
                                 int nthreads) {
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
  for (int b = 0; b < batch; ++b)
    out[b] = oracle_backward_error(n[b], A0[b], lda0[b], Lf[b], ldl[b], info[b]);
}

/* LU with partial pivoting of the m x n column-major a (leading dim lda), in place: on return
 * the strict lower part holds L (unit diagonal not stored), the upper part U; ipiv[k] (1-based)
 * is the row interchanged with row k (k < min(m,n)). Returns LAPACK info (0, or the 1-based
 * index of the first exactly-zero pivot). */
int oracle_dgetrf(int m, int n, double* a, int lda, int* ipiv) {
  const int kmax = m < n ? m : n;
  int info = 0;
  for (int k = 0; k < kmax; ++k) {
    int p = k;
    double best = fabs(a[IDX(k, k, lda)]);
    for (int i = k + 1; i < m; ++i) {
      const double v = fabs(a[IDX(i, k, lda)]);
      if (v > best) { best = v; p = i; }
    }
    ipiv[k] = p + 1;
    if (a[IDX(p, k, lda)] != 0.0) {
      if (p != k)
        for (int j = 0; j < n; ++j) {
          const double t = a[IDX(k, j, lda)];
          a[IDX(k, j, lda)] = a[IDX(p, j, lda)];
          a[IDX(p, j, lda)] = t;
        }
      const double piv = a[IDX(k, k, lda)];
      for (int i = k + 1; i < m; ++i) a[IDX(i, k, lda)] = a[IDX(i, k, lda)] / piv;
    } else if (info == 0) {
      info = k + 1;
    }
    for (int j = k + 1; j < n; ++j) {
      const double ukj = a[IDX(k, j, lda)];
      for (int i = k + 1; i < m; ++i) a[IDX(i, j, lda)] = a[IDX(i, j, lda)] - a[IDX(i, k, lda)] * ukj;
    }
  }
  return info;
}

/* ||P A - L U||_F / (max(m,n) ||A||_F eps), eps = 2^-53, long double. A0: the original m x n
 * matrix; F: the factored one (L strictly below the diagonal, unit diagonal implied; U on and
 * above); ipiv as returned by DGETRF. P A is formed by applying the interchanges in order. */
double oracle_getrf_backward_error(int m, int n, const double* A0, int lda0, const double* F,
                                   int ldf, const int* ipiv) {
  const int kmax = m < n ? m : n;
  if (m <= 0 || n <= 0) return 0.0;
  long double* PA = (long double*)malloc(sizeof(long double) * (size_t)m * (size_t)n);
  for (int j = 0; j < n; ++j)
    for (int i = 0; i < m; ++i) PA[(size_t)j * m + i] = (long double)A0[IDX(i, j, lda0)];
  for (int k = 0; k < kmax; ++k) {
    const int p = ipiv[k] - 1;
    if (p != k)
      for (int j = 0; j < n; ++j) {
        const long double t = PA[(size_t)j * m + k];
        PA[(size_t)j * m + k] = PA[(size_t)j * m + p];
        PA[(size_t)j * m + p] = t;
      }
  }
  long double num = 0.0L, den = 0.0L;
  for (int j = 0; j < n; ++j)
    for (int i = 0; i < m; ++i) {
      long double s = 0.0L;
      const int kk = (i < j ? i : j) < kmax ? (i < j ? i : j) : kmax - 1;
      for (int k = 0; k <= kk && k < kmax; ++k) {
        const long double l = (i == k) ? 1.0L : (i > k ? (long double)F[IDX(i, k, ldf)] : 0.0L);
        const long double u = (k <= j) ? (long double)F[IDX(k, j, ldf)] : 0.0L;
        s += l * u;
      }
      const long double d = PA[(size_t)j * m + i] - s;
      num += d * d;
      den += PA[(size_t)j * m + i] * PA[(size_t)j * m + i];
    }
  free(PA);
  if (den == 0.0L) return num == 0.0L ? 0.0 : INFINITY;
  const long double eps = ldexpl(1.0L, -53);
  const int mx = m > n ? m : n;
  return (double)(sqrtl(num) / ((long double)mx * sqrtl(den) * eps));
}

/* Complex Cholesky-Crout on the lower triangle of an interleaved column-major n x n Hermitian
 * matrix (element (i,j) at a[2*(i + j*lda)] (re), [.. + 1] (im)). Returns LAPACK info. */
#define ZPOTRF_BODY(T, SQRT)                                                                    \
  if (n <= 0) return 0;                                                                        \
  T* w = (T*)malloc(sizeof(T) * 2 * (size_t)n * (size_t)n); /* row-major lower: w[2*(i*n+j)] */ \
  if (!w) return -1000;                                                                        \
  for (int i = 0; i < n; ++i)                                                                  \
    for (int j = 0; j <= i; ++j) {                                                             \
      w[2 * ((size_t)i * n + j)] = a[2 * IDX(i, j, lda)];                                      \
      w[2 * ((size_t)i * n + j) + 1] = (i == j) ? (T)0 : a[2 * IDX(i, j, lda) + 1];            \
    }                                                                                          \
  int info = 0, done = n;                                                                      \
  for (int j = 0; j < n; ++j) {                                                                \
    const T* lj = w + 2 * (size_t)j * n;                                                       \
    T s = lj[2 * j];                                                                           \
    for (int k = 0; k < j; ++k) s = s - (lj[2 * k] * lj[2 * k] + lj[2 * k + 1] * lj[2 * k + 1]); \
    if (!(s > (T)0)) {                                                                         \
      w[2 * ((size_t)j * n + j)] = s;                                                          \
      info = j + 1;                                                                            \
      done = j;                                                                                \
      break;                                                                                   \
    }                                                                                          \
    const T ljj = SQRT(s);                                                                     \
    w[2 * ((size_t)j * n + j)] = ljj;                                                          \
    w[2 * ((size_t)j * n + j) + 1] = (T)0;                                                     \
    for (int i = j + 1; i < n; ++i) {                                                          \
      T* li = w + 2 * (size_t)i * n;                                                           \
      T tr = li[2 * j], ti = li[2 * j + 1];                                                    \
      for (int k = 0; k < j; ++k) {                                                            \
        /* l_ik conj(l_jk) = (ar + i ai)(br - i bi) = (ar br + ai bi) + i (ai br - ar bi) */  \
        const T ar = li[2 * k], ai = li[2 * k + 1], br = lj[2 * k], bi = lj[2 * k + 1];        \
        tr = tr - (ar * br + ai * bi);                                                         \
        ti = ti - (ai * br - ar * bi);                                                         \
      }                                                                                        \
      li[2 * j] = tr / ljj;                                                                    \
      li[2 * j + 1] = ti / ljj;                                                                \
    }                                                                                          \
  }                                                                                            \
  for (int j = 0; j < done; ++j)                                                               \
    for (int i = j; i < n; ++i) {                                                              \
      a[2 * IDX(i, j, lda)] = w[2 * ((size_t)i * n + j)];                                      \
      a[2 * IDX(i, j, lda) + 1] = w[2 * ((size_t)i * n + j) + 1];                              \
    }                                                                                          \
  if (info > 0) {                                                                              \
    a[2 * IDX(info - 1, info - 1, lda)] = w[2 * ((size_t)(info - 1) * n + (info - 1))];        \
    a[2 * IDX(info - 1, info - 1, lda) + 1] = (T)0;                                            \
  }                                                                                            \
  free(w);                                                                                     \
  return info;

int oracle_zpotrf_lower(int n, double* a, int lda) { ZPOTRF_BODY(double, sqrt) }
int oracle_cpotrf_lower(int n, float* a, int lda) { ZPOTRF_BODY(float, sqrtf) }

/* ||A - L L^H||_F / (nb ||A||_F eps), eps = 2^-53, long double; A Hermitian rebuilt from the
 * lower triangle of A0 (diagonal imaginary part ignored), L = lower triangle of Lf (upper taken
 * as zero, diagonal imaginary part as stored). nb = n, or info-1 on failure. */
double oracle_zpotrf_backward_error(int n, const double* A0, int lda0, const double* Lf, int ldl,
                                    int info) {
  int nb = info > 0 ? info - 1 : n;
  if (nb <= 0) return 0.0;
  long double num = 0.0L, den = 0.0L;
  for (int j = 0; j < nb; ++j)
    for (int i = 0; i < nb; ++i) {
      long double ar, ai;
      if (i > j) { ar = A0[2 * IDX(i, j, lda0)]; ai = A0[2 * IDX(i, j, lda0) + 1]; }
      else if (i < j) { ar = A0[2 * IDX(j, i, lda0)]; ai = -(long double)A0[2 * IDX(j, i, lda0) + 1]; }
      else { ar = A0[2 * IDX(i, i, lda0)]; ai = 0.0L; }
      long double sr = 0.0L, si = 0.0L;
      const int kmax = i < j ? i : j;
      for (int k = 0; k <= kmax; ++k) {
        const long double xr = Lf[2 * IDX(i, k, ldl)], xi = Lf[2 * IDX(i, k, ldl) + 1];
        const long double yr = Lf[2 * IDX(j, k, ldl)], yi = Lf[2 * IDX(j, k, ldl) + 1];
        sr += xr * yr + xi * yi;
        si += xi * yr - xr * yi;
      }
      const long double dr = ar - sr, di = ai - si;
      num += dr * dr + di * di;
      den += ar * ar + ai * ai;
    }
  if (den == 0.0L) return num == 0.0L ? 0.0 : INFINITY;
  const long double eps = ldexpl(1.0L, -53);
  return (double)(sqrtl(num) / ((long double)nb * sqrtl(den) * eps));
}

/* Householder QR of the m x n column-major a (leading dim lda), in place; tau[min(m,n)]. */
void oracle_dgeqrf(int m, int n, double* a, int lda, double* tau) {
  const int kmax = m < n ? m : n;
  for (int k = 0; k < kmax; ++k) {
    double* x = a + IDX(k, k, lda);
    const double alpha = x[0];
    double ss = 0.0;
    for (int i = 1; i < m - k; ++i) ss = ss + x[i] * x[i];
    const double xnorm = sqrt(ss);
    if (xnorm == 0.0) {
      tau[k] = 0.0;
      continue; /* H = I: nothing to apply */
    }
    const double r = sqrt(alpha * alpha + xnorm * xnorm);
    const double beta = alpha >= 0.0 ? -r : r;
    tau[k] = (beta - alpha) / beta;
    const double den = alpha - beta;
    for (int i = 1; i < m - k; ++i) x[i] = x[i] / den;
    x[0] = beta;
    for (int j = k + 1; j < n; ++j) {
      double* y = a + IDX(k, j, lda);
      double w = y[0]; /* v_0 = 1 */
      for (int i = 1; i < m - k; ++i) w = w + x[i] * y[i];
      const double tw = tau[k] * w;
      y[0] = y[0] - tw;
      for (int i = 1; i < m - k; ++i) y[i] = y[i] - tw * x[i];
    }
  }
}

/* QR gates in long double: bwd = ||A - Q R||_F / (max(m,n) ||A||_F eps) and
 * orth = ||Q^T Q - I||_F / (m eps), with Q = H_0 H_1 ... H_(k-1) (m x m) formed explicitly
 * from the compact factor F (v below the diagonal, v_0 = 1) and tau; eps = 2^-53. */
void oracle_geqrf_errors(int m, int n, const double* A0, int lda0, const double* F, int ldf,
                         const double* tau, double* bwd, double* orth) {
  const int kmax = m < n ? m : n;
  *bwd = 0.0;
  *orth = 0.0;
  if (m <= 0 || n <= 0) return;
  long double* Q = (long double*)calloc((size_t)m * m, sizeof(long double));
  for (int i = 0; i < m; ++i) Q[(size_t)i * m + i] = 1.0L;
  /* Q = H_0 ... H_(k-1): apply in reverse to I from the left */
  for (int k = kmax - 1; k >= 0; --k) {
    for (int j = 0; j < m; ++j) {
      long double* q = Q + (size_t)j * m;
      long double w = q[k];
      for (int i = k + 1; i < m; ++i) w += (long double)F[IDX(i, k, ldf)] * q[i];
      const long double tw = (long double)tau[k] * w;
      q[k] -= tw;
      for (int i = k + 1; i < m; ++i) q[i] -= tw * (long double)F[IDX(i, k, ldf)];
    }
  }
  long double num = 0.0L, den = 0.0L;
  for (int j = 0; j < n; ++j)
    for (int i = 0; i < m; ++i) {
      long double s = 0.0L;
      for (int k = 0; k <= j && k < kmax; ++k) s += Q[(size_t)k * m + i] * (long double)F[IDX(k, j, ldf)];
      const long double a = A0[IDX(i, j, lda0)];
      num += (a - s) * (a - s);
      den += a * a;
    }
  long double on = 0.0L;
  for (int j = 0; j < m; ++j)
    for (int i = 0; i < m; ++i) {
      long double s = 0.0L;
      for (int k = 0; k < m; ++k) s += Q[(size_t)i * m + k] * Q[(size_t)j * m + k];
      const long double d = s - (i == j ? 1.0L : 0.0L);
      on += d * d;
    }
  free(Q);
  const long double eps = ldexpl(1.0L, -53);
  const int mx = m > n ? m : n;
  *bwd = den == 0.0L ? (num == 0.0L ? 0.0 : INFINITY) : (double)(sqrtl(num) / ((long double)mx * sqrtl(den) * eps));
  *orth = (double)(sqrtl(on) / ((long double)m * eps));
}
