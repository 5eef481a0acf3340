/*
 * oracle/bqr_ref.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct double-precision CPU Householder QR used as
 * the parity oracle for the CUDA path.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the product library
 * (paper_conf_ipps_andersonsk12_b200/csrc); neither side includes the other.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:L<n>"):
 *   - Householder QR "because it is consistent with LAPACK" (Sec. III-C)
 *     -> LAPACK xGEQR2 with xLARFG / xLARF semantics, step by step, in the
 *     order the paper's Table VI lists for one column:
 *       column norm -> (sqrt, two divides, two multiplies) -> scale the column
 *       -> matrix-vector multiply -> rank-1 update.
 *   - Q formation (xORG2R / xUNG2R) for bqr_orgqr_batched, and Q^H B
 *     (xORM2R / xUNM2R, SIDE='L', TRANS='T'/'C') for bqr_apply_qh_batched,
 *     the latter being the paper's least-squares use "apply Q^T to b"
 *     (Sec. III-D).
 *   - Real (double) and complex (double _Complex, interleaved re/im) flavours;
 *     the complex one is the paper's STAP workload (Sec. VII).
 *
 * Readings of silent / garbled passages (DESIGN.md "Readings" Q1-Q10):
 *   Q2  k = min(m,n) reflectors; real: a 1-row reflector is the identity
 *       (tau = 0), complex: a 1-row reflector with Im(alpha) != 0 is NOT
 *       skipped (it makes R's diagonal real), as in ZLARFG.
 *   Q3  beta = -sign(Re alpha) * sqrt(|alpha|^2 + ||x||^2)  (LAPACK sign rule)
 *   Q4  sign taken with copysign semantics: alpha = -0.0 gives beta = +nu.
 *   Q5  ||x|| == 0 (and Im alpha == 0 for complex) -> tau = 0, column untouched.
 *   Q6  no dnrm2-style scaling and no safmin rescale loop: plain serial sum of
 *       squares (the paper's "serial reduction by thread 0", Table VI).
 *   Q9  the trailing update applies H^H = I - conj(tau) v v^H  (ZGEQR2).
 *
 * Pins (tests/test_oracle_*.py): hand-worked 2x2/3x3 reflectors and edge cases,
 * LAPACK (scipy dgeqrf/zgeqrf, dorgqr/zungqr, dormqr/zunmqr), invariants
 * (||R e_j|| = ||A e_j||, R = D chol(A^H A)^H, |det R| = |det A|, tau ranges,
 * augmented least squares), Givens brute force on tiny inputs.
 *
 * Layout: batch of column-major matrices, matrix b at A + b*lda*n elements,
 * tau of matrix b at tau + b*min(m,n).  Complex arrays are interleaved
 * (re, im) doubles, i.e. numpy complex128.
 */
#include <complex.h>
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef double _Complex zc;

static int g_threads = 0; /* 0 -> OpenMP default (all available cores) */

void bqr_ref_set_threads(int n) { g_threads = n; }

int bqr_ref_max_threads(void) {
#ifdef _OPENMP
  return g_threads > 0 ? g_threads : omp_get_max_threads();
#else
  return 1;
#endif
}

static inline int imin(int a, int b) { return a < b ? a : b; }

/* ------------------------------------------------------------------------ */
/* Real double                                                               */
/* ------------------------------------------------------------------------ */

/* xLARFG (real), P:L689 / Table VI "Column": norm of the sub-column, then
 * "a square root, two divides, and two multiplies" by one thread.
 * alpha = a[0], x = a[1..len-1].  Returns tau; writes beta into a[0] and
 * v[1..] = x/(alpha-beta) into a[1..].  *margin = |alpha| / nu (sign-tie
 * detector for the comparator), 1 when the reflector is skipped. */
static double larfg_d(int len, double *a, double *margin) {
  *margin = 1.0;
  if (len <= 1) return 0.0;
  double alpha = a[0];
  double sigma = 0.0;
  for (int r = 1; r < len; ++r) sigma += a[r] * a[r];
  if (sigma == 0.0) return 0.0;
  double nu = sqrt(alpha * alpha + sigma);
  double beta = -copysign(nu, alpha);
  double tau = (beta - alpha) / beta;
  double scal = 1.0 / (alpha - beta);
  for (int r = 1; r < len; ++r) a[r] *= scal;
  a[0] = beta;
  *margin = fabs(alpha) / nu;
  return tau;
}

/* Apply (I - t v v^T) from the left to the rows x cols block C (ldc), where
 * v[0] = 1 implicitly and v[1..rows-1] = vtail[0..rows-2].
 * Table VI "Trailing Matrix": matrix-vector multiply w = C^T v, then the
 * rank-1 update C -= t v w^T (Listing 7). */
static void larf_left_d(int rows, int cols, const double *vtail, double t,
                        double *C, int ldc) {
  if (t == 0.0) return;
  for (int j = 0; j < cols; ++j) {
    double *c = C + (size_t)j * ldc;
    double w = c[0];
    for (int r = 1; r < rows; ++r) w += vtail[r - 1] * c[r];
    double tw = t * w;
    c[0] -= tw;
    for (int r = 1; r < rows; ++r) c[r] -= vtail[r - 1] * tw;
  }
}

/* One matrix, LAPACK DGEQR2.  margin may be NULL. */
static void geqr2_d(int m, int n, double *A, int lda, double *tau,
                    double *margin) {
  int k = imin(m, n);
  for (int i = 0; i < k; ++i) {
    double *col = A + (size_t)i * lda + i;
    double mg;
    double t = larfg_d(m - i, col, &mg);
    tau[i] = t;
    if (margin) margin[i] = mg;
    if (i < n - 1)
      larf_left_d(m - i, n - i - 1, col + 1, t, col + lda, lda);
  }
}

/* LAPACK DORG2R: A (m x n, first k columns hold the reflectors) <- first n
 * columns of Q = H_0 H_1 ... H_{k-1}. */
static void org2r_d(int m, int n, int k, double *A, int lda, const double *tau) {
  for (int j = k; j < n; ++j) {
    double *c = A + (size_t)j * lda;
    for (int r = 0; r < m; ++r) c[r] = 0.0;
    c[j] = 1.0;
  }
  for (int i = k - 1; i >= 0; --i) {
    double *col = A + (size_t)i * lda + i;
    if (i < n - 1)
      larf_left_d(m - i, n - i - 1, col + 1, tau[i], col + lda, lda);
    for (int r = 1; r < m - i; ++r) col[r] *= -tau[i];
    col[0] = 1.0 - tau[i];
    for (int r = 0; r < i; ++r) A[(size_t)i * lda + r] = 0.0;
  }
}

/* LAPACK DORM2R('L','T'): B (m x nrhs) <- Q^T B, Q = H_0 ... H_{k-1}, i.e.
 * apply H_0 first.  The paper's least-squares step. */
static void apply_qt_d(int m, int k, int nrhs, const double *A, int lda,
                       const double *tau, double *B, int ldb) {
  for (int i = 0; i < k; ++i)
    larf_left_d(m - i, nrhs, A + (size_t)i * lda + i + 1, tau[i], B + i, ldb);
}

/* ------------------------------------------------------------------------ */
/* Complex double (STAP)                                       */
/* ------------------------------------------------------------------------ */

static inline double abs2(zc z) { return creal(z) * creal(z) + cimag(z) * cimag(z); }

/* ZLARFG: alpha complex; the result beta is real; tau = ((beta - Re a)/beta,
 * -Im a / beta); x scaled by 1/(alpha - beta). */
static zc larfg_z(int len, zc *a, double *margin) {
  *margin = 1.0;
  if (len <= 0) return 0.0;
  zc alpha = a[0];
  double sigma = 0.0;
  for (int r = 1; r < len; ++r) sigma += abs2(a[r]);
  double ar = creal(alpha), ai = cimag(alpha);
  if (sigma == 0.0 && ai == 0.0) return 0.0;
  double nu = sqrt(ar * ar + ai * ai + sigma);
  double beta = -copysign(nu, ar);
  zc tau = CMPLX((beta - ar) / beta, -ai / beta);
  zc scal = 1.0 / (alpha - beta);
  for (int r = 1; r < len; ++r) a[r] *= scal;
  a[0] = CMPLX(beta, 0.0);
  *margin = fabs(ar) / nu;
  return tau;
}

/* Apply (I - t v v^H) from the left: w_j = sum_r conj(v_r) C[r,j];
 * C[r,j] -= t v_r w_j. */
static void larf_left_z(int rows, int cols, const zc *vtail, zc t, zc *C,
                        int ldc) {
  if (t == 0.0) return;
  for (int j = 0; j < cols; ++j) {
    zc *c = C + (size_t)j * ldc;
    zc w = c[0];
    for (int r = 1; r < rows; ++r) w += conj(vtail[r - 1]) * c[r];
    zc tw = t * w;
    c[0] -= tw;
    for (int r = 1; r < rows; ++r) c[r] -= vtail[r - 1] * tw;
  }
}

/* ZGEQR2: the trailing update applies H_i^H = I - conj(tau_i) v v^H (Q9). */
static void geqr2_z(int m, int n, zc *A, int lda, zc *tau, double *margin) {
  int k = imin(m, n);
  for (int i = 0; i < k; ++i) {
    zc *col = A + (size_t)i * lda + i;
    double mg;
    zc t = larfg_z(m - i, col, &mg);
    tau[i] = t;
    if (margin) margin[i] = mg;
    if (i < n - 1)
      larf_left_z(m - i, n - i - 1, col + 1, conj(t), col + lda, lda);
  }
}

/* ZUNG2R: Q = H_0 H_1 ... H_{k-1}, H_i = I - tau_i v v^H. */
static void org2r_z(int m, int n, int k, zc *A, int lda, const zc *tau) {
  for (int j = k; j < n; ++j) {
    zc *c = A + (size_t)j * lda;
    for (int r = 0; r < m; ++r) c[r] = 0.0;
    c[j] = 1.0;
  }
  for (int i = k - 1; i >= 0; --i) {
    zc *col = A + (size_t)i * lda + i;
    if (i < n - 1)
      larf_left_z(m - i, n - i - 1, col + 1, tau[i], col + lda, lda);
    for (int r = 1; r < m - i; ++r) col[r] *= -tau[i];
    col[0] = 1.0 - tau[i];
    for (int r = 0; r < i; ++r) A[(size_t)i * lda + r] = 0.0;
  }
}

/* ZUNM2R('L','C'): B <- Q^H B = H_{k-1}^H ... H_0^H B. */
static void apply_qh_z(int m, int k, int nrhs, const zc *A, int lda,
                       const zc *tau, zc *B, int ldb) {
  for (int i = 0; i < k; ++i)
    larf_left_z(m - i, nrhs, A + (size_t)i * lda + i + 1, conj(tau[i]), B + i,
                ldb);
}

/* ------------------------------------------------------------------------ */
/* Batched entry points (OpenMP over independent matrices)            */
/* ------------------------------------------------------------------------ */

#define OMP_FOR _Pragma("omp parallel for schedule(static) num_threads(bqr_ref_max_threads())")

void bqr_ref_geqrf_d(int m, int n, int64_t batch, double *A, int lda,
                     double *tau, double *margin) {
  int k = imin(m, n);
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b)
    geqr2_d(m, n, A + b * (int64_t)lda * n, lda, tau + b * k,
            margin ? margin + b * k : NULL);
}

void bqr_ref_geqrf_z(int m, int n, int64_t batch, double *A, int lda,
                     double *tau, double *margin) {
  int k = imin(m, n);
  zc *Az = (zc *)A, *tz = (zc *)tau;
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b)
    geqr2_z(m, n, Az + b * (int64_t)lda * n, lda, tz + b * k,
            margin ? margin + b * k : NULL);
}

void bqr_ref_orgqr_d(int m, int n, int k, int64_t batch, double *A, int lda,
                     const double *tau) {
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b)
    org2r_d(m, n, k, A + b * (int64_t)lda * n, lda, tau + b * k);
}

void bqr_ref_orgqr_z(int m, int n, int k, int64_t batch, double *A, int lda,
                     const double *tau) {
  zc *Az = (zc *)A;
  const zc *tz = (const zc *)tau;
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b)
    org2r_z(m, n, k, Az + b * (int64_t)lda * n, lda, tz + b * k);
}

/* A holds n columns per matrix (batch stride lda*n) of which the first k are
 * reflectors; tau stride is k; B stride ldb*nrhs. */
void bqr_ref_apply_qh_d(int m, int n, int k, int nrhs, int64_t batch,
                        const double *A, int lda, const double *tau, double *B,
                        int ldb) {
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b)
    apply_qt_d(m, k, nrhs, A + b * (int64_t)lda * n, lda, tau + b * k,
               B + b * (int64_t)ldb * nrhs, ldb);
}

void bqr_ref_apply_qh_z(int m, int n, int k, int nrhs, int64_t batch,
                        const double *A, int lda, const double *tau, double *B,
                        int ldb) {
  const zc *Az = (const zc *)A, *tz = (const zc *)tau;
  zc *Bz = (zc *)B;
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b)
    apply_qh_z(m, k, nrhs, Az + b * (int64_t)lda * n, lda, tz + b * k,
               Bz + b * (int64_t)ldb * nrhs, ldb);
}

/* ------------------------------------------------------------------------ */
/* Least squares (paper Sec. III-D):                             */
/*   "find the QR factorization of A, apply Q^T to b, and solve the          */
/*    resulting upper triangular system for x ... We compute Q^T b by        */
/*    appending b to the right side of the matrix during the factorization.  */
/*    We then solve the upper triangular system using row operations."       */
/* Here: geqr2 of A, Q^H B (the appended columns, xORM2R), then backward     */
/* elimination on [R | c] by row operations: for j = n-1 .. 0,               */
/* x_j = c_j / R_jj, then row j times x_j is subtracted from rows 0..j-1.    */
/* On exit B[0:n] = X and B[n:m] = the residual components (Q^H B)[n:m]      */
/* (LAPACK xGELS convention: ||A x - b||^2 = sum of their squares).          */
/* info = 0, or j+1 for the first j with R_jj == 0 (solution undefined).     */
/* ------------------------------------------------------------------------ */

static int backsolve_d(int n, int nrhs, const double *R, int lda, double *B,
                       int ldb) {
  int info = 0;
  for (int j = 0; j < n; ++j)
    if (R[(size_t)j * lda + j] == 0.0 && !info) info = j + 1;
  for (int r = 0; r < nrhs; ++r) {
    double *c = B + (size_t)r * ldb;
    for (int j = n - 1; j >= 0; --j) {
      const double xj = c[j] / R[(size_t)j * lda + j];
      c[j] = xj;
      for (int i = 0; i < j; ++i) c[i] -= R[(size_t)j * lda + i] * xj;
    }
  }
  return info;
}

static int backsolve_z(int n, int nrhs, const zc *R, int lda, zc *B, int ldb) {
  int info = 0;
  for (int j = 0; j < n; ++j)
    if (R[(size_t)j * lda + j] == 0.0 && !info) info = j + 1;
  for (int r = 0; r < nrhs; ++r) {
    zc *c = B + (size_t)r * ldb;
    for (int j = n - 1; j >= 0; --j) {
      const zc xj = c[j] / R[(size_t)j * lda + j];
      c[j] = xj;
      for (int i = 0; i < j; ++i) c[i] -= R[(size_t)j * lda + i] * xj;
    }
  }
  return info;
}

/* A (m x n, m >= n) is overwritten by its QR factorization, tau (stride n),
 * B (m x nrhs, stride ldb*nrhs) by [X; residual components]. */
void bqr_ref_gels_d(int m, int n, int nrhs, int64_t batch, double *A, int lda,
                    double *tau, double *B, int ldb, int *info) {
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b) {
    double *Ab = A + b * (int64_t)lda * n, *Bb = B + b * (int64_t)ldb * nrhs;
    geqr2_d(m, n, Ab, lda, tau + b * n, NULL);
    apply_qt_d(m, n, nrhs, Ab, lda, tau + b * n, Bb, ldb);
    const int inf = backsolve_d(n, nrhs, Ab, lda, Bb, ldb);
    if (info) info[b] = inf;
  }
}

void bqr_ref_gels_z(int m, int n, int nrhs, int64_t batch, double *A, int lda,
                    double *tau, double *B, int ldb, int *info) {
  zc *Az = (zc *)A, *tz = (zc *)tau, *Bz = (zc *)B;
  OMP_FOR
  for (int64_t b = 0; b < batch; ++b) {
    zc *Ab = Az + b * (int64_t)lda * n, *Bb = Bz + b * (int64_t)ldb * nrhs;
    geqr2_z(m, n, Ab, lda, tz + b * n, NULL);
    apply_qh_z(m, n, nrhs, Ab, lda, tz + b * n, Bb, ldb);
    const int inf = backsolve_z(n, nrhs, Ab, lda, Bb, ldb);
    if (info) info[b] = inf;
  }
}

