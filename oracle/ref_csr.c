/* oracle/ref_csr.c — O1: the plain definition y = A·x.
 * TEST INFRASTRUCTURE ONLY (see oracle/__init__.py): only tests/, smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.
 *
 * y[i] = sum_j A[i][j] * x[j] over the CSR row, accumulated with the compensated dot
 * product Dot2 of Ogita, Rump & Oishi (TwoProduct via fma + TwoSum), in fp64, in column
 * order.  For fp32 inputs the operands are widened to fp64 first (each product is then
 * exact).  bound[i] = sum_j |A[i][j]| * |x[j]| (plain fp64) scales the tolerance
 * (BASELINE.json north_star: |y - y_ref| <= tol * bound).
 * Rows are independent; OpenMP splits them dynamically (skewed rows).
 * Must be compiled with -ffp-contract=off (TwoSum/TwoProduct need unfused a*b and +).
 */
#include <stdint.h>
#include <math.h>
#include <omp.h>

#define DOT2_BODY(VT, XT)                                                          \
  _Pragma("omp parallel for schedule(dynamic, 256)")                               \
  for (int64_t i = 0; i < m; ++i) {                                                \
    double s = 0.0, c = 0.0, bnd = 0.0;                                            \
    for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k) {                        \
      double a = (double)((const VT*)val)[k];                                      \
      double b = (double)((const XT*)x)[col[k]];                                   \
      double p = a * b;                                                            \
      double pe = fma(a, b, -p);               /* TwoProduct error term */         \
      double t = s + p;                        /* TwoSum(s, p) */                  \
      double z = t - s;                                                            \
      double se = (s - (t - z)) + (p - z);                                         \
      s = t;                                                                       \
      c += pe + se;                                                                \
      bnd += fabs(a) * fabs(b);                                                    \
    }                                                                              \
    y[i] = s + c;                                                                  \
    if (bound) bound[i] = bnd;                                                     \
  }

/* dtype: 0 = fp32 (val and x float), 1 = fp64 */
int ref_spmv_dot2(int64_t m, const int64_t* row_ptr, const int32_t* col, const void* val,
                  const void* x, int dtype, double* y, double* bound) {
  if (dtype == 0) { DOT2_BODY(float, float) }
  else if (dtype == 1) { DOT2_BODY(double, double) }
  else return -1;
  return 0;
}

/* The same definition on a subset of rows (sampled-row parity at full size). */
int ref_spmv_rows(int64_t nrows, const int64_t* rows, const int64_t* row_ptr, const int32_t* col,
                  const void* val, const void* x, int dtype, double* y, double* bound) {
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t q = 0; q < nrows; ++q) {
    int64_t i = rows[q];
    double s = 0.0, c = 0.0, bnd = 0.0;
    for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k) {
      double a = dtype == 0 ? (double)((const float*)val)[k] : ((const double*)val)[k];
      double b = dtype == 0 ? (double)((const float*)x)[col[k]] : ((const double*)x)[col[k]];
      double p = a * b;
      double pe = fma(a, b, -p);
      double t = s + p;
      double z = t - s;
      double se = (s - (t - z)) + (p - z);
      s = t;
      c += pe + se;
      bnd += fabs(a) * fabs(b);
    }
    y[q] = s + c;
    if (bound) bound[q] = bnd;
  }
  return 0;
}

int ref_num_threads(void) {
  int n = 1;
#pragma omp parallel
  {
#pragma omp single
    n = omp_get_num_threads();
  }
  return n;
}
