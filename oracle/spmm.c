/* oracle/spmm.c — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
 *
 * Plain fp64 sparse products used by the CPU oracle of the GNN-RDM hot path.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may
 * load this library; the product path (paper_conf_ipps_kurtysps23_b200/)
 * never does.  Shares no code with the CUDA path.
 *
 * Definitions followed:
 *   eq. (1) L71  Z^l = A^T H^{l-1} W^l           -> oracle_spmm_t  (A^T X)
 *   eq. (3) L77  G^{l-1} = A G^l (W^l)^T ⊙ ...    -> oracle_spmm    (A X)
 *   eq. (4) L79  Y^l = (H^{l-1})^T A G^l          -> oracle_spmm    (A X)
 * A is an N x N CSR matrix (int64 rowptr, int32 col, fp32 values promoted to
 * fp64); X, Y are dense row-major fp64 N x f.
 */
#include <stdint.h>
#include <string.h>
#include <omp.h>

/* Y = A X :  Y[i,:] = sum_{p in row i} a_p * X[col_p, :] */
void oracle_spmm(int64_t n, const int64_t* rowptr, const int32_t* col, const float* val,
                 const double* X, int64_t f, double* Y) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double* y = Y + i * f;
    for (int64_t c = 0; c < f; ++c) y[c] = 0.0;
    for (int64_t p = rowptr[i]; p < rowptr[i + 1]; ++p) {
      const double a = (double)val[p];
      const double* x = X + (int64_t)col[p] * f;
      for (int64_t c = 0; c < f; ++c) y[c] += a * x[c];
    }
  }
}

/* Y = A^T X :  for every stored a_ij,  Y[j,:] += a_ij * X[i,:]
 * (the definition of the transpose product, written as a scatter; each
 * thread owns a disjoint range of feature columns so no two threads write
 * the same element). */
void oracle_spmm_t(int64_t n, const int64_t* rowptr, const int32_t* col, const float* val,
                   const double* X, int64_t f, double* Y) {
  memset(Y, 0, sizeof(double) * (size_t)(n * f));
#pragma omp parallel
  {
    int nt = omp_get_num_threads(), t = omp_get_thread_num();
    int64_t c0 = f * t / nt, c1 = f * (t + 1) / nt;
    if (c1 > c0) {
      for (int64_t i = 0; i < n; ++i) {
        const double* x = X + i * f;
        for (int64_t p = rowptr[i]; p < rowptr[i + 1]; ++p) {
          const double a = (double)val[p];
          double* y = Y + (int64_t)col[p] * f;
          for (int64_t c = c0; c < c1; ++c) y[c] += a * x[c];
        }
      }
    }
  }
}

/* Selected rows of A X (rows[0..m)), X given with leading dimension ldx and
 * f columns; Y is m x f.  Used for sampled parity at full sizes: one output
 * row needs only that row's neighbours. */
void oracle_spmm_rows(const int64_t* rowptr, const int32_t* col, const float* val,
                      const float* X, int64_t ldx, int64_t f, const int64_t* rows, int64_t m,
                      double* Y) {
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t r = 0; r < m; ++r) {
    const int64_t i = rows[r];
    double* y = Y + r * f;
    for (int64_t c = 0; c < f; ++c) y[c] = 0.0;
    for (int64_t p = rowptr[i]; p < rowptr[i + 1]; ++p) {
      const double a = (double)val[p];
      const float* x = X + (int64_t)col[p] * ldx;
      for (int64_t c = 0; c < f; ++c) y[c] += a * (double)x[c];
    }
  }
}

int oracle_num_threads(void) { return omp_get_max_threads(); }

/* Thread count of the loops above (bench.py times the oracle at nproc and at 1). */
void oracle_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }
