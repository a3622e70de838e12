/* fp64 CPU oracle in plain C — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
 *
 * The same definitions as oracle/spmv.py (SURVEY c-1) and oracle/sgemm.py
 * (c-2), as straight loops: used for the CPU baseline timing in bench.py and
 * pinned against the numpy oracle and a triple loop in tests/test_oracle_sgemm.py
 * (test_c_oracle_spmv, test_c_oracle_gemm).
 *   y_i = sum_{k in row i} (double)val_k * (double)x[col_k]   (CSR order;
 *         SHOC spmv-csr scalar, §4.2)
 *   C   = alpha * A B + beta * C0, row-major, fp64 accumulation
 *         (Parboil sgemm, §4.3)
 * Threads: rows (SpMV) and rows of C (GEMM) are split statically over
 * `nthreads` OpenMP threads; each output is computed by exactly one thread in
 * the sequential order above, so the result does not depend on nthreads.
 */
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

void oracle_spmv_f64(int64_t n, const int32_t *row_ptr, const int32_t *col,
                     const float *val, const float *x, double *y, int nthreads) {
#pragma omp parallel for schedule(static) num_threads(nthreads)
  for (int64_t i = 0; i < n; ++i) {
    double s = 0.0;
    for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k)
      s += (double)val[k] * (double)x[col[k]];
    y[i] = s;
  }
}

void oracle_gemm_f64(int64_t M, int64_t N, int64_t K, double alpha,
                     const float *A, const float *B, double beta,
                     const float *C0, double *C, int nthreads) {
#pragma omp parallel for schedule(static) num_threads(nthreads)
  for (int64_t i = 0; i < M; ++i) {
    for (int64_t j = 0; j < N; ++j) C[i * N + j] = 0.0;
    for (int64_t k = 0; k < K; ++k) {          /* ikj: row of B streamed */
      double a = (double)A[i * K + k];
      for (int64_t j = 0; j < N; ++j) C[i * N + j] += a * (double)B[k * N + j];
    }
    for (int64_t j = 0; j < N; ++j)
      C[i * N + j] = alpha * C[i * N + j] + beta * (double)C0[i * N + j];
  }
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
