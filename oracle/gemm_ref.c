/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg may load this library.  The product path
 * (paper_conf_ppopp_li0yjl19_b200/) never links, imports or calls it.
 *
 * Plain definition of the result (PAPER.md P31, §1; restated at P133, §2.2):
 *
 *     C_i = alpha_i * A_i x B_i + beta_i * C_i,   A_i in R^{M_i x K_i}, B_i in R^{K_i x N_i}
 *
 * computed as a textbook triple loop in fp64 over inputs that were converted exactly to fp64
 * (bf16 / fp16 / fp32 -> fp64 is exact).  Row-major storage with leading dimensions in
 * elements (reading C-15).  BLAS rules (reading C-16): beta == 0 means C is not
 * read (so NaN in C does not propagate); M == 0 or N == 0 is a no-op; K == 0 gives
 * C = beta * C.  No blocking, no fusion, no reordering beyond the i-k-j loop order.
 *
 * Work is split over (gemm, row) pairs with OpenMP so both big batches and a single large
 * GEMM use every host core; each C element is still produced by exactly one thread with
 * the same summation order (k ascending), so the result does not depend on thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static int64_t find_gemm(const int64_t *row_start, int64_t batch, int64_t t) {
  /* largest g with row_start[g] <= t */
  int64_t lo = 0, hi = batch - 1;
  while (lo < hi) {
    int64_t mid = (lo + hi + 1) / 2;
    if (row_start[mid] <= t) lo = mid; else hi = mid - 1;
  }
  return lo;
}

int vbref_gemm(int64_t batch, const int64_t *M, const int64_t *N, const int64_t *K,
               const double *const *A, const int64_t *lda,
               const double *const *B, const int64_t *ldb,
               double *const *C, const int64_t *ldc,
               const double *alpha, const double *beta, int nthreads) {
  if (batch < 0) return 1;
  if (batch == 0) return 0;
  int64_t *row_start = (int64_t *)malloc(sizeof(int64_t) * (size_t)(batch + 1));
  if (!row_start) return 2;
  int64_t total = 0, maxn = 0;
  for (int64_t g = 0; g < batch; ++g) {
    if (M[g] < 0 || N[g] < 0 || K[g] < 0) { free(row_start); return 1; }
    row_start[g] = total;
    total += (N[g] > 0) ? M[g] : 0;
    if (N[g] > maxn) maxn = N[g];
  }
  row_start[batch] = total;
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
#pragma omp parallel
  {
    double *acc = (double *)malloc(sizeof(double) * (size_t)(maxn > 0 ? maxn : 1));
#pragma omp for schedule(dynamic, 16)
    for (int64_t t = 0; t < total; ++t) {
      int64_t g = find_gemm(row_start, batch, t); /* empty GEMMs share a start; the last wins */
      int64_t i = t - row_start[g];
      int64_t n = N[g], k = K[g];
      const double *a = A[g] + i * lda[g];
      double *c = C[g] + i * ldc[g];
      for (int64_t j = 0; j < n; ++j) acc[j] = 0.0;
      for (int64_t p = 0; p < k; ++p) {            /* i-k-j order */
        const double aip = a[p];
        const double *b = B[g] + p * ldb[g];
        for (int64_t j = 0; j < n; ++j) acc[j] += aip * b[j];
      }
      const double al = alpha[g], be = beta[g];
      if (be == 0.0) {
        for (int64_t j = 0; j < n; ++j) c[j] = al * acc[j];
      } else {
        for (int64_t j = 0; j < n; ++j) c[j] = al * acc[j] + be * c[j];
      }
    }
    free(acc);
  }
  free(row_start);
  return 0;
}

int vbref_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
