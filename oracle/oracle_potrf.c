/*
 * ORACLE -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU Cholesky factorisation used to check the
 * CUDA path.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this file's library.  It shares no code,
 * header, table or helper with paper_conf_sc_augonnetasg24_b200/ (the product).
 *
 * What it computes (the plain definition, SURVEY.md §8(c) "Definition"):
 *   for symmetric positive definite A (lower triangle referenced), the unique
 *   lower-triangular L with positive diagonal such that A = L * L^T
 *   ("Cholesky decomposition", §VII-C; tiled
 *   algorithm of ref. [17]).  The tiled right-looking method the
 *   GPU runs is a reordering of the same elimination with the same n^3/3
 *   flops, so the oracle is the element-wise definition of A = L L^T solved
 *   column by column (unblocked Cholesky-Crout):
 *
 *     for j = 0 .. n-1:
 *         s = A[j][j] - sum_{k<j} L[j][k]^2           (k ascending)
 *         if !(s > 0): return info = j+1               (also catches NaN)
 *         L[j][j] = sqrt(s)                            (IEEE correctly rounded)
 *         for i = j+1 .. n-1:                          (OpenMP over rows)
 *             L[i][j] = (A[i][j] - sum_{k<j} L[i][k]*L[j][k]) / L[j][j]
 *     L[i][j] = 0 for j > i
 *
 * No blocking, no reordering, no fused multiply-add (built with
 * -ffp-contract=off).  L is stored row-major so both dot products walk
 * contiguous memory.
 *
 * Non-SPD input (LAPACK convention): the return value is
 * the 1-based index of the first column whose pivot s is not > 0; L is then
 * defined only for the columns before it.
 *
 * Build: gcc -O3 -fopenmp -ffp-contract=off -shared -fPIC -o liboracle.so oracle_potrf.c -lm
 */
#include <math.h>
#include <stdint.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* A: n x n column-major, leading dimension lda (only i >= j read).
 * L: n x n row-major output (L[i*n + k]); strictly upper part set to 0.
 * nthreads <= 0 -> OpenMP default.  Returns info (0 = success). */
int64_t oracle_potrf(int64_t n, const double *A, int64_t lda, double *L, int nthreads) {
  if (n <= 0) return 0;
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
  memset(L, 0, (size_t)n * (size_t)n * sizeof(double));
  for (int64_t j = 0; j < n; ++j) {
    const double *Lj = L + j * n;
    double s = A[j + j * lda];
    for (int64_t k = 0; k < j; ++k) s -= Lj[k] * Lj[k];
    if (!(s > 0.0)) return j + 1;
    const double d = sqrt(s);
    L[j * n + j] = d;
#pragma omp parallel for schedule(static)
    for (int64_t i = j + 1; i < n; ++i) {
      const double *Li = L + i * n;
      double t = A[i + j * lda];
      for (int64_t k = 0; k < j; ++k) t -= Li[k] * Lj[k];
      L[i * n + j] = t / d;
    }
  }
  return 0;
}

/* Threads OpenMP will use for the parallel loop (reported as `cores`). */
int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
