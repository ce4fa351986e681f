/* orc_par.c — the "CPU-parallel" CONTEXT line of SURVEY §8d (test/bench infrastructure only,
 * like orc.c; never linked into the product): the SpMV and PageRank oracle loops of orc.c
 * with their independent outer loop (rows / pages) split over OpenMP threads.  Every row's
 * inner loop and every other sum keep orc.c's order (the dangling sum stays serial), so the
 * results are bit-identical to orc_spmv / orc_pagerank (pinned in tests/test_oracle_spmv.py
 * and tests/test_oracle_pagerank.py).  It is a reported baseline only; orc.c stays the
 * parity reference.  Passages: P5@10072 (SpMV), P5@9262 / P5@9781 (PageRank). */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <omp.h>

int orc_par_threads(void) { return omp_get_max_threads(); }

int orc_spmv_par(int64_t n_rows, const int64_t *row_ptr, const int32_t *col_idx, const float *val,
                 const float *x, double *y) {
  if (n_rows < 0 || !row_ptr || (n_rows > 0 && !y)) return -1;
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t i = 0; i < n_rows; ++i) {
    double s = 0.0;
    for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k)
      s += (double)val[k] * (double)x[col_idx[k]];
    y[i] = s;
  }
  return 0;
}

int orc_pagerank_par(int64_t n, const int64_t *in_row_ptr, const int32_t *in_col_idx,
                     const int32_t *out_degree, double damping, int32_t iterations, double *rank) {
  if (n < 0 || iterations < 0 || !(damping >= 0.0 && damping < 1.0)) return -1;
  if (n == 0) return 0;
  if (!in_row_ptr || !out_degree || !rank) return -1;
  double *next = (double *)malloc(sizeof(double) * (size_t)n);
  if (!next) return -2;
  for (int64_t v = 0; v < n; ++v) rank[v] = 1.0 / (double)n;
  for (int32_t t = 0; t < iterations; ++t) {
    double dangling = 0.0; /* serial, as in orc.c */
    for (int64_t u = 0; u < n; ++u)
      if (out_degree[u] == 0) dangling += rank[u];
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < n; ++v) {
      double s = 0.0;
      for (int64_t k = in_row_ptr[v]; k < in_row_ptr[v + 1]; ++k) {
        int32_t u = in_col_idx[k];
        s += rank[u] / (double)out_degree[u];
      }
      next[v] = (1.0 - damping) / (double)n + damping * (s + dangling / (double)n);
    }
    memcpy(rank, next, sizeof(double) * (size_t)n);
  }
  free(next);
  return 0;
}
