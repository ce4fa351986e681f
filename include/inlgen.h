/* inlgen.h — C-ABI of the seeded synthetic-input generator (module `inlgen/`).
 *
 * INPUT SIDE ONLY: nothing here computes any step of the paper's method
 * (Li, Wu, Becchi, ICPP'15).  The generator builds the CSR graphs the paper's
 * irregular nested loop runs over (PAPER.md P11@2195 "CSR", P5@9967 SpMV over
 * "Compressed Sparse Row"), with the shapes of SURVEY.md §8 (R-MAT, power-law
 * degrees), and the seeded values / weights / vectors.  Both the oracle tests
 * and the CUDA path consume these inputs; the host and device builders produce
 * bit-identical graphs (checked by tests/test_inlgen*.py).
 *
 * Conventions: every function returns 0 on success, a negative code on error
 * (-1 invalid argument, -2 out of memory, -3 CUDA error); inlgen_last_error()
 * returns a thread-local message.  CSR: row_ptr int64 [n_rows+1] with
 * row_ptr[0] == 0, col_idx int32 [nnz] global column ids, sorted and unique
 * within each row, no self-loops.
 */
#ifndef INLGEN_H
#define INLGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum {
  INLGEN_SYMMETRIC = 1, /* add (v,u) for every (u,v): undirected graph (SSSP/BFS) */
  INLGEN_TRANSPOSE = 2  /* store the in-edge CSR (rows = destinations) + out_degree (PageRank) */
};

typedef struct inlgen_graph_s *inlgen_graph;

const char *inlgen_last_error(void);

/* Philox4x32-10 block (known-answer tests). */
void inlgen_philox(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* The relabel bijection on [0, 2^scale). */
uint64_t inlgen_relabel(uint64_t x, int scale, uint64_t seed);
/* Raw R-MAT tuples e in [e_begin, e_begin+count), after relabel, self-loops kept. */
int inlgen_rmat_tuples(int scale, uint64_t seed, uint64_t e_begin, int64_t count, int64_t *u,
                       int64_t *v);

/* R-MAT graph with 2^scale vertices and edge_factor * 2^scale tuples; self-loops
 * dropped, duplicates merged, columns sorted.  Rows [row_begin, row_end) only
 * (row_end < 0 means n).  Host build: plain C (small scales).  Device build:
 * CUDA + CUB on the current device, stream = cudaStream_t (may be NULL). */
int inlgen_host_build(int scale, int edge_factor, uint64_t seed, int flags, int64_t row_begin,
                      int64_t row_end, inlgen_graph *out);
int inlgen_dev_build(int scale, int edge_factor, uint64_t seed, int flags, int64_t row_begin,
                     int64_t row_end, void *stream, inlgen_graph *out);
/* Sizes. on_device = 1 if the arrays live in device memory. */
int inlgen_graph_info(inlgen_graph g, int64_t *n_global, int64_t *n_rows, int64_t *row_begin,
                      int64_t *nnz, int *on_device);
/* Copy into caller buffers (host or device, any combination; cudaMemcpyDefault for
 * device graphs).  out_degree [n_global] is only available for INLGEN_TRANSPOSE
 * graphs (pass NULL otherwise). */
int inlgen_graph_export(inlgen_graph g, int64_t *row_ptr, int32_t *col_idx, int32_t *out_degree,
                        void *stream);
void inlgen_graph_free(inlgen_graph g);

/* Per-entry inputs for a (local) CSR whose row 0 is global row `row_begin`.
 * *_host: host arrays.  *_dev: device arrays, asynchronous on `stream`. */
int inlgen_weights_host(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                        const int32_t *col_idx, uint64_t seed, uint32_t *w);
int inlgen_weights_dev(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                       const int32_t *col_idx, uint64_t seed, uint32_t *w, void *stream);
/* mode 0: U[0,1) fp32; mode 1: integers 1..255 (bit-exact integer SpMV test). */
int inlgen_values_host(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                       const int32_t *col_idx, uint64_t seed, int mode, float *val);
int inlgen_values_dev(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                      const int32_t *col_idx, uint64_t seed, int mode, float *val, void *stream);
/* x[i] for global i in [begin, begin+n). mode 0: U[0,1); mode 1: integers 0..15. */
int inlgen_vector_host(int64_t n, int64_t begin, uint64_t seed, int mode, float *x);
int inlgen_vector_dev(int64_t n, int64_t begin, uint64_t seed, int mode, float *x, void *stream);

#ifdef __cplusplus
}
#endif
#endif
