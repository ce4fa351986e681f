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

/* ---- loaders and the CiteSeer-shaped generator: host graphs ---- */
/* MatrixMarket coordinate file (real / integer / pattern; general / symmetric; 1-based):
 * self-loops dropped, repeated (row, col) pairs merged keeping the FIRST value, columns sorted.
 * flags: INLGEN_SYMMETRIC adds (v,u) for every (u,v); INLGEN_TRANSPOSE stores the in-edge CSR
 * + out_degree (both need a square matrix).  Values (non-pattern files) via
 * inlgen_graph_values.  Returns 0, -1 bad argument, -2 out of memory, -3 file / format error. */
int inlgen_load_mtx(const char *path, int flags, inlgen_graph *out);
/* .inlcsr binary file (little-endian): 8-byte magic "INLCSR\0\1"; int64 n_global, n_rows,
 * row_begin, nnz, flags (1: values follow, 2: out_degree follows); int64 row_ptr[n_rows+1];
 * int32 col_idx[nnz]; [float val[nnz]]; [int32 out_degree[n_global]].  Loading checks the
 * structure (row_ptr[0] = 0, non-decreasing, = nnz at the end, columns in range). */
int inlgen_save_csr(const char *path, inlgen_graph g);
int inlgen_load_csr(const char *path, inlgen_graph *out);
/* A host graph from caller arrays (copied; val / out_degree may be NULL). */
int inlgen_graph_from_csr(int64_t n_global, int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                          const int32_t *col_idx, const float *val, const int32_t *out_degree,
                          inlgen_graph *out);
int inlgen_graph_values(inlgen_graph g, float *val); /* -1 if the graph has none */
/* Undirected configuration-model graph on n vertices whose degree sequence follows a discrete
 * truncated power law on [dmin, dmax] with the given mean (exponent solved by bisection);
 * stubs paired by a Philox-keyed shuffle; both directions stored, self-loops and repeated
 * pairs removed (so realised degrees can be slightly lower).  The CiteSeer shape of PAPER.md
 * P5@12491-13052: n = 434102, dmin = 1, dmax = 1188, mean 73.9 (~32.1 M CSR entries). */
int inlgen_powerlaw_build(int64_t n, int dmin, int dmax, double mean, uint64_t seed, int flags,
                          inlgen_graph *out);

/* Synthetic tree of PAPER.md §III.C: `depth` levels, every non-leaf node
 * has `outdegree` children, a node below the last level has children with probability
 * (1/2)^sparsity (the root always).  Level-order ids (root 0, siblings consecutive); the
 * children CSR is the graph, parent[] (parent[0] = -1) via inlgen_graph_parent. */
int inlgen_tree_build(int depth, int outdegree, int sparsity, uint64_t seed, inlgen_graph *out);
int inlgen_graph_parent(inlgen_graph g, int32_t *parent);

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
