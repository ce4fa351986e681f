/* inlgen_graph.h — private graph handle of the inlgen module. */
#ifndef INLGEN_GRAPH_H
#define INLGEN_GRAPH_H
#include <stdint.h>

struct inlgen_graph_s {
  int64_t n_global;
  int64_t n_rows;
  int64_t row_begin;
  int64_t nnz;
  int on_device;
  int64_t *row_ptr;    /* [n_rows+1] */
  int32_t *col_idx;    /* [nnz] */
  int32_t *out_degree; /* [n_global] or NULL */
  float *val;          /* [nnz] or NULL (loaded matrices with values; host graphs only) */
  int32_t *parent;     /* [n_global] or NULL (trees from inlgen_tree_build) */
};

#ifdef __cplusplus
extern "C" {
#endif
void inlgen_set_error(const char *fmt, ...);
#ifdef __cplusplus
}
#endif

#endif
