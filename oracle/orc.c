/* orc.c — the ORACLE (test infrastructure only; see orc.h).
 *
 * Plain single-threaded C99, fp64 for floating point.  Each function is the
 * textbook definition of the application the paper evaluates, written out
 * with no blocking, fusion or reordering, so it can be checked by eye.
 *
 * Paper: Li, Wu, Becchi, "Nested Parallelism on GPU: Exploring
 * Parallelization Templates for Irregular Loops and Recursive Computations",
 * ICPP 2015 — /root/reference/PAPER.md (citations P<line>@<char offset>).
 * The parallelization templates (thread/block mapping, dual queue, delayed
 * buffer; P3@9322, P5@2078, P5@2721) only re-map this loop nest, so every
 * template must produce the result computed here.  Readings of silent or
 * ambiguous points are listed in DESIGN.md §3 ("Readings").
 *
 * Pins (tests/test_oracle_*.py, run with -m "not gpu") tie every function to
 * closed forms, brute force and library routines independent of this file.
 */
#include "orc.h"

#include <stdlib.h>
#include <string.h>

const char *orc_version(void) { return "orc 1.0 (fp64 CPU oracle)"; }

/* SpMV — P5@10072: "calculates the product of a sparse matrix and a dense
 * vector"; P5@10497: "the sparse matrix is represented in Compressed Sparse
 * Row format, the nested loop within the matrix multiplication algorithm is
 * irregular."  Outer loop over rows i, inner loop over the row's nonzeros
 * (Fig. 1(a) pattern, P3@9300).  The fp32 inputs are promoted to fp64 and
 * accumulated in row order (reading R2). */
int orc_spmv(int64_t n_rows, const int64_t *row_ptr, const int32_t *col_idx, const float *val,
             const float *x, double *y) {
  if (n_rows < 0 || !row_ptr || (n_rows > 0 && !y)) return -1;
  for (int64_t i = 0; i < n_rows; ++i) {
    double s = 0.0;
    for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k)
      s += (double)val[k] * (double)x[col_idx[k]];
    y[i] = s;
  }
  return 0;
}

/* PageRank — P5@9262 ("PageRank is a popular graph analysis algorithm to rank
 * web pages ... implementation described in [7]") and P5@9781: "each
 * iteration of the outer loop processes a different webpage (node in a
 * graph); the inner loop collects ranks from the neighbors of the considered
 * node" — a pull over in-neighbours.  The paper gives no formula; reading R1
 * (DESIGN.md): damping d, teleport (1-d)/n, PR^0 = 1/n, the rank of dangling
 * pages (out-degree 0) redistributed uniformly, a fixed iteration count. */
int orc_pagerank(int64_t n, const int64_t *in_row_ptr, const int32_t *in_col_idx,
                 const int32_t *out_degree, double damping, int32_t iterations, double *rank) {
  if (n < 0 || iterations < 0 || !(damping >= 0.0 && damping < 1.0)) return -1;
  if (n == 0) return 0;
  if (!in_row_ptr || !out_degree || !rank) return -1;
  double *next = (double *)malloc(sizeof(double) * (size_t)n);
  if (!next) return -2;
  for (int64_t v = 0; v < n; ++v) rank[v] = 1.0 / (double)n;
  for (int32_t t = 0; t < iterations; ++t) {
    double dangling = 0.0; /* D^t = sum of PR^t over pages with no out-links */
    for (int64_t u = 0; u < n; ++u)
      if (out_degree[u] == 0) dangling += rank[u];
    for (int64_t v = 0; v < n; ++v) {
      double s = 0.0; /* inner loop: collect ranks from the in-neighbours */
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

/* SSSP — P5@10183/P5@10241: "For SSSP, we used the thread-mapped
 * implementation described in [5] as baseline"; P11@2218: the graph is
 * "encode[d] ... in Compressed Sparse Row (CSR) format" and "its traversal
 * assumes the form of the nested loop in Figure 1(a), where the outer loop
 * iterates over the nodes in the graph, and the inner loop over [their]
 * neighbors".  [5] (Harish & Narayanan) iterates Bellman-Ford relaxations to
 * a fixed point; with non-negative weights that fixed point is the unique
 * vector of shortest-path distances, which Dijkstra computes directly
 * (reading R4).  Binary heap with lazy deletion; int64 accumulator. */
typedef struct { uint64_t d; int64_t v; } orc_heap_item;

static void heap_push(orc_heap_item *h, int64_t *sz, uint64_t d, int64_t v) {
  int64_t i = (*sz)++;
  h[i].d = d;
  h[i].v = v;
  while (i > 0) {
    int64_t p = (i - 1) / 2;
    if (h[p].d <= h[i].d) break;
    orc_heap_item t = h[p]; h[p] = h[i]; h[i] = t;
    i = p;
  }
}

static orc_heap_item heap_pop(orc_heap_item *h, int64_t *sz) {
  orc_heap_item top = h[0];
  h[0] = h[--(*sz)];
  int64_t i = 0;
  for (;;) {
    int64_t l = 2 * i + 1, r = l + 1, m = i;
    if (l < *sz && h[l].d < h[m].d) m = l;
    if (r < *sz && h[r].d < h[m].d) m = r;
    if (m == i) break;
    orc_heap_item t = h[m]; h[m] = h[i]; h[i] = t;
    i = m;
  }
  return top;
}

int orc_sssp_dijkstra(int64_t n, const int64_t *row_ptr, const int32_t *col_idx,
                      const uint32_t *w, int64_t source, uint32_t *dist) {
  if (n < 0 || source < 0 || source >= n || !row_ptr || !dist) return -1;
  const uint64_t INF = UINT64_MAX;
  uint64_t *d = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)n);
  int64_t nnz = row_ptr[n];
  orc_heap_item *h = (orc_heap_item *)malloc(sizeof(orc_heap_item) * (size_t)(nnz + 1));
  if (!d || !h) { free(d); free(h); return -2; }
  for (int64_t v = 0; v < n; ++v) d[v] = INF;
  int64_t sz = 0;
  d[source] = 0;
  heap_push(h, &sz, 0, source);
  while (sz > 0) {
    orc_heap_item it = heap_pop(h, &sz);
    if (it.d != d[it.v]) continue; /* stale entry (lazy deletion) */
    int64_t u = it.v;
    for (int64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
      int64_t v = col_idx[k];
      uint64_t nd = d[u] + (uint64_t)w[k];
      if (nd < d[v]) {
        d[v] = nd;
        heap_push(h, &sz, nd, v);
      }
    }
  }
  int rc = 0;
  for (int64_t v = 0; v < n; ++v) {
    if (d[v] == INF) dist[v] = UINT32_MAX;
    else if (d[v] >= (uint64_t)UINT32_MAX) { dist[v] = UINT32_MAX; rc = -4; }
    else dist[v] = (uint32_t)d[v];
  }
  free(d);
  free(h);
  return rc;
}

/* BFS — P5@11250/P5@11591: "For BFS, we used the thread-mapped implementation
 * described in [5] ... This implementation is work-efficient and traverses
 * the graph level by level."  A FIFO queue visits vertices in level order;
 * level[v] = number of edges on a shortest path from source (reading R5). */
int orc_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t source,
            int32_t *level) {
  if (n < 0 || source < 0 || source >= n || !row_ptr || !level) return -1;
  int64_t *queue = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  if (!queue) return -2;
  for (int64_t v = 0; v < n; ++v) level[v] = -1;
  int64_t head = 0, tail = 0;
  level[source] = 0;
  queue[tail++] = source;
  while (head < tail) {
    int64_t u = queue[head++];
    for (int64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
      int64_t v = col_idx[k];
      if (level[v] == -1) {
        level[v] = level[u] + 1;
        queue[tail++] = v;
      }
    }
  }
  free(queue);
  return 0;
}

/* Betweenness centrality: Brandes, "A faster algorithm for betweenness centrality"
 * (J. Math. Sociol. 2001), Algorithm 1 for unweighted graphs, the method the paper's [6]
 * parallelises (P5@8911: "First, it constructs the shortest paths tree using BFS ...;
 * second, it computes the BC value by traversing the shortest path tree").  Per source:
 * FIFO BFS recording sigma (shortest-path counts) and the visit order S; then vertices in
 * reverse visit order accumulate delta; bc[w] += delta[w] for w != s. */
int orc_bc(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const int64_t *sources,
           int64_t n_sources, double *bc) {
  if (n < 0 || n_sources < 0 || !row_ptr || (n > 0 && !bc) || (n_sources > 0 && !sources)) return -1;
  for (int64_t i = 0; i < n_sources; ++i)
    if (sources[i] < 0 || sources[i] >= n) return -1;
  for (int64_t v = 0; v < n; ++v) bc[v] = 0.0;
  if (n == 0) return 0;
  int64_t *S = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  int64_t *dist = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  double *sigma = (double *)malloc(sizeof(double) * (size_t)n);
  double *delta = (double *)malloc(sizeof(double) * (size_t)n);
  if (!S || !dist || !sigma || !delta) {
    free(S); free(dist); free(sigma); free(delta);
    return -2;
  }
  for (int64_t i = 0; i < n_sources; ++i) {
    const int64_t s = sources[i];
    for (int64_t v = 0; v < n; ++v) {
      dist[v] = -1;
      sigma[v] = 0.0;
      delta[v] = 0.0;
    }
    dist[s] = 0;
    sigma[s] = 1.0;
    int64_t head = 0, tail = 0; /* S doubles as the BFS queue: visit order */
    S[tail++] = s;
    while (head < tail) {
      const int64_t v = S[head++];
      for (int64_t k = row_ptr[v]; k < row_ptr[v + 1]; ++k) {
        const int64_t w = col_idx[k];
        if (dist[w] < 0) {
          dist[w] = dist[v] + 1;
          S[tail++] = w;
        }
        if (dist[w] == dist[v] + 1) sigma[w] += sigma[v];
      }
    }
    /* reverse visit order: every successor of w is finished before w */
    for (int64_t j = tail - 1; j >= 0; --j) {
      const int64_t w = S[j];
      for (int64_t k = row_ptr[w]; k < row_ptr[w + 1]; ++k) {
        const int64_t v = col_idx[k];
        if (dist[v] == dist[w] + 1) delta[w] += sigma[w] / sigma[v] * (1.0 + delta[v]);
      }
      if (w != s) bc[w] += delta[w];
    }
  }
  free(S);
  free(dist);
  free(sigma);
  free(delta);
  return 0;
}

/* Tree descendants and heights — PAPER.md §II.C (P5@5170-7323, Fig. 3(a)): "the recursive
 * computation of the number of descendants in a tree ... the descendants array, which stores
 * the number of descendants of all nodes, is initialized to all 1s (that is, every node is a
 * descendant of itself)"; Tree Heights is "similar code" (P5@11250).  Fig. 3(a)'s recursion
 *   descendants(v) = 1 + sum_{c child of v} descendants(c)
 *   height(v)      = 1 + max_{c child of v} height(c)   (a leaf: 1; reading R14)
 * evaluated without recursion: nodes in BFS order from the root, then in reverse, so every
 * child is finished before its parent.  Input: the children CSR; nodes not reachable from
 * `root` get 0. */
static int orc_tree_order(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t root,
                          int64_t *order, int64_t *count) {
  if (n <= 0 || root < 0 || root >= n) return -1;
  char *seen = (char *)calloc((size_t)n, 1);
  if (!seen) return -2;
  int64_t head = 0, tail = 0;
  order[tail++] = root;
  seen[root] = 1;
  while (head < tail) {
    const int64_t v = order[head++];
    for (int64_t k = row_ptr[v]; k < row_ptr[v + 1]; ++k) {
      const int64_t c = col_idx[k];
      if (c < 0 || c >= n || seen[c]) { free(seen); return -1; } /* not a tree */
      seen[c] = 1;
      order[tail++] = c;
    }
  }
  free(seen);
  *count = tail;
  return 0;
}

int orc_tree_descendants(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t root,
                         int64_t *desc) {
  if (n < 0 || (n > 0 && (!row_ptr || !desc))) return -1;
  if (n == 0) return 0;
  int64_t *order = (int64_t *)malloc(sizeof(int64_t) * (size_t)n), cnt = 0;
  if (!order) return -2;
  const int rc = orc_tree_order(n, row_ptr, col_idx, root, order, &cnt);
  if (rc) { free(order); return rc; }
  for (int64_t v = 0; v < n; ++v) desc[v] = 0;
  for (int64_t j = cnt - 1; j >= 0; --j) {
    const int64_t v = order[j];
    int64_t s = 1;
    for (int64_t k = row_ptr[v]; k < row_ptr[v + 1]; ++k) s += desc[col_idx[k]];
    desc[v] = s;
  }
  free(order);
  return 0;
}

int orc_tree_heights(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t root,
                     int64_t *height) {
  if (n < 0 || (n > 0 && (!row_ptr || !height))) return -1;
  if (n == 0) return 0;
  int64_t *order = (int64_t *)malloc(sizeof(int64_t) * (size_t)n), cnt = 0;
  if (!order) return -2;
  const int rc = orc_tree_order(n, row_ptr, col_idx, root, order, &cnt);
  if (rc) { free(order); return rc; }
  for (int64_t v = 0; v < n; ++v) height[v] = 0;
  for (int64_t j = cnt - 1; j >= 0; --j) {
    const int64_t v = order[j];
    int64_t h = 0;
    for (int64_t k = row_ptr[v]; k < row_ptr[v + 1]; ++k)
      if (height[col_idx[k]] > h) h = height[col_idx[k]];
    height[v] = 1 + h;
  }
  free(order);
  return 0;
}
