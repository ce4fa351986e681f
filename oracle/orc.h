/* orc.h — the ORACLE: plain, slow, obviously-correct CPU reference for the
 * paper's irregular-nested-loop applications (Li, Wu, Becchi, ICPP'15,
 * /root/reference/PAPER.md; citations P<line>@<char> as in SURVEY.md §0).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py (cpu_baseline leg and --impl reference) may load liborc.so.  The
 * product path (libinl.so, paper_conf_icpp_liwb15_b200/) never includes,
 * links or calls anything here, and this file includes nothing from it.
 *
 * Single-threaded C, fp64 arithmetic for floating point, int64 for integer
 * path lengths.  No blocking, fusion or reordering: each function is the
 * textbook definition written out (see oracle/orc.c for the passages).
 *
 * Return codes: 0 ok, -1 invalid argument, -2 out of memory,
 *               -4 result does not fit the output type (SSSP distance >= 2^32-1).
 */
#ifndef ORC_H
#define ORC_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

const char *orc_version(void);

/* SpMV: y[i] = sum_{k in [row_ptr[i], row_ptr[i+1])} val[k] * x[col_idx[k]]   (fp64) */
int orc_spmv(int64_t n_rows, const int64_t *row_ptr, const int32_t *col_idx, const float *val,
             const float *x, double *y);

/* PageRank (pull over the in-edge CSR), `iterations` synchronous steps:
 *   PR^0 = 1/n;  D^t = sum_{outdeg(u)=0} PR^t(u)
 *   PR^{t+1}(v) = (1-d)/n + d * ( sum_{u->v} PR^t(u)/outdeg(u) + D^t/n )        (fp64) */
int orc_pagerank(int64_t n, const int64_t *in_row_ptr, const int32_t *in_col_idx,
                 const int32_t *out_degree, double damping, int32_t iterations, double *rank);

/* SSSP: exact distances by Dijkstra (binary heap, lazy deletion), weights >= 0.
 * dist[v] = UINT32_MAX if unreachable. */
int orc_sssp_dijkstra(int64_t n, const int64_t *row_ptr, const int32_t *col_idx,
                      const uint32_t *w, int64_t source, uint32_t *dist);

/* BFS: hop levels by a FIFO queue; level[v] = -1 if unreachable, level[source] = 0. */
int orc_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t source,
            int32_t *level);

/* Betweenness centrality (PAPER.md P5@8318-8911: "equal to the number of shortest paths
 * from all nodes to all others that pass through that node"; two phases after [6]: a BFS
 * shortest-path tree of the unweighted graph, then a backward pass over it).  Reading
 * R10: Freeman/Brandes betweenness over ordered pairs of the given sources,
 *   bc[v] = sum_{s in sources} sum_{t != s, t != v} sigma_st(v) / sigma_st
 * computed by Brandes' recurrence delta_s(w) = sum_{v: w in P_s(v)} sigma_sw/sigma_sv (1 + delta_s(v)),
 * sigma and delta in fp64.  All n vertices as sources = exact BC. */
int orc_bc(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const int64_t *sources,
           int64_t n_sources, double *bc);

/* Tree descendants / heights (§II.C Fig. 3(a), §III.C) over the
 * children CSR of a tree rooted at `root`:
 *   desc[v]   = 1 + sum_{c child of v} desc[c]          (every node descends from itself)
 *   height[v] = 1 + max_{c child of v} height[c]         (a leaf has height 1; reading R14)
 * int64; nodes not reachable from root get 0.  -1 if the CSR is not a tree below root. */
int orc_tree_descendants(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t root,
                         int64_t *desc);
int orc_tree_heights(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, int64_t root,
                     int64_t *height);

#ifdef __cplusplus
}
#endif
#endif
