/* inl.h — C-ABI of libinl.so: the B200-native (sm_100a) hot path of
 *   Li, Wu, Becchi, "Nested Parallelism on GPU: Exploring Parallelization
 *   Templates for Irregular Loops and Recursive Computations", ICPP 2015
 *   (/root/reference/PAPER.md; citations P<line>@<char offset>).
 *
 * The hot path is the paper's irregular nested loop (Fig. 1(a), P3@9300):
 *     for i in outer (CSR rows / vertices):  for j < f(i) (nonzeros / edges): work(i, j)
 * load-balanced by the degree f(i) against thresholds (lbTHRES, P5@366,
 * P11@1197): small rows thread-mapped; larger rows deferred to warp-, block-
 * or grid-mapped buffers (the dual-queue / delayed-buffer templates, P5@2078,
 * P5@2721, P5@3623), instantiated for SpMV (P5@10072), SSSP (P5@10241),
 * PageRank (P5@9262) and BFS (P5@11591).
 *
 * Conventions (all entry points):
 *   - Return inl_status; nothing aborts and no C++ exception crosses the ABI.
 *     On failure, inl_last_error(ctx) holds a message for that ctx.
 *   - Array arguments may be DEVICE pointers (the fast path: results are
 *     produced asynchronously on the ctx stream for SpMV/PageRank) or HOST
 *     pointers (pageable or pinned): host inputs are copied to device scratch
 *     owned by the ctx and host outputs copied back before the call returns
 *     (the end-to-end path).  The caller owns every array; the library never
 *     frees or retains caller memory and never writes inputs.
 *   - CSR: row_ptr int64 [n_rows+1], row_ptr[0] == 0, non-decreasing;
 *     col_idx int32 [nnz] global column ids in [0, n_global).  Contents are
 *     not checked on the hot path (malformed CSR = undefined behaviour unless
 *     inl_csr_validate is called).  Rows are local to a rank: global row id =
 *     row_begin + local row (row_begin = 0, n_rows = n_global on one GPU).
 *   - A ctx is not thread-safe; use one ctx per host thread / rank.
 *   - Multi-GPU: every rank calls the same ops in the same order (NCCL rule);
 *     ranks own contiguous row blocks from inl_partition_rows.
 */
#ifndef INL_H
#define INL_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  INL_OK = 0,
  INL_ERR_INVALID_ARGUMENT = 1,
  INL_ERR_OUT_OF_MEMORY = 2,
  INL_ERR_CUDA = 3,
  INL_ERR_NCCL = 4,
  INL_ERR_NOT_INITIALIZED = 5,
  INL_ERR_UNSUPPORTED = 6,
  INL_ERR_INTERNAL = 7
} inl_status;

typedef struct inl_ctx_s *inl_ctx;   /* device, stream, optional NCCL comm, scratch arena */
typedef struct inl_plan_s *inl_plan; /* degree bins / work queues for one CSR on one ctx */

typedef struct {
  int64_t n_rows;         /* local rows on this rank (= n_global on one GPU) */
  int64_t n_global;       /* global vertex / column count n */
  int64_t row_begin;      /* global id of local row 0 (0 on one GPU) */
  int64_t nnz;            /* local nnz = row_ptr[n_rows] */
  const int64_t *row_ptr; /* [n_rows+1] */
  const int32_t *col_idx; /* [nnz] */
} inl_csr;

/* Load-balancing thresholds (the paper's lbTHRES, P5@366; 0 = default).
 *
 * What each kernel family actually reads (a threshold not listed is ignored by it):
 *  - DEFAULT fused kernels (no template flag).  The deferral threshold lbTHRES is t_warp:
 *      SpMV / PageRank (k_gather): rows of degree <= t_warp form row tiles (one warp per
 *        tile; inside a tile a row contained in one lane's 8 entries is summed serially by
 *        that lane — thread-mapped — and a row crossing lanes by the warp's segmented scan
 *        — warp-mapped; which of the two a row gets depends on its length and alignment,
 *        not on t_thread); rows of degree > t_warp are cut into grid_chunk pieces, one warp
 *        each, combined in piece order (the delayed buffer).  t_block only splits the
 *        reported counts (rows_block / rows_grid); t_thread only splits rows_thread /
 *        rows_warp in inl_plan_info.
 *      SSSP / BFS (k_expand_flat, k_expand_grid): frontier vertices of degree <= t_warp are
 *        buffered in shared memory and expanded CTA-wide, 8 edges per thread
 *        (dbuf-shared); larger ones go to the global buffer as min(grid_chunk, 2048)-edge
 *        pieces (dbuf-global).  t_thread and t_block are not read.
 *  - The paper's templates (INL_BINS_TPL_*) and the T1 baseline: lbTHRES = t_thread, CTA =
 *    cta_threads; the rows / vertices of degree > t_thread are block-mapped (SSSP/BFS
 *    dbuf-global: through the global buffer in min(grid_chunk, 2048)-edge pieces).
 * Ties go to the lower class (reading R6 of DESIGN.md: "f(i) greater than lbTHRES is
 * processed block-mapped", P11@1197).  t_thread = -1 means 0.
 * flags: INL_BINS_THREAD_ONLY runs the paper's baseline (thread-mapped outer loop,
 * no load balancing, P5@14490).  INL_BINS_COLBLOCK (opt-in; measured slower at the
 * bench configs) processes SpMV/PR rows of degree > max(t_warp,
 * 4 * column blocks) column-blocked: a CTA holds one block of x in shared memory and
 * sums the row's entries in that block (one partial per (row, block) run, combined in
 * block order).  SSSP on one GPU runs its near-far step loop on the device as ONE CUDA-graph
 * launch per source (a conditional WHILE node; one host round trip per call);
 * INL_BINS_SSSP_DEVLOOP keeps that device loop even when the environment variable
 * INL_SSSP_LOOP=host selects the host-driven loop (measurement switch).  At most one
 * INL_BINS_TPL_* flag, and none combined with another flag (else INL_ERR_INVALID_ARGUMENT
 * from inl_plan_create). */
enum {
  INL_BINS_THREAD_ONLY = 1,
  INL_BINS_COLBLOCK = 2,
  INL_BINS_SSSP_DEVLOOP = 4,
  /* The paper's templates, as it describes them (template study):
   * lbTHRES = t_thread (rows / vertices of degree > t_thread are block-mapped).
   * SpMV: dual-queue (Fig. 1(b), P5@2074), dbuf-global and dbuf-shared (Fig. 1(c),
   * P5@2717), CTA = cta_threads.  SSSP / BFS: dual-queue (a pre-pass splits the frontier;
   * thread- and block-mapped kernels), dbuf-shared and dbuf-global (256-thread CTAs; plain
   * frontier Bellman-Ford / top-down BFS like the T1 baseline).  PageRank (one GPU): each
   * iteration is the template SpMV with unit values over the in-CSR, then an elementwise
   * update (INL_BINS_THREAD_ONLY: the T1 gather). */
  INL_BINS_TPL_DUAL_QUEUE = 8,
  INL_BINS_TPL_DBUF_GLOBAL = 16,
  INL_BINS_TPL_DBUF_SHARED = 32
};
typedef struct {
  int32_t t_thread;    /* default 8; <= t_warp */
  int32_t t_warp;      /* default 1024, in [16, 4096] (SpMV/PR tiles hold < 2048 + t_warp nnz) */
  int32_t t_block;     /* default 16384, >= t_warp */
  int32_t grid_chunk;  /* default 8192 nnz per SpMV/PR long-row piece (one warp each), in [32, 2^20];
                          SSSP/BFS pieces are min(grid_chunk, 2048) edges */
  int32_t cta_threads; /* CTA size of the INL_BINS_TPL_* templates (multiple of 32 in [32, 1024],
                          default 256); the default kernels use fixed CTA shapes */
  int32_t flags;
} inl_bins;

typedef struct {
  int32_t iterations;     /* frontier iterations / BFS levels executed */
  int64_t edges_relaxed;  /* edges examined: the degrees of all frontier vertices expanded (top-down /
                             push steps) + the neighbours read by BFS bottom-up steps */
  int64_t frontier_total; /* sum of frontier sizes over the iterations */
  int64_t launches;       /* kernels the call launched (memsets and copies excluded) */
  int64_t host_syncs;     /* host <-> device round trips of the iteration loop */
  int64_t exchange_bytes; /* P > 1: bytes this rank moved through the exchange:
                             collectives by the ring model (allreduce 2(P-1)/P * size, allgather
                             (P-1)/P * size); NEXT-1 peer-memory exchange: 4 B per remote atomic
                             (counted on the device) + the peers' bitmap words read */
} inl_stats;

/* Plan summary (for tests and the bench; counts per bin). */
typedef struct {
  int64_t n_tiles;        /* row tiles holding the rows of degree <= t_warp */
  /* degree-class histogram by the thresholds (f <= t_thread, <= t_warp, <= t_block, above):
     a diagnostic of the CSR's shape — see inl_bins for which classes a kernel maps differently */
  int64_t rows_thread, rows_warp, rows_block, rows_grid;
  int64_t nnz_thread, nnz_warp, nnz_block, nnz_grid;
  int64_t n_grid_chunks;  /* CTAs of the grid/long-row kernel */
  inl_bins bins;          /* thresholds in effect */
  int64_t cb_rows;        /* SpMV rows processed column-blocked (0: none) */
  int64_t cb_runs;        /* their (row, column block) runs = partial sums */
  int64_t cb_nnz;         /* their nonzeros */
  int64_t cb_width;       /* column-block width K (x floats held in shared memory) */
  int64_t cb_threshold;   /* rows of degree > cb_threshold are column-blocked */
  int64_t symmetric;      /* 1: every edge's reverse is present (full square CSR with sorted rows);
                             enables BFS bottom-up and BC pull steps for calls using this plan */
} inl_plan_info;

const char *inl_version(void);
const char *inl_status_string(inl_status s);
const char *inl_last_error(inl_ctx ctx);

/* device: CUDA ordinal; cuda_stream: cudaStream_t (NULL = legacy default stream). */
inl_status inl_ctx_create(inl_ctx *out, int device, void *cuda_stream);
inl_status inl_ctx_set_stream(inl_ctx ctx, void *cuda_stream);
inl_status inl_ctx_destroy(inl_ctx ctx);

/* Row-block partition (host only, no GPU needed): bounds[p] = min(p*B, n),
 * B = ceil(n / nranks), p = 0..nranks.  Equal block sizes keep the NCCL
 * allgather counts equal (the last block is padded). */
inl_status inl_partition_rows(int64_t n, int32_t nranks, int64_t *bounds);

/* NCCL bootstrap: rank 0 calls inl_nccl_unique_id and broadcasts the 128 bytes
 * (torch.distributed in the Python binding); every rank then calls inl_comm_init.
 * Once a ctx has a communicator it is one rank of a row-block job: its CSR is
 * the row block [rank*B, rank*B + n_rows), B = ceil(n_global / nranks), and the ops run the
 * exchange of SURVEY §8a row a12: PageRank allgathers its contributions in K row sub-blocks
 * overlapped with the gather; SpMV allgathers y in inl_spmv_allgather; BFS and
 * SSSP use the fused peer-memory exchange of SURVEY §8f NEXT-1 — discovered vertices set bits
 * in their owners' next-frontier bitmaps, improved distances are atomicMin'd into their owners'
 * arrays, over NVLink peer memory mapped with CUDA IPC (handles exchanged through NCCL), one
 * barrier / one 4-byte allreduce per round — or, with the environment variables
 * INL_BFS_EXCHANGE=bytemap / INL_SSSP_EXCHANGE=dense, an n-byte allreduce-max / a 4n-byte
 * allreduce-min per round.  While waiting, NCCL ranks poll ncclCommGetAsyncError: a failed peer
 * or a collective stuck for INL_NCCL_TIMEOUT_S seconds (default 600) aborts the communicator
 * and the call returns INL_ERR_NCCL.  nranks = 1 is allowed (the same code path). */
inl_status inl_nccl_unique_id(uint8_t out[128]);
inl_status inl_comm_init(inl_ctx ctx, const uint8_t uid[128], int32_t nranks, int32_t rank);

/* Loopback communicator (tests and single-GPU studies of the multi-GPU path): P row-block
 * contexts on ONE device exchange through the same calls as NCCL ranks, with device copies
 * and a reduction kernel.  inl_loop_create makes a host object for nranks ranks; each rank's
 * ctx (its own stream) joins it with inl_comm_init_loopback, and each rank must be driven by
 * its own host thread, every rank calling the same ops in the same order (the NCCL rule):
 * collectives block their host thread until all ranks reach them.  A rank whose call fails
 * aborts the group, so its peers fail with INL_ERR_NCCL instead of hanging (also after a
 * 300 s barrier timeout).  The group lives until it is destroyed AND every member ctx is. */
typedef struct inl_loop_s *inl_loop;
inl_status inl_loop_create(int32_t nranks, inl_loop *out);  /* nranks in [1, 64] */
inl_status inl_loop_destroy(inl_loop group);
inl_status inl_comm_init_loopback(inl_ctx ctx, inl_loop group, int32_t rank);

/* Degree binning, built once and reused across calls on the
 * same CSR (device pointers only).  bins may be NULL (defaults). */
inl_status inl_plan_create(inl_ctx ctx, const inl_csr *A, const inl_bins *bins, inl_plan *out);
inl_status inl_plan_get_info(inl_plan plan, inl_plan_info *info);
inl_status inl_plan_destroy(inl_plan plan);

/* O(nnz) device check of the CSR invariants (never on the hot path). */
inl_status inl_csr_validate(inl_ctx ctx, const inl_csr *A);

/* SpMV (P5@10072, P5@10497): y[i] = sum_{k in row i} val[k] * x[col_idx[k]] for the
 * n_rows local rows; x has n_global entries.  fp32 in, fp32 accumulate, fp32 out.
 * Deterministic: bit-identical run to run for the same CSR, bins and partition.  Across
 * row-block partitions a row's fp32 summation order can differ (lane groups are aligned to
 * the local work item), so y agrees within fp32 rounding, and bit-exactly when every partial
 * sum is exactly representable (integer-valued data; reading R11).  plan: NULL =
 * transient bins built inside the call (cost included), else a plan created from this
 * same inl_csr. */
inl_status inl_spmv(inl_ctx ctx, const inl_csr *A, const float *val, const float *x, float *y,
                    inl_plan plan);

/* SpMV with a replicated result (the form an iterated SpMV needs): every rank
 * computes y for its row block (same kernels as inl_spmv) and the blocks are allgathered, so
 * y_global [n_global] = A * x on every rank.  A must be this rank's block of
 * inl_partition_rows (the whole CSR without a communicator).  Asynchronous on the ctx stream
 * for device pointers. */
inl_status inl_spmv_allgather(inl_ctx ctx, const inl_csr *A, const float *val, const float *x,
                              float *y_global, inl_plan plan);

/* PageRank (P5@9262, P5@9781; reading R1): A_in = in-edge CSR (rows =
 * destinations, cols = sources), out_degree [n_global].  PR^0 = 1/n;
 * PR^{t+1}(v) = (1-d)/n + d*(sum_{u->v} PR^t(u)/outdeg(u) + D^t/n), D^t = rank of
 * dangling pages.  rank [n_global] fp32 (replicated on every rank).  damping in
 * [0,1), iterations >= 0. */
inl_status inl_pagerank(inl_ctx ctx, const inl_csr *A_in, const int32_t *out_degree, float damping,
                        int32_t iterations, float *rank, inl_plan plan);

/* SSSP (P5@10241, P11@2218): frontier Bellman-Ford relaxation (atomicMin) until no distance
 * changes (one GPU: near-far scheduled with bitmap frontiers, the step loop as one CUDA-graph
 * launch).  w [nnz]
 * uint32 >= 1, dist [n_global] uint32 with UINT32_MAX = unreachable (replicated).  Distances
 * must stay < 2^32 - 2^8.  Blocks until converged. */
inl_status inl_sssp(inl_ctx ctx, const inl_csr *G, const uint32_t *w, int64_t source,
                    uint32_t *dist, inl_stats *stats, inl_plan plan);

/* BFS (P5@11591): level-synchronous frontier expansion (one GPU: direction-optimizing when the
 * plan found the graph symmetric, bottom-up levels over degree-binned worklists of the unvisited
 * vertices — the first bottom-up level reads the plan's static degree bins, which a symmetric
 * plan builds at creation: 8 B per vertex in the plan's memory); level
 * [n_global] int32, -1 = unreachable, level[source] = 0 (replicated).
 * Blocks until converged. */
inl_status inl_bfs(inl_ctx ctx, const inl_csr *G, int64_t source, int32_t *level,
                   inl_stats *stats, inl_plan plan);

/* Betweenness centrality (P5@8318-8911; reading R10 of DESIGN.md): for each of the
 * n_sources vertices in `sources` (a HOST array of global ids), a BFS shortest-path DAG
 * with path counts sigma, then Brandes' backward dependency sweep;
 *   bc[v] = sum_{s in sources} sum_{t != s, v} sigma_st(v) / sigma_st      (fp64)
 * bc [n_global] double (device or host), overwritten.  All vertices as sources = exact
 * BC (ordered pairs; an undirected graph's usual value is half).  One GPU (no row
 * blocks).  Two paths, chosen by a cost model (environment INL_BC_MODE=level|src forces one):
 * level-synchronous (every source through grid-wide level steps, degree-binned, pull steps on
 * a symmetric plan) and source-parallel (one CTA per source, both sweeps inside the CTA, state
 * in shared memory when 20 B x n_global fits; for many sources on small graphs).  A plan whose
 * bins.flags name one of the paper's templates (INL_BINS_TPL_*, lbTHRES = t_thread, CTA =
 * cta_threads) or INL_BINS_THREAD_ONLY runs both sweeps of every level through that template
 * (the template study).  Deterministic for a given path and source list.
 * stats: iterations = forward levels over all sources.  Blocks until done. */
inl_status inl_bc(inl_ctx ctx, const inl_csr *G, const int64_t *sources, int64_t n_sources, double *bc,
                  inl_stats *stats, inl_plan plan);

/* Tree descendants / heights (§II.C Fig. 3, §III.C) of the tree
 * below `root` given as its children CSR T (one GPU, whole CSR; every node reachable from
 * root at most once):
 *   desc[v]   = 1 + sum_{c child of v} desc[c]     (inl_tree_descendants)
 *   height[v] = 1 + max_{c child of v} height[c]    (inl_tree_heights; a leaf has height 1)
 * out [n_global] int64 (device or host), 0 for nodes not reachable from root.
 * method INL_TREE_FLAT: the paper's flat template (Fig. 3(c)): one thread per node walks up
 * parent[] (int32 [n_global], parent[root] = -1; required) with atomicAdd / atomicMax into the
 * ancestors; stats->edges_relaxed = atomics performed (the sum of node depths for descendants).
 * method INL_TREE_LEVELS: the B200 form of the hierarchical template (Fig. 3(e)) without
 * nested launches: nodes grouped by level (top-down BFS + radix sort), one launch per level,
 * deepest first, 8-lane groups pull their node's children; no atomics; parent may be NULL.
 * stats->iterations = levels, launches = kernels of the method.  Blocks until done. */
enum { INL_TREE_FLAT = 0, INL_TREE_LEVELS = 1 };
inl_status inl_tree_descendants(inl_ctx ctx, const inl_csr *T, const int32_t *parent, int64_t root,
                                int32_t method, int64_t *desc, inl_stats *stats);
inl_status inl_tree_heights(inl_ctx ctx, const inl_csr *T, const int32_t *parent, int64_t root,
                            int32_t method, int64_t *height, inl_stats *stats);

/* Kernel timer (measurement only; off by default).  While enabled, every launch of the
 * path's main kernels ("k_gather", "k_gather_thread_only", "k_expand_flat",
 * "k_expand_grid", "k_bfs_bottom_up") is bracketed by CUDA events recorded on the ctx
 * stream — stream-ordered, so the asynchronous SpMV / PageRank calls stay asynchronous.
 * inl_ktimer_enable(ctx, 1) clears the counters; inl_ktimer_read synchronizes the ctx
 * stream and returns, for the named kernel, the number of launches and the summed
 * device duration in ms (0 / 0 if it never ran).  Unknown names are not an error. */
inl_status inl_ktimer_enable(inl_ctx ctx, int32_t enable);
inl_status inl_ktimer_read(inl_ctx ctx, const char *kernel, int64_t *launches, double *total_ms);

#ifdef __cplusplus
}
#endif
#endif
