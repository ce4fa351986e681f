// inl_internal.cuh — shared internals of libinl.so (product path; no oracle code).
#pragma once
#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>

#include <string>
#include <cstdlib>
#include <vector>

#include "inl.h"

namespace inl {

constexpr int kTileRows = 256;  // max rows per SpMV/PR warp tile
constexpr int kMaxDevices = 64;  // per-device caches of kernel attributes
constexpr int kCtxEvents = 16;   // events a ctx keeps for cross-stream ordering

// One unit of work of the fused gather kernel (one warp): a tile (j < 0: rows [r0, r1),
// all of degree <= t_warp, nonzeros [s, e), tile index t into the plan's non-empty-row
// masks) or one chunk c of long row r0 (j = long-row index, nonzeros [s, e), nch chunks,
// partial slots from pbase).
struct __align__(16) WorkItem {
  int64_t s, e;
  int32_t r0, r1, j, c, nch, pbase, t, pad1;
};

struct Status {
  inl_status code = INL_OK;
  std::string msg;
};

// Error carried from a failing CUDA/NCCL call up to the C-ABI boundary.
struct Error {
  inl_status code;
  std::string msg;
};

[[noreturn]] void raise(inl_status code, const std::string &msg);

#define INL_CUDA(call)                                                                     \
  do {                                                                                     \
    cudaError_t e_ = (call);                                                               \
    if (e_ != cudaSuccess)                                                                 \
      ::inl::raise(INL_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_) + " (" \
                                     __FILE__ ":" + std::to_string(__LINE__) + ")");       \
  } while (0)

#define INL_NCCL(call)                                                                          \
  do {                                                                                          \
    ncclResult_t r_ = (call);                                                                   \
    if (r_ != ncclSuccess)                                                                      \
      ::inl::raise(INL_ERR_NCCL, std::string(#call) + ": " + ncclGetErrorString(r_) + " (" \
                                     __FILE__ ":" + std::to_string(__LINE__) + ")");            \
  } while (0)

#define INL_CHECK(cond, msg)                                      \
  do {                                                            \
    if (!(cond)) ::inl::raise(INL_ERR_INVALID_ARGUMENT, (msg));   \
  } while (0)

// Growable device scratch buffer owned by a ctx or plan.
struct DevBuf {
  void *p = nullptr;
  size_t bytes = 0;
  void *get(size_t need);  // grows (cudaFree + cudaMalloc) when too small
  void release();
  ~DevBuf() { release(); }
};

struct Bins {
  int t_thread, t_warp, t_block, grid_chunk, cta, flags;
};
Bins resolve_bins(const inl_bins *b);

// One (column block, row) run of a column-blocked row (colblock.cu): entries
// [cs, cs + len) of the CSR, whose columns all lie in one column block; their local
// column offsets are cbcol[cb, cb + len).  j = index of the row in CbPlan::rows.
struct __align__(8) CbPair {
  int64_t cs, cb;
  int32_t len, j;
};

// Column-blocked deferred bin: rows of degree > t_cb are split by column
// block (K consecutive columns = one shared-memory copy of x); a CTA loads one block of x
// and sums every run of that block into a per-run partial; a combine kernel adds each
// row's partials in block order.  Built per column space (SpMV: the CSR's; PageRank: the
// compacted contribution space).
struct CbPlan {
  bool active = false;
  int K = 0;                // column-block width (x slots in shared memory)
  int64_t ncols = 0, nblocks = 0;
  int32_t t_cb = 0;         // rows of degree > t_cb are column-blocked
  int64_t n_rows = 0, n_pairs = 0, n_entries = 0;
  int grid = 0;             // CTAs of k_cb (entry ranges in cta_lo)
  DevBuf rows;              // int32 [n_rows] local row ids
  DevBuf rp_base;           // int64 [n_rows + 1] first run (row order) of each row
  DevBuf pos_of;            // int64 [n_pairs] position of run q (row order) in `pairs`
  DevBuf pairs;             // CbPair [n_pairs] sorted by (block, length desc, row)
  DevBuf blk_first;         // int64 [nblocks + 1] first pair of each block
  DevBuf cta_lo;            // int64 [grid + 1] first pair of each CTA (equal entry shares)
  DevBuf cbcol;             // uint16 [n_entries] column offsets within the block
  DevBuf partials;          // float [n_pairs]
  int64_t n_items = 0;      // gather work items without the column-blocked rows
  DevBuf items;             // WorkItem [n_items]
};

}  // namespace inl

namespace inl {
struct LoopGroup;  // loopback.cu: P row-block contexts on one device standing in for NCCL
// Per-kernel launch timer (inl_ktimer_*): event pairs pending on the ctx stream, resolved
// into (launches, ms) totals when read.
struct KTimer {
  struct Slot {
    std::string name;
    int64_t launches = 0;
    double ms = 0.0;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> pending;
  };
  bool on = false;
  std::vector<Slot> slots;
  std::vector<cudaEvent_t> pool;
  Slot &slot(const char *name);
  cudaEvent_t ev();
  void resolve();  // caller synchronized the stream
  void clear();
  ~KTimer();
};
}  // namespace inl

struct inl_ctx_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  int num_sms = 148;
  std::string last_error;
  ncclComm_t comm = nullptr;
  inl::LoopGroup *loop = nullptr;  // loopback group (inl_comm_init_loopback) instead of NCCL
  cudaStream_t comm_stream = nullptr;  // second stream: exchanges overlapped with the gather
  cudaEvent_t events[inl::kCtxEvents] = {};
  void *sssp_graph = nullptr;  // cached executable graph of the one-GPU SSSP loop (frontier.cu)
  // peer mappings of one exchange buffer (comm_peer_bases): every rank's base pointer, the
  // local buffer they belong to, and the CUDA IPC mappings to close when it changes
  std::vector<void *> peer_bases, ipc_open;
  void *peer_mine = nullptr;
  size_t peer_bytes = 0;
  inl::DevBuf s_xch;   // NEXT-1 exchange buffers (frontier bitmaps peers write into)
  inl::DevBuf s_xtab;  // device tables of peer pointers into s_xch
  inl::DevBuf s_bar;   // NCCL barrier word
  int nranks = 1, rank = 0;
  // scratch
  inl::DevBuf s_tmp, s_a, s_b, s_c, s_d, s_e, s_f, s_g;
  inl::DevBuf h_rp, h_ci, h_val, h_x, h_y, h_w, h_od;  // host-staging device copies
  inl::DevBuf s_loop;                                  // loopback allreduce scratch
  inl::DevBuf s_pad;                                   // padded replicated vectors (P > 1)
  inl::DevBuf s_bu;                                    // BFS bottom-up worklists
  inl::DevBuf s_h;                                     // tree levels (tree.cu)
  inl::DevBuf s_t;                                     // SSSP step trace (INL_SSSP_TRACE, measurement)
  inl::DevBuf s_bcb;                                   // BC next-level bitmap (heavy push levels)
  int64_t *pinned = nullptr;                           // small pinned host scalars
  int live_plans = 0;    // plans created on this ctx and not yet destroyed
  struct inl_plan_s *tplan = nullptr;  // reusable transient plan (plan = NULL calls)
  bool closed = false;   // inl_ctx_destroy called; freed when the last plan goes
  inl::KTimer ktimer;
};

struct inl_plan_s {
  inl_ctx ctx = nullptr;
  // identity of the CSR it was built from
  int64_t n_rows = 0, n_global = 0, row_begin = 0, nnz = 0;
  const int64_t *row_ptr = nullptr;
  const int32_t *col_idx = nullptr;
  inl::Bins bins{};
  // tiles: rows [tile_lo[t], tile_hi[t]) with every row of degree <= t_warp
  int64_t n_tiles = 0;
  inl::DevBuf tiles;  // int2 {lo, hi}
  inl::DevBuf tile_nz;  // uint32 [n_tiles * 8]: bit r of tile t = row lo_t + r is non-empty
  // long rows: degree > t_warp, cut into grid_chunk-sized chunks
  int64_t n_long = 0, n_chunks = 0;
  inl::DevBuf long_rows;    // int32 [n_long]
  inl::DevBuf chunk_items;  // int2 {long index, chunk index} [n_chunks]
  inl::DevBuf chunk_base;   // int32 [n_long] first chunk of each long row
  inl::DevBuf partials;     // float [n_chunks]
  inl::DevBuf tickets;      // int32 [n_long], zero between calls
  inl::DevBuf dpart;        // double [n_items] (PageRank dangling partials, one per item)
  // hot-column remap (plan-time): the n_hot most frequent columns are read from a
  // shared-memory copy of x; pcol is col_idx with hot entries encoded 0x80000000 | h.
  int64_t n_hot = 0;
  inl::DevBuf hot_cols;     // int32 [n_hot] original column of hot slot h
  inl::DevBuf pcol;         // int32 [nnz]
  inl::DevBuf x_hot;        // float [n_hot] per-call copy of x[hot_cols]
  inl::DevBuf rs_bits;      // uint32 [nnz/32 + 1]: bit k = entry k starts a non-empty row
  inl::DevBuf ticket;       // uint64 dynamic-schedule counter of the gather kernel
  unsigned long long ticket_base = 0;  // its value at the start of the next launch
  int64_t n_items = 0;
  inl::DevBuf items;        // WorkItem [n_items]: grid-bin chunks first, then tiles
  inl_plan_info info{};
  bool transient = false;  // built inside a call: no hot-column remap (pcol unused)
  // PageRank: contributions live in the compacted space of non-dangling vertices
  // (every column of an in-CSR is a page with out-links), cached per out_degree array
  const int32_t *pr_od = nullptr;
  int64_t pr_bc = 0;           // compact slots per (rank block, sub-block) group
  int pr_P = 0, pr_K = 0;      // ranks and row sub-blocks the compaction was built for
  int64_t pr_Bs = 0;           // sub-block width in rows (a multiple of kTileRows)
  std::vector<int64_t> pr_iofs;  // [pr_K + 1] first work item of each sub-block in pr_items
  inl::DevBuf pr_items;        // WorkItem [n_items] grouped by sub-block (pr_K > 1)
  inl::DevBuf pr_cidx;         // int32 [n_global]: exchange-space index, -1 if dangling
  inl::DevBuf pr_col;          // int32 [nnz]: gather columns in the compact space (hot kept)
  inl::DevBuf pr_hot;          // int32 [pr_nhot]: hot slots in the compact space
  int64_t pr_nhot = 0;         // PageRank's hot slots (a prefix of the plan's)
  bool symmetric = false;  // every edge's reverse is present (checked at plan time, sorted rows)
  // static bottom-up bins of a symmetric plan (frontier.cu bu_static_build): thread bin
  // [0, bu_ns), warp bin [n_global, n_global + bu_nl) of bu_lists
  inl::DevBuf bu_lists;
  int64_t bu_ns = 0, bu_nl = 0;
  // column-blocked long rows: SpMV (the CSR's column space) and PageRank (compact space)
  inl::CbPlan cb, pr_cb;
};

namespace inl {
// RAII bracket of one kernel launch for the kernel timer (no-op unless enabled).
struct KScope {
  inl_ctx ctx;
  KTimer::Slot *sl = nullptr;
  cudaEvent_t e0 = nullptr;
  KScope(inl_ctx c, const char *name) : ctx(c) {
    if (!c->ktimer.on) return;
    sl = &c->ktimer.slot(name);
    e0 = c->ktimer.ev();
    cudaEventRecord(e0, c->stream);
  }
  ~KScope() {
    if (!sl) return;
    cudaEvent_t e1 = ctx->ktimer.ev();
    cudaEventRecord(e1, ctx->stream);
    sl->pending.emplace_back(e0, e1);
  }
};
// plan.cu
void build_plan(inl_plan p);
// spmv.cu
void spmv_run(inl_ctx ctx, inl_plan p, const float *val, const float *x, float *y);
void spmv_thread_only(inl_ctx ctx, const inl_csr &A, const float *val, const float *x, float *y);
// pagerank.cu
void pagerank_run(inl_ctx ctx, inl_plan p, const int32_t *out_degree, float damping, int iters,
                  float *rank);
// frontier.cu
void sssp_run(inl_ctx ctx, const inl_csr &G, const Bins &b, const uint32_t *w, int64_t source,
              uint32_t *dist, inl_stats *st);
// symmetric: the plan verified that every edge (u, v) has its reverse (v, u), so a vertex's
// row lists its predecessors too (bottom-up / pull steps are valid)
struct BuStatic {  // a plan's static bottom-up bins (s == nullptr: none)
  const int32_t *s = nullptr, *l = nullptr;
  int64_t ns = 0, nl = 0;
};
void bfs_run(inl_ctx ctx, const inl_csr &G, const Bins &b, int64_t source, int32_t *level,
             inl_stats *st, bool symmetric, const BuStatic &bus = BuStatic());
void bu_static_build(inl_plan p);
// templates.cu: the paper's dual-queue / dbuf-global / dbuf-shared SpMV (false: no template flag)
constexpr int kTemplateFlags = INL_BINS_TPL_DUAL_QUEUE | INL_BINS_TPL_DBUF_GLOBAL | INL_BINS_TPL_DBUF_SHARED;
bool spmv_template(inl_ctx ctx, const inl_csr &A, const Bins &b, const float *val, const float *x, float *y);
// colblock.cu: builds `cb` for the column space `cols` (raw ids in [0, ncols), CSR order)
void cb_build(inl_plan p, CbPlan &cb, const int32_t *cols, int64_t ncols, bool sort_rows = false);
// tree.cu: descendants (heights = false) or heights of the tree below `root`
void tree_run(inl_ctx ctx, const inl_csr &T, const int32_t *parent, int64_t root, int method, bool heights,
              int64_t *out, inl_stats *stats);
// bc.cu
void bc_run(inl_ctx ctx, const inl_csr &G, const Bins &b, const int64_t *sources, int64_t n_sources, double *bc,
            inl_stats *stats, bool symmetric);
// validate
void csr_validate(inl_ctx ctx, const inl_csr &A);
// Wait for the ctx stream.  NCCL ranks poll instead (ncclCommGetAsyncError): a failed peer or
// a stuck collective surfaces as INL_ERR_NCCL (communicator aborted) instead of a hang; the
// limit is INL_NCCL_TIMEOUT_S seconds (default 600).  api.cu.
void ctx_sync(inl_ctx ctx);
// NVTX range around a C-ABI call (visible in nsys / ncu timelines; free without a tool)
struct NvtxRange {
  explicit NvtxRange(const char *name);
  ~NvtxRange();
};
void sssp_graph_free(void *g);  // frontier.cu
}  // namespace inl
