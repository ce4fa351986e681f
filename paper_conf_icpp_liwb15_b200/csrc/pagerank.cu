// pagerank.cu — PageRank pull iterations (PAPER.md P5@9262, P5@9781; reading R1)
// on the binned gather.  One iteration = one fused gather launch (tiles + long
// rows; epilogue computes PR', the next contribution and the dangling partials)
// + one single-CTA fixed-order reduction of the dangling partials.  On P > 1
// ranks the contribution slice and the rank's dangling sum are allgathered.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <cstdlib>
#include <string>
#include <vector>

#include "comm.h"
#include "gather.cuh"

namespace inl {

namespace {

// c[cidx(v)] = PR^0(v) / outdeg(v) with PR^0 = 1/n; dangling count for D^0.
__global__ void k_pr_init(const int32_t *__restrict__ od, const int32_t *__restrict__ cidx, int64_t n,
                          float *__restrict__ c, unsigned long long *__restrict__ n_dangling) {
  const float pr0 = (float)(1.0 / (double)n);
  unsigned long long cnt = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int d = od[v];
    if (d > 0) c[cidx[v]] = pr0 / (float)d;
    cnt += d == 0;
  }
  for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(n_dangling, cnt);
}

__global__ void k_pr_base0(const unsigned long long *__restrict__ n_dangling, int64_t n, double d,
                           float *__restrict__ base) {
  const double D = (double)*n_dangling * (1.0 / (double)n);  // sum of PR^0 over dangling pages
  *base = (float)((1.0 - d) / (double)n + d * D / (double)n);
}

// Fixed-order sum of the dangling partials of this rank -> dloc.
__global__ void __launch_bounds__(1024) k_pr_dsum(const double *__restrict__ dpart, int64_t m,
                                                  double *__restrict__ dloc) {
  __shared__ double red[32];
  double s = 0.0;
  for (int64_t i = threadIdx.x; i < m; i += 1024) s += dpart[i];
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int i = 0; i < 32; ++i) t += red[i];
    *dloc = t;
  }
}

// Stage 1 of the fixed-order dangling sum for large m: CTA b sums the b-th contiguous chunk of
// the partials (the same tree as k_pr_dsum) into part[b]; k_pr_dsum then adds the part[] in
// order.  Deterministic for a given m and grid; one CTA alone took 43 us at scale 25.
__global__ void __launch_bounds__(1024) k_pr_dsum_part(const double *__restrict__ dpart, int64_t m,
                                                       double *__restrict__ part) {
  __shared__ double red[32];
  const int64_t per = (m + gridDim.x - 1) / gridDim.x;
  const int64_t lo = blockIdx.x * per, hi = min(m, lo + per);
  double s = 0.0;
  for (int64_t i = lo + threadIdx.x; i < hi; i += 1024) s += dpart[i];
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int i = 0; i < 32; ++i) t += red[i];
    part[blockIdx.x] = t;
  }
}

// D = sum over ranks in rank order; base = (1-d)/n + d*D/n.
__global__ void k_pr_base(const double *__restrict__ dall, int nranks, int64_t n, double d,
                          float *__restrict__ base) {
  double D = 0.0;
  for (int r = 0; r < nranks; ++r) D += dall[r];
  *base = (float)((1.0 - d) / (double)n + d * D / (double)n);
}

__global__ void k_fill(float *__restrict__ a, int64_t n, float v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    a[i] = v;
}

// ---- compaction of the contribution space to pages with out-links ----
__global__ void k_nd_flags(const int32_t *__restrict__ od, int64_t n, int32_t *__restrict__ f) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n;
       v += (int64_t)gridDim.x * blockDim.x)
    f[v] = v < n && od[v] > 0;
}

// Exchange-space layout (DESIGN.md §5 "PageRank exchange"): rank block q = v / B is cut into
// K row sub-blocks of Bs rows; group (q, k) holds its pages with out-links in slots
//   k * (P * Bck) + q * Bck + i,   i < Bck,
// so sub-block k of every rank is one contiguous, rank-major range: its allgather is NCCL's
// in-place layout and can start as soon as sub-block k's gather is done.  K = 1 is the plain
// rank-major layout q * Bck + i.
struct GroupMap {
  int64_t B, Bs, Bck;
  int P;
  __device__ __forceinline__ int64_t q_of(int64_t v) const { return v / B; }
  __device__ __forceinline__ int64_t k_of(int64_t v, int64_t q) const { return (v - q * B) / Bs; }
  __device__ __forceinline__ int64_t start(int64_t q, int64_t k) const { return q * B + k * Bs; }
  __device__ __forceinline__ int64_t slot(int64_t q, int64_t k, int64_t i) const {
    return k * ((int64_t)P * Bck) + q * Bck + i;
  }
};

// vertex order inside a group: i = rank among the group's pages with out-links
__global__ void k_cidx(const int32_t *__restrict__ od, const int32_t *__restrict__ pos, int64_t n, GroupMap gm,
                       int32_t *__restrict__ cidx) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = gm.q_of(v), k = gm.k_of(v, q);
    cidx[v] = od[v] > 0 ? (int32_t)gm.slot(q, k, pos[v] - pos[gm.start(q, k)]) : -1;
  }
}

// degree order: key = (group, ~out_degree) so that, after a stable sort, group g's pages with
// out-links come first in descending out-degree (ties by id), dangling last
__global__ void k_deg_keys(const int32_t *__restrict__ od, int64_t n, GroupMap gm, int K,
                           uint64_t *__restrict__ key, int32_t *__restrict__ ids) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = gm.q_of(v), g = q * K + gm.k_of(v, q);
    key[v] = ((uint64_t)g << 32) | (uint64_t)(~(uint32_t)max(od[v], 0));
    ids[v] = (int32_t)v;
  }
}

// slot of the i-th vertex of the sorted order within its group (groups are contiguous runs of
// vertex ids, so group (q, k) occupies sorted positions [start(q, k), ...))
__global__ void k_cidx_sorted(const int32_t *__restrict__ od, const int32_t *__restrict__ ids, int64_t n,
                              GroupMap gm, int32_t *__restrict__ cidx) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = ids[i];
    const int64_t q = gm.q_of(v), k = gm.k_of(v, q);
    cidx[v] = od[v] > 0 ? (int32_t)gm.slot(q, k, i - gm.start(q, k)) : -1;
  }
}

// gather columns in the compact space (hot slots kept); a column without out-links
// (inconsistent input) reads the zero slot
__global__ void k_remap_cols(const int32_t *__restrict__ col, int64_t nnz, const int32_t *__restrict__ cidx,
                             int32_t zero_slot, int32_t *__restrict__ out, const int32_t *__restrict__ hot_cols = nullptr,
                             int n_hot = 0) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
       k += (int64_t)gridDim.x * blockDim.x) {
    int32_t c = col[k];
    if (c < 0 && (c & 0x7FFFFFFF) >= n_hot) c = hot_cols[c & 0x7FFFFFFF];  // beyond PageRank's hot set
    if (c < 0) {
      out[k] = c;
    } else {
      const int32_t m = cidx[c];
      out[k] = m >= 0 ? m : zero_slot;
    }
  }
}

__global__ void k_remap_hot(const int32_t *__restrict__ hot, int n_hot, const int32_t *__restrict__ cidx,
                            int32_t zero_slot, int32_t *__restrict__ out) {
  for (int h = blockIdx.x * blockDim.x + threadIdx.x; h < n_hot; h += gridDim.x * blockDim.x) {
    const int32_t m = cidx[hot[h]];
    out[h] = m >= 0 ? m : zero_slot;
  }
}

// Template-study PageRank (the paper's Fig. 6 / Table II PageRank rows): contributions in vertex
// space; c[v] = PR^0/outdeg for v with out-links, 0 otherwise; dangling count for D^0.
__global__ void k_pr_init_v(const int32_t *__restrict__ od, int64_t n, float *__restrict__ c,
                            unsigned long long *__restrict__ n_dangling) {
  const float pr0 = (float)(1.0 / (double)n);
  unsigned long long cnt = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const int d = od[v];
    c[v] = d > 0 ? pr0 / (float)d : 0.0f;
    cnt += d == 0;
  }
  for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(n_dangling, cnt);
}

// PR'(v) = base + d * s(v); the next contribution in place of c (the gather that read c is
// done); the rank on the last step; one fixed-order fp64 dangling partial per CTA
__global__ void __launch_bounds__(256) k_pr_apply_v(const float *__restrict__ s, const int32_t *__restrict__ od,
                                                    const float *__restrict__ base_p, float damping, int64_t n,
                                                    float *__restrict__ c, float *__restrict__ rank_out,
                                                    double *__restrict__ dpart) {
  __shared__ double red[8];
  const float base = *base_p;
  double dsum = 0.0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const float pr = fmaf(damping, s[v], base);
    const int d = od[v];
    c[v] = d > 0 ? pr / (float)d : 0.0f;
    if (rank_out) rank_out[v] = pr;
    if (d == 0) dsum += (double)pr;
  }
  for (int o = 16; o > 0; o >>= 1) dsum += __shfl_xor_sync(0xffffffffu, dsum, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = dsum;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int q = 0; q < 8; ++q) t += red[q];
    dpart[blockIdx.x] = t;
  }
}

int grid_for(int64_t n, int sms) {
  int64_t g = (n + 255) / 256;
  if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
  return g < 1 ? 1 : (int)g;
}

}  // namespace

// Compact (exchange-space) numbering of the pages with out-links, the gather columns in
// that space, and the slots per (rank block, sub-block) group.  Cached in the plan per
// (out_degree array, P, K).  Inside a group the slots follow descending out-degree (= how
// often a page's contribution is gathered), so the frequently read contributions share cache
// lines and stay L2-resident; INL_PR_ORDER=vertex keeps vertex order (measurement switch).
static void pr_compact(inl_ctx ctx, inl_plan p, const int32_t *od, int64_t B, int P, int K) {
  if (p->pr_od == od && p->pr_P == P && p->pr_K == K) return;
  cudaStream_t st = ctx->stream;
  const int64_t n = p->n_global;
  // sub-block width: a multiple of kTileRows, so that no row tile of the plan straddles two
  const int64_t Bs = K > 1 ? ((B + K - 1) / K + kTileRows - 1) / kTileRows * kTileRows : std::max<int64_t>(B, 1);
  int32_t *flags = (int32_t *)ctx->s_e.get(sizeof(int32_t) * (n + 1));
  int32_t *pos = (int32_t *)ctx->s_f.get(sizeof(int32_t) * (n + 1));
  k_nd_flags<<<grid_for(n + 1, ctx->num_sms), 256, 0, st>>>(od, n, flags);
  size_t need = 0;
  INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, flags, pos, n + 1, st));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(ctx->s_tmp.get(need), need, flags, pos, n + 1, st));
  // pages with out-links per group = pos[group end] - pos[group start]
  std::vector<int64_t> gb;  // group boundaries (vertex ids), 2 per group
  for (int q = 0; q < P; ++q)
    for (int k = 0; k < K; ++k) {
      const int64_t hi_q = std::min<int64_t>((int64_t)(q + 1) * B, n);
      const int64_t lo = std::min<int64_t>((int64_t)q * B + k * Bs, hi_q);
      const int64_t hi = std::min<int64_t>((int64_t)q * B + (int64_t)(k + 1) * Bs, hi_q);
      gb.push_back(lo);
      gb.push_back(hi);
    }
  std::vector<int32_t> at(gb.size());
  for (size_t i = 0; i < gb.size(); ++i)
    INL_CUDA(cudaMemcpyAsync(&at[i], pos + gb[i], sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  ctx_sync(ctx);
  int64_t bck = 1;
  for (size_t i = 0; i < gb.size(); i += 2) bck = std::max<int64_t>(bck, (int64_t)at[i + 1] - at[i]);
  p->pr_bc = bck;
  p->pr_Bs = Bs;
  const GroupMap gm{B, Bs, bck, P};
  int32_t *cidx = (int32_t *)p->pr_cidx.get(sizeof(int32_t) * (n > 0 ? n : 1));
  static int vorder = -1;
  if (vorder < 0) {
    const char *e = getenv("INL_PR_ORDER");
    vorder = e && std::string(e) == "vertex";
  }
  if (vorder || n <= 1) {
    k_cidx<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(od, pos, n, gm, cidx);
  } else {
    uint64_t *k0 = (uint64_t *)ctx->s_a.get(sizeof(uint64_t) * n);
    uint64_t *k1 = (uint64_t *)ctx->s_b.get(sizeof(uint64_t) * n);
    int32_t *i0 = flags, *i1 = pos;  // the scan results are no longer needed
    k_deg_keys<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(od, n, gm, K, k0, i0);
    int end_bit = 32;
    while (end_bit < 64 && ((uint64_t)(P * K - 1) >> (end_bit - 32))) ++end_bit;
    cub::DoubleBuffer<uint64_t> kb(k0, k1);
    cub::DoubleBuffer<int32_t> vb(i0, i1);
    size_t sneed = 0;
    INL_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, sneed, kb, vb, n, 0, end_bit, st));
    INL_CUDA(cub::DeviceRadixSort::SortPairs(ctx->s_tmp.get(sneed), sneed, kb, vb, n, 0, end_bit, st));
    k_cidx_sorted<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(od, vb.Current(), n, gm, cidx);
  }
  const int32_t zero_slot = (int32_t)(bck * P * K);
  const int32_t *src = p->n_hot > 0 ? (const int32_t *)p->pcol.p : p->col_idx;
  int32_t *pc = (int32_t *)p->pr_col.get(sizeof(int32_t) * (p->nnz > 0 ? p->nnz : 1));
  // PageRank's own hot set: the first pr_nhot slots of the plan's (ranked by frequency);
  // fewer than SpMV's because the contribution gathers miss L2 more often and profit from
  // the L1 capacity a smaller shared-memory copy leaves (measured, profiles/r01)
  int64_t nh = 16384;
  if (const char *e = getenv("INL_PR_HOT_K")) nh = atoll(e);
  if (nh > p->n_hot) nh = p->n_hot;
  if (nh < 0) nh = 0;
  p->pr_nhot = nh & ~(int64_t)3;
  if (p->n_hot > 0 && p->pr_nhot < 4) p->pr_nhot = 0;
  if (p->nnz > 0)
    k_remap_cols<<<grid_for(p->nnz, ctx->num_sms), 256, 0, st>>>(src, p->nnz, cidx, zero_slot, pc,
                                                                 (const int32_t *)p->hot_cols.p, (int)p->pr_nhot);
  if (p->pr_nhot > 0) {
    int32_t *ph = (int32_t *)p->pr_hot.get(sizeof(int32_t) * p->pr_nhot);
    k_remap_hot<<<grid_for(p->pr_nhot, ctx->num_sms), 256, 0, st>>>((const int32_t *)p->hot_cols.p, (int)p->pr_nhot,
                                                                 cidx, zero_slot, ph);
  }
  INL_CUDA(cudaGetLastError());
  {  // column-blocked bin in the compact space (raw compact columns, no hot tags)
    DevBuf raw;
    int32_t *rc = (int32_t *)raw.get(sizeof(int32_t) * (p->nnz > 0 ? p->nnz : 1));
    if (p->nnz > 0)
      k_remap_cols<<<grid_for(p->nnz, ctx->num_sms), 256, 0, st>>>(p->col_idx, p->nnz, cidx, zero_slot, rc);
    INL_CUDA(cudaGetLastError());
    cb_build(p, p->pr_cb, rc, bck * P * K + 1, /*sort_rows=*/!vorder);
  }
  // the gather's work items grouped by sub-block (stable: longest-first inside each), so that
  // sub-block k is one launch over items [pr_iofs[k], pr_iofs[k+1])
  p->pr_iofs.assign(K + 1, 0);
  p->pr_iofs[K] = p->n_items;
  if (K > 1 && p->n_items > 0) {
    std::vector<WorkItem> h(p->n_items), o;
    INL_CUDA(cudaMemcpyAsync(h.data(), p->items.p, sizeof(WorkItem) * h.size(), cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    o.reserve(h.size());
    for (int k = 0; k < K; ++k) {
      p->pr_iofs[k] = (int64_t)o.size();
      for (const WorkItem &w : h)
        if (std::min<int64_t>(w.r0 / Bs, K - 1) == k) o.push_back(w);
    }
    INL_CHECK(o.size() == h.size(), "pagerank: sub-block item split lost items");
    WorkItem *d = (WorkItem *)p->pr_items.get(sizeof(WorkItem) * o.size());
    INL_CUDA(cudaMemcpyAsync(d, o.data(), sizeof(WorkItem) * o.size(), cudaMemcpyHostToDevice, st));
    ctx_sync(ctx);
  }
  p->pr_od = od;
  p->pr_P = P;
  p->pr_K = K;
}

// Row sub-blocks per rank for the pipelined exchange (P > 1): env INL_PR_SUBBLOCKS, default 4;
// 1 = one allgather after the whole gather.
static int pr_subblocks() {
  int k = 4;
  if (const char *e = getenv("INL_PR_SUBBLOCKS")) k = atoi(e);
  return k < 1 ? 1 : k > 16 ? 16 : k;
}

// PageRank through the paper's templates (INL_BINS_TPL_*) or its thread-mapped baseline T1
// (INL_BINS_THREAD_ONLY), one GPU, for the template study: per
// iteration the template SpMV with implicit unit values gathers s(v) = sum of c(u) over the
// in-CSR, then k_pr_apply_v forms PR', the next contributions and the dangling partials.
static void pagerank_template(inl_ctx ctx, inl_plan p, const int32_t *od, float damping, int iters, float *rank) {
  cudaStream_t st = ctx->stream;
  const int64_t n = p->n_global;
  inl_csr A{p->n_rows, p->n_global, p->row_begin, p->nnz, p->row_ptr, p->col_idx};
  // not s_a / s_b / s_f: spmv_template's queues and counters live there
  float *c = (float *)ctx->s_d.get(sizeof(float) * (size_t)n);
  float *s = (float *)ctx->s_e.get(sizeof(float) * (size_t)n);
  const int grid = grid_for(n, ctx->num_sms);
  char *scal = (char *)ctx->s_g.get(256 + sizeof(double) * (size_t)grid);
  float *base = (float *)scal;
  unsigned long long *ndang = (unsigned long long *)(scal + 8);
  double *dall = (double *)(scal + 16);
  double *dpart = (double *)(scal + 256);
  INL_CUDA(cudaMemsetAsync(ndang, 0, sizeof(unsigned long long), st));
  k_pr_init_v<<<grid, 256, 0, st>>>(od, n, c, ndang);
  k_pr_base0<<<1, 1, 0, st>>>(ndang, n, (double)damping, base);
  INL_CUDA(cudaGetLastError());
  for (int t = 0; t < iters; ++t) {
    const bool last = t + 1 == iters;
    if (p->bins.flags & INL_BINS_THREAD_ONLY) spmv_thread_only(ctx, A, nullptr, c, s);  // the T1 baseline
    else spmv_template(ctx, A, p->bins, nullptr, c, s);
    k_pr_apply_v<<<grid, 256, 0, st>>>(s, od, base, damping, n, c, last ? rank : nullptr, dpart);
    if (!last) {
      k_pr_dsum<<<1, 1024, 0, st>>>(dpart, grid, dall);
      k_pr_base<<<1, 1, 0, st>>>(dall, 1, n, (double)damping, base);
    }
    INL_CUDA(cudaGetLastError());
  }
}

void pagerank_run(inl_ctx ctx, inl_plan p, const int32_t *out_degree, float damping, int iters,
                  float *rank) {
  if (p->bins.flags & (kTemplateFlags | INL_BINS_THREAD_ONLY)) {
    INL_CHECK(!has_comm(ctx), "pagerank: the paper's templates / T1 run on one GPU (no communicator)");
    if (p->n_global == 0) return;
    if (iters == 0) {
      k_fill<<<grid_for(p->n_global, ctx->num_sms), 256, 0, ctx->stream>>>(rank, p->n_global,
                                                                           (float)(1.0 / (double)p->n_global));
      INL_CUDA(cudaGetLastError());
      return;
    }
    pagerank_template(ctx, p, out_degree, damping, iters, rank);
    return;
  }
  cudaStream_t st = ctx->stream;
  const int64_t n = p->n_global;
  if (n == 0) return;
  if (iters == 0) {
    k_fill<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(rank, n, (float)(1.0 / (double)n));
    INL_CUDA(cudaGetLastError());
    return;
  }
  const int P = ctx->nranks;
  const bool DIST = has_comm(ctx);  // row-block mode with an exchange (NCCL or loopback; also P = 1)
  const int64_t B = DIST ? (n + P - 1) / P : n;  // row block (inl_partition_rows)
  const int64_t npad = B * P;
  // pipelined exchange: sub-block k's allgather (on the comm stream) overlaps the gathers of
  // sub-blocks k+1.. (the column-blocked opt-in keeps one launch per iteration)
  int K = DIST && P > 1 ? pr_subblocks() : 1;
  if (p->bins.flags & INL_BINS_COLBLOCK) K = 1;
  pr_compact(ctx, p, out_degree, B, DIST ? P : 1, K);
  if (p->pr_cb.active) K = 1;
  const int64_t Bc = p->pr_bc;                        // slots per (rank, sub-block) group
  const int64_t span = Bc * (DIST ? P : 1);           // slots per sub-block (all ranks)
  const int64_t ncomp = span * p->pr_K + 1;           // + the zero slot
  float *c_cur = (float *)ctx->s_a.get(sizeof(float) * ncomp);
  float *c_next = (float *)ctx->s_b.get(sizeof(float) * ncomp);
  INL_CUDA(cudaMemsetAsync(c_cur, 0, sizeof(float) * ncomp, st));
  INL_CUDA(cudaMemsetAsync(c_next, 0, sizeof(float) * ncomp, st));
  const int32_t *cidx = (const int32_t *)p->pr_cidx.p;
  constexpr int kDsumParts = 1024;  // stage-1 partials of the dangling sum (<= num_sms CTAs)
  char *scal = (char *)ctx->s_c.get(256 + sizeof(double) * (P + 1 + kDsumParts));
  float *base = (float *)scal;
  unsigned long long *ndang = (unsigned long long *)(scal + 8);
  double *dloc = (double *)(scal + 16);
  double *dall = (double *)(scal + 256);
  double *dparts = dall + P + 1;
  // fixed-order dangling sum of m partials: one CTA for small m, else stage 1 over G CTAs first
  auto dsum = [&](const double *src, int64_t cnt, double *out) {
    const int G = (int)std::min<int64_t>(std::min(ctx->num_sms, kDsumParts), cnt / 8192);
    if (G > 1) {
      k_pr_dsum_part<<<G, 1024, 0, st>>>(src, cnt, dparts);
      k_pr_dsum<<<1, 1024, 0, st>>>(dparts, G, out);
    } else {
      k_pr_dsum<<<1, 1024, 0, st>>>(src, cnt, out);
    }
  };
  float *rank_pad = nullptr;
  if (DIST) rank_pad = (float *)ctx->s_d.get(sizeof(float) * npad);

  INL_CUDA(cudaMemsetAsync(ndang, 0, sizeof(unsigned long long), st));
  k_pr_init<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(out_degree, cidx, n, c_cur, ndang);
  k_pr_base0<<<1, 1, 0, st>>>(ndang, n, (double)damping, base);
  INL_CUDA(cudaGetLastError());

  const int64_t m = gather_dpart_count(p, &p->pr_cb);
  double *dpart = (double *)p->dpart.p;
  const int32_t *pr_hot = p->pr_nhot > 0 ? (const int32_t *)p->pr_hot.p : nullptr;
  cudaStream_t cs = K > 1 ? comm_stream(ctx) : st;
  // leave SMs to NCCL's kernels while they overlap the gather (the loopback copies use the
  // copy engines instead)
  const int max_ctas = K > 1 && ctx->comm ? ctx->num_sms - 16 : 0;
  for (int t = 0; t < iters; ++t) {
    const bool last = t + 1 == iters;
    GatherArgs a{p->row_ptr, p->col_idx, nullptr, c_cur, p->nnz, p->n_rows,
                 p->bins.t_thread, p->bins.t_warp, p->bins.t_block, p->bins.grid_chunk, false};
    PrEpi epi{out_degree, c_next, cidx, last ? (DIST ? rank_pad : rank) : nullptr, base, damping,
              p->row_begin, 0.0f};
    if (K == 1) {
      launch_gather<false>(ctx, p, a, epi, dpart, (const int32_t *)p->pr_col.p, pr_hot, &p->pr_cb, p->pr_nhot);
      if (!last) {
        dsum(dpart, m, DIST ? dloc : dall);
        INL_CUDA(cudaGetLastError());
        if (DIST) comm_allgather(ctx, c_next + (int64_t)ctx->rank * Bc, c_next, Bc, ncclFloat32, dloc, dall);
      }
    } else {
      const WorkItem *items = (const WorkItem *)p->pr_items.p;
      for (int k = 0; k < K; ++k) {
        GatherRange rg;
        rg.items = items + p->pr_iofs[k];
        rg.n = p->pr_iofs[k + 1] - p->pr_iofs[k];
        rg.max_ctas = max_ctas;
        rg.skip_xhot = k > 0;  // x_hot (c_cur's hot slots) is copied once per iteration
        if (rg.n > 0)
          launch_gather<false>(ctx, p, a, epi, dpart + p->pr_iofs[k], (const int32_t *)p->pr_col.p, pr_hot, nullptr,
                               p->pr_nhot, &rg);
        if (!last) {  // sub-block k's contributions go out while k+1.. are gathered
          cudaEvent_t ev = ctx_event(ctx, 0);  // a wait captures the record made just before it
          INL_CUDA(cudaEventRecord(ev, st));
          INL_CUDA(cudaStreamWaitEvent(cs, ev, 0));
          float *blk = c_next + (int64_t)k * span;
          comm_allgather(ctx, blk + (int64_t)ctx->rank * Bc, blk, Bc, ncclFloat32, nullptr, nullptr, cs);
        }
      }
      if (!last) {
        dsum(dpart, m, dloc);
        INL_CUDA(cudaGetLastError());
        cudaEvent_t ev = ctx_event(ctx, 1);
        INL_CUDA(cudaEventRecord(ev, st));
        INL_CUDA(cudaStreamWaitEvent(cs, ev, 0));
        comm_allgather(ctx, dloc, dall, 1, ncclFloat64, nullptr, nullptr, cs);
        cudaEvent_t done = ctx_event(ctx, 2);
        INL_CUDA(cudaEventRecord(done, cs));
        INL_CUDA(cudaStreamWaitEvent(st, done, 0));  // the next iteration reads every block
      }
    }
    if (!last) {
      k_pr_base<<<1, 1, 0, st>>>(dall, DIST ? P : 1, n, (double)damping, base);
      INL_CUDA(cudaGetLastError());
      float *tmp = c_cur;
      c_cur = c_next;
      c_next = tmp;
    }
  }
  if (DIST) {
    comm_allgather(ctx, rank_pad + (int64_t)ctx->rank * B, rank_pad, B, ncclFloat32, nullptr, nullptr);
    INL_CUDA(cudaMemcpyAsync(rank, rank_pad, sizeof(float) * n, cudaMemcpyDeviceToDevice, st));
  }
}

}  // namespace inl
