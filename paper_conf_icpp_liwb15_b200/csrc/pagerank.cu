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

// exchange-space index: block q = v / B holds slots [q*Bc, (q+1)*Bc); -1 for dangling pages
__global__ void k_cidx(const int32_t *__restrict__ od, const int32_t *__restrict__ pos, int64_t n, int64_t B,
                       int64_t Bc, int32_t *__restrict__ cidx) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = v / B;
    cidx[v] = od[v] > 0 ? (int32_t)(q * Bc + (pos[v] - pos[q * B])) : -1;
  }
}

// degree order: key = (rank block q, ~out_degree) so that, after a stable sort, block q's
// pages with out-links come first in descending out-degree (ties by id), dangling last
__global__ void k_deg_keys(const int32_t *__restrict__ od, int64_t n, int64_t B, uint64_t *__restrict__ key,
                           int32_t *__restrict__ ids) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    key[v] = ((uint64_t)(v / B) << 32) | (uint64_t)(~(uint32_t)max(od[v], 0));
    ids[v] = (int32_t)v;
  }
}

// slot of the i-th vertex of the sorted order within its block (blocks are contiguous runs
// of B positions in the sorted order)
__global__ void k_cidx_sorted(const int32_t *__restrict__ od, const int32_t *__restrict__ ids, int64_t n,
                              int64_t B, int64_t Bc, int32_t *__restrict__ cidx) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = ids[i];
    const int64_t q = v / B;
    cidx[v] = od[v] > 0 ? (int32_t)(q * Bc + (i - q * B)) : -1;
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

int grid_for(int64_t n, int sms) {
  int64_t g = (n + 255) / 256;
  if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
  return g < 1 ? 1 : (int)g;
}

}  // namespace

// Compact (exchange-space) numbering of the pages with out-links, the gather columns in
// that space, and the slots per rank block.  Cached in the plan per out_degree array.
// Inside a rank block the slots follow descending out-degree (= how often a page's
// contribution is gathered), so the frequently read contributions share cache lines
// and stay L2-resident; INL_PR_ORDER=vertex keeps vertex order (measurement switch).
static void pr_compact(inl_ctx ctx, inl_plan p, const int32_t *od, int64_t B, int P) {
  if (p->pr_od == od) return;
  cudaStream_t st = ctx->stream;
  const int64_t n = p->n_global;
  int32_t *flags = (int32_t *)ctx->s_e.get(sizeof(int32_t) * (n + 1));
  int32_t *pos = (int32_t *)ctx->s_f.get(sizeof(int32_t) * (n + 1));
  k_nd_flags<<<grid_for(n + 1, ctx->num_sms), 256, 0, st>>>(od, n, flags);
  size_t need = 0;
  INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, flags, pos, n + 1, st));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(ctx->s_tmp.get(need), need, flags, pos, n + 1, st));
  std::vector<int32_t> at(P + 1);
  for (int q = 0; q <= P; ++q) {
    const int64_t v = std::min<int64_t>((int64_t)q * B, n);
    INL_CUDA(cudaMemcpyAsync(&at[q], pos + v, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
  }
  INL_CUDA(cudaStreamSynchronize(st));
  int64_t bc = 1;
  for (int q = 0; q < P; ++q) bc = std::max<int64_t>(bc, (int64_t)at[q + 1] - at[q]);
  p->pr_bc = bc;
  int32_t *cidx = (int32_t *)p->pr_cidx.get(sizeof(int32_t) * (n > 0 ? n : 1));
  static int vorder = -1;
  if (vorder < 0) {
    const char *e = getenv("INL_PR_ORDER");
    vorder = e && std::string(e) == "vertex";
  }
  if (vorder || n <= 1) {
    k_cidx<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(od, pos, n, B, bc, cidx);
  } else {
    uint64_t *k0 = (uint64_t *)ctx->s_a.get(sizeof(uint64_t) * n);
    uint64_t *k1 = (uint64_t *)ctx->s_b.get(sizeof(uint64_t) * n);
    int32_t *i0 = flags, *i1 = pos;  // the scan results are no longer needed
    k_deg_keys<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(od, n, B, k0, i0);
    int end_bit = 32;
    while (end_bit < 64 && ((uint64_t)(P - 1) >> (end_bit - 32))) ++end_bit;
    cub::DoubleBuffer<uint64_t> kb(k0, k1);
    cub::DoubleBuffer<int32_t> vb(i0, i1);
    size_t sneed = 0;
    INL_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, sneed, kb, vb, n, 0, end_bit, st));
    INL_CUDA(cub::DeviceRadixSort::SortPairs(ctx->s_tmp.get(sneed), sneed, kb, vb, n, 0, end_bit, st));
    k_cidx_sorted<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(od, vb.Current(), n, B, bc, cidx);
  }
  const int32_t zero_slot = (int32_t)(bc * P);
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
    cb_build(p, p->pr_cb, rc, bc * P + 1, /*sort_rows=*/!vorder);
  }
  p->pr_od = od;
}

void pagerank_run(inl_ctx ctx, inl_plan p, const int32_t *out_degree, float damping, int iters,
                  float *rank) {
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
  pr_compact(ctx, p, out_degree, B, DIST ? P : 1);
  const int64_t Bc = p->pr_bc;                    // compact slots per block (exchange count)
  const int64_t ncomp = Bc * (DIST ? P : 1) + 1;  // + the zero slot
  float *c_cur = (float *)ctx->s_a.get(sizeof(float) * ncomp);
  float *c_next = (float *)ctx->s_b.get(sizeof(float) * ncomp);
  INL_CUDA(cudaMemsetAsync(c_cur, 0, sizeof(float) * ncomp, st));
  INL_CUDA(cudaMemsetAsync(c_next, 0, sizeof(float) * ncomp, st));
  const int32_t *cidx = (const int32_t *)p->pr_cidx.p;
  char *scal = (char *)ctx->s_c.get(256 + sizeof(double) * (P + 1));
  float *base = (float *)scal;
  unsigned long long *ndang = (unsigned long long *)(scal + 8);
  double *dloc = (double *)(scal + 16);
  double *dall = (double *)(scal + 256);
  float *rank_pad = nullptr;
  if (DIST) rank_pad = (float *)ctx->s_d.get(sizeof(float) * npad);

  INL_CUDA(cudaMemsetAsync(ndang, 0, sizeof(unsigned long long), st));
  k_pr_init<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(out_degree, cidx, n, c_cur, ndang);
  k_pr_base0<<<1, 1, 0, st>>>(ndang, n, (double)damping, base);
  INL_CUDA(cudaGetLastError());

  const int64_t m = gather_dpart_count(p, &p->pr_cb);
  double *dpart = (double *)p->dpart.p;
  for (int t = 0; t < iters; ++t) {
    const bool last = t + 1 == iters;
    GatherArgs a{p->row_ptr, p->col_idx, nullptr, c_cur, p->nnz, p->n_rows,
                 p->bins.t_thread, p->bins.t_warp, p->bins.t_block, p->bins.grid_chunk, false};
    PrEpi epi{out_degree, c_next, cidx, last ? (DIST ? rank_pad : rank) : nullptr, base, damping,
              p->row_begin, 0.0f};
    launch_gather<false>(ctx, p, a, epi, dpart, (const int32_t *)p->pr_col.p,
                         p->pr_nhot > 0 ? (const int32_t *)p->pr_hot.p : nullptr, &p->pr_cb, p->pr_nhot);
    if (!last) {
      k_pr_dsum<<<1, 1024, 0, st>>>(dpart, m, DIST ? dloc : dall);
      INL_CUDA(cudaGetLastError());
      if (DIST) {
        comm_allgather(ctx, c_next + (int64_t)ctx->rank * Bc, c_next, Bc, ncclFloat32, dloc, dall);
      }
      k_pr_base<<<1, 1, 0, st>>>(dall, P, n, (double)damping, base);
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
