// plan.cu — static degree binning (the paper's dual-queue /
// delayed-buffer split by lbTHRES, P5@2078, P5@2721, P11@1197).
//
// Output of the plan for a CSR with n rows:
//  * tiles: contiguous row ranges [lo, hi) whose rows all have degree <= t_warp
//    (thread and warp bins, processed by one warp — dbuf-shared).  A tile starts
//    at every multiple of kTileRows rows, at every row after a long row, and
//    wherever floor(P[i] / kTileSpan) changes, P = exclusive prefix sum of the
//    short-row degrees.  Hence a tile holds <= kTileRows rows and < kTileSpan +
//    t_warp nonzeros.
//  * hot columns: the n_hot most frequent columns get shared-memory slots; pcol
//    is col_idx with their entries encoded 0x80000000 | slot (gather.cuh).
//  * long rows: degree > t_warp (the global deferral buffer — dbuf-global), cut
//    into grid_chunk-sized chunks at row-relative offsets; one warp per chunk
//    (block bin: degree <= t_block, grid bin: above).
// The plan is built on the GPU with CUB scans / selects, once per CSR.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>
#include <thrust/iterator/counting_iterator.h>

#include "gather.cuh"
#include "inl_internal.cuh"

namespace inl {

namespace {

__global__ void k_classify(const int64_t *__restrict__ rp, int64_t n, int t_long,
                           int32_t *__restrict__ short_deg, uint8_t *__restrict__ is_long) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = rp[i + 1] - rp[i];
    const bool lg = d > t_long;
    is_long[i] = lg;
    short_deg[i] = lg ? 0 : (int32_t)d;
  }
}

__global__ void k_boundary(const int64_t *__restrict__ P, const uint8_t *__restrict__ is_long,
                           int64_t n, int stride, uint8_t *__restrict__ flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    bool b = (i % kTileRows) == 0 || is_long[i];
    if (i > 0 && !b) b = is_long[i - 1] || (P[i] / stride) != (P[i - 1] / stride);
    flag[i] = b;
  }
}

__global__ void k_emit_tiles(const int32_t *__restrict__ S, const int64_t *__restrict__ nS,
                             const uint8_t *__restrict__ is_long, int64_t n,
                             int2 *__restrict__ cand, uint8_t *__restrict__ valid) {
  const int64_t K = *nS;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < K;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = S[k];
    const int32_t end = (k + 1 < K) ? S[k + 1] : (int32_t)n;
    cand[k] = make_int2(r, end);
    valid[k] = !is_long[r];
  }
}

__global__ void k_long_chunks(const int64_t *__restrict__ rp, const int32_t *__restrict__ long_rows,
                              int64_t n_long, int chunk, int32_t *__restrict__ nch) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n_long;
       j += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = long_rows[j];
    nch[j] = (int32_t)((rp[r + 1] - rp[r] + chunk - 1) / chunk);
  }
}

__global__ void k_chunk_items(const int32_t *__restrict__ nch, const int32_t *__restrict__ base,
                              int64_t n_long, int2 *__restrict__ items) {
  for (int64_t j = blockIdx.x; j < n_long; j += gridDim.x)
    for (int c = threadIdx.x; c < nch[j]; c += blockDim.x) items[base[j] + c] = make_int2((int)j, c);
}

// Work items of the fused gather: chunks of long rows first (the longest work), then tiles.
__global__ void k_build_items(const int64_t *__restrict__ rp, const int2 *__restrict__ tiles,
                              int64_t n_tiles, const int2 *__restrict__ citems,
                              const int32_t *__restrict__ long_rows, const int32_t *__restrict__ nch,
                              const int32_t *__restrict__ base, int64_t n_chunks, int chunk,
                              WorkItem *__restrict__ out) {
  const int64_t total = n_chunks + n_tiles;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    WorkItem w;
    w.t = w.pad1 = 0;
    if (i < n_chunks) {
      const int2 ci = citems[i];
      const int32_t r = long_rows[ci.x];
      const int64_t rs = rp[r], re = rp[r + 1];
      w.s = rs + (int64_t)ci.y * chunk;
      w.e = min(w.s + (int64_t)chunk, re);
      w.r0 = r;
      w.r1 = r + 1;
      w.j = ci.x;
      w.c = ci.y;
      w.nch = nch[ci.x];
      w.pbase = base[ci.x];
    } else {
      const int2 t = tiles[i - n_chunks];
      w.s = rp[t.x];
      w.e = rp[t.y];
      w.r0 = t.x;
      w.r1 = t.y;
      w.j = -1;
      w.t = (int32_t)(i - n_chunks);
      w.c = 0;
      w.nch = 0;
      w.pbase = 0;
    }
    out[i] = w;
  }
}

// Non-empty-row masks of the tiles (one warp per tile): the gather kernel builds its
// per-tile row lists from them instead of re-reading row_ptr.
__global__ void k_tile_nz(const int64_t *__restrict__ rp, const int2 *__restrict__ tiles, int64_t n_tiles,
                          uint32_t *__restrict__ nz) {
  const int lane = threadIdx.x & 31;
  for (int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; t < n_tiles;
       t += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int2 tl = tiles[t];
    for (int rb = 0; rb < kTileRows; rb += 32) {
      const int r = tl.x + rb + lane;
      const bool ne = r < tl.y && rp[r + 1] > rp[r];
      const unsigned m = __ballot_sync(0xffffffffu, ne);
      if (lane == 0) nz[8 * t + rb / 32] = m;
    }
  }
}

__global__ void k_col_count(const int32_t *__restrict__ col, int64_t nnz, int32_t *__restrict__ cnt) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
       k += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + col[k], 1);
}

__global__ void k_iota(int32_t *__restrict__ a, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    a[i] = (int32_t)i;
}

__global__ void k_hot_rank(const int32_t *__restrict__ sorted_cols, int64_t n_hot,
                           int32_t *__restrict__ hot_rank, int32_t *__restrict__ hot_cols) {
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_hot;
       h += (int64_t)gridDim.x * blockDim.x) {
    hot_rank[sorted_cols[h]] = (int32_t)h;
    hot_cols[h] = sorted_cols[h];
  }
}

__global__ void k_remap(const int32_t *__restrict__ col, int64_t nnz, const int32_t *__restrict__ hot_rank,
                        int32_t *__restrict__ pcol) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = col[k];
    const int32_t h = hot_rank[c];
    pcol[k] = h >= 0 ? (int32_t)(0x80000000u | (uint32_t)h) : c;
  }
}

__global__ void k_rowstart_bits(const int64_t *__restrict__ rp, int64_t n, uint32_t *__restrict__ bits) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n;
       r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = rp[r];
    if (rp[r + 1] > b) atomicOr(bits + (b >> 5), 1u << (b & 31));
  }
}

// Per-bin row / nnz counts (plan info; not on the hot path).
__global__ void k_bin_stats(const int64_t *__restrict__ rp, int64_t n, Bins b,
                            unsigned long long *__restrict__ st) {
  unsigned long long c[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = rp[i + 1] - rp[i];
    const int bin = d <= b.t_thread ? 0 : d <= b.t_warp ? 1 : d <= b.t_block ? 2 : 3;
    c[bin] += 1;
    c[4 + bin] += (unsigned long long)d;
  }
  for (int q = 0; q < 8; ++q) {
    unsigned long long v = c[q];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(st + q, v);
  }
}

// symmetry check: every entry (r, c) of a square CSR has (c, r) — binary search of r in row
// c (rows sorted; an unsorted row just fails the check, which only disables bottom-up)
__global__ void k_check_symmetric(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n,
                                  int *__restrict__ bad) {
  const int lane = threadIdx.x & 31;
  for (int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; r < n;
       r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    bool ok = true;
    for (int64_t k = rp[r] + lane; k < rp[r + 1]; k += 32) {
      const int32_t c = col[k];
      if (c < 0 || c >= n) {
        ok = false;
        break;
      }
      int64_t lo = rp[c], hi = rp[c + 1];
      while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (col[mid] < r) lo = mid + 1;
        else hi = mid;
      }
      if (lo >= rp[c + 1] || col[lo] != r) {
        ok = false;
        break;
      }
    }
    if (__any_sync(0xffffffffu, !ok) && lane == 0) atomicExch(bad, 1);
  }
}

int grid_for(int64_t n, int num_sms) {
  int64_t g = (n + 255) / 256;
  const int64_t cap = (int64_t)num_sms * 16;
  if (g > cap) g = cap;
  return g < 1 ? 1 : (int)g;
}

}  // namespace

// Hot-column remap: rank columns by their number of nonzeros (stable radix sort, so
// ties keep column order and the plan is deterministic) and give the top n_hot a
// shared-memory slot.
void build_hot_remap(inl_plan p) {
  inl_ctx ctx = p->ctx;
  cudaStream_t st = ctx->stream;
  const int64_t ng = p->n_global, nnz = p->nnz;
  int64_t n_hot = hot_capacity(p->bins.t_warp);
  if (const char *e = getenv("INL_HOT_K")) n_hot = atoll(e) & ~(int64_t)3;
  if (p->transient) n_hot = 0;  // a one-shot call does not amortise the remap
  if (n_hot > ng) n_hot = ng;
  if (nnz == 0) n_hot = 0;
  p->n_hot = n_hot;
  if (n_hot == 0) return;  // the gather reads col_idx directly
  int32_t *pcol = (int32_t *)p->pcol.get(sizeof(int32_t) * (nnz > 0 ? nnz : 1));
  int32_t *cnt = (int32_t *)ctx->s_a.get(sizeof(int32_t) * ng);
  int32_t *cnt_sorted = (int32_t *)ctx->s_b.get(sizeof(int32_t) * ng);
  int32_t *ids = (int32_t *)ctx->s_c.get(sizeof(int32_t) * ng);
  int32_t *ids_sorted = (int32_t *)ctx->s_d.get(sizeof(int32_t) * ng);
  int32_t *hot_rank = (int32_t *)ctx->s_e.get(sizeof(int32_t) * ng);
  const int G = grid_for(nnz, ctx->num_sms);
  INL_CUDA(cudaMemsetAsync(cnt, 0, sizeof(int32_t) * ng, st));
  k_col_count<<<G, 256, 0, st>>>(p->col_idx, nnz, cnt);
  k_iota<<<grid_for(ng, ctx->num_sms), 256, 0, st>>>(ids, ng);
  INL_CUDA(cudaGetLastError());
  size_t need = 0;
  INL_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, need, cnt, cnt_sorted, ids, ids_sorted, ng, 0, 32, st));
  INL_CUDA(cub::DeviceRadixSort::SortPairsDescending(ctx->s_tmp.get(need), need, cnt, cnt_sorted, ids, ids_sorted,
                                                     ng, 0, 32, st));
  INL_CUDA(cudaMemsetAsync(hot_rank, 0xFF, sizeof(int32_t) * ng, st));
  int32_t *hot_cols = (int32_t *)p->hot_cols.get(sizeof(int32_t) * n_hot);
  k_hot_rank<<<grid_for(n_hot, ctx->num_sms), 256, 0, st>>>(ids_sorted, n_hot, hot_rank, hot_cols);
  k_remap<<<G, 256, 0, st>>>(p->col_idx, nnz, hot_rank, pcol);
  INL_CUDA(cudaGetLastError());
  float *xh = (float *)p->x_hot.get(sizeof(float) * ((n_hot + 3) & ~3));
  INL_CUDA(cudaMemsetAsync(xh, 0, sizeof(float) * ((n_hot + 3) & ~3), st));
  INL_CUDA(cudaStreamSynchronize(st));
}

void build_plan(inl_plan p) {
  inl_ctx ctx = p->ctx;
  cudaStream_t st = ctx->stream;
  const int64_t n = p->n_rows;
  const Bins &b = p->bins;
  p->info.bins = {b.t_thread, b.t_warp, b.t_block, b.grid_chunk, b.cta, b.flags};
  p->pr_od = nullptr;  // PageRank compaction is rebuilt for a (re)built plan
  p->n_tiles = p->n_long = p->n_chunks = 0;
  if (n == 0) return;
  INL_CHECK(n < INT32_MAX, "plan: n_rows must be < 2^31");
  const int G = grid_for(n, ctx->num_sms);

  // scratch layout (ctx-owned, reused across plans)
  int32_t *short_deg = (int32_t *)ctx->s_a.get(sizeof(int32_t) * n);
  uint8_t *is_long = (uint8_t *)ctx->s_b.get(n);
  int64_t *P = (int64_t *)ctx->s_c.get(sizeof(int64_t) * n);
  uint8_t *flag = (uint8_t *)ctx->s_d.get(n);
  int32_t *S = (int32_t *)ctx->s_e.get(sizeof(int32_t) * n);
  int64_t *d_cnt = (int64_t *)ctx->s_f.get(sizeof(int64_t) * 8 + sizeof(unsigned long long) * 8);
  unsigned long long *d_stats = (unsigned long long *)(d_cnt + 8);

  k_classify<<<G, 256, 0, st>>>(p->row_ptr, n, b.t_warp, short_deg, is_long);
  INL_CUDA(cudaGetLastError());
  size_t need = 0;
  INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, short_deg, P, n, st));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(ctx->s_tmp.get(need), need, short_deg, P, n, st));
  k_boundary<<<G, 256, 0, st>>>(P, is_long, n, tile_stride(b.t_warp), flag);
  INL_CUDA(cudaGetLastError());
  thrust::counting_iterator<int32_t> iota(0);
  INL_CUDA(cub::DeviceSelect::Flagged(nullptr, need, iota, flag, S, d_cnt, n, st));
  INL_CUDA(cub::DeviceSelect::Flagged(ctx->s_tmp.get(need), need, iota, flag, S, d_cnt, n, st));
  // long rows (reuse `flag` semantics through is_long)
  int32_t *long_tmp = short_deg;  // short_deg is dead after the scan
  INL_CUDA(cub::DeviceSelect::Flagged(nullptr, need, iota, is_long, long_tmp, d_cnt + 1, n, st));
  INL_CUDA(cub::DeviceSelect::Flagged(ctx->s_tmp.get(need), need, iota, is_long, long_tmp, d_cnt + 1, n,
                                      st));
  int64_t h_cnt[2] = {0, 0};
  INL_CUDA(cudaMemcpyAsync(h_cnt, d_cnt, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  const int64_t K = h_cnt[0];
  p->n_long = h_cnt[1];

  // tiles = boundary segments that do not start at a long row
  int2 *cand = (int2 *)P;             // P is dead now; 8 B per entry fits (K <= n)
  uint8_t *valid = flag;              // flag is dead after the select
  k_emit_tiles<<<grid_for(K, ctx->num_sms), 256, 0, st>>>(S, d_cnt, is_long, n, cand, valid);
  INL_CUDA(cudaGetLastError());
  int2 *tiles = (int2 *)p->tiles.get(sizeof(int2) * (K > 0 ? K : 1));
  INL_CUDA(cub::DeviceSelect::Flagged(nullptr, need, cand, valid, tiles, d_cnt + 2, K, st));
  INL_CUDA(cub::DeviceSelect::Flagged(ctx->s_tmp.get(need), need, cand, valid, tiles, d_cnt + 2, K, st));

  // long rows -> chunks
  if (p->n_long > 0) {
    int32_t *long_rows = (int32_t *)p->long_rows.get(sizeof(int32_t) * p->n_long);
    INL_CUDA(cudaMemcpyAsync(long_rows, long_tmp, sizeof(int32_t) * p->n_long, cudaMemcpyDeviceToDevice, st));
    int32_t *nch = (int32_t *)ctx->s_e.get(sizeof(int32_t) * n);  // S is dead now
    int32_t *base = (int32_t *)p->chunk_base.get(sizeof(int32_t) * p->n_long);
    k_long_chunks<<<grid_for(p->n_long, ctx->num_sms), 256, 0, st>>>(p->row_ptr, long_rows, p->n_long,
                                                                     b.grid_chunk, nch);
    INL_CUDA(cudaGetLastError());
    INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, nch, base, p->n_long, st));
    INL_CUDA(cub::DeviceScan::ExclusiveSum(ctx->s_tmp.get(need), need, nch, base, p->n_long, st));
    int32_t last[2] = {0, 0};
    INL_CUDA(cudaMemcpyAsync(&last[0], base + p->n_long - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    INL_CUDA(cudaMemcpyAsync(&last[1], nch + p->n_long - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    INL_CUDA(cudaStreamSynchronize(st));
    p->n_chunks = (int64_t)last[0] + last[1];
    int2 *items = (int2 *)p->chunk_items.get(sizeof(int2) * p->n_chunks);
    k_chunk_items<<<grid_for(p->n_long * 32, ctx->num_sms), 128, 0, st>>>(nch, base, p->n_long, items);
    INL_CUDA(cudaGetLastError());
    p->partials.get(sizeof(float) * p->n_chunks);
    int *tk = (int *)p->tickets.get(sizeof(int) * p->n_long);
    INL_CUDA(cudaMemsetAsync(tk, 0, sizeof(int) * p->n_long, st));
  }
  INL_CUDA(cudaMemsetAsync(d_stats, 0, sizeof(unsigned long long) * 8, st));
  k_bin_stats<<<G, 256, 0, st>>>(p->row_ptr, n, b, d_stats);
  INL_CUDA(cudaGetLastError());
  unsigned long long h_st[8];
  int64_t h_nt = 0;
  INL_CUDA(cudaMemcpyAsync(h_st, d_stats, sizeof h_st, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaMemcpyAsync(&h_nt, d_cnt + 2, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  p->n_tiles = h_nt;
  p->n_items = p->n_tiles + p->n_chunks;
  {
    WorkItem *items = (WorkItem *)p->items.get(sizeof(WorkItem) * (p->n_items > 0 ? p->n_items : 1));
    const int32_t *nch = (const int32_t *)ctx->s_e.p;  // valid when n_long > 0
    k_build_items<<<grid_for(p->n_items, ctx->num_sms), 256, 0, st>>>(
        p->row_ptr, tiles, p->n_tiles, (const int2 *)p->chunk_items.p, (const int32_t *)p->long_rows.p,
        nch, (const int32_t *)p->chunk_base.p, p->n_chunks, b.grid_chunk, items);
    INL_CUDA(cudaGetLastError());
  }
  if (p->n_tiles > 0) {
    uint32_t *nz = (uint32_t *)p->tile_nz.get(sizeof(uint32_t) * 8 * p->n_tiles);
    k_tile_nz<<<grid_for(p->n_tiles * 32, ctx->num_sms), 256, 0, st>>>(p->row_ptr, tiles, p->n_tiles, nz);
    INL_CUDA(cudaGetLastError());
  }
  p->dpart.get(sizeof(double) * (p->n_items + 1));
  {
    const int64_t nw = p->nnz / 32 + 2;
    uint32_t *bits = (uint32_t *)p->rs_bits.get(sizeof(uint32_t) * nw);
    INL_CUDA(cudaMemsetAsync(bits, 0, sizeof(uint32_t) * nw, st));
    k_rowstart_bits<<<G, 256, 0, st>>>(p->row_ptr, n, bits);
    INL_CUDA(cudaGetLastError());
  }
  build_hot_remap(p);
  p->symmetric = false;
  if (!p->transient && p->n_rows == p->n_global && p->row_begin == 0) {  // one-shot calls skip it
    int *bad = (int *)ctx->s_f.get(64);
    INL_CUDA(cudaMemsetAsync(bad, 0, sizeof(int), st));
    k_check_symmetric<<<grid_for(n * 32, ctx->num_sms), 256, 0, st>>>(p->row_ptr, p->col_idx, n, bad);
    INL_CUDA(cudaGetLastError());
    int h_bad = 1;
    INL_CUDA(cudaMemcpyAsync(&h_bad, bad, sizeof(int), cudaMemcpyDeviceToHost, st));
    INL_CUDA(cudaStreamSynchronize(st));
    p->symmetric = h_bad == 0;
    if (p->symmetric) bu_static_build(p);
  }
  p->info.symmetric = p->symmetric ? 1 : 0;
  cb_build(p, p->cb, p->col_idx, p->n_global);
  p->pr_cb.active = false;
  INL_CUDA(cudaMemsetAsync(p->ticket.get(16), 0, 16, st));
  p->ticket_base = 0;
  p->info.n_tiles = p->n_tiles;
  p->info.rows_thread = (int64_t)h_st[0];
  p->info.rows_warp = (int64_t)h_st[1];
  p->info.rows_block = (int64_t)h_st[2];
  p->info.rows_grid = (int64_t)h_st[3];
  p->info.nnz_thread = (int64_t)h_st[4];
  p->info.nnz_warp = (int64_t)h_st[5];
  p->info.nnz_block = (int64_t)h_st[6];
  p->info.nnz_grid = (int64_t)h_st[7];
  p->info.n_grid_chunks = p->n_chunks;
  p->info.cb_rows = p->cb.active ? p->cb.n_rows : 0;
  p->info.cb_runs = p->cb.active ? p->cb.n_pairs : 0;
  p->info.cb_nnz = p->cb.active ? p->cb.n_entries : 0;
  p->info.cb_width = p->cb.active ? p->cb.K : 0;
  p->info.cb_threshold = p->cb.active ? p->cb.t_cb : 0;
}

}  // namespace inl
