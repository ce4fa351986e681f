// colblock.cu — plan side of the column-blocked deferred bin (colblock.cuh).
//
// For the rows of degree > t_cb = max(t_warp, mult * nblocks) of a plan, in the column
// space `cols` (raw ids in [0, ncols)):
//   runs   — maximal stretches of a row whose columns share one block b = col / K (rows
//            are column-sorted, so a row's runs follow block order);
//   pairs  — the runs sorted by (block, length descending, row), with their entries'
//            offsets within the block copied to cbcol (uint16);
//   cta_lo — equal shares of the run entries, one per CTA of k_cb;
//   items  — the plan's gather work items without the chunks of those rows.
// Built once per plan (SpMV) or per compacted PageRank space; never on the hot path.
// sort_rows: the rows' columns are copied and sorted per row first (a column space that
// does not keep CSR rows sorted; only for value-free gathers — runs' cs then index that
// copy, not the CSR).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>
#include <cub/device/device_select.cuh>

#include <cstdlib>

#include "colblock.cuh"
#include "gather.cuh"

namespace inl {

namespace {

int grid_of(int64_t n, int sms) {
  int64_t g = (n + 255) / 256;
  if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
  return g < 1 ? 1 : (int)g;
}

__global__ void k_cb_rowflag(const int64_t *__restrict__ rp, const int32_t *__restrict__ long_rows, int64_t n_long,
                             int t_cb, uint8_t *__restrict__ f) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n_long;
       j += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = long_rows[j];
    f[j] = rp[r + 1] - rp[r] > t_cb;
  }
}

// entry range of each column-blocked row in the run source: the CSR itself ...
__global__ void k_cb_ranges(const int64_t *__restrict__ rp, const int32_t *__restrict__ rows, int64_t n_rows,
                            int64_t *__restrict__ rs, int64_t *__restrict__ re) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n_rows;
       j += (int64_t)gridDim.x * blockDim.x) {
    rs[j] = rp[rows[j]];
    re[j] = rp[rows[j] + 1];
  }
}

// ... or a copy of the rows' columns (goff = exclusive scan of their degrees), sorted per
// row afterwards when the column space does not keep rows column-sorted (PageRank's
// degree-ordered compact space; no values, so the entry order within a row is free)
__global__ void k_cb_degrees(const int64_t *__restrict__ rp, const int32_t *__restrict__ rows, int64_t n_rows,
                             int64_t *__restrict__ deg) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n_rows;
       j += (int64_t)gridDim.x * blockDim.x)
    deg[j] = rp[rows[j] + 1] - rp[rows[j]];
}

__global__ void k_cb_copy_rows(const int64_t *__restrict__ rp, const int32_t *__restrict__ rows, int64_t n_rows,
                               const int32_t *__restrict__ cols, const int64_t *__restrict__ goff,
                               int32_t *__restrict__ out, int64_t *__restrict__ re) {
  const int lane = threadIdx.x & 31;
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_rows;
       j += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int64_t s = rp[rows[j]], d = rp[rows[j] + 1] - s, o = goff[j];
    for (int64_t t = lane; t < d; t += 32) out[o + t] = cols[s + t];
    if (lane == 0) re[j] = o + d;
  }
}

// one warp per row: number of runs (entries whose block differs from the previous one's)
__global__ void k_cb_count(const int64_t *__restrict__ rs, const int64_t *__restrict__ re, int64_t n_rows,
                           const int32_t *__restrict__ cols, int K, int64_t *__restrict__ cnt) {
  const int lane = threadIdx.x & 31;
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_rows;
       j += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int64_t s = rs[j], e = re[j];
    int64_t c = 0;
    for (int64_t k = s + lane; k < e; k += 32) c += k == s || cols[k] / K != cols[k - 1] / K;
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0) cnt[j] = c;
  }
}

// one warp per row: run starts in row order (q = rp_base[j] + rank)
__global__ void k_cb_emit(const int64_t *__restrict__ rs, const int64_t *__restrict__ re, int64_t n_rows,
                          const int32_t *__restrict__ cols, int K, const int64_t *__restrict__ base,
                          int64_t *__restrict__ qs, int32_t *__restrict__ qj) {
  const int lane = threadIdx.x & 31;
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_rows;
       j += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int64_t s = rs[j], e = re[j];
    int64_t q = base[j];
    for (int64_t k0 = s; k0 < e; k0 += 32) {
      const int64_t k = k0 + lane;
      const bool st = k < e && (k == s || cols[k] / K != cols[k - 1] / K);
      const unsigned m = __ballot_sync(0xffffffffu, st);
      if (st) {
        const int64_t qq = q + __popc(m & ((1u << lane) - 1u));
        qs[qq] = k;
        qj[qq] = (int32_t)j;
      }
      q += __popc(m);
    }
  }
}

// run lengths and sort keys (block, ~length)
__global__ void k_cb_keys(const int64_t *__restrict__ re, const int64_t *__restrict__ base,
                          const int64_t *__restrict__ qs,
                          const int32_t *__restrict__ qj, const int32_t *__restrict__ cols, int K, int64_t n_pairs,
                          int32_t *__restrict__ len, uint64_t *__restrict__ key, int64_t *__restrict__ ids) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n_pairs;
       q += (int64_t)gridDim.x * blockDim.x) {
    const int32_t j = qj[q];
    const int64_t end = q + 1 < base[j + 1] ? qs[q + 1] : re[j];
    const int32_t l = (int32_t)(end - qs[q]);
    len[q] = l;
    key[q] = ((uint64_t)(uint32_t)(cols[qs[q]] / K) << 32) | (uint64_t)(~(uint32_t)l);
    ids[q] = q;
  }
}

__global__ void k_cb_sorted_len(const int64_t *__restrict__ ord, const int32_t *__restrict__ len, int64_t n,
                                int64_t *__restrict__ slen, int64_t *__restrict__ pos_of) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = ord[i];
    slen[i] = len[q];
    pos_of[q] = i;
  }
}

__global__ void k_cb_pairs(const int64_t *__restrict__ ord, const int64_t *__restrict__ qs,
                           const int32_t *__restrict__ qj, const int32_t *__restrict__ len,
                           const int64_t *__restrict__ cbs, int64_t n, CbPair *__restrict__ pairs) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = ord[i];
    CbPair p;
    p.cs = qs[q];
    p.cb = cbs[i];
    p.len = len[q];
    p.j = qj[q];
    pairs[i] = p;
  }
}

// one warp per pair: local column offsets
__global__ void k_cb_cols(const CbPair *__restrict__ pairs, int64_t n, const int32_t *__restrict__ cols, int K,
                          uint16_t *__restrict__ cbcol) {
  const int lane = threadIdx.x & 31;
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n;
       i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const CbPair p = pairs[i];
    const int32_t c0 = cols[p.cs] / K * K;
    for (int t = lane; t < p.len; t += 32) cbcol[p.cb + t] = (uint16_t)(cols[p.cs + t] - c0);
  }
}

// blk_first[b] = first sorted pair with block >= b (b in [0, nblocks])
__global__ void k_cb_blk_first(const uint64_t *__restrict__ skey, int64_t n, int64_t nblocks,
                               int64_t *__restrict__ bf) {
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b <= nblocks;
       b += (int64_t)gridDim.x * blockDim.x) {
    int64_t lo = 0, hi = n;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if ((int64_t)(skey[mid] >> 32) < b) lo = mid + 1;
      else hi = mid;
    }
    bf[b] = lo;
  }
}

// cta_lo[c] = first pair whose entries start at or after c * E / G
__global__ void k_cb_cta_lo(const int64_t *__restrict__ cbs, int64_t n, int64_t E, int G,
                            int64_t *__restrict__ lo_out) {
  for (int c = blockIdx.x * blockDim.x + threadIdx.x; c <= G; c += gridDim.x * blockDim.x) {
    if (c == G) {
      lo_out[c] = n;
      continue;
    }
    const int64_t target = (int64_t)((__int128)E * c / G);
    int64_t lo = 0, hi = n;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (cbs[mid] < target) lo = mid + 1;
      else hi = mid;
    }
    lo_out[c] = lo;
  }
}

__global__ void k_cb_itemflag(const WorkItem *__restrict__ items, int64_t n, const int64_t *__restrict__ rp,
                              int t_cb, uint8_t *__restrict__ f) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const WorkItem w = items[i];
    f[i] = w.j < 0 || rp[w.r0 + 1] - rp[w.r0] <= t_cb;
  }
}

}  // namespace

void cb_build(inl_plan p, CbPlan &cb, const int32_t *cols, int64_t ncols, bool sort_rows) {
  inl_ctx ctx = p->ctx;
  cudaStream_t st = ctx->stream;
  cb.active = false;
  cb.n_rows = cb.n_pairs = cb.n_entries = 0;
  if (p->transient || !(p->bins.flags & INL_BINS_COLBLOCK) || (p->bins.flags & INL_BINS_THREAD_ONLY) ||
      p->n_long == 0 || ncols <= 0)
    return;
  int K = 49152;  // 192 KB of x per CTA: leaves ~60 KB of L1 for the in-flight run loads
  if (const char *e = getenv("INL_CB_K")) K = atoi(e);
  if (K > 57344) K = 57344;
  if (K < 32) K = 32;
  K &= ~3;
  int mult = 4;
  if (const char *e = getenv("INL_CB_MULT")) mult = atoi(e);
  cb.K = K;
  cb.ncols = ncols;
  cb.nblocks = (ncols + K - 1) / K;
  const int64_t tcb = (int64_t)mult * cb.nblocks;
  cb.t_cb = (int32_t)(tcb > p->bins.t_warp ? (tcb > INT32_MAX / 2 ? INT32_MAX / 2 : tcb) : p->bins.t_warp);
  const int64_t n_long = p->n_long;
  const int32_t *long_rows = (const int32_t *)p->long_rows.p;

  // rows
  DevBuf flag, tmp, cnt_b;
  uint8_t *f = (uint8_t *)flag.get(n_long > p->n_items ? n_long : p->n_items);
  int64_t *d_n = (int64_t *)cnt_b.get(16);
  k_cb_rowflag<<<grid_of(n_long, ctx->num_sms), 256, 0, st>>>(p->row_ptr, long_rows, n_long, cb.t_cb, f);
  int32_t *rows = (int32_t *)cb.rows.get(sizeof(int32_t) * n_long);
  size_t need = 0;
  INL_CUDA(cub::DeviceSelect::Flagged(nullptr, need, long_rows, f, rows, d_n, n_long, st));
  INL_CUDA(cub::DeviceSelect::Flagged(tmp.get(need), need, long_rows, f, rows, d_n, n_long, st));
  int64_t h = 0;
  INL_CUDA(cudaMemcpyAsync(&h, d_n, sizeof h, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  cb.n_rows = h;
  if (h == 0) return;
  const int64_t nr = cb.n_rows;

  // entry ranges of the rows in the run source `src`
  DevBuf b_rs, b_re, b_src, b_src2;
  int64_t *rs = (int64_t *)b_rs.get(sizeof(int64_t) * (nr + 1));
  int64_t *re = (int64_t *)b_re.get(sizeof(int64_t) * (nr + 1));
  const int32_t *src = cols;
  if (!sort_rows) {
    k_cb_ranges<<<grid_of(nr, ctx->num_sms), 256, 0, st>>>(p->row_ptr, rows, nr, rs, re);
  } else {
    int64_t *deg = re;
    k_cb_degrees<<<grid_of(nr, ctx->num_sms), 256, 0, st>>>(p->row_ptr, rows, nr, deg);
    INL_CUDA(cudaMemsetAsync(deg + nr, 0, sizeof(int64_t), st));
    INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, deg, rs, nr + 1, st));
    INL_CUDA(cub::DeviceScan::ExclusiveSum(tmp.get(need), need, deg, rs, nr + 1, st));
    int64_t tot = 0;
    INL_CUDA(cudaMemcpyAsync(&tot, rs + nr, sizeof tot, cudaMemcpyDeviceToHost, st));
    INL_CUDA(cudaStreamSynchronize(st));
    INL_CHECK(tot < INT32_MAX, "column-blocked PageRank rows: more than 2^31 entries on one rank");
    int32_t *g0 = (int32_t *)b_src.get(sizeof(int32_t) * (tot + 1));
    int32_t *g1 = (int32_t *)b_src2.get(sizeof(int32_t) * (tot + 1));
    k_cb_copy_rows<<<grid_of(nr * 32, ctx->num_sms), 256, 0, st>>>(p->row_ptr, rows, nr, cols, rs, g0, re);
    INL_CUDA(cudaGetLastError());
    INL_CUDA(cub::DeviceSegmentedSort::SortKeys(nullptr, need, g0, g1, (int)tot, (int)nr, rs, re, st));
    INL_CUDA(cub::DeviceSegmentedSort::SortKeys(tmp.get(need), need, g0, g1, (int)tot, (int)nr, rs, re, st));
    src = g1;
  }
  // runs per row -> rp_base
  DevBuf cnt;
  int64_t *c = (int64_t *)cnt.get(sizeof(int64_t) * (nr + 1));
  k_cb_count<<<grid_of(nr * 32, ctx->num_sms), 256, 0, st>>>(rs, re, nr, src, K, c);
  INL_CUDA(cudaMemsetAsync(c + nr, 0, sizeof(int64_t), st));
  int64_t *base = (int64_t *)cb.rp_base.get(sizeof(int64_t) * (nr + 1));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, c, base, nr + 1, st));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(tmp.get(need), need, c, base, nr + 1, st));
  INL_CUDA(cudaMemcpyAsync(&h, base + nr, sizeof h, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  const int64_t np = cb.n_pairs = h;

  // runs in row order, sorted by (block, length desc) — stable, so ties keep row order
  DevBuf b_qs, b_qj, b_len, b_k0, b_k1, b_i0, b_i1, b_slen, b_cbs;
  int64_t *qs = (int64_t *)b_qs.get(sizeof(int64_t) * np);
  int32_t *qj = (int32_t *)b_qj.get(sizeof(int32_t) * np);
  int32_t *len = (int32_t *)b_len.get(sizeof(int32_t) * np);
  uint64_t *k0 = (uint64_t *)b_k0.get(sizeof(uint64_t) * np), *k1 = (uint64_t *)b_k1.get(sizeof(uint64_t) * np);
  int64_t *i0 = (int64_t *)b_i0.get(sizeof(int64_t) * np), *i1 = (int64_t *)b_i1.get(sizeof(int64_t) * np);
  k_cb_emit<<<grid_of(nr * 32, ctx->num_sms), 256, 0, st>>>(rs, re, nr, src, K, base, qs, qj);
  k_cb_keys<<<grid_of(np, ctx->num_sms), 256, 0, st>>>(re, base, qs, qj, src, K, np, len, k0, i0);
  INL_CUDA(cudaGetLastError());
  int end_bit = 32;
  while (end_bit < 64 && ((uint64_t)(cb.nblocks - 1) >> (end_bit - 32))) ++end_bit;
  cub::DoubleBuffer<uint64_t> kb(k0, k1);
  cub::DoubleBuffer<int64_t> vb(i0, i1);
  INL_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, need, kb, vb, np, 0, end_bit, st));
  INL_CUDA(cub::DeviceRadixSort::SortPairs(tmp.get(need), need, kb, vb, np, 0, end_bit, st));
  const int64_t *ord = vb.Current();
  int64_t *slen = (int64_t *)b_slen.get(sizeof(int64_t) * (np + 1));
  int64_t *pos_of = (int64_t *)cb.pos_of.get(sizeof(int64_t) * np);
  k_cb_sorted_len<<<grid_of(np, ctx->num_sms), 256, 0, st>>>(ord, len, np, slen, pos_of);
  INL_CUDA(cudaMemsetAsync(slen + np, 0, sizeof(int64_t), st));
  int64_t *cbs = (int64_t *)b_cbs.get(sizeof(int64_t) * (np + 1));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, need, slen, cbs, np + 1, st));
  INL_CUDA(cub::DeviceScan::ExclusiveSum(tmp.get(need), need, slen, cbs, np + 1, st));
  INL_CUDA(cudaMemcpyAsync(&h, cbs + np, sizeof h, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  cb.n_entries = h;
  CbPair *pairs = (CbPair *)cb.pairs.get(sizeof(CbPair) * np);
  k_cb_pairs<<<grid_of(np, ctx->num_sms), 256, 0, st>>>(ord, qs, qj, len, cbs, np, pairs);
  uint16_t *cbcol = (uint16_t *)cb.cbcol.get(sizeof(uint16_t) * (cb.n_entries + 16));
  k_cb_cols<<<grid_of(np * 32, ctx->num_sms), 256, 0, st>>>(pairs, np, src, K, cbcol);
  int64_t *bf = (int64_t *)cb.blk_first.get(sizeof(int64_t) * (cb.nblocks + 1));
  k_cb_blk_first<<<grid_of(cb.nblocks + 1, ctx->num_sms), 256, 0, st>>>(kb.Current(), np, cb.nblocks, bf);
  cb.grid = ctx->num_sms;
  int64_t *clo = (int64_t *)cb.cta_lo.get(sizeof(int64_t) * (cb.grid + 1));
  k_cb_cta_lo<<<1, 256, 0, st>>>(cbs, np, cb.n_entries, cb.grid, clo);
  cb.partials.get(sizeof(float) * np);
  INL_CUDA(cudaGetLastError());

  // gather items without the column-blocked rows' chunks (stable: longest first stays)
  k_cb_itemflag<<<grid_of(p->n_items, ctx->num_sms), 256, 0, st>>>((const WorkItem *)p->items.p, p->n_items,
                                                                    p->row_ptr, cb.t_cb, f);
  WorkItem *it = (WorkItem *)cb.items.get(sizeof(WorkItem) * (p->n_items > 0 ? p->n_items : 1));
  INL_CUDA(cub::DeviceSelect::Flagged(nullptr, need, (const WorkItem *)p->items.p, f, it, d_n, p->n_items, st));
  INL_CUDA(cub::DeviceSelect::Flagged(tmp.get(need), need, (const WorkItem *)p->items.p, f, it, d_n, p->n_items, st));
  INL_CUDA(cudaMemcpyAsync(&h, d_n, sizeof h, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  cb.n_items = h;
  cb.active = true;
}

}  // namespace inl
