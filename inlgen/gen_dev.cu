// gen_dev.cu — device (CUDA) twin of gen_host.cpp: bit-identical graphs, built
// on the GPU so the large configurations (R-MAT scale 22..26) are generated in
// seconds.  Input side only; none of the method's arithmetic lives here.
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>
#include <cstdlib>
#include <cstring>

#include "../include/inlgen.h"
#include "inlgen_core.h"
#include "inlgen_graph.h"

#define IG_CUDA(call)                                                             \
  do {                                                                            \
    cudaError_t e_ = (call);                                                      \
    if (e_ != cudaSuccess) {                                                      \
      inlgen_set_error("%s:%d %s: %s", __FILE__, __LINE__, #call,                 \
                       cudaGetErrorString(e_));                                   \
      rc = -3;                                                                    \
      goto done;                                                                  \
    }                                                                             \
  } while (0)

__global__ void k_gen_keys(uint64_t *keys, uint64_t m, int scale, uint64_t seed, int flags,
                           uint64_t sentinel) {
  const bool sym = flags & INLGEN_SYMMETRIC, tr = flags & INLGEN_TRANSPOSE;
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m;
       e += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t a, b;
    ig_rmat_edge(seed, scale, e, &a, &b);
    uint64_t u = ig_relabel(a, scale, seed), v = ig_relabel(b, scale, seed);
    if (sym) {
      keys[2 * e] = (u == v) ? sentinel : ((u << scale) | v);
      keys[2 * e + 1] = (u == v) ? sentinel : ((v << scale) | u);
    } else {
      keys[e] = (u == v) ? sentinel : (tr ? ((v << scale) | u) : ((u << scale) | v));
    }
  }
}

__device__ __forceinline__ int64_t lower_bound_u64(const uint64_t *a, int64_t n, uint64_t key) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] < key) lo = mid + 1; else hi = mid;
  }
  return lo;
}

__global__ void k_row_ptr(const uint64_t *keys, int64_t nkeys, int scale, int64_t row_begin,
                          int64_t n_rows, int64_t base, int64_t *row_ptr) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r <= n_rows;
       r += (int64_t)gridDim.x * blockDim.x)
    row_ptr[r] = lower_bound_u64(keys, nkeys, (uint64_t)(row_begin + r) << scale) - base;
}

__global__ void k_cols(const uint64_t *keys, int64_t lo, int64_t cnt, uint64_t mask,
                       int32_t *col) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt;
       i += (int64_t)gridDim.x * blockDim.x)
    col[i] = (int32_t)(keys[lo + i] & mask);
}

__global__ void k_outdeg(const uint64_t *keys, int64_t cnt, uint64_t mask, int32_t *deg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt;
       i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&deg[keys[i] & mask], 1);
}

__global__ void k_find_range(const uint64_t *keys, int64_t nkeys, int scale, int64_t rb,
                             int64_t re, int64_t *out) {
  out[0] = lower_bound_u64(keys, nkeys, (uint64_t)rb << scale);
  out[1] = lower_bound_u64(keys, nkeys, (uint64_t)re << scale);
}

static int grid_for(int64_t n) {
  int64_t g = (n + 255) / 256;
  if (g > 148 * 64) g = 148 * 64;
  return g < 1 ? 1 : (int)g;
}

extern "C" int inlgen_dev_build(int scale, int edge_factor, uint64_t seed, int flags,
                                int64_t row_begin, int64_t row_end, void *stream_,
                                inlgen_graph *out) {
  int rc = 0;
  cudaStream_t st = (cudaStream_t)stream_;
  uint64_t *k0 = nullptr, *k1 = nullptr;
  int64_t *d_cnt = nullptr;
  void *tmp = nullptr;
  size_t tmp_bytes = 0, need = 0;
  inlgen_graph g = nullptr;
  int64_t h_cnt[2] = {0, 0}, h_range[2] = {0, 0};
  if (!out || scale < 1 || scale > 30 || edge_factor < 1) {
    inlgen_set_error("inlgen_dev_build: bad argument (scale 1..30, edge_factor >= 1)");
    return -1;
  }
  const int64_t n = (int64_t)1 << scale;
  if (row_end < 0) row_end = n;
  if (row_begin < 0 || row_begin > row_end || row_end > n) {
    inlgen_set_error("inlgen_dev_build: bad row range");
    return -1;
  }
  const uint64_t m = (uint64_t)edge_factor << scale;
  const bool sym = flags & INLGEN_SYMMETRIC;
  const int64_t nk = (int64_t)(sym ? 2 * m : m);
  const int bits = 2 * scale;
  const uint64_t mask = ((uint64_t)1 << scale) - 1;
  const uint64_t sentinel = (mask << scale) | mask;  // (n-1, n-1): a self-loop, sorts last
  cub::DoubleBuffer<uint64_t> db;
  int64_t nu = 0;

  g = (inlgen_graph)calloc(1, sizeof(*g));
  if (!g) return -2;
  g->n_global = n;
  g->row_begin = row_begin;
  g->n_rows = row_end - row_begin;
  g->on_device = 1;

  IG_CUDA(cudaMalloc(&k0, sizeof(uint64_t) * nk));
  IG_CUDA(cudaMalloc(&k1, sizeof(uint64_t) * nk));
  IG_CUDA(cudaMalloc(&d_cnt, sizeof(int64_t) * 4));
  k_gen_keys<<<grid_for((int64_t)m), 256, 0, st>>>(k0, m, scale, seed, flags, sentinel);
  IG_CUDA(cudaGetLastError());
  db = cub::DoubleBuffer<uint64_t>(k0, k1);
  IG_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, need, db, nk, 0, bits, st));
  tmp_bytes = need;
  IG_CUDA(cub::DeviceSelect::Unique(nullptr, need, db.Current(), db.Alternate(), d_cnt, nk, st));
  if (need > tmp_bytes) tmp_bytes = need;
  IG_CUDA(cudaMalloc(&tmp, tmp_bytes));
  IG_CUDA(cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, db, nk, 0, bits, st));
  IG_CUDA(cub::DeviceSelect::Unique(tmp, tmp_bytes, db.Current(), db.Alternate(), d_cnt, nk, st));
  IG_CUDA(cudaMemcpyAsync(h_cnt, d_cnt, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  IG_CUDA(cudaStreamSynchronize(st));
  {
    // unique keys are in db.Alternate(); drop the trailing sentinel if present
    uint64_t last = 0;
    nu = h_cnt[0];
    if (nu > 0) {
      IG_CUDA(cudaMemcpy(&last, db.Alternate() + nu - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost));
      if (last == sentinel) --nu;
    }
  }
  {
    const uint64_t *uk = db.Alternate();
    if (flags & INLGEN_TRANSPOSE) {
      IG_CUDA(cudaMalloc(&g->out_degree, sizeof(int32_t) * n));
      IG_CUDA(cudaMemsetAsync(g->out_degree, 0, sizeof(int32_t) * n, st));
      if (nu > 0) k_outdeg<<<grid_for(nu), 256, 0, st>>>(uk, nu, mask, g->out_degree);
      IG_CUDA(cudaGetLastError());
    }
    k_find_range<<<1, 1, 0, st>>>(uk, nu, scale, row_begin, row_end, d_cnt + 2);
    IG_CUDA(cudaMemcpyAsync(h_range, d_cnt + 2, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    IG_CUDA(cudaStreamSynchronize(st));
    g->nnz = h_range[1] - h_range[0];
    IG_CUDA(cudaMalloc(&g->row_ptr, sizeof(int64_t) * (g->n_rows + 1)));
    IG_CUDA(cudaMalloc(&g->col_idx, sizeof(int32_t) * (g->nnz > 0 ? g->nnz : 1)));
    k_row_ptr<<<grid_for(g->n_rows + 1), 256, 0, st>>>(uk, nu, scale, row_begin, g->n_rows,
                                                        h_range[0], g->row_ptr);
    IG_CUDA(cudaGetLastError());
    if (g->nnz > 0)
      k_cols<<<grid_for(g->nnz), 256, 0, st>>>(uk, h_range[0], g->nnz, mask, g->col_idx);
    IG_CUDA(cudaGetLastError());
    IG_CUDA(cudaStreamSynchronize(st));
  }
done:
  cudaFree(k0);
  cudaFree(k1);
  cudaFree(d_cnt);
  cudaFree(tmp);
  if (rc) {
    inlgen_graph_free(g);
    return rc;
  }
  *out = g;
  return 0;
}

extern "C" int inlgen_graph_export(inlgen_graph g, int64_t *row_ptr, int32_t *col_idx,
                                   int32_t *out_degree, void *stream_) {
  int rc = 0;
  cudaStream_t st = (cudaStream_t)stream_;
  if (!g) return -1;
  if (out_degree && !g->out_degree) {
    inlgen_set_error("inlgen_graph_export: graph has no out_degree (build with INLGEN_TRANSPOSE)");
    return -1;
  }
  if (!g->on_device) {
    // host graph: plain host copies (the destination must be host memory)
    if (row_ptr) memcpy(row_ptr, g->row_ptr, sizeof(int64_t) * (g->n_rows + 1));
    if (col_idx && g->nnz) memcpy(col_idx, g->col_idx, sizeof(int32_t) * g->nnz);
    if (out_degree) memcpy(out_degree, g->out_degree, sizeof(int32_t) * g->n_global);
    return 0;
  }
  if (row_ptr)
    IG_CUDA(cudaMemcpyAsync(row_ptr, g->row_ptr, sizeof(int64_t) * (g->n_rows + 1),
                            cudaMemcpyDefault, st));
  if (col_idx && g->nnz)
    IG_CUDA(cudaMemcpyAsync(col_idx, g->col_idx, sizeof(int32_t) * g->nnz, cudaMemcpyDefault, st));
  if (out_degree)
    IG_CUDA(cudaMemcpyAsync(out_degree, g->out_degree, sizeof(int32_t) * g->n_global,
                            cudaMemcpyDefault, st));
  IG_CUDA(cudaStreamSynchronize(st));
done:
  return rc;
}

extern "C" void inlgen_graph_free(inlgen_graph g) {
  if (!g) return;
  if (g->on_device) {
    cudaFree(g->row_ptr);
    cudaFree(g->col_idx);
    cudaFree(g->out_degree);
  } else {
    free(g->row_ptr);
    free(g->col_idx);
    free(g->out_degree);
    free(g->val);
    free(g->parent);
  }
  free(g);
}

__global__ void k_weights(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                          const int32_t *col, uint64_t seed, uint32_t *w) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n_rows;
       r += (int64_t)gridDim.x * blockDim.x)
    for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
      w[k] = ig_weight(seed, (uint64_t)(row_begin + r), (uint64_t)col[k]);
}

__global__ void k_values(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                         const int32_t *col, uint64_t seed, int mode, float *val) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n_rows;
       r += (int64_t)gridDim.x * blockDim.x)
    for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
      val[k] = ig_value(seed, (uint64_t)(row_begin + r), (uint64_t)col[k], mode);
}

__global__ void k_vector(int64_t n, int64_t begin, uint64_t seed, int mode, float *x) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    x[i] = ig_vector(seed, (uint64_t)(begin + i), mode);
}

extern "C" int inlgen_weights_dev(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                                  const int32_t *col_idx, uint64_t seed, uint32_t *w,
                                  void *stream) {
  if (n_rows < 0) return -1;
  if (n_rows == 0) return 0;
  k_weights<<<grid_for(n_rows), 256, 0, (cudaStream_t)stream>>>(n_rows, row_begin, row_ptr,
                                                                 col_idx, seed, w);
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

extern "C" int inlgen_values_dev(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                                 const int32_t *col_idx, uint64_t seed, int mode, float *val,
                                 void *stream) {
  if (n_rows < 0) return -1;
  if (n_rows == 0) return 0;
  k_values<<<grid_for(n_rows), 256, 0, (cudaStream_t)stream>>>(n_rows, row_begin, row_ptr,
                                                                col_idx, seed, mode, val);
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

extern "C" int inlgen_vector_dev(int64_t n, int64_t begin, uint64_t seed, int mode, float *x,
                                 void *stream) {
  if (n < 0) return -1;
  if (n == 0) return 0;
  k_vector<<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(n, begin, seed, mode, x);
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
