// templates.cu — the paper's load-balancing templates for the irregular nested loop,
// written as the paper describes them (prior art on B200, for the template study of
// SURVEY §8f NEXT-2; the default SpMV path is the fused gather of gather.cuh).
//
// PAPER.md P5@2074-3874 (Fig. 1(b, c)), lbTHRES = bins.t_thread (P5@332), CTA size =
// bins.cta_threads (P5@11808, P11@1656):
//   * dual-queue (Fig. 1(b)): a pre-pass "divides the elements processed in the outer
//     loop in two queues depending on the number of iterations they require in the
//     inner-loop and processes those queues separately using thread- and block-based
//     mapping" — k_tpl_queues, then k_tpl_thread over the small queue and k_tpl_block
//     over the large one.
//   * dbuf-global (Fig. 1(c)): a thread-mapped kernel "delays the execution of large
//     iterations of the outer loop by queuing them in a buffer" in global memory; a second
//     kernel processes the buffer block-mapped, "redistributing the work among
//     thread-blocks" — k_tpl_dbuf_global, then k_tpl_block.
//   * dbuf-shared: the buffer lives in shared memory; "a single kernel invocation but
//     possibly leading to uneven work distribution among thread-blocks" —
//     k_tpl_dbuf_shared.
// val == nullptr: implicit unit values (PageRank's pull through the templates, pagerank.cu).
// Row sums: serial in one thread (thread mapping) or strided over the CTA plus a fixed
// shared-memory tree (block mapping): deterministic.  Queue order from atomics may vary;
// each row's sum does not.
#include <cub/device/device_select.cuh>

#include "inl_internal.cuh"

namespace inl {

namespace {

__device__ __forceinline__ float row_serial(const int64_t *rp, const int32_t *col, const float *val,
                                            const float *x, int64_t r) {
  float acc = 0.0f;
  for (int64_t k = rp[r]; k < rp[r + 1]; ++k) acc += (val ? val[k] : 1.0f) * __ldg(x + col[k]);
  return acc;
}

// block-mapped row: threads stride the inner loop, then a fixed tree over the CTA
__device__ __forceinline__ float row_block(const int64_t *rp, const int32_t *col, const float *val,
                                           const float *x, int64_t r, float *red) {
  float acc = 0.0f;
  for (int64_t k = rp[r] + threadIdx.x; k < rp[r + 1]; k += blockDim.x)
    acc += (val ? val[k] : 1.0f) * __ldg(x + col[k]);
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  const int warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  __syncthreads();  // red[] reuse
  if ((threadIdx.x & 31) == 0) red[warp] = acc;
  __syncthreads();
  float s = 0.0f;
  if (threadIdx.x == 0)
    for (int q = 0; q < nw; ++q) s += red[q];
  return s;  // valid in thread 0
}

// dual-queue pre-pass: rows of degree <= lbt -> small queue, others -> large queue
__global__ void k_tpl_queues(const int64_t *__restrict__ rp, int64_t n, int lbt, int32_t *qs, int *ns, int32_t *ql,
                             int *nl) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = rp[r + 1] - rp[r];
    if (d <= lbt) qs[atomicAdd(ns, 1)] = (int32_t)r;
    else ql[atomicAdd(nl, 1)] = (int32_t)r;
  }
}

// thread mapping over a queue (count read on the device)
__global__ void k_tpl_thread(const int32_t *__restrict__ q, const int *__restrict__ nq, const int64_t *rp,
                             const int32_t *col, const float *val, const float *x, float *y) {
  const int n = *nq;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t r = q[i];
    y[r] = row_serial(rp, col, val, x, r);
  }
}

// block mapping over a queue: one CTA per row, grid-stride (count read on the device)
__global__ void k_tpl_block(const int32_t *__restrict__ q, const int *__restrict__ nq, const int64_t *rp,
                            const int32_t *col, const float *val, const float *x, float *y) {
  __shared__ float red[32];
  const int n = *nq;
  for (int i = blockIdx.x; i < n; i += gridDim.x) {
    const int32_t r = q[i];
    const float s = row_block(rp, col, val, x, r, red);
    if (threadIdx.x == 0) y[r] = s;
  }
}

// dbuf-global phase 1: thread per row; large rows queued in a global buffer
__global__ void k_tpl_dbuf_global(const int64_t *__restrict__ rp, int64_t n, int lbt, const int32_t *col,
                                  const float *val, const float *x, float *y, int32_t *buf, int *nbuf) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
    if (rp[r + 1] - rp[r] <= lbt) y[r] = row_serial(rp, col, val, x, r);
    else buf[atomicAdd(nbuf, 1)] = (int32_t)r;
  }
}

// dbuf-shared: thread per row; large rows queued in shared memory and processed
// block-mapped by the same CTA after __syncthreads
__global__ void k_tpl_dbuf_shared(const int64_t *__restrict__ rp, int64_t n, int lbt, const int32_t *col,
                                  const float *val, const float *x, float *y) {
  extern __shared__ int32_t sbuf[];  // [blockDim.x]
  __shared__ int ns;
  __shared__ float red[32];
  for (int64_t r0 = blockIdx.x * (int64_t)blockDim.x; r0 < n; r0 += (int64_t)gridDim.x * blockDim.x) {
    if (threadIdx.x == 0) ns = 0;
    __syncthreads();
    const int64_t r = r0 + threadIdx.x;
    if (r < n) {
      if (rp[r + 1] - rp[r] <= lbt) y[r] = row_serial(rp, col, val, x, r);
      else sbuf[atomicAdd(&ns, 1)] = (int32_t)r;
    }
    __syncthreads();
    const int m = ns;
    for (int j = 0; j < m; ++j) {
      const int32_t rr = sbuf[j];
      const float s = row_block(rp, col, val, x, rr, red);
      if (threadIdx.x == 0) y[rr] = s;
    }
    __syncthreads();
  }
}

int tpl_grid(int64_t work, int cta, int sms) {
  int64_t g = (work + cta - 1) / cta;
  const int64_t cap = (int64_t)sms * 32;
  if (g > cap) g = cap;
  return g < 1 ? 1 : (int)g;
}

}  // namespace

bool spmv_template(inl_ctx ctx, const inl_csr &A, const Bins &b, const float *val, const float *x, float *y) {
  const int which = b.flags & (INL_BINS_TPL_DUAL_QUEUE | INL_BINS_TPL_DBUF_GLOBAL | INL_BINS_TPL_DBUF_SHARED);
  if (!which) return false;
  INL_CHECK(which == INL_BINS_TPL_DUAL_QUEUE || which == INL_BINS_TPL_DBUF_GLOBAL ||
                which == INL_BINS_TPL_DBUF_SHARED,
            "bins.flags: at most one paper template");
  const int64_t n = A.n_rows;
  if (n == 0) return true;
  INL_CHECK(n < INT32_MAX, "template kernels: n_rows must be < 2^31");
  cudaStream_t st = ctx->stream;
  const int cta = b.cta, lbt = b.t_thread;
  const int sms = ctx->num_sms;
  int *cnt = (int *)ctx->s_f.get(64);
  INL_CUDA(cudaMemsetAsync(cnt, 0, 2 * sizeof(int), st));
  if (which == INL_BINS_TPL_DUAL_QUEUE) {
    int32_t *qs = (int32_t *)ctx->s_a.get(sizeof(int32_t) * n);
    int32_t *ql = (int32_t *)ctx->s_b.get(sizeof(int32_t) * n);
    {
      KScope ks(ctx, "k_tpl_queues");
      k_tpl_queues<<<tpl_grid(n, 256, sms), 256, 0, st>>>(A.row_ptr, n, lbt, qs, cnt, ql, cnt + 1);
    }
    {
      KScope ks(ctx, "k_tpl_thread");
      k_tpl_thread<<<tpl_grid(n, cta, sms), cta, 0, st>>>(qs, cnt, A.row_ptr, A.col_idx, val, x, y);
    }
    KScope ks(ctx, "k_tpl_block");
    k_tpl_block<<<sms * 16, cta, 0, st>>>(ql, cnt + 1, A.row_ptr, A.col_idx, val, x, y);
  } else if (which == INL_BINS_TPL_DBUF_GLOBAL) {
    int32_t *buf = (int32_t *)ctx->s_a.get(sizeof(int32_t) * n);
    {
      KScope ks(ctx, "k_tpl_dbuf_global");
      k_tpl_dbuf_global<<<tpl_grid(n, cta, sms), cta, 0, st>>>(A.row_ptr, n, lbt, A.col_idx, val, x, y, buf, cnt);
    }
    KScope ks(ctx, "k_tpl_block");
    k_tpl_block<<<sms * 16, cta, 0, st>>>(buf, cnt, A.row_ptr, A.col_idx, val, x, y);
  } else {
    KScope ks(ctx, "k_tpl_dbuf_shared");
    k_tpl_dbuf_shared<<<tpl_grid(n, cta, sms), cta, sizeof(int32_t) * cta, st>>>(A.row_ptr, n, lbt, A.col_idx, val,
                                                                                x, y);
  }
  INL_CUDA(cudaGetLastError());
  return true;
}

}  // namespace inl
