// Microbenchmark (not product code): the memory-system ceilings of the SpMV stream on B200.
//   k_stream: sum of col+val streamed with 128-bit loads            -> DRAM streaming bound
//   k_gather: the same stream + x[col] random gather (read-only)      -> + L2 gather bound
// Timed with CUDA events, best of `iters`.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

__global__ void k_stream(const int4 *__restrict__ col, const float4 *__restrict__ val, int64_t n4,
                         float *out) {
  float acc = 0.f;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    int4 c = __ldcs(col + i);
    float4 v = __ldcs(val + i);
    acc += v.x + v.y + v.z + v.w + (float)(c.x ^ c.y ^ c.z ^ c.w);
  }
  if (acc == 1234.5f) out[0] = acc;
}

template <int U>
__global__ void k_gather(const int4 *__restrict__ col, const float4 *__restrict__ val, int64_t n4,
                         const float *__restrict__ x, float *out) {
  float acc = 0.f;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += stride * U) {
    int4 c[U];
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      int64_t k = i + u * stride;
      if (k < n4) { c[u] = __ldcs(col + k); v[u] = __ldcs(val + k); }
      else { c[u] = make_int4(0, 0, 0, 0); v[u] = make_float4(0, 0, 0, 0); }
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
      acc += v[u].x * __ldg(x + c[u].x) + v[u].y * __ldg(x + c[u].y) + v[u].z * __ldg(x + c[u].z) +
             v[u].w * __ldg(x + c[u].w);
  }
  if (acc == 1234.5f) out[0] = acc;
}

// hot columns (encoded c < 0: ~c is the hot index) read from a shared-memory copy of x_hot
template <int U>
__global__ void __launch_bounds__(1024, 1) k_gather_hot(const int4 *__restrict__ col, const float4 *__restrict__ val, int64_t n4,
                             const float *__restrict__ x, const float *__restrict__ xhot, int nhot, float *out) {
  extern __shared__ float xs[];
  for (int i = threadIdx.x; i < nhot; i += blockDim.x) xs[i] = xhot[i];
  __syncthreads();
  float acc = 0.f;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += stride * U) {
    int4 c[U];
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      int64_t k = i + u * stride;
      if (k < n4) { c[u] = __ldcs(col + k); v[u] = __ldcs(val + k); }
      else { c[u] = make_int4(0, 0, 0, 0); v[u] = make_float4(0, 0, 0, 0); }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      int cc[4] = {c[u].x, c[u].y, c[u].z, c[u].w};
      float vv[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
#pragma unroll
      for (int j = 0; j < 4; ++j) acc += vv[j] * (cc[j] < 0 ? xs[~cc[j]] : __ldg(x + cc[j]));
    }
  }
  if (acc == 1234.5f) out[0] = acc;
}

extern "C" int mb_run_hot(const int32_t *col, const float *val, int64_t nnz, const float *x, const float *xhot,
                          int nhot, int block, int iters, float *best_ms, int unroll) {
  float *out;
  cudaMalloc(&out, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  size_t smem = (size_t)nhot * 4;
  cudaFuncSetAttribute(k_gather_hot<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_gather_hot<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_gather_hot<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e30f;
  for (int it = 0; it < iters; ++it) {
    cudaEventRecord(a);
    if (unroll == 4) k_gather_hot<4><<<sms, block, smem>>>((const int4 *)col, (const float4 *)val, nnz / 4, x, xhot, nhot, out);
    else if (unroll == 1) k_gather_hot<1><<<sms, block, smem>>>((const int4 *)col, (const float4 *)val, nnz / 4, x, xhot, nhot, out);
    else k_gather_hot<2><<<sms, block, smem>>>((const int4 *)col, (const float4 *)val, nnz / 4, x, xhot, nhot, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  *best_ms = best;
  cudaFree(out);
  return (int)cudaGetLastError();
}

extern "C" int mb_run(const int32_t *col, const float *val, int64_t nnz, const float *x, int which,
                      int grid_mult, int block, int iters, float *best_ms) {
  float *out;
  cudaMalloc(&out, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t n4 = nnz / 4;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e30f;
  for (int it = 0; it < iters; ++it) {
    cudaEventRecord(a);
    if (which == 0) k_stream<<<sms * grid_mult, block>>>((const int4 *)col, (const float4 *)val, n4, out);
    else if (which == 1) k_gather<1><<<sms * grid_mult, block>>>((const int4 *)col, (const float4 *)val, n4, x, out);
    else k_gather<4><<<sms * grid_mult, block>>>((const int4 *)col, (const float4 *)val, n4, x, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  *best_ms = best;
  cudaFree(out);
  return (int)cudaGetLastError();
}
