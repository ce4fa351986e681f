// Microbenchmark (not product code): random 4-byte gather throughput on B200 from
//   (a) the CTA's own shared memory, (b) distributed shared memory of a thread-block
//   cluster of C CTAs (mapa + ld.shared::cluster), (c) an L2-resident global array.
// Question it answers: can a cluster-wide shared-memory copy of the hot part of x
// (C x ~190 KB) serve SpMV gathers faster than L1TEX (1 wavefront per distinct line)?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o dsmem_gather dsmem_gather.cu
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

namespace cg = cooperative_groups;

#define CK(x)                                                                   \
  do {                                                                          \
    cudaError_t e_ = (x);                                                       \
    if (e_ != cudaSuccess) {                                                    \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      return 1;                                                                 \
    }                                                                           \
  } while (0)

constexpr int kThreads = 1024;
constexpr int kIters = 2048;  // gathers per thread (8 independent chains of 256)

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

// MODE 0: local smem, 1: cluster DSMEM (uniform over the cluster), 2: global
template <int MODE>
__global__ void __launch_bounds__(kThreads, 1) k_gather(const float *__restrict__ g, uint32_t gmask, int S,
                                                       float *out) {
  extern __shared__ float xs[];
  for (int i = threadIdx.x; i < S; i += kThreads) xs[i] = (float)(i & 7);
  uint32_t nct = 1, myrank = 0;
  if (MODE == 1) {
    cg::cluster_group cl = cg::this_cluster();
    nct = cl.num_blocks();
    myrank = cl.block_rank();
    cl.sync();
  } else {
    __syncthreads();
  }
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(xs);
  uint32_t st[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) st[u] = hash32(blockIdx.x * kThreads + threadIdx.x + u * 0x9e3779b9u);
  float acc = 0.f;
  for (int it = 0; it < kIters / 8; ++it) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      st[u] = st[u] * 1664525u + 1013904223u;
      const uint32_t r = st[u] >> 8;
      float v;
      if (MODE == 0) {
        const uint32_t a = base + (r % (uint32_t)S) * 4u;
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
      } else if (MODE == 1) {
        const uint32_t idx = r % ((uint32_t)S * nct);
        const uint32_t cta = idx / (uint32_t)S, off = idx - cta * (uint32_t)S;
        uint32_t ra;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(base + off * 4u), "r"(cta));
        asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(ra));
      } else {
        v = __ldg(g + (r & gmask));
      }
      acc += v;
    }
  }
  (void)myrank;
  if (MODE == 1) cg::this_cluster().sync();
  if (acc == 1234.5f) out[0] = acc;
}

template <int MODE>
static int run(const char *name, int cluster, int S, const float *g, uint32_t gmask, float *out, int nsm,
               double clk_ghz) {
  auto kern = k_gather<MODE>;
  const size_t smem = (size_t)S * 4;
  CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  if (cluster > 8) CK(cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  int grid = nsm;
  if (cluster > 1) grid = (nsm / cluster) * cluster;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = cluster;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  if (cluster > 1) {
    int ncl = 0;
    CK(cudaOccupancyMaxActiveClusters(&ncl, kern, &cfg));
    if (ncl * cluster < grid) grid = ncl * cluster;
    cfg.gridDim = dim3(grid);
  }
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  float best = 1e30f;
  for (int rep = 0; rep < 6; ++rep) {
    CK(cudaEventRecord(a));
    CK(cudaLaunchKernelEx(&cfg, kern, g, gmask, S, out));
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    if (rep > 0 && ms < best) best = ms;
  }
  const double loads = (double)grid * kThreads * kIters;
  const double per_sm_cyc = loads / (best * 1e-3 * clk_ghz * 1e9 * grid);
  printf("%-10s cluster=%2d S=%6d grid=%3d : %8.1f us  %6.2f lane-loads/SM-cycle  %6.3f cyc per warp-load\n",
         name, cluster, S, grid, best * 1e3, per_sm_cyc, 32.0 / per_sm_cyc);
  return 0;
}

int main() {
  int nsm = 0, clk_khz = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0));
  const double clk = clk_khz * 1e-6;
  printf("SMs %d, clock %.3f GHz (nominal; timing uses it for cycles)\n", nsm, clk);
  float *g, *out;
  CK(cudaMalloc(&g, (size_t)(1 << 24) * 4));
  CK(cudaMemset(g, 0, (size_t)(1 << 24) * 4));
  CK(cudaMalloc(&out, 4));
  const int S = 48 * 1024;
  if (run<0>("smem", 1, S, g, 0, out, nsm, clk)) return 1;
  for (int c : {2, 4, 8, 16})
    if (run<1>("dsmem", c, S, g, 0, out, nsm, clk)) return 1;
  if (run<2>("global4M", 1, 1024, g, (1u << 22) - 1, out, nsm, clk)) return 1;
  if (run<2>("global16M", 1, 1024, g, (1u << 24) - 1, out, nsm, clk)) return 1;
  return 0;
}
