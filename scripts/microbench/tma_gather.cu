// Microbenchmark (not product code): random 4-byte gather throughput per SM on B200 via
//   (0) LDG (ld.global.cg) — one L1TEX wavefront per distinct 128-B line, ~1 line/SM-cycle
//   (1) TMA tile::gather4 — x viewed as a [n/4][4] fp32 tensor, one gather4 fetches four
//       random 16-B rows into shared memory (mbarrier complete_tx), then 1 LDS per value
//   (2) both at once (half of each lane's gathers on each path).
// Question it answers: does the TMA unit give SpMV's cold x[col] gathers a second path
// around the L1TEX wavefront limit?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_gather tma_gather.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#define CK(x)                                                                          \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess) {                                                           \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      exit(1);                                                                         \
    }                                                                                  \
  } while (0)

constexpr int W = 16;      // warps per CTA
constexpr int S = 3;       // pipeline stages per warp
constexpr int G = 1;       // gather4 per lane per stage (smem: W*S*32*G*PITCH <= 227 KB)
constexpr int PITCH = 128;  // bytes per lane-group of 4 rows (TMA destinations are 128-B aligned)

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

__device__ __forceinline__ void mbar_init(uint32_t a, int c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(c));
}
__device__ __forceinline__ void mbar_expect(uint32_t a, uint32_t tx) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t par) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra W;\n\t}" ::"r"(a),
      "r"(par)
      : "memory");
}
__device__ __forceinline__ void gather4(uint32_t dst, const CUtensorMap *tm, uint32_t mbar, int r0, int r1, int r2,
                                        int r3) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
      "l"(tm), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(mbar)
      : "memory");
}

// MODE 0: LDG only; MODE 1: TMA only; MODE 2: half / half; MODE 3: TMA, values not read
template <int MODE>
__global__ void __launch_bounds__(W * 32, 1) k_bench(const __grid_constant__ CUtensorMap tm, const float *x,
                                                     uint32_t n, int iters, float *out) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ __align__(8) uint64_t mbar[W][S];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t buf = (uint32_t)__cvta_generic_to_shared(sm) + (uint32_t)warp * S * 32 * G * PITCH;
  if (lane == 0)
    for (int s = 0; s < S; ++s) mbar_init((uint32_t)__cvta_generic_to_shared(&mbar[warp][s]), 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t st = hash32(blockIdx.x * W * 32 + threadIdx.x);
  float acc = 0.f;
  constexpr int GL = 4 * G;  // gathers per lane per stage on each path
  auto issue = [&](int s, uint32_t &seed, uint32_t (&sel)[GL]) {
    const uint32_t mb = (uint32_t)__cvta_generic_to_shared(&mbar[warp][s]);
    if (lane == 0) mbar_expect(mb, 32 * G * 64);
    __syncwarp();
#pragma unroll
    for (int g = 0; g < G; ++g) {
      int r[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        seed = seed * 1664525u + 1013904223u;
        const uint32_t i = (uint32_t)(((uint64_t)(seed >> 4) * n) >> 28);
        r[q] = (int)(i >> 2);
        sel[4 * g + q] = i & 3;
      }
      gather4(buf + (uint32_t)((s * G + g) * 32 + lane) * PITCH, &tm, mb, r[0], r[1], r[2], r[3]);
    }
  };
  if (MODE == 0) {
    for (int it = 0; it < iters; ++it) {
      float v[GL];
#pragma unroll
      for (int u = 0; u < GL; ++u) {
        st = st * 1664525u + 1013904223u;
        const uint32_t i = (uint32_t)(((uint64_t)(st >> 4) * n) >> 28);
        asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v[u]) : "l"(x + i));
      }
#pragma unroll
      for (int u = 0; u < GL; ++u) acc += v[u];
    }
  } else {
    uint32_t sel[S][GL];
    uint32_t tseed = st ^ 0x5bd1e995u;
#pragma unroll
    for (int s = 0; s < S; ++s) issue(s, tseed, sel[s]);
    for (int it = 0; it < iters; it += S) {
#pragma unroll
      for (int s = 0; s < S; ++s) {
        float v[GL];
        if (MODE == 2) {
#pragma unroll
          for (int u = 0; u < GL; ++u) {
            st = st * 1664525u + 1013904223u;
            const uint32_t i = (uint32_t)(((uint64_t)(st >> 4) * n) >> 28);
            asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v[u]) : "l"(x + i));
          }
        }
        mbar_wait((uint32_t)__cvta_generic_to_shared(&mbar[warp][s]), (uint32_t)((it / S) & 1));
#pragma unroll
        for (int g = 0; g < G; ++g)
#pragma unroll
          for (int q = 0; q < (MODE == 3 ? 0 : 4); ++q) {
            float t;
            const uint32_t a = buf + (uint32_t)((s * G + g) * 32 + lane) * PITCH + q * 16 + sel[s][4 * g + q] * 4;
            asm volatile("ld.shared.f32 %0, [%1];" : "=f"(t) : "r"(a));
            acc += t;
          }
        if (MODE == 2) {
#pragma unroll
          for (int u = 0; u < GL; ++u) acc += v[u];
        }
        __syncwarp();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (it + S < iters) issue(s, tseed, sel[s]);
      }
    }
  }
  if (acc == -1.f) out[0] = acc;
}

int main(int argc, char **argv) {
  const uint32_t n = argc > 1 ? (uint32_t)atol(argv[1]) : (1u << 22);
  const int iters = 510;  // stages per warp (a multiple of S)
  int sms = 0, clk = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0));
  float *x, *out;
  CK(cudaMalloc(&x, (size_t)n * 4));
  CK(cudaMemset(x, 0, (size_t)n * 4));
  CK(cudaMalloc(&out, 4));
  auto enc = cuTensorMapEncodeTiled;
  CUtensorMap tm;
  cuuint64_t dims[2] = {4, n / 4};
  cuuint64_t strides[1] = {16};
  cuuint32_t box[2] = {4, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, x, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    printf("encode failed %d\n", (int)r);
    return 1;
  }
  const int smem = W * S * 32 * G * PITCH;
  auto run = [&](auto kern, const char *name, double gathers_per_thread) {
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    kern<<<sms, W * 32, smem>>>(tm, x, n, iters, out);
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(a));
    const int reps = 5;
    for (int i = 0; i < reps; ++i) kern<<<sms, W * 32, smem>>>(tm, x, n, iters, out);
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    ms /= reps;
    const double g = gathers_per_thread * W * 32;  // per SM
    const double cyc = ms * 1e-3 * clk * 1e3;
    printf("%-10s n=%10u: %8.1f us  %.2f gathers/SM-cycle (%.0f per SM)\n", name, n, ms * 1e3, g / cyc, g);
  };
  run(k_bench<0>, "ldg", (double)iters * 4 * G);
  run(k_bench<1>, "tma", (double)iters * 4 * G);
  run(k_bench<2>, "ldg+tma", (double)iters * 8 * G);
  run(k_bench<3>, "tma-noread", (double)iters * 4 * G);
  return 0;
}
