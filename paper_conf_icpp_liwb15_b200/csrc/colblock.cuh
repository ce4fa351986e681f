// colblock.cuh — the column-blocked deferred bin of the SpMV / PageRank gather.
//
// Paper: long inner loops are deferred to a buffer and processed block-mapped
// (dbuf-global, P5@2721; "f(i) greater than lbTHRES is processed block-mapped",
// P11@1197).  B200 form: a random x[col] gather from global memory costs
// one L1TEX wavefront per distinct 128-B line (~1 per SM-cycle), a gather from shared
// memory ~1/7 of that.  So rows of degree > t_cb (>= 4 entries per column block on
// average) are split by column block: CTA c holds block b of x (K floats) in shared
// memory and sums every (row, block) run of its share into partials[run]; k_cb_combine
// adds a row's partials in block order (fp64) and applies the epilogue.  Each sum's
// order depends only on the row's columns and K — never on the CTA split — so results
// are deterministic and partition-invariant.
#pragma once
#include "inl_internal.cuh"
#include "ptx.cuh"

namespace inl {

struct CbArgs {
  const CbPair *pairs;
  const uint16_t *cbcol;
  const int64_t *blk_first;  // [nblocks + 1]
  const int64_t *cta_lo;     // [grid + 1]
  float *partials;
  int64_t ncols, nblocks;
  int K;
  // combine
  const int32_t *rows;
  const int64_t *rp_base;
  const int64_t *pos_of;
  int64_t n_rows;
};

constexpr int kCbWarps = 32;   // 1 CTA per SM (x block in shared memory)
constexpr int kCbLanes = 4;    // lanes per run
constexpr int kCbUnroll = 8;   // entries per lane in flight

// Runs of one CTA: pairs [cta_lo[c], cta_lo[c+1]), walked block by block.
template <bool VALS>
__global__ void __launch_bounds__(kCbWarps * 32, 1) k_cb(CbArgs c, const float *__restrict__ val,
                                                         const float *__restrict__ x) {
  extern __shared__ __align__(16) float xs[];
  constexpr int RPW = 32 / kCbLanes;       // runs per warp per step
  constexpr int RPC = kCbWarps * RPW;      // runs per CTA per step
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int sub = lane % kCbLanes;
  int64_t i0 = c.cta_lo[blockIdx.x];
  const int64_t i1 = c.cta_lo[blockIdx.x + 1];
  if (i0 >= i1) return;
  // block of the first run: last b with blk_first[b] <= i0
  int64_t lo = 0, hi = c.nblocks - 1;
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (c.blk_first[mid] <= i0) lo = mid;
    else hi = mid - 1;
  }
  int64_t b = lo;
  while (i0 < i1) {
    int64_t bend = c.blk_first[b + 1];
    if (bend <= i0) {  // empty block(s)
      ++b;
      continue;
    }
    const int64_t iend = bend < i1 ? bend : i1;
    // x block b -> shared memory
    const int64_t c0 = b * (int64_t)c.K;
    const int w = (int)((c.ncols - c0) < c.K ? (c.ncols - c0) : c.K);
    __syncthreads();  // the previous block's readers are done
    if ((c0 & 3) == 0) {
      const float4 *src = reinterpret_cast<const float4 *>(x + c0);
      for (int t = tid; t < (w >> 2); t += kCbWarps * 32) reinterpret_cast<float4 *>(xs)[t] = __ldg(src + t);
      for (int t = (w & ~3) + tid; t < w; t += kCbWarps * 32) xs[t] = __ldg(x + c0 + t);
    } else {
      for (int t = tid; t < w; t += kCbWarps * 32) xs[t] = __ldg(x + c0 + t);
    }
    __syncthreads();
    // the next step's run descriptors are loaded before the current step's entries
    int64_t ib = i0 + (int64_t)warp * RPW;
    CbPair nx{0, 0, 0, 0};
    bool nok = ib + lane / kCbLanes < iend;
    if (nok) nx = c.pairs[ib + lane / kCbLanes];
    for (; ib < iend; ib += RPC) {  // warp-uniform trip count
      const int64_t i = ib + lane / kCbLanes;
      const CbPair pr = nx;
      const bool ok = nok;
      nok = i + RPC < iend;
      if (nok) nx = c.pairs[i + RPC];
      float s = 0.0f;
      if (ok) {
        for (int t0 = 0; t0 < pr.len; t0 += kCbLanes * kCbUnroll) {
          uint32_t cc[kCbUnroll];
          float vv[kCbUnroll];
#pragma unroll
          for (int u = 0; u < kCbUnroll; ++u) {
            const int t = t0 + u * kCbLanes + sub;
            const bool in = t < pr.len;
            cc[u] = in ? (uint32_t)__ldcs(c.cbcol + pr.cb + t) : 0u;
            vv[u] = VALS ? (in ? __ldcs(val + pr.cs + t) : 0.0f) : (in ? 1.0f : 0.0f);
          }
#pragma unroll
          for (int u = 0; u < kCbUnroll; ++u) s = fmaf(vv[u], xs[cc[u]], s);
        }
      }
#pragma unroll
      for (int o = kCbLanes / 2; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (ok && sub == 0) c.partials[i] = s;
    }
    i0 = iend;
    ++b;
  }
}

// One warp per column-blocked row: partials in block order (fixed fp64 tree per 32 runs,
// chunks added in order), then the epilogue.  dpart[j] = the epilogue's dangling value.
template <class Epi>
__global__ void __launch_bounds__(256) k_cb_combine(CbArgs c, Epi epi, double *dpart) {
  epi.init();
  const int lane = threadIdx.x & 31;
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < c.n_rows;
       j += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int64_t q0 = c.rp_base[j], q1 = c.rp_base[j + 1];
    double tot = 0.0;
    for (int64_t q = q0; q < q1; q += 32) {
      double v = q + lane < q1 ? (double)c.partials[c.pos_of[q + lane]] : 0.0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
      tot += v;
    }
    if (lane == 0) {
      const double d = epi(c.rows[j], (float)tot);
      if (dpart) dpart[j] = d;
    }
  }
}

inline CbArgs cb_args(const CbPlan &cb) {
  CbArgs a;
  a.pairs = (const CbPair *)cb.pairs.p;
  a.cbcol = (const uint16_t *)cb.cbcol.p;
  a.blk_first = (const int64_t *)cb.blk_first.p;
  a.cta_lo = (const int64_t *)cb.cta_lo.p;
  a.partials = (float *)cb.partials.p;
  a.ncols = cb.ncols;
  a.nblocks = cb.nblocks;
  a.K = cb.K;
  a.rows = (const int32_t *)cb.rows.p;
  a.rp_base = (const int64_t *)cb.rp_base.p;
  a.pos_of = (const int64_t *)cb.pos_of.p;
  a.n_rows = cb.n_rows;
  return a;
}

template <bool VALS, class Epi>
void launch_cb(inl_ctx ctx, const CbPlan &cb, const float *val, const float *x, const Epi &epi, double *dpart) {
  const CbArgs a = cb_args(cb);
  const size_t smem = (size_t)cb.K * 4;
  static size_t configured[kMaxDevices] = {};  // per instantiation AND device
  size_t &cf = configured[ctx->device % kMaxDevices];
  if (smem > cf) {
    INL_CUDA(cudaFuncSetAttribute(k_cb<VALS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    cf = smem;
  }
  {
    KScope ks(ctx, "k_cb");
    k_cb<VALS><<<cb.grid, kCbWarps * 32, smem, ctx->stream>>>(a, val, x);
    INL_CUDA(cudaGetLastError());
  }
  int64_t g = (cb.n_rows * 32 + 255) / 256;
  if (g > (int64_t)ctx->num_sms * 8) g = (int64_t)ctx->num_sms * 8;
  KScope ks(ctx, "k_cb_combine");
  k_cb_combine<Epi><<<(int)(g < 1 ? 1 : g), 256, 0, ctx->stream>>>(a, epi, dpart);
  INL_CUDA(cudaGetLastError());
}

}  // namespace inl
