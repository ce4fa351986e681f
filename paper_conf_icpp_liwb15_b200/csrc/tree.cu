// tree.cu — tree descendants / heights (§II.C Fig. 3, §III.C):
// the paper's flat template against the B200 form of its hierarchical one, without CUDA
// dynamic parallelism.
//
//  * INL_TREE_FLAT — Fig. 3(c), "parallelizes the iterative version of the code using
//    thread-based mapping": one thread per node walks up the parent chain; descendants adds 1 to
//    every ancestor (atomicAdd), heights pushes (distance + 1) into every ancestor of a leaf
//    (atomicMax).  Atomics = sum of node depths (d + 2d^2 + 3d^3 on a regular depth-4 tree, the
//    Fig. 7(c) "Atomic" column), counted into stats.edges_relaxed.
//  * INL_TREE_LEVELS — Fig. 3(e)'s hierarchical mapping (a block over the children of a node,
//    threads over them) recast for B200 without nested launches: the nodes are grouped by level
//    (a top-down BFS over the children CSR + a radix sort by level), then one launch per level,
//    deepest first, in which 8-lane groups pull their node's children (the irregular nested loop
//    of Fig. 1(a): outer loop over the level's nodes, inner loop over the children) — no atomics,
//    `depth` launches instead of the 1 + d nested grids of rec-hier (Fig. 7(c) "KCalls").
#include <cub/device/device_radix_sort.cuh>

#include <algorithm>
#include <vector>

#include "comm.h"
#include "inl_internal.cuh"

namespace inl {

namespace {

int tgrid(int64_t n, int sms) {
  int64_t g = (n + 255) / 256;
  if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
  return g < 1 ? 1 : (int)g;
}

__global__ void k_tree_fill(int64_t *__restrict__ out, int64_t n, const int32_t *__restrict__ level) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    out[v] = level[v] >= 0 ? 1 : 0;  // unreachable from the root: 0 (as the oracle)
}

// Fig. 3(c): every node adds itself to each ancestor's count
__global__ void k_tree_flat_desc(const int32_t *__restrict__ parent, const int32_t *__restrict__ level, int64_t n,
                                 unsigned long long *desc, unsigned long long *atomics) {
  unsigned long long c = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    if (level[v] < 0) continue;
    for (int32_t u = parent[v]; u >= 0; u = parent[u]) {
      atomicAdd(desc + u, 1ull);
      ++c;
    }
  }
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(atomics, c);
}

// heights, flat: every leaf pushes its distance + 1 into each ancestor
__global__ void k_tree_flat_height(const int64_t *__restrict__ rp, const int32_t *__restrict__ parent,
                                   const int32_t *__restrict__ level, int64_t n, unsigned long long *height,
                                   unsigned long long *atomics) {
  unsigned long long c = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    if (level[v] < 0 || rp[v + 1] > rp[v]) continue;  // leaves only
    unsigned long long h = 1;
    for (int32_t u = parent[v]; u >= 0; u = parent[u]) {
      atomicMax(height + u, ++h);
      ++c;
    }
  }
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(atomics, c);
}

// one level, deepest first: 8-lane groups pull the children of their node (sum or max + 1)
template <bool HEIGHT>
__global__ void k_tree_level(const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                             const int32_t *__restrict__ nodes, int64_t count, int64_t *out) {
  constexpr int G = 8;
  const int gl = threadIdx.x & (G - 1);
  const int64_t ng = ((int64_t)gridDim.x * blockDim.x) / G;
  const int64_t nn = (count + 3) / 4 * 4;  // a warp's 4 groups iterate together
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / G; i < nn; i += ng) {
    int64_t acc = 0;
    int32_t v = -1;
    if (i < count) {
      v = nodes[i];
      for (int64_t k = rp[v] + gl; k < rp[v + 1]; k += G) {
        const int64_t x = out[col[k]];
        acc = HEIGHT ? (x > acc ? x : acc) : acc + x;
      }
    }
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) {
      const int64_t y = __shfl_xor_sync(0xffffffffu, acc, o);
      acc = HEIGHT ? (y > acc ? y : acc) : acc + y;
    }
    if (gl == 0 && v >= 0) out[v] = 1 + acc;
  }
}

// nodes per level: a per-CTA shared histogram when the tree is shallow (the paper's trees have
// 4-6 levels: a global histogram would be a same-address atomic storm), global atomics otherwise
constexpr int kHistSmem = 8192;
__global__ void k_level_hist(const int32_t *__restrict__ level, int64_t n, int depth, unsigned long long *hist) {
  extern __shared__ unsigned int sh[];
  const bool shm = depth <= kHistSmem;
  if (shm)
    for (int i = threadIdx.x; i < depth; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const int L = level[v];
    if (L < 0 || L >= depth) continue;
    if (shm) atomicAdd(sh + L, 1u);
    else atomicAdd(hist + L, 1ull);
  }
  __syncthreads();
  if (shm)
    for (int i = threadIdx.x; i < depth; i += blockDim.x)
      if (sh[i]) atomicAdd(hist + i, (unsigned long long)sh[i]);
}

__global__ void k_level_keys(const int32_t *__restrict__ level, int64_t n, uint32_t *__restrict__ key,
                             int32_t *__restrict__ ids) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    key[v] = level[v] < 0 ? 0xFFFFFFFFu : (uint32_t)level[v];  // unreachable last
    ids[v] = (int32_t)v;
  }
}

}  // namespace

void tree_run(inl_ctx ctx, const inl_csr &T, const int32_t *parent, int64_t root, int method, bool heights,
              int64_t *out, inl_stats *stats) {
  cudaStream_t st = ctx->stream;
  const int64_t n = T.n_global;
  if (n == 0) return;
  INL_CHECK(n < INT32_MAX, "tree: n must be < 2^31");
  // node levels: a top-down BFS from the root over the children CSR
  int32_t *level = (int32_t *)ctx->s_h.get(sizeof(int32_t) * (size_t)n);
  inl_stats bst{};
  bfs_run(ctx, T, resolve_bins(nullptr), root, level, &bst, false);
  unsigned long long *atomics = (unsigned long long *)ctx->s_f.get(64) + 4;
  INL_CUDA(cudaMemsetAsync(atomics, 0, sizeof(unsigned long long), st));
  int64_t launches = 1;
  k_tree_fill<<<tgrid(n, ctx->num_sms), 256, 0, st>>>(out, n, level);
  if (method == INL_TREE_FLAT) {
    INL_CHECK(parent != nullptr, "tree: INL_TREE_FLAT needs parent[]");
    if (heights) {
      KScope ks(ctx, "k_tree_flat");
      k_tree_flat_height<<<tgrid(n, ctx->num_sms), 256, 0, st>>>(T.row_ptr, parent, level, n,
                                                                 (unsigned long long *)out, atomics);
    } else {
      KScope ks(ctx, "k_tree_flat");
      k_tree_flat_desc<<<tgrid(n, ctx->num_sms), 256, 0, st>>>(parent, level, n, (unsigned long long *)out, atomics);
    }
    INL_CUDA(cudaGetLastError());
    launches += 1;
  } else {
    // nodes sorted by level (stable: level order inside a level), then levels deepest first
    uint32_t *k0 = (uint32_t *)ctx->s_a.get(sizeof(uint32_t) * (size_t)n);
    uint32_t *k1 = (uint32_t *)ctx->s_b.get(sizeof(uint32_t) * (size_t)n);
    int32_t *i0 = (int32_t *)ctx->s_c.get(sizeof(int32_t) * (size_t)n);
    int32_t *i1 = (int32_t *)ctx->s_e.get(sizeof(int32_t) * (size_t)n);
    k_level_keys<<<tgrid(n, ctx->num_sms), 256, 0, st>>>(level, n, k0, i0);
    cub::DoubleBuffer<uint32_t> kb(k0, k1);
    cub::DoubleBuffer<int32_t> vb(i0, i1);
    size_t need = 0;
    INL_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, need, kb, vb, (int)n, 0, 32, st));
    INL_CUDA(cub::DeviceRadixSort::SortPairs(ctx->s_tmp.get(need), need, kb, vb, (int)n, 0, 32, st));
    // level sizes (a histogram over the BFS's levels 0 .. iterations-1) -> boundaries on the host
    const int depth = bst.iterations > 0 ? bst.iterations : 1;
    unsigned long long *hist = (unsigned long long *)ctx->s_g.get(sizeof(unsigned long long) * (size_t)(depth + 1));
    INL_CUDA(cudaMemsetAsync(hist, 0, sizeof(unsigned long long) * (size_t)(depth + 1), st));
    k_level_hist<<<tgrid(n, ctx->num_sms), 256, depth <= kHistSmem ? sizeof(unsigned int) * depth : 0, st>>>(
        level, n, depth, hist);
    INL_CUDA(cudaGetLastError());
    std::vector<unsigned long long> hc((size_t)depth);
    INL_CUDA(cudaMemcpyAsync(hc.data(), hist, sizeof(unsigned long long) * (size_t)depth, cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    std::vector<int64_t> lo((size_t)depth + 1, 0);
    for (int L = 0; L < depth; ++L) lo[(size_t)L + 1] = lo[(size_t)L] + (int64_t)hc[(size_t)L];
    const int32_t *nodes = vb.Current();
    for (int L = depth - 1; L >= 0; --L) {
      const int64_t cnt = lo[(size_t)L + 1] - lo[(size_t)L];
      if (cnt <= 0) continue;
      KScope ks(ctx, "k_tree_level");
      if (heights)
        k_tree_level<true><<<tgrid(cnt * 8, ctx->num_sms), 256, 0, st>>>(T.row_ptr, T.col_idx, nodes + lo[(size_t)L],
                                                                         cnt, out);
      else
        k_tree_level<false><<<tgrid(cnt * 8, ctx->num_sms), 256, 0, st>>>(T.row_ptr, T.col_idx, nodes + lo[(size_t)L],
                                                                          cnt, out);
      INL_CUDA(cudaGetLastError());
      ++launches;
    }
  }
  if (stats) {
    unsigned long long a = 0;
    INL_CUDA(cudaMemcpyAsync(&a, atomics, sizeof a, cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    stats->iterations = bst.iterations;      // levels
    stats->edges_relaxed = (int64_t)a;       // atomics (INL_TREE_FLAT), 0 for INL_TREE_LEVELS
    stats->frontier_total = bst.frontier_total;
    stats->launches = launches;
    stats->host_syncs = bst.host_syncs + 1;
    stats->exchange_bytes = 0;
  }
}

}  // namespace inl
