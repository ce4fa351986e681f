// bc.cu — betweenness centrality (PAPER.md P5@8318-8911; reading R10):
// per source, (1) a level-synchronous BFS that builds the shortest-path DAG and the path
// counts sigma, (2) a backward sweep over the levels that accumulates the dependencies
// delta (Brandes' recurrence) into bc.  Both phases are the paper's irregular nested loop
// (outer: the vertices of one level, inner: their adjacency), load-balanced with its
// templates: a CTA takes 256 level vertices; degree <= kBcThread runs serially in one
// thread, larger ones are deferred to shared-memory buffers and run by 8-lane groups
// (<= kBcGroup) or warps (dbuf-shared, P5@3623), the largest are cut into pieces in a
// global buffer that a second kernel runs CTA-mapped (dbuf-global, P5@2721).
//   forward  (level L):  v unvisited -> claimed for L+1 (atomicCAS), enqueued; every edge
//                        into level L+1 adds sigma[u] to sigma[v] (fp64 atomicAdd: path
//                        counts are integers, exact below 2^53).
//   backward (level L):  delta[w] = sum_{v in N(w), level[v] = L+1} sigma[w]/sigma[v] (1+delta[v])
//                        (pull, no atomics; fixed order per vertex), bc[w] += delta[w]; a
//                        finished w leaves (1+delta)/sigma, its level and the sweep's tag in
//                        one 16-B record (one gather per backward edge).
#include <cooperative_groups.h>

#include <cstdlib>
#include <vector>

#include "inl_internal.cuh"

namespace cg = cooperative_groups;

namespace inl {

namespace {

constexpr int kBcNT = 256;
constexpr int kBcThread = 2;     // degree <= 2: one thread (thread-mapped inner loop)
constexpr int kBcGroup = 64;     // degree <= 64: 8 lanes (a quarter warp)
constexpr int kBcWarp = 256;     // degree <= 256: one warp; above: kBcChunk-edge pieces, one CTA each
constexpr int kBcChunk = 2048;   // (global buffer; backward pieces combined in piece order)

// A finished vertex of the backward sweep: (1 + delta) / sigma, its level, and the tag
// (source number + 1) of the sweep that wrote it — one 16-B gather per backward edge
// instead of level + sigma + delta.
struct __align__(16) BcPk {
  double coef;
  int32_t level, tag;
};

struct BcArgs {
  const int64_t *rp;
  const int32_t *col;
  int32_t *level;
  double *sigma, *delta, *bc;
  int32_t *Q;       // visit order (levels contiguous)
  int lo, hi;       // this level's slice of Q
  int L;
  int *qcount;      // forward: vertices enqueued for level L+1 (at Q[hi + i])
  unsigned long long *mf;  // forward: degree sum of the vertices enqueued for level L+1
  int2 *big;        // global buffer: (vertex, piece) of the largest-degree vertices
  int *bigcount;
  int4 *bigv;       // (vertex, first piece, pieces) per large vertex (backward combine)
  int *bigvcount;
  double *bigpart;  // backward partial sum per piece
  int32_t source;
  BcPk *pk;
  int32_t tag;
};

// append v to level L+1 (one counter atomic per coalesced group)
__device__ __forceinline__ void enqueue(const BcArgs &a, int32_t v) {
  cg::coalesced_group g = cg::coalesced_threads();
  int pos = 0;
  if (g.thread_rank() == 0) pos = atomicAdd(a.qcount, (int)g.size());
  pos = g.shfl(pos, 0) + (int)g.thread_rank();
  a.Q[a.hi + pos] = v;
}

// m_f of the level just built: degree sum of Q[hi, hi + *qcount) (Beamer's frontier edge
// count for the push / pull choice), one atomic per warp
__global__ void k_bc_degsum(BcArgs a) {
  const int cntv = *(volatile int *)a.qcount;
  unsigned long long s = 0;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < cntv; i += gridDim.x * blockDim.x) {
    const int32_t v = a.Q[a.hi + i];
    s += (unsigned long long)(a.rp[v + 1] - a.rp[v]);
  }
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(a.mf, s);
}

// forward edge (u at level L, sigma su) -> v
__device__ __forceinline__ void fwd_edge(const BcArgs &a, double su, int32_t v) {
  int lv = a.level[v];
  if (lv == -1) {
    const int old = atomicCAS(a.level + v, -1, a.L + 1);
    if (old == -1) enqueue(a, v);
    lv = a.L + 1;  // whoever won, only level L+1 is claimed in this step
  }
  if (lv == a.L + 1) atomicAdd(a.sigma + v, su);
}

// backward term of edge w -> v: sigma_w / sigma_v (1 + delta_v) for a successor v
__device__ __forceinline__ double bwd_term(const BcArgs &a, double sw, int32_t v) {
  const BcPk p = a.pk[v];
  return p.tag == a.tag && p.level == a.L + 1 ? sw * p.coef : 0.0;
}

__device__ __forceinline__ void bwd_finish(const BcArgs &a, int32_t w, double d) {
  BcPk p;
  p.coef = (1.0 + d) / a.sigma[w];
  p.level = a.L;
  p.tag = a.tag;
  a.pk[w] = p;
  if (w != a.source) a.bc[w] += d;
}

template <bool FWD>
__global__ void __launch_bounds__(kBcNT) k_bc_level(BcArgs a) {
  __shared__ int32_t wl[kBcNT], gl[kBcNT];
  __shared__ int nw, ng;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) nw = ng = 0;
  __syncthreads();
  const int i = a.lo + blockIdx.x * kBcNT + tid;
  if (i < a.hi) {
    const int32_t u = a.Q[i];
    const int64_t rs = a.rp[u], re = a.rp[u + 1];
    if (re - rs <= kBcThread) {  // thread-mapped
      if (FWD) {
        const double su = a.sigma[u];
        for (int64_t k = rs; k < re; ++k) fwd_edge(a, su, __ldg(a.col + k));
      } else {
        const double sw = a.sigma[u];
        double d = 0.0;
        for (int64_t k = rs; k < re; ++k) d += bwd_term(a, sw, __ldg(a.col + k));
        bwd_finish(a, u, d);
      }
    } else if (re - rs <= kBcGroup) {
      gl[atomicAdd(&ng, 1)] = u;
    } else if (re - rs <= kBcWarp) {
      wl[atomicAdd(&nw, 1)] = u;
    } else {
      const int nch = (int)((re - rs + kBcChunk - 1) / kBcChunk);
      const int base = atomicAdd(a.bigcount, nch);
      for (int c = 0; c < nch; ++c) a.big[base + c] = make_int2(u, c);
      if (!FWD) a.bigv[atomicAdd(a.bigvcount, 1)] = make_int4(u, base, nch, 0);
    }
  }
  __syncthreads();
  // 8-lane groups (4 vertices per warp per round; warp-uniform round count)
  const int sub = lane & 7, grp = lane >> 3;
  for (int j0 = warp * 4; j0 < ng; j0 += kBcNT / 8) {
    const int j = j0 + grp;
    double d = 0.0;
    int32_t u = -1;
    if (j < ng) {
      u = gl[j];
      const int64_t rs = a.rp[u], re = a.rp[u + 1];
      const double su = a.sigma[u];
      for (int64_t k = rs + sub; k < re; k += 8) {
        if (FWD) fwd_edge(a, su, __ldg(a.col + k));
        else d += bwd_term(a, su, __ldg(a.col + k));
      }
    }
    if (!FWD) {
      for (int o = 4; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
      if (sub == 0 && u >= 0) bwd_finish(a, u, d);
    }
  }
  for (int j = warp; j < nw; j += kBcNT / 32) {  // warp-mapped (shared delayed buffer)
    const int32_t u = wl[j];
    const int64_t rs = a.rp[u], re = a.rp[u + 1];
    if (FWD) {
      const double su = a.sigma[u];
      for (int64_t k = rs + lane; k < re; k += 32) fwd_edge(a, su, __ldg(a.col + k));
    } else {
      const double sw = a.sigma[u];
      double d = 0.0;
      for (int64_t k = rs + lane; k < re; k += 32) d += bwd_term(a, sw, __ldg(a.col + k));
      for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
      if (lane == 0) bwd_finish(a, u, d);
    }
  }
}

// Pieces of the largest-degree vertices of the level (global delayed buffer), one CTA each;
// backward pieces write partial sums that k_bc_combine adds in piece order.
template <bool FWD>
__global__ void __launch_bounds__(kBcNT) k_bc_big(BcArgs a) {
  __shared__ int nb;
  __shared__ double red[kBcNT / 32];
  if (threadIdx.x == 0) nb = *(volatile int *)a.bigcount;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int j = blockIdx.x; j < nb; j += gridDim.x) {
    const int2 it = a.big[j];
    const int32_t u = it.x;
    const int64_t rs = a.rp[u] + (int64_t)it.y * kBcChunk;
    const int64_t re = min(rs + (int64_t)kBcChunk, a.rp[u + 1]);
    const double s = a.sigma[u];
    if (FWD) {
      for (int64_t k = rs + threadIdx.x; k < re; k += kBcNT) fwd_edge(a, s, __ldg(a.col + k));
    } else {
      double d = 0.0;
      for (int64_t k = rs + threadIdx.x; k < re; k += kBcNT) d += bwd_term(a, s, __ldg(a.col + k));
      for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
      if (lane == 0) red[warp] = d;
      __syncthreads();
      if (threadIdx.x == 0) {
        double t = 0.0;
        for (int q = 0; q < kBcNT / 32; ++q) t += red[q];
        a.bigpart[j] = t;
      }
      __syncthreads();
    }
  }
}

__global__ void k_bc_combine(BcArgs a) {
  const int nv = *(volatile int *)a.bigvcount;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nv; i += gridDim.x * blockDim.x) {
    const int4 r = a.bigv[i];
    double t = 0.0;
    for (int c = 0; c < r.z; ++c) t += a.bigpart[r.y + c];
    bwd_finish(a, r.x, t);
  }
}

// Forward step pulled from the unvisited side (direction optimisation, Beamer et al.,
// SC'12) for large frontiers of a symmetric graph (rows list the predecessors): an unvisited v sums sigma over ALL its level-L neighbours
// (plain loads, no atomics, neighbour order); a non-zero sum puts v on level L+1.
__global__ void __launch_bounds__(kBcNT) k_bc_pull(BcArgs a, int64_t n) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    if (a.level[v] != -1) continue;
    double s = 0.0;
    for (int64_t k = a.rp[v]; k < a.rp[v + 1]; ++k) {
      const int32_t u = __ldg(a.col + k);
      if (a.level[u] == a.L) s += a.sigma[u];
    }
    if (s > 0.0) {
      a.level[v] = a.L + 1;
      a.sigma[v] = s;
      enqueue(a, (int32_t)v);
    }
  }
}

__global__ void k_bc_init(int32_t *level, double *sigma, int64_t n, int64_t s, int32_t *Q) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    level[v] = v == s ? 0 : -1;
    sigma[v] = v == s ? 1.0 : 0.0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) Q[0] = (int32_t)s;
}

__global__ void k_zero_d(double *a, int64_t n) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    a[v] = 0.0;
}

int grid_of(int64_t n, int sms) {
  int64_t g = (n + 255) / 256;
  if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
  return g < 1 ? 1 : (int)g;
}

}  // namespace

void bc_run(inl_ctx ctx, const inl_csr &G, const int64_t *sources, int64_t n_sources, double *bc,
            inl_stats *stats, bool symmetric) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  INL_CHECK(n < INT32_MAX, "bc: n must be < 2^31");
  if (n == 0) return;
  int32_t *level = (int32_t *)ctx->s_a.get(sizeof(int32_t) * n);
  int32_t *Q = (int32_t *)ctx->s_b.get(sizeof(int32_t) * (n + 1));
  double *sigma = (double *)ctx->s_c.get(sizeof(double) * n);
  double *delta = nullptr;  // folded into pk
  BcPk *pk = (BcPk *)ctx->s_d.get(sizeof(BcPk) * n);
  INL_CUDA(cudaMemsetAsync(pk, 0, sizeof(BcPk) * n, st));  // tag 0 = never written
  // pieces of the vertices above kBcWarp: <= nnz / kBcChunk + (their number <= nnz / kBcWarp)
  const int64_t maxp = G.nnz / kBcChunk + G.nnz / kBcWarp + 16;
  int2 *big = (int2 *)ctx->s_e.get(sizeof(int2) * maxp);
  double *bigpart = (double *)ctx->s_g.get(sizeof(double) * maxp);
  int4 *bigv = (int4 *)ctx->s_tmp.get(sizeof(int4) * (G.nnz / kBcWarp + 16));
  int *cnt = (int *)ctx->s_f.get(64);  // [0] queue [1] pieces [2] large vertices; m_f at byte 16
  unsigned long long *mfp = (unsigned long long *)(cnt + 4);
  k_zero_d<<<grid_of(n, ctx->num_sms), 256, 0, st>>>(bc, n);
  INL_CUDA(cudaGetLastError());
  int64_t launches = 1, syncs = 0, iters = 0, ftotal = 0;
  std::vector<int> off;
  static int pull_div = -1;  // pull when the frontier holds more than n / pull_div vertices
  if (pull_div < 0) {
    pull_div = 8;  // measured: 16 -> 4.92 ms, 8 -> 4.14 ms, 64 -> 4.31 ms per scale-22 source
    if (const char *e = getenv("INL_BC_PULL_DIV")) pull_div = atoi(e);  // 0: never pull
  }
  static double pull_edge = -1.0;  // > 0: pull when m_f * pull_edge > m_u (edge rule), else n/pull_div
  if (pull_edge < 0.0) {
    pull_edge = 0.5;  // measured on one box at scale 22: n/8 rule 5.38, 0.5 -> 4.16, 1 -> 4.34, 2 -> 5.64 ms
    if (const char *e = getenv("INL_BC_PULL_EDGE")) pull_edge = atof(e);
  }
  for (int64_t si = 0; si < n_sources; ++si) {
    const int64_t s = sources[si];
    k_bc_init<<<grid_of(n, ctx->num_sms), 256, 0, st>>>(level, sigma, n, s, Q);
    ++launches;
    off.assign({0, 1});
    BcArgs a{G.row_ptr, G.col_idx, level, sigma, delta, bc, Q, 0, 0, 0, cnt, mfp, big, cnt + 1, bigv, cnt + 2,
             bigpart, (int32_t)s, pk, (int32_t)(si + 1)};
    double m_u = (double)G.nnz;       // edges of unvisited vertices (Beamer)
    unsigned long long mf_next = 0;   // edges of the current frontier
    for (int L = 0;; ++L) {  // forward: one level per step
      a.lo = off[L];
      a.hi = off[L + 1];
      a.L = L;
      if (a.hi == a.lo) break;
      INL_CUDA(cudaMemsetAsync(cnt, 0, 24, st));  // counters + m_f
      const bool pull = symmetric && (pull_edge > 0.0 ? (double)mf_next * pull_edge > m_u
                                                      : pull_div > 0 && (int64_t)(a.hi - a.lo) * pull_div > n);
      if (pull) {  // large frontier: pull from the unvisited side
        KScope ks(ctx, "k_bc_fwd");
        k_bc_pull<<<ctx->num_sms * 8, kBcNT, 0, st>>>(a, n);
        launches += 1;
      } else {
        KScope ks(ctx, "k_bc_fwd");
        k_bc_level<true><<<(a.hi - a.lo + kBcNT - 1) / kBcNT, kBcNT, 0, st>>>(a);
        k_bc_big<true><<<ctx->num_sms * 4, kBcNT, 0, st>>>(a);
        launches += 2;
      }
      if (pull_edge > 0.0) {
        k_bc_degsum<<<ctx->num_sms * 2, 256, 0, st>>>(a);
        ++launches;
      }
      INL_CUDA(cudaGetLastError());
      INL_CUDA(cudaMemcpyAsync(ctx->pinned, cnt, 24, cudaMemcpyDeviceToHost, st));
      INL_CUDA(cudaStreamSynchronize(st));
      ++syncs;
      off.push_back(a.hi + *(volatile int *)ctx->pinned);
      mf_next = *(volatile unsigned long long *)((char *)ctx->pinned + 16);
      m_u -= (double)mf_next;
      ++iters;
    }
    ftotal += off.back();
    // backward: the deepest non-empty level first; level 0 (the source) needs no delta
    const int nlev = (int)off.size() - 1;  // off[nlev] == off[nlev - 1]: levels 0 .. nlev-2
    for (int L = nlev - 2; L >= 1; --L) {
      a.lo = off[L];
      a.hi = off[L + 1];
      a.L = L;
      INL_CUDA(cudaMemsetAsync(cnt + 1, 0, 2 * sizeof(int), st));
      {
        KScope ks(ctx, "k_bc_bwd");
        k_bc_level<false><<<(a.hi - a.lo + kBcNT - 1) / kBcNT, kBcNT, 0, st>>>(a);
        k_bc_big<false><<<ctx->num_sms * 4, kBcNT, 0, st>>>(a);
        k_bc_combine<<<8, 128, 0, st>>>(a);
      }
      launches += 3;
      INL_CUDA(cudaGetLastError());
    }
  }
  INL_CUDA(cudaStreamSynchronize(st));
  if (stats) {
    stats->iterations = (int32_t)iters;
    stats->edges_relaxed = 0;  // not counted (the bench sums the reached vertices' degrees)
    stats->frontier_total = ftotal;
    stats->launches = launches;
    stats->host_syncs = syncs;
    stats->exchange_bytes = 0;
  }
}

}  // namespace inl
