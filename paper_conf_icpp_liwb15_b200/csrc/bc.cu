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

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "inl_internal.cuh"
#include "ptx.cuh"

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
  // heavy push levels: claims are plain level stores + a fire-and-forget bit in nbits (no
  // returning atomicCAS, no queue counter); k_bc_bits_to_q appends the level in vertex order
  uint32_t *nbits = nullptr;
};

// append v to level L+1 (one counter atomic per coalesced group)
__device__ __forceinline__ void enqueue(const BcArgs &a, int32_t v) {
  cg::coalesced_group g = cg::coalesced_threads();
  int pos = 0;
  if (g.thread_rank() == 0) pos = atomicAdd(a.qcount, (int)g.size());
  pos = g.shfl(pos, 0) + (int)g.thread_rank();
  a.Q[a.hi + pos] = v;
}

// the level claimed through nbits -> Q[hi, hi + count) in vertex order, count in *qcount (one
// counter atomic per warp)
__global__ void k_bc_bits_to_q(const uint32_t *__restrict__ nb, int64_t nwords, int32_t *Qn, int *qcount) {
  const int64_t nr = (nwords + 31) / 32 * 32;
  const int lane = threadIdx.x & 31;
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nr; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t b = w < nwords ? nb[w] : 0u;
    if (!__any_sync(0xffffffffu, b != 0u)) continue;
    const int c = __popc(b);
    int incl = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    int base = 0;
    if (lane == 31) base = atomicAdd(qcount, incl);
    int pos = __shfl_sync(0xffffffffu, base, 31) + incl - c;
    for (; b; b &= b - 1) Qn[pos++] = (int32_t)(w * 32 + __ffs(b) - 1);
  }
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
    if (a.nbits) {  // every discoverer stores the same level; the bitmap deduplicates
      a.level[v] = a.L + 1;
      red_or_b32(a.nbits + (v >> 5), 1u << (v & 31));
    } else {
      const int old = atomicCAS(a.level + v, -1, a.L + 1);
      if (old == -1) enqueue(a, v);
    }
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

// ---- the paper's templates (template study, Fig. 6 BC bars / Table II BC row) ----------
// Outer loop: the vertices Q[lo, hi) of one level; inner loop: their adjacency.  lbTHRES =
// bins.t_thread, CTA size = bins.cta; forward and backward use the same mapping.
//   T1 (INL_BINS_THREAD_ONLY): k_bct_thread over the whole level (thread-mapped, the
//     paper's baseline); dual-queue: k_bct_split -> k_bct_thread (small) + k_bct_block
//     (large); dbuf-global: k_bct_dbuf_global (defers large vertices to a global buffer) +
//     k_bct_block; dbuf-shared: k_bct_dbuf_shared (shared buffer, same CTA).
// Backward sums: thread-serial in edge order, block-mapped over a fixed CTA tree.

// one vertex, thread-mapped (serial inner loop)
template <bool FWD>
__device__ __forceinline__ void bct_serial(const BcArgs &a, int32_t u) {
  const int64_t rs = a.rp[u], re = a.rp[u + 1];
  const double su = a.sigma[u];
  if (FWD) {
    for (int64_t k = rs; k < re; ++k) fwd_edge(a, su, __ldg(a.col + k));
  } else {
    double d = 0.0;
    for (int64_t k = rs; k < re; ++k) d += bwd_term(a, su, __ldg(a.col + k));
    bwd_finish(a, u, d);
  }
}

// one vertex, block-mapped (threads stride the inner loop; backward: fixed CTA tree)
template <bool FWD>
__device__ __forceinline__ void bct_block(const BcArgs &a, int32_t u, double *red) {
  const int64_t rs = a.rp[u], re = a.rp[u + 1];
  const double su = a.sigma[u];
  if (FWD) {
    for (int64_t k = rs + threadIdx.x; k < re; k += blockDim.x) fwd_edge(a, su, __ldg(a.col + k));
    return;
  }
  double d = 0.0;
  for (int64_t k = rs + threadIdx.x; k < re; k += blockDim.x) d += bwd_term(a, su, __ldg(a.col + k));
  for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
  __syncthreads();  // red[] reuse
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = d;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int q = 0; q < (int)(blockDim.x >> 5); ++q) t += red[q];
    bwd_finish(a, u, t);
  }
}

// dual-queue pre-pass over the level: degree <= lbt -> small queue, else large queue
__global__ void k_bct_split(BcArgs a, int lbt, int32_t *qs, int *ns, int32_t *ql, int *nl) {
  for (int i = a.lo + blockIdx.x * blockDim.x + threadIdx.x; i < a.hi; i += gridDim.x * blockDim.x) {
    const int32_t u = a.Q[i];
    if (a.rp[u + 1] - a.rp[u] <= lbt) qs[atomicAdd(ns, 1)] = u;
    else ql[atomicAdd(nl, 1)] = u;
  }
}

// thread mapping over a queue (q == nullptr: the level itself)
template <bool FWD>
__global__ void k_bct_thread(BcArgs a, const int32_t *q, const int *nq) {
  const int n = q ? *nq : a.hi - a.lo;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    bct_serial<FWD>(a, q ? q[i] : a.Q[a.lo + i]);
}

// block mapping over a queue: one CTA per vertex, grid-stride (count read on the device)
template <bool FWD>
__global__ void k_bct_block(BcArgs a, const int32_t *q, const int *nq) {
  __shared__ double red[32];
  const int n = *(volatile const int *)nq;
  for (int i = blockIdx.x; i < n; i += gridDim.x) bct_block<FWD>(a, q[i], red);
}

// dbuf-global phase 1: thread per level vertex; large ones go to a global buffer
template <bool FWD>
__global__ void k_bct_dbuf_global(BcArgs a, int lbt, int32_t *buf, int *nbuf) {
  for (int i = a.lo + blockIdx.x * blockDim.x + threadIdx.x; i < a.hi; i += gridDim.x * blockDim.x) {
    const int32_t u = a.Q[i];
    if (a.rp[u + 1] - a.rp[u] <= lbt) bct_serial<FWD>(a, u);
    else buf[atomicAdd(nbuf, 1)] = u;
  }
}

// dbuf-shared: thread per level vertex; large ones queued in shared memory and run
// block-mapped by the same CTA after __syncthreads
template <bool FWD>
__global__ void k_bct_dbuf_shared(BcArgs a, int lbt) {
  extern __shared__ int32_t sbuf[];  // [blockDim.x]
  __shared__ int ns;
  __shared__ double red[32];
  for (int i0 = a.lo + blockIdx.x * blockDim.x; i0 < a.hi; i0 += gridDim.x * blockDim.x) {
    if (threadIdx.x == 0) ns = 0;
    __syncthreads();
    const int i = i0 + threadIdx.x;
    if (i < a.hi) {
      const int32_t u = a.Q[i];
      if (a.rp[u + 1] - a.rp[u] <= lbt) bct_serial<FWD>(a, u);
      else sbuf[atomicAdd(&ns, 1)] = u;
    }
    __syncthreads();
    const int m = ns;
    for (int j = 0; j < m; ++j) bct_block<FWD>(a, sbuf[j], red);
    __syncthreads();
  }
}

// ---- source-parallel BC (many sources): one CTA per source -------------------------------
// The paper's BC runs every source through grid-wide level steps (a launch pair and a host
// sync per level).  With many sources and a graph whose per-source state fits one SM, the
// sources themselves are the outer parallel loop: CTA c runs sources c, c + G, c + 2G, ...
// (static, so the result is deterministic), each with both sweeps inside the CTA
// (__syncthreads between levels, no launches, no host syncs).  The level's nested loop keeps
// the paper's binning inside the CTA (dbuf-shared, P5@3623): a thread per frontier vertex,
// degree > kSrcThread deferred to shared lists run by 8-lane groups (<= kSrcGroup) or warps.
// State per CTA — level int32, sigma f64, coef f64 ((1 + delta) / sigma of a finished
// vertex) — sits in shared memory when 20 B x n fits (SMEM), else in global slices
// (L2-resident for small n); the visit order Q and the level offsets are global; bc partial
// sums per CTA (bc_part[c][v], plain stores) are added in CTA order by k_bc_src_reduce.
constexpr int kSrcNT = 1024;
constexpr int kSrcThread = 4;
constexpr int kSrcGroup = 64;

struct SrcArgs {
  const int64_t *rp;
  const int32_t *col;
  int32_t n;
  const int32_t *sources;
  int32_t n_sources;
  int32_t *g_level;          // [G][n] (global state only)
  double *g_sigma, *g_coef;  // [G][n]
  int32_t *g_Q;              // [G][n]
  int32_t *g_off;            // [G][n + 2] level offsets into Q
  double *bc_part;           // [G][n]
  unsigned long long *levels;   // forward levels over all sources (stats)
  unsigned long long *reached;  // vertices reached over all sources (stats)
};

__device__ __forceinline__ void src_enqueue(int32_t *Q, int *tail, int32_t v) {
  cg::coalesced_group g = cg::coalesced_threads();
  int pos = 0;
  if (g.thread_rank() == 0) pos = atomicAdd(tail, (int)g.size());
  pos = g.shfl(pos, 0) + (int)g.thread_rank();
  Q[pos] = v;
}

// per-CTA state of one source's sweeps
struct SrcState {
  int32_t *level;
  double *sigma, *coef;
  int32_t *Q;
  int *tail;
  int L;
};

// forward edge u (level L, sigma su) -> v
__device__ __forceinline__ void src_fwd(const SrcState &S, double su, int32_t v) {
  int lv = ((volatile int32_t *)S.level)[v];
  if (lv == -1) {
    if (atomicCAS(S.level + v, -1, S.L + 1) == -1) src_enqueue(S.Q, S.tail, v);
    lv = S.L + 1;
  }
  if (lv == S.L + 1) atomicAdd(S.sigma + v, su);
}

// backward term of edge w -> v (sw = sigma[w]); S.L = level of w
__device__ __forceinline__ double src_bwd(const SrcState &S, double sw, int32_t v) {
  return S.level[v] == S.L + 1 ? sw * S.coef[v] : 0.0;
}

__device__ __forceinline__ void src_finish(const SrcState &S, double *part, int32_t w, double sw, double d) {
  S.coef[w] = (1.0 + d) / sw;
  part[w] += d;
}

// one level (forward: FWD) of the CTA's source over Q[lo, hi): thread / 8-lane group / warp
template <bool FWD>
__device__ __forceinline__ void src_level(const SrcArgs &a, const SrcState &S, double *part, int lo, int hi,
                                          int32_t *gl, int32_t *wl, int *ng, int *nw, int &ph) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int base = lo; base < hi; base += kSrcNT) {
    const int i = base + tid;
    if (i < hi) {
      const int32_t u = S.Q[i];
      const int64_t rs = a.rp[u], re = a.rp[u + 1];
      if (re - rs <= kSrcThread) {
        const double su = S.sigma[u];
        if (FWD) {
          for (int64_t k = rs; k < re; ++k) src_fwd(S, su, __ldg(a.col + k));
        } else {
          double d = 0.0;
          for (int64_t k = rs; k < re; ++k) d += src_bwd(S, su, __ldg(a.col + k));
          src_finish(S, part, u, su, d);
        }
      } else if (re - rs <= kSrcGroup) {
        gl[atomicAdd(&ng[ph], 1)] = u;
      } else {
        wl[atomicAdd(&nw[ph], 1)] = u;
      }
    }
    __syncthreads();
    const int mg = ng[ph], mw = nw[ph];
    if (tid == 0) ng[ph ^ 1] = nw[ph ^ 1] = 0;  // the other pair is reset for the next chunk
    const int sub = lane & 7, grp = lane >> 3;
    for (int j0 = warp * 4; j0 < mg; j0 += kSrcNT / 8) {  // 8-lane groups (warp-uniform rounds)
      const int j = j0 + grp;
      double d = 0.0, su = 0.0;
      int32_t u = -1;
      if (j < mg) {
        u = gl[j];
        su = S.sigma[u];
        for (int64_t k = a.rp[u] + sub; k < a.rp[u + 1]; k += 8) {
          if (FWD) src_fwd(S, su, __ldg(a.col + k));
          else d += src_bwd(S, su, __ldg(a.col + k));
        }
      }
      if (!FWD) {
        for (int o = 4; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
        if (sub == 0 && u >= 0) src_finish(S, part, u, su, d);
      }
    }
    for (int j = warp; j < mw; j += kSrcNT / 32) {  // warps
      const int32_t u = wl[j];
      const double su = S.sigma[u];
      double d = 0.0;
      for (int64_t k = a.rp[u] + lane; k < a.rp[u + 1]; k += 32) {
        if (FWD) src_fwd(S, su, __ldg(a.col + k));
        else d += src_bwd(S, su, __ldg(a.col + k));
      }
      if (!FWD) {
        for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
        if (lane == 0) src_finish(S, part, u, su, d);
      }
    }
    __syncthreads();
    ph ^= 1;
  }
}

template <bool SMEM>
__global__ void __launch_bounds__(kSrcNT, 1) k_bc_src(SrcArgs a) {
  extern __shared__ __align__(16) unsigned char sm[];
  __shared__ int32_t gl[kSrcNT], wl[kSrcNT];
  __shared__ int ng[2], nw[2], tail;  // list counters: ping-pong per chunk
  const int tid = threadIdx.x;
  const int n = a.n;
  const size_t c = blockIdx.x;
  SrcState S;
  if (SMEM) {
    S.sigma = (double *)sm;
    S.coef = S.sigma + n;
    S.level = (int32_t *)(S.coef + n);
  } else {
    S.level = a.g_level + c * n;
    S.sigma = a.g_sigma + c * n;
    S.coef = a.g_coef + c * n;
  }
  S.Q = a.g_Q + c * n;
  S.tail = &tail;
  int32_t *off = a.g_off + c * (size_t)(n + 2);
  double *part = a.bc_part + c * n;
  for (int v = tid; v < n; v += kSrcNT) part[v] = 0.0;
  unsigned long long nlev = 0, nreach = 0;
  int ph = 0;
  for (int si = blockIdx.x; si < a.n_sources; si += gridDim.x) {
    const int32_t s = a.sources[si];
    for (int v = tid; v < n; v += kSrcNT) {
      S.level[v] = v == s ? 0 : -1;
      S.sigma[v] = v == s ? 1.0 : 0.0;
    }
    if (tid == 0) {
      S.Q[0] = s;
      off[0] = 0;
      off[1] = 1;
      tail = 1;
      ng[0] = ng[1] = nw[0] = nw[1] = 0;
    }
    __syncthreads();
    int L = 0, lo = 0, hi = 1;
    while (lo < hi) {  // forward: level L = Q[lo, hi)
      S.L = L;
      src_level<true>(a, S, part, lo, hi, gl, wl, ng, nw, ph);
      lo = hi;
      hi = *(volatile int *)&tail;
      ++L;
      if (tid == 0) off[L + 1] = hi;
      __syncthreads();  // everyone has read tail before the next level appends
    }
    if (tid == 0) {
      nlev += L;
      nreach += lo;
    }
    // levels 0 .. L-1 are non-empty; backward from the deepest, level 0 (the source) skipped
    for (int l = L - 1; l >= 1; --l) {
      S.L = l;
      src_level<false>(a, S, part, off[l], off[l + 1], gl, wl, ng, nw, ph);
    }
    __syncthreads();
  }
  if (tid == 0 && nlev) {
    atomicAdd(a.levels, nlev);
    atomicAdd(a.reached, nreach);
  }
}

// bc[v] = sum over CTAs c (in order) of bc_part[c][v]
__global__ void k_bc_src_reduce(const double *__restrict__ part, int G, int64_t n, double *bc) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    double t = 0.0;
    for (int c = 0; c < G; ++c) t += part[(size_t)c * n + v];
    bc[v] = t;
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


// shared-memory bytes of one CTA's state (sigma, coef, level), 0 if it does not fit
size_t src_smem_bytes(inl_ctx ctx, int64_t n) {
  static int optin[kMaxDevices] = {};
  int &o = optin[ctx->device % kMaxDevices];
  if (!o) INL_CUDA(cudaDeviceGetAttribute(&o, cudaDevAttrMaxSharedMemoryPerBlockOptin, ctx->device));
  const size_t need = (size_t)n * 20;
  const size_t stat = 2 * sizeof(int32_t) * kSrcNT + 1024 + 64;  // k_bc_src static + reserved shared memory
  return need + stat <= (size_t)o ? need : 0;
}

// global scratch bytes per CTA of the source-parallel path
size_t src_global_bytes(int64_t n, bool smem) {
  return (size_t)n * (smem ? 16 : 36) + 8 * 2 + 16;
}

// Source-parallel when its modelled time beats the level-synchronous path's (INL_BC_MODE=
// level|src overrides).  Model fitted to profiles/r02/bc_mode_sweep.jsonl (B200, symmetric
// R-MAT 14..20 and the Wiki-vote-shaped graph): one source on one SM costs ~3.3 ns per CSR
// entry while the per-CTA state stays in L2 (~6 ns beyond), the sources run ceil(ns / G)
// deep; a level-synchronous source costs max(0.4 ms (launches + a host sync per level),
// 0.033 ns per entry).
bool bc_use_src(inl_ctx ctx, const inl_csr &G, int64_t n_sources) {
  const char *e = getenv("INL_BC_MODE");
  if (e && !strcmp(e, "level")) return false;
  const int64_t n = G.n_global;
  const int64_t Gc = std::min<int64_t>(n_sources, ctx->num_sms);
  const bool smem = src_smem_bytes(ctx, n) > 0;
  const double bytes = (double)Gc * (double)src_global_bytes(n, smem);
  const bool fits = n < INT32_MAX && n_sources < INT32_MAX && bytes <= 4.0e9;
  if (e && !strcmp(e, "src")) {
    INL_CHECK(fits, "INL_BC_MODE=src: the per-CTA state does not fit");
    return true;
  }
  if (!fits) return false;
  const double nnz = (double)G.nnz;
  const double per_edge = smem || bytes <= 64.0e6 ? 3.3e-9 : 6.0e-9;
  const double t_src = (double)((n_sources + Gc - 1) / Gc) * nnz * per_edge;
  const double t_level = (double)n_sources * std::max(0.4e-3, nnz * 0.033e-9);
  return t_src < t_level;
}

void bc_src_run(inl_ctx ctx, const inl_csr &G, const int64_t *sources, int64_t n_sources, double *bc,
                inl_stats *stats) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  const int Gc = (int)std::min<int64_t>(n_sources, ctx->num_sms);
  const size_t smem = src_smem_bytes(ctx, n);
  SrcArgs a{};
  a.rp = G.row_ptr;
  a.col = G.col_idx;
  a.n = (int32_t)n;
  a.n_sources = (int32_t)n_sources;
  std::vector<int32_t> hs((size_t)n_sources);
  for (int64_t i = 0; i < n_sources; ++i) hs[(size_t)i] = (int32_t)sources[i];
  int32_t *dsrc = (int32_t *)ctx->s_tmp.get(sizeof(int32_t) * n_sources);
  INL_CUDA(cudaMemcpyAsync(dsrc, hs.data(), sizeof(int32_t) * n_sources, cudaMemcpyHostToDevice, st));
  a.sources = dsrc;
  const size_t gn = (size_t)Gc * n;
  a.bc_part = (double *)ctx->s_a.get(sizeof(double) * gn);
  a.g_Q = (int32_t *)ctx->s_b.get(sizeof(int32_t) * gn);
  a.g_off = (int32_t *)ctx->s_c.get(sizeof(int32_t) * (size_t)Gc * (n + 2));
  if (!smem) {
    a.g_sigma = (double *)ctx->s_d.get(sizeof(double) * gn);
    a.g_coef = (double *)ctx->s_e.get(sizeof(double) * gn);
    a.g_level = (int32_t *)ctx->s_g.get(sizeof(int32_t) * gn);
  }
  unsigned long long *cnt = (unsigned long long *)ctx->s_f.get(64);
  a.levels = cnt;
  a.reached = cnt + 1;
  INL_CUDA(cudaMemsetAsync(cnt, 0, 16, st));
  static size_t configured[kMaxDevices] = {};
  size_t &cf = configured[ctx->device % kMaxDevices];
  if (smem > cf) {
    INL_CUDA(cudaFuncSetAttribute(k_bc_src<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    cf = smem;
  }
  {
    KScope ks(ctx, "k_bc_src");
    if (smem) k_bc_src<true><<<Gc, kSrcNT, smem, st>>>(a);
    else k_bc_src<false><<<Gc, kSrcNT, 0, st>>>(a);
    INL_CUDA(cudaGetLastError());
  }
  k_bc_src_reduce<<<grid_of(n, ctx->num_sms), 256, 0, st>>>(a.bc_part, Gc, n, bc);
  INL_CUDA(cudaGetLastError());
  INL_CUDA(cudaMemcpyAsync(ctx->pinned, cnt, 16, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  if (stats) {
    stats->iterations = (int32_t)((volatile unsigned long long *)ctx->pinned)[0];
    stats->edges_relaxed = 0;
    stats->frontier_total = (int64_t)((volatile unsigned long long *)ctx->pinned)[1];
    stats->launches = 2;
    stats->host_syncs = 0;
    stats->exchange_bytes = 0;
  }
}

}  // namespace

// fire-and-forget claims on heavy push levels (INL_BC_MARKS=0 keeps atomicCAS + queue pushes)
static bool bc_marks() {
  static int v = -1;
  if (v < 0) {
    const char *e = getenv("INL_BC_MARKS");
    v = e ? atoi(e) != 0 : 1;
  }
  return v == 1;
}

void bc_run(inl_ctx ctx, const inl_csr &G, const Bins &b, const int64_t *sources, int64_t n_sources, double *bc,
            inl_stats *stats, bool symmetric) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  INL_CHECK(n < INT32_MAX, "bc: n must be < 2^31");
  if (n == 0) return;
  const int tpl = b.flags & (INL_BINS_THREAD_ONLY | kTemplateFlags);
  if (!tpl && n_sources > 0 && bc_use_src(ctx, G, n_sources)) {
    bc_src_run(ctx, G, sources, n_sources, bc, stats);
    return;
  }
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
  const int64_t nwb = (n + 31) / 32;
  uint32_t *nbits = (uint32_t *)ctx->s_bcb.get(sizeof(uint32_t) * (nwb + 1));
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
  // the paper's templates / T1 baseline (bins flags): plain push levels, no pull
  if (tpl) symmetric = false;
  int32_t *tq = tpl == INL_BINS_TPL_DUAL_QUEUE || tpl == INL_BINS_TPL_DBUF_GLOBAL
                    ? (int32_t *)ctx->s_h.get(sizeof(int32_t) * 2 * n) : nullptr;
  // one level of either sweep through the template; returns the launches
  auto tpl_level = [&](const BcArgs &a, bool fwd) -> int {
    const int m = a.hi - a.lo, cta = b.cta, lbt = b.t_thread, sms = ctx->num_sms;
    int g = (m + cta - 1) / cta;
    if (g > sms * 32) g = sms * 32;
    int *tc = cnt + 8;  // template queue counters
    if (tpl == INL_BINS_THREAD_ONLY) {
      if (fwd) k_bct_thread<true><<<g, cta, 0, st>>>(a, nullptr, nullptr);
      else k_bct_thread<false><<<g, cta, 0, st>>>(a, nullptr, nullptr);
      return 1;
    }
    if (tpl == INL_BINS_TPL_DBUF_SHARED) {
      if (fwd) k_bct_dbuf_shared<true><<<g, cta, sizeof(int32_t) * cta, st>>>(a, lbt);
      else k_bct_dbuf_shared<false><<<g, cta, sizeof(int32_t) * cta, st>>>(a, lbt);
      return 1;
    }
    INL_CUDA(cudaMemsetAsync(tc, 0, 2 * sizeof(int), st));
    if (tpl == INL_BINS_TPL_DUAL_QUEUE) {
      int gs = (m + 255) / 256;
      if (gs > sms * 16) gs = sms * 16;
      k_bct_split<<<gs, 256, 0, st>>>(a, lbt, tq, tc, tq + n, tc + 1);
      if (fwd) {
        k_bct_thread<true><<<g, cta, 0, st>>>(a, tq, tc);
        k_bct_block<true><<<sms * 16, cta, 0, st>>>(a, tq + n, tc + 1);
      } else {
        k_bct_thread<false><<<g, cta, 0, st>>>(a, tq, tc);
        k_bct_block<false><<<sms * 16, cta, 0, st>>>(a, tq + n, tc + 1);
      }
      return 3;
    }
    if (fwd) {
      k_bct_dbuf_global<true><<<g, cta, 0, st>>>(a, lbt, tq, tc);
      k_bct_block<true><<<sms * 16, cta, 0, st>>>(a, tq, tc);
    } else {
      k_bct_dbuf_global<false><<<g, cta, 0, st>>>(a, lbt, tq, tc);
      k_bct_block<false><<<sms * 16, cta, 0, st>>>(a, tq, tc);
    }
    return 2;
  };
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
      if (tpl) {
        KScope ks(ctx, "k_bc_fwd");
        launches += tpl_level(a, true);
      } else if (pull) {  // large frontier: pull from the unvisited side
        KScope ks(ctx, "k_bc_fwd");
        k_bc_pull<<<ctx->num_sms * 8, kBcNT, 0, st>>>(a, n);
        launches += 1;
      } else {
        KScope ks(ctx, "k_bc_fwd");
        // heavy push level (frontier edges > nnz / 256): fire-and-forget claims, see BcArgs::nbits
        const bool marks = bc_marks() && (double)mf_next * 256.0 > (double)G.nnz;
        if (marks) {
          a.nbits = nbits;
          INL_CUDA(cudaMemsetAsync(nbits, 0, sizeof(uint32_t) * nwb, st));
        }
        k_bc_level<true><<<(a.hi - a.lo + kBcNT - 1) / kBcNT, kBcNT, 0, st>>>(a);
        k_bc_big<true><<<ctx->num_sms * 4, kBcNT, 0, st>>>(a);
        launches += 2;
        if (marks) {
          k_bc_bits_to_q<<<grid_of(nwb, ctx->num_sms), 256, 0, st>>>(nbits, nwb, Q + a.hi, cnt);
          ++launches;
          a.nbits = nullptr;
        }
      }
      if (pull_edge > 0.0 && !tpl) {
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
      if (tpl) {
        KScope ks(ctx, "k_bc_bwd");
        launches += tpl_level(a, false);
        INL_CUDA(cudaGetLastError());
        continue;
      }
      INL_CUDA(cudaMemsetAsync(cnt + 1, 0, 2 * sizeof(int), st));
      {
        KScope ks(ctx, "k_bc_bwd");
        k_bc_level<false><<<(a.hi - a.lo + kBcNT - 1) / kBcNT, kBcNT, 0, st>>>(a);
        k_bc_big<false><<<ctx->num_sms * 4, kBcNT, 0, st>>>(a);
        k_bc_combine<<<ctx->num_sms * 4, 128, 0, st>>>(a);  // one thread per large vertex (8 CTAs: 256 us at scale 22)
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
