// frontier.cu — SSSP (PAPER.md P5@10241, P11@2218) and BFS (P5@11591) as a
// frontier worklist over the CSR, load-balanced with the paper's delayed-buffer
// templates:
//   * k_expand: one thread per frontier vertex (thread-mapped outer loop).  A
//     vertex with degree <= t_thread runs its inner loop serially in that lane;
//     larger ones are deferred to a shared-memory buffer and processed, after
//     __syncthreads, warp-mapped (<= t_warp) or block-mapped (<= t_block) by the
//     same CTA (dbuf-shared, P5@3623); the largest are appended as grid_chunk
//     chunks to a global buffer (dbuf-global, P5@2721) that k_expand_grid
//     processes with one CTA per chunk.
//   * SSSP relaxation: nd = dist[u] + w; atomicMin(&dist[v], nd); an improved v
//     is claimed once per iteration (iteration stamp) and enqueued with one
//     atomicAdd per coalesced group.  The asynchronous (single-array) variant
//     converges to the same unique distances (reading R4).
//   * BFS claim: atomicOr on a visited bitmap (8.4 MB at scale 26, L2-resident);
//     the winner writes level[v] = L + 1 and enqueues v.
//   * P > 1 ranks (row blocks): synchronous rounds; SSSP allreduce-min of dist,
//     BFS allreduce-max of an n-byte next-frontier map, each with a
//     trailing termination word.
#include <cooperative_groups.h>
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <cstdlib>

#include <cub/block/block_scan.cuh>
#include <cub/device/device_partition.cuh>
#include <cub/device/device_select.cuh>
#include <thrust/iterator/discard_iterator.h>
#include <thrust/iterator/counting_iterator.h>

#include "comm.h"
#include "inl_internal.cuh"
#include "ptx.cuh"

namespace cg = cooperative_groups;

namespace inl {

namespace {

constexpr int NT = 256;
constexpr int NW = NT / 32;
// resident CTAs per SM the expansion kernels are compiled for (register cap 65536 / (NT * it)):
// 4 (64 registers, 32 warps / SM) measured best with the bitmap SSSP loop (scale 23: 4.94 ->
// 4.48 ms per source; 3: 4.62, 5 and 6 spill: 4.90 / 5.43) and neutral for BFS
// (profiles/r02/sssp_bitmap_sweeps.txt)
#ifndef INL_EXPAND_MINB
#define INL_EXPAND_MINB 4
#endif

__device__ __forceinline__ void push(int32_t *q, int *cnt, int32_t v) {
  cg::coalesced_group g = cg::coalesced_threads();
  int pos = 0;
  if (g.thread_rank() == 0) pos = atomicAdd(cnt, (int)g.size());
  pos = g.shfl(pos, 0) + (int)g.thread_rank();
  q[pos] = v;
}

// Warp-aggregated enqueue of the slots of m (bit j: v[j]) — one counter atomic per warp.
// All 32 lanes must call it (warp-uniform control flow).
template <int K>
__device__ __forceinline__ void push_batch(int32_t *q, int *cnt, const int32_t (&v)[K], unsigned m) {
  if (!__any_sync(0xffffffffu, m != 0u)) return;
  const int lane = threadIdx.x & 31;
  const int c = __popc(m);
  int incl = c;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int t = __shfl_up_sync(0xffffffffu, incl, d);
    if (lane >= d) incl += t;
  }
  int base = 0;
  if (lane == 31) base = atomicAdd(cnt, incl);
  int pos = __shfl_sync(0xffffffffu, base, 31) + incl - c;
#pragma unroll
  for (int j = 0; j < K; ++j)
    if ((m >> j) & 1u) q[pos++] = v[j];
}

struct SsspOp {
  uint32_t *dist;       // [n_global (+1 flag word on P > 1)]
  const uint32_t *w;    // [nnz]
  uint32_t *inq;        // !DIST: bitmap "already in the next frontier", cleared per iteration
  uint32_t *flag;       // P > 1: dist[n] cleared on any improvement
  int iter;
  int64_t row_begin;
  bool enqueue;         // !DIST: enqueue improved vertices directly
  uint64_t pol_stream;  // L2 evict-first for the edge stream
  uint32_t thr;         // near-far: vertices reaching dist >= thr go to the far pile
  int32_t *far;         // far pile (each vertex at most once: `infar` bitmap)
  int *far_count;
  uint32_t *infar;
  // NEXT-1 sparse exchange (DIST): vertex v's distance is OWNED by rank q = v / B; a
  // relaxation that beats this rank's (stale, upper-bound) copy dist[v] does atomicMin in the
  // owner's array (peer memory) and, if that improved it, sets v's bit in the owner's
  // changed-bitmap of the round; nimp counts those improvements (summed by the one allreduce
  // per round, which is also the barrier and the termination test)
  uint32_t *const *xd = nullptr;   // [P] owners' distance arrays (xd[rank] == dist)
  uint32_t *const *xc = nullptr;   // [P] owners' changed bitmaps of this round
  int64_t B = 0;
  unsigned int *nimp = nullptr;
  unsigned long long *xops = nullptr;  // remote atomics issued (the exchange volume)
  // bitmap frontier (the one-GPU graph loop): an improvement is a fire-and-forget atomicMin
  // plus a fire-and-forget bit in the next-frontier (nbits) or far (fbits) bitmap — no
  // queue counter, no atomic whose result a warp waits for; k_sssp_bcompact turns the bits
  // into the next step's worklist.  A lost race only adds a vertex to the frontier (it is
  // expanded with its true distance then), never loses an improvement.
  uint32_t *nbits = nullptr;
  uint32_t *fbits = nullptr;
  unsigned long long *tmark = nullptr;  // INL_SSSP_TRACE only: improvements marked
  __device__ __forceinline__ void mark(int32_t v, uint32_t nd) const {
    red_min_u32(dist + v, nd);
    red_or_b32((nd >= thr ? fbits : nbits) + (v >> 5), 1u << (v & 31));
  }
  __device__ __forceinline__ bool xrelax(int32_t v, uint32_t nd) const {
    uint32_t *o = xd[v / B];
    if (o != dist) atomicMin(dist + v, nd);  // keep the local filter tight
    if (atomicMin(o + v, nd) <= nd) return false;
    atomicOr(xc[v / B] + (v >> 5), 1u << (v & 31));
    return true;
  }
  __device__ __forceinline__ uint32_t load(int32_t u) const {
    return *(volatile uint32_t *)(dist + row_begin + u);
  }
  __device__ __forceinline__ void fence() const {
    if (xd) __threadfence_system();  // the owners read these after the round's allreduce
  }
  __device__ __forceinline__ void improve(int32_t v, uint32_t nd, int32_t *q, int *cnt) const {
    if (xd) {
      const bool r = xd[v / B] != dist;
      const bool imp = xrelax(v, nd);
      if (imp) atomicAdd(nimp, 1u);
      if (r) atomicAdd(xops, imp ? 2ull : 1ull);
      return;
    }
    if (nbits) {
      mark(v, nd);
      return;
    }
    const uint32_t old = atomicMin(dist + v, nd);
    if (nd < old) {
      if (enqueue) {
        const uint32_t bit = 1u << (v & 31);
        if (nd >= thr) {
          if (!(atomicOr(infar + (v >> 5), bit) & bit)) push(far, far_count, v);
        } else {
          if (!(atomicOr(inq + (v >> 5), bit) & bit)) push(q, cnt, v);
        }
      } else {
        *flag = 0u;
      }
    }
  }
  __device__ __forceinline__ void edge(uint32_t du, int64_t k, int32_t v, int32_t *q, int *cnt) const {
    const uint32_t nd = du + __ldg(w + k);
    if (nd < dist[v]) improve(v, nd, q, cnt);
  }
  // K edges per lane at once, every stage issued back to back so the latencies overlap
  // (memory-level parallelism K): weight loads, dist gathers, atomicMin of the candidate
  // improvements, claim bits of the improved vertices, one warp-aggregated enqueue.
  // Out-of-range slots have in[j] = false.  All 32 lanes must call it.
  template <int K>
  __device__ __forceinline__ void edges(const uint32_t (&du)[K], const int64_t (&kk)[K], const int32_t (&vv)[K],
                                        const bool (&in)[K], int32_t *q, int *cnt) const {
    uint32_t nd[K], dv[K], old[K];
#pragma unroll
    for (int j = 0; j < K; ++j) nd[j] = in[j] ? du[j] + ld_stream_pol(w + kk[j], pol_stream) : 0xFFFFFFFFu;
#pragma unroll
    for (int j = 0; j < K; ++j) dv[j] = in[j] ? dist[vv[j]] : 0u;
    if (xd) {  // NEXT-1: improvements go to the owners
      unsigned c = 0, rem = 0;
#pragma unroll
      for (int j = 0; j < K; ++j)
        if (nd[j] < dv[j]) {
          const bool r = xd[vv[j] / B] != dist;
          const bool imp = xrelax(vv[j], nd[j]);
          c += imp;
          rem += r ? 1u + (imp ? 1u : 0u) : 0u;  // the remote atomicMin (+ the changed bit)
        }
      for (int o = 16; o > 0; o >>= 1) {
        c += __shfl_xor_sync(0xffffffffu, c, o);
        rem += __shfl_xor_sync(0xffffffffu, rem, o);
      }
      if ((threadIdx.x & 31) == 0) {
        if (c) atomicAdd(nimp, c);
        if (rem) atomicAdd(xops, (unsigned long long)rem);
      }
      return;
    }
    if (nbits) {
      unsigned m = 0;
#pragma unroll
      for (int j = 0; j < K; ++j)
        if (nd[j] < dv[j]) {
          mark(vv[j], nd[j]);
          ++m;
        }
      if (tmark) {
        m = __reduce_add_sync(0xffffffffu, m);
        if ((threadIdx.x & 31) == 0 && m) atomicAdd(tmark, (unsigned long long)m);
      }
      return;
    }
#pragma unroll
    for (int j = 0; j < K; ++j) old[j] = nd[j] < dv[j] ? atomicMin(dist + vv[j], nd[j]) : 0u;
    unsigned imp = 0u;
#pragma unroll
    for (int j = 0; j < K; ++j)
      if (nd[j] < dv[j] && nd[j] < old[j]) imp |= 1u << j;
    if (!enqueue) {
      if (imp) *flag = 0u;
      return;
    }
    uint32_t ob[K];
#pragma unroll
    for (int j = 0; j < K; ++j)
      ob[j] = (imp >> j) & 1u ? atomicOr((nd[j] >= thr ? infar : inq) + (vv[j] >> 5), 1u << (vv[j] & 31)) : 0u;
    unsigned nearm = 0u, farm = 0u;
#pragma unroll
    for (int j = 0; j < K; ++j)
      if (((imp >> j) & 1u) && !((ob[j] >> (vv[j] & 31)) & 1u)) {
        if (nd[j] >= thr) farm |= 1u << j;
        else nearm |= 1u << j;
      }
    push_batch(q, cnt, vv, nearm);
    push_batch(far, far_count, vv, farm);
  }
};

struct BfsOp {
  uint32_t *bitmap;  // visited, [ceil(n/32)]
  int32_t *level;    // [n_global]
  uint8_t *next;     // P > 1: n-byte next map (+ flag byte at [n])
  int64_t n;
  int L;
  bool enqueue;      // !DIST
  uint64_t pol_stream;
  const int64_t *rp = nullptr;       // !DIST: degree sum of the next frontier -> *mf
  unsigned long long *mf = nullptr;  //   (Beamer's m_f, for the direction switch)
  // NEXT-1 fused exchange (DIST): a discovered vertex v sets its bit in the next-frontier
  // bitmap of its OWNER q = v / B, in q's memory (NVLink peer memory; the same device for the
  // loopback), during the expansion itself — no byte map, no allreduce
  // one-GPU top-down with fire-and-forget marks: a candidate sets its visited bit and its bit
  // in nbits (the next frontier) with red.or and stores level L+1 (every discoverer stores the
  // same value) — no returning atomicOr, no queue push; k_bfs_next_queue builds the queue and
  // m_f from nbits afterwards
  uint32_t *nbits = nullptr;
  uint32_t *const *xtab = nullptr;   // [P] owners' bitmaps of this level
  int64_t B = 0;                     // row block
  const uint32_t *xself = nullptr;   // this rank's own bitmap (local sets are not exchange)
  unsigned long long *xops = nullptr;  // remote atomics issued
  __device__ __forceinline__ void xset(int32_t v) const {
    atomicOr(xtab[v / B] + (v >> 5), 1u << (v & 31));
  }
  __device__ __forceinline__ void fence() const {
    if (xtab) __threadfence_system();  // the peers read these bits after the barrier
  }
  __device__ __forceinline__ uint32_t load(int32_t) const { return 0u; }
  __device__ __forceinline__ void visit(int32_t v, int32_t *q, int *cnt) const {
    if (!enqueue && xtab) {
      xset(v);
      if (xtab[v / B] != xself) atomicAdd(xops, 1ull);
    } else if (enqueue) {
      const uint32_t bit = 1u << (v & 31);
      const uint32_t old = atomicOr(bitmap + (v >> 5), bit);
      if (!(old & bit)) {
        level[v] = L + 1;
        if (mf) atomicAdd(mf, (unsigned long long)(rp[v + 1] - rp[v]));
        push(q, cnt, v);
      }
    } else {
      next[v] = 1;
      next[n] = 1;
    }
  }
  __device__ __forceinline__ void edge(uint32_t, int64_t, int32_t v, int32_t *q, int *cnt) const {
    const uint32_t bit = 1u << (v & 31);
    if (!(bitmap[v >> 5] & bit)) visit(v, q, cnt);
  }
  // K edges per lane at once (see SsspOp::edges); all 32 lanes must call it.
  template <int K>
  __device__ __forceinline__ void edges(const uint32_t (&)[K], const int64_t (&)[K], const int32_t (&vv)[K],
                                        const bool (&in)[K], int32_t *q, int *cnt) const {
    uint32_t bw[K];
#pragma unroll
    for (int j = 0; j < K; ++j) bw[j] = in[j] ? bitmap[vv[j] >> 5] : 0xFFFFFFFFu;
    unsigned cand = 0u;
#pragma unroll
    for (int j = 0; j < K; ++j)
      if (!((bw[j] >> (vv[j] & 31)) & 1u)) cand |= 1u << j;
    if (nbits) {
#pragma unroll
      for (int j = 0; j < K; ++j)
        if ((cand >> j) & 1u) {
          const uint32_t bit = 1u << (vv[j] & 31);
          red_or_b32(bitmap + (vv[j] >> 5), bit);
          red_or_b32(nbits + (vv[j] >> 5), bit);
          level[vv[j]] = L + 1;
        }
      return;
    }
    if (!enqueue) {
      if (xtab) {
        unsigned rem = 0;
#pragma unroll
        for (int j = 0; j < K; ++j)
          if ((cand >> j) & 1u) {
            xset(vv[j]);
            rem += xtab[vv[j] / B] != xself;
          }
        for (int o = 16; o > 0; o >>= 1) rem += __shfl_xor_sync(0xffffffffu, rem, o);
        if ((threadIdx.x & 31) == 0 && rem) atomicAdd(xops, (unsigned long long)rem);
        return;
      }
#pragma unroll
      for (int j = 0; j < K; ++j)
        if ((cand >> j) & 1u) next[vv[j]] = 1;
      if (cand) next[n] = 1;
      return;
    }
#pragma unroll
    for (int j = 0; j < K; ++j)
      bw[j] = (cand >> j) & 1u ? atomicOr(bitmap + (vv[j] >> 5), 1u << (vv[j] & 31)) : 0xFFFFFFFFu;
    unsigned won = 0u;
#pragma unroll
    for (int j = 0; j < K; ++j)
      if (((cand >> j) & 1u) && !((bw[j] >> (vv[j] & 31)) & 1u)) {
        won |= 1u << j;
        level[vv[j]] = L + 1;
      }
    if (mf) {  // degree sum of the claimed vertices (one atomic per warp)
      unsigned long long dsum = 0;
#pragma unroll
      for (int j = 0; j < K; ++j)
        if ((won >> j) & 1u) dsum += (unsigned long long)(rp[vv[j] + 1] - rp[vv[j]]);
      for (int o = 16; o > 0; o >>= 1) dsum += __shfl_xor_sync(0xffffffffu, dsum, o);
      if ((threadIdx.x & 31) == 0 && dsum) atomicAdd(mf, dsum);
    }
    push_batch(q, cnt, vv, won);
  }
};

// Device-driven near-far SSSP (one GPU): the loop state lives on the device, so the
// host enqueues several steps (split, expand, grid expand, post) per round trip.
struct __align__(16) SsspDev {
  int nF;       // input frontier size of this step (0: the step starts with a far split)
  int cnt;      // next-frontier counter
  int gcount;   // grid-bin chunk counter
  int nsplit;   // near vertices the split moved into the frontier
  int nfar, nfar2;  // far pile sizes (current, split output + this step's far pushes)
  int par, fpar;    // frontier / far buffer parity
  int iter, done;
  uint32_t thr, delta;
  int slice;    // dynamic slice counter of k_expand_flat
  int pad;      // steps run (k_sssp_post); done = 2 if it ever exceeds kSsspMaxSteps
  unsigned long long ftotal;
};
struct SsspDyn {
  SsspDev *s;  // nullptr: static (host-driven) launch
  int32_t *buf[2];
  int32_t *far[2];
  uint32_t *inq[2];  // claim bitmaps of even / odd iterations (bitmap mode: frontier C / next N by par)
  uint32_t *keep;    // in-far-pile bitmap (bitmap mode: the far pile itself)
  bool bits;         // bitmap frontier (k_sssp_bcompact / k_sssp_bsplit / k_sssp_bpost)
  int64_t nwords4;   // bitmap mode: words per bitmap, a multiple of 4 (uint4 scans)
};

// element i & 1 of a two-entry array held in a kernel parameter, without indexing it: a
// run-time index forces the whole parameter struct into a per-thread stack copy (~200 B of
// local stores per thread at kernel entry, ~10 us per launch of an otherwise idle grid)
template <class T>
__device__ __forceinline__ T pick2(T const (&v)[2], int i) { return (i & 1) ? v[1] : v[0]; }

__device__ __forceinline__ uint32_t sat_add(uint32_t a, uint32_t b) { return a > 0xFFFFFFFFu - b ? 0xFFFFFFFFu : a + b; }

struct ExpandArgs {
  const int32_t *F;  // frontier (local row ids)
  int nF;
  const int64_t *rp;
  const int32_t *col;
  int t_thread, t_warp, t_block, chunk;
  int2 *gitems;  // grid-bin chunk buffer [gcap]
  int *gcount;
  int gcap;      // its capacity (frontier_cfg: an upper bound of what one expansion emits)
  int *oflow;    // set if an expansion ever needed more (-> INL_ERR_INTERNAL; never expected)
  int32_t *Fout;
  int *fcount;
  unsigned long long *relaxed;
  SsspDyn dyn;
};

// The step state, read once per CTA (4 lanes, 16-B L2 loads) into shared memory: every
// thread reading it from global memory would hammer one L2 slice.
__device__ __forceinline__ void load_state(const SsspDev *g, SsspDev *sh) {
  if (threadIdx.x < (int)(sizeof(SsspDev) / 16))
    reinterpret_cast<int4 *>(sh)[threadIdx.x] = __ldcg(reinterpret_cast<const int4 *>(g) + threadIdx.x);
  __syncthreads();
}

// Dynamic launches read this step's frontier / far-pile / claim-bitmap roles from the
// device state; returns false when the step has nothing to expand.
template <class Op>
__device__ __forceinline__ bool dyn_bind(ExpandArgs &a, Op &op, uint32_t **inq_prev) {
  *inq_prev = nullptr;
  return true;
}
template <>
__device__ __forceinline__ bool dyn_bind<SsspOp>(ExpandArgs &a, SsspOp &op, uint32_t **inq_prev) {
  *inq_prev = nullptr;
  if (!a.dyn.s) return true;
  __shared__ __align__(16) SsspDev st_s;
  load_state(a.dyn.s, &st_s);
  const SsspDev &s = st_s;
  if (s.done) return false;
  const bool split = s.nF == 0;
  const int nF = split ? s.nsplit : s.nF;
  if (nF == 0) return false;
  if (a.dyn.bits) {  // worklist built by k_sssp_bcompact (or the split) in buf[0]
    a.nF = nF;
    a.F = a.dyn.buf[0];
    a.gcount = &a.dyn.s->gcount;
    op.thr = split ? sat_add(s.thr, s.delta) : s.thr;
    op.nbits = pick2(a.dyn.inq, s.par ^ 1);
    op.fbits = a.dyn.keep;
    return true;
  }
  const int par = s.par, fpar = s.fpar, it = s.iter;
  a.nF = nF;
  a.F = pick2(a.dyn.buf, par);
  a.Fout = pick2(a.dyn.buf, par ^ 1);
  a.fcount = &a.dyn.s->cnt;
  a.gcount = &a.dyn.s->gcount;
  op.thr = split ? sat_add(s.thr, s.delta) : s.thr;
  op.inq = pick2(a.dyn.inq, it & 1);
  op.far = pick2(a.dyn.far, split ? fpar ^ 1 : fpar);
  op.far_count = split ? &a.dyn.s->nfar2 : &a.dyn.s->nfar;
  op.infar = a.dyn.keep;
  *inq_prev = pick2(a.dyn.inq, (it & 1) ^ 1);
  return true;
}

// The bitmap graph loop's relaxation alone (SsspOp::edges minus the NEXT-1 and worklist
// paths): the expansion kernels instantiated for it carry no registers for the paths they never
// take (64 registers without spills at 4 resident CTAs / SM; SsspOp spills ~200 B there).
struct SsspBitsOp : SsspOp {
  template <int K>
  __device__ __forceinline__ void edges(const uint32_t (&du)[K], const int64_t (&kk)[K], const int32_t (&vv)[K],
                                        const bool (&in)[K], int32_t *, int *) const {
    uint32_t nd[K], dv[K];
#pragma unroll
    for (int j = 0; j < K; ++j) nd[j] = in[j] ? du[j] + ld_stream_pol(w + kk[j], pol_stream) : 0xFFFFFFFFu;
#pragma unroll
    for (int j = 0; j < K; ++j) dv[j] = in[j] ? dist[vv[j]] : 0u;
    unsigned m = 0;
#pragma unroll
    for (int j = 0; j < K; ++j)
      if (nd[j] < dv[j]) {
        mark(vv[j], nd[j]);
        ++m;
      }
    if (tmark) {
      m = __reduce_add_sync(0xffffffffu, m);
      if ((threadIdx.x & 31) == 0 && m) atomicAdd(tmark, (unsigned long long)m);
    }
  }
};
template <>
__device__ __forceinline__ bool dyn_bind<SsspBitsOp>(ExpandArgs &a, SsspBitsOp &op, uint32_t **inq_prev) {
  *inq_prev = nullptr;
  __shared__ __align__(16) SsspDev st_s;
  load_state(a.dyn.s, &st_s);
  const SsspDev &s = st_s;
  if (s.done) return false;
  const bool split = s.nF == 0;
  const int nF = split ? s.nsplit : s.nF;
  if (nF == 0) return false;
  a.nF = nF;  // worklist built by k_sssp_bcompact (or the split) in buf[0]
  a.F = a.dyn.buf[0];
  a.gcount = &a.dyn.s->gcount;
  op.thr = split ? sat_add(s.thr, s.delta) : s.thr;
  op.nbits = pick2(a.dyn.inq, s.par ^ 1);
  op.fbits = a.dyn.keep;
  return true;
}

// ---- the paper's dual-queue template on the frontier (Fig. 1(b), P5@2074): a pre-pass
// "divides the elements processed in the outer loop in two queues depending on the number of
// iterations they require in the inner-loop and processes those queues separately using thread-
// and block-based mapping" — k_dq_split, then k_dq_thread over the small queue (one thread per
// vertex, serial inner loop) and k_dq_block over the large one (one CTA per vertex).  Queue
// sizes are read on the device (no host round trip).
__global__ void k_dq_split(const int32_t *__restrict__ F, int nF, const int64_t *__restrict__ rp, int lbt,
                           int32_t *qs, int *ns, int32_t *ql, int *nl, unsigned long long *relaxed) {
  unsigned long long dsum = 0;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nF; i += gridDim.x * blockDim.x) {
    const int32_t u = F[i];
    const int64_t d = rp[u + 1] - rp[u];
    dsum += (unsigned long long)d;
    if (d <= lbt) push(qs, ns, u);
    else push(ql, nl, u);
  }
  for (int o = 16; o > 0; o >>= 1) dsum += __shfl_xor_sync(0xffffffffu, dsum, o);
  if ((threadIdx.x & 31) == 0 && dsum) atomicAdd(relaxed, dsum);
}

template <class Op>
__global__ void __launch_bounds__(NT) k_dq_thread(const int32_t *__restrict__ q, const int *__restrict__ nq,
                                                  const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                                                  Op op, int32_t *Fout, int *fcount) {
  op.pol_stream = policy_evict_first();
  const int n = __ldcg(nq);
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int32_t u = q[i];
    const uint32_t su = op.load(u);
    for (int64_t k = rp[u]; k < rp[u + 1]; ++k) op.edge(su, k, __ldg(col + k), Fout, fcount);
  }
  op.fence();
}

template <class Op>
__global__ void __launch_bounds__(NT) k_dq_block(const int32_t *__restrict__ q, const int *__restrict__ nq,
                                                 const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                                                 Op op, int32_t *Fout, int *fcount) {
  op.pol_stream = policy_evict_first();
  __shared__ int n_s;
  if (threadIdx.x == 0) n_s = __ldcg(nq);
  __syncthreads();
  for (int j = blockIdx.x; j < n_s; j += gridDim.x) {
    const int32_t u = q[j];
    const uint32_t su = op.load(u);
    for (int64_t k = rp[u] + threadIdx.x; k < rp[u + 1]; k += NT) op.edge(su, k, __ldg(col + k), Fout, fcount);
  }
  op.fence();
}

// Append the ceil(d / chunk) pieces of frontier vertex u to the grid buffer.  The buffer
// holds gcap pieces, an upper bound of one expansion's output (frontier_cfg); a write past
// it is dropped and flagged instead (the host turns the flag into INL_ERR_INTERNAL).
__device__ __forceinline__ void emit_pieces(const ExpandArgs &a, int32_t u, int64_t d) {
  const int nch = (int)((d + a.chunk - 1) / a.chunk);
  const int base = atomicAdd(a.gcount, nch);
  if (base + nch > a.gcap) {
    atomicOr(a.oflow, 1);
    return;
  }
  for (int c = 0; c < nch; ++c) a.gitems[base + c] = make_int2(u, c);
}

template <class Op>
__global__ void __launch_bounds__(NT) k_expand(ExpandArgs a, Op op) {
  op.pol_stream = policy_evict_first();
  __shared__ int32_t lw[NT], lb[NT];
  __shared__ int nw, nb;
  __shared__ unsigned long long red[NW];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    nw = 0;
    nb = 0;
  }
  __syncthreads();
  const int i = blockIdx.x * NT + tid;
  unsigned long long mydeg = 0;
  if (i < a.nF) {
    const int32_t u = a.F[i];
    const int64_t rs = a.rp[u], re = a.rp[u + 1];
    const int64_t d = re - rs;
    mydeg = (unsigned long long)d;
    if (d <= a.t_thread) {  // thread bin: serial inner loop in this lane
      const uint32_t su = op.load(u);
      for (int64_t k = rs; k < re; ++k) op.edge(su, k, __ldg(a.col + k), a.Fout, a.fcount);
    } else if (d <= a.t_warp) {
      lw[atomicAdd(&nw, 1)] = u;
    } else if (d <= a.t_block) {
      lb[atomicAdd(&nb, 1)] = u;
    } else {  // grid bin: global delayed buffer
      emit_pieces(a, u, d);
    }
  }
  __syncthreads();
  for (int j = warp; j < nw; j += NW) {  // warp bin
    const int32_t u = lw[j];
    const int64_t rs = a.rp[u], re = a.rp[u + 1];
    const uint32_t su = op.load(u);
    for (int64_t k = rs + lane; k < re; k += 32) op.edge(su, k, __ldg(a.col + k), a.Fout, a.fcount);
  }
  for (int j = 0; j < nb; ++j) {  // block bin
    const int32_t u = lb[j];
    const int64_t rs = a.rp[u], re = a.rp[u + 1];
    const uint32_t su = op.load(u);
    for (int64_t k = rs + tid; k < re; k += NT) op.edge(su, k, __ldg(a.col + k), a.Fout, a.fcount);
  }
  for (int o = 16; o > 0; o >>= 1) mydeg += __shfl_xor_sync(0xffffffffu, mydeg, o);
  if (lane == 0) red[warp] = mydeg;
  __syncthreads();
  if (tid == 0) {
    unsigned long long s = 0;
    for (int q = 0; q < NW; ++q) s += red[q];
    if (s) atomicAdd(a.relaxed, s);
  }
  op.fence();
}

// Default expansion (dbuf-shared, P5@3623, B200 form): every frontier vertex of the
// CTA's slice with degree <= t_warp is deferred to a shared-memory buffer of runs
// (edge offset, degree prefix, dist); the CTA then runs the buffered inner loops over
// their concatenation in windows of NT*kEdgesPerThread edges — thread t takes 8
// consecutive edges of the window (one upper-bound search per window, then a walk),
// so all threads do equal work and a warp touches consecutive edges.  Vertices of
// larger degree go to the global grid buffer (dbuf-global) as grid_chunk pieces.
#ifndef INL_EPT
#define INL_EPT 8
#endif
constexpr int kEdgesPerThread = INL_EPT;  // edges in flight per thread in the expansion kernels

template <class Op>
__global__ void __launch_bounds__(NT, INL_EXPAND_MINB) k_expand_flat(ExpandArgs a, Op op) {
  if (a.dyn.s) {  // device-sized step: CTAs beyond the frontier's slices leave before any setup
    const int nf = __ldcg(&a.dyn.s->nF);
    if ((int64_t)blockIdx.x * NT >= (nf ? nf : __ldcg(&a.dyn.s->nsplit))) return;
  }
  op.pol_stream = policy_evict_first();
  uint32_t *inq_prev;
  if (!dyn_bind(a, op, &inq_prev)) return;
  using Scan = cub::BlockScan<int, NT>;
  __shared__ typename Scan::TempStorage scan_tmp;
  __shared__ int64_t rs_s[NT];
  __shared__ int off_s[NT + 1];
  __shared__ uint32_t su_s[NT];
  __shared__ unsigned long long red[NW];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  unsigned long long mydeg = 0;
  // static launches have one slice of NT frontier vertices per CTA; dynamic ones a fixed
  // grid whose CTAs take slices from a counter (load balance across the grid)
  __shared__ int slice_s;
  int base = blockIdx.x * NT;
  if (a.dyn.s) {
    if (tid == 0) slice_s = atomicAdd(&a.dyn.s->slice, 1);
    __syncthreads();
    base = slice_s * NT;
  }
  while (base < a.nF) {
  const int i = base + tid;
  int d = 0;
  int64_t rs = 0;
  uint32_t su = 0;
  if (i < a.nF) {
    const int32_t u = a.F[i];
    if (inq_prev) inq_prev[u >> 5] = 0u;  // its claim bit of the previous iteration
    rs = a.rp[u];
    const int64_t dd = a.rp[u + 1] - rs;
    mydeg += (unsigned long long)dd;
    su = op.load(u);
    if (dd > a.t_warp) {  // grid bin: global delayed buffer
      emit_pieces(a, u, dd);
    } else {
      d = (int)dd;
    }
  }
  // compact the non-empty runs (the buffer), then their edge offsets
  int2 cnt_off = make_int2(d > 0 ? 1 : 0, d);
  int2 excl, tot;
  {
    using Scan2 = cub::BlockScan<int2, NT>;
    __shared__ typename Scan2::TempStorage scan2_tmp;
    struct Add2 {
      __device__ int2 operator()(int2 x, int2 y) const { return make_int2(x.x + y.x, x.y + y.y); }
    };
    Scan2(scan2_tmp).ExclusiveScan(cnt_off, excl, make_int2(0, 0), Add2(), tot);
  }
  (void)scan_tmp;
  if (d > 0) {
    rs_s[excl.x] = rs;
    off_s[excl.x] = excl.y;
    su_s[excl.x] = su;
  }
  const int nruns = tot.x, total = tot.y;
  if (tid == 0) off_s[nruns] = total;
  __syncthreads();
  // each warp takes 32*K consecutive edges of the window; lane l takes edges l, l+32, ...
  // (every load instruction of the warp reads 32 consecutive edges: coalesced)
  for (int w0 = warp * 32 * kEdgesPerThread; w0 < total; w0 += NT * kEdgesPerThread) {
    const int e0 = w0 + lane;
    int lo = 0, hi = nruns;  // last run with off_s[run] <= e0
    const int es = e0 < total ? e0 : total - 1;
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (off_s[mid] <= es) lo = mid; else hi = mid;
    }
    int run = lo;
    int64_t kk[kEdgesPerThread];
    uint32_t du[kEdgesPerThread];
    int32_t vv[kEdgesPerThread];
    bool in[kEdgesPerThread];
#pragma unroll
    for (int j = 0; j < kEdgesPerThread; ++j) {
      const int e = e0 + 32 * j;
      in[j] = e < total;
      if (in[j])
        while (off_s[run + 1] <= e) ++run;  // runs are non-empty: forward walk
      kk[j] = rs_s[run] + (e - off_s[run]);
      du[j] = su_s[run];
    }
#pragma unroll
    for (int j = 0; j < kEdgesPerThread; ++j) vv[j] = in[j] ? (int32_t)ld_stream_pol(a.col + kk[j], op.pol_stream) : 0;
    op.edges(du, kk, vv, in, a.Fout, a.fcount);
  }
  __syncthreads();  // the run buffer is rewritten by the next slice
  if (a.dyn.s) {
    if (tid == 0) slice_s = atomicAdd(&a.dyn.s->slice, 1);
    __syncthreads();
    base = slice_s * NT;
  } else {
    base += gridDim.x * NT;
  }
  }
  for (int o = 16; o > 0; o >>= 1) mydeg += __shfl_xor_sync(0xffffffffu, mydeg, o);
  if (lane == 0) red[warp] = mydeg;
  __syncthreads();
  if (tid == 0) {
    unsigned long long s = 0;
    for (int q = 0; q < NW; ++q) s += red[q];
    if (s) atomicAdd(a.relaxed, s);
  }
  op.fence();
}

// Grid bin (dbuf-global, P5@2721): pieces of grid_chunk edges of the large-degree
// frontier vertices, one CTA per piece (grid-stride); each thread keeps 8 edges in flight.
template <class Op>
__global__ void __launch_bounds__(NT, INL_EXPAND_MINB) k_expand_grid(ExpandArgs a, Op op) {
  // device-sized step: CTAs beyond the pieces the flat kernel emitted leave before any setup
  if (a.dyn.s && blockIdx.x >= min(__ldcg(&a.dyn.s->gcount), a.gcap)) return;
  op.pol_stream = policy_evict_first();
  uint32_t *inq_prev;
  if (!dyn_bind(a, op, &inq_prev)) return;
  __shared__ int n_s;  // one L2 read per CTA (every thread reading it would hit one L2 slice)
  if (threadIdx.x == 0) n_s = min(__ldcg(a.gcount), a.gcap);  // dropped pieces were flagged
  __syncthreads();
  const int n = n_s;
  for (int it = blockIdx.x; it < n; it += gridDim.x) {
    const int2 g = a.gitems[it];
    const int64_t rs = a.rp[g.x], re = a.rp[g.x + 1];
    const int64_t ks = rs + (int64_t)g.y * a.chunk;
    const int64_t ke = min(ks + (int64_t)a.chunk, re);
    const uint32_t su = op.load(g.x);
    for (int64_t kb = ks; kb < ke; kb += NT * kEdgesPerThread) {  // block-uniform trip count
      const int64_t k0 = kb + threadIdx.x;
      int32_t vv[kEdgesPerThread];
      int64_t kk[kEdgesPerThread];
      uint32_t du[kEdgesPerThread];
      bool in[kEdgesPerThread];
#pragma unroll
      for (int j = 0; j < kEdgesPerThread; ++j) {
        kk[j] = k0 + (int64_t)j * NT;
        in[j] = kk[j] < ke;
        du[j] = su;
        vv[j] = in[j] ? (int32_t)ld_stream_pol(a.col + kk[j], op.pol_stream) : 0;
      }
      op.edges(du, kk, vv, in, a.Fout, a.fcount);
    }
  }
  op.fence();
}

__global__ void k_init_sssp(uint32_t *dist, int64_t n, int64_t s) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    dist[i] = i == s ? 0u : 0xFFFFFFFFu;
}

__global__ void k_init_bfs(int32_t *level, uint32_t *bm, int64_t n, int64_t s) {
  const int64_t nw = (n + 31) / 32;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n || i < nw;
       i += (int64_t)gridDim.x * blockDim.x) {
    if (i < n) level[i] = i == s ? 0 : -1;
    if (i < nw) bm[i] = (i == (s >> 5)) ? (1u << (s & 31)) : 0u;
  }
}

// Near-far: move far-pile vertices with lo <= dist < hi into the near frontier (once each);
// keep those still >= hi (deduplicated through `keep`); drop the rest (already settled
// in an earlier phase at a smaller distance).
__global__ void k_far_split(const int32_t *__restrict__ far, int nfar, const uint32_t *__restrict__ dist,
                            uint32_t lo, uint32_t hi, uint32_t *inq, uint32_t *keep, int32_t *q, int *qcnt,
                            int32_t *far2, int *far2cnt) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nfar; i += gridDim.x * blockDim.x) {
    const int32_t v = far[i];
    const uint32_t d = dist[v];
    const uint32_t bit = 1u << (v & 31);
    if (d >= lo && d < hi) {
      if (!(atomicOr(inq + (v >> 5), bit) & bit)) push(q, qcnt, v);
    } else if (d >= hi) {
      if (!(atomicOr(keep + (v >> 5), bit) & bit)) push(far2, far2cnt, v);
    }
  }
}

// Device-driven step, part 1: when the near frontier is empty, advance the threshold and
// split the far pile (duplicate-free): lo <= dist < hi -> frontier, dist >= hi -> the other
// far buffer (stays marked in `keep`), dist < lo -> settled earlier, dropped.
__global__ void k_sssp_split(SsspDyn dy, const uint32_t *__restrict__ dist) {
  __shared__ __align__(16) SsspDev st_s;
  load_state(dy.s, &st_s);
  const SsspDev *s = &st_s;
  if (s->done || s->nF != 0) return;
  const int nfar = s->nfar;
  if (nfar == 0) {
    if (blockIdx.x == 0 && threadIdx.x == 0) dy.s->done = 1;
    return;
  }
  const uint32_t lo = s->thr, hi = sat_add(lo, s->delta);
  const int fpar = s->fpar, par = s->par;
  const int32_t *far = pick2(dy.far, fpar);
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nfar; i += gridDim.x * blockDim.x) {
    const int32_t v = far[i];
    const uint32_t d = dist[v];
    if (d >= hi) {
      push(pick2(dy.far, fpar ^ 1), &dy.s->nfar2, v);
    } else {
      atomicAnd(dy.keep + (v >> 5), ~(1u << (v & 31)));
      if (d >= lo) push(pick2(dy.buf, par), &dy.s->nsplit, v);
    }
  }
}

// ---- bitmap-frontier step (one GPU, CUDA-graph loop) -------------------------------------
// Step: k_sssp_bcompact (frontier bitmap C -> worklist, C zeroed) -> k_sssp_bsplit (C was
// empty: far bitmap -> worklist for [thr, thr + delta)) -> k_expand_flat / k_expand_grid
// (improvements set bits in N = the other bitmap, or in the far bitmap) -> k_sssp_bpost
// (N becomes C).  The worklist is in vertex order within each CTA's word range.
constexpr int kCompactNT = 256;

// C -> buf[0] (count in s->nF), C zeroed; one counter atomic per CTA.
__global__ void __launch_bounds__(kCompactNT) k_sssp_bcompact(SsspDyn dy) {
  __shared__ __align__(16) SsspDev st_s;
  load_state(dy.s, &st_s);
  if (st_s.done) return;
  using Scan = cub::BlockScan<int, kCompactNT>;
  __shared__ typename Scan::TempStorage tmp;
  __shared__ int base_s;
  uint4 *C = reinterpret_cast<uint4 *>(pick2(dy.inq, st_s.par));
  int32_t *F = dy.buf[0];
  const int64_t nv = dy.nwords4 / 4;  // uint4 vectors
  for (int64_t c0 = (int64_t)blockIdx.x * kCompactNT; c0 < nv; c0 += (int64_t)gridDim.x * kCompactNT) {
    const int64_t i = c0 + threadIdx.x;
    uint4 w = make_uint4(0, 0, 0, 0);
    if (i < nv) w = C[i];
    const int cnt = __popc(w.x) + __popc(w.y) + __popc(w.z) + __popc(w.w);
    int off, tot;
    Scan(tmp).ExclusiveSum(cnt, off, tot);
    if (threadIdx.x == 0) base_s = tot ? atomicAdd(&dy.s->nF, tot) : 0;
    __syncthreads();
    if (cnt) {
      int pos = base_s + off;
      const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
      for (int q = 0; q < 4; ++q)
        for (uint32_t b = ws[q]; b; b &= b - 1) F[pos++] = (int32_t)((i * 4 + q) * 32 + __ffs(b) - 1);
      C[i] = make_uint4(0, 0, 0, 0);
    }
    __syncthreads();  // tmp / base_s reuse
  }
}

// Near frontier empty: the far bitmap's vertices with thr <= dist < thr + delta -> buf[0]
// (count in s->nsplit), those with dist < thr (settled at a smaller distance) dropped, the
// rest kept (count in s->nfar).
__global__ void __launch_bounds__(kCompactNT) k_sssp_bsplit(SsspDyn dy, const uint32_t *__restrict__ dist) {
  __shared__ __align__(16) SsspDev st_s;
  load_state(dy.s, &st_s);
  const SsspDev *s = &st_s;
  if (s->done || s->nF != 0) return;
  const uint32_t lo = s->thr, hi = sat_add(lo, s->delta);
  uint4 *Fb = reinterpret_cast<uint4 *>(dy.keep);
  const int64_t nv = dy.nwords4 / 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t nvr = (nv + 31) / 32 * 32;  // whole warps iterate together (warp-aggregated pushes)
  const int lane = threadIdx.x & 31;
  int kept = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nvr; i += stride) {
    const uint4 w = i < nv ? Fb[i] : make_uint4(0, 0, 0, 0);
    uint32_t ws[4] = {w.x, w.y, w.z, w.w}, pm[4] = {0u, 0u, 0u, 0u};
    int c = 0;
    if (w.x | w.y | w.z | w.w) {
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint32_t keepw = 0;
        for (uint32_t b = ws[q]; b; b &= b - 1) {
          const int bit = __ffs(b) - 1;
          const uint32_t d = dist[(i * 4 + q) * 32 + bit];
          if (d >= hi) keepw |= 1u << bit;
          else if (d >= lo) pm[q] |= 1u << bit;
        }
        c += __popc(pm[q]);
        kept += __popc(keepw);
        ws[q] = keepw;
      }
      Fb[i] = make_uint4(ws[0], ws[1], ws[2], ws[3]);
    }
    if (!__any_sync(0xffffffffu, c != 0)) continue;
    int incl = c;  // one counter atomic per warp instead of one per moved vertex
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    int base = 0;
    if (lane == 31) base = atomicAdd(&dy.s->nsplit, incl);
    int pos = __shfl_sync(0xffffffffu, base, 31) + incl - c;
#pragma unroll
    for (int q = 0; q < 4; ++q)
      for (uint32_t b = pm[q]; b; b &= b - 1) dy.buf[0][pos++] = (int32_t)((i * 4 + q) * 32 + __ffs(b) - 1);
  }
  for (int o = 16; o > 0; o >>= 1) kept += __shfl_xor_sync(0xffffffffu, kept, o);
  if ((threadIdx.x & 31) == 0 && kept) atomicAdd(&dy.s->nfar, kept);
}

// Roll over: N becomes C; a split step that moved nothing with nothing kept ends the loop.
__global__ void k_sssp_bpost(SsspDyn dy, cudaGraphConditionalHandle cond, int use_cond) {
  SsspDev *s = dy.s;
  if (!s->done) {
    if (++s->pad > (1 << 20)) s->done = 2;
    const bool split = s->nF == 0;
    if (split && s->nsplit == 0 && s->nfar == 0) s->done = 1;
    if (!s->done) {
      if (split) s->thr = sat_add(s->thr, s->delta);
      const int size = split ? s->nsplit : s->nF;
      if (size > 0) {
        s->ftotal += (unsigned long long)size;
        s->iter += 1;
      }
      s->par ^= 1;
      s->nF = 0;
      s->nsplit = 0;
      s->nfar = 0;
      s->gcount = 0;
      s->slice = 0;
    }
  }
  if (use_cond) cudaGraphSetConditional(cond, s->done ? 0u : 1u);
}

// INL_SSSP_TRACE=<file> (measurement only): a one-thread kernel between the step kernels of the
// bitmap graph loop stamps %globaltimer, so the host can print each step's kernel durations and
// frontier sizes.  slot 0..5: step start, after compact, split, flat, grid, post; 6: nF | nsplit.
constexpr int kTraceSlots = 12, kTraceSteps = 4096;
__global__ void k_sssp_trace(const SsspDev *s, unsigned long long *tr, int slot, const unsigned long long *relaxed,
                             const unsigned long long *marks) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  const int step = s->pad;
  if (step >= kTraceSteps) return;
  unsigned long long *r = tr + step * kTraceSlots;
  r[slot] = t;
  if (slot == 3) r[6] = (unsigned long long)(unsigned)s->nF | ((unsigned long long)(unsigned)s->nsplit << 32);
  if (slot == 4) r[11] = (unsigned long long)(unsigned)s->gcount;  // grid-bin pieces of the step
  if (slot == 3 || slot == 4) {  // 7 / 8: relaxed / marked after the flat kernel; 9 / 10 after the grid kernel
    r[slot == 3 ? 7 : 9] = *relaxed;
    r[slot == 3 ? 8 : 10] = marks ? *marks : 0ull;
  }
}

// Device-driven step, part 4: roll the state over to the next step.  In the CUDA-graph loop
// (a conditional WHILE node around the four kernels) it also sets the loop condition; a step
// count far beyond any converging run (kSsspMaxSteps) stops the loop with an error flag
// instead of letting a bug spin the GPU.
constexpr int kSsspMaxSteps = 1 << 20;
__global__ void k_sssp_post(SsspDyn dy, cudaGraphConditionalHandle cond, int use_cond) {
  SsspDev *s = dy.s;
  if (!s->done && ++s->pad > kSsspMaxSteps) s->done = 2;
  if (use_cond) cudaGraphSetConditional(cond, s->done ? 0u : 1u);
  if (s->done) return;
  const bool split = s->nF == 0;
  if (split) {
    s->thr = sat_add(s->thr, s->delta);
    s->nfar = s->nfar2;
    s->nfar2 = 0;
    s->fpar ^= 1;
  }
  const int size = split ? s->nsplit : s->nF;
  s->nsplit = 0;
  if (size > 0) {
    s->ftotal += (unsigned long long)size;
    s->iter += 1;
    s->nF = s->cnt;
    s->par ^= 1;
  }
  s->cnt = 0;
  s->gcount = 0;
  s->slice = 0;
}

// P > 1: vertices of the owned slice whose distance dropped -> next frontier.
__global__ void k_sssp_collect(const uint32_t *__restrict__ dist, uint32_t *__restrict__ prev,
                               int64_t row_begin, int64_t n_rows, int32_t *q, int *cnt) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n_rows;
       v += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t d = dist[row_begin + v];
    if (d < prev[v]) {
      prev[v] = d;
      push(q, cnt, (int32_t)v);
    }
  }
}

// NEXT-1: the owned vertices whose distance improved this round (their bits in this rank's
// changed-bitmap, set by every rank's relaxations) -> next local frontier
__global__ void k_sssp_collect_xbits(const uint32_t *__restrict__ chg, int64_t row_begin, int64_t n_rows, int32_t *q,
                                     int *cnt) {
  const int64_t w0 = row_begin / 32, w1 = (row_begin + n_rows + 31) / 32;
  for (int64_t w = w0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < w1; w += (int64_t)gridDim.x * blockDim.x) {
    for (uint32_t b = chg[w]; b; b &= b - 1) {
      const int64_t v = w * 32 + __ffs(b) - 1;
      if (v >= row_begin && v < row_begin + n_rows) push(q, cnt, (int32_t)(v - row_begin));
    }
  }
}

__global__ void k_copy_u32(const uint32_t *__restrict__ a, uint32_t *__restrict__ b, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    b[i] = a[i];
}

// P > 1: apply the allreduced next map: new vertices get level L+1; owned ones
// form the next local frontier.
__global__ void k_bfs_apply(const uint8_t *__restrict__ next, int64_t n, int32_t *level,
                            uint32_t *bm, int L, int64_t row_begin, int64_t n_rows, int32_t *q,
                            int *cnt) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    if (next[v] && level[v] < 0) {
      level[v] = L + 1;
      atomicOr(bm + (v >> 5), 1u << (v & 31));
      if (v >= row_begin && v < row_begin + n_rows) push(q, cnt, (int32_t)(v - row_begin));
    }
  }
}

// NEXT-1 apply (P > 1): the level's new-frontier bitmap is the OR over the owners' buffers (an
// owner's buffer holds the bits every rank set for its vertices; a word straddling two row
// blocks reads both).  New vertices (not yet visited) get level L+1 on EVERY rank — the level
// vector stays replicated with no allgather — and the owned ones form the next local frontier.
// *total counts the new vertices of the whole graph: the same on every rank, so the ranks agree
// on termination without a collective.
__global__ void k_bfs_apply_xbits(uint32_t *const *__restrict__ xtab, int64_t B, int64_t n, uint32_t *bm,
                                  int32_t *level, int L, int64_t row_begin, int64_t n_rows, int32_t *q, int *cnt,
                                  unsigned long long *total) {
  const int64_t nwords = (n + 31) / 32;
  const int64_t nn = (nwords + 31) / 32 * 32;
  unsigned long long c = 0;
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nn; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t nw = 0;
    if (w < nwords) {
      const int64_t lo = w * 32, hi = min(lo + 32, n);
      uint32_t bits = 0;
      for (int64_t o = lo / B; o <= (hi - 1) / B; ++o) bits |= __ldcg(xtab[o] + w);
      nw = bits & ~bm[w];
      if (nw) {
        bm[w] |= nw;
        c += (unsigned long long)__popc(nw);
        for (uint32_t b = nw; b; b &= b - 1) {
          const int64_t v = lo + __ffs(b) - 1;
          level[v] = L + 1;
          if (v >= row_begin && v < row_begin + n_rows) push(q, cnt, (int32_t)(v - row_begin));
        }
      }
    }
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(total, c);
    c = 0;
  }
}

// ---- direction-optimizing BFS (single GPU): bottom-up steps for large frontiers ----
// One warp owns 32 consecutive vertices = one word of each bitmap, so no atomics: an
// unvisited vertex scans its neighbours (thread-mapped, early exit at the first one in
// the current frontier bitmap).
__global__ void k_bfs_bottom_up(const int64_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n,
                                uint32_t *__restrict__ visited, const uint32_t *__restrict__ fcur,
                                uint32_t *__restrict__ fnext, int32_t *__restrict__ level, int L,
                                int *__restrict__ count, unsigned long long *__restrict__ mf) {
  const int lane = threadIdx.x & 31;
  const int64_t nwords = (n + 31) / 32;
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w < nwords;
       w += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t vis = visited[w];
    const int64_t v = w * 32 + lane;
    bool found = false;
    unsigned long long dg = 0;
    if (v < n && !((vis >> lane) & 1u)) {
      const int64_t e = rp[v + 1];
      // 4 neighbours per step: their column loads, then their frontier-bit loads, are
      // issued back to back (the scan is a chain of dependent loads otherwise)
      for (int64_t k = rp[v]; k < e && !found; k += 4) {
        int32_t u[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) u[j] = k + j < e ? __ldg(col + k + j) : -1;
        uint32_t fw[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) fw[j] = u[j] >= 0 ? __ldg(fcur + (u[j] >> 5)) : 0u;
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (u[j] >= 0 && ((fw[j] >> (u[j] & 31)) & 1u)) found = true;
      }
      if (found) {
        level[v] = L + 1;
        dg = (unsigned long long)(e - rp[v]);
      }
    }
    for (int o = 16; o > 0; o >>= 1) dg += __shfl_xor_sync(0xffffffffu, dg, o);
    if (lane == 0 && dg) atomicAdd(mf, dg);
    const uint32_t nw = __ballot_sync(0xffffffffu, found);
    if (lane == 0) {
      fnext[w] = nw;
      if (nw) {
        visited[w] = vis | nw;
        atomicAdd(count, __popc(nw));
      }
    }
  }
}

// ---- bottom-up with the paper's template: the unvisited vertices of
// degree > 0 are kept in two worklists by degree — thread-mapped (<= kBuThread neighbours:
// one lane scans serially, 8 neighbour loads in flight) and warp-mapped (above: the warp
// scans 64 neighbours per step, early exit on __any_sync) — so no lane idles on a visited
// vertex and no warp waits on one long serial scan (the T1 form above).  A vertex that
// finds no parent is carried over to the next level's list (order-preserving within a warp).
constexpr int kBuThread = 32;

// Worklist maintenance through CUB's decoupled look-back selects (stable, one pass each):
// a per-warp counter atomic on one address serialises at its L2 slice (measured: 2.7 ms to
// build the lists at scale 26 that way).
struct BuBin {  // unvisited, degree in (lo, hi]
  const int64_t *rp;
  const uint32_t *visited;
  int64_t lo, hi;
  __device__ __forceinline__ bool operator()(int32_t v) const {
    if ((visited[v >> 5] >> (v & 31)) & 1u) return false;
    const int64_t d = rp[v + 1] - rp[v];
    return d > lo && d <= hi;
  }
};
struct BuDeg {  // degree in (lo, hi]
  const int64_t *rp;
  int64_t lo, hi;
  __device__ __forceinline__ bool operator()(int32_t v) const {
    const int64_t d = rp[v + 1] - rp[v];
    return d > lo && d <= hi;
  }
};
struct BuUnvisited {
  const uint32_t *visited;
  __device__ __forceinline__ bool operator()(int32_t v) const { return !((visited[v >> 5] >> (v & 31)) & 1u); }
};

struct BuArgs {
  const int64_t *rp;
  const int32_t *col;
  const uint32_t *fcur;  // current frontier bitmap
  uint32_t *fnext;       // next frontier bitmap (cleared before the level)
  uint32_t *visited;
  int32_t *level;
  int L;
  const int32_t *in;     // this level's list
  int n_in;
  int *found;            // newly visited vertices
  unsigned long long *mf;  // their degree sum (Beamer's m_f)
  uint64_t pol;
  unsigned long long *examined;  // neighbours read (the stats' edges_relaxed)
  // `in` is the plan's static degree bin (every vertex of degree > 0, visited or not): skip the
  // visited ones (the first bottom-up level; later levels read the compacted unvisited lists)
  bool check_visited = false;
};

__device__ __forceinline__ bool bu_skip(const BuArgs &a, int32_t v) {
  return a.check_visited && ((__ldg(a.visited + (v >> 5)) >> (v & 31)) & 1u);
}

__device__ __forceinline__ void bu_visit(const BuArgs &a, int32_t v) {
  const uint32_t bit = 1u << (v & 31);
  a.level[v] = a.L + 1;
  atomicOr(a.fnext + (v >> 5), bit);
  atomicOr(a.visited + (v >> 5), bit);
}

// thread bin: one lane per vertex, its <= kBuThread neighbours 8 at a time
template <int K1>  // neighbours probed in the first batch (then 8 per batch)
__global__ void __launch_bounds__(256) k_bu_thread(BuArgs a) {
  a.pol = policy_evict_first();
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t nn = ((int64_t)a.n_in + 31) / 32 * 32;
  int fcnt = 0;
  unsigned long long dg = 0, ex = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nn; i += stride) {
    bool valid = i < a.n_in;
    const int32_t v = valid ? a.in[i] : 0;
    if (valid && bu_skip(a, v)) valid = false;
    bool found = false;
    int64_t s = 0, e = 0;
    if (valid) {
      s = a.rp[v];
      e = a.rp[v + 1];
    }
    int64_t k = s;
    if (K1 < 8 && k < e) {  // a short first batch: most vertices find a parent among their first neighbours
      ex += (unsigned long long)min((int64_t)K1, e - k);
      int32_t u[K1];
#pragma unroll
      for (int j = 0; j < K1; ++j) u[j] = k + j < e ? (int32_t)ld_stream_pol(a.col + k + j, a.pol) : -1;
      uint32_t fw[K1];
#pragma unroll
      for (int j = 0; j < K1; ++j) fw[j] = u[j] >= 0 ? __ldg(a.fcur + (u[j] >> 5)) : 0u;
#pragma unroll
      for (int j = 0; j < K1; ++j)
        if (u[j] >= 0 && ((fw[j] >> (u[j] & 31)) & 1u)) found = true;
      k += K1;
    }
    for (; k < e && !found; k += 8) {
      ex += (unsigned long long)min((int64_t)8, e - k);
      int32_t u[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) u[j] = k + j < e ? (int32_t)ld_stream_pol(a.col + k + j, a.pol) : -1;
      uint32_t fw[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) fw[j] = u[j] >= 0 ? __ldg(a.fcur + (u[j] >> 5)) : 0u;
#pragma unroll
      for (int j = 0; j < 8; ++j)
        if (u[j] >= 0 && ((fw[j] >> (u[j] & 31)) & 1u)) found = true;
    }
    if (found) {
      bu_visit(a, v);
      ++fcnt;
      dg += (unsigned long long)(e - s);
    }
  }
  for (int o = 16; o > 0; o >>= 1) {
    fcnt += __shfl_xor_sync(0xffffffffu, fcnt, o);
    dg += __shfl_xor_sync(0xffffffffu, dg, o);
    ex += __shfl_xor_sync(0xffffffffu, ex, o);
  }
  if ((threadIdx.x & 31) == 0) {
    if (fcnt) {
      atomicAdd(a.found, fcnt);
      atomicAdd(a.mf, dg);
    }
    if (ex) atomicAdd(a.examined, ex);
  }
}

// Group-mapped bottom-up scan: G lanes per vertex (32/G vertices per warp), 2G neighbours per
// step (two loads per lane in flight, consecutive lanes on consecutive neighbours: one sector
// serves a group's load instead of one per lane), early exit on the group's ballot, at most
// SPAN neighbours; with DEFER a vertex whose first SPAN neighbours hold no parent goes to the
// deep list.  Warp bin: G = 8, SPAN = 64 — in a bottom-up level almost every high-degree vertex
// has a frontier neighbour among its first few (R-MAT scale 22: median position 4, 90th
// percentile 14), so a whole warp per vertex would mostly read wasted lanes.  Thread bin (the
// vertices of <= kBuThread neighbours) as 4-lane groups (INL_BFS_SMALL=group): 4x fewer L1TEX
// wavefronts for the column loads than one lane per vertex, but measured no faster (scale 26:
// 0.47 vs 0.43 ms per launch) — the random frontier-bit probes bound it; k_bu_thread stays.
// lanes per vertex of the warp bin: 2 (4 neighbours per step, 16 vertices per warp) measured
// best — scale 26: 8 lanes 2.50, 4 lanes 2.35, 2 lanes 2.29, 1 lane 2.33 ms per BFS
// (profiles/r02/bfs_group_sweep.txt); INL_BFS_GROUP = 1 / 4 / 8 / 16 to measure
constexpr int kBuGroup = 2;
constexpr int kBuGroupSpan = 64;

template <int G, int SPAN, bool DEFER>
__global__ void __launch_bounds__(256) k_bu_group(BuArgs a, int32_t *deep, int *n_deep) {
  a.pol = policy_evict_first();
  const int lane = threadIdx.x & 31, gl = lane & (G - 1), gsh = lane & ~(G - 1);
  constexpr unsigned GM = G == 32 ? 0xffffffffu : ((1u << G) - 1u);
  const int64_t ngroups = ((int64_t)gridDim.x * blockDim.x) / G;
  const int64_t nn = ((int64_t)a.n_in + (32 / G) - 1) / (32 / G) * (32 / G);  // a warp's groups iterate together
  int fcnt = 0;
  unsigned long long dg = 0, ex = 0;
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / G; i < nn; i += ngroups) {
    bool valid = i < a.n_in;
    const int32_t v = valid ? a.in[i] : 0;
    if (valid && bu_skip(a, v)) valid = false;
    int64_t s = 0, e = 0;
    if (valid) {
      s = a.rp[v];
      e = a.rp[v + 1];
    }
    const int64_t stop = min(e, s + SPAN);
    bool found = false;
    for (int64_t k = s;; k += 2 * G) {
      const bool act = k < stop && !found;
      if (!__any_sync(0xffffffffu, act)) break;
      bool hit = false;
      if (act) {
        const int64_t k0 = k + gl, k1 = k + G + gl;
        const int32_t u0 = k0 < stop ? (int32_t)ld_stream_pol(a.col + k0, a.pol) : -1;
        const int32_t u1 = k1 < stop ? (int32_t)ld_stream_pol(a.col + k1, a.pol) : -1;
        const uint32_t f0 = u0 >= 0 ? __ldg(a.fcur + (u0 >> 5)) : 0u;
        const uint32_t f1 = u1 >= 0 ? __ldg(a.fcur + (u1 >> 5)) : 0u;
        hit = (u0 >= 0 && ((f0 >> (u0 & 31)) & 1u)) || (u1 >= 0 && ((f1 >> (u1 & 31)) & 1u));
        if (gl == 0) ex += (unsigned long long)min((int64_t)(2 * G), stop - k);
      }
      const unsigned m = __ballot_sync(0xffffffffu, hit);
      if ((m >> gsh) & GM) found = true;
    }
    if (gl == 0 && valid) {
      if (found) {
        bu_visit(a, v);
        ++fcnt;
        dg += (unsigned long long)(e - s);
      } else if (DEFER && e > stop) {
        deep[atomicAdd(n_deep, 1)] = v;  // rare: no parent among the first SPAN
      }
    }
  }
  for (int o = 16; o > 0; o >>= 1) {
    fcnt += __shfl_xor_sync(0xffffffffu, fcnt, o);
    dg += __shfl_xor_sync(0xffffffffu, dg, o);
    ex += __shfl_xor_sync(0xffffffffu, ex, o);
  }
  if (lane == 0) {
    if (fcnt) {
      atomicAdd(a.found, fcnt);
      atomicAdd(a.mf, dg);
    }
    if (ex) atomicAdd(a.examined, ex);
  }
}

// warp bin, deep pass: one warp per deferred vertex from neighbour kBuGroupSpan on, 64 per step,
// early exit on __any_sync.  The count is read on the device (no host round trip).
__global__ void __launch_bounds__(256) k_bu_deep(BuArgs a, const int32_t *deep, const int *n_deep) {
  a.pol = policy_evict_first();
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int n = *n_deep;
  int fcnt = 0;
  unsigned long long dg = 0, ex = 0;
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n; i += nw) {
    const int32_t v = deep[i];
    const int64_t s = a.rp[v], e = a.rp[v + 1];
    bool found = false;
    for (int64_t k = s + kBuGroupSpan; k < e; k += 64) {
      ex += (unsigned long long)min((int64_t)64, e - k);
      const int64_t k0 = k + lane, k1 = k + 32 + lane;
      const int32_t u0 = k0 < e ? (int32_t)ld_stream_pol(a.col + k0, a.pol) : -1;
      const int32_t u1 = k1 < e ? (int32_t)ld_stream_pol(a.col + k1, a.pol) : -1;
      const uint32_t f0 = u0 >= 0 ? __ldg(a.fcur + (u0 >> 5)) : 0u;
      const uint32_t f1 = u1 >= 0 ? __ldg(a.fcur + (u1 >> 5)) : 0u;
      const bool hit = (u0 >= 0 && ((f0 >> (u0 & 31)) & 1u)) || (u1 >= 0 && ((f1 >> (u1 & 31)) & 1u));
      if (__any_sync(0xffffffffu, hit)) {
        found = true;
        break;
      }
    }
    if (lane == 0 && found) {
      bu_visit(a, v);
      ++fcnt;
      dg += (unsigned long long)(e - s);
    }
  }
  if (lane == 0) {
    if (fcnt) {
      atomicAdd(a.found, fcnt);
      atomicAdd(a.mf, dg);
    }
    if (ex) atomicAdd(a.examined, ex);
  }
}

__global__ void k_queue_to_bitmap(const int32_t *__restrict__ q, int nq, uint32_t *__restrict__ bm) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nq; i += gridDim.x * blockDim.x)
    atomicOr(bm + (q[i] >> 5), 1u << (q[i] & 31));
}

// next frontier bitmap -> queue (one counter atomic per warp) and its degree sum (Beamer's m_f)
__global__ void k_bfs_next_queue(const uint32_t *__restrict__ nb, int64_t nwords, const int64_t *__restrict__ rp,
                                 int32_t *q, int *cnt, unsigned long long *mf) {
  const int64_t nr = (nwords + 31) / 32 * 32;  // whole warps iterate together
  const int lane = threadIdx.x & 31;
  unsigned long long dg = 0;
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
    if (lane == 31) base = atomicAdd(cnt, incl);
    int pos = __shfl_sync(0xffffffffu, base, 31) + incl - c;
    for (; b; b &= b - 1) {
      const int32_t v = (int32_t)(w * 32 + __ffs(b) - 1);
      q[pos++] = v;
      dg += (unsigned long long)(rp[v + 1] - rp[v]);
    }
  }
  for (int o = 16; o > 0; o >>= 1) dg += __shfl_xor_sync(0xffffffffu, dg, o);
  if (lane == 0 && dg) atomicAdd(mf, dg);
}

__global__ void k_bitmap_to_queue(const uint32_t *__restrict__ bm, int64_t n, int32_t *q, int *cnt) {
  const int64_t nwords = (n + 31) / 32;
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nwords;
       w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t b = bm[w];
    while (b) {
      const int t = __ffs(b) - 1;
      b &= b - 1;
      push(q, cnt, (int32_t)(w * 32 + t));
    }
  }
}

int grid_for(int64_t n, int sms) {
  int64_t g = (n + 255) / 256;
  if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
  return g < 1 ? 1 : (int)g;
}

// Near-far bucket width (Davidson et al., IPDPS'14, "near-far" delta stepping); env
// INL_SSSP_DELTA overrides (0xFFFFFFFF = plain frontier Bellman-Ford).
uint32_t sssp_delta() {
  static uint32_t d = 0;
  if (!d) {
    // near-far delta on R-MAT scale 23, w in [1, 255]: 48 with the round-1 worklists
    // (profiles/r01/sssp_delta_sweep2.txt); 96 with the bitmap loop at 32 warps / SM (4.33 ->
    // 4.03 ms; 128..384 within 2% but more wasted relaxations; profiles/r02/sssp_bitmap_sweeps.txt)
    d = 96;
    if (const char *e = getenv("INL_SSSP_DELTA")) d = (uint32_t)strtoul(e, nullptr, 10);
    if (!d) d = 0xFFFFFFFFu;
  }
  return d;
}

struct FrontierBufs {
  int32_t *F, *Fout;
  int2 *gitems;
  int64_t gcap;
  int *counts;  // [0] fcount [1] gcount [2] grid-buffer overflow flag; u64 at [8] relaxed, [10] m_f
  unsigned long long *relaxed;
  int *h_counts;  // pinned
};

// Thresholds the expansion kernels use, and the grid-buffer capacity they imply.
//  * default: k_expand_flat defers vertices of degree > t_warp to the grid buffer;
//  * the paper's templates / the T1 baseline: k_expand (lbTHRES = t_thread; dbuf-global sends
//    everything above it to the grid buffer, dbuf-shared and T1 nothing).
// A frontier holds each vertex at most once, and a vertex of degree d > T emits ceil(d / C)
// <= d / C + 1 pieces, so one expansion emits at most nnz / C + min(n_rows, nnz / (T + 1)).
struct ExpandCfg {
  int t_thread, t_warp, t_block, chunk;
  bool flat;     // k_expand_flat (else k_expand)
  int64_t gcap;  // grid-buffer capacity in pieces
};

ExpandCfg expand_cfg(const inl_csr &G, const Bins &b) {
  ExpandCfg c{b.t_thread, b.t_warp, b.t_block, std::min(b.grid_chunk, 2048), true, 0};
  const int tpl = b.flags & kTemplateFlags;
  if (tpl) {  // the paper's templates (template study): lbTHRES = t_thread
    c.t_warp = b.t_thread;  // no warp bin: above lbTHRES is block-mapped ...
    // ... in smem (dbuf-shared), via the grid buffer (dbuf-global), or from the large queue of
    // the pre-pass (dual-queue: no grid buffer)
    c.t_block = tpl == INL_BINS_TPL_DBUF_GLOBAL ? b.t_thread : INT32_MAX / 2;
  }
  c.flat = !((b.flags & INL_BINS_THREAD_ONLY) || tpl);
  const int64_t T = c.flat ? c.t_warp : c.t_block;
  c.gcap = G.nnz / c.chunk + std::min<int64_t>(G.n_rows, G.nnz / (T + 1)) + 64;
  INL_CHECK(c.gcap < INT32_MAX, "frontier: grid buffer capacity exceeds 2^31 pieces");
  return c;
}

FrontierBufs frontier_bufs(inl_ctx ctx, const inl_csr &G, const Bins &b) {
  FrontierBufs f;
  const int64_t n = G.n_global;
  f.F = (int32_t *)ctx->s_a.get(sizeof(int32_t) * (n + 1));
  f.Fout = (int32_t *)ctx->s_b.get(sizeof(int32_t) * (n + 1));
  f.gcap = expand_cfg(G, b).gcap;
  f.gitems = (int2 *)ctx->s_c.get(sizeof(int2) * f.gcap);
  f.counts = (int *)ctx->s_f.get(64);
  f.relaxed = (unsigned long long *)(f.counts + 8);
  f.h_counts = (int *)ctx->pinned;
  INL_CUDA(cudaMemsetAsync(f.counts, 0, 64, ctx->stream));
  return f;
}

// The grid-buffer overflow flag (never expected: gcap is an upper bound) -> INL_ERR_INTERNAL.
void check_overflow(inl_ctx ctx, const FrontierBufs &f) {
  int h = 0;
  INL_CUDA(cudaMemcpyAsync(&h, f.counts + 2, sizeof(int), cudaMemcpyDeviceToHost, ctx->stream));
  ctx_sync(ctx);
  if (h) raise(INL_ERR_INTERNAL, "frontier grid buffer overflow (capacity " + std::to_string(f.gcap) + " pieces)");
}

template <class Op>
void expand(inl_ctx ctx, const inl_csr &G, const Bins &b, FrontierBufs &f, int nF, const Op &op) {
  cudaStream_t st = ctx->stream;
  INL_CUDA(cudaMemsetAsync(f.counts, 0, 2 * sizeof(int), st));
  const ExpandCfg c = expand_cfg(G, b);
  ExpandArgs a{f.F, nF, G.row_ptr, G.col_idx, c.t_thread, c.t_warp, c.t_block, c.chunk,
               f.gitems, f.counts + 1, (int)f.gcap, f.counts + 2, f.Fout, f.counts, f.relaxed};
  if ((b.flags & kTemplateFlags) == INL_BINS_TPL_DUAL_QUEUE) {
    int32_t *qs = (int32_t *)ctx->s_bu.get(sizeof(int32_t) * 2 * (size_t)(G.n_rows + 1));
    int32_t *ql = qs + G.n_rows + 1;
    INL_CUDA(cudaMemsetAsync(f.counts + 4, 0, 2 * sizeof(int), st));
    if (nF > 0) {
      {
        KScope ks(ctx, "k_dq_split");
        k_dq_split<<<grid_for(nF, ctx->num_sms), NT, 0, st>>>(f.F, nF, G.row_ptr, c.t_thread, qs, f.counts + 4, ql,
                                                             f.counts + 5, f.relaxed);
      }
      {
        KScope ks(ctx, "k_dq_thread");
        k_dq_thread<Op><<<grid_for(nF, ctx->num_sms), NT, 0, st>>>(qs, f.counts + 4, G.row_ptr, G.col_idx, op, f.Fout,
                                                                  f.counts);
      }
      KScope ks(ctx, "k_dq_block");
      k_dq_block<Op><<<ctx->num_sms * 8, NT, 0, st>>>(ql, f.counts + 5, G.row_ptr, G.col_idx, op, f.Fout, f.counts);
    }
    INL_CUDA(cudaGetLastError());
    return;
  }
  if (nF > 0) {
    if (!c.flat) {  // the paper's baseline (thread-mapped) / templates
      KScope ks(ctx, "k_expand");
      k_expand<Op><<<(nF + NT - 1) / NT, NT, 0, st>>>(a, op);
    } else {
      KScope ks(ctx, "k_expand_flat");
      k_expand_flat<Op><<<(nF + NT - 1) / NT, NT, 0, st>>>(a, op);
    }
  }
  {
    KScope ks(ctx, "k_expand_grid");
    k_expand_grid<Op><<<ctx->num_sms * 8, NT, 0, st>>>(a, op);
  }
  INL_CUDA(cudaGetLastError());
}

int read_count(inl_ctx ctx, const int *d) {
  INL_CUDA(cudaMemcpyAsync(ctx->pinned, d, sizeof(int), cudaMemcpyDeviceToHost, ctx->stream));
  ctx_sync(ctx);
  return *(volatile int *)ctx->pinned;
}

// xbytes: exchange bytes counted on the host; the device adds 4 B per remote atomic (counts[12])
void finish_stats(inl_ctx ctx, FrontierBufs &f, inl_stats *st, int iters, int64_t ftotal, int64_t xbytes = 0) {
  check_overflow(ctx, f);
  if (!st) return;
  unsigned long long r[3] = {0, 0, 0};  // relaxed (counts[8]), m_f / total (counts[10]), remote atomics (counts[12])
  INL_CUDA(cudaMemcpyAsync(r, f.relaxed, sizeof r, cudaMemcpyDeviceToHost, ctx->stream));
  ctx_sync(ctx);
  st->iterations = iters;
  st->edges_relaxed = (int64_t)r[0];
  st->frontier_total = ftotal;
  st->launches = 0;  // host-driven loops: not counted
  st->host_syncs = iters;
  st->exchange_bytes = xbytes + 4 * (int64_t)r[2];
}

}  // namespace

// One GPU, near-far: the step loop runs on the device (k_sssp_split, k_expand_flat,
// k_expand_grid, k_sssp_post per step, fixed grids); the host enqueues `batch` steps per
// round trip and reads back the `done` flag.  Same fixed point as the host-driven loop.
static void sssp_run_dyn(inl_ctx ctx, const inl_csr &G, const Bins &b, const uint32_t *w, int64_t source,
                         uint32_t *dist, inl_stats *stats) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  FrontierBufs f = frontier_bufs(ctx, G, b);
  INL_CUDA(cudaMemsetAsync(f.relaxed, 0, sizeof(unsigned long long), st));
  // the polling loop keeps the queue-counter worklists; INL_SSSP_DYN_BITS=1 runs the graph loop's
  // bitmap step kernels stream-launched instead (so ncu can profile them: it skips kernels inside
  // conditional graph nodes)
  const char *dbe = getenv("INL_SSSP_DYN_BITS");
  const int bmode = dbe && atoi(dbe) != 0;
  const int64_t nwb = ((n + 31) / 32 + 1 + 3) / 4 * 4;  // a multiple of 4 words (uint4 scans)
  SsspDyn dy{};
  uint32_t *bits = (uint32_t *)ctx->s_d.get(sizeof(uint32_t) * 3 * nwb);
  dy.inq[0] = bits;
  dy.inq[1] = bits + nwb;
  dy.keep = bits + 2 * nwb;
  dy.bits = bmode != 0;
  dy.nwords4 = nwb;
  INL_CUDA(cudaMemsetAsync(bits, 0, sizeof(uint32_t) * 3 * nwb, st));
  dy.far[0] = (int32_t *)ctx->s_g.get(sizeof(int32_t) * (2 * n + 16));
  dy.far[1] = dy.far[0] + n + 8;
  dy.buf[0] = f.F;
  dy.buf[1] = f.Fout;
  dy.s = (SsspDev *)ctx->s_e.get(sizeof(SsspDev));
  static_assert(sizeof(SsspDev) <= 64, "SsspDev is read back through the ctx's 64-B pinned buffer");
  const bool owned = source >= G.row_begin && source < G.row_begin + G.n_rows;
  SsspDev h{};
  h.nF = owned && !dy.bits ? 1 : 0;
  h.thr = h.delta = sssp_delta();
  INL_CUDA(cudaMemcpyAsync(dy.s, &h, sizeof h, cudaMemcpyHostToDevice, st));
  const int32_t s0 = (int32_t)(owned ? source - G.row_begin : 0);
  if (dy.bits) {  // the source's bit in C = inq[0]
    if (owned) {
      uint32_t *hw = (uint32_t *)ctx->pinned;
      hw[0] = 1u << (s0 & 31);
      INL_CUDA(cudaMemcpyAsync(dy.inq[0] + (s0 >> 5), hw, sizeof(uint32_t), cudaMemcpyHostToDevice, st));
    }
  } else {
    INL_CUDA(cudaMemcpyAsync(f.F, &s0, sizeof(int32_t), cudaMemcpyHostToDevice, st));
  }
  k_init_sssp<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(dist, n, source);
  INL_CUDA(cudaGetLastError());
  const ExpandCfg c = expand_cfg(G, b);
  ExpandArgs a{f.F, 0, G.row_ptr, G.col_idx, c.t_thread, c.t_warp, c.t_block, c.chunk,
               f.gitems, nullptr, (int)f.gcap, f.counts + 2, f.Fout, nullptr, f.relaxed};
  a.dyn = dy;
  SsspOp op{dist, w, nullptr, nullptr, 0, 0, true, 0, 0, nullptr, nullptr, nullptr};
  static int gmul = -1;  // grid multipliers (env INL_SSSP_GRIDS=split,flat,grid for tuning)
  static int gm[3] = {2, 8, 2};
  if (gmul < 0) {
    gmul = 1;
    if (bmode) gm[1] = 6, gm[2] = 8;  // the graph loop's bitmap-step grids
    if (const char *e = getenv("INL_SSSP_GRIDS")) sscanf(e, "%d,%d,%d", &gm[0], &gm[1], &gm[2]);
  }
  const int gsplit = ctx->num_sms * gm[0], gflat = ctx->num_sms * gm[1], ggrid = ctx->num_sms * gm[2];
  SsspBitsOp bop;
  static_cast<SsspOp &>(bop) = op;
  const int64_t nv4 = nwb / 4;
  const int gc = (int)std::max<int64_t>(1, std::min<int64_t>((nv4 + kCompactNT - 1) / kCompactNT, (int64_t)ctx->num_sms * 8));
  int64_t launches = 1, syncs = 0;
  int batch = 4;
  SsspDev *hs = (SsspDev *)ctx->pinned;  // pinned scratch (>= 64 B)
  for (;;) {
    for (int k = 0; k < batch && bmode; ++k) {
      k_sssp_bcompact<<<gc, kCompactNT, 0, st>>>(dy);
      k_sssp_bsplit<<<gc, kCompactNT, 0, st>>>(dy, dist);
      {
        KScope ks(ctx, "k_expand_flat");
        k_expand_flat<SsspBitsOp><<<gflat, NT, 0, st>>>(a, bop);
      }
      {
        KScope ks(ctx, "k_expand_grid");
        k_expand_grid<SsspBitsOp><<<ggrid, NT, 0, st>>>(a, bop);
      }
      k_sssp_bpost<<<1, 1, 0, st>>>(dy, 0, 0);
      launches += 5;
    }
    for (int k = 0; k < batch && !bmode; ++k) {
      {
        KScope ks(ctx, "k_sssp_split");
        k_sssp_split<<<gsplit, 256, 0, st>>>(dy, dist);
      }
      {
        KScope ks(ctx, "k_expand_flat");
        k_expand_flat<SsspOp><<<gflat, NT, 0, st>>>(a, op);
      }
      {
        KScope ks(ctx, "k_expand_grid");
        k_expand_grid<SsspOp><<<ggrid, NT, 0, st>>>(a, op);
      }
      k_sssp_post<<<1, 1, 0, st>>>(dy, 0, 0);
      launches += 4;
    }
    INL_CUDA(cudaGetLastError());
    INL_CUDA(cudaMemcpyAsync(hs, dy.s, sizeof(SsspDev), cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    ++syncs;
    if (((volatile SsspDev *)hs)->done) break;
    if (batch < 16) batch *= 2;
  }
  check_overflow(ctx, f);
  if (stats) {
    unsigned long long r = 0;
    INL_CUDA(cudaMemcpyAsync(&r, f.relaxed, sizeof r, cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    stats->iterations = hs->iter;
    stats->edges_relaxed = (int64_t)r;
    stats->frontier_total = (int64_t)hs->ftotal;
    stats->launches = launches;
    stats->host_syncs = syncs;
    stats->exchange_bytes = 0;
  }
}

// One GPU, near-far, CUDA graph: the step (k_sssp_split, k_expand_flat, k_expand_grid,
// k_sssp_post) is the body of a conditional WHILE node that k_sssp_post keeps enabled until
// the near frontier and the far pile are both empty — the whole source runs as ONE graph
// launch with no host round trip (host_syncs = 1: the final stats read).  The executable
// graph is cached in the ctx and rebuilt only when an argument it captured changes.
struct SsspGraphKey {
  const int64_t *rp;
  const int32_t *col;
  const uint32_t *w;
  uint32_t *dist;
  void *bufs[6];
  int64_t n, nnz, gcap;
  int t_warp, chunk, gm0, gm1, gm2;
  uint32_t delta;
  int bits;
  void *trace;
  bool operator==(const SsspGraphKey &o) const { return memcmp(this, &o, sizeof(*this)) == 0; }
};

struct SsspGraph {
  SsspGraphKey key{};
  cudaGraphExec_t exec = nullptr;
  cudaGraph_t graph = nullptr;
  ~SsspGraph() {
    if (exec) cudaGraphExecDestroy(exec);
    if (graph) cudaGraphDestroy(graph);
  }
};

void sssp_graph_free(void *g) { delete static_cast<SsspGraph *>(g); }

static void sssp_run_graph(inl_ctx ctx, const inl_csr &G, const Bins &b, const uint32_t *w, int64_t source,
                           uint32_t *dist, inl_stats *stats) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  FrontierBufs f = frontier_bufs(ctx, G, b);
  INL_CUDA(cudaMemsetAsync(f.relaxed, 0, sizeof(unsigned long long), st));
  // bitmap frontier by default (INL_SSSP_FRONTIER=list: the r02 queue-counter worklists)
  const char *fe = getenv("INL_SSSP_FRONTIER");
  const int bmode = !(fe && !strcmp(fe, "list"));
  const int64_t nwb = ((n + 31) / 32 + 1 + 3) / 4 * 4;  // a multiple of 4 words (uint4 scans)
  SsspDyn dy{};
  uint32_t *bits = (uint32_t *)ctx->s_d.get(sizeof(uint32_t) * 3 * nwb);
  dy.inq[0] = bits;
  dy.inq[1] = bits + nwb;
  dy.keep = bits + 2 * nwb;
  dy.bits = bmode != 0;
  dy.nwords4 = nwb;
  INL_CUDA(cudaMemsetAsync(bits, 0, sizeof(uint32_t) * 3 * nwb, st));
  dy.far[0] = (int32_t *)ctx->s_g.get(sizeof(int32_t) * (2 * n + 16));
  dy.far[1] = dy.far[0] + n + 8;
  dy.buf[0] = f.F;
  dy.buf[1] = f.Fout;
  dy.s = (SsspDev *)ctx->s_e.get(sizeof(SsspDev));
  const bool owned = source >= G.row_begin && source < G.row_begin + G.n_rows;
  SsspDev h{};
  h.nF = owned && !dy.bits ? 1 : 0;
  h.thr = h.delta = sssp_delta();
  INL_CUDA(cudaMemcpyAsync(dy.s, &h, sizeof h, cudaMemcpyHostToDevice, st));
  const int32_t s0 = (int32_t)(owned ? source - G.row_begin : 0);
  if (dy.bits) {  // the source's bit in C = inq[0]
    if (owned) {
      uint32_t *hw = (uint32_t *)ctx->pinned;
      hw[0] = 1u << (s0 & 31);
      INL_CUDA(cudaMemcpyAsync(dy.inq[0] + (s0 >> 5), hw, sizeof(uint32_t), cudaMemcpyHostToDevice, st));
    }
  } else {
    INL_CUDA(cudaMemcpyAsync(f.F, &s0, sizeof(int32_t), cudaMemcpyHostToDevice, st));
  }
  k_init_sssp<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(dist, n, source);
  INL_CUDA(cudaGetLastError());
  const ExpandCfg c = expand_cfg(G, b);
  ExpandArgs a{f.F, 0, G.row_ptr, G.col_idx, c.t_thread, c.t_warp, c.t_block, c.chunk,
               f.gitems, nullptr, (int)f.gcap, f.counts + 2, f.Fout, nullptr, f.relaxed};
  a.dyn = dy;
  SsspOp op{dist, w, nullptr, nullptr, 0, 0, true, 0, 0, nullptr, nullptr, nullptr};
  static int gm[3] = {2, 6, 8};  // split, flat, grid CTAs per SM (sweep: profiles/r02/sssp_bitmap_sweeps.txt)
  static bool gm_read = false;
  if (!gm_read) {
    gm_read = true;
    if (const char *e = getenv("INL_SSSP_GRIDS")) sscanf(e, "%d,%d,%d", &gm[0], &gm[1], &gm[2]);
  }
  SsspGraphKey key{};
  key.rp = G.row_ptr;
  key.col = G.col_idx;
  key.w = w;
  key.dist = dist;
  void *bufs[6] = {dy.s, dy.far[0], bits, f.F, f.Fout, f.gitems};
  memcpy(key.bufs, bufs, sizeof bufs);
  key.n = n;
  key.nnz = G.nnz;
  key.gcap = f.gcap;
  key.t_warp = c.t_warp;
  key.chunk = c.chunk;
  key.gm0 = gm[0];
  key.gm1 = gm[1];
  key.gm2 = gm[2];
  key.delta = h.delta;
  key.bits = dy.bits;
  const char *trace_path = getenv("INL_SSSP_TRACE");
  unsigned long long *trace = nullptr;
  if (trace_path && dy.bits) {
    trace = (unsigned long long *)ctx->s_t.get(sizeof(unsigned long long) * (kTraceSlots * kTraceSteps + 1));
    INL_CUDA(cudaMemsetAsync(trace, 0, sizeof(unsigned long long) * (kTraceSlots * kTraceSteps + 1), st));
    // the improvement counter (one same-address atomic per warp-call) slows the step kernels
    // severalfold, so it is on only with INL_SSSP_TRACE_MARKS (counts from one run, times from another)
    if (getenv("INL_SSSP_TRACE_MARKS")) op.tmark = trace + kTraceSlots * kTraceSteps;
  }
  key.trace = trace;
  SsspGraph *sg = static_cast<SsspGraph *>(ctx->sssp_graph);
  if (!sg || !(sg->key == key)) {
    delete sg;
    ctx->sssp_graph = sg = new SsspGraph();
    sg->key = key;
    INL_CUDA(cudaGraphCreate(&sg->graph, 0));
    cudaGraphConditionalHandle cond;
    INL_CUDA(cudaGraphConditionalHandleCreate(&cond, sg->graph, 1, cudaGraphCondAssignDefault));
    cudaGraphNodeParams cp{};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = cond;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t node;
    INL_CUDA(cudaGraphAddNode(&node, sg->graph, nullptr, 0, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    // the body: captured into the conditional node's graph on a private stream (the ctx
    // stream may be the legacy default stream, which cannot capture); it runs on the ctx stream
    cudaStream_t cap = nullptr;
    INL_CUDA(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
    cudaError_t ce = cudaStreamBeginCaptureToGraph(cap, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal);
    if (ce == cudaSuccess) {
      const int gsplit = ctx->num_sms * gm[0], gflat = ctx->num_sms * gm[1], ggrid = ctx->num_sms * gm[2];
      if (dy.bits) {
        const int64_t nv = nwb / 4;
        int gc = (int)std::min<int64_t>((nv + kCompactNT - 1) / kCompactNT, (int64_t)ctx->num_sms * 8);
        auto tr = [&](int slot) {
          if (trace) k_sssp_trace<<<1, 1, 0, cap>>>(dy.s, trace, slot, f.relaxed, op.tmark);
        };
        tr(0);
        k_sssp_bcompact<<<gc < 1 ? 1 : gc, kCompactNT, 0, cap>>>(dy);
        tr(1);
        k_sssp_bsplit<<<gc < 1 ? 1 : gc, kCompactNT, 0, cap>>>(dy, dist);
        tr(2);
        SsspBitsOp bop;
        static_cast<SsspOp &>(bop) = op;
        k_expand_flat<SsspBitsOp><<<gflat, NT, 0, cap>>>(a, bop);
        tr(3);
        k_expand_grid<SsspBitsOp><<<ggrid, NT, 0, cap>>>(a, bop);
        tr(4);
        k_sssp_bpost<<<1, 1, 0, cap>>>(dy, cond, 1);
        tr(5);
      } else {
        k_sssp_split<<<gsplit, 256, 0, cap>>>(dy, dist);
        k_expand_flat<SsspOp><<<gflat, NT, 0, cap>>>(a, op);
        k_expand_grid<SsspOp><<<ggrid, NT, 0, cap>>>(a, op);
        k_sssp_post<<<1, 1, 0, cap>>>(dy, cond, 1);
      }
      cudaGraph_t captured = nullptr;
      ce = cudaStreamEndCapture(cap, &captured);
    }
    cudaStreamDestroy(cap);
    if (ce != cudaSuccess) {
      ctx->sssp_graph = nullptr;
      delete sg;
    }
    INL_CUDA(ce);
    INL_CUDA(cudaGraphInstantiate(&sg->exec, sg->graph, 0));
  }
  {
    KScope ks(ctx, "sssp_graph");
    INL_CUDA(cudaGraphLaunch(sg->exec, st));
  }
  SsspDev *hs = (SsspDev *)ctx->pinned;
  INL_CUDA(cudaMemcpyAsync(hs, dy.s, sizeof(SsspDev), cudaMemcpyDeviceToHost, st));
  ctx_sync(ctx);
  if (((volatile SsspDev *)hs)->done == 2)
    raise(INL_ERR_INTERNAL, "sssp graph loop exceeded its step bound");
  if (trace) {  // measurement only: append this call's per-step trace to the file
    const int steps = std::min(hs->pad + 1, kTraceSteps);
    std::vector<unsigned long long> h((size_t)steps * kTraceSlots);
    INL_CUDA(cudaMemcpy(h.data(), trace, h.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost));
    if (FILE *fp = fopen(trace_path, "a")) {
      fprintf(fp, "# source %lld\n", (long long)source);
      for (int i = 0; i < steps; ++i) {
        const unsigned long long *r = &h[(size_t)i * kTraceSlots];
        fprintf(fp, "%d", i);
        for (int k = 0; k < 6; ++k) fprintf(fp, " %llu", r[k]);
        fprintf(fp, " %u %u", (unsigned)(r[6] & 0xffffffffu), (unsigned)(r[6] >> 32));
        for (int k = 7; k < 12; ++k) fprintf(fp, " %llu", r[k]);
        fprintf(fp, "\n");
      }
      fclose(fp);
    }
  }
  check_overflow(ctx, f);
  if (stats) {
    unsigned long long r = 0;
    INL_CUDA(cudaMemcpyAsync(&r, f.relaxed, sizeof r, cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    stats->iterations = hs->iter;
    stats->edges_relaxed = (int64_t)r;
    stats->frontier_total = (int64_t)hs->ftotal;
    stats->launches = 1 + (dy.bits ? 5LL : 4LL) * hs->pad;  // init + 4 or 5 kernels per step (one graph launch)
    stats->host_syncs = 1;
    stats->exchange_bytes = 0;
  }
}

void sssp_run(inl_ctx ctx, const inl_csr &G, const Bins &b, const uint32_t *w, int64_t source,
              uint32_t *dist, inl_stats *stats) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  const bool DIST = has_comm(ctx);  // row-block mode with an exchange (NCCL or loopback; also P = 1)
  // One GPU, near-far: by default the whole step loop is ONE CUDA-graph launch (sssp_run_graph,
  // 7.40 vs 7.84 ms per scale-23 source for the host-driven loop, profiles/r02/sssp_loops.txt).
  // INL_SSSP_LOOP=host (the r01 default: one host round trip per step) or =dyn (device loop,
  // host polling every 4-16 steps) select the others for measurement; INL_BINS_SSSP_DEVLOOP
  // forces a device loop even then.
  const char *lp = getenv("INL_SSSP_LOOP");
  const bool host_loop = lp && std::string(lp) == "host" && !(b.flags & INL_BINS_SSSP_DEVLOOP);
  const bool dyn_loop = lp && std::string(lp) == "dyn";
  if (!DIST && !(b.flags & (INL_BINS_THREAD_ONLY | kTemplateFlags)) && !host_loop && sssp_delta() != 0xFFFFFFFFu &&
      n > 0) {
    if (dyn_loop) sssp_run_dyn(ctx, G, b, w, source, dist, stats);
    else sssp_run_graph(ctx, G, b, w, source, dist, stats);
    return;
  }
  FrontierBufs f = frontier_bufs(ctx, G, b);
  INL_CUDA(cudaMemsetAsync(f.relaxed, 0, sizeof(unsigned long long), st));
  uint32_t *D = dist;
  uint32_t *prev = nullptr;
  uint32_t *inq = nullptr, *keep = nullptr;
  const int64_t nwb = (n + 31) / 32 + 1;
  int32_t *far_a = nullptr, *far_b = nullptr;
  int *farcnt = nullptr;
  int nfar = 0;
  uint32_t delta = 0xFFFFFFFFu, thr = 0xFFFFFFFFu;
  // P > 1 exchange: NEXT-1 sparse owner updates (default) or the r01 dense allreduce-min of the
  // whole distance vector (INL_SSSP_EXCHANGE=dense, measurement switch)
  const char *xe = getenv("INL_SSSP_EXCHANGE");
  const bool xsparse = DIST && n > 0 && !(xe && std::string(xe) == "dense");
  const int P = DIST ? ctx->nranks : 1;
  const int64_t Bk = (n + P - 1) / P;
  const int64_t xw = ((n + 31) / 32 + 31) / 32 * 32;  // words per changed-bitmap (128-B aligned)
  const int64_t dlen = (Bk * P + 31) / 32 * 32;      // padded replicated distance vector
  uint32_t *xchg = nullptr, **xtab = nullptr;
  unsigned int *nimp = (unsigned int *)(f.counts + 3);
  unsigned long long *xops = (unsigned long long *)(f.counts + 12);  // remote atomics (exchange volume)
  int64_t xbytes = 0;  // exchange bytes of the collectives (ring model)
  if (xsparse) {
    // one exchange buffer: [distances (dlen)] [3 changed-bitmaps (xw each), round r uses r % 3]
    const size_t bytes = sizeof(uint32_t) * ((size_t)dlen + 3 * (size_t)xw);
    D = (uint32_t *)ctx->s_xch.get(bytes);
    xchg = D + dlen;
    INL_CUDA(cudaMemsetAsync(xchg, 0, sizeof(uint32_t) * 3 * (size_t)xw, st));
    const std::vector<void *> &bases = comm_peer_bases(ctx, ctx->s_xch.p, ctx->s_xch.bytes);
    std::vector<uint32_t *> tab((size_t)4 * P);  // [0]: distances, [1 + r]: changed-bitmap r
    for (int q = 0; q < P; ++q) {
      tab[q] = (uint32_t *)bases[q];
      for (int r = 0; r < 3; ++r) tab[(size_t)(1 + r) * P + q] = (uint32_t *)bases[q] + dlen + (size_t)r * xw;
    }
    xtab = (uint32_t **)ctx->s_xtab.get(sizeof(uint32_t *) * tab.size());
    INL_CUDA(cudaMemcpyAsync(xtab, tab.data(), sizeof(uint32_t *) * tab.size(), cudaMemcpyHostToDevice, st));
    ctx_sync(ctx);
  } else if (DIST) {
    D = (uint32_t *)ctx->s_d.get(sizeof(uint32_t) * (n + 1));
    prev = (uint32_t *)ctx->s_e.get(sizeof(uint32_t) * (G.n_rows + 1));
  } else {
    inq = (uint32_t *)ctx->s_d.get(sizeof(uint32_t) * 2 * nwb);
    keep = inq + nwb;
    // far piles hold each vertex at most once (`keep` doubles as the in-far bitmap)
    far_a = (int32_t *)ctx->s_g.get(sizeof(int32_t) * (2 * n + 16));
    far_b = far_a + n + 8;
    farcnt = (int *)ctx->s_e.get(16);
    INL_CUDA(cudaMemsetAsync(farcnt, 0, 16, st));
    INL_CUDA(cudaMemsetAsync(keep, 0, sizeof(uint32_t) * nwb, st));
    // the baseline and the paper's templates run [5]'s plain frontier Bellman-Ford
    delta = b.flags & (INL_BINS_THREAD_ONLY | kTemplateFlags) ? 0xFFFFFFFFu : sssp_delta();
    thr = delta;
  }
  k_init_sssp<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(D, n, source);
  INL_CUDA(cudaGetLastError());
  int nF = 0;
  const bool owned = source >= G.row_begin && source < G.row_begin + G.n_rows;
  if (owned) {
    const int32_t s_local = (int32_t)(source - G.row_begin);
    INL_CUDA(cudaMemcpyAsync(f.F, &s_local, sizeof(int32_t), cudaMemcpyHostToDevice, st));
    nF = 1;
  }
  if (DIST && !xsparse) k_copy_u32<<<grid_for(G.n_rows, ctx->num_sms), 256, 0, st>>>(D + G.row_begin, prev, G.n_rows);
  if (xsparse) comm_barrier(ctx);  // every rank's distances / bitmaps are initialised before peers write
  int iters = 0;
  int64_t ftotal = 0;
  for (;;) {
    ftotal += nF;
    if (!DIST) {
      if (nF == 0) {  // near frontier exhausted: advance the threshold, pull in the far pile
        if (nfar == 0) break;
        const uint32_t lo = thr;
        thr = thr > 0xFFFFFFFFu - delta ? 0xFFFFFFFFu : thr + delta;
        INL_CUDA(cudaMemsetAsync(inq, 0, sizeof(uint32_t) * nwb, st));
        INL_CUDA(cudaMemsetAsync(keep, 0, sizeof(uint32_t) * nwb, st));
        INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
        INL_CUDA(cudaMemsetAsync(farcnt + 1, 0, sizeof(int), st));
        k_far_split<<<grid_for(nfar, ctx->num_sms), 256, 0, st>>>(far_a, nfar, D, lo, thr, inq, keep, f.F,
                                                                 f.counts, far_b, farcnt + 1);
        INL_CUDA(cudaGetLastError());
        INL_CUDA(cudaMemcpyAsync(ctx->pinned, f.counts, sizeof(int), cudaMemcpyDeviceToHost, st));
        INL_CUDA(cudaMemcpyAsync((int *)ctx->pinned + 1, farcnt + 1, sizeof(int), cudaMemcpyDeviceToHost, st));
        ctx_sync(ctx);
        nF = ((volatile int *)ctx->pinned)[0];
        nfar = ((volatile int *)ctx->pinned)[1];
        std::swap(far_a, far_b);
        INL_CUDA(cudaMemcpyAsync(farcnt, farcnt + 1, sizeof(int), cudaMemcpyDeviceToDevice, st));
        continue;
      }
      INL_CUDA(cudaMemsetAsync(inq, 0, sizeof(uint32_t) * nwb, st));
      SsspOp op{D, w, inq, nullptr, iters, 0, true, 0, thr, far_a, farcnt, keep};
      expand(ctx, G, b, f, nF, op);
      ++iters;
      INL_CUDA(cudaMemcpyAsync(ctx->pinned, f.counts, sizeof(int), cudaMemcpyDeviceToHost, st));
      INL_CUDA(cudaMemcpyAsync((int *)ctx->pinned + 1, farcnt, sizeof(int), cudaMemcpyDeviceToHost, st));
      ctx_sync(ctx);
      nF = ((volatile int *)ctx->pinned)[0];
      nfar = ((volatile int *)ctx->pinned)[1];
      std::swap(f.F, f.Fout);
    } else if (xsparse) {
      const int r = iters % 3;
      INL_CUDA(cudaMemsetAsync(xchg + (size_t)((iters + 1) % 3) * xw, 0, sizeof(uint32_t) * xw, st));
      INL_CUDA(cudaMemsetAsync(nimp, 0, sizeof(unsigned int), st));
      SsspOp op{D, w, nullptr, nullptr, iters, G.row_begin, false, 0, 0xFFFFFFFFu, nullptr, nullptr, nullptr};
      op.xd = xtab;
      op.xc = xtab + (size_t)(1 + r) * P;
      op.B = Bk;
      op.nimp = nimp;
      op.xops = xops;
      expand(ctx, G, b, f, nF, op);
      comm_allreduce(ctx, nimp, 1, ncclUint32, ncclSum);  // the round's barrier + termination test
      xbytes += 2 * (int64_t)(P - 1) * 4 / P;
      ++iters;
      INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
      k_sssp_collect_xbits<<<grid_for((G.n_rows + 31) / 32 + 1, ctx->num_sms), 256, 0, st>>>(
          xchg + (size_t)r * xw, G.row_begin, G.n_rows, f.F, f.counts);
      INL_CUDA(cudaGetLastError());
      INL_CUDA(cudaMemcpyAsync(ctx->pinned, f.counts, 16, cudaMemcpyDeviceToHost, st));
      ctx_sync(ctx);
      nF = ((volatile int *)ctx->pinned)[0];
      if (((volatile unsigned int *)ctx->pinned)[3] == 0u) break;
    } else {
      // flag word D[n] = 1 ("no change"), cleared by any improvement on any rank
      const uint32_t one = 1u;
      INL_CUDA(cudaMemcpyAsync(D + n, &one, sizeof(uint32_t), cudaMemcpyHostToDevice, st));
      SsspOp op{D, w, nullptr, D + n, iters, G.row_begin, false, 0, 0xFFFFFFFFu, nullptr, nullptr, nullptr};
      expand(ctx, G, b, f, nF, op);
      comm_allreduce(ctx, D, n + 1, ncclUint32, ncclMin);
      xbytes += 2 * (int64_t)(P - 1) * 4 * (n + 1) / P;
      ++iters;
      INL_CUDA(cudaMemcpyAsync(ctx->pinned, D + n, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
      ctx_sync(ctx);
      if (*(volatile uint32_t *)ctx->pinned == 1u) break;
      INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
      k_sssp_collect<<<grid_for(G.n_rows, ctx->num_sms), 256, 0, st>>>(D, prev, G.row_begin, G.n_rows,
                                                                      f.F, f.counts);
      INL_CUDA(cudaGetLastError());
      nF = read_count(ctx, f.counts);
    }
  }
  if (xsparse) {  // replicate: the owners' slices (in place, padded to P equal blocks)
    comm_allgather(ctx, D + (size_t)ctx->rank * Bk, D, Bk, ncclUint32, nullptr, nullptr);
    xbytes += 4 * Bk * (int64_t)(P - 1);
  }
  if (DIST)
    INL_CUDA(cudaMemcpyAsync(dist, D, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, st));
  finish_stats(ctx, f, stats, iters, ftotal, xbytes);
}

// The plan's static bottom-up bins (a3's degree binning applied to the bottom-up loop): every
// vertex of degree in (0, kBuThread] (thread bin), then every vertex of larger degree (warp bin),
// each in vertex order.  The first bottom-up level of a BFS reads them (skipping visited
// vertices) instead of partitioning all n vertices on the device at that level.
void bu_static_build(inl_plan p) {
  inl_ctx ctx = p->ctx;
  cudaStream_t st = ctx->stream;
  const int64_t n = p->n_global;
  p->bu_ns = p->bu_nl = 0;
  if (n < 4096 || n > INT32_MAX - 1) return;  // BFS takes bottom-up steps only from n >= 4096
  int32_t *lists = (int32_t *)p->bu_lists.get(sizeof(int32_t) * 2 * (size_t)n);
  int *cnt = (int *)ctx->s_f.get(64);
  thrust::counting_iterator<int32_t> iota(0);
  thrust::discard_iterator<> none;
  const BuDeg sm{p->row_ptr, 0, kBuThread}, lg{p->row_ptr, kBuThread, INT64_MAX};
  size_t need = 0;
  INL_CUDA(cub::DevicePartition::If(nullptr, need, iota, lists, lists + n, none, cnt, (int)n, sm, lg, st));
  INL_CUDA(cub::DevicePartition::If(ctx->s_tmp.get(need), need, iota, lists, lists + n, none, cnt, (int)n, sm, lg, st));
  int h[2] = {0, 0};
  INL_CUDA(cudaMemcpyAsync(h, cnt, sizeof h, cudaMemcpyDeviceToHost, st));
  INL_CUDA(cudaStreamSynchronize(st));
  p->bu_ns = h[0];
  p->bu_nl = h[1];
}

void bfs_run(inl_ctx ctx, const inl_csr &G, const Bins &b, int64_t source, int32_t *level,
             inl_stats *stats, bool symmetric, const BuStatic &bus) {
  cudaStream_t st = ctx->stream;
  const int64_t n = G.n_global;
  const bool DIST = has_comm(ctx);  // row-block mode with an exchange (NCCL or loopback; also P = 1)
  FrontierBufs f = frontier_bufs(ctx, G, b);
  INL_CUDA(cudaMemsetAsync(f.relaxed, 0, sizeof(unsigned long long), st));
  uint32_t *bm = (uint32_t *)ctx->s_d.get(sizeof(uint32_t) * ((n + 31) / 32 + 1));
  // P > 1 exchange: NEXT-1 bit-packed owner bitmaps (default) or the r01 byte map + allreduce-max
  // (INL_BFS_EXCHANGE=bytemap, measurement switch)
  const char *xe = getenv("INL_BFS_EXCHANGE");
  const bool xbits = DIST && !(xe && std::string(xe) == "bytemap");
  uint8_t *next = DIST && !xbits ? (uint8_t *)ctx->s_e.get(n + 1) : nullptr;
  k_init_bfs<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(level, bm, n, source);
  INL_CUDA(cudaGetLastError());
  const int P = DIST ? ctx->nranks : 1;
  const int64_t B = (n + P - 1) / P;
  const int64_t xw = ((n + 31) / 32 + 31) / 32 * 32;  // words per level buffer (128-B aligned)
  uint32_t *xb = nullptr;
  uint32_t **xtab = nullptr;
  unsigned long long *xtotal = (unsigned long long *)(f.counts + 10);
  unsigned long long *xops = (unsigned long long *)(f.counts + 12);  // remote atomics (exchange volume)
  int64_t xbytes = 0;  // exchange bytes counted on the host (collectives, bitmap reads)
  if (xbits && n > 0) {
    // three level buffers (level L writes buffer L % 3; a rank clears buffer (L+1) % 3 before
    // its level-L expansion: every rank read it at level L-2, before the level L-1 barrier, and
    // peers write it only after the level-L barrier) — one barrier per level
    const size_t bytes = sizeof(uint32_t) * 3 * (size_t)xw;
    xb = (uint32_t *)ctx->s_xch.get(bytes);
    INL_CUDA(cudaMemsetAsync(xb, 0, bytes, st));
    const std::vector<void *> &bases = comm_peer_bases(ctx, ctx->s_xch.p, ctx->s_xch.bytes);
    std::vector<uint32_t *> tab((size_t)3 * P);
    for (int bb = 0; bb < 3; ++bb)
      for (int q = 0; q < P; ++q) tab[(size_t)bb * P + q] = (uint32_t *)bases[q] + (size_t)bb * xw;
    xtab = (uint32_t **)ctx->s_xtab.get(sizeof(uint32_t *) * tab.size());
    INL_CUDA(cudaMemcpyAsync(xtab, tab.data(), sizeof(uint32_t *) * tab.size(), cudaMemcpyHostToDevice, st));
    ctx_sync(ctx);  // `tab` is a host temporary
    comm_barrier(ctx);  // every rank's buffers are zero before any peer writes into them
  }
  int nF = 0;
  if (source >= G.row_begin && source < G.row_begin + G.n_rows) {
    const int32_t s_local = (int32_t)(source - G.row_begin);
    INL_CUDA(cudaMemcpyAsync(f.F, &s_local, sizeof(int32_t), cudaMemcpyHostToDevice, st));
    nF = 1;
  }
  int L = 0;
  int64_t ftotal = 0;
  // direction optimisation (Beamer et al.): bottom-up while the frontier holds more than
  // n / kBuEnter vertices, top-down again once it falls below n / kBuLeave
  const int64_t nwords = (n + 31) / 32;
  uint32_t *fa = nullptr, *fb = nullptr, *tdb = nullptr;  // tdb: top-down next-frontier bitmap
  bool bu = false;       // direction of the previous step
  bool queue_ok = true;  // f.F holds the frontier (else the bitmap fa does)
  // bottom-up scans a vertex's row for frontier parents: valid only when rows list the
  // predecessors too (a symmetric graph, verified by the plan)
  const bool allow_bu = symmetric && !(b.flags & (INL_BINS_THREAD_ONLY | kTemplateFlags)) && n >= 4096;
  // top-down steps with fire-and-forget marks (BfsOp::nbits) where the flat / grid kernels run
  // (INL_BFS_TD=atomic keeps the claim-by-atomicOr queue pushes, for A/B)
  static int td_env = -1;
  if (td_env < 0) {
    const char *e = getenv("INL_BFS_TD");
    td_env = e && std::string(e) == "atomic" ? 0 : 1;
  }
  const bool td_red = allow_bu && td_env == 1 && expand_cfg(G, b).flat;
  // Beamer's m_f (degree sum of the next frontier) and m_u (edges of unvisited vertices)
  unsigned long long *mfp = (unsigned long long *)(f.counts + 10);
  unsigned long long mf_next = 0;
  double m_u = (double)G.nnz;
  auto read_level = [&](int *nf, unsigned long long *mfn) {
    INL_CUDA(cudaMemcpyAsync(ctx->pinned, f.counts, 48, cudaMemcpyDeviceToHost, st));
    ctx_sync(ctx);
    *nf = ((volatile int *)ctx->pinned)[0];
    *mfn = *(volatile unsigned long long *)((int *)ctx->pinned + 10);
    m_u -= (double)*mfn;
  };
  // binned bottom-up worklists (thread / warp bins, current and next); INL_BFS_BU=word keeps
  // the one-thread-per-vertex word kernel (measurement switch)
  static int bu_word = -1;
  if (bu_word < 0) {
    const char *e = getenv("INL_BFS_BU");
    bu_word = e && std::string(e) == "word";
  }
  // thread bin: one lane per vertex (default) or 4-lane groups (INL_BFS_SMALL=group: coalesced
  // column loads, measured no faster — the frontier-bit probes, not the column loads, bound it)
  const char *bs_env = getenv("INL_BFS_SMALL");
  const bool bu_small_thread = !(bs_env && std::string(bs_env) == "group");
  int32_t *bl_s[2] = {nullptr, nullptr}, *bl_l[2] = {nullptr, nullptr};
  int n_small = 0, n_large = 0, bl_cur = 0;
  bool lists_ok = false;  // the worklists hold exactly the unvisited vertices of degree > 0
  if (allow_bu) {
    fa = (uint32_t *)ctx->s_g.get(sizeof(uint32_t) * 3 * (nwords + 1));
    tdb = fa + 2 * (nwords + 1);  // fixed: fa / fb swap roles every bottom-up level
    fb = fa + nwords + 1;
    if (!bu_word) {
      int32_t *L4 = (int32_t *)ctx->s_bu.get(sizeof(int32_t) * 4 * (size_t)(n + 1));
      for (int q = 0; q < 2; ++q) {
        bl_s[q] = L4 + (size_t)q * (n + 1);
        bl_l[q] = L4 + (size_t)(2 + q) * (n + 1);
      }
    }
  }
  for (;;) {
    ftotal += nF;
    if (!DIST) {
      if (nF == 0) break;
      // Beamer's switch: enter bottom-up when the frontier's edges exceed the unvisited
      // edges / 14 (or it holds > n/24 vertices), leave it below n/256 vertices
      static double alpha = -1.0, beta = -1.0;  // Beamer's alpha (14) and beta (24); INL_BFS_AB=a,b to measure
      if (alpha < 0.0) {
        alpha = 14.0, beta = 24.0;
        if (const char *e = getenv("INL_BFS_AB")) sscanf(e, "%lf,%lf", &alpha, &beta);
      }
      const bool want_bu = allow_bu && (bu ? nF > n / 256 : (nF > (int64_t)(n / beta) || (double)mf_next * alpha > (double)m_u));
      if (want_bu) {
        if (queue_ok) {  // frontier queue -> bitmap
          INL_CUDA(cudaMemsetAsync(fa, 0, sizeof(uint32_t) * nwords, st));
          k_queue_to_bitmap<<<grid_for(nF, ctx->num_sms), 256, 0, st>>>(f.F, nF, fa);
        }
        INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
        INL_CUDA(cudaMemsetAsync(mfp, 0, sizeof(unsigned long long), st));
        if (bu_word) {
          KScope ks(ctx, "k_bfs_bottom_up");
          k_bfs_bottom_up<<<ctx->num_sms * 8, 256, 0, st>>>(G.row_ptr, G.col_idx, n, bm, fa, fb, level, L,
                                                           f.counts, mfp);
          INL_CUDA(cudaGetLastError());
          read_level(&nF, &mf_next);
        } else {
          const bool from_static = !lists_ok && bus.s;  // the plan's degree bins, visited ones skipped
          if (from_static) {
            n_small = (int)bus.ns;
            n_large = (int)bus.nl;
            bl_cur = 0;
            lists_ok = true;
          }
          if (!lists_ok) {  // entering bottom-up: the unvisited vertices, binned by degree
            thrust::counting_iterator<int32_t> iota(0);
            size_t need = 0;
            const BuBin sm{G.row_ptr, bm, 0, kBuThread}, lg{G.row_ptr, bm, kBuThread, INT64_MAX};
            thrust::discard_iterator<> none;
            INL_CUDA(cub::DevicePartition::If(nullptr, need, iota, bl_s[0], bl_l[0], none, f.counts + 4, (int)n, sm, lg, st));
            INL_CUDA(cub::DevicePartition::If(ctx->s_tmp.get(need), need, iota, bl_s[0], bl_l[0], none, f.counts + 4,
                                              (int)n, sm, lg, st));
            INL_CUDA(cudaMemcpyAsync(ctx->pinned, f.counts + 4, 2 * sizeof(int), cudaMemcpyDeviceToHost, st));
            ctx_sync(ctx);
            n_small = ((volatile int *)ctx->pinned)[0];
            n_large = ((volatile int *)ctx->pinned)[1];
            bl_cur = 0;
            lists_ok = true;
          }
          INL_CUDA(cudaMemsetAsync(fb, 0, sizeof(uint32_t) * nwords, st));
          INL_CUDA(cudaMemsetAsync(f.counts + 6, 0, 2 * sizeof(int), st));
          const int32_t *in_s = from_static ? bus.s : bl_s[bl_cur], *in_l = from_static ? bus.l : bl_l[bl_cur];
          BuArgs ba{G.row_ptr, G.col_idx, fa, fb, bm, level, L, in_s, n_small, f.counts, mfp, 0, f.relaxed, from_static};
          if (n_small > 0) {
            if (bu_small_thread) {
              KScope ks(ctx, "k_bu_thread");
              // first-batch width: 2 (scale 26: 2.70 -> 2.50 ms per BFS; 4: 2.56, 1: 2.52; scale 23
              // within noise; profiles/r02/bfs_k1_sweep.txt); INL_BFS_K1 = 1 / 2 / 4 / 8 to measure
              static int k1 = -1;
              if (k1 < 0) k1 = getenv("INL_BFS_K1") ? atoi(getenv("INL_BFS_K1")) : 2;
              const int gb = (int)grid_for(n_small, ctx->num_sms);
              if (k1 == 1) k_bu_thread<1><<<gb, 256, 0, st>>>(ba);
              else if (k1 == 2) k_bu_thread<2><<<gb, 256, 0, st>>>(ba);
              else if (k1 == 4) k_bu_thread<4><<<gb, 256, 0, st>>>(ba);
              else k_bu_thread<8><<<gb, 256, 0, st>>>(ba);
            } else {
              KScope ks(ctx, "k_bu_small");
              k_bu_group<4, kBuThread, false><<<grid_for((int64_t)n_small * 4, ctx->num_sms), 256, 0, st>>>(ba, nullptr,
                                                                                                   nullptr);
            }
          }
          ba.in = in_l;
          ba.n_in = n_large;
          if (n_large > 0) {
            int32_t *deep = bl_l[bl_cur ^ 1];  // the next large list is written only after k_bu_deep
            INL_CUDA(cudaMemsetAsync(f.counts + 3, 0, sizeof(int), st));
            {
              KScope ks(ctx, "k_bu_warp");
              static int gsz = -1;  // INL_BFS_GROUP: group width of the warp bin (measurement)
              if (gsz < 0) gsz = getenv("INL_BFS_GROUP") ? atoi(getenv("INL_BFS_GROUP")) : kBuGroup;
              if (gsz == 1)
                k_bu_group<1, kBuGroupSpan, true><<<grid_for((int64_t)n_large, ctx->num_sms), 256, 0, st>>>(
                    ba, deep, f.counts + 3);
              else if (gsz == 2)
                k_bu_group<2, kBuGroupSpan, true><<<grid_for((int64_t)n_large * 2, ctx->num_sms), 256, 0, st>>>(
                    ba, deep, f.counts + 3);
              else if (gsz == 4)
                k_bu_group<4, kBuGroupSpan, true><<<grid_for((int64_t)n_large * 4, ctx->num_sms), 256, 0, st>>>(
                    ba, deep, f.counts + 3);
              else if (gsz == 8)
                k_bu_group<8, kBuGroupSpan, true><<<grid_for((int64_t)n_large * 8, ctx->num_sms), 256, 0, st>>>(
                    ba, deep, f.counts + 3);
              else if (gsz == 16)
                k_bu_group<16, kBuGroupSpan, true><<<grid_for((int64_t)n_large * 16, ctx->num_sms), 256, 0, st>>>(
                    ba, deep, f.counts + 3);
              else
                k_bu_group<kBuGroup, kBuGroupSpan, true><<<grid_for((int64_t)n_large * kBuGroup, ctx->num_sms), 256, 0,
                                                            st>>>(ba, deep, f.counts + 3);
            }
            KScope ks(ctx, "k_bu_deep");
            k_bu_deep<<<ctx->num_sms * 2, 256, 0, st>>>(ba, deep, f.counts + 3);
          }
          INL_CUDA(cudaGetLastError());
          // carry the vertices still without a parent over to the next level's lists
          const BuUnvisited un{bm};
          if (n_small > 0) {
            size_t need = 0;
            INL_CUDA(cub::DeviceSelect::If(nullptr, need, in_s, bl_s[bl_cur ^ 1], f.counts + 6, n_small, un, st));
            INL_CUDA(cub::DeviceSelect::If(ctx->s_tmp.get(need), need, in_s, bl_s[bl_cur ^ 1], f.counts + 6,
                                           n_small, un, st));
          }
          if (n_large > 0) {
            size_t need = 0;
            INL_CUDA(cub::DeviceSelect::If(nullptr, need, in_l, bl_l[bl_cur ^ 1], f.counts + 7, n_large, un, st));
            INL_CUDA(cub::DeviceSelect::If(ctx->s_tmp.get(need), need, in_l, bl_l[bl_cur ^ 1], f.counts + 7,
                                           n_large, un, st));
          }
          read_level(&nF, &mf_next);
          n_small = ((volatile int *)ctx->pinned)[6];
          n_large = ((volatile int *)ctx->pinned)[7];
          bl_cur ^= 1;
        }
        std::swap(fa, fb);
        queue_ok = false;
      } else {
        if (!queue_ok) {  // bitmap -> frontier queue
          INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
          k_bitmap_to_queue<<<grid_for(nwords, ctx->num_sms), 256, 0, st>>>(fa, n, f.F, f.counts);
          INL_CUDA(cudaGetLastError());
        }
        lists_ok = false;  // top-down visits vertices the worklists still hold
        BfsOp op{bm, level, nullptr, n, L, true, 0, G.row_ptr, allow_bu ? mfp : nullptr};  // m_f only when it decides
        INL_CUDA(cudaMemsetAsync(mfp, 0, sizeof(unsigned long long), st));
        // fire-and-forget marks pay for their bitmap clear + scan only on a heavy level (edges
        // of the frontier > nnz / 256: scale 26 2.30 -> 2.02 ms per BFS, the heaviest level
        // 1.70 -> 0.48 ms; on every level scale 23 lost 4%; divisors 16 / 64 / 256 / 1024:
        // profiles/r02/bfs_td_marks.txt); INL_BFS_TD_DIV to measure
        static double td_div = -1.0;
        if (td_div < 0.0) td_div = getenv("INL_BFS_TD_DIV") ? atof(getenv("INL_BFS_TD_DIV")) : 256.0;
        if (td_red && (double)mf_next * td_div > (double)G.nnz) {
          uint32_t *nb = tdb;
          INL_CUDA(cudaMemsetAsync(nb, 0, sizeof(uint32_t) * nwords, st));
          op.nbits = nb;
          op.mf = nullptr;
          expand(ctx, G, b, f, nF, op);  // clears the queue counter; no pushes
          k_bfs_next_queue<<<grid_for(nwords, ctx->num_sms), 256, 0, st>>>(nb, nwords, G.row_ptr, f.Fout, f.counts, mfp);
          INL_CUDA(cudaGetLastError());
        } else {
          expand(ctx, G, b, f, nF, op);
        }
        read_level(&nF, &mf_next);
        std::swap(f.F, f.Fout);
        queue_ok = true;
      }
      bu = want_bu;
      ++L;
    } else if (xbits) {  // NEXT-1: bits straight into the owners' buffers, one barrier per level
      const int buf = L % 3;
      INL_CUDA(cudaMemsetAsync(xb + (size_t)((L + 1) % 3) * xw, 0, sizeof(uint32_t) * xw, st));
      BfsOp op{bm, level, nullptr, n, L, false, 0};
      op.xtab = xtab + (size_t)buf * P;
      op.B = B;
      op.xself = xb + (size_t)buf * xw;
      op.xops = xops;
      expand(ctx, G, b, f, nF, op);
      // the apply reads every word of the level bitmap outside this rank's block from its owner
      xbytes += 4 * ((n + 31) / 32 - ((G.row_begin + G.n_rows + 31) / 32 - G.row_begin / 32));
      comm_barrier(ctx);
      INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
      INL_CUDA(cudaMemsetAsync(xtotal, 0, sizeof(unsigned long long), st));
      k_bfs_apply_xbits<<<grid_for((n + 31) / 32, ctx->num_sms), 256, 0, st>>>(xtab + (size_t)buf * P, B, n, bm, level,
                                                                                L, G.row_begin, G.n_rows, f.F, f.counts,
                                                                                xtotal);
      INL_CUDA(cudaGetLastError());
      INL_CUDA(cudaMemcpyAsync(ctx->pinned, f.counts, 48, cudaMemcpyDeviceToHost, st));
      ctx_sync(ctx);
      nF = ((volatile int *)ctx->pinned)[0];
      const unsigned long long tot = *(volatile unsigned long long *)((int *)ctx->pinned + 10);
      if (tot == 0) break;
      ++L;
    } else {
      INL_CUDA(cudaMemsetAsync(next, 0, n + 1, st));
      BfsOp op{bm, level, next, n, L, false, 0};
      expand(ctx, G, b, f, nF, op);
      comm_allreduce(ctx, next, n + 1, ncclUint8, ncclMax);
      xbytes += 2 * (int64_t)(P - 1) * (n + 1) / P;
      INL_CUDA(cudaMemcpyAsync(ctx->pinned, next + n, 1, cudaMemcpyDeviceToHost, st));
      ctx_sync(ctx);
      if (*(volatile uint8_t *)ctx->pinned == 0) break;
      INL_CUDA(cudaMemsetAsync(f.counts, 0, sizeof(int), st));
      k_bfs_apply<<<grid_for(n, ctx->num_sms), 256, 0, st>>>(next, n, level, bm, L, G.row_begin,
                                                            G.n_rows, f.F, f.counts);
      INL_CUDA(cudaGetLastError());
      nF = read_count(ctx, f.counts);
      ++L;
    }
  }
  finish_stats(ctx, f, stats, L, ftotal, xbytes);
}

}  // namespace inl
