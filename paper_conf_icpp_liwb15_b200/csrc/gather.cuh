// gather.cuh — the load-balanced irregular-nested-loop gather (SpMV, PageRank pull).
//
// Paper: the loop nest of Fig. 1(a) (P3@9300) — outer loop over CSR rows, inner
// loop over the row's nonzeros — with the load-balancing templates of Fig. 1(b,c):
// rows whose inner loop is short are thread-mapped; longer ones are deferred to a
// buffer and processed by a wider group of threads — in the same kernel
// (dbuf-shared, P5@3623) or spread over the grid (dbuf-global, P5@2721).
//
// B200 design.  Measured ceilings on B200 (scripts/microbench,
// profiles/): streaming col_idx+val alone runs at 6.7 TB/s, but every random
// x[col] gather costs one L1TEX wavefront per distinct 128-B line, ~1 per SM-cycle,
// so plain gathers cap SpMV at ~230 us on R-MAT scale 22.  Hence:
//  * HOT COLUMNS IN SHARED MEMORY: the plan ranks columns by in-degree and remaps the
//    n_hot most frequent ones (~53% of all gathers at scale 22) to slots of a
//    shared-memory copy of x (bank-conflict cost instead of one line per lane).
//  * ONE CTA PER SM, 32 WARPS, and every unit of work belongs to ONE WARP — no
//    CTA-wide barrier after the x_hot fill.  Work items (plan.cu): TILES =
//    contiguous row ranges (<= kTileRows rows) of rows of degree <= t_warp whose
//    nonzeros form one contiguous span (< 2*t_warp - 14 entries); CHUNKS = grid_chunk
//    pieces of rows of degree > t_warp cut at row-relative offsets (a warp streams a
//    chunk in passes of 2*t_warp - 32 entries).
//  * Per item: 256-bit evict-first loads of the (remapped) col_idx and val span,
//    the gathers (smem for hot, read-only path with L2 evict-last for cold), the
//    products staged in a per-warp shared buffer; then THREAD bin: a lane sums its
//    row serially (degree <= t_thread); WARP bin: rows above t_thread are deferred
//    in a ballot mask (the shared delayed buffer of dbuf-shared, held in registers)
//    and summed by the warp (lane stride + xor tree).  A chunk is summed by the
//    warp; the last chunk of a row (atomic ticket) combines the partials in chunk
//    order (fp64).  Chunked rows of degree <= t_block are the BLOCK bin (their
//    pieces go to consecutive warps), longer ones the GRID bin.
//  * No float atomics: results are bit-identical run to run.  A row's summation order
//    depends on where its entries fall in the 8-entry lane groups and 256-entry passes of
//    its work item (aligned to the item's start), so a different row-block partition can
//    round fp32 sums differently (within the fp32 bound; integer-valued data stays exact).
//    DESIGN.md §3 reading R11.
#pragma once
#include <cuda/atomic>

#include "colblock.cuh"
#include "inl_internal.cuh"
#include "ptx.cuh"

namespace inl {

constexpr int kGatherWarps = 32;          // warps per CTA (1 CTA per SM)
constexpr int kSmemBudget = 224 * 1024;   // dynamic shared memory of the gather CTA
constexpr int kMaxHot = 32768;            // measured best x_hot size at scale 22 (128 KB)

constexpr int kTileSpan = 2048;  // target nonzeros per tile (tiles hold < kTileSpan + t_warp)
__host__ __device__ constexpr int tile_stride(int t_warp) { return kTileSpan; }

// Per-warp shared scratch of a tile: the non-empty rows in order (start offset within the
// tile span, local row id) and the row-start bitmap of the current 256-entry pass.
struct WarpTileSmem {
  short nzrow[kTileRows];
};

// hot slots that fit next to the per-warp tile scratch
inline int64_t hot_capacity(int t_warp) {
  (void)t_warp;
  int64_t b = kSmemBudget - (int64_t)kGatherWarps * (int64_t)sizeof(WarpTileSmem) - 2048;
  int64_t k = b / 4;
  if (k > kMaxHot) k = kMaxHot;
  return k < 0 ? 0 : (k & ~(int64_t)3);
}

// Epilogue for SpMV: y[r] = sum.
struct SpmvEpi {
  float *y;
  static constexpr bool kDangling = false;
  __device__ __forceinline__ void init() {}
  __device__ __forceinline__ double operator()(int64_t r, float s) const {
    y[r] = s;
    return 0.0;
  }
};

// Epilogue for one PageRank step (reading R1): PR'(v) = base + d * s(v) with
// base = (1-d)/n + d*D/n; writes the next contribution c'(v) = PR'(v)/outdeg(v)
// (0 for dangling pages) and, on the last step, the rank.  Returns PR'(v) for
// dangling pages so the warp can form its fixed-order partial of D'.
struct PrEpi {
  const int32_t *out_degree;  // [n_global]
  float *c_next;              // compacted contributions; this rank writes its own rows
  const int32_t *cidx;        // [n_global] compact (exchange-space) index of v, -1 if dangling
  float *rank_out;            // [n_global] or nullptr
  const float *base_ptr;      // device scalar
  float damping;
  int64_t row_begin;
  float base;
  static constexpr bool kDangling = true;
  __device__ __forceinline__ void init() { base = *base_ptr; }
  __device__ __forceinline__ double operator()(int64_t r, float s) const {
    const int64_t v = row_begin + r;
    const float pr = fmaf(damping, s, base);
    const int od = __ldg(out_degree + v);  // L1-cached: neighbouring rows share lines
    if (od > 0) c_next[__ldg(cidx + v)] = pr / (float)od;
    if (rank_out) rank_out[v] = pr;
    return od == 0 ? (double)pr : 0.0;
  }
};

struct GatherArgs {
  const int64_t *row_ptr;
  const int32_t *col_idx;  // the plan's remapped copy (hot entries 0x80000000 | h)
  const float *val;        // nullptr => implicit 1 (PageRank pull)
  const float *x;
  int64_t nnz, n_rows;
  int t_thread, t_warp, t_block, chunk;
  bool vec;  // col_idx / val 32-B aligned: 256-bit loads allowed
};

struct GatherPlan {
  const WorkItem *items;
  int n_items;
  float *partials;
  int *tickets;
  double *dpart;        // [n_items] or nullptr
  const float *x_hot;   // [n_hot]
  int n_hot;
  const uint32_t *rs_bits;  // [nnz/32 + 1] bit k set iff entry k starts a non-empty row
  const uint32_t *tile_nz;  // [n_tiles * 8] non-empty-row masks of the tiles
  unsigned long long *ticket;  // work counter (monotone across launches)
  unsigned long long base;     // its value at the start of this launch
};


// x[c] for a remapped column: hot slots (c = 0x80000000 | slot) from shared memory at
// xs + (c << 2) (the shift drops the tag bit), cold columns from global memory
// (ld.global.cg: cold columns have no L1 reuse).  Two complementary predicated loads into
// ONE register: no select.
__device__ __forceinline__ float gx(int32_t c, uint32_t xs_base, const float *x, uint64_t pol) {
  float r;
  asm("{\n\t"
      ".reg .pred h;\n\t"
      ".reg .b32 sa;\n\t"
      ".reg .b64 ga;\n\t"
      "setp.lt.s32 h, %1, 0;\n\t"
      "shl.b32 sa, %1, 2;\n\t"
      "add.u32 sa, sa, %2;\n\t"
      "mad.wide.s32 ga, %1, 4, %3;\n\t"
      "@h ld.shared.f32 %0, [sa];\n\t"
#if defined(INL_GX_NA)
      "@!h ld.global.nc.L1::no_allocate.f32 %0, [ga];\n\t"
#elif defined(INL_GX_NC)
      "@!h ld.global.nc.f32 %0, [ga];\n\t"
#elif defined(INL_GX_EL)
      "@!h ld.global.cg.L2::cache_hint.f32 %0, [ga], %4;\n\t"
#else  // cache-global (L2 only): measured 4% faster than the read-only path (profiles/r01)
      "@!h ld.global.cg.f32 %0, [ga];\n\t"
#endif
      "}"
      : "=f"(r)
      : "r"(c), "r"(xs_base), "l"(x), "l"(pol));
  return r;
}

// L2 prefetch of entries [lo, hi) of the col/val streams (short range: one pass ahead keeps
// the in-flight prefetch of all 4.7K warps at ~10 MB, far below the 126 MB L2).
template <bool VALS>
__device__ __forceinline__ void prefetch_entries(const GatherArgs &a, int64_t lo, int64_t hi) {
  prefetch_span(a.col_idx + lo, a.col_idx + hi, a.col_idx + a.nnz);
  if (VALS) prefetch_span(a.val + lo, a.val + hi, a.val + a.nnz);
}

template <bool VALS>
__device__ __forceinline__ void prefetch_item(const GatherArgs &a, const WorkItem &it) {
  prefetch_entries<VALS>(a, it.s, min(it.e, it.s + 256));
}

// Stream registers of one pass: lane l holds the (remapped) columns of entries
// q0 .. q0+E-1 of the item span and the 32-bit word of the row-start bit array that
// covers them (double-buffered: they feed the gathers); the values are single-buffered
// (loaded once the current pass's products are formed).
template <int E>
struct ColRegs {
  uint32_t cv[E];
  uint32_t fw;
};

// Lanes whose group lies wholly outside the item load nothing (their entries are masked
// before use).
template <int E>
__device__ __forceinline__ void load_cols(const GatherArgs &a, const uint32_t *rs_bits, int64_t s, int len,
                                          int q0, ColRegs<E> &r, uint64_t pol_ef) {
  const int64_t k0 = s + q0;  // E-aligned, >= 0
  if (q0 >= len || q0 + E <= 0) return;
  r.fw = ld_stream_pol(rs_bits + (k0 >> 5), pol_ef);
  if (a.vec && k0 + E <= a.nnz) {
#pragma unroll
    for (int h = 0; h < E / 8; ++h) {
      const U32x8 c = ld_stream_256(a.col_idx + k0 + 8 * h);
#pragma unroll
      for (int j = 0; j < 8; ++j) r.cv[8 * h + j] = c.v[j];
    }
  } else {
#pragma unroll
    for (int j = 0; j < E; ++j) r.cv[j] = ld_stream_pred(a.col_idx + k0 + j, (unsigned)(q0 + j) < (unsigned)len);
  }
}

template <int E>
__device__ __forceinline__ void load_vals(const GatherArgs &a, int64_t s, int len, int q0, float (&vv)[E]) {
  const int64_t k0 = s + q0;
  if (q0 >= len || q0 + E <= 0) return;
  if (a.vec && k0 + E <= a.nnz) {
#pragma unroll
    for (int h = 0; h < E / 8; ++h) {
      const U32x8 v = ld_stream_256(a.val + k0 + 8 * h);
#pragma unroll
      for (int j = 0; j < 8; ++j) vv[8 * h + j] = __uint_as_float(v.v[j]);
    }
  } else {
#pragma unroll
    for (int j = 0; j < E; ++j)
      vv[j] = __uint_as_float(ld_stream_pred(a.val + k0 + j, (unsigned)(q0 + j) < (unsigned)len));
  }
}

// The first pass of an item starts at p0 = -(s mod E) (E-entry aligned groups); a pass
// is 32*E consecutive entries, lane l takes entries E*l .. E*l+E-1 of it, summed serially
// then across lanes — tiles and chunks take the same path.
template <int E>
__device__ __forceinline__ int first_p0(const WorkItem &it) { return -(int)(it.s & (E - 1)); }

template <int E, bool VALS, class Epi, int NWARP = 256 / E>
__global__ void __launch_bounds__(NWARP * 32, 1) k_gather(GatherPlan gp, GatherArgs a, Epi epi) {
  // NWARP: 32 warps for E = 8 (64 registers), 24 (85 registers) or 16 for E = 16
  constexpr int P = 32 * E;                     // entries per pass
  constexpr unsigned EM = E == 32 ? 0xffffffffu : ((1u << E) - 1u);
  extern __shared__ __align__(128) unsigned char smem_raw[];
  float *xs = reinterpret_cast<float *>(smem_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __shared__ WarpTileSmem ws_all[NWARP];
  WarpTileSmem &ws = ws_all[warp];
  const int gw = blockIdx.x * NWARP + warp, nwarps = gridDim.x * NWARP;
  if (lane == 0 && gw < gp.n_items) prefetch_item<VALS>(a, gp.items[gw]);
  for (int i = threadIdx.x * 4; i < gp.n_hot; i += NWARP * 32 * 4)
    *reinterpret_cast<float4 *>(xs + i) = __ldg(reinterpret_cast<const float4 *>(gp.x_hot + i));
  if (threadIdx.x == 0) xs[gp.n_hot] = 0.0f;  // the zero slot (masked entries gather it)
  __syncthreads();
  epi.init();
  const uint32_t xs_base = smem_u32(xs);
  const uint32_t ZS = 0x80000000u | (uint32_t)gp.n_hot;  // remapped column of the zero slot
  const uint64_t pol_ef = policy_evict_first();  // plan metadata streams (row-start bits, masks)
#if defined(INL_GX_EL)
  const uint64_t pol = policy_evict_last();
#else
  const uint64_t pol = 0;
#endif
  const unsigned lt = (1u << lane) - 1u;
  const unsigned le = 0xffffffffu >> (31 - lane);
  if (gw >= gp.n_items) return;

  // dynamic schedule: a warp's first item is gw, later ones come from the work counter
  // (items are ordered longest-first by the plan, so the tail is made of short tiles)
  auto grab = [&]() -> int {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(gp.ticket, 1ull) - gp.base;
    t = __shfl_sync(0xffffffffu, t, 0);
    return (int)min(t + (unsigned long long)nwarps, (unsigned long long)gp.n_items);
  };
  int idx = gw;
  WorkItem it = gp.items[idx];
  int nidx = grab();
  int64_t ns = 0, ne = 0;  // the next item's span (its full descriptor is re-read at the switch)
  if (nidx < gp.n_items) {
    ns = gp.items[nidx].s;
    ne = gp.items[nidx].e;
  }
  // column registers of the next pass (a pass copies them, then refills them with the
  // loads of the pass after it); one value set (reloaded once a pass's products are formed)
  ColRegs<E> nx;
  float vv[E];
  load_cols<E>(a, gp.rs_bits, it.s, (int)(it.e - it.s), first_p0<E>(it) + E * lane, nx, pol_ef);
  if (VALS) load_vals<E>(a, it.s, (int)(it.e - it.s), first_p0<E>(it) + E * lane, vv);
  for (;;) {
    const int64_t s = it.s;
    const int len = (int)(it.e - s);
    const bool has_next = nidx < gp.n_items;
    const bool chunk = it.j >= 0;
    if (lane == 0 && has_next) prefetch_item<VALS>(a, gp.items[nidx]);
    double dacc = 0.0;
    int nnzr = 0;
    if (!chunk) {  // tile: non-empty rows -> list (plan masks); empty rows finish here (y = 0)
      const int nr = it.r1 - it.r0;
      const uint32_t *nzm = gp.tile_nz + 8 * (int64_t)it.t;
      for (int rb0 = 0; rb0 < nr; rb0 += 32) {
        const int r = rb0 + lane;
        const unsigned nz = ld_stream_pol(nzm + (rb0 >> 5), pol_ef);
        const bool ne = (nz >> lane) & 1u;
        if (ne) ws.nzrow[nnzr + __popc(nz & lt)] = (short)r;
        if (r < nr && !ne) dacc += epi(it.r0 + r, 0.0f);
        nnzr += __popc(nz);
      }
    } else {  // a chunk is one row: its only start is offset 0
      if (lane == 0) ws.nzrow[0] = 0;
    }
    __syncwarp();
    int kcur = 0;        // number of row starts consumed so far in this item
    int open_row = -1;   // local row open across the pass boundary
    float carry = 0.0f;  // its partial sum

    for (int p0 = first_p0<E>(it);; p0 += P) {  // >= 1 pass: it also hands the pipeline over
      ColRegs<E> cur = nx;
      const int q0 = p0 + E * lane;
      const bool more = p0 + P < len;
      // (1) the next pass's columns (same item, or the next item's first pass)
      if (more) load_cols<E>(a, gp.rs_bits, s, len, q0 + P, nx, pol_ef);
      else if (has_next)
        load_cols<E>(a, gp.rs_bits, ns, (int)(ne - ns), -(int)(ns & (E - 1)) + E * lane, nx, pol_ef);
      // (2) my E row-start flags; entries outside the item gather the zero slot
      unsigned fl = (cur.fw >> (int)((s + q0) & 31)) & EM;
      if (!(p0 >= 0 && p0 + P <= len)) {  // edge pass of the item (warp-uniform)
        const int lo = q0 < 0 ? -q0 : 0, hi = len - q0 < E ? len - q0 : E;
        fl = (lo < hi && hi > 0 && lo < E) ? fl & (EM << lo) & (EM >> (E - hi)) : 0u;
#pragma unroll
        for (int j = 0; j < E; ++j) {
          if ((unsigned)(q0 + j) >= (unsigned)len) {
            cur.cv[j] = ZS;
            vv[j] = 0.0f;
          }
        }
      }
      if (chunk && q0 <= 0 && q0 + E > 0) fl |= 1u << (-q0);  // a chunk (re)starts its row
      // (3) gathers
      float pr[E];
#pragma unroll
      for (int j = 0; j < E; ++j) {
        const float xv = gx((int32_t)cur.cv[j], xs_base, a.x, pol);
        pr[j] = VALS ? vv[j] * xv : xv;
      }
      if (VALS) {  // the next pass's values
        if (more) load_vals<E>(a, s, len, q0 + P, vv);
        else if (has_next) load_vals<E>(a, ns, (int)(ne - ns), -(int)(ns & (E - 1)) + E * lane, vv);
      }
      const int nf = __popc(fl);
      const unsigned fmask = __ballot_sync(0xffffffffu, nf != 0);
      const int kpass = kcur;
      float head = 0.0f, tail = 0.0f;
      int before;
      if (__any_sync(0xffffffffu, nf >= 2)) {
        // THREAD-mapped rows complete inside my segment are emitted here
        before = nf;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const int t = __shfl_up_sync(0xffffffffu, before, d);
          if (lane >= d) before += t;
        }
        kcur += __shfl_sync(0xffffffffu, before, 31);
        before -= nf;
        int rank = before - 1;
#pragma unroll
        for (int j = 0; j < E; ++j) {
          if (fl & (1u << j)) {
            if (rank < before) head = tail;  // first start: what came before belongs to the open row
            else dacc += epi(it.r0 + ws.nzrow[kpass + rank], tail);
            ++rank;
            tail = 0.0f;
          }
          tail += pr[j];
        }
        if (!fl) head = tail;
      } else {  // at most one start per lane (warp-bin rows and chunks): one serial chain
        before = __popc(fmask & lt);
        kcur += __popc(fmask);
#pragma unroll
        for (int j = 0; j < E; ++j) {
          const bool f = (fl >> j) & 1u;
          if (f) head = tail;
          tail = (f ? 0.0f : tail) + pr[j];
        }
        if (!fl) head = tail;
      }
      // WARP-mapped rows: segmented inclusive scan across lanes; a segment starts at the
      // last lane <= me holding a start (span = lanes below me in my segment)
      if (lane == 0) head += carry;
      const bool F = nf != 0;
      float S = F ? tail : head;
      const unsigned hm = fmask & le;
      const int span = hm ? lane - (31 - __clz(hm)) : lane;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const float t = __shfl_up_sync(0xffffffffu, S, d);
        if (span >= d) S += t;
      }
      float Ein = __shfl_up_sync(0xffffffffu, S, 1);  // value entering my segment
      if (lane == 0) Ein = 0.0f;
      if (F) {  // the row open at my segment start ends at my first start
        const int rr = before > 0 ? ws.nzrow[kpass + before - 1] : open_row;
        if (rr >= 0) dacc += epi(it.r0 + rr, Ein + head);
      }
      carry = __shfl_sync(0xffffffffu, S, 31);
      if (fmask) open_row = ws.nzrow[chunk ? 0 : kcur - 1];
      if (!more) break;
    }
    __syncwarp();
    // the row still open at the end of the item
    if (lane == 0 && open_row >= 0) {
      if (!chunk || it.nch == 1) {
        dacc += epi(it.r0 + open_row, carry);
      } else {  // grid bin: partial of chunk c; the last chunk to finish combines in order
        gp.partials[it.pbase + it.c] = carry;
        cuda::atomic_ref<int, cuda::thread_scope_device> tk(gp.tickets[it.j]);
        if (tk.fetch_add(1, cuda::memory_order_acq_rel) == it.nch - 1) {
          double tot = 0.0;  // partials combined in chunk order, fp64 accumulator
          for (int q = 0; q < it.nch; ++q) {
            cuda::atomic_ref<float, cuda::thread_scope_device> pq(gp.partials[it.pbase + q]);
            tot += (double)pq.load(cuda::memory_order_relaxed);
          }
          dacc += epi(it.r0, (float)tot);
          tk.store(0, cuda::memory_order_relaxed);  // ready for the next call
        }
      }
    }
    if (Epi::kDangling) {
      const double t = warp_sum_d(dacc);
      if (lane == 0) gp.dpart[idx] = t;
    }
    __syncwarp();
    if (!has_next) break;
    idx = nidx;
    it = gp.items[idx];
    nidx = grab();
    if (nidx < gp.n_items) {
      ns = gp.items[nidx].s;
      ne = gp.items[nidx].e;
    }
  }
}

// Long-row pieces alone (the grid / block bins of rows longer than t_warp; dbuf-global,
// P5@2721).  A piece is part of one row, so there is no row bookkeeping: a warp streams it in
// passes of 256 entries (lane l: entries 8l..8l+7) with the NEXT pass's columns and values in
// flight while this pass's gathers run (both double-buffered: this kernel has the registers
// the tile kernel spends on row tracking), sums the 8 products per lane, chains the pass sums
// per lane and reduces across the warp once per piece; the last piece of a row (acq_rel
// ticket) adds the row's partials in piece order in fp64, as k_gather does.  Worst-case
// rounding depth per piece: 8 + passes + 5 (relative error <= depth * 2^-24 for the
// non-negative data of the configs).  Runs before k_gather on items [0, n_chunks).
template <bool VALS, class Epi>
__global__ void __launch_bounds__(1024, 1) k_gather_chunks(GatherPlan gp, GatherArgs a, Epi epi) {
  constexpr int E = 8, P = 256;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  float *xs = reinterpret_cast<float *>(smem_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, NWARP = blockDim.x >> 5;
  const int gw = blockIdx.x * NWARP + warp, nwarps = gridDim.x * NWARP;
  for (int i = threadIdx.x * 4; i < gp.n_hot; i += blockDim.x * 4)
    *reinterpret_cast<float4 *>(xs + i) = __ldg(reinterpret_cast<const float4 *>(gp.x_hot + i));
  if (threadIdx.x == 0) xs[gp.n_hot] = 0.0f;
  __syncthreads();
  epi.init();
  const uint32_t xs_base = smem_u32(xs);
  const uint32_t ZS = 0x80000000u | (uint32_t)gp.n_hot;
  const uint64_t pol = 0;
  if (gw >= gp.n_items) return;
  auto grab = [&]() -> int {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(gp.ticket, 1ull) - gp.base;
    t = __shfl_sync(0xffffffffu, t, 0);
    return (int)min(t + (unsigned long long)nwarps, (unsigned long long)gp.n_items);
  };
  // columns (resp. values) of entries [k0, k0 + 8) of an item spanning [s, e); outside it the
  // zero slot (resp. 0)
  auto load_c = [&](int64_t s, int64_t e, int64_t k0, uint32_t (&cv)[E]) {
    if (a.vec && k0 >= s && k0 + E <= e) {
      const U32x8 c = ld_stream_256(a.col_idx + k0);
#pragma unroll
      for (int j = 0; j < E; ++j) cv[j] = c.v[j];
    } else {
#pragma unroll
      for (int j = 0; j < E; ++j) {
        const bool in = k0 + j >= s && k0 + j < e;
        const uint32_t c = ld_stream_pred(a.col_idx + k0 + j, in);
        cv[j] = in ? c : ZS;
      }
    }
  };
  auto load_v = [&](int64_t s, int64_t e, int64_t k0, float (&v)[E]) {
    if (a.vec && k0 >= s && k0 + E <= e) {
      const U32x8 w = ld_stream_256(a.val + k0);
#pragma unroll
      for (int j = 0; j < E; ++j) v[j] = __uint_as_float(w.v[j]);
    } else {
#pragma unroll
      for (int j = 0; j < E; ++j) {
        const bool in = k0 + j >= s && k0 + j < e;
        const float x = __uint_as_float(ld_stream_pred(a.val + k0 + j, in));
        v[j] = in ? x : 0.0f;
      }
    }
  };
  int idx = gw;
  int64_t is = gp.items[idx].s, ie = gp.items[idx].e;  // the rest of the descriptor is re-read at the end
  uint32_t cv[E];
  load_c(is, ie, (is & ~(int64_t)(E - 1)) + E * lane, cv);
  for (;;) {
    const int nidx = grab();
    const bool has_next = nidx < gp.n_items;
    int64_t ns = 0, ne = 0;
    if (has_next) {
      ns = gp.items[nidx].s;
      ne = gp.items[nidx].e;
    }
    const int64_t a0 = is & ~(int64_t)(E - 1);
    float acc = 0.0f;
    for (int64_t kb = a0;; kb += P) {
      // this pass's values (in flight with its gathers), the next pass's columns
      float vv[E];
      if (VALS) load_v(is, ie, kb + E * lane, vv);
      uint32_t cn[E];
      const bool more = kb + P < ie;
      if (more) load_c(is, ie, kb + P + E * lane, cn);
      else if (has_next) load_c(ns, ne, (ns & ~(int64_t)(E - 1)) + E * lane, cn);
      float ps = 0.0f;
#pragma unroll
      for (int j = 0; j < E; ++j) {
        const float xv = gx((int32_t)cv[j], xs_base, a.x, pol);
        ps += VALS ? vv[j] * xv : xv;
      }
      acc += ps;
#pragma unroll
      for (int j = 0; j < E; ++j) cv[j] = cn[j];
      if (!more) break;
    }
    const float tot = warp_sum(acc);
    if (lane == 0) {
      const WorkItem it = gp.items[idx];
      double dacc = 0.0;
      if (it.nch == 1) {
        dacc = epi(it.r0, tot);
      } else {
        gp.partials[it.pbase + it.c] = tot;
        cuda::atomic_ref<int, cuda::thread_scope_device> tk(gp.tickets[it.j]);
        if (tk.fetch_add(1, cuda::memory_order_acq_rel) == it.nch - 1) {
          double t = 0.0;  // partials combined in piece order, fp64 accumulator
          for (int q = 0; q < it.nch; ++q) {
            cuda::atomic_ref<float, cuda::thread_scope_device> pq(gp.partials[it.pbase + q]);
            t += (double)pq.load(cuda::memory_order_relaxed);
          }
          dacc = epi(it.r0, (float)t);
          tk.store(0, cuda::memory_order_relaxed);
        }
      }
      if (Epi::kDangling) gp.dpart[idx] = dacc;
    }
    __syncwarp();
    if (!has_next) break;
    idx = nidx;
    is = ns;
    ie = ne;
  }
}

// The paper's baseline (T1, P3@9322, P5@14490): one thread per row, serial inner
// loop, no load balancing.  Used only as the in-build comparator.
template <class Epi>
__global__ void __launch_bounds__(256) k_gather_thread_only(int64_t n_rows, GatherArgs a, Epi epi) {
  epi.init();
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n_rows;
       r += (int64_t)gridDim.x * blockDim.x) {
    float acc = 0.0f;
    for (int64_t k = a.row_ptr[r]; k < a.row_ptr[r + 1]; ++k)
      acc += (a.val ? a.val[k] : 1.0f) * a.x[a.col_idx[k]];
    epi(r, acc);
  }
}

// x_hot[h] = x[hot_cols[h]] (per call; zero-padded to a multiple of 4) — spmv.cu.
// hot_cols: NULL = the plan's list, else a list in another column space.
void build_xhot(inl_ctx ctx, inl_plan p, const float *x, const int32_t *hot_cols = nullptr, int64_t n_hot = -1);

template <int E, bool VALS, class Epi, int NWARP = 256 / E>
void launch_gather_t(inl_ctx ctx, const GatherPlan &gp, const GatherArgs &a, const Epi &epi, int max_ctas = 0) {
  const size_t smem = (size_t)gp.n_hot * 4 + 16;  // xs[0] is read (then discarded) by cold gathers
  auto kern = k_gather<E, VALS, Epi, NWARP>;
  static size_t configured[kMaxDevices] = {};  // per instantiation AND device (the attribute is per device)
  size_t &cf = configured[ctx->device % kMaxDevices];
  if (smem > cf) {
    INL_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    cf = smem;
  }
  int64_t grid = max_ctas > 0 && max_ctas < ctx->num_sms ? max_ctas : ctx->num_sms;
  const int64_t need = (gp.n_items + NWARP - 1) / NWARP;
  if (grid > need) grid = need;
  KScope ks(ctx, "k_gather");
  kern<<<(int)grid, NWARP * 32, smem, ctx->stream>>>(gp, a, epi);
  INL_CUDA(cudaGetLastError());
}

// INL_GATHER_SPLIT=1 (opt-in experiment): long-row pieces in k_gather_chunks, then the tiles in
// k_gather.  Default 0: every item in k_gather.  Measured at scale 22 (profiles/r02/
// spmv_chunk_split.txt): 74-91 us for the pieces + 134 us for the tiles vs 185-188 us for the
// fused kernel — both kernels gather at the same ~310 G entries/s, the L1TEX wavefront rate of
// the x gathers, so removing the row bookkeeping from the pieces buys nothing and the split
// loses the fused kernel's overlap of long and short items.
inline int gather_split() {
  static int v = -1;
  if (v < 0) {
    const char *e = getenv("INL_GATHER_SPLIT");
    v = e ? atoi(e) != 0 : 0;
  }
  return v;
}

template <bool VALS, class Epi>
void launch_gather_chunks(inl_ctx ctx, const GatherPlan &gp, const GatherArgs &a, const Epi &epi) {
  const size_t smem = (size_t)gp.n_hot * 4 + 16;
  auto kern = k_gather_chunks<VALS, Epi>;
  static size_t configured[kMaxDevices] = {};
  size_t &cf = configured[ctx->device % kMaxDevices];
  if (smem > cf) {
    INL_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    cf = smem;
  }
  int64_t grid = ctx->num_sms;
  const int64_t need = (gp.n_items + 31) / 32;
  if (grid > need) grid = need;
  KScope ks(ctx, "k_gather_chunks");
  kern<<<(int)grid, 1024, smem, ctx->stream>>>(gp, a, epi);
  INL_CUDA(cudaGetLastError());
}

inline int gather_entries_per_lane() {
  static int e = 0;
  if (!e) {  // 8 entries / lane with 32 warps measured best at scale 22 (16 / lane: 16 warps, slower)
    e = 8;
    if (const char *v = getenv("INL_GATHER_E")) e = atoi(v) == 16 ? 16 : 8;
  }
  return e;
}

// A sub-range of a plan's work items for one launch (PageRank's pipelined sub-blocks): items
// [items, items + n) write their dangling partials to dpart[0, n); max_ctas caps the grid
// (leaves SMs to a concurrent NCCL kernel); skip_xhot: x_hot is already current.
struct GatherRange {
  const WorkItem *items = nullptr;  // nullptr: every item of the plan
  int64_t n = 0;
  int max_ctas = 0;
  bool skip_xhot = false;
};

// Host-side launcher for one full gather (tiles + long-row chunks) on a plan; x is the
// dense vector (n_global) whose hot part is copied to the plan's x_hot first.
// col_over / hot_over: a column space other than the plan's (PageRank's compacted one).
// cb: the column-blocked bin of that column space (its rows leave the gather's items and
// are summed by k_cb + k_cb_combine; their dangling values go to dpart[n_items + j]).
template <bool VALS, class Epi>
void launch_gather(inl_ctx ctx, inl_plan p, const GatherArgs &a_in, const Epi &epi, double *dpart,
                   const int32_t *col_over = nullptr, const int32_t *hot_over = nullptr,
                   const CbPlan *cb = nullptr, int64_t n_hot_over = -1, const GatherRange *range = nullptr) {
  if (p->n_items == 0) return;
  const int64_t n_hot = n_hot_over >= 0 ? n_hot_over : p->n_hot;
  const bool use_cb = cb && cb->active;
  const bool ranged = range && range->items;
  const int64_t n_items = ranged ? range->n : use_cb ? cb->n_items : p->n_items;
  GatherArgs a = a_in;
  if (col_over) a.col_idx = col_over;
  else if (p->n_hot > 0) a.col_idx = (const int32_t *)p->pcol.p;  // hot columns remapped
  if (n_items > 0) {
    GatherPlan gp;
    gp.items = ranged ? range->items : (const WorkItem *)(use_cb ? cb->items.p : p->items.p);
    gp.n_items = (int)n_items;
    gp.partials = (float *)p->partials.p;
    gp.tickets = (int *)p->tickets.p;
    gp.dpart = dpart;
    gp.x_hot = (const float *)p->x_hot.p;
    gp.n_hot = (int)((n_hot + 3) & ~3);
    gp.rs_bits = (const uint32_t *)p->rs_bits.p;
    gp.tile_nz = (const uint32_t *)p->tile_nz.p;
    gp.ticket = (unsigned long long *)p->ticket.p;
    // each launch advances the counter by exactly n_items (successful grabs + one failing
    // grab per active warp), so the next launch's base is known on the host: no reset
    gp.base = p->ticket_base;
    if (!(ranged && range->skip_xhot)) build_xhot(ctx, p, a.x, hot_over, n_hot);
    a.vec = ((uintptr_t)a.col_idx % 32 == 0) && (!VALS || (uintptr_t)a.val % 32 == 0);
    static int w24 = -1;
    if (w24 < 0) w24 = getenv("INL_GATHER_W24") ? 1 : 0;
    const int mc = ranged ? range->max_ctas : 0;
    const int64_t n_split = (!ranged && !use_cb && gather_split()) ? p->n_chunks : 0;
    if (n_split > 0) {  // long-row pieces first, in their own kernel (items [0, n_chunks))
      GatherPlan gc = gp;
      gc.n_items = (int)n_split;
      launch_gather_chunks<VALS>(ctx, gc, a, epi);
      gp.items += n_split;
      gp.n_items -= (int)n_split;
      if (gp.dpart) gp.dpart += n_split;
      gp.base += (unsigned long long)n_split;
    }
    if (gp.n_items > 0) {
      if (gather_entries_per_lane() == 16) launch_gather_t<16, VALS>(ctx, gp, a, epi, mc);
      else if (w24) launch_gather_t<8, VALS, Epi, 24>(ctx, gp, a, epi, mc);
      else launch_gather_t<8, VALS>(ctx, gp, a, epi, mc);
    }
    p->ticket_base += (unsigned long long)n_items;  // only once the launch was accepted
  }
  if (use_cb && !ranged) launch_cb<VALS>(ctx, *cb, a_in.val, a_in.x, epi, dpart ? dpart + n_items : nullptr);
}

// number of dangling partials launch_gather writes
inline int64_t gather_dpart_count(inl_plan p, const CbPlan *cb) {
  return cb && cb->active ? cb->n_items + cb->n_rows : p->n_items;
}

}  // namespace inl
