/* inlgen_core.h — counter-based input recipe shared by the host and device
 * generators of the `inlgen` module (seeded synthetic inputs only).
 *
 * This header holds NO arithmetic of the paper's method (no SpMV, PageRank,
 * SSSP or BFS step): only the random draws that define the synthetic inputs.
 * Both the oracle side (tests/, bench.py cpu_baseline) and the CUDA side read
 * the inputs this module produces; neither side includes this header.
 *
 * Recipe (DESIGN.md §"Input recipe"):
 *   - Philox4x32-10 (Salmon et al., Random123), key = seed, counter =
 *     (index_lo, index_hi, sub, stream).  Identical on host and device.
 *   - R-MAT/Graph500 Kronecker edges with (A,B,C,D) = (.57,.19,.19,.05) as
 *     integer thresholds on the raw 32-bit draw (no float compare).
 *   - Vertex relabel: stateless bijection on [0, 2^scale).
 *   - SpMV values / x: U[0,1) = (r >> 8) * 2^-24 (exact in fp32), or small
 *     integers for the bit-exact integer mode.
 *   - SSSP weights: 1 + r mod 255, keyed by the unordered pair {u, v}.
 */
#ifndef INLGEN_CORE_H
#define INLGEN_CORE_H
#include <stdint.h>

#if defined(__CUDACC__)
#define IG_HD __host__ __device__ __forceinline__
#else
#define IG_HD static inline
#endif

enum {
  IG_STREAM_RMAT = 1,
  IG_STREAM_WEIGHT = 2,
  IG_STREAM_VALUE = 3,
  IG_STREAM_VECTOR = 4,
  IG_STREAM_RELABEL = 5,
  IG_STREAM_SOURCE = 6,
  IG_STREAM_PL_DEGREE = 7,  /* power-law degree sequence (loader.cpp) */
  IG_STREAM_PL_SHUFFLE = 8, /* its stub shuffle */
  IG_STREAM_TREE = 9        /* synthetic trees: does node v have children */
};

typedef struct { uint32_t v[4]; } ig_u32x4;

IG_HD uint32_t ig_mulhilo(uint32_t a, uint32_t b, uint32_t *hi) {
  uint64_t p = (uint64_t)a * (uint64_t)b;
  *hi = (uint32_t)(p >> 32);
  return (uint32_t)p;
}

/* Philox4x32 with 10 rounds; Random123 round/bump order. */
IG_HD ig_u32x4 ig_philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                         uint32_t k0, uint32_t k1) {
  const uint32_t M0 = 0xD2511F53u, M1 = 0xCD9E8D57u;
  const uint32_t W0 = 0x9E3779B9u, W1 = 0xBB67AE85u;
  for (int r = 0; r < 10; ++r) {
    if (r) { k0 += W0; k1 += W1; }
    uint32_t hi0, hi1;
    uint32_t lo0 = ig_mulhilo(M0, c0, &hi0);
    uint32_t lo1 = ig_mulhilo(M1, c2, &hi1);
    uint32_t n0 = hi1 ^ c1 ^ k0, n1 = lo1, n2 = hi0 ^ c3 ^ k1, n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  ig_u32x4 out;
  out.v[0] = c0; out.v[1] = c1; out.v[2] = c2; out.v[3] = c3;
  return out;
}

IG_HD uint32_t ig_draw(uint64_t seed, uint32_t stream, uint64_t index, uint32_t sub,
                       int word) {
  ig_u32x4 r = ig_philox((uint32_t)index, (uint32_t)(index >> 32), sub, stream,
                         (uint32_t)seed, (uint32_t)(seed >> 32));
  return r.v[word & 3];
}

/* Stateless bijection on [0, 2^scale): 4 rounds of (odd multiply + add) mod 2^s
 * followed by an xorshift-right; every step is invertible mod 2^s. */
IG_HD uint64_t ig_relabel(uint64_t x, int scale, uint64_t seed) {
  if (scale <= 0) return 0;
  const uint64_t mask = (scale >= 64) ? ~0ull : ((1ull << scale) - 1ull);
  const int sh = (scale + 1) / 2;
  for (uint32_t r = 0; r < 4; ++r) {
    ig_u32x4 k = ig_philox(r, 0, 0, IG_STREAM_RELABEL, (uint32_t)seed, (uint32_t)(seed >> 32));
    uint64_t a = (((uint64_t)k.v[0] << 32) | k.v[1]) | 1ull;
    uint64_t b = ((uint64_t)k.v[2] << 32) | k.v[3];
    x = (x * a + b) & mask;
    x ^= (x >> sh);
  }
  return x;
}

/* R-MAT quadrant thresholds: floor(p * 2^32) for p = .57, .76, .95 */
#define IG_RMAT_TA 2448131358u
#define IG_RMAT_TAB 3264175144u
#define IG_RMAT_TABC 4080218931u

/* Edge tuple e in [0, edge_factor * 2^scale): (u, v) before relabel. */
IG_HD void ig_rmat_edge(uint64_t seed, int scale, uint64_t e, uint64_t *u, uint64_t *v) {
  uint64_t uu = 0, vv = 0;
  ig_u32x4 r;
  r.v[0] = r.v[1] = r.v[2] = r.v[3] = 0;
  for (int l = 0; l < scale; ++l) {
    if ((l & 3) == 0)
      r = ig_philox((uint32_t)e, (uint32_t)(e >> 32), (uint32_t)(l >> 2), IG_STREAM_RMAT,
                    (uint32_t)seed, (uint32_t)(seed >> 32));
    uint32_t x = r.v[l & 3];
    uint64_t bu = (x >= IG_RMAT_TAB) ? 1u : 0u;                 /* C or D quadrant */
    uint64_t bv = (x >= IG_RMAT_TA && x < IG_RMAT_TAB) || (x >= IG_RMAT_TABC) ? 1u : 0u;
    uu |= bu << l;
    vv |= bv << l;
  }
  *u = uu;
  *v = vv;
}

/* SSSP weight in [1, 255], symmetric in (u, v). */
IG_HD uint32_t ig_weight(uint64_t seed, uint64_t u, uint64_t v) {
  uint64_t a = u < v ? u : v, b = u < v ? v : u;
  ig_u32x4 r = ig_philox((uint32_t)a, (uint32_t)(a >> 32) ^ ((uint32_t)(b >> 32) << 16), (uint32_t)b,
                         IG_STREAM_WEIGHT, (uint32_t)seed, (uint32_t)(seed >> 32));
  return 1u + r.v[0] % 255u;
}

/* Matrix value for entry (row, col). mode 0: U[0,1); mode 1: integer 1..255. */
IG_HD float ig_value(uint64_t seed, uint64_t row, uint64_t col, int mode) {
  ig_u32x4 r = ig_philox((uint32_t)row, (uint32_t)(row >> 32) ^ ((uint32_t)(col >> 32) << 16),
                         (uint32_t)col, IG_STREAM_VALUE, (uint32_t)seed, (uint32_t)(seed >> 32));
  if (mode == 1) return (float)(1u + r.v[0] % 255u);
  return (float)(r.v[0] >> 8) * (1.0f / 16777216.0f);
}

/* Dense vector element i. mode 0: U[0,1); mode 1: integer 0..15. */
IG_HD float ig_vector(uint64_t seed, uint64_t i, int mode) {
  ig_u32x4 r = ig_philox((uint32_t)i, (uint32_t)(i >> 32), 0, IG_STREAM_VECTOR, (uint32_t)seed,
                         (uint32_t)(seed >> 32));
  if (mode == 1) return (float)(r.v[0] & 15u);
  return (float)(r.v[0] >> 8) * (1.0f / 16777216.0f);
}

#endif
