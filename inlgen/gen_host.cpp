// gen_host.cpp — host (CPU) builder of the seeded synthetic inputs.
// Input side only (see include/inlgen.h); holds none of the method's arithmetic.
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "../include/inlgen.h"
#include "inlgen_core.h"
#include "inlgen_graph.h"

static thread_local char g_err[512];

extern "C" void inlgen_set_error(const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof g_err, fmt, ap);
  va_end(ap);
}

extern "C" const char *inlgen_last_error(void) { return g_err; }

extern "C" void inlgen_philox(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  ig_u32x4 r = ig_philox(ctr[0], ctr[1], ctr[2], ctr[3], key[0], key[1]);
  for (int i = 0; i < 4; ++i) out[i] = r.v[i];
}

extern "C" uint64_t inlgen_relabel(uint64_t x, int scale, uint64_t seed) {
  return ig_relabel(x, scale, seed);
}

extern "C" int inlgen_rmat_tuples(int scale, uint64_t seed, uint64_t e_begin, int64_t count,
                                  int64_t *u, int64_t *v) {
  if (scale < 1 || scale > 30 || count < 0 || !u || !v) {
    inlgen_set_error("inlgen_rmat_tuples: bad argument");
    return -1;
  }
  for (int64_t i = 0; i < count; ++i) {
    uint64_t a, b;
    ig_rmat_edge(seed, scale, e_begin + (uint64_t)i, &a, &b);
    u[i] = (int64_t)ig_relabel(a, scale, seed);
    v[i] = (int64_t)ig_relabel(b, scale, seed);
  }
  return 0;
}

// LSD radix sort of 64-bit keys on the low `bits` bits (11-bit digits).
static void radix_sort_u64(std::vector<uint64_t> &a, int bits) {
  std::vector<uint64_t> tmp(a.size());
  const int D = 11;
  const size_t R = 1u << D;
  std::vector<size_t> cnt(R);
  for (int sh = 0; sh < bits; sh += D) {
    std::fill(cnt.begin(), cnt.end(), 0);
    for (uint64_t k : a) cnt[(k >> sh) & (R - 1)]++;
    size_t s = 0;
    for (size_t d = 0; d < R; ++d) {
      size_t c = cnt[d];
      cnt[d] = s;
      s += c;
    }
    for (uint64_t k : a) tmp[cnt[(k >> sh) & (R - 1)]++] = k;
    a.swap(tmp);
  }
}

extern "C" int inlgen_host_build(int scale, int edge_factor, uint64_t seed, int flags,
                                 int64_t row_begin, int64_t row_end, inlgen_graph *out) {
  if (!out || scale < 1 || scale > 26 || edge_factor < 1) {
    inlgen_set_error("inlgen_host_build: bad argument (scale 1..26, edge_factor >= 1)");
    return -1;
  }
  const int64_t n = (int64_t)1 << scale;
  if (row_end < 0) row_end = n;
  if (row_begin < 0 || row_begin > row_end || row_end > n) {
    inlgen_set_error("inlgen_host_build: bad row range [%lld, %lld)", (long long)row_begin,
                     (long long)row_end);
    return -1;
  }
  const uint64_t m = (uint64_t)edge_factor << scale;
  const bool sym = flags & INLGEN_SYMMETRIC, tr = flags & INLGEN_TRANSPOSE;
  std::vector<uint64_t> keys;
  keys.reserve(sym ? 2 * m : m);
  for (uint64_t e = 0; e < m; ++e) {
    uint64_t a, b;
    ig_rmat_edge(seed, scale, e, &a, &b);
    uint64_t u = ig_relabel(a, scale, seed), v = ig_relabel(b, scale, seed);
    if (u == v) continue;
    if (sym) {
      keys.push_back((u << scale) | v);
      keys.push_back((v << scale) | u);
    } else if (tr) {
      keys.push_back((v << scale) | u);
    } else {
      keys.push_back((u << scale) | v);
    }
  }
  radix_sort_u64(keys, 2 * scale);
  size_t w = 0;
  for (size_t i = 0; i < keys.size(); ++i)
    if (i == 0 || keys[i] != keys[i - 1]) keys[w++] = keys[i];
  keys.resize(w);

  inlgen_graph g = (inlgen_graph)calloc(1, sizeof(*g));
  if (!g) return -2;
  g->n_global = n;
  g->row_begin = row_begin;
  g->n_rows = row_end - row_begin;
  g->on_device = 0;
  const uint64_t mask = (uint64_t(1) << scale) - 1;
  if (tr) {
    g->out_degree = (int32_t *)calloc((size_t)n, sizeof(int32_t));
    for (uint64_t k : keys) g->out_degree[k & mask]++;
  }
  size_t lo = 0;
  while (lo < keys.size() && (int64_t)(keys[lo] >> scale) < row_begin) ++lo;
  size_t hi = lo;
  while (hi < keys.size() && (int64_t)(keys[hi] >> scale) < row_end) ++hi;
  g->nnz = (int64_t)(hi - lo);
  g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(g->n_rows + 1));
  g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(g->nnz > 0 ? g->nnz : 1));
  if (!g->row_ptr || !g->col_idx) {
    inlgen_graph_free(g);
    return -2;
  }
  std::vector<int64_t> cnt((size_t)g->n_rows + 1, 0);
  for (size_t i = lo; i < hi; ++i) {
    cnt[(size_t)((int64_t)(keys[i] >> scale) - row_begin) + 1]++;
    g->col_idx[i - lo] = (int32_t)(keys[i] & mask);
  }
  g->row_ptr[0] = 0;
  for (int64_t r = 0; r < g->n_rows; ++r) g->row_ptr[r + 1] = g->row_ptr[r] + cnt[(size_t)r + 1];
  *out = g;
  return 0;
}

extern "C" int inlgen_graph_info(inlgen_graph g, int64_t *n_global, int64_t *n_rows,
                                 int64_t *row_begin, int64_t *nnz, int *on_device) {
  if (!g) return -1;
  if (n_global) *n_global = g->n_global;
  if (n_rows) *n_rows = g->n_rows;
  if (row_begin) *row_begin = g->row_begin;
  if (nnz) *nnz = g->nnz;
  if (on_device) *on_device = g->on_device;
  return 0;
}

extern "C" int inlgen_weights_host(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                                   const int32_t *col_idx, uint64_t seed, uint32_t *w) {
  if (n_rows < 0 || !row_ptr || (!w && row_ptr[n_rows] > 0)) return -1;
  for (int64_t r = 0; r < n_rows; ++r)
    for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
      w[k] = ig_weight(seed, (uint64_t)(row_begin + r), (uint64_t)col_idx[k]);
  return 0;
}

extern "C" int inlgen_values_host(int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                                  const int32_t *col_idx, uint64_t seed, int mode, float *val) {
  if (n_rows < 0 || !row_ptr || (!val && row_ptr[n_rows] > 0)) return -1;
  for (int64_t r = 0; r < n_rows; ++r)
    for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
      val[k] = ig_value(seed, (uint64_t)(row_begin + r), (uint64_t)col_idx[k], mode);
  return 0;
}

extern "C" int inlgen_vector_host(int64_t n, int64_t begin, uint64_t seed, int mode, float *x) {
  if (n < 0 || (!x && n > 0)) return -1;
  for (int64_t i = 0; i < n; ++i) x[i] = ig_vector(seed, (uint64_t)(begin + i), mode);
  return 0;
}
