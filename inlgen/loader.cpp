// loader.cpp — CSR loaders and the CiteSeer-shaped generator of the input module (SURVEY §8a
// row a1: "a CSR generator and loader"; §III.B P11@2099: graphs are encoded in
// CSR; L5 §III.A P5@12491-13052: CiteSeer, "434,102 nodes and 16 million edges", out-degree
// 1..1,188, average 73.9).  INPUT SIDE ONLY: nothing here computes a step of the method.
//
//  * MatrixMarket (coordinate; real / integer / pattern; general / symmetric): 1-based
//    entries -> a CSR with sorted columns; self-loops dropped and duplicate (row, col) pairs
//    merged keeping the FIRST value (the recipe's reading R7/R8: a graph has one edge per
//    pair; an SpMV user who wants summed duplicates must pre-merge them).  INLGEN_SYMMETRIC
//    adds (v, u) for every (u, v); INLGEN_TRANSPOSE stores the in-edge CSR + out-degrees.
//  * .inlcsr: a little-endian binary dump of one (local) CSR, with optional values and
//    out-degrees (layout in include/inlgen.h).
//  * inlgen_powerlaw_build: a configuration-model graph whose degree sequence follows a
//    discrete truncated power law on [dmin, dmax] with the requested mean (stubs paired by a
//    Philox-keyed Fisher-Yates shuffle, symmetric, self-loops / duplicates removed).
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "inlgen.h"
#include "inlgen_core.h"
#include "inlgen_graph.h"

namespace {

constexpr char kMagic[8] = {'I', 'N', 'L', 'C', 'S', 'R', 0, 1};
enum { F_VALUES = 1, F_OUTDEG = 2 };

struct Entry {
  int64_t r, c;
  float v;
  int64_t ord;  // input order (duplicates keep the first)
};

// CSR of n_rows x n_global from (r, c, v) entries: sort by (r, c, input order), drop
// self-loops and repeated pairs.
int build_csr(std::vector<Entry> &e, int64_t n_rows, int64_t n_global, bool values, bool outdeg,
              inlgen_graph *out) {
  std::sort(e.begin(), e.end(), [](const Entry &a, const Entry &b) {
    return a.r != b.r ? a.r < b.r : a.c != b.c ? a.c < b.c : a.ord < b.ord;
  });
  size_t w = 0;
  for (size_t i = 0; i < e.size(); ++i) {
    if (e[i].r == e[i].c) continue;
    if (w > 0 && e[w - 1].r == e[i].r && e[w - 1].c == e[i].c) continue;
    e[w++] = e[i];
  }
  e.resize(w);
  inlgen_graph g = (inlgen_graph)calloc(1, sizeof(*g));
  if (!g) return -2;
  g->n_global = n_global;
  g->n_rows = n_rows;
  g->row_begin = 0;
  g->nnz = (int64_t)w;
  g->row_ptr = (int64_t *)calloc((size_t)n_rows + 1, sizeof(int64_t));
  g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (w > 0 ? w : 1));
  if (values) g->val = (float *)malloc(sizeof(float) * (w > 0 ? w : 1));
  if (outdeg) g->out_degree = (int32_t *)calloc((size_t)n_global, sizeof(int32_t));
  if (!g->row_ptr || !g->col_idx || (values && !g->val) || (outdeg && !g->out_degree)) {
    inlgen_graph_free(g);
    return -2;
  }
  for (size_t i = 0; i < w; ++i) {
    g->row_ptr[e[i].r + 1]++;
    g->col_idx[i] = (int32_t)e[i].c;
    if (values) g->val[i] = e[i].v;
    if (outdeg) g->out_degree[e[i].c]++;  // in-CSR: column = source
  }
  for (int64_t r = 0; r < n_rows; ++r) g->row_ptr[r + 1] += g->row_ptr[r];
  *out = g;
  return 0;
}

// (u, v, val) list -> the requested orientation (SYMMETRIC adds reverses, TRANSPOSE swaps)
void orient(std::vector<Entry> &e, int flags) {
  const size_t m = e.size();
  if (flags & INLGEN_SYMMETRIC) {
    e.reserve(2 * m);
    for (size_t i = 0; i < m; ++i) e.push_back(Entry{e[i].c, e[i].r, e[i].v, e[i].ord});
  } else if (flags & INLGEN_TRANSPOSE) {
    for (auto &x : e) std::swap(x.r, x.c);
  }
}

bool lower_eq(std::string a, const char *b) {
  for (auto &ch : a) ch = (char)tolower((unsigned char)ch);
  return a == b;
}

template <class T>
bool wr(FILE *f, const T *p, size_t n) {
  return n == 0 || fwrite(p, sizeof(T), n, f) == n;
}
template <class T>
bool rd(FILE *f, T *p, size_t n) {
  return n == 0 || fread(p, sizeof(T), n, f) == n;
}

}  // namespace

extern "C" int inlgen_load_mtx(const char *path, int flags, inlgen_graph *out) {
  if (!path || !out) return -1;
  FILE *f = fopen(path, "r");
  if (!f) {
    inlgen_set_error("inlgen_load_mtx: cannot open %s", path);
    return -3;
  }
  char line[4096];
  if (!fgets(line, sizeof line, f)) {
    fclose(f);
    inlgen_set_error("inlgen_load_mtx: empty file");
    return -3;
  }
  char bnr[64] = {0}, obj[64] = {0}, fmt[64] = {0}, field[64] = {0}, sym[64] = {0};
  if (sscanf(line, "%63s %63s %63s %63s %63s", bnr, obj, fmt, field, sym) != 5 ||
      std::string(bnr) != "%%MatrixMarket" || !lower_eq(obj, "matrix") || !lower_eq(fmt, "coordinate")) {
    fclose(f);
    inlgen_set_error("inlgen_load_mtx: not a MatrixMarket coordinate matrix");
    return -3;
  }
  const bool pattern = lower_eq(field, "pattern");
  if (!pattern && !lower_eq(field, "real") && !lower_eq(field, "integer") && !lower_eq(field, "double")) {
    fclose(f);
    inlgen_set_error("inlgen_load_mtx: field '%s' not supported (real, integer, pattern)", field);
    return -3;
  }
  const bool msym = lower_eq(sym, "symmetric");
  if (!msym && !lower_eq(sym, "general")) {
    fclose(f);
    inlgen_set_error("inlgen_load_mtx: symmetry '%s' not supported (general, symmetric)", sym);
    return -3;
  }
  long long M = -1, N = -1, L = -1;
  while (fgets(line, sizeof line, f)) {
    if (line[0] == '%') continue;
    if (sscanf(line, "%lld %lld %lld", &M, &N, &L) == 3) break;
  }
  if (M < 0 || N < 0 || L < 0 || M >= INT32_MAX || N >= INT32_MAX) {
    fclose(f);
    inlgen_set_error("inlgen_load_mtx: bad size line");
    return -3;
  }
  std::vector<Entry> e;
  e.reserve((size_t)L * (msym ? 2 : 1));
  for (long long i = 0; i < L; ++i) {
    long long r, c;
    double v = 1.0;
    int got = 0;
    bool have = false;
    while (fgets(line, sizeof line, f)) {
      if (line[0] != '%' && line[0] != '\n') {
        have = true;
        break;
      }
    }
    if (have) got = pattern ? sscanf(line, "%lld %lld", &r, &c) : sscanf(line, "%lld %lld %lf", &r, &c, &v);
    if (got != (pattern ? 2 : 3) || r < 1 || r > M || c < 1 || c > N) {
      fclose(f);
      inlgen_set_error("inlgen_load_mtx: bad entry %lld of %lld", i + 1, L);
      return -3;
    }
    e.push_back(Entry{r - 1, c - 1, (float)v, (int64_t)i});
    if (msym && r != c) e.push_back(Entry{c - 1, r - 1, (float)v, (int64_t)i});
  }
  fclose(f);
  if ((flags & (INLGEN_SYMMETRIC | INLGEN_TRANSPOSE)) && M != N) {
    inlgen_set_error("inlgen_load_mtx: SYMMETRIC / TRANSPOSE need a square matrix");
    return -1;
  }
  orient(e, flags);
  const int64_t n_global = std::max<int64_t>(M, N);
  const int64_t n_rows = (flags & INLGEN_TRANSPOSE) ? N : M;
  return build_csr(e, n_rows, n_global, !pattern, (flags & INLGEN_TRANSPOSE) != 0, out);
}

extern "C" int inlgen_graph_from_csr(int64_t n_global, int64_t n_rows, int64_t row_begin, const int64_t *row_ptr,
                                     const int32_t *col_idx, const float *val, const int32_t *out_degree,
                                     inlgen_graph *out) {
  if (!out || !row_ptr || n_rows < 0 || n_global < 0 || row_begin < 0) return -1;
  const int64_t nnz = row_ptr[n_rows];
  inlgen_graph g = (inlgen_graph)calloc(1, sizeof(*g));
  if (!g) return -2;
  g->n_global = n_global;
  g->n_rows = n_rows;
  g->row_begin = row_begin;
  g->nnz = nnz;
  g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n_rows + 1));
  g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
  if (val) g->val = (float *)malloc(sizeof(float) * (size_t)(nnz > 0 ? nnz : 1));
  if (out_degree) g->out_degree = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n_global > 0 ? n_global : 1));
  if (!g->row_ptr || !g->col_idx || (val && !g->val) || (out_degree && !g->out_degree)) {
    inlgen_graph_free(g);
    return -2;
  }
  memcpy(g->row_ptr, row_ptr, sizeof(int64_t) * (size_t)(n_rows + 1));
  if (nnz) memcpy(g->col_idx, col_idx, sizeof(int32_t) * (size_t)nnz);
  if (val && nnz) memcpy(g->val, val, sizeof(float) * (size_t)nnz);
  if (out_degree && n_global) memcpy(g->out_degree, out_degree, sizeof(int32_t) * (size_t)n_global);
  *out = g;
  return 0;
}

extern "C" int inlgen_save_csr(const char *path, inlgen_graph g) {
  if (!path || !g) return -1;
  if (g->on_device) {
    inlgen_set_error("inlgen_save_csr: host graphs only");
    return -1;
  }
  FILE *f = fopen(path, "wb");
  if (!f) {
    inlgen_set_error("inlgen_save_csr: cannot create %s", path);
    return -3;
  }
  const int64_t hdr[5] = {g->n_global, g->n_rows, g->row_begin, g->nnz,
                          (g->val ? F_VALUES : 0) | (g->out_degree ? F_OUTDEG : 0)};
  bool ok = wr(f, kMagic, 8) && wr(f, hdr, 5) && wr(f, g->row_ptr, (size_t)g->n_rows + 1) &&
            wr(f, g->col_idx, (size_t)g->nnz);
  if (ok && g->val) ok = wr(f, g->val, (size_t)g->nnz);
  if (ok && g->out_degree) ok = wr(f, g->out_degree, (size_t)g->n_global);
  ok = (fclose(f) == 0) && ok;
  if (!ok) inlgen_set_error("inlgen_save_csr: write failed");
  return ok ? 0 : -3;
}

extern "C" int inlgen_load_csr(const char *path, inlgen_graph *out) {
  if (!path || !out) return -1;
  FILE *f = fopen(path, "rb");
  if (!f) {
    inlgen_set_error("inlgen_load_csr: cannot open %s", path);
    return -3;
  }
  char mg[8];
  int64_t hdr[5];
  if (!rd(f, mg, 8) || memcmp(mg, kMagic, 8) != 0 || !rd(f, hdr, 5) || hdr[0] < 0 || hdr[1] < 0 || hdr[2] < 0 ||
      hdr[3] < 0 || hdr[2] + hdr[1] > hdr[0] || hdr[0] >= INT32_MAX) {
    fclose(f);
    inlgen_set_error("inlgen_load_csr: %s is not an .inlcsr file", path);
    return -3;
  }
  inlgen_graph g = (inlgen_graph)calloc(1, sizeof(*g));
  if (!g) {
    fclose(f);
    return -2;
  }
  g->n_global = hdr[0];
  g->n_rows = hdr[1];
  g->row_begin = hdr[2];
  g->nnz = hdr[3];
  g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(g->n_rows + 1));
  g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(g->nnz > 0 ? g->nnz : 1));
  if (hdr[4] & F_VALUES) g->val = (float *)malloc(sizeof(float) * (size_t)(g->nnz > 0 ? g->nnz : 1));
  if (hdr[4] & F_OUTDEG) g->out_degree = (int32_t *)malloc(sizeof(int32_t) * (size_t)(g->n_global > 0 ? g->n_global : 1));
  bool ok = g->row_ptr && g->col_idx && (!(hdr[4] & F_VALUES) || g->val) && (!(hdr[4] & F_OUTDEG) || g->out_degree);
  ok = ok && rd(f, g->row_ptr, (size_t)g->n_rows + 1) && rd(f, g->col_idx, (size_t)g->nnz);
  if (ok && g->val) ok = rd(f, g->val, (size_t)g->nnz);
  if (ok && g->out_degree) ok = rd(f, g->out_degree, (size_t)g->n_global);
  fclose(f);
  // structural checks: row_ptr[0] = 0, non-decreasing, ends at nnz, columns in range
  if (ok) ok = g->row_ptr[0] == 0 && g->row_ptr[g->n_rows] == g->nnz;
  for (int64_t r = 0; ok && r < g->n_rows; ++r) ok = g->row_ptr[r] <= g->row_ptr[r + 1];
  for (int64_t k = 0; ok && k < g->nnz; ++k) ok = g->col_idx[k] >= 0 && g->col_idx[k] < g->n_global;
  if (!ok) {
    inlgen_graph_free(g);
    inlgen_set_error("inlgen_load_csr: %s is truncated or malformed", path);
    return -3;
  }
  *out = g;
  return 0;
}

extern "C" int inlgen_graph_values(inlgen_graph g, float *val) {
  if (!g || !val) return -1;
  if (!g->val) {
    inlgen_set_error("inlgen_graph_values: the graph has no values");
    return -1;
  }
  if (g->on_device) return -1;
  if (g->nnz) memcpy(val, g->val, sizeof(float) * (size_t)g->nnz);
  return 0;
}

// P(d) ~ d^-alpha on [dmin, dmax]; mean(alpha) decreases in alpha: bisection for the target.
static double pl_mean(double alpha, int dmin, int dmax) {
  double s = 0, sd = 0;
  for (int d = dmin; d <= dmax; ++d) {
    const double p = pow((double)d, -alpha);
    s += p;
    sd += p * d;
  }
  return sd / s;
}

static int powerlaw_once(int64_t n, int dmin, int dmax, double mean, uint64_t seed, inlgen_graph *out);

// Merging repeated pairs (hub-hub multi-edges of the configuration model) lowers the realised
// mean degree; the target of the degree law is raised until the realised mean is within 0.5%.
extern "C" int inlgen_powerlaw_build(int64_t n, int dmin, int dmax, double mean, uint64_t seed, int flags,
                                     inlgen_graph *out) {
  if (!out || n < 2 || n >= INT32_MAX || dmin < 1 || dmax < dmin || dmax >= n || mean < dmin || mean > dmax) {
    inlgen_set_error("inlgen_powerlaw_build: bad argument");
    return -1;
  }
  (void)flags;
  double target = mean;
  for (int it = 0;; ++it) {
    inlgen_graph g = nullptr;
    const int rc = powerlaw_once(n, dmin, dmax, target, seed, &g);
    if (rc) return rc;
    const double got = (double)g->nnz / (double)n;
    if (it == 5 || fabs(got - mean) <= 0.005 * mean || target >= dmax) {
      *out = g;
      return 0;
    }
    inlgen_graph_free(g);
    target = std::min((double)dmax, target * mean / got);
  }
}

static int powerlaw_once(int64_t n, int dmin, int dmax, double mean, uint64_t seed, inlgen_graph *out) {
  double lo = -4.0, hi = 8.0;  // alpha < 0 puts mass on large degrees
  for (int it = 0; it < 100; ++it) {
    const double mid = 0.5 * (lo + hi);
    if (pl_mean(mid, dmin, dmax) > mean) lo = mid;
    else hi = mid;
  }
  const double alpha = 0.5 * (lo + hi);
  std::vector<double> cdf((size_t)(dmax - dmin + 1));
  double s = 0;
  for (int d = dmin; d <= dmax; ++d) {
    s += pow((double)d, -alpha);
    cdf[(size_t)(d - dmin)] = s;
  }
  // degree of vertex i: inverse CDF of a 53-bit Philox uniform keyed by (seed, i)
  std::vector<int32_t> deg((size_t)n);
  int64_t stubs = 0;
  for (int64_t i = 0; i < n; ++i) {
    const uint64_t r = ((uint64_t)ig_draw(seed, IG_STREAM_PL_DEGREE, (uint64_t)i, 0, 0) << 21) ^
                       (uint64_t)ig_draw(seed, IG_STREAM_PL_DEGREE, (uint64_t)i, 0, 1);
    const double u = (double)(r & ((1ull << 53) - 1)) * (1.0 / 9007199254740992.0) * s;
    const size_t k = (size_t)(std::upper_bound(cdf.begin(), cdf.end(), u) - cdf.begin());
    deg[(size_t)i] = dmin + (int32_t)std::min(k, cdf.size() - 1);
    stubs += deg[(size_t)i];
  }
  if (stubs & 1) {  // an even stub count: the last vertex takes one more (or one less)
    deg[(size_t)n - 1] += deg[(size_t)n - 1] < dmax ? 1 : -1;
    stubs += deg[(size_t)n - 1] < dmax ? 1 : -1;
  }
  std::vector<int32_t> st;
  st.reserve((size_t)stubs);
  for (int64_t i = 0; i < n; ++i)
    for (int32_t j = 0; j < deg[(size_t)i]; ++j) st.push_back((int32_t)i);
  // Fisher-Yates with Philox-keyed draws (deterministic for a seed)
  for (int64_t i = (int64_t)st.size() - 1; i > 0; --i) {
    const uint64_t r = ((uint64_t)ig_draw(seed, IG_STREAM_PL_SHUFFLE, (uint64_t)i, 0, 0) << 32) |
                       ig_draw(seed, IG_STREAM_PL_SHUFFLE, (uint64_t)i, 0, 1);
    const int64_t j = (int64_t)(r % (uint64_t)(i + 1));
    std::swap(st[(size_t)i], st[(size_t)j]);
  }
  std::vector<Entry> e;
  e.reserve(st.size());
  for (size_t i = 0; i + 1 < st.size(); i += 2) e.push_back(Entry{st[i], st[i + 1], 1.0f, (int64_t)i});
  st.clear();
  st.shrink_to_fit();
  // the configuration model is undirected: both directions always (SURVEY §8c.12 "CSR entries")
  orient(e, INLGEN_SYMMETRIC);
  return build_csr(e, n, n, false, false, out);
}

// ---- synthetic trees (§III.C P11@8056: "three parameters: tree
// depth, node outdegree and sparsity ... All non-leaf nodes have the same number of children,
// which is given by the node outdegree parameter.  The probability rho of the non-leaf nodes
// having children is defined as rho = (1/2)^sparsity" — reading R14: the garbled formula is
// (1/2)^sparsity; the root always has children; `depth` counts levels, so the leaves of a
// regular tree are at level depth-1 and the flat kernel's atomics are d + 2d^2 + 3d^3 at
// depth 4, Fig. 7(c)).  Node ids are level order (BFS numbering): the root is 0 and a node's
// children are consecutive.  Children CSR in row_ptr / col_idx; parent[] via inlgen_graph_parent
// (parent[0] = -1).  Node v (below the last level) has children iff a Philox draw keyed by
// (seed, v) is below rho * 2^32.
extern "C" int inlgen_tree_build(int depth, int outdegree, int sparsity, uint64_t seed, inlgen_graph *out) {
  if (!out || depth < 1 || outdegree < 1 || sparsity < 0 || sparsity > 31) {
    inlgen_set_error("inlgen_tree_build: bad argument (depth >= 1, outdegree >= 1, sparsity in [0, 31])");
    return -1;
  }
  const uint64_t thr = sparsity == 0 ? 0x100000000ull : (0x100000000ull >> sparsity);  // rho * 2^32
  std::vector<int64_t> rp(1, 0);
  std::vector<int32_t> col, par(1, -1);
  int64_t lo = 0, hi = 1;  // the current level's nodes
  for (int lev = 0; lev < depth; ++lev) {
    for (int64_t v = lo; v < hi; ++v) {
      const bool kids = lev + 1 < depth && (v == 0 || (uint64_t)ig_draw(seed, IG_STREAM_TREE, (uint64_t)v, 0, 0) < thr);
      if (kids) {
        if ((int64_t)par.size() + outdegree >= INT32_MAX) {
          inlgen_set_error("inlgen_tree_build: more than 2^31 nodes");
          return -1;
        }
        for (int c = 0; c < outdegree; ++c) {
          col.push_back((int32_t)par.size());
          par.push_back((int32_t)v);
        }
      }
      rp.push_back((int64_t)col.size());
    }
    lo = hi;
    hi = (int64_t)par.size();
  }
  const int64_t n = (int64_t)par.size();
  inlgen_graph g = (inlgen_graph)calloc(1, sizeof(*g));
  if (!g) return -2;
  g->n_global = g->n_rows = n;
  g->nnz = (int64_t)col.size();
  g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (col.empty() ? 1 : col.size()));
  g->parent = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  if (!g->row_ptr || !g->col_idx || !g->parent) {
    inlgen_graph_free(g);
    return -2;
  }
  memcpy(g->row_ptr, rp.data(), sizeof(int64_t) * (size_t)(n + 1));
  if (!col.empty()) memcpy(g->col_idx, col.data(), sizeof(int32_t) * col.size());
  memcpy(g->parent, par.data(), sizeof(int32_t) * (size_t)n);
  *out = g;
  return 0;
}

extern "C" int inlgen_graph_parent(inlgen_graph g, int32_t *parent) {
  if (!g || !parent || !g->parent || g->on_device) {
    inlgen_set_error("inlgen_graph_parent: not a tree from inlgen_tree_build");
    return -1;
  }
  memcpy(parent, g->parent, sizeof(int32_t) * (size_t)g->n_global);
  return 0;
}
