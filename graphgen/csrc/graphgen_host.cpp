// graphgen_host.cpp -- host (CPU) builders of the seeded synthetic inputs.
// Input module: shared by oracle-side tests and CUDA-side tests as the only
// common code; none of the Louvain arithmetic lives here.  Graph recipes are
// SURVEY.md 8(d) C1..C5.
#include "graphgen.h"
#include "gg_internal.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

static thread_local std::string g_err;
void gg_set_error(const char* msg) { g_err = msg; }
extern "C" const char* gg_last_error(void) { return g_err.c_str(); }

// ---------------------------------------------------------------- handle
gg_graph_s* gg_alloc_host(int64_t n, int64_t nnz) {
  gg_graph_s* g = new gg_graph_s();
  g->n = n;
  g->nnz = nnz;
  g->device = 0;
  g->rowptr = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  g->col = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
  g->labels = nullptr;
  return g;
}

extern "C" int64_t gg_n(gg_graph_t g) { return g ? g->n : -1; }
extern "C" int64_t gg_nnz(gg_graph_t g) { return g ? g->nnz : -1; }
extern "C" int gg_on_device(gg_graph_t g) { return g ? g->device : 0; }
extern "C" const int64_t* gg_rowptr(gg_graph_t g) { return g ? g->rowptr : nullptr; }
extern "C" const int32_t* gg_col(gg_graph_t g) { return g ? g->col : nullptr; }
extern "C" const int32_t* gg_labels(gg_graph_t g) { return g ? g->labels : nullptr; }

extern "C" void gg_free(gg_graph_t g) {
  if (!g) return;
  if (g->device) {
    gg_device_free(g);
  } else {
    free(g->rowptr);
    free(g->col);
  }
  free(g->labels);
  delete g;
}

extern "C" int gg_copy_out(gg_graph_t g, int64_t* rowptr_dst, int32_t* col_dst) {
  if (!g) { gg_set_error("null graph"); return -1; }
  if (g->device) return gg_device_copy_out(g, rowptr_dst, col_dst);
  // Host source: destination may still be device memory.
  return gg_copy_any(rowptr_dst, g->rowptr, sizeof(int64_t) * (size_t)(g->n + 1), col_dst, g->col,
                     sizeof(int32_t) * (size_t)g->nnz);
}

// ---------------------------------------------------------------- canonical CSR builder
// LSD radix sort of 64-bit keys, 16-bit digits, skipping constant digits.
static void radix_sort_u64(std::vector<uint64_t>& keys) {
  size_t N = keys.size();
  if (N < 2) return;
  std::vector<uint64_t> tmp(N);
  uint64_t orv = 0, andv = ~0ull;
  for (uint64_t k : keys) { orv |= k; andv &= k; }
  std::vector<size_t> cnt(65537);
  for (int shift = 0; shift < 64; shift += 16) {
    if ((((orv ^ andv) >> shift) & 0xFFFFull) == 0) continue;  // digit constant
    std::fill(cnt.begin(), cnt.end(), 0);
    for (size_t i = 0; i < N; ++i) cnt[((keys[i] >> shift) & 0xFFFF) + 1]++;
    for (int d = 0; d < 65536; ++d) cnt[d + 1] += cnt[d];
    for (size_t i = 0; i < N; ++i) tmp[cnt[(keys[i] >> shift) & 0xFFFF]++] = keys[i];
    keys.swap(tmp);
  }
}

// keys: directed entries (u << 32 | v), both directions already present, u != v.
// Sorts, dedups, optionally compacts isolated vertices (order preserving, R21).
// If labels_in is given (size n) the labels of surviving vertices are kept.
gg_graph_s* gg_build_csr_host(int64_t n, std::vector<uint64_t>& keys, int compact,
                              const int32_t* labels_in) {
  radix_sort_u64(keys);
  keys.erase(std::unique(keys.begin(), keys.end()), keys.end());
  std::vector<int64_t> deg((size_t)n, 0);
  for (uint64_t k : keys) deg[(size_t)(k >> 32)]++;
  std::vector<int32_t> newid((size_t)n);
  int64_t nn = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (!compact || deg[(size_t)i] > 0) newid[(size_t)i] = (int32_t)nn++;
    else newid[(size_t)i] = -1;
  }
  gg_graph_s* g = gg_alloc_host(nn, (int64_t)keys.size());
  g->rowptr[0] = 0;
  int64_t r = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (newid[(size_t)i] < 0) continue;
    g->rowptr[r + 1] = g->rowptr[r] + deg[(size_t)i];
    ++r;
  }
  for (size_t e = 0; e < keys.size(); ++e) g->col[e] = newid[(size_t)(keys[e] & 0xFFFFFFFFu)];
  if (labels_in) {
    g->labels = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nn > 0 ? nn : 1));
    for (int64_t i = 0; i < n; ++i)
      if (newid[(size_t)i] >= 0) g->labels[newid[(size_t)i]] = labels_in[i];
  }
  return g;
}

static void push_edge(std::vector<uint64_t>& keys, uint32_t u, uint32_t v) {
  if (u == v) return;  // self-loops dropped (R1: level-0 graphs are simple)
  keys.push_back(((uint64_t)u << 32) | v);
  keys.push_back(((uint64_t)v << 32) | u);
}

extern "C" int gg_from_edges(int64_t n, int64_t m, const int32_t* u, const int32_t* v, int compact,
                             gg_graph_t* out) {
  if (!out || n < 0 || m < 0 || (m > 0 && (!u || !v))) { gg_set_error("bad args"); return -1; }
  if (n > INT32_MAX) { gg_set_error("n too large"); return -1; }
  std::vector<uint64_t> keys;
  keys.reserve((size_t)(2 * m));
  for (int64_t e = 0; e < m; ++e) {
    if (u[e] < 0 || u[e] >= n || v[e] < 0 || v[e] >= n) { gg_set_error("edge endpoint out of range"); return -2; }
    push_edge(keys, (uint32_t)u[e], (uint32_t)v[e]);
  }
  *out = gg_build_csr_host(n, keys, compact, nullptr);
  return 0;
}

// ---------------------------------------------------------------- C1 karate
static const uint8_t kKarate[78][2] = {
    {0, 1},   {0, 2},   {0, 3},   {0, 4},   {0, 5},   {0, 6},   {0, 7},   {0, 8},   {0, 10},
    {0, 11},  {0, 12},  {0, 13},  {0, 17},  {0, 19},  {0, 21},  {0, 31},  {1, 2},   {1, 3},
    {1, 7},   {1, 13},  {1, 17},  {1, 19},  {1, 21},  {1, 30},  {2, 3},   {2, 7},   {2, 8},
    {2, 9},   {2, 13},  {2, 27},  {2, 28},  {2, 32},  {3, 7},   {3, 12},  {3, 13},  {4, 6},
    {4, 10},  {5, 6},   {5, 10},  {5, 16},  {6, 16},  {8, 30},  {8, 32},  {8, 33},  {9, 33},
    {13, 33}, {14, 32}, {14, 33}, {15, 32}, {15, 33}, {18, 32}, {18, 33}, {19, 33}, {20, 32},
    {20, 33}, {22, 32}, {22, 33}, {23, 25}, {23, 27}, {23, 29}, {23, 32}, {23, 33}, {24, 25},
    {24, 27}, {24, 31}, {25, 31}, {26, 29}, {26, 33}, {27, 33}, {28, 31}, {28, 33}, {29, 32},
    {29, 33}, {30, 32}, {30, 33}, {31, 32}, {31, 33}, {32, 33}};

extern "C" int gg_karate(gg_graph_t* out) {
  if (!out) { gg_set_error("bad args"); return -1; }
  std::vector<uint64_t> keys;
  for (int e = 0; e < 78; ++e) push_edge(keys, kKarate[e][0], kKarate[e][1]);
  *out = gg_build_csr_host(34, keys, 1, nullptr);
  return 0;
}

// ---------------------------------------------------------------- R-MAT (C3, C5)
void gg_rmat_thresholds(double a, double b, double c, uint32_t* tA, uint32_t* tAB, uint32_t* tABC) {
  *tA = (uint32_t)std::floor(a * 4294967296.0);
  *tAB = (uint32_t)std::floor((a + b) * 4294967296.0);
  *tABC = (uint32_t)std::floor((a + b + c) * 4294967296.0);
}

extern "C" int gg_rmat_host(int scale, int64_t ntuples, uint64_t seed, double a, double b, double c,
                            int compact, gg_graph_t* out) {
  if (!out || scale < 1 || scale > 31 || ntuples < 0) { gg_set_error("bad args"); return -1; }
  uint32_t tA, tAB, tABC;
  gg_rmat_thresholds(a, b, c, &tA, &tAB, &tABC);
  std::vector<uint64_t> keys;
  keys.reserve((size_t)(2 * ntuples));
  for (int64_t t = 0; t < ntuples; ++t) {
    uint32_t u, v;
    gg_rmat_tuple(seed, (uint64_t)t, scale, tA, tAB, tABC, &u, &v);
    push_edge(keys, u, v);
  }
  *out = gg_build_csr_host((int64_t)1 << scale, keys, compact, nullptr);
  return 0;
}

// ---------------------------------------------------------------- 3-D mesh (C4a)
int gg_mesh_bits(int L) {
  int bits = 0;
  while ((1 << bits) < L) ++bits;
  return bits;
}

extern "C" int gg_mesh3d_host(int L, int morton, gg_graph_t* out) {
  if (!out || L < 1 || L > 1024) { gg_set_error("bad args"); return -1; }
  int64_t n = (int64_t)L * L * L;
  if (n > INT32_MAX) { gg_set_error("mesh too large"); return -1; }
  // id[x,y,z] (row-major index x + L*(y + L*z)) -> vertex id
  std::vector<int32_t> id((size_t)n);
  if (morton) {
    int bits = gg_mesh_bits(L);
    uint64_t ncodes = 1ull << (3 * bits);
    int32_t next = 0;
    for (uint64_t code = 0; code < ncodes; ++code) {
      uint32_t x, y, z;
      gg_morton3_decode(code, bits, &x, &y, &z);
      if ((int)x < L && (int)y < L && (int)z < L) id[(size_t)x + (size_t)L * (y + (size_t)L * z)] = next++;
    }
  } else {
    for (int64_t i = 0; i < n; ++i) id[(size_t)i] = (int32_t)i;
  }
  std::vector<int32_t> inv((size_t)n);
  for (int64_t i = 0; i < n; ++i) inv[(size_t)id[(size_t)i]] = (int32_t)i;
  int64_t nnz = 6 * n - 6 * (int64_t)L * L;  // 2 * 3 * L^2 * (L-1)
  gg_graph_s* g = gg_alloc_host(n, nnz);
  int64_t e = 0;
  g->rowptr[0] = 0;
  for (int64_t vid = 0; vid < n; ++vid) {
    int64_t p = inv[(size_t)vid];
    int x = (int)(p % L), y = (int)((p / L) % L), z = (int)(p / ((int64_t)L * L));
    int32_t nb[6];
    int k = 0;
    if (x > 0) nb[k++] = id[(size_t)(p - 1)];
    if (x < L - 1) nb[k++] = id[(size_t)(p + 1)];
    if (y > 0) nb[k++] = id[(size_t)(p - L)];
    if (y < L - 1) nb[k++] = id[(size_t)(p + L)];
    if (z > 0) nb[k++] = id[(size_t)(p - (int64_t)L * L)];
    if (z < L - 1) nb[k++] = id[(size_t)(p + (int64_t)L * L)];
    std::sort(nb, nb + k);
    for (int j = 0; j < k; ++j) g->col[e++] = nb[j];
    g->rowptr[vid + 1] = e;
  }
  *out = g;
  return 0;
}

// ---------------------------------------------------------------- RGG (C4b)
// Points: x = u01(w0,w1), y = u01(w2,w3) of Philox(seed, stream "RGG ", item i).
// Cell grid G = floor(1/r) per side (side >= r).  Ids: sort by (row-major cell, x, y, i).
// Edge iff dx*dx + dy*dy < r*r, evaluated in double without contraction.
double gg_rgg_radius(int64_t n, double rfac) {
  return rfac * std::sqrt(std::log((double)n) / (double)n);
}

extern "C" int gg_rgg_host(int64_t n, double rfac, uint64_t seed, int compact, gg_graph_t* out) {
  if (!out || n < 2 || n > INT32_MAX) { gg_set_error("bad args"); return -1; }
  double r = gg_rgg_radius(n, rfac);
  double r2 = r * r;
  int64_t G = (int64_t)std::floor(1.0 / r);
  if (G < 1) G = 1;
  struct P { double x, y; int64_t cell; int32_t i; };
  std::vector<P> pts((size_t)n);
  for (int64_t i = 0; i < n; ++i) {
    gg_u32x4 w = gg_philox4x32_10((uint32_t)i, (uint32_t)((uint64_t)i >> 32), 0u, 0x52474720u,
                                  (uint32_t)seed, (uint32_t)(seed >> 32));
    double x = gg_u01(w.v[0], w.v[1]), y = gg_u01(w.v[2], w.v[3]);
    int64_t cx = (int64_t)(x * (double)G), cy = (int64_t)(y * (double)G);
    if (cx >= G) cx = G - 1;
    if (cy >= G) cy = G - 1;
    pts[(size_t)i] = P{x, y, cy * G + cx, (int32_t)i};
  }
  std::sort(pts.begin(), pts.end(), [](const P& p, const P& q) {
    if (p.cell != q.cell) return p.cell < q.cell;
    if (p.x != q.x) return p.x < q.x;
    if (p.y != q.y) return p.y < q.y;
    return p.i < q.i;
  });
  // cell start offsets (points sorted by cell; new id == position)
  std::vector<int64_t> cstart((size_t)(G * G + 1), 0);
  for (int64_t i = 0; i < n; ++i) cstart[(size_t)pts[(size_t)i].cell + 1]++;
  for (int64_t c = 0; c < G * G; ++c) cstart[(size_t)c + 1] += cstart[(size_t)c];
  std::vector<uint64_t> keys;
  keys.reserve((size_t)(n * 20));
  for (int64_t i = 0; i < n; ++i) {
    const P& p = pts[(size_t)i];
    int64_t cx = p.cell % G, cy = p.cell / G;
    for (int64_t dy = -1; dy <= 1; ++dy) {
      int64_t yy = cy + dy;
      if (yy < 0 || yy >= G) continue;
      for (int64_t dx = -1; dx <= 1; ++dx) {
        int64_t xx = cx + dx;
        if (xx < 0 || xx >= G) continue;
        int64_t c = yy * G + xx;
        for (int64_t j = cstart[(size_t)c]; j < cstart[(size_t)c + 1]; ++j) {
          if (j == i) continue;
          double ex = p.x - pts[(size_t)j].x, ey = p.y - pts[(size_t)j].y;
          double d2 = ex * ex + ey * ey;
          if (d2 < r2) keys.push_back(((uint64_t)i << 32) | (uint64_t)j);
        }
      }
    }
  }
  *out = gg_build_csr_host(n, keys, compact, nullptr);
  return 0;
}

// ---------------------------------------------------------------- LFR-style (C2)
// SURVEY 8(d) C2.  Host only (n = 1e6 builds in seconds).
static inline uint32_t lfr_rand(uint64_t seed, uint32_t stream, uint64_t item) {
  return gg_rand_u32(seed, stream, item, 0);
}
static inline double lfr_u01(uint64_t seed, uint32_t stream, uint64_t item) {
  gg_u32x4 w = gg_philox4x32_10((uint32_t)item, (uint32_t)(item >> 32), 1u, stream, (uint32_t)seed,
                                (uint32_t)(seed >> 32));
  return gg_u01(w.v[0], w.v[1]);
}
static int64_t powerlaw_int(double u, double e, double lo, double hi) {
  double a = std::pow(lo, 1.0 - e), b = std::pow(hi, 1.0 - e);
  double k = std::pow(a + u * (b - a), 1.0 / (1.0 - e));
  int64_t ki = (int64_t)std::floor(k);
  if (ki < (int64_t)lo) ki = (int64_t)lo;
  if (ki > (int64_t)hi) ki = (int64_t)hi;
  return ki;
}
template <class T>
static void philox_shuffle(std::vector<T>& a, uint64_t seed, uint32_t stream, uint64_t base) {
  for (size_t i = a.size(); i > 1; --i) {
    uint64_t r = lfr_rand(seed, stream, base + i);
    size_t j = (size_t)((r * (uint64_t)i) >> 32);
    std::swap(a[i - 1], a[j]);
  }
}

extern "C" int gg_lfr_host(int64_t n, double gamma, int32_t kmin, int32_t kmax, double beta,
                           int32_t smin, int32_t smax, double mu, uint64_t seed, gg_graph_t* out) {
  if (!out || n < 2 || n > INT32_MAX || kmin < 1 || kmax < kmin || smin < 2 || smax < smin || mu < 0 ||
      mu > 1) {
    gg_set_error("bad args");
    return -1;
  }
  const uint32_t S_DEG = 0x4C464431u, S_SIZE = 0x4C464432u, S_PICK = 0x4C464433u,
                 S_INTRA = 0x4C464434u, S_INTER = 0x4C464435u, S_PERM = 0x4C464436u;
  std::vector<int32_t> kin((size_t)n), kout((size_t)n);
  for (int64_t i = 0; i < n; ++i) {
    int64_t k = powerlaw_int(lfr_u01(seed, S_DEG, (uint64_t)i), gamma, kmin, kmax);
    int64_t ki = (int64_t)std::floor((1.0 - mu) * (double)k + 0.5);
    kin[(size_t)i] = (int32_t)ki;
    kout[(size_t)i] = (int32_t)(k - ki);
  }
  // community sizes
  std::vector<int64_t> csize;
  int64_t sum = 0;
  for (uint64_t j = 0; sum < n; ++j) {
    int64_t s = powerlaw_int(lfr_u01(seed, S_SIZE, j), beta, smin, smax);
    if (sum + s > n) s = n - sum;
    if (s < smin && !csize.empty()) { csize.back() += s; sum += s; break; }
    csize.push_back(s);
    sum += s;
  }
  int64_t nc = (int64_t)csize.size();
  // open communities sorted by size descending (stable by index)
  std::vector<int32_t> open((size_t)nc);
  for (int64_t c = 0; c < nc; ++c) open[(size_t)c] = (int32_t)c;
  std::stable_sort(open.begin(), open.end(), [&](int32_t p, int32_t q) { return csize[(size_t)p] > csize[(size_t)q]; });
  std::vector<int64_t> fill((size_t)nc, 0);
  // vertices by intra degree descending (stable by id)
  std::vector<int32_t> order((size_t)n);
  for (int64_t i = 0; i < n; ++i) order[(size_t)i] = (int32_t)i;
  std::stable_sort(order.begin(), order.end(), [&](int32_t p, int32_t q) { return kin[(size_t)p] > kin[(size_t)q]; });
  std::vector<int32_t> comm((size_t)n);
  for (int64_t t = 0; t < n; ++t) {
    int32_t i = order[(size_t)t];
    // eligible prefix: size > kin
    size_t lo = 0, hi = open.size();
    while (lo < hi) {
      size_t mid = (lo + hi) / 2;
      if (csize[(size_t)open[mid]] > kin[(size_t)i]) lo = mid + 1; else hi = mid;
    }
    size_t pref = lo;
    size_t pick;
    if (pref == 0) {
      pick = 0;  // none large enough: largest open community, cap intra degree
      int32_t cap = (int32_t)csize[(size_t)open[0]] - 1;
      kout[(size_t)i] += kin[(size_t)i] - cap;
      kin[(size_t)i] = cap;
    } else {
      pick = (size_t)(((uint64_t)lfr_rand(seed, S_PICK, (uint64_t)t) * (uint64_t)pref) >> 32);
    }
    int32_t c = open[pick];
    comm[(size_t)i] = c;
    if (++fill[(size_t)c] == csize[(size_t)c]) open.erase(open.begin() + (ptrdiff_t)pick);
  }
  // members per community
  std::vector<std::vector<int32_t>> members((size_t)nc);
  for (int64_t i = 0; i < n; ++i) members[(size_t)comm[(size_t)i]].push_back((int32_t)i);
  // random id permutation (ids random w.r.t. communities)
  std::vector<int32_t> perm((size_t)n);
  for (int64_t i = 0; i < n; ++i) perm[(size_t)i] = (int32_t)i;
  philox_shuffle(perm, seed, S_PERM, 0);
  std::vector<uint64_t> keys;
  keys.reserve((size_t)(n * (kmin + kmax) / 4));
  uint64_t base = 0;
  for (int64_t c = 0; c < nc; ++c) {
    std::vector<int32_t> stubs;
    for (int32_t v : members[(size_t)c])
      for (int32_t s = 0; s < kin[(size_t)v]; ++s) stubs.push_back(v);
    philox_shuffle(stubs, seed, S_INTRA, base);
    base += stubs.size() + 1;
    for (size_t s = 0; s + 1 < stubs.size(); s += 2)
      push_edge(keys, (uint32_t)perm[(size_t)stubs[s]], (uint32_t)perm[(size_t)stubs[s + 1]]);
  }
  {
    std::vector<int32_t> stubs;
    for (int64_t i = 0; i < n; ++i)
      for (int32_t s = 0; s < kout[(size_t)i]; ++s) stubs.push_back((int32_t)i);
    philox_shuffle(stubs, seed, S_INTER, 0);
    for (size_t s = 0; s + 1 < stubs.size(); s += 2)
      push_edge(keys, (uint32_t)perm[(size_t)stubs[s]], (uint32_t)perm[(size_t)stubs[s + 1]]);
  }
  std::vector<int32_t> gt((size_t)n);
  for (int64_t i = 0; i < n; ++i) gt[(size_t)perm[(size_t)i]] = comm[(size_t)i];
  *out = gg_build_csr_host(n, keys, 1, gt.data());
  return 0;
}
