// graph_io.cpp -- graph file loader / writer (input module, host C++).
//
// The paper stores every graph as CSR with both directions of each edge
// and reads its 55 inputs from files (Table 1); this is
// the loader for real graph files next to the seeded generators.  Formats:
//   * Matrix Market coordinate (.mtx): field pattern | integer | real (values must
//     be positive integers: the method's weights are uint32, R4/R20), symmetry
//     general | symmetric; 1-based (the format's rule).
//   * Edge list (.txt, .el, .edges, .tsv): one edge "u v [w]" per line, '#' or '%'
//     comment lines, 0-based unless one_based = 1 (-1: guess 1-based when no id is 0).
//   * .csrbin: this repo's binary CSR container (magic "LVCSRB01", int64 n, int64 nnz,
//     uint32 flags (bit 0 = weighted), uint32 0, rowptr int64[n+1], col int32[nnz],
//     w uint32[nnz] if weighted), stored and loaded as is (validated on load).
// Text inputs describe UNDIRECTED graphs; the CSR follows R1: each edge {u, v},
// u != v, stored as (u, v) and (v, u), a self-loop once; rows sorted by column.
// Repeated edges: without weights (pattern / two columns) the graph is simple
// (repeats and reversed repeats collapse, unit weight -- the generators'
// convention); with weights every occurrence adds its weight (a file listing both
// directions doubles every weight uniformly, which leaves Q and every decision
// unchanged except the relative weight of self-loops).
// Holds none of the Louvain method's arithmetic.
#include <errno.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "graphgen.h"

static thread_local std::string g_io_err;

struct gg_csr_s {
  int64_t n = 0, nnz = 0;
  std::vector<int64_t> rowptr;
  std::vector<int32_t> col;
  std::vector<uint32_t> w;  // empty = unit weights
};

static int fail(const std::string& m) {
  g_io_err = m;
  return -1;
}

extern "C" const char* gg_io_last_error(void) { return g_io_err.c_str(); }
extern "C" int64_t gg_csr_n(gg_csr_t g) { return g ? g->n : -1; }
extern "C" int64_t gg_csr_nnz(gg_csr_t g) { return g ? g->nnz : -1; }
extern "C" const int64_t* gg_csr_rowptr(gg_csr_t g) { return g ? g->rowptr.data() : nullptr; }
extern "C" const int32_t* gg_csr_col(gg_csr_t g) { return g && g->nnz ? g->col.data() : nullptr; }
extern "C" const uint32_t* gg_csr_w(gg_csr_t g) { return g && !g->w.empty() ? g->w.data() : nullptr; }
extern "C" void gg_csr_free(gg_csr_t g) { delete g; }

namespace {

bool read_file(const char* path, std::string* buf) {
  FILE* f = fopen(path, "rb");
  if (!f) return false;
  fseek(f, 0, SEEK_END);
  long sz = ftell(f);
  fseek(f, 0, SEEK_SET);
  buf->resize(sz > 0 ? (size_t)sz : 0);
  size_t got = sz > 0 ? fread(&(*buf)[0], 1, (size_t)sz, f) : 0;
  fclose(f);
  return got == buf->size();
}

struct Edge {
  int64_t u, v;
  uint64_t w;
};

// Undirected edges -> R1 CSR.  weighted: sum repeated edges; else collapse them.
int build(int64_t n, std::vector<Edge>& edges, bool weighted, gg_csr_t* out) {
  std::vector<std::pair<uint64_t, uint64_t>> ent;  // (u << 32 | v, w)
  ent.reserve(2 * edges.size());
  for (const Edge& e : edges) {
    if (e.u < 0 || e.v < 0 || e.u >= n || e.v >= n) return fail("vertex id out of range [0, n)");
    ent.emplace_back(((uint64_t)e.u << 32) | (uint64_t)e.v, e.w);
    if (e.u != e.v) ent.emplace_back(((uint64_t)e.v << 32) | (uint64_t)e.u, e.w);
  }
  std::sort(ent.begin(), ent.end(), [](const auto& a, const auto& b) { return a.first < b.first; });
  gg_csr_s* g = new gg_csr_s();
  g->n = n;
  g->rowptr.assign(n + 1, 0);
  for (size_t i = 0; i < ent.size();) {
    size_t j = i;
    uint64_t ws = 0;
    while (j < ent.size() && ent[j].first == ent[i].first) ws += ent[j++].second;
    if (!weighted) ws = 1;
    if (ws > 0xFFFFFFFFull) {
      delete g;
      return fail("merged edge weight exceeds 2^32 - 1");
    }
    g->col.push_back((int32_t)(ent[i].first & 0xFFFFFFFFull));
    if (weighted) g->w.push_back((uint32_t)ws);
    g->rowptr[(ent[i].first >> 32) + 1] += 1;
    i = j;
  }
  for (int64_t r = 0; r < n; ++r) g->rowptr[r + 1] += g->rowptr[r];
  g->nnz = (int64_t)g->col.size();
  *out = g;
  return 0;
}

// next token as integer (returns false at end of line / buffer)
inline void skip_blank(const char*& p, const char* e) {
  while (p < e && (*p == ' ' || *p == '\t' || *p == '\r')) ++p;
}
inline void next_line(const char*& p, const char* e) {
  while (p < e && *p != '\n') ++p;
  if (p < e) ++p;
}
bool parse_int(const char*& p, const char* e, int64_t* v) {
  skip_blank(p, e);
  if (p >= e || *p == '\n') return false;
  char* q = nullptr;
  errno = 0;
  long long x = strtoll(p, &q, 10);
  if (q == p || errno) return false;
  p = q;
  *v = x;
  return true;
}
// a positive integral weight (text "3", "3.0", "3e0"); 0 = malformed / non-integral / <= 0
bool parse_weight(const char*& p, const char* e, uint64_t* w, bool* present) {
  skip_blank(p, e);
  *present = !(p >= e || *p == '\n' || *p == '#' || *p == '%');
  if (!*present) return true;
  char* q = nullptr;
  double x = strtod(p, &q);
  if (q == p) return false;
  p = q;
  if (!(x >= 1.0) || x != (double)(uint64_t)x || x > 4294967295.0) return false;
  *w = (uint64_t)x;
  return true;
}

int load_mtx(const std::string& buf, gg_csr_t* out) {
  const char* p = buf.data();
  const char* e = p + buf.size();
  std::string head(p, std::find(p, e, '\n'));
  for (auto& c : head) c = (char)tolower(c);
  if (head.rfind("%%matrixmarket", 0) != 0) return fail("not a Matrix Market file (missing %%MatrixMarket header)");
  if (head.find("coordinate") == std::string::npos) return fail("Matrix Market: only the coordinate format is supported");
  const bool pattern = head.find("pattern") != std::string::npos;
  const bool symmetric = head.find("symmetric") != std::string::npos;
  if (head.find("complex") != std::string::npos) return fail("Matrix Market: complex values are not graph weights");
  if (!symmetric && head.find("general") == std::string::npos)
    return fail("Matrix Market: symmetry must be general or symmetric");
  next_line(p, e);
  while (p < e && *p == '%') next_line(p, e);
  int64_t rows = 0, cols = 0, nz = 0;
  if (!parse_int(p, e, &rows) || !parse_int(p, e, &cols) || !parse_int(p, e, &nz))
    return fail("Matrix Market: bad size line");
  if (rows != cols || rows < 0 || nz < 0) return fail("Matrix Market: the adjacency matrix must be square");
  if (rows > INT32_MAX - 1) return fail("Matrix Market: n >= 2^31 - 1");
  next_line(p, e);
  std::vector<Edge> edges;
  edges.reserve((size_t)nz);
  for (int64_t k = 0; k < nz; ++k) {
    while (p < e && (*p == '%' || *p == '\n')) next_line(p, e);
    int64_t i = 0, j = 0;
    if (!parse_int(p, e, &i) || !parse_int(p, e, &j)) return fail("Matrix Market: truncated entry list");
    uint64_t w = 1;
    bool present = false;
    if (!pattern && (!parse_weight(p, e, &w, &present) || !present))
      return fail("Matrix Market: weights must be positive integers (uint32)");
    edges.push_back(Edge{i - 1, j - 1, w});
    next_line(p, e);
  }
  (void)symmetric;  // either way each entry is one undirected edge (R1 stores both directions)
  return build(rows, edges, !pattern, out);
}

int load_edgelist(const std::string& buf, int one_based, gg_csr_t* out) {
  const char* p = buf.data();
  const char* e = p + buf.size();
  std::vector<Edge> edges;
  int weighted = -1;
  int64_t mx = -1, mn = INT64_MAX;
  int64_t line = 0;
  while (p < e) {
    ++line;
    skip_blank(p, e);
    if (p >= e) break;
    if (*p == '\n' || *p == '#' || *p == '%') {
      next_line(p, e);
      continue;
    }
    int64_t u = 0, v = 0;
    if (!parse_int(p, e, &u) || !parse_int(p, e, &v))
      return fail("edge list: line " + std::to_string(line) + " is not 'u v [w]'");
    uint64_t w = 1;
    bool present = false;
    if (!parse_weight(p, e, &w, &present))
      return fail("edge list: line " + std::to_string(line) + ": weights must be positive integers (uint32)");
    if (weighted < 0) weighted = present ? 1 : 0;
    if ((weighted == 1) != present) return fail("edge list: every line or none must carry a weight");
    edges.push_back(Edge{u, v, w});
    mx = std::max(mx, std::max(u, v));
    mn = std::min(mn, std::min(u, v));
    next_line(p, e);
  }
  if (one_based < 0) one_based = (!edges.empty() && mn >= 1) ? 1 : 0;
  if (one_based) {
    for (Edge& x : edges) {
      x.u -= 1;
      x.v -= 1;
    }
    mx -= 1;
  }
  if (mx + 1 > INT32_MAX - 1) return fail("edge list: n >= 2^31 - 1");
  return build(mx + 1, edges, weighted == 1, out);
}

const char kMagic[8] = {'L', 'V', 'C', 'S', 'R', 'B', '0', '1'};

int load_csrbin(const std::string& buf, gg_csr_t* out) {
  if (buf.size() < 32 || memcmp(buf.data(), kMagic, 8) != 0) return fail(".csrbin: bad magic");
  int64_t n = 0, nnz = 0;
  uint32_t flags = 0;
  memcpy(&n, buf.data() + 8, 8);
  memcpy(&nnz, buf.data() + 16, 8);
  memcpy(&flags, buf.data() + 24, 4);
  const bool weighted = flags & 1u;
  if (n < 0 || nnz < 0 || n > INT32_MAX - 1) return fail(".csrbin: bad sizes");
  const size_t need = 32 + 8 * (size_t)(n + 1) + 4 * (size_t)nnz * (weighted ? 2 : 1);
  if (buf.size() != need) return fail(".csrbin: file size does not match its header");
  gg_csr_s* g = new gg_csr_s();
  g->n = n;
  g->nnz = nnz;
  g->rowptr.resize(n + 1);
  g->col.resize(nnz);
  const char* p = buf.data() + 32;
  memcpy(g->rowptr.data(), p, 8 * (size_t)(n + 1));
  p += 8 * (size_t)(n + 1);
  if (nnz) memcpy(g->col.data(), p, 4 * (size_t)nnz);
  p += 4 * (size_t)nnz;
  if (weighted) {
    g->w.resize(nnz);
    if (nnz) memcpy(g->w.data(), p, 4 * (size_t)nnz);
  }
  bool ok = g->rowptr[0] == 0 && g->rowptr[n] == nnz;
  for (int64_t r = 0; ok && r < n; ++r) ok = g->rowptr[r] <= g->rowptr[r + 1];
  for (int64_t k = 0; ok && k < nnz; ++k) ok = g->col[k] >= 0 && g->col[k] < n;
  for (size_t k = 0; ok && k < g->w.size(); ++k) ok = g->w[k] > 0;
  if (!ok) {
    delete g;
    return fail(".csrbin: invalid CSR (rowptr, column range or zero weight)");
  }
  *out = g;
  return 0;
}

std::string ext_of(const char* path) {
  std::string s(path);
  size_t d = s.rfind('.');
  std::string x = d == std::string::npos ? "" : s.substr(d + 1);
  for (auto& c : x) c = (char)tolower(c);
  return x;
}

}  // namespace

// format: 0 = by extension, 1 = Matrix Market, 2 = edge list, 3 = .csrbin
extern "C" int gg_load(const char* path, int format, int one_based, gg_csr_t* out) {
  if (!path || !out) return fail("gg_load: null argument");
  *out = nullptr;
  if (format == 0) {
    const std::string x = ext_of(path);
    format = (x == "mtx") ? 1 : (x == "csrbin") ? 3 : 2;
  }
  std::string buf;
  if (!read_file(path, &buf)) return fail(std::string("cannot read ") + path);
  switch (format) {
    case 1: return load_mtx(buf, out);
    case 2: return load_edgelist(buf, one_based, out);
    case 3: return load_csrbin(buf, out);
    default: return fail("gg_load: unknown format");
  }
}

extern "C" int gg_save_csrbin(const char* path, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                              const uint32_t* w) {
  if (!path || n < 0 || nnz < 0 || !rowptr || (nnz && !col)) return fail("gg_save_csrbin: bad argument");
  FILE* f = fopen(path, "wb");
  if (!f) return fail(std::string("cannot write ") + path);
  uint32_t flags = w ? 1u : 0u, pad = 0;
  bool ok = fwrite(kMagic, 1, 8, f) == 8 && fwrite(&n, 8, 1, f) == 1 && fwrite(&nnz, 8, 1, f) == 1 &&
            fwrite(&flags, 4, 1, f) == 1 && fwrite(&pad, 4, 1, f) == 1 &&
            fwrite(rowptr, 8, (size_t)(n + 1), f) == (size_t)(n + 1) &&
            (nnz == 0 || fwrite(col, 4, (size_t)nnz, f) == (size_t)nnz) &&
            (!w || nnz == 0 || fwrite(w, 4, (size_t)nnz, f) == (size_t)nnz);
  ok = (fclose(f) == 0) && ok;
  return ok ? 0 : fail(std::string("write failed: ") + path);
}
