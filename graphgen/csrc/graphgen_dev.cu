// graphgen_dev.cu -- device (B200) builders of the seeded synthetic inputs.
// Same recipes and bit-identical output as graphgen_host.cpp; used for the
// full-size configs (R-MAT scale 24/27, mesh 368^3, RGG 5e7) that the host
// builder would take minutes on.  Input module only (no Louvain arithmetic).
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>
#include <string>

#include "graphgen.h"
#include "gg_internal.h"

#define GG_CUDA(call)                                                          \
  do {                                                                         \
    cudaError_t e_ = (call);                                                   \
    if (e_ != cudaSuccess) {                                                   \
      char buf_[256];                                                          \
      snprintf(buf_, sizeof buf_, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
      gg_set_error(buf_);                                                      \
      return -5;                                                               \
    }                                                                          \
  } while (0)

namespace {

template <class T>
struct DevBuf {
  T* p = nullptr;
  size_t n = 0;
  cudaError_t alloc(size_t count) {
    n = count;
    return cudaMalloc(&p, sizeof(T) * (count ? count : 1));
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
  }
  ~DevBuf() { release(); }
};

inline unsigned blocks_for(int64_t n, int threads) {
  int64_t b = (n + threads - 1) / threads;
  if (b > 148LL * 64) b = 148LL * 64;  // grid-stride beyond this
  return (unsigned)(b < 1 ? 1 : b);
}

__global__ void k_rmat_keys(uint64_t seed, int64_t T, int scale, uint32_t tA, uint32_t tAB, uint32_t tABC,
                            uint64_t* keys) {
  const uint64_t sentinel = (scale >= 32) ? ~0ull : ((1ull << (2 * scale)) - 1ull);
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
    uint32_t u, v;
    gg_rmat_tuple(seed, (uint64_t)t, scale, tA, tAB, tABC, &u, &v);
    if (u == v) {
      keys[2 * t] = sentinel;
      keys[2 * t + 1] = sentinel;
    } else {
      keys[2 * t] = ((uint64_t)u << scale) | v;
      keys[2 * t + 1] = ((uint64_t)v << scale) | u;
    }
  }
}

__global__ void k_row_degree(const uint64_t* keys, int64_t M, int sb, int32_t* deg) {
  const unsigned lane = threadIdx.x & 31;
  int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < M; base += stride) {
    int64_t e = base + threadIdx.x;
    bool valid = e < M;
    uint32_t u = valid ? (uint32_t)(keys[e] >> sb) : 0xFFFFFFFFu;
    unsigned mask = __match_any_sync(0xFFFFFFFFu, u);
    if (valid && (__ffs(mask) - 1) == (int)lane) atomicAdd(&deg[u], __popc(mask));
  }
}

__global__ void k_flag_nonzero(const int32_t* deg, int64_t n, int compact, int32_t* flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    flag[i] = (!compact || deg[i] > 0) ? 1 : 0;
}

__global__ void k_scatter_deg(const int32_t* deg, const int32_t* newid, int64_t n, int compact, int64_t* rowcnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    if (!compact || deg[i] > 0) rowcnt[newid[i] + 1] = deg[i];
}

__global__ void k_col_from_keys(const uint64_t* keys, int64_t M, int sb, const int32_t* newid, int32_t* col) {
  const uint64_t vmask = (sb >= 64) ? ~0ull : ((1ull << sb) - 1ull);
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < M; e += (int64_t)gridDim.x * blockDim.x)
    col[e] = newid[keys[e] & vmask];
}

__global__ void k_remap_col(int32_t* col, int64_t M, const int32_t* newid) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < M; e += (int64_t)gridDim.x * blockDim.x)
    col[e] = newid[col[e]];
}

// Sorted unique keys (u << sb | v) over vertex space nfull -> compacted CSR.
int build_csr_from_sorted_unique(const uint64_t* d_keys, int64_t M, int sb, int64_t nfull, int compact,
                                 gg_graph_s** out) {
  DevBuf<int32_t> deg, flag, newid;
  GG_CUDA(deg.alloc((size_t)nfull));
  GG_CUDA(flag.alloc((size_t)nfull));
  GG_CUDA(newid.alloc((size_t)nfull + 1));
  GG_CUDA(cudaMemset(deg.p, 0, sizeof(int32_t) * (size_t)nfull));
  if (M > 0) k_row_degree<<<blocks_for(M, 256), 256>>>(d_keys, M, sb, deg.p);
  k_flag_nonzero<<<blocks_for(nfull, 256), 256>>>(deg.p, nfull, compact, flag.p);
  size_t tb = 0;
  GG_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, flag.p, newid.p, (int64_t)nfull + 0));
  DevBuf<char> tmp;
  GG_CUDA(tmp.alloc(tb));
  GG_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tb, flag.p, newid.p, (int64_t)nfull));
  int32_t last_new = 0, last_flag = 0;
  GG_CUDA(cudaMemcpy(&last_new, newid.p + nfull - 1, 4, cudaMemcpyDeviceToHost));
  GG_CUDA(cudaMemcpy(&last_flag, flag.p + nfull - 1, 4, cudaMemcpyDeviceToHost));
  int64_t nn = (int64_t)last_new + last_flag;
  gg_graph_s* g = new gg_graph_s();
  g->n = nn;
  g->nnz = M;
  g->device = 1;
  g->labels = nullptr;
  g->rowptr = nullptr;
  g->col = nullptr;
  if (cudaMalloc(&g->rowptr, sizeof(int64_t) * (size_t)(nn + 1)) != cudaSuccess ||
      cudaMalloc(&g->col, sizeof(int32_t) * (size_t)(M > 0 ? M : 1)) != cudaSuccess) {
    gg_device_free(g);
    delete g;
    gg_set_error("cudaMalloc failed for output graph");
    return -4;
  }
  DevBuf<int64_t> rowcnt;
  GG_CUDA(rowcnt.alloc((size_t)nn + 1));
  GG_CUDA(cudaMemset(rowcnt.p, 0, sizeof(int64_t) * (size_t)(nn + 1)));
  k_scatter_deg<<<blocks_for(nfull, 256), 256>>>(deg.p, newid.p, nfull, compact, rowcnt.p);
  size_t tb2 = 0;
  GG_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb2, rowcnt.p, g->rowptr, (int64_t)nn + 1));
  DevBuf<char> tmp2;
  GG_CUDA(tmp2.alloc(tb2));
  GG_CUDA(cub::DeviceScan::InclusiveSum(tmp2.p, tb2, rowcnt.p, g->rowptr, (int64_t)nn + 1));
  if (M > 0) k_col_from_keys<<<blocks_for(M, 256), 256>>>(d_keys, M, sb, newid.p, g->col);
  GG_CUDA(cudaGetLastError());
  GG_CUDA(cudaDeviceSynchronize());
  *out = g;
  return 0;
}

// ------------------------------------------------------------------ mesh
__global__ void k_mesh_valid(uint64_t ncodes, int bits, int L, int morton, int32_t* flag) {
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < ncodes; c += (uint64_t)gridDim.x * blockDim.x) {
    if (morton) {
      uint32_t x, y, z;
      gg_morton3_decode(c, bits, &x, &y, &z);
      flag[c] = ((int)x < L && (int)y < L && (int)z < L) ? 1 : 0;
    } else {
      flag[c] = 1;
    }
  }
}

__global__ void k_mesh_inverse(uint64_t ncodes, const int32_t* flag, const int32_t* id_of_code, int64_t* code_of_id) {
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < ncodes; c += (uint64_t)gridDim.x * blockDim.x)
    if (flag[c]) code_of_id[id_of_code[c]] = (int64_t)c;
}

__device__ __forceinline__ void mesh_coords(int64_t code, int bits, int L, int morton, int* x, int* y, int* z) {
  if (morton) {
    uint32_t a, b, c;
    gg_morton3_decode((uint64_t)code, bits, &a, &b, &c);
    *x = (int)a; *y = (int)b; *z = (int)c;
  } else {
    *x = (int)(code % L);
    *y = (int)((code / L) % L);
    *z = (int)(code / ((int64_t)L * L));
  }
}

__device__ __forceinline__ int64_t mesh_code(int x, int y, int z, int bits, int L, int morton) {
  if (morton) return (int64_t)gg_morton3((uint32_t)x, (uint32_t)y, (uint32_t)z, bits);
  return (int64_t)x + (int64_t)L * (y + (int64_t)L * z);
}

__global__ void k_mesh_rows(int64_t n, int bits, int L, int morton, const int64_t* code_of_id,
                            const int32_t* id_of_code, const int64_t* rowptr, int64_t* rowcnt, int32_t* col) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    int x, y, z;
    mesh_coords(code_of_id[v], bits, L, morton, &x, &y, &z);
    int32_t nb[6];
    int k = 0;
    if (x > 0) nb[k++] = id_of_code[mesh_code(x - 1, y, z, bits, L, morton)];
    if (x < L - 1) nb[k++] = id_of_code[mesh_code(x + 1, y, z, bits, L, morton)];
    if (y > 0) nb[k++] = id_of_code[mesh_code(x, y - 1, z, bits, L, morton)];
    if (y < L - 1) nb[k++] = id_of_code[mesh_code(x, y + 1, z, bits, L, morton)];
    if (z > 0) nb[k++] = id_of_code[mesh_code(x, y, z - 1, bits, L, morton)];
    if (z < L - 1) nb[k++] = id_of_code[mesh_code(x, y, z + 1, bits, L, morton)];
    if (rowptr == nullptr) {
      rowcnt[v + 1] = k;
    } else {
      for (int i = 1; i < k; ++i) {  // insertion sort of <= 6 ids
        int32_t t = nb[i];
        int j = i - 1;
        while (j >= 0 && nb[j] > t) { nb[j + 1] = nb[j]; --j; }
        nb[j + 1] = t;
      }
      int64_t e = rowptr[v];
      for (int i = 0; i < k; ++i) col[e + i] = nb[i];
    }
  }
}

// ------------------------------------------------------------------ RGG
__global__ void k_rgg_points(int64_t n, uint64_t seed, int64_t G, double* x, double* y, uint32_t* cell, int32_t* idx) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    gg_u32x4 w = gg_philox4x32_10((uint32_t)i, (uint32_t)((uint64_t)i >> 32), 0u, 0x52474720u, (uint32_t)seed,
                                  (uint32_t)(seed >> 32));
    double px = gg_u01(w.v[0], w.v[1]), py = gg_u01(w.v[2], w.v[3]);
    int64_t cx = (int64_t)__dmul_rn(px, (double)G), cy = (int64_t)__dmul_rn(py, (double)G);
    if (cx >= G) cx = G - 1;
    if (cy >= G) cy = G - 1;
    x[i] = px;
    y[i] = py;
    cell[i] = (uint32_t)(cy * G + cx);
    idx[i] = (int32_t)i;
  }
}

__global__ void k_gather_d(const int32_t* perm, const double* src, double* dst, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = src[perm[i]];
}
__global__ void k_gather_u(const int32_t* perm, const uint32_t* src, uint32_t* dst, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = src[perm[i]];
}
__global__ void k_bits_of(const double* v, uint64_t* bits, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    bits[i] = (uint64_t)__double_as_longlong(v[i]);  // non-negative doubles order like their bits
}
__global__ void k_cell_count(const uint32_t* cell, int64_t n, int64_t* cstart) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd((unsigned long long*)&cstart[cell[i] + 1], 1ull);
}
__global__ void k_rgg_rows(int64_t n, int64_t G, double r2, const double* x, const double* y, const uint32_t* cell,
                           const int64_t* cstart, const int64_t* rowptr, int64_t* rowcnt, int32_t* col) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t c = cell[i];
    int64_t cx = c % G, cy = c / G;
    double px = x[i], py = y[i];
    int64_t cnt = 0;
    int64_t e = rowptr ? rowptr[i] : 0;
    for (int64_t dy = -1; dy <= 1; ++dy) {
      int64_t yy = cy + dy;
      if (yy < 0 || yy >= G) continue;
      for (int64_t dx = -1; dx <= 1; ++dx) {
        int64_t xx = cx + dx;
        if (xx < 0 || xx >= G) continue;
        int64_t cc = yy * G + xx;
        for (int64_t j = cstart[cc]; j < cstart[cc + 1]; ++j) {
          if (j == i) continue;
          double ex = __dsub_rn(px, x[j]), ey = __dsub_rn(py, y[j]);
          double d2 = __dadd_rn(__dmul_rn(ex, ex), __dmul_rn(ey, ey));
          if (d2 < r2) {
            if (rowptr) col[e + cnt] = (int32_t)j;
            ++cnt;
          }
        }
      }
    }
    if (!rowptr) rowcnt[i + 1] = cnt;
  }
}
__global__ void k_deg_from_rowptr(const int64_t* rowptr, int64_t n, int32_t* deg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    deg[i] = (int32_t)(rowptr[i + 1] - rowptr[i]);
}

}  // namespace

void gg_device_free(gg_graph_s* g) {
  if (g->rowptr) cudaFree(g->rowptr);
  if (g->col) cudaFree(g->col);
  g->rowptr = nullptr;
  g->col = nullptr;
}

int gg_device_copy_out(gg_graph_s* g, int64_t* rowptr_dst, int32_t* col_dst) {
  return gg_copy_any(rowptr_dst, g->rowptr, sizeof(int64_t) * (size_t)(g->n + 1), col_dst, g->col,
                     sizeof(int32_t) * (size_t)g->nnz);
}

static bool is_device_ptr(const void* p) {
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();  // no driver / unregistered host memory: treat as host
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

static int copy_one(void* d, const void* s, size_t b) {
  if (!d || !b) return 0;
  if (!is_device_ptr(d) && !is_device_ptr(s)) {
    memcpy(d, s, b);
    return 0;
  }
  GG_CUDA(cudaMemcpy(d, s, b, cudaMemcpyDefault));
  return 0;
}

int gg_copy_any(void* d0, const void* s0, size_t b0, void* d1, const void* s1, size_t b1) {
  int rc = copy_one(d0, s0, b0);
  if (rc) return rc;
  return copy_one(d1, s1, b1);
}

extern "C" int gg_rmat_device(int scale, int64_t ntuples, uint64_t seed, double a, double b, double c, int compact,
                              gg_graph_t* out) {
  if (!out || scale < 1 || scale > 31 || ntuples < 0) { gg_set_error("bad args"); return -1; }
  uint32_t tA, tAB, tABC;
  gg_rmat_thresholds(a, b, c, &tA, &tAB, &tABC);
  int64_t N = 2 * ntuples;
  int bits = 2 * scale;
  const uint64_t sentinel = (1ull << bits) - 1ull;
  int64_t nfull = (int64_t)1 << scale;
  DevBuf<uint64_t> k0, k1;
  GG_CUDA(k0.alloc((size_t)N));
  GG_CUDA(k1.alloc((size_t)N));
  if (ntuples > 0) k_rmat_keys<<<blocks_for(ntuples, 256), 256>>>(seed, ntuples, scale, tA, tAB, tABC, k0.p);
  GG_CUDA(cudaGetLastError());
  cub::DoubleBuffer<uint64_t> db(k0.p, k1.p);
  size_t tb = 0;
  GG_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tb, db, N, 0, bits));
  {
    DevBuf<char> tmp;
    GG_CUDA(tmp.alloc(tb));
    GG_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, tb, db, N, 0, bits));
  }
  uint64_t* sorted = db.Current();
  uint64_t* other = db.Alternate();
  DevBuf<int64_t> nsel;
  GG_CUDA(nsel.alloc(1));
  size_t tu = 0;
  GG_CUDA(cub::DeviceSelect::Unique(nullptr, tu, sorted, other, nsel.p, N));
  int64_t M = 0;
  {
    DevBuf<char> tmp;
    GG_CUDA(tmp.alloc(tu));
    GG_CUDA(cub::DeviceSelect::Unique(tmp.p, tu, sorted, other, nsel.p, N));
    GG_CUDA(cudaMemcpy(&M, nsel.p, 8, cudaMemcpyDeviceToHost));
  }
  if (M > 0) {
    uint64_t lastk = 0;
    GG_CUDA(cudaMemcpy(&lastk, other + M - 1, 8, cudaMemcpyDeviceToHost));
    if (lastk == sentinel) --M;  // self-loop sentinel sorts last
  }
  // release the sorted copy before building (keeps peak memory at 2 key buffers)
  if (sorted == k0.p) k0.release(); else k1.release();
  return build_csr_from_sorted_unique(other, M, scale, nfull, compact, out);
}

extern "C" int gg_mesh3d_device(int L, int morton, gg_graph_t* out) {
  if (!out || L < 1 || L > 1024) { gg_set_error("bad args"); return -1; }
  int64_t n = (int64_t)L * L * L;
  if (n > INT32_MAX) { gg_set_error("mesh too large"); return -1; }
  int bits = gg_mesh_bits(L);
  uint64_t ncodes = morton ? (1ull << (3 * bits)) : (uint64_t)n;
  DevBuf<int32_t> flag, idc;
  DevBuf<int64_t> coi;
  GG_CUDA(flag.alloc(ncodes));
  GG_CUDA(idc.alloc(ncodes));
  GG_CUDA(coi.alloc((size_t)n));
  k_mesh_valid<<<blocks_for((int64_t)ncodes, 256), 256>>>(ncodes, bits, L, morton, flag.p);
  size_t tb = 0;
  GG_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, flag.p, idc.p, (int64_t)ncodes));
  {
    DevBuf<char> tmp;
    GG_CUDA(tmp.alloc(tb));
    GG_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tb, flag.p, idc.p, (int64_t)ncodes));
  }
  k_mesh_inverse<<<blocks_for((int64_t)ncodes, 256), 256>>>(ncodes, flag.p, idc.p, coi.p);
  flag.release();
  int64_t nnz = 6 * n - 6 * (int64_t)L * L;
  gg_graph_s* g = new gg_graph_s();
  g->n = n; g->nnz = nnz; g->device = 1; g->labels = nullptr; g->rowptr = nullptr; g->col = nullptr;
  if (cudaMalloc(&g->rowptr, sizeof(int64_t) * (size_t)(n + 1)) != cudaSuccess ||
      cudaMalloc(&g->col, sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1)) != cudaSuccess) {
    gg_device_free(g); delete g; gg_set_error("cudaMalloc failed"); return -4;
  }
  DevBuf<int64_t> rowcnt;
  GG_CUDA(rowcnt.alloc((size_t)n + 1));
  GG_CUDA(cudaMemset(rowcnt.p, 0, sizeof(int64_t) * (size_t)(n + 1)));
  k_mesh_rows<<<blocks_for(n, 256), 256>>>(n, bits, L, morton, coi.p, idc.p, nullptr, rowcnt.p, nullptr);
  size_t tb2 = 0;
  GG_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb2, rowcnt.p, g->rowptr, (int64_t)n + 1));
  {
    DevBuf<char> tmp;
    GG_CUDA(tmp.alloc(tb2));
    GG_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb2, rowcnt.p, g->rowptr, (int64_t)n + 1));
  }
  k_mesh_rows<<<blocks_for(n, 256), 256>>>(n, bits, L, morton, coi.p, idc.p, g->rowptr, nullptr, g->col);
  GG_CUDA(cudaGetLastError());
  GG_CUDA(cudaDeviceSynchronize());
  *out = g;
  return 0;
}

extern "C" int gg_rgg_device(int64_t n, double rfac, uint64_t seed, int compact, gg_graph_t* out) {
  if (!out || n < 2 || n > INT32_MAX) { gg_set_error("bad args"); return -1; }
  double r = gg_rgg_radius(n, rfac);
  double r2 = r * r;
  int64_t G = (int64_t)(1.0 / r);
  if (G < 1) G = 1;
  if (G * G >= (int64_t)UINT32_MAX) { gg_set_error("grid too fine"); return -1; }
  DevBuf<double> x, y, x2, y2;
  DevBuf<uint32_t> cell, cell2;
  DevBuf<int32_t> idx, idx2;
  DevBuf<uint64_t> kb, kb2;
  GG_CUDA(x.alloc(n)); GG_CUDA(y.alloc(n)); GG_CUDA(x2.alloc(n)); GG_CUDA(y2.alloc(n));
  GG_CUDA(cell.alloc(n)); GG_CUDA(cell2.alloc(n)); GG_CUDA(idx.alloc(n)); GG_CUDA(idx2.alloc(n));
  GG_CUDA(kb.alloc(n)); GG_CUDA(kb2.alloc(n));
  k_rgg_points<<<blocks_for(n, 256), 256>>>(n, seed, G, x.p, y.p, cell.p, idx.p);
  // Stable LSD sort by (cell, x, y, i): permutation idx sorted by y, then x, then cell.
  size_t tb = 0, tbc = 0;
  GG_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, kb.p, kb2.p, idx.p, idx2.p, n));
  GG_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tbc, cell.p, cell2.p, idx.p, idx2.p, n));
  DevBuf<char> tmp;
  GG_CUDA(tmp.alloc(tb > tbc ? tb : tbc));
  size_t tbm = tmp.n;
  // pass 1: key y
  k_bits_of<<<blocks_for(n, 256), 256>>>(y.p, kb.p, n);
  GG_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tbm, kb.p, kb2.p, idx.p, idx2.p, n));
  // pass 2: key x (gathered through the current permutation)
  k_gather_d<<<blocks_for(n, 256), 256>>>(idx2.p, x.p, x2.p, n);
  k_bits_of<<<blocks_for(n, 256), 256>>>(x2.p, kb.p, n);
  tbm = tmp.n;
  GG_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tbm, kb.p, kb2.p, idx2.p, idx.p, n));
  // pass 3: key cell
  k_gather_u<<<blocks_for(n, 256), 256>>>(idx.p, cell.p, cell2.p, n);
  tbm = tmp.n;
  GG_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tbm, cell2.p, cell.p, idx.p, idx2.p, n));
  // now idx2 = permutation (new id -> original point); cell holds sorted cells
  k_gather_d<<<blocks_for(n, 256), 256>>>(idx2.p, x.p, x2.p, n);
  k_gather_d<<<blocks_for(n, 256), 256>>>(idx2.p, y.p, y2.p, n);
  x.release(); y.release(); kb.release(); kb2.release(); idx.release(); cell2.release();
  DevBuf<int64_t> cstart;
  GG_CUDA(cstart.alloc((size_t)(G * G + 1)));
  GG_CUDA(cudaMemset(cstart.p, 0, sizeof(int64_t) * (size_t)(G * G + 1)));
  k_cell_count<<<blocks_for(n, 256), 256>>>(cell.p, n, cstart.p);
  size_t tb3 = 0;
  GG_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb3, cstart.p, cstart.p, G * G + 1));
  {
    DevBuf<char> t3;
    GG_CUDA(t3.alloc(tb3));
    GG_CUDA(cub::DeviceScan::InclusiveSum(t3.p, tb3, cstart.p, cstart.p, G * G + 1));
  }
  DevBuf<int64_t> rowcnt, rowptr;
  GG_CUDA(rowcnt.alloc(n + 1)); GG_CUDA(rowptr.alloc(n + 1));
  GG_CUDA(cudaMemset(rowcnt.p, 0, sizeof(int64_t) * (size_t)(n + 1)));
  k_rgg_rows<<<blocks_for(n, 256), 256>>>(n, G, r2, x2.p, y2.p, cell.p, cstart.p, nullptr, rowcnt.p, nullptr);
  size_t tb4 = 0;
  GG_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb4, rowcnt.p, rowptr.p, n + 1));
  {
    DevBuf<char> t4;
    GG_CUDA(t4.alloc(tb4));
    GG_CUDA(cub::DeviceScan::InclusiveSum(t4.p, tb4, rowcnt.p, rowptr.p, n + 1));
  }
  int64_t nnz = 0;
  GG_CUDA(cudaMemcpy(&nnz, rowptr.p + n, 8, cudaMemcpyDeviceToHost));
  DevBuf<int32_t> col;
  GG_CUDA(col.alloc((size_t)nnz));
  k_rgg_rows<<<blocks_for(n, 256), 256>>>(n, G, r2, x2.p, y2.p, cell.p, cstart.p, rowptr.p, nullptr, col.p);
  GG_CUDA(cudaGetLastError());
  // compaction of isolated points (order preserving)
  DevBuf<int32_t> deg, flag, newid;
  GG_CUDA(deg.alloc(n)); GG_CUDA(flag.alloc(n)); GG_CUDA(newid.alloc(n));
  k_deg_from_rowptr<<<blocks_for(n, 256), 256>>>(rowptr.p, n, deg.p);
  k_flag_nonzero<<<blocks_for(n, 256), 256>>>(deg.p, n, compact, flag.p);
  size_t tb5 = 0;
  GG_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb5, flag.p, newid.p, n));
  {
    DevBuf<char> t5;
    GG_CUDA(t5.alloc(tb5));
    GG_CUDA(cub::DeviceScan::ExclusiveSum(t5.p, tb5, flag.p, newid.p, n));
  }
  int32_t last_new = 0, last_flag = 0;
  GG_CUDA(cudaMemcpy(&last_new, newid.p + n - 1, 4, cudaMemcpyDeviceToHost));
  GG_CUDA(cudaMemcpy(&last_flag, flag.p + n - 1, 4, cudaMemcpyDeviceToHost));
  int64_t nn = (int64_t)last_new + last_flag;
  gg_graph_s* g = new gg_graph_s();
  g->n = nn; g->nnz = nnz; g->device = 1; g->labels = nullptr; g->rowptr = nullptr; g->col = nullptr;
  if (cudaMalloc(&g->rowptr, sizeof(int64_t) * (size_t)(nn + 1)) != cudaSuccess) {
    delete g; gg_set_error("cudaMalloc failed"); return -4;
  }
  GG_CUDA(cudaMemset(rowcnt.p, 0, sizeof(int64_t) * (size_t)(n + 1)));
  k_scatter_deg<<<blocks_for(n, 256), 256>>>(deg.p, newid.p, n, compact, rowcnt.p);
  size_t tb6 = 0;
  GG_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb6, rowcnt.p, g->rowptr, nn + 1));
  {
    DevBuf<char> t6;
    GG_CUDA(t6.alloc(tb6));
    GG_CUDA(cub::DeviceScan::InclusiveSum(t6.p, tb6, rowcnt.p, g->rowptr, nn + 1));
  }
  if (nnz > 0) k_remap_col<<<blocks_for(nnz, 256), 256>>>(col.p, nnz, newid.p);
  GG_CUDA(cudaGetLastError());
  GG_CUDA(cudaDeviceSynchronize());
  g->col = col.p;
  col.p = nullptr;  // ownership moves to the graph
  *out = g;
  return 0;
}
