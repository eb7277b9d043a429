// lv_level.cu -- per-level kernels of the GPU Louvain hot path (sm_100a):
// level setup (Alg. 1 l.2), degree binning, commit
// (Alg. 1 l.8-11), exact modularity (Eq. 1) and
// contraction (Alg. 3).  See DESIGN.md for the byte model of each.
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "lv_device.cuh"
#include "lv_internal.cuh"

namespace lv {

namespace {

constexpr int kTileEdges = 2048;  // edges per block tile in edge-centric kernels
constexpr int kTileRows = 2048;   // rowptr entries staged in smem per tile

__global__ void k_degrees_unit(const int64_t* rowptr, int64_t n, uint32_t* k) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    k[i] = (uint32_t)(rowptr[i + 1] - rowptr[i]);
}

__global__ void k_init_singletons(const uint32_t* k, int64_t n, uint2* ca, int32_t* size, int32_t* C) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    ca[i] = make_uint2((uint32_t)i, k[i]);  // C[i] = i, a_C(i) = k_i
    C[i] = (int32_t)i;
    size[i] = 1;
  }
}

// C[i] = labels[i] (or i), a = 0, size = 0; the C write keeps the packed record's a word.
__global__ void k_set_C(const int32_t* labels, int64_t n, uint2* ca, int32_t* size, int32_t* C) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    ca[i] = make_uint2(labels ? (uint32_t)labels[i] : (uint32_t)i, 0u);
    C[i] = labels ? labels[i] : (int32_t)i;
    size[i] = 0;
  }
}

// a_c = sum_{i in c} k_i and size_c; the lanes of a warp holding the same
// label are merged first (__match_any_sync): a final partition has few, large
// communities, and one atomic per vertex on them serialises.
__global__ void k_totals_add(const uint2* ca, const uint32_t* k, int64_t n, int32_t* size, unsigned long long* bad) {
  uint32_t* a = const_cast<uint32_t*>(reinterpret_cast<const uint32_t*>(ca)) + 1;  // a word, stride 2
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t base = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; base < n; base += nw * 32) {
    const int64_t i = base + lane;
    int32_t c = (i < n) ? (int32_t)ca[i].x : -1;
    if (i < n && (c < 0 || c >= n)) {
      atomicAdd(bad, 1ull);
      c = -1;
    }
    const bool valid = c >= 0;
    const uint32_t ki = valid ? k[i] : 0u;
    const unsigned m = __match_any_sync(kFull, valid ? c : (int32_t)(0x80000000u | (unsigned)lane));
    const uint32_t ks = __reduce_add_sync(m, ki);
    if (valid && lane == __ffs(m) - 1) {
      atomicAdd(&a[2 * (int64_t)c], ks);
      atomicAdd(&size[c], __popc(m));
    }
  }
}

// a_c of an external labelling (louvain_modularity with labels != NULL)
__global__ void k_ext_totals(const int32_t* C, const uint32_t* k, int64_t n, uint32_t* a, unsigned long long* bad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = C[i];
    if (c < 0 || c >= n) { atomicAdd(bad, 1ull); continue; }
    atomicAdd(&a[c], k[i]);
  }
}

__global__ void k_get_C(const uint2* ca, int64_t n, int32_t* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (int32_t)ca[i].x;
}

__global__ void k_get_a(const uint2* ca, int64_t n, uint32_t* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = ca[i].y;
}

// class = 8*bucket + sub  (lv_internal.cuh)
__global__ void k_classify(const int64_t* rowptr, int64_t n, int64_t b0, int64_t b1, int64_t b2, int64_t b3,
                           int64_t b4, int64_t b5, int64_t lo, int64_t hi, uint8_t* cls, int32_t* iota,
                           unsigned long long* hist) {
  __shared__ unsigned long long sh[kNumClasses];
  if (threadIdx.x < kNumClasses) sh[threadIdx.x] = 0;
  __syncthreads();
  // uniform trip count per warp so the class counts can be merged with __match_any_sync
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i0 = blockIdx.x * (int64_t)blockDim.x + (threadIdx.x & ~31); i0 < n; i0 += stride) {
    const int64_t i = i0 + (threadIdx.x & 31);
    const bool has = i < n;
    const int64_t d = has ? rowptr[i + 1] - rowptr[i] : 0;  // R11: row length incl. self-loop
    int b;
    if (d == 0 || i < lo || i >= hi) b = 0;  // not decided here (no edges, or owned by another rank)
    else if (d <= b0) b = 1;
    else if (d <= b1) b = 2;
    else if (d <= b2) b = 3;
    else if (d <= b3) b = 4;
    else if (d <= b4) b = 5;
    else if (d <= b5) b = 6;
    else b = 7;
    // buckets whose bound is <= 32 (the register kernels): sub-class by the power of two
    // of the degree, so each vertex gets a lane group of its own size (deg 1: one lane)
    const int64_t bound = b == 1 ? b0 : b == 2 ? b1 : b == 3 ? b2 : b == 4 ? b3 : b == 5 ? b4 : b == 6 ? b5 : INT64_MAX;
    const int sub = (b >= 1 && bound <= kSmallMaxDeg) ? small_sub_of_degree(d) : sub_of_degree(d);
    const uint8_t c = (uint8_t)(kSubPerBucket * b + sub);
    if (has) {
      cls[i] = c;
      iota[i] = (int32_t)i;
    }
    const unsigned m = __match_any_sync(0xffffffffu, has ? (int)c : -1);  // one smem atomic per class per warp
    if (has && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(&sh[c], (unsigned long long)__popc(m));
  }
  __syncthreads();
  if (threadIdx.x < kNumClasses && sh[threadIdx.x]) atomicAdd(&hist[threadIdx.x], sh[threadIdx.x]);
}

__global__ void k_hub_degrees(const int32_t* hv, int64_t nh, const int64_t* rowptr, int64_t* deg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nh; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t v = hv[i];
    deg[i] = rowptr[v + 1] - rowptr[v];
    deg[nh + i] = rowptr[v];
  }
}

__global__ void k_bin_degrees(const int32_t* bv, int64_t n, const int64_t* rowptr, int64_t* dg, int64_t* brb) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x) {
    if (i < n) {
      const int64_t rb = rowptr[bv[i]];
      dg[i] = rowptr[bv[i] + 1] - rb;
      brb[i] = rb;
    } else {
      dg[i] = 0;
    }
  }
}

__global__ void k_fill_u64(unsigned long long* p, int64_t n, unsigned long long v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}
__global__ void k_fill_u32v(uint32_t* p, int64_t n, uint32_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}

// Commit of one bucket (Alg. 1 l.8-11): C[i] = newComm[i] and the exact
// integer a_c / size_c deltas (identical to recomputing a_c, R12).
__global__ void k_commit(DevCtl* ctl, int bucket, const int32_t* mv_v, const int32_t* mv_new, int32_t* mv_old,
                         uint2* ca, int32_t* size, const uint32_t* k, int32_t* C, const int64_t* rowptr,
                         uint2* pcn) {
  const unsigned long long start = ctl->bounds[bucket];
  const unsigned long long end = *(volatile unsigned long long*)&ctl->logn;
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->bounds[bucket + 1] = end;
  uint32_t* w32 = reinterpret_cast<uint32_t*>(ca);
  unsigned long long md = 0;
  const int lane = threadIdx.x & 31;
  // warp-uniform trips: moves into one community (a hub absorbing its degree-1
  // neighbours) are summed per warp first, one atomic pair per distinct label
  for (unsigned long long b = start + blockIdx.x * (unsigned long long)blockDim.x + (threadIdx.x - lane); b < end;
       b += (unsigned long long)gridDim.x * blockDim.x) {
    const unsigned long long p = b + lane;
    const bool act = p < end;
    int32_t i = 0, t = -1 - lane, old = -1 - lane;  // idle lanes: distinct negative labels
    uint32_t ki = 0;
    if (act) {
      i = mv_v[p];
      t = mv_new[p];
      old = (int32_t)w32[2 * (int64_t)i];
      mv_old[p] = old;
      w32[2 * (int64_t)i] = (uint32_t)t;
      C[i] = t;
      if (pcn) pcn[i].y = (uint32_t)t;
      ki = k[i];
      if (rowptr) md += (unsigned long long)(rowptr[i + 1] - rowptr[i]);
    }
#pragma unroll
    for (int side = 0; side < 2; ++side) {
      const int32_t c = side ? old : t;
      unsigned m = 1u << lane;
      uint32_t x = ki;
      if (__any_sync(kFull, c == __shfl_xor_sync(kFull, c, 1))) {
        m = __match_any_sync(kFull, c);
        x = __reduce_add_sync(m, ki);
      }
      if (c >= 0 && lane == __ffs(m) - 1) {
        if (side) {
          atomicSub(&w32[2 * (int64_t)c + 1], x);
          atomicSub(&size[c], __popc(m));
        } else {
          atomicAdd(&w32[2 * (int64_t)c + 1], x);
          atomicAdd(&size[c], __popc(m));
        }
      }
    }
  }
  md = warp_sum_u64(md);
  if ((threadIdx.x & 31) == 0 && md) atomicAdd(&ctl->mdeg, md);
}

// Undo every move of the sweep (R15).
__global__ void k_revert(const DevCtl* ctl, const int32_t* mv_v, const int32_t* mv_new, const int32_t* mv_old,
                         uint2* ca, int32_t* size, const uint32_t* k, int32_t* C) {
  const unsigned long long end = ctl->logn;
  uint32_t* w32 = reinterpret_cast<uint32_t*>(ca);
  for (unsigned long long p = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; p < end;
       p += (unsigned long long)gridDim.x * blockDim.x) {
    const int32_t i = mv_v[p], t = mv_new[p], old = mv_old[p];
    w32[2 * (int64_t)i] = (uint32_t)old;
    C[i] = old;
    const uint32_t ki = k[i];
    atomicSub(&w32[2 * (int64_t)t + 1], ki);
    atomicAdd(&w32[2 * (int64_t)old + 1], ki);
    atomicSub(&size[t], 1);
    atomicAdd(&size[old], 1);
  }
}

// Edge-centric tile walker: calls f(u, e) for every CSR entry e of the tile
// [e0, e1) with its source row u.  The tile's rowptr window is staged in smem
// and each thread binary-searches it (coalesced col/w loads; degree-skew free).
// tr = tile plan (tile_starts): rows tr[tile] .. tr[tile + 1] cover the tile.
template <class F>
__device__ __forceinline__ void for_tile_edges(const int64_t* rowptr, int64_t n, int64_t e0, int64_t e1,
                                               const int64_t* tr, int64_t tile, int64_t* sh_rows, int64_t* sh_u0,
                                               int* sh_nr, F f) {
  if (threadIdx.x == 0) {
    const int64_t u0 = tr[tile];
    const int64_t u1 = tr[tile + 1];
    *sh_u0 = u0;
    *sh_nr = (u1 - u0 + 2 <= kTileRows) ? (int)(u1 - u0 + 2) : -1;
  }
  __syncthreads();
  const int64_t u0 = *sh_u0;
  const int nr = *sh_nr;
  for (int t = threadIdx.x; t < nr; t += blockDim.x) sh_rows[t] = rowptr[u0 + t];
  __syncthreads();
  for (int64_t e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
    int64_t u;
    if (nr > 0) {
      int lo = 0, hi = nr - 2;  // largest r with sh_rows[r] <= e
      while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (sh_rows[mid] <= e) lo = mid; else hi = mid - 1;
      }
      u = u0 + lo;
    } else {
      u = row_of(rowptr, n, e);
    }
    f(u, e);
  }
  __syncthreads();
}

// Eq. (1): L = sum of w over entries (u,v) with C[u] = C[v] (self-loops
// included, R2); S = sum_c a_c^2.  Integer atomics: deterministic.  Labels come
// from the packed records (C = ca.x, a = ca.y) or from an external labelling.
// SINGLE: the partition is known to be singletons (distinct labels, level start,
// P:164), so C(u) = C(v) iff u = v: L = sum of self-loop weights, no label gathers.
template <bool PACKED, bool SINGLE = false>
__global__ void __launch_bounds__(256) k_modularity(const int64_t* rowptr, int64_t n, const int32_t* col,
                                                    const uint32_t* w, const uint2* ca, const int32_t* C,
                                                    const uint32_t* a, int64_t e_begin, int64_t nnz,
                                                    const int64_t* __restrict__ tr, unsigned long long* Lout,
                                                    unsigned long long* Sout, const DevCtl* gate = nullptr) {
  if (gate && delta_chosen(*gate, nnz)) return;  // the delta pass evaluates this sweep
  __shared__ int64_t sh_rows[kTileRows];
  __shared__ int64_t sh_u0;
  __shared__ int sh_nr;
  const uint32_t* lab = reinterpret_cast<const uint32_t*>(C);  // 4-byte labels (the level's copy, or external)
  unsigned long long acc = 0;
  const int64_t ntiles = (nnz - e_begin + kTileEdges - 1) / kTileEdges;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t e0 = e_begin + tile * kTileEdges, e1 = min(nnz, e0 + kTileEdges);
    for_tile_edges(rowptr, n, e0, e1, tr, tile, sh_rows, &sh_u0, &sh_nr, [&](int64_t u, int64_t e) {
      // the CSR is symmetric (both directions stored; a precondition of
      // every louvain_* call), so each pair u < v is counted twice from row u and
      // row v's copy is skipped: half the random label gathers, same L
      const int32_t v = __ldcs(&col[e]);
      if (v >= (int32_t)u) {
        const uint32_t we = w ? __ldcs(&w[e]) : 1u;
        if (v == (int32_t)u) acc += we;  // self-loop (stored once, R2)
        else if (!SINGLE && __ldg(&lab[v]) == __ldg(&lab[u])) acc += 2ull * we;
      }
    });
  }
  unsigned long long s2 = 0;
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long x = PACKED ? ca[c].y : a[c];
    s2 += x * x;
  }
  acc = warp_sum_u64(acc);
  s2 = warp_sum_u64(s2);
  if ((threadIdx.x & 31) == 0) {
    if (acc) atomicAdd(Lout, acc);
    if (s2) atomicAdd(Sout, s2);
  }
}

// Delta pass of Eq. (1) after a sweep (used by louvain_run when the moved vertices
// hold <= nnz/LV_DELTA_DIV entries; default: always).  L = sum over directed entries (u->v) of w [C(u) == C(v)]
// (self-loops once, R2) changes only on entries with a moved endpoint.  For a moved
// i (old label o, new t) and each entry (i->j), j != i:
//   d = [C'(j) == t] - [C(j) == o]     (C = labels at the sweep start, C' = after)
// counts for both directions (x2) when j did not move -- the mirror (j->i) holds
// the same w and the same d (symmetric CSR) -- and once when j moved too (its own
// row supplies (j->i)).  Self-loops never change.  Exact integers, any order.
constexpr int64_t kDeltaBigDeg = 4096;  // rows longer than this: one CTA each
__device__ __forceinline__ long long delta_entry(const uint2* __restrict__ P, int32_t i, int32_t j, uint32_t we,
                                                 int32_t t, int32_t o) {
  if (j == i) return 0;
  const uint2 pj = __ldg(&P[j]);  // {C(j), C'(j)}: one sector for both labels
  const int d = (int)((int32_t)pj.y == t) - (int)((int32_t)pj.x == o);
  return d ? (long long)d * (long long)we * (pj.x != pj.y ? 1 : 2) : 0;
}

__global__ void k_snapshot(const int32_t* __restrict__ C, int64_t n, uint2* P) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t c = (uint32_t)C[i];
    P[i] = make_uint2(c, c);
  }
}

constexpr int64_t kDeltaThrDeg = 32;    // rows up to this length: one thread each
__global__ void __launch_bounds__(256) k_mod_delta_thr(DevCtl* ctl, const int32_t* __restrict__ mv_v,
                                                       const int32_t* __restrict__ mv_new,
                                                       const int32_t* __restrict__ mv_old,
                                                       const int64_t* __restrict__ rowptr,
                                                       const int32_t* __restrict__ col,
                                                       const uint32_t* __restrict__ w, const uint2* __restrict__ P,
                                                       int64_t nnz, int32_t* mid,
                                                       int32_t* big, int64_t own_lo, int64_t own_hi) {
  if (!delta_chosen(*ctl, nnz)) return;
  const long long logn = (long long)ctl->logn;
  long long acc = 0;
  for (long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x; p < logn; p += (long long)gridDim.x * blockDim.x) {
    const int32_t i = mv_v[p];
    if (i < own_lo || i >= own_hi) continue;  // sharded run: another rank sums this moved row
    const int64_t b = rowptr[i], e = rowptr[i + 1];
    if (e - b > kDeltaBigDeg) {
      big[atomicAdd(&ctl->nbig, 1ull)] = (int32_t)p;
    } else if (e - b > kDeltaThrDeg) {
      mid[atomicAdd(&ctl->nmid, 1ull)] = (int32_t)p;
    } else {
      const int32_t t = mv_new[p], o = mv_old[p];
      for (int64_t q = b; q < e; q += 4) {  // 4 independent gathers in flight
        int32_t j[4];
        uint32_t x[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          j[u] = q + u < e ? __ldcs(&col[q + u]) : i;  // j = i contributes 0 without a gather
          x[u] = (w && q + u < e) ? __ldcs(&w[q + u]) : 1u;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) acc += delta_entry(P, i, j[u], x[u], t, o);
      }
    }
  }
  const unsigned long long s = warp_sum_u64((unsigned long long)acc);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(&ctl->dL, s);
}

__global__ void __launch_bounds__(256) k_mod_delta_warp(DevCtl* ctl, const int32_t* __restrict__ mid,
                                                        const int32_t* __restrict__ mv_v,
                                                        const int32_t* __restrict__ mv_new,
                                                        const int32_t* __restrict__ mv_old,
                                                        const int64_t* __restrict__ rowptr,
                                                        const int32_t* __restrict__ col,
                                                        const uint32_t* __restrict__ w, const uint2* __restrict__ P,
                                                        int64_t nnz) {
  if (!delta_chosen(*ctl, nnz)) return;
  const long long nmid = (long long)ctl->nmid;
  const int lane = threadIdx.x & 31;
  const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
  long long acc = 0;
  for (long long k = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < nmid; k += nw) {
    const int32_t p = mid[k];
    const int32_t i = mv_v[p], t = mv_new[p], o = mv_old[p];
    const int64_t b = rowptr[i], e = rowptr[i + 1];
    for (int64_t q = b + lane; q < e; q += 64) {  // 2 independent gathers in flight per lane
      const bool has1 = q + 32 < e;
      const int32_t j0 = __ldcs(&col[q]), j1 = has1 ? __ldcs(&col[q + 32]) : i;
      const uint32_t x0 = w ? __ldcs(&w[q]) : 1u, x1 = (w && has1) ? __ldcs(&w[q + 32]) : 1u;
      acc += delta_entry(P, i, j0, x0, t, o) + delta_entry(P, i, j1, x1, t, o);
    }
  }
  const unsigned long long s = warp_sum_u64((unsigned long long)acc);
  if (lane == 0 && s) atomicAdd(&ctl->dL, s);
}

// Long rows of the delta pass (one CTA per moved vertex) and S = sum_c a_c^2.
__global__ void __launch_bounds__(512) k_mod_delta_cta(DevCtl* ctl, const int32_t* __restrict__ big,
                                                       const int32_t* __restrict__ mv_v,
                                                       const int32_t* __restrict__ mv_new,
                                                       const int32_t* __restrict__ mv_old,
                                                       const int64_t* __restrict__ rowptr,
                                                       const int32_t* __restrict__ col,
                                                       const uint32_t* __restrict__ w, const uint2* __restrict__ P,
                                                       int64_t nnz, const uint2* ca,
                                                       int64_t n) {
  if (!delta_chosen(*ctl, nnz)) return;
  const unsigned long long nbig = ctl->nbig;
  long long acc = 0;
  for (unsigned long long k = blockIdx.x; k < nbig; k += gridDim.x) {
    const int32_t p = big[k];
    const int32_t i = mv_v[p], t = mv_new[p], o = mv_old[p];
    for (int64_t q = rowptr[i] + threadIdx.x; q < rowptr[i + 1]; q += blockDim.x)
      acc += delta_entry(P, i, __ldcs(&col[q]), w ? __ldcs(&w[q]) : 1u, t, o);
  }
  unsigned long long s2 = 0;
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long x = ca[c].y;
    s2 += x * x;
  }
  const unsigned long long s = warp_sum_u64((unsigned long long)acc);
  s2 = warp_sum_u64(s2);
  if ((threadIdx.x & 31) == 0) {
    if (s) atomicAdd(&ctl->dL, s);
    if (s2) atomicAdd(&ctl->S, s2);
  }
}

// ---------------------------------------------------------------- contraction
__global__ void k_flags_nonempty(const int32_t* size, int64_t n, int32_t* flag) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x)
    flag[c] = size[c] > 0 ? 1 : 0;
}

// Degree of a contracted vertex = total of its community (R18: the merged row
// sums every member's row), so the next level's k needs no reduction.
__global__ void k_next_degrees(const uint2* ca, const int32_t* size, const int32_t* newID, int64_t n, uint32_t* kout) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x)
    if (size[c] > 0) kout[newID[c]] = ca[c].y;
}

__global__ void k_map(const uint2* ca, const int32_t* newID, int64_t n, int32_t* map) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    map[i] = newID[ca[i].x];  // R17: new ids in label order
}

__global__ void __launch_bounds__(256) k_emit_keys(const int64_t* rowptr, int64_t n, const int32_t* col,
                                                   const uint32_t* w, const int32_t* map, int64_t nnz, uint64_t np,
                                                   const int64_t* __restrict__ tr, unsigned long long* keys,
                                                   uint32_t* vals) {
  __shared__ int64_t sh_rows[kTileRows];
  __shared__ int64_t sh_u0;
  __shared__ int sh_nr;
  const int64_t ntiles = (nnz + kTileEdges - 1) / kTileEdges;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t e0 = tile * kTileEdges, e1 = min(nnz, e0 + kTileEdges);
    for_tile_edges(rowptr, n, e0, e1, tr, tile, sh_rows, &sh_u0, &sh_nr, [&](int64_t u, int64_t e) {
      keys[e] = (unsigned long long)map[u] * np + (unsigned long long)map[col[e]];  // (newID[C[u]], newID[C[v]])
      if (vals) vals[e] = w[e];
    });
  }
}

__global__ void k_row_counts(const unsigned long long* keys, int64_t m, uint64_t np, int64_t* cnt) {
  const unsigned lane = threadIdx.x & 31;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < m; base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = base + threadIdx.x;
    const bool valid = e < m;
    const uint32_t r = valid ? (uint32_t)(keys[e] / np) : 0xFFFFFFFFu;
    const unsigned mask = __match_any_sync(kFull, r);
    if (valid && (__ffs(mask) - 1) == (int)lane) atomicAdd((unsigned long long*)&cnt[r + 1], (unsigned long long)__popc(mask));
  }
}

__global__ void k_split_keys(const unsigned long long* keys, int64_t m, uint64_t np, int32_t* col) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m; e += (int64_t)gridDim.x * blockDim.x)
    col[e] = (int32_t)(keys[e] % np);
}

__global__ void k_compose(int32_t* lab, int64_t n0, const int32_t* map) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n0; i += (int64_t)gridDim.x * blockDim.x)
    lab[i] = map[lab[i]];
}
__global__ void k_compose_ca(int32_t* lab, int64_t n0, const uint2* ca) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n0; i += (int64_t)gridDim.x * blockDim.x)
    lab[i] = (int32_t)ca[lab[i]].x;
}

__global__ void k_sum_u32(const uint32_t* x, int64_t n, unsigned long long* out) {
  unsigned long long acc = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) acc += x[i];
  acc = warp_sum_u64(acc);
  if ((threadIdx.x & 31) == 0 && acc) atomicAdd(out, acc);
}

__global__ void k_tile_starts(const int64_t* __restrict__ offs, int64_t lo, int64_t hi, int64_t base, int64_t end,
                              int64_t T, int64_t ntiles, int64_t* out) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t <= ntiles; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = min(base + t * T, end - 1);
    int64_t a = lo, b = hi - 1;  // largest i in [lo, hi) with offs[i] <= x
    while (a < b) {
      const int64_t mid = (a + b + 1) >> 1;
      if (offs[mid] <= x) a = mid; else b = mid - 1;
    }
    out[t] = a;
  }
}

}  // namespace

int32_t tile_starts(Handle& h, const int64_t* offs, int64_t lo, int64_t hi, int64_t base, int64_t end, int64_t T,
                    const int64_t** out) {
  const int64_t ntiles = (end - base + T - 1) / T;
  void* p = nullptr;
  LV_TRY(scratch_get(h, SC_TILES, 8 * (size_t)(ntiles + 1), &p));
  k_tile_starts<<<grid_for(ntiles + 1, 256), 256, 0, h.stream>>>(offs, lo, hi, base, end, T, ntiles,
                                                                 static_cast<int64_t*>(p));
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  *out = static_cast<const int64_t*>(p);
  return LOUVAIN_OK;
}

// ======================================================================== host side
int32_t level_alloc_state(Level& L, cudaStream_t s) {
  LV_TRY(dalloc(&L.k, L.n, s));
  LV_TRY(dalloc(&L.ca, L.n, s));
  LV_TRY(dalloc(&L.C, L.n, s));
  LV_TRY(dalloc(&L.size, L.n, s));
  LV_TRY(dalloc(&L.mv_v, L.n, s));
  LV_TRY(dalloc(&L.mv_new, L.n, s));
  LV_TRY(dalloc(&L.mv_old, L.n, s));
  LV_TRY(dalloc(&L.bin_vertices, L.n, s));
  return LOUVAIN_OK;
}

static void part_free(PartPlan& Q, cudaStream_t s);
// Most partitions a vertex may get on the label-partitioned path (more: hub kernel).
// LV_PART_MAXP lowers it (tests use it to exercise the cooperative hub kernel).
static int64_t part_maxp() {
  static const int64_t v = [] {
    const char* e = getenv("LV_PART_MAXP");
    const long long x = e ? atoll(e) : 0;
    return (x >= 1 && x < kPartMaxP) ? (int64_t)x : (int64_t)kPartMaxP;
  }();
  return v;
}
// Vertices with more partitions than this take the pre-partitioned tasks, the
// others stream.  Measured on C5 with kPartLabels = 10240 (per 2 sweeps, levels
// 0/1/2): everything streaming 21.3 / 11.2 / 68.1 ms; P > 16 pre-partitioned
// 21.2 / 10.4 / 27.1 ms; the earlier rule (pre-partition all hubs of levels with
// mean degree >= 256, else P > 64) 21.8 / 10.8 / 31.7 ms.
static void hub_free(HubPlan& P, cudaStream_t s) {
  dfree(P.ins, s); dfree(P.scans, s); dfree(P.ins_off, s); dfree(P.scan_off, s); dfree(P.wave_hub, s);
  dfree(P.info, s); dfree(P.ring, s);
  dfree(P.partial, s);
  P = HubPlan();
}

int32_t level_alloc_scratch(Handle& h, Level& L, int parity) {
  const size_t n = (size_t)std::max<int64_t>(L.n, 1);
  auto get = [&](int a, size_t bytes, void** out) { return scratch_get(h, SC_LVL0 + 2 * a + parity, bytes, out); };
  LV_TRY(get(LA_K, 4 * n, (void**)&L.k));
  LV_TRY(get(LA_CA, 8 * n, (void**)&L.ca));
  LV_TRY(get(LA_C, 4 * n, (void**)&L.C));
  LV_TRY(get(LA_SIZE, 4 * n, (void**)&L.size));
  LV_TRY(get(LA_MVV, 4 * n, (void**)&L.mv_v));
  LV_TRY(get(LA_MVN, 4 * n, (void**)&L.mv_new));
  LV_TRY(get(LA_MVO, 4 * n, (void**)&L.mv_old));
  LV_TRY(get(LA_BIN, 4 * n, (void**)&L.bin_vertices));
  LV_TRY(get(LA_SOFF, 8 * (n + 1), (void**)&L.soff));
  LV_TRY(get(LA_BINRB, 8 * n, (void**)&L.bin_rb));
  L.scratch_backed = true;
  L.parity = parity;
  L.owns_csr = false;
  // peer-memory commits: the level's partition state lives in a replica set every rank
  // writes into (odd depth -> set 2, even depth -> set 1; the handle's level 0 -> set 0)
  if (dist_p2p(h)) LV_TRY(dist_bind_state(h, L, parity == 1 ? 2 : 1));
  return LOUVAIN_OK;
}

void level_free(Level& L, cudaStream_t s) {
  if (L.scratch_backed) {  // arrays belong to the handle's scratch; plans are per level
    dfree(L.mv_stamp, s);
    hub_free(L.hub, s);
    part_free(L.part, s);
    L = Level();
    return;
  }
  if (L.owns_csr) {
    dfree(L.rowptr, s);
    dfree(L.col, s);
    dfree(L.w, s);
  }
  dfree(L.k, s);
  if (!L.state_external) {  // else: a replica set of the distributed handle (lv_dist.cu)
    dfree(L.ca, s);
    dfree(L.C, s);
    dfree(L.size, s);
  }
  dfree(L.mv_v, s); dfree(L.mv_new, s); dfree(L.mv_old, s); dfree(L.bin_vertices, s); dfree(L.mv_stamp, s);
  dfree(L.soff, s);  // L.stage lives in the handle's scratch
  dfree(L.bin_rb, s);
  hub_free(L.hub, s);
  part_free(L.part, s);
  L = Level();
}

int32_t level_setup(Handle& h, Level& L) {
  cudaStream_t s = h.stream;
  const int64_t n = L.n;
  if (n == 0) { L.W = 0; return LOUVAIN_OK; }
  if (L.k_ready) {  // contracted level: k = community totals, W unchanged (set by level_contract)
    k_init_singletons<<<grid_for(n, 256), 256, 0, s>>>(L.k, n, L.ca, L.size, L.C);
    LV_LAUNCHED();
    LV_CUDA(cudaGetLastError());
    return LOUVAIN_OK;
  }
  if (L.w) {
    // k_i = weighted row sum
    size_t tb = 0;
    LV_CUDA(cub::DeviceSegmentedReduce::Sum(nullptr, tb, L.w, L.k, (int)n, L.rowptr, L.rowptr + 1, s));
    void* tmp = nullptr;
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceSegmentedReduce::Sum(tmp, tb, L.w, L.k, (int)n, L.rowptr, L.rowptr + 1, s)); LV_CUB();
    dfree(tmp, s);
  } else {
    k_degrees_unit<<<grid_for(n, 256), 256, 0, s>>>(L.rowptr, n, L.k);
    LV_LAUNCHED();
  }
  // W = sum_i k_i = 2m (R1)
  unsigned long long* dW = &h.ctl->L;  // reuse a ctl word as scratch
  LV_CUDA(cudaMemsetAsync(dW, 0, 8, s));
  k_sum_u32<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(L.k, n, dW);
  LV_LAUNCHED();
  unsigned long long W = 0;
  LV_CUDA(cudaMemcpyAsync(&W, dW, 8, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaStreamSynchronize(s));
  L.W = W;
  if (W > kWGuard) {
    set_error("W = 2m exceeds 3,037,000,499 (int64 gain guard, R4)");
    return LOUVAIN_E_OVERFLOW;
  }
  k_init_singletons<<<grid_for(n, 256), 256, 0, s>>>(L.k, n, L.ca, L.size, L.C);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t level_set_labels(Handle& h, Level& L, const int32_t* d_labels) {
  cudaStream_t s = h.stream;
  L.sweeps_done = d_labels ? 1 : 0;
  if (L.n == 0) return LOUVAIN_OK;
  if (!d_labels) {  // singletons: a = k, size = 1 directly
    k_init_singletons<<<grid_for(L.n, 256), 256, 0, s>>>(L.k, L.n, L.ca, L.size, L.C);
    LV_LAUNCHED();
    LV_CUDA(cudaGetLastError());
    return LOUVAIN_OK;
  }
  k_set_C<<<grid_for(L.n, 256), 256, 0, s>>>(d_labels, L.n, L.ca, L.size, L.C);
  LV_LAUNCHED();
  LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, s));
  k_totals_add<<<grid_for(L.n, 256), 256, 0, s>>>(L.ca, L.k, L.n, L.size, &h.ctl->bad);
  LV_LAUNCHED();
  unsigned long long bad = 0;
  LV_CUDA(cudaMemcpyAsync(&bad, &h.ctl->bad, 8, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaStreamSynchronize(s));
  if (bad) {
    set_error("labels out of range [0, n)");
    return LOUVAIN_E_INVALID_ARG;
  }
  return LOUVAIN_OK;
}

// Final partition of a run on the input level (labels in the last level's id
// space [0, n_last)): a_c is the last level's total of c (contraction preserves
// totals, R18) and size_c counts the input vertices labelled c -- one shared-memory
// histogram per CTA instead of global atomics on a few giant communities.
__global__ void k_copy_a(const uint2* __restrict__ ca_last, int64_t n_last, uint2* ca) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n_last; c += (int64_t)gridDim.x * blockDim.x)
    ca[c].y = ca_last[c].y;
}
__global__ void __launch_bounds__(1024) k_size_hist(const int32_t* __restrict__ lab, int64_t n, int nl, int32_t* size) {
  extern __shared__ int32_t hs[];
  for (int c = threadIdx.x; c < nl; c += blockDim.x) hs[c] = 0;
  __syncthreads();
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i0 = blockIdx.x * (int64_t)blockDim.x + (threadIdx.x & ~31); i0 < n; i0 += stride) {
    const int64_t i = i0 + (threadIdx.x & 31);
    const int32_t c = i < n ? lab[i] : -1;
    const unsigned m = __match_any_sync(0xffffffffu, c);
    if (c >= 0 && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(&hs[c], __popc(m));
  }
  __syncthreads();
  for (int c = threadIdx.x; c < nl; c += blockDim.x)
    if (hs[c]) atomicAdd(&size[c], hs[c]);
}

int32_t level_set_final(Handle& h, Level& L, const int32_t* d_labels, const uint2* ca_last, int64_t n_last) {
  cudaStream_t s = h.stream;
  L.sweeps_done = 1;
  if (L.n == 0) return LOUVAIN_OK;
  k_set_C<<<grid_for(L.n, 256), 256, 0, s>>>(d_labels, L.n, L.ca, L.size, L.C);
  LV_LAUNCHED();
  k_copy_a<<<grid_for(n_last, 256), 256, 0, s>>>(ca_last, n_last, L.ca);
  LV_LAUNCHED();
  const int smem = (int)(4 * n_last);
  LV_CUDA(cudaFuncSetAttribute(k_size_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  k_size_hist<<<148, 1024, smem, s>>>(d_labels, L.n, (int)n_last, L.size);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t level_get_labels(Handle& h, Level& L, int32_t* d_out) {
  if (L.n == 0) return LOUVAIN_OK;
  k_get_C<<<grid_for(L.n, 256), 256, 0, h.stream>>>(L.ca, L.n, d_out);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t level_get_a(Handle& h, Level& L, uint32_t* d_out) {
  if (L.n == 0) return LOUVAIN_OK;
  k_get_a<<<grid_for(L.n, 256), 256, 0, h.stream>>>(L.ca, L.n, d_out);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

// Hub plan (vertices of sub-class kSubHub with more than kPartMaxP partitions, of any bucket): work items
// in hub order -- inserts (kHubChunkEdges edges each), scans (kHubScanSlots
// slots each), final -- and a ring of table slots reused hub after hub.
static int32_t build_hub_plan(Handle& h, Level& L) {
  cudaStream_t s = h.stream;
  HubPlan& P = L.hub;
  std::vector<int32_t> hv;
  std::vector<int64_t> hdeg, rb, hsoff;
  std::vector<int32_t> hbucket;
  for (int b = 1; b <= 7; ++b) {
    if (b <= 6 && L.bins_bounds_pending[b - 1] <= kSmallMaxDeg) continue;  // register-kernel bucket: no hubs
    const int c = kSubPerBucket * b + kSubPart;  // partitioned sub-classes (P > part_maxp() only)
    const int64_t off = L.class_off[c], cnt = L.class_off[kSubPerBucket * (b + 1)] - off;
    if (cnt <= 0) continue;
    std::vector<int32_t> v(cnt);
    std::vector<int64_t> d(2 * cnt);
    int64_t* dd = nullptr;
    LV_TRY(dalloc(&dd, 2 * cnt, s));
    k_hub_degrees<<<grid_for(cnt, 256), 256, 0, s>>>(L.bin_vertices + off, cnt, L.rowptr, dd);
    LV_LAUNCHED();
    std::vector<int64_t> so(cnt);
    LV_CUDA(cudaMemcpyAsync(v.data(), L.bin_vertices + off, 4 * cnt, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaMemcpyAsync(d.data(), dd, 16 * cnt, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaMemcpyAsync(so.data(), L.soff + off, 8 * cnt, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    dfree(dd, s);
    for (int64_t i = 0; i < cnt; ++i) {
      if ((d[i] + kPartLabels - 1) / kPartLabels <= part_maxp()) continue;  // label-partitioned path
      hsoff.push_back(so[i]);
      hv.push_back(v[i]);
      hdeg.push_back(d[i]);
      rb.push_back(d[cnt + i]);
      hbucket.push_back(b);
    }
  }
  P.nh = (int64_t)hv.size();
  std::fill(P.bucket_wave, P.bucket_wave + 9, 0);
  if (P.nh == 0) return LOUVAIN_OK;
  std::vector<HubInfo> info(P.nh);
  std::vector<HubItem> ins, scans;
  std::vector<int64_t> ins_off, scan_off, wave_hub;
  auto cap_of = [](int64_t d) { return ((2 * d + 3) / 4) * 4; };  // load <= 1/2, whole 4-slot buckets
  int64_t seg = kHubWaveSlots;
  for (int64_t i = 0; i < P.nh; ++i) seg = std::max(seg, cap_of(hdeg[i]));
  int64_t acc = 0;
  for (int64_t i = 0; i < P.nh; ++i) {
    const int64_t cap = cap_of(hdeg[i]);
    if (wave_hub.empty() || acc + cap > seg || hbucket[i] != hbucket[i - 1]) {  // a wave never spans buckets
      for (int b = (i == 0) ? 1 : hbucket[i - 1] + 1; b <= hbucket[i]; ++b) P.bucket_wave[b - 1] = (int64_t)wave_hub.size();
      wave_hub.push_back(i);
      ins_off.push_back((int64_t)ins.size());
      scan_off.push_back((int64_t)scans.size());
      acc = 0;
    }
    HubInfo& hi = info[i];
    hi.v = hv[i];
    hi.cap = cap;
    hi.off = acc;
    hi.sbase = hsoff[i] - rb[i];
    acc += cap;
    for (int64_t e = 0; e < hdeg[i]; e += kHubChunkEdges)
      ins.push_back(HubItem{(int32_t)i, 0, rb[i] + e, rb[i] + std::min(hdeg[i], e + kHubChunkEdges)});
    hi.scan_first = (int64_t)scans.size();
    hi.nscan = 0;
    for (int64_t t = 0; t < cap; t += kHubScanSlots) {
      scans.push_back(HubItem{(int32_t)i, 0, t, std::min(cap, t + kHubScanSlots)});
      hi.nscan++;
    }
  }
  P.nwaves = (int64_t)wave_hub.size();
  for (int b = hbucket[P.nh - 1] + 1; b <= 8; ++b) P.bucket_wave[b - 1] = P.nwaves;
  wave_hub.push_back(P.nh);
  ins_off.push_back((int64_t)ins.size());
  scan_off.push_back((int64_t)scans.size());
  P.seg = seg;
  P.nins = (int64_t)ins.size();
  P.nscan = (int64_t)scans.size();
  LV_TRY(dalloc(&P.ins, ins.size(), s));
  LV_TRY(dalloc(&P.scans, scans.size(), s));
  LV_TRY(dalloc(&P.ins_off, ins_off.size(), s));
  LV_TRY(dalloc(&P.scan_off, scan_off.size(), s));
  LV_TRY(dalloc(&P.wave_hub, wave_hub.size(), s));
  LV_TRY(dalloc(&P.info, info.size(), s));
  // one allocation: {label|e} slots then a_c words
  LV_TRY(dmalloc(reinterpret_cast<void**>(&P.ring), 12 * (size_t)(2 * seg), s));
  P.ring_a = reinterpret_cast<uint32_t*>(P.ring + 2 * seg);
  LV_TRY(dmalloc(&P.partial, hub_partial_bytes() * (size_t)P.nscan, s));
  LV_CUDA(cudaMemcpyAsync(P.ins, ins.data(), sizeof(HubItem) * ins.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(P.scans, scans.data(), sizeof(HubItem) * scans.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(P.ins_off, ins_off.data(), 8 * ins_off.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(P.scan_off, scan_off.data(), 8 * scan_off.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(P.wave_hub, wave_hub.data(), 8 * wave_hub.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(P.info, info.data(), sizeof(HubInfo) * info.size(), cudaMemcpyHostToDevice, s));
  k_fill_u64<<<grid_for(2 * seg, 256), 256, 0, s>>>(P.ring, 2 * seg, kEmpty);
  LV_LAUNCHED();
  k_fill_u32v<<<grid_for(2 * seg, 256), 256, 0, s>>>(P.ring_a, 2 * seg, 0xFFFFFFFFu);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  LV_CUDA(cudaStreamSynchronize(s));  // host vectors die here
  return LOUVAIN_OK;
}

static void part_free(PartPlan& Q, cudaStream_t s) {
  dfree(Q.task_vpos, s); dfree(Q.task_p, s); dfree(Q.vert_pos, s); dfree(Q.vert_P, s); dfree(Q.vert_first, s);
  dfree(Q.vert_pbase, s); dfree(Q.done, s); dfree(Q.partial, s); dfree(Q.poff, s); dfree(Q.pcur, s);
  dfree(Q.chunks, s);
  Q = PartPlan();
}

// Partition plan for every vertex of sub-classes kSubPart.. (deg >= kSub5Min) with
// P <= kPartMaxP, any bucket.
int32_t build_part_plan(Handle& h, Level& L) {
  cudaStream_t s = h.stream;
  PartPlan& Q = L.part;
  part_free(Q, s);
  std::vector<int32_t> vpos, vP, vfirst, tv, tp;
  std::vector<int64_t> vpb;
  std::vector<PartChunk> ch;
  int64_t pb = 0;
  for (int b = 1; b <= 7; ++b) {
    Q.bucket_task[b - 1] = (int64_t)tv.size();
    Q.bucket_vert[b - 1] = (int64_t)vpos.size();
    Q.bucket_chunk[b - 1] = (int64_t)ch.size();
    Q.bucket_vsplit[b - 1] = (int64_t)vpos.size();
    Q.bucket_tsplit[b - 1] = (int64_t)tv.size();
    if (b <= 6 && L.bins_bounds_pending[b - 1] <= kSmallMaxDeg) continue;  // register-kernel bucket: no hubs
    const int c0 = kSubPerBucket * b + kSubPart, c1 = kSubPerBucket * (b + 1);
    const int64_t off = L.class_off[c0], cnt = L.class_off[c1] - off;
    if (cnt <= 0) continue;
    std::vector<int64_t> so(cnt + 1);
    LV_CUDA(cudaMemcpyAsync(so.data(), L.soff + off, 8 * (cnt + 1), cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    // longest first: a CTA walks all partitions of one vertex (sweep_part)
    std::vector<int64_t> ord(cnt);
    for (int64_t i = 0; i < cnt; ++i) ord[i] = i;
    std::stable_sort(ord.begin(), ord.end(),
                     [&](int64_t a, int64_t b) { return so[a + 1] - so[a] > so[b + 1] - so[b]; });
    for (int64_t i : ord) {
      const int64_t deg = so[i + 1] - so[i];
      const int64_t P = (deg + kPartLabels - 1) / kPartLabels;
      if (P > part_maxp()) continue;  // giant: cooperative hub kernel
      const int32_t vi = (int32_t)vpos.size();
      vpos.push_back((int32_t)(off + i));
      vP.push_back((int32_t)P);
      vfirst.push_back((int32_t)tv.size());
      vpb.push_back(pb);
      pb += P + 1;
      for (int32_t q = 0; q < (int32_t)P; ++q) {
        tv.push_back(vi);
        tp.push_back(q);
      }
      if (P > kStreamMaxP) {  // pre-partitioned (a prefix: degrees descending)
        for (int64_t e = 0; e < deg; e += kPartChunk) ch.push_back(PartChunk{vi, 0, e, std::min(deg, e + kPartChunk)});
        Q.bucket_vsplit[b - 1] = (int64_t)vpos.size();
        Q.bucket_tsplit[b - 1] = (int64_t)tv.size();
      }
    }
  }
  Q.nverts = (int64_t)vpos.size();
  Q.ntasks = (int64_t)tv.size();
  Q.nchunks = (int64_t)ch.size();
  Q.npoff = pb;
  Q.bucket_task[7] = Q.ntasks;
  Q.bucket_vert[7] = Q.nverts;
  Q.bucket_chunk[7] = Q.nchunks;
  if (Q.nverts == 0) return LOUVAIN_OK;
  LV_TRY(dalloc(&Q.task_vpos, Q.ntasks, s));
  LV_TRY(dalloc(&Q.task_p, Q.ntasks, s));
  LV_TRY(dalloc(&Q.vert_pos, Q.nverts, s));
  LV_TRY(dalloc(&Q.vert_P, Q.nverts, s));
  LV_TRY(dalloc(&Q.vert_first, Q.nverts, s));
  LV_TRY(dalloc(&Q.vert_pbase, Q.nverts, s));
  LV_TRY(dalloc(&Q.done, Q.nverts, s));
  LV_TRY(dmalloc(&Q.partial, hub_partial_bytes() * (size_t)Q.ntasks, s));
  LV_TRY(dalloc(&Q.poff, Q.npoff, s));
  LV_TRY(dalloc(&Q.pcur, Q.ntasks, s));
  LV_TRY(dalloc(&Q.chunks, Q.nchunks, s));
  LV_CUDA(cudaMemcpyAsync(Q.task_vpos, tv.data(), 4 * tv.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(Q.task_p, tp.data(), 4 * tp.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(Q.vert_pos, vpos.data(), 4 * vpos.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(Q.vert_P, vP.data(), 4 * vP.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(Q.vert_first, vfirst.data(), 4 * vfirst.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(Q.vert_pbase, vpb.data(), 8 * vpb.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaMemcpyAsync(Q.chunks, ch.data(), sizeof(PartChunk) * ch.size(), cudaMemcpyHostToDevice, s));
  LV_CUDA(cudaStreamSynchronize(s));  // host vectors die here
  return LOUVAIN_OK;
}

int32_t level_binning(Handle& h, Level& L, const louvain_params_t& p) {
  bool same = L.bins_valid;
  for (int t = 0; t < 6 && same; ++t) same = (L.bins_bounds[t] == p.deg_bounds[t]);
  if (same) return LOUVAIN_OK;
  cudaStream_t s = h.stream;
  const int64_t n = L.n;
  std::memcpy(L.bins_bounds_pending, p.deg_bounds, sizeof L.bins_bounds_pending);
  hub_free(L.hub, s);
  std::fill(L.class_off, L.class_off + kNumClasses + 1, 0);
  if (n > 0) {
    uint8_t *cls = nullptr, *cls2 = nullptr;
    int32_t* iota = nullptr;
    unsigned long long* hist = nullptr;
    LV_TRY(dalloc(&cls, n, s));
    LV_TRY(dalloc(&cls2, n, s));
    LV_TRY(dalloc(&iota, n, s));
    LV_TRY(dalloc(&hist, kNumClasses, s));
    LV_CUDA(cudaMemsetAsync(hist, 0, 8 * kNumClasses, s));
    const int64_t lo = L.own_hi < 0 ? 0 : L.own_lo, hi = L.own_hi < 0 ? n : L.own_hi;
    k_classify<<<grid_for(n, 256), 256, 0, s>>>(L.rowptr, n, p.deg_bounds[0], p.deg_bounds[1], p.deg_bounds[2],
                                                p.deg_bounds[3], p.deg_bounds[4], p.deg_bounds[5], lo, hi, cls,
                                                iota, hist);
    LV_LAUNCHED();
    LV_CUDA(cudaGetLastError());
    // stable sort by class (6 bits): vertices of a class stay in ascending id order
    size_t tb = 0;
    LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, cls, cls2, iota, L.bin_vertices, n, 0, 6, s));
    void* tmp = nullptr;
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, cls, cls2, iota, L.bin_vertices, n, 0, 6, s)); LV_CUB();
    dfree(tmp, s);
    unsigned long long hh[kNumClasses];
    LV_CUDA(cudaMemcpyAsync(hh, hist, sizeof hh, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    dfree(cls, s); dfree(cls2, s); dfree(iota, s); dfree(hist, s);
    for (int c = 0; c < kNumClasses; ++c) L.class_off[c + 1] = L.class_off[c] + (int64_t)hh[c];
    // staging offsets: exclusive scan of the degrees in bin order
    if (!L.soff) LV_TRY(dalloc(&L.soff, n + 1, s));  // scratch-backed levels have them already
    if (!L.bin_rb) LV_TRY(dalloc(&L.bin_rb, n, s));
    {
      void* st = nullptr;
      LV_TRY(scratch_get(h, SC_STAGE, sizeof(uint2) * (size_t)std::max<int64_t>(L.nnz, 1), &st));
      L.stage = static_cast<uint2*>(st);
    }
    int64_t* dg = nullptr;
    LV_TRY(dalloc(&dg, n + 1, s));
    k_bin_degrees<<<grid_for(n, 256), 256, 0, s>>>(L.bin_vertices, n, L.rowptr, dg, L.bin_rb);
    LV_LAUNCHED();
    size_t tb2 = 0;
    LV_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb2, dg, L.soff, n + 1, s));
    void* tmp2 = nullptr;
    LV_TRY(dmalloc(&tmp2, tb2, s));
    LV_CUDA(cub::DeviceScan::ExclusiveSum(tmp2, tb2, dg, L.soff, n + 1, s)); LV_CUB();
    dfree(tmp2, s);
    dfree(dg, s);
    // staged-entry offsets of every class boundary, for host-side tile plans
    for (int c = 0; c <= kNumClasses; ++c)
      LV_CUDA(cudaMemcpyAsync(&L.class_soff[c], L.soff + L.class_off[c], 8, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
  } else {
    std::fill(L.class_soff, L.class_soff + kNumClasses + 1, 0);
  }
  LV_TRY(build_hub_plan(h, L));
  LV_TRY(build_part_plan(h, L));
  std::memcpy(L.bins_bounds, p.deg_bounds, sizeof L.bins_bounds);
  L.bins_valid = true;
  return LOUVAIN_OK;
}

// Eq. (1) parts into ctl->L / ctl->S (stream-ordered, no sync).  d_C == nullptr:
// the level's own partition with its maintained a_c; else an external labelling.
int32_t launch_modularity(Handle& h, Level& L, const int32_t* d_C, bool singletons) {
  cudaStream_t s = h.stream;
  LV_CUDA(cudaMemsetAsync(&h.ctl->L, 0, 16, s));
  if (L.n == 0) return LOUVAIN_OK;
  const int64_t e0 = (d_C || L.own_hi < 0) ? 0 : L.own_e0, e1 = (d_C || L.own_hi < 0) ? L.nnz : L.own_e1;
  const int64_t ntiles = (e1 - e0 + kTileEdges - 1) / kTileEdges;
  const unsigned grid = grid_for(std::max<int64_t>(ntiles, (L.n + 255) / 256), 1, 148 * 8);
  const int64_t* tr = nullptr;
  if (e1 > e0) {
    LV_TRY(tile_starts(h, L.rowptr, 0, L.n, e0, e1, kTileEdges, &tr));
  } else {
    LV_TRY(tile_starts(h, L.rowptr, 0, L.n, 0, 1, kTileEdges, &tr));  // unused (no tiles)
  }
  if (!d_C && singletons) {
    k_modularity<true, true><<<grid, 256, 0, s>>>(L.rowptr, L.n, L.col, L.w, L.ca, L.C, nullptr, e0, e1, tr,
                                                  &h.ctl->L, &h.ctl->S);
    LV_LAUNCHED();
  } else if (!d_C) {
    k_modularity<true><<<grid, 256, 0, s>>>(L.rowptr, L.n, L.col, L.w, L.ca, L.C, nullptr, e0, e1, tr, &h.ctl->L,
                                            &h.ctl->S);
    LV_LAUNCHED();
  } else {
    uint32_t* a_tmp = nullptr;
    LV_TRY(dalloc(&a_tmp, L.n, s));
    LV_CUDA(cudaMemsetAsync(a_tmp, 0, 4 * L.n, s));
    k_ext_totals<<<grid_for(L.n, 256), 256, 0, s>>>(d_C, L.k, L.n, a_tmp, &h.ctl->bad);
    LV_LAUNCHED();
    k_modularity<false><<<grid, 256, 0, s>>>(L.rowptr, L.n, L.col, L.w, nullptr, d_C, a_tmp, 0, L.nnz, tr,
                                             &h.ctl->L, &h.ctl->S);
    LV_LAUNCHED();
    dfree(a_tmp, s);
  }
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

// Delta pass iff moved entries <= nnz / LV_DELTA_DIV.  Default 1 (always; the
// commit then skips the moved-degree sum): measured faster than the full pass on
// every config even at 84% moved entries (DESIGN 13); LV_DELTA_DIV=1000000 forces
// the full pass.
unsigned long long delta_div() {
  static const unsigned long long d = getenv("LV_DELTA_DIV") ? strtoull(getenv("LV_DELTA_DIV"), nullptr, 10) : 1ull;
  return d;
}

int32_t launch_snapshot(Handle& h, Level& L) {
  if (L.n == 0) return LOUVAIN_OK;
  k_snapshot<<<grid_for(L.n, 256), 256, 0, h.stream>>>(L.C, L.n, h.pcn);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t launch_modularity_delta(Handle& h, Level& L) {
  const uint2* P = h.pcn;
  cudaStream_t s = h.stream;
  LV_CUDA(cudaMemsetAsync(&h.ctl->L, 0, 16, s));
  LV_CUDA(cudaMemsetAsync(&h.ctl->dL, 0, 24, s));
  LV_TRY(set_ctl_u64(h, &h.ctl->ddiv, delta_div()));
  if (L.n == 0) return LOUVAIN_OK;
  const size_t nbig = (size_t)(L.nnz / kDeltaBigDeg + 1), nmid = (size_t)(L.nnz / kDeltaThrDeg + 1);
  if (h.dl_big_n < nbig) {
    dfree(h.dl_big, s);
    h.dl_big = nullptr;
    h.dl_big_n = 0;
    LV_TRY(dalloc(&h.dl_big, nbig, s));
    h.dl_big_n = nbig;
  }
  if (h.dl_mid_n < nmid) {
    dfree(h.dl_mid, s);
    h.dl_mid = nullptr;
    h.dl_mid_n = 0;
    LV_TRY(dalloc(&h.dl_mid, nmid, s));
    h.dl_mid_n = nmid;
  }
  int32_t *big = h.dl_big, *mid = h.dl_mid;
  // a distributed handle sums the moved rows it owns (the ranks' parts are all-reduced)
  const int64_t own_lo = (h.dist && L.own_hi >= 0) ? L.own_lo : 0;
  const int64_t own_hi = (h.dist && L.own_hi >= 0) ? L.own_hi : L.n;
  k_mod_delta_thr<<<148 * 8, 256, 0, s>>>(h.ctl, L.mv_v, L.mv_new, L.mv_old, L.rowptr, L.col, L.w, P,
                                          L.nnz, mid, big, own_lo, own_hi);
  LV_LAUNCHED();
  k_mod_delta_warp<<<148 * 8, 256, 0, s>>>(h.ctl, mid, L.mv_v, L.mv_new, L.mv_old, L.rowptr, L.col, L.w, P,
                                           L.nnz);
  LV_LAUNCHED();
  k_mod_delta_cta<<<148 * 4, 512, 0, s>>>(h.ctl, big, L.mv_v, L.mv_new, L.mv_old, L.rowptr, L.col, L.w, P,
                                          L.nnz, L.ca, L.n);
  LV_LAUNCHED();
  // full pass, skipped on the device when the delta pass was chosen
  const int64_t ntiles = (L.nnz + kTileEdges - 1) / kTileEdges;
  const unsigned grid = grid_for(std::max<int64_t>(ntiles, (L.n + 255) / 256), 1, 148 * 8);
  const int64_t* tr = nullptr;
  LV_TRY(tile_starts(h, L.rowptr, 0, L.n, 0, std::max<int64_t>(L.nnz, 1), kTileEdges, &tr));
  k_modularity<true><<<grid, 256, 0, s>>>(L.rowptr, L.n, L.col, L.w, L.ca, L.C, nullptr, 0, L.nnz, tr, &h.ctl->L,
                                          &h.ctl->S, h.ctl);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t level_modularity(Handle& h, Level& L, const int32_t* d_C, uint64_t* Lout, uint64_t* Sout, bool singletons) {
  LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, h.stream));
  LV_TRY(launch_modularity(h, L, d_C, singletons));
  LV_CUDA(cudaMemcpyAsync(h.h_ctl, h.ctl, sizeof(DevCtl), cudaMemcpyDeviceToHost, h.stream));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  if (h.h_ctl->bad) {
    set_error("labels out of range [0, n)");
    return LOUVAIN_E_INVALID_ARG;
  }
  *Lout = h.h_ctl->L;
  *Sout = h.h_ctl->S;
  return LOUVAIN_OK;
}

int32_t launch_commit(Handle& h, Level& L, int bucket) {
  if (dist_p2p(h)) return dist_commit_p2p(h, L, bucket);
  k_commit<<<148 * 4, 256, 0, h.stream>>>(h.ctl, bucket, L.mv_v, L.mv_new, L.mv_old, L.ca, L.size, L.k, L.C,
                                         (h.pcn && delta_div() > 1) ? L.rowptr : nullptr, h.pcn);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

namespace {
__global__ void k_set_u64(unsigned long long* p, unsigned long long v) { *p = v; }
__global__ void k_pack_moves(const int32_t* mv_v, const int32_t* mv_new, int64_t c0, int64_t cnt, int32_t* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x) {
    out[2 * i] = mv_v[c0 + i];
    out[2 * i + 1] = mv_new[c0 + i];
  }
}
// (v, new) pairs -> move log.  Caller-supplied ids are validated before any
// commit: v and new in [0, n), and no vertex twice in one sweep (stamp[v] holds
// the id of the last sweep that moved v); a violation sets ctl->bad.
__global__ void k_unpack_moves(const int32_t* in, int64_t c0, int64_t cnt, int64_t n, int32_t* mv_v, int32_t* mv_new,
                               int32_t* stamp, int32_t sweep_id, DevCtl* ctl) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = in[2 * i], t = in[2 * i + 1];
    if (v < 0 || v >= n || t < 0 || t >= n || atomicExch(&stamp[v], sweep_id) == sweep_id) {
      atomicOr(&ctl->bad, 1ull);
      mv_v[c0 + i] = 0;  // never committed: the host refuses the call
      mv_new[c0 + i] = 0;
      continue;
    }
    mv_v[c0 + i] = v;
    mv_new[c0 + i] = t;
  }
}
}  // namespace

int32_t set_ctl_u64(Handle& h, unsigned long long* dst, unsigned long long v) {
  k_set_u64<<<1, 1, 0, h.stream>>>(dst, v);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t pack_moves(Handle& h, Level& L, int64_t c0, int64_t cnt, int32_t* out) {
  if (cnt <= 0) return LOUVAIN_OK;
  k_pack_moves<<<grid_for(cnt, 256), 256, 0, h.stream>>>(L.mv_v, L.mv_new, c0, cnt, out);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t unpack_moves(Handle& h, Level& L, int64_t c0, int64_t cnt, const int32_t* in) {
  if (cnt <= 0) return LOUVAIN_OK;
  if (!L.mv_stamp) {
    LV_TRY(dalloc(&L.mv_stamp, L.n, h.stream));
    LV_CUDA(cudaMemsetAsync(L.mv_stamp, 0xFF, 4 * (size_t)std::max<int64_t>(L.n, 1), h.stream));  // -1: never
  }
  LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, h.stream));
  k_unpack_moves<<<grid_for(cnt, 256), 256, 0, h.stream>>>(in, c0, cnt, L.n, L.mv_v, L.mv_new, L.mv_stamp,
                                                          L.stamp_id, h.ctl);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  unsigned long long bad = 0;
  LV_CUDA(cudaMemcpyAsync(&bad, &h.ctl->bad, 8, cudaMemcpyDeviceToHost, h.stream));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  if (bad) {
    // undo the stamps of this call's valid entries is not needed: the handle's
    // sweep is refused as a whole (the caller must revert or restart the sweep)
    LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, h.stream));
    set_error("louvain_commit_moves: vertex or label out of [0, n), or a vertex moved twice in one sweep");
    return LOUVAIN_E_INVALID_ARG;
  }
  return LOUVAIN_OK;
}

int32_t launch_revert(Handle& h, Level& L) {
  if (dist_p2p(h)) return dist_revert_p2p(h, L);
  k_revert<<<148 * 4, 256, 0, h.stream>>>(h.ctl, L.mv_v, L.mv_new, L.mv_old, L.ca, L.size, L.k, L.C);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t compose_labels(Handle& h, int32_t* lab, int64_t n0, const int32_t* map) {
  if (n0 == 0) return LOUVAIN_OK;
  k_compose<<<grid_for(n0, 256), 256, 0, h.stream>>>(lab, n0, map);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

int32_t compose_labels_ca(Handle& h, int32_t* lab, int64_t n0, const uint2* ca) {
  if (n0 == 0) return LOUVAIN_OK;
  k_compose_ca<<<grid_for(n0, 256), 256, 0, h.stream>>>(lab, n0, ca);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

// Alg. 3 as renumber-by-scan + sort-by-key + segmented reduce:
//  newID = exclusive scan of [size_c > 0] (Alg. 3 l.7-12, R17);
//  every entry (u,v,w) emits key (newID[C[u]], newID[C[v]]) (R18: mergeCommunity
//  hashes all neighbours of all members); radix sort; equal keys summed
//  (run-length counts at unit weight); CSR' rows sorted by column.
int32_t level_contract(Handle& h, Level& L, Level& out, int32_t* d_map, int parity) {
  cudaStream_t s = h.stream;
  const int64_t n = L.n, nnz = L.nnz;
  out = Level();
  out.W = L.W;
  const bool scr = parity >= 0;  // inside louvain_run: every big array from the handle's scratch
  auto lvl = [&](int a, size_t bytes, void** o) { return scratch_get(h, SC_LVL0 + 2 * a + parity, bytes, o); };
  if (n == 0) {
    LV_TRY(dalloc(&out.rowptr, 1, s));
    LV_CUDA(cudaMemsetAsync(out.rowptr, 0, 8, s));
    return level_alloc_state(out, s);
  }
  int32_t *flag = nullptr, *newID = nullptr;
  LV_TRY(dalloc(&flag, n, s));
  LV_TRY(dalloc(&newID, n, s));
  k_flags_nonempty<<<grid_for(n, 256), 256, 0, s>>>(L.size, n, flag);
  LV_LAUNCHED();
  size_t tb = 0;
  LV_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, flag, newID, n, s));
  void* tmp = nullptr;
  LV_TRY(dmalloc(&tmp, tb, s));
  LV_CUDA(cub::DeviceScan::ExclusiveSum(tmp, tb, flag, newID, n, s)); LV_CUB();
  dfree(tmp, s);
  int32_t last[2];
  LV_CUDA(cudaMemcpyAsync(&last[0], newID + n - 1, 4, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaMemcpyAsync(&last[1], flag + n - 1, 4, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaStreamSynchronize(s));
  const int64_t np = (int64_t)last[0] + last[1];
  k_map<<<grid_for(n, 256), 256, 0, s>>>(L.ca, newID, n, d_map);
  LV_LAUNCHED();
  dfree(flag, s);
  out.n = np;
  if (scr) LV_TRY(lvl(LA_ROWPTR, 8 * (size_t)(np + 1), (void**)&out.rowptr));
  else LV_TRY(dalloc(&out.rowptr, np + 1, s));
  LV_CUDA(cudaMemsetAsync(out.rowptr, 0, 8 * (np + 1), s));
  if (nnz == 0) {
    out.nnz = 0;
    if (scr) {
      LV_TRY(lvl(LA_COL, 4, (void**)&out.col));
      LV_TRY(lvl(LA_W, 4, (void**)&out.w));
      LV_TRY(level_alloc_scratch(h, out, parity));
    } else {
      LV_TRY(dalloc(&out.col, 1, s));
      LV_TRY(dalloc(&out.w, 1, s));
      LV_TRY(level_alloc_state(out, s));
    }
    k_next_degrees<<<grid_for(n, 256), 256, 0, s>>>(L.ca, L.size, newID, n, out.k);
    LV_LAUNCHED();
    dfree(newID, s);
    out.k_ready = true;
    return LOUVAIN_OK;
  }
  const bool weighted = L.w != nullptr;
  unsigned long long *k0 = nullptr, *k1 = nullptr;
  uint32_t *v0 = nullptr, *v1 = nullptr;
  if (scr) {
    LV_TRY(scratch_get(h, SC_STAGE, 8 * (size_t)nnz, (void**)&k0));  // the level's stage is dead now
    LV_TRY(scratch_get(h, SC_K1, 8 * (size_t)nnz, (void**)&k1));
    LV_TRY(scratch_get(h, SC_V0, 4 * (size_t)nnz, (void**)&v0));
    if (weighted) LV_TRY(scratch_get(h, SC_V1, 4 * (size_t)nnz, (void**)&v1));
  } else {
    LV_TRY(dalloc(&k0, nnz, s));
    LV_TRY(dalloc(&k1, nnz, s));
    LV_TRY(dalloc(&v0, nnz, s));
    if (weighted) LV_TRY(dalloc(&v1, nnz, s));
  }
  {
    const int64_t ntiles = (nnz + kTileEdges - 1) / kTileEdges;
    const int64_t* tr = nullptr;
    LV_TRY(tile_starts(h, L.rowptr, 0, n, 0, nnz, kTileEdges, &tr));
    k_emit_keys<<<grid_for(ntiles, 1, 148 * 8), 256, 0, s>>>(L.rowptr, n, L.col, L.w, d_map, nnz, (uint64_t)np, tr,
                                                             k0, weighted ? v0 : nullptr);
    LV_LAUNCHED();
    LV_CUDA(cudaGetLastError());
  }
  int bits = 1;
  while (bits < 64 && ((unsigned long long)1 << bits) < (unsigned long long)np * (unsigned long long)np) ++bits;
  cub::DoubleBuffer<unsigned long long> kb(k0, k1);
  cub::DoubleBuffer<uint32_t> vb(v0, v1);
  tb = 0;
  if (weighted) LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, kb, vb, nnz, 0, bits, s));
  else LV_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tb, kb, nnz, 0, bits, s));
  LV_TRY(dmalloc(&tmp, tb, s));
  if (weighted) LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, kb, vb, nnz, 0, bits, s));
  else LV_CUDA(cub::DeviceRadixSort::SortKeys(tmp, tb, kb, nnz, 0, bits, s));
  LV_CUB();
  dfree(tmp, s);
  unsigned long long* sorted = kb.Current();
  unsigned long long* uniq = kb.Alternate();
  uint32_t* sums = weighted ? vb.Alternate() : v0;
  int64_t* d_num = reinterpret_cast<int64_t*>(&h.ctl->bad);
  tb = 0;
  if (weighted) {
    LV_CUDA(cub::DeviceReduce::ReduceByKey(nullptr, tb, sorted, uniq, vb.Current(), sums, d_num, cub::Sum(), nnz, s));
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceReduce::ReduceByKey(tmp, tb, sorted, uniq, vb.Current(), sums, d_num, cub::Sum(), nnz, s)); LV_CUB();
  } else {
    LV_CUDA(cub::DeviceRunLengthEncode::Encode(nullptr, tb, sorted, uniq, sums, d_num, nnz, s));
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceRunLengthEncode::Encode(tmp, tb, sorted, uniq, sums, d_num, nnz, s)); LV_CUB();
  }
  dfree(tmp, s);
  int64_t m = 0;
  LV_CUDA(cudaMemcpyAsync(&m, d_num, 8, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaStreamSynchronize(s));
  if (!scr) dfree(sorted, s);
  out.nnz = m;
  if (scr) {
    LV_TRY(lvl(LA_COL, 4 * (size_t)std::max<int64_t>(m, 1), (void**)&out.col));
    LV_TRY(lvl(LA_W, 4 * (size_t)std::max<int64_t>(m, 1), (void**)&out.w));
  } else {
    LV_TRY(dalloc(&out.col, m, s));
    LV_TRY(dalloc(&out.w, m, s));
  }
  int64_t* cnt = nullptr;
  LV_TRY(dalloc(&cnt, np + 1, s));
  LV_CUDA(cudaMemsetAsync(cnt, 0, 8 * (np + 1), s));
  k_row_counts<<<grid_for(m, 256), 256, 0, s>>>(uniq, m, (uint64_t)np, cnt);
  LV_LAUNCHED();
  tb = 0;
  LV_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, cnt, out.rowptr, np + 1, s));
  LV_TRY(dmalloc(&tmp, tb, s));
  LV_CUDA(cub::DeviceScan::InclusiveSum(tmp, tb, cnt, out.rowptr, np + 1, s)); LV_CUB();
  dfree(tmp, s);
  dfree(cnt, s);
  k_split_keys<<<grid_for(m, 256), 256, 0, s>>>(uniq, m, (uint64_t)np, out.col);
  LV_LAUNCHED();
  LV_CUDA(cudaMemcpyAsync(out.w, sums, 4 * m, cudaMemcpyDeviceToDevice, s));
  LV_CUDA(cudaGetLastError());
  if (!scr) {
    dfree(uniq, s);
    dfree(v0, s);
    if (v1) dfree(v1, s);
  }
  if (scr) LV_TRY(level_alloc_scratch(h, out, parity));
  else LV_TRY(level_alloc_state(out, s));
  k_next_degrees<<<grid_for(n, 256), 256, 0, s>>>(L.ca, L.size, newID, n, out.k);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  dfree(newID, s);
  out.k_ready = true;
  return LOUVAIN_OK;
}

// Host-side CSR validation (LOUVAIN_VALIDATE): rowptr monotone with rowptr[0]=0
// and rowptr[n]=nnz, 0 <= col < n, w > 0, W guard, and symmetry (the multiset
// of (u,v,w) equals that of (v,u,w); R1).
int32_t validate_csr_host(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                          bool full, uint64_t* Wout) {
  if (rowptr[0] != 0 || rowptr[n] != nnz) {
    set_error("rowptr[0] must be 0 and rowptr[n] must equal nnz");
    return LOUVAIN_E_INVALID_GRAPH;
  }
  if (!full) return LOUVAIN_OK;
  uint64_t W = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (rowptr[i + 1] < rowptr[i]) { set_error("rowptr not monotone"); return LOUVAIN_E_INVALID_GRAPH; }
    for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
      if (col[e] < 0 || col[e] >= n) { set_error("col out of range"); return LOUVAIN_E_INVALID_GRAPH; }
      uint32_t we = w ? w[e] : 1u;
      if (we == 0) { set_error("zero weight"); return LOUVAIN_E_INVALID_GRAPH; }
      W += we;
    }
  }
  if (W > kWGuard) { set_error("W = 2m exceeds 3,037,000,499"); return LOUVAIN_E_OVERFLOW; }
  struct T { int32_t u, v; uint32_t w; };
  std::vector<T> f, b;
  f.reserve(nnz);
  b.reserve(nnz);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
      uint32_t we = w ? w[e] : 1u;
      f.push_back(T{(int32_t)i, col[e], we});
      b.push_back(T{col[e], (int32_t)i, we});
    }
  auto lt = [](const T& x, const T& y) {
    if (x.u != y.u) return x.u < y.u;
    if (x.v != y.v) return x.v < y.v;
    return x.w < y.w;
  };
  std::sort(f.begin(), f.end(), lt);
  std::sort(b.begin(), b.end(), lt);
  for (size_t t = 0; t < f.size(); ++t)
    if (f[t].u != b[t].u || f[t].v != b[t].v || f[t].w != b[t].w) {
      set_error("graph is not symmetric (each non-loop edge must be stored in both directions)");
      return LOUVAIN_E_INVALID_GRAPH;
    }
  if (Wout) *Wout = W;
  return LOUVAIN_OK;
}

}  // namespace lv
