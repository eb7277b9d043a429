// lv_contract.cu -- the aggregation phase used inside louvain_run (Alg. 3,
// PAPER.md P:238-294) without a global sort of all entries.
//
//   1. newID = exclusive scan of [size_c > 0] (Alg. 3 l.7-12, R17); map[v] = newID[C[v]];
//      degree of new vertex = a_c (the merged row sums all member rows, R18).
//   2. Members grouped by new vertex (radix sort of n keys; Alg. 3 l.15-19's com[]),
//      member degrees prefix-summed (Alg. 3 l.13-14's edgePos, an upper bound).
//   3. Every member row is copied into its community's segment as (map[col], w)
//      (edge-parallel, one random gather per entry).
//   4. Each segment is merged (mergeCommunity): equal neighbours summed.
//      Segments <= 32 entries: a warp, __match_any_sync/__reduce_add_sync;
//      <= 4096: a CTA with a shared-memory table; larger: one device-wide
//      radix sort of (segment rank, neighbour) keys + run-length reduction.
//   5. Distinct counts prefix-summed into rowptr', entries compacted.
// Rows of the result are not sorted by column (nothing downstream depends on
// the order inside a row: every later step is an order-independent integer
// sum or a total-order argmax); louvain_aggregate keeps the canonical sorted
// variant (level_contract in lv_level.cu).
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "lv_device.cuh"
#include "lv_internal.cuh"

namespace lv {
namespace {

constexpr int kCTile = 4096;       // grouped entries per copy tile
constexpr int kCRows = 2048;       // member rows staged per copy tile
constexpr int kWarpMax = 512;      // segments merged by one warp (1024-slot table)
constexpr int kWarpSlots = 1024;
constexpr int kMidMax = 8192;      // segments merged by one CTA (16384-slot table)
constexpr int kMidSlots = 16384;

__global__ void k_flags(const int32_t* size, int64_t n, int32_t* flag) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x)
    flag[c] = size[c] > 0 ? 1 : 0;
}

__global__ void k_map_iota(const uint2* ca, const int32_t* newID, int64_t n, int32_t* map, int32_t* iota) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    map[i] = newID[ca[i].x];
    iota[i] = (int32_t)i;
  }
}

__global__ void k_kdeg(const uint2* ca, const int32_t* size, const int32_t* newID, int64_t n, uint32_t* kout) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x)
    if (size[c] > 0) kout[newID[c]] = ca[c].y;
}

// member degrees in grouped order; first member position of every new row
__global__ void k_group_meta(const int32_t* skey, const int32_t* vorder, int64_t n, const int64_t* rowptr,
                             int64_t* mdeg, int64_t* rfirst) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x) {
    if (i == n) {
      mdeg[n] = 0;
      continue;
    }
    const int32_t v = vorder[i];
    mdeg[i] = rowptr[v + 1] - rowptr[v];
    if (i == 0 || skey[i] != skey[i - 1]) rfirst[skey[i]] = i;
  }
}

__global__ void k_seg_bounds(const int64_t* rfirst, const int64_t* gpos, int64_t np, int64_t n, int64_t* sstart,
                             uint8_t* scls, int32_t* rid, unsigned long long* hist) {
  __shared__ unsigned long long sh[4];
  if (threadIdx.x < 4) sh[threadIdx.x] = 0;
  __syncthreads();
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < np; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = gpos[rfirst[r]], e = gpos[(r + 1 < np) ? rfirst[r + 1] : n];
    sstart[r] = b;
    const int64_t len = e - b;
    const int c = len <= 32 ? 0 : (len <= kWarpMax ? 1 : (len <= kMidMax ? 2 : 3));
    scls[r] = (uint8_t)c;
    rid[r] = (int32_t)r;
    atomicAdd(&sh[c], 1ull);
  }
  __syncthreads();
  if (threadIdx.x < 4 && sh[threadIdx.x]) atomicAdd(&hist[threadIdx.x], sh[threadIdx.x]);
}

// Step 3: grouped[t] = (map[col[e]], w[e]) for the t-th grouped entry.
__global__ void __launch_bounds__(256) k_group_copy(const int32_t* __restrict__ vorder,
                                                    const int64_t* __restrict__ gpos, int64_t n,
                                                    const int64_t* __restrict__ rowptr,
                                                    const int32_t* __restrict__ col, const uint32_t* __restrict__ w,
                                                    const int32_t* __restrict__ map, const int64_t* __restrict__ tr,
                                                    int32_t* gc, uint32_t* gw) {
  __shared__ int64_t sh_g[kCRows + 1];
  __shared__ int64_t sh_rb[kCRows];
  __shared__ int64_t sh_i0;
  __shared__ int sh_nr;
  const int64_t total = gpos[n];
  const int64_t ntiles = (total + kCTile - 1) / kCTile;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t t0 = tile * kCTile, t1 = min(total, t0 + kCTile);
    if (threadIdx.x == 0) {  // tile plan (tile_starts)
      const int64_t i0 = tr[tile], i1 = tr[tile + 1];
      sh_i0 = i0;
      sh_nr = (i1 - i0 + 1 <= kCRows) ? (int)(i1 - i0 + 1) : -1;
    }
    __syncthreads();
    const int64_t i0 = sh_i0;
    const int nr = sh_nr;
    for (int r = threadIdx.x; r < nr; r += blockDim.x) {
      sh_g[r] = gpos[i0 + r];
      sh_rb[r] = rowptr[vorder[i0 + r]];
    }
    __syncthreads();
    for (int64_t base = t0 + threadIdx.x; base < t1; base += 4 * (int64_t)blockDim.x) {
      int32_t jj[4];
      int64_t ee[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + (int64_t)q * blockDim.x;
        jj[q] = -1;
        ee[q] = 0;
        if (t < t1) {
          if (nr > 0) {
            int lo = 0, hi = nr - 1;
            while (lo < hi) {
              const int mid = (lo + hi + 1) >> 1;
              if (sh_g[mid] <= t) lo = mid; else hi = mid - 1;
            }
            ee[q] = sh_rb[lo] + (t - sh_g[lo]);
          } else {
            int64_t lo = 0, hi = n - 1;
            while (lo < hi) {
              const int64_t mid = (lo + hi + 1) >> 1;
              if (gpos[mid] <= t) lo = mid; else hi = mid - 1;
            }
            ee[q] = rowptr[vorder[lo]] + (t - gpos[lo]);
          }
          jj[q] = __ldcs(&col[ee[q]]);
        }
      }
      int32_t mm[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) mm[q] = jj[q] >= 0 ? __ldg(&map[jj[q]]) : 0;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + (int64_t)q * blockDim.x;
        if (t < t1) {  // evict-first: streamed once, must not displace map[] in L2
          __stcs(&gc[t], mm[q]);
          if (gw) __stcs(&gw[t], w ? __ldcs(&w[ee[q]]) : 1u);
        }
      }
    }
    __syncthreads();
  }
}

// Step 4a: segments of <= 32 entries, one warp each; distinct neighbours written
// compactly from the segment start; cnt[r] = distinct count.
__global__ void __launch_bounds__(256) k_merge_small(const int32_t* __restrict__ rows, int64_t nr,
                                                     const int64_t* __restrict__ sstart,
                                                     const int64_t* __restrict__ send_, const int32_t* __restrict__ gc,
                                                     const uint32_t* __restrict__ gw, int32_t* oc, uint32_t* ow,
                                                     int64_t* cnt) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t k = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < nr; k += warps) {
    const int32_t r = rows[k];
    const int64_t b = sstart[r], len = send_[r] - b;
    const bool has = lane < len;
    const int32_t c = has ? gc[b + lane] : (int32_t)(0x80000000u | (unsigned)lane);
    const uint32_t x = has ? (gw ? gw[b + lane] : 1u) : 0u;
    const unsigned m = __match_any_sync(kFull, c);
    const uint32_t sum = __reduce_add_sync(m, x);
    const bool leader = has && lane == __ffs(m) - 1;
    const unsigned lm = __ballot_sync(kFull, leader);
    if (leader) {
      const int pos = __popc(lm & ((1u << lane) - 1u));
      oc[b + pos] = c;
      ow[b + pos] = sum;
    }
    if (lane == 0) cnt[r] = __popc(lm);
  }
}

// Step 4b: segments of 33..512 entries, one warp each with a 1024-slot smem table.
__global__ void __launch_bounds__(128) k_merge_warp(const int32_t* __restrict__ rows, int64_t nr,
                                                    const int64_t* __restrict__ sstart,
                                                    const int64_t* __restrict__ send_, const int32_t* __restrict__ gc,
                                                    const uint32_t* __restrict__ gw, int32_t* oc, uint32_t* ow,
                                                    int64_t* cnt) {
  __shared__ unsigned long long tab[4][kWarpSlots];  // 4 warps x 8 KB
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  unsigned long long* T = tab[wl];
  for (int t = lane; t < kWarpSlots; t += 32) T[t] = kEmpty;
  __syncwarp();
  const int64_t warps = (int64_t)gridDim.x * 4;
  for (int64_t k = (int64_t)blockIdx.x * 4 + wl; k < nr; k += warps) {
    const int32_t r = rows[k];
    const int64_t b = sstart[r], len = send_[r] - b;
    const uint32_t cap = (uint32_t)(2 * len);
    for (int64_t t = lane; t < len; t += 32) {
      const int32_t c = gc[b + t];
      const uint32_t x = gw ? gw[b + t] : 1u;
      const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
      uint32_t h = hash_slot(c, cap);
      for (;;) {
        const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
        if (old == kEmpty) break;
        if ((old >> 32) == (unsigned long long)(uint32_t)c) {
          atomicAdd(&T[h], (unsigned long long)x);
          break;
        }
        h = (h + 1 == cap) ? 0 : h + 1;
      }
    }
    __syncwarp();
    int base = 0;
    for (uint32_t t0 = 0; t0 < cap; t0 += 32) {
      const uint32_t t = t0 + lane;
      const unsigned long long x = (t < cap) ? T[t] : kEmpty;
      const bool has = x != kEmpty;
      const unsigned m = __ballot_sync(kFull, has);
      if (has) {
        T[t] = kEmpty;
        const int pos = base + __popc(m & ((1u << lane) - 1u));
        oc[b + pos] = (int32_t)(x >> 32);
        ow[b + pos] = (uint32_t)x;
      }
      base += __popc(m);
    }
    if (lane == 0) cnt[r] = base;
    __syncwarp();
  }
}

// Step 4c: segments of 513..8192 entries, one CTA each (persistent), smem table.
__global__ void __launch_bounds__(512) k_merge_mid(const int32_t* __restrict__ rows, int64_t nr,
                                                   const int64_t* __restrict__ sstart,
                                                   const int64_t* __restrict__ send_, const int32_t* __restrict__ gc,
                                                   const uint32_t* __restrict__ gw, int32_t* oc, uint32_t* ow,
                                                   int64_t* cnt) {
  extern __shared__ unsigned long long T[];  // kMidSlots slots (dynamic: 64 KB)
  __shared__ unsigned ncnt;
  for (int t = threadIdx.x; t < kMidSlots; t += blockDim.x) T[t] = kEmpty;
  if (threadIdx.x == 0) ncnt = 0;
  __syncthreads();
  for (int64_t k = blockIdx.x; k < nr; k += gridDim.x) {
    const int32_t r = rows[k];
    const int64_t b = sstart[r], len = send_[r] - b;
    const uint32_t cap = (uint32_t)((2 * len < (int64_t)kMidSlots) ? 2 * len : (int64_t)kMidSlots);
    for (int64_t t = threadIdx.x; t < len; t += blockDim.x) {
      const int32_t c = gc[b + t];
      const uint32_t x = gw ? gw[b + t] : 1u;
      const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
      uint32_t h = hash_slot(c, cap);
      for (;;) {
        const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
        if (old == kEmpty) break;
        if ((old >> 32) == (unsigned long long)(uint32_t)c) {
          atomicAdd(&T[h], (unsigned long long)x);
          break;
        }
        h = (h + 1 == cap) ? 0 : h + 1;
      }
    }
    __syncthreads();
    for (uint32_t t = threadIdx.x; t < cap; t += blockDim.x) {
      const unsigned long long x = T[t];
      if (x == kEmpty) continue;
      T[t] = kEmpty;
      const unsigned pos = atomicAdd(&ncnt, 1u);
      oc[b + pos] = (int32_t)(x >> 32);
      ow[b + pos] = (uint32_t)x;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      cnt[r] = ncnt;
      ncnt = 0;
    }
    __syncthreads();
  }
}

// Step 4d: big segments.  keys = (rank of segment among big ones) << nb | neighbour,
// edge-parallel over the concatenated big segments (boff = their prefix offsets).
__global__ void k_big_keys(const int32_t* __restrict__ rows, int64_t nbig, const int64_t* __restrict__ sstart,
                           const int64_t* __restrict__ boff, const int32_t* __restrict__ gc,
                           const uint32_t* __restrict__ gw, int nb, unsigned long long* keys, uint32_t* vals) {
  const int64_t m = boff[nbig];
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x) {
    int64_t lo = 0, hi = nbig - 1;  // largest k with boff[k] <= t
    while (lo < hi) {
      const int64_t mid = (lo + hi + 1) >> 1;
      if (boff[mid] <= t) lo = mid; else hi = mid - 1;
    }
    const int64_t src = sstart[rows[lo]] + (t - boff[lo]);
    keys[t] = ((unsigned long long)lo << nb) | (unsigned long long)(uint32_t)gc[src];
    vals[t] = gw ? gw[src] : 1u;
  }
}

__global__ void k_big_first(const unsigned long long* __restrict__ ukeys, int64_t nruns, int nb, int64_t* first_run) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nruns; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = (int64_t)(ukeys[i] >> nb);
    if (i == 0 || (int64_t)(ukeys[i - 1] >> nb) != k) first_run[k] = i;
  }
}

__global__ void k_big_place(const unsigned long long* __restrict__ ukeys, const uint32_t* __restrict__ sums,
                            int64_t nruns, int nb, const int32_t* __restrict__ rows,
                            const int64_t* __restrict__ sstart, const int64_t* __restrict__ first_run, int32_t* oc,
                            uint32_t* ow, int64_t* cnt) {
  const unsigned long long mask = (1ull << nb) - 1ull;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nruns; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = (int64_t)(ukeys[i] >> nb);
    const int32_t r = rows[k];
    const int64_t local = i - first_run[k];
    oc[sstart[r] + local] = (int32_t)(ukeys[i] & mask);
    ow[sstart[r] + local] = sums[i];
    if (i == nruns - 1 || (int64_t)(ukeys[i + 1] >> nb) != k) cnt[r] = local + 1;
  }
}


// Step 4d (default): big segments merged in global-memory hash tables kept
// L2-resident by processing the segments in waves (each wave's tables <= kBigWaveSlots
// slots).  Table of a segment: cap = 2 * min(len, n') slots (load <= 1/2), split into
// 4-slot buckets read with two 16-byte loads; a label is claimed at the first
// empty slot of its probe sequence (one CAS) and summed with atomicAdd afterwards.
struct BigSeg {
  int64_t src;   // segment start in gc/gw and in oc/ow
  int64_t toff;  // table offset in the wave table
  int64_t cap;   // slots, multiple of 4
  int32_t row;
  int32_t pad;
};
struct BigItem {
  int32_t seg;
  int32_t pad;
  int64_t begin, end;  // insert: entries [begin, end) of the segment; extract: slots
};
constexpr int64_t kBigWaveSlots = 6 << 20;  // 48 MB of 8-byte slots per wave
constexpr int64_t kBigChunk = 4096;

__device__ __forceinline__ void big_insert4(unsigned long long* T, uint32_t cap, const int32_t c[4],
                                            const uint32_t x[4], bool todo[4]) {
  const uint32_t nb = cap >> 2;
  uint32_t b[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) b[q] = todo[q] ? (hash_slot(c[q], nb) << 2) : 0u;
  while (todo[0] || todo[1] || todo[2] || todo[3]) {
    unsigned long long k[4][4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (!todo[q]) continue;
      const ulonglong2 lo = __ldcg(reinterpret_cast<const ulonglong2*>(&T[b[q]]));
      const ulonglong2 hi = __ldcg(reinterpret_cast<const ulonglong2*>(&T[b[q] + 2]));
      k[q][0] = lo.x; k[q][1] = lo.y; k[q][2] = hi.x; k[q][3] = hi.y;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (!todo[q]) continue;
      int tgt = -1;
      bool found = false;
#pragma unroll
      for (int u = 3; u >= 0; --u)
        if (k[q][u] == kEmpty) tgt = u;
#pragma unroll
      for (int u = 3; u >= 0; --u)
        if (k[q][u] != kEmpty && (k[q][u] >> 32) == (unsigned long long)(uint32_t)c[q]) { tgt = u; found = true; }
      if (tgt < 0) {  // bucket full: next bucket
        b[q] = (b[q] + 4 >= cap) ? 0u : b[q] + 4;
        continue;
      }
      if (!found) {
        const unsigned long long old =
            atomicCAS(&T[b[q] + tgt], kEmpty, (((unsigned long long)(uint32_t)c[q]) << 32) | x[q]);
        if (old == kEmpty) { todo[q] = false; continue; }
        if ((old >> 32) != (unsigned long long)(uint32_t)c[q]) continue;  // lost the slot: re-read the bucket
      }
      atomicAdd(&T[b[q] + tgt], (unsigned long long)x[q]);
      todo[q] = false;
    }
  }
}

__global__ void __launch_bounds__(256) k_big_insert(const BigItem* __restrict__ items, int64_t nitems,
                                                    const BigSeg* __restrict__ segs, const int32_t* __restrict__ gc,
                                                    const uint32_t* __restrict__ gw, unsigned long long* T) {
  for (int64_t it = blockIdx.x; it < nitems; it += gridDim.x) {
    const BigItem item = items[it];
    const BigSeg sg = segs[item.seg];
    unsigned long long* Ts = T + sg.toff;
    for (int64_t base = item.begin + threadIdx.x; base < item.end; base += 4 * (int64_t)blockDim.x) {
      int32_t c[4];
      uint32_t x[4];
      bool todo[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + (int64_t)q * blockDim.x;
        todo[q] = t < item.end;
        c[q] = todo[q] ? __ldcs(&gc[sg.src + t]) : 0;
        x[q] = todo[q] ? (gw ? __ldcs(&gw[sg.src + t]) : 1u) : 0u;
      }
      big_insert4(Ts, (uint32_t)sg.cap, c, x, todo);
    }
  }
}

__global__ void __launch_bounds__(256) k_big_extract(const BigItem* __restrict__ items, int64_t nitems,
                                                     const BigSeg* __restrict__ segs, unsigned long long* T,
                                                     int32_t* oc, uint32_t* ow, int64_t* cnt) {
  const int lane = threadIdx.x & 31;
  for (int64_t it = blockIdx.x; it < nitems; it += gridDim.x) {
    const BigItem item = items[it];
    const BigSeg sg = segs[item.seg];
    unsigned long long* Ts = T + sg.toff;
    for (int64_t t0 = item.begin + (threadIdx.x - lane); t0 < item.end; t0 += blockDim.x) {  // warp-uniform trips
      const int64_t t = t0 + lane;
      unsigned long long x = kEmpty;
      if (t < item.end) {
        x = __ldcg(&Ts[t]);
        if (x != kEmpty) Ts[t] = kEmpty;  // clean for the next wave
      }
      const bool has = x != kEmpty;
      const unsigned m = __ballot_sync(kFull, has);
      if (!m) continue;
      unsigned long long base = 0;
      const int leader = __ffs(m) - 1;
      if (lane == leader) base = atomicAdd(reinterpret_cast<unsigned long long*>(&cnt[sg.row]), (unsigned long long)__popc(m));
      base = __shfl_sync(kFull, base, leader);
      if (has) {
        const int64_t pos = sg.src + (int64_t)base + __popc(m & ((1u << lane) - 1u));
        oc[pos] = (int32_t)(x >> 32);
        ow[pos] = (uint32_t)x;
      }
    }
  }
}

__global__ void k_fill_empty(unsigned long long* p, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = kEmpty;
}

// Step 5: compaction into the final CSR, edge-parallel over the output entries
// (tile of 4096 outputs: its rows' bounds staged in smem, binary search).
__global__ void __launch_bounds__(256) k_compact(const int64_t* __restrict__ sstart,
                                                 const int64_t* __restrict__ rowptr_out, int64_t np,
                                                 const int32_t* __restrict__ oc, const uint32_t* __restrict__ ow,
                                                 const int64_t* __restrict__ tr, int32_t* col, uint32_t* w) {
  __shared__ int64_t sh_r[kCRows + 1];
  __shared__ int64_t sh_s[kCRows];
  __shared__ int64_t sh_r0;
  __shared__ int sh_nr;
  const int64_t total = rowptr_out[np];
  const int64_t ntiles = (total + kCTile - 1) / kCTile;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t q0 = tile * kCTile, q1 = min(total, q0 + kCTile);
    if (threadIdx.x == 0) {  // tile plan (tile_starts)
      const int64_t r0 = tr[tile], r1 = tr[tile + 1];
      sh_r0 = r0;
      sh_nr = (r1 - r0 + 1 <= kCRows) ? (int)(r1 - r0 + 1) : -1;
    }
    __syncthreads();
    const int64_t r0 = sh_r0;
    const int nr = sh_nr;
    for (int r = threadIdx.x; r < nr; r += blockDim.x) {
      sh_r[r] = rowptr_out[r0 + r];
      sh_s[r] = sstart[r0 + r];
    }
    __syncthreads();
    for (int64_t q = q0 + threadIdx.x; q < q1; q += blockDim.x) {
      int64_t src;
      if (nr > 0) {
        int lo = 0, hi = nr - 1;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (sh_r[mid] <= q) lo = mid; else hi = mid - 1;
        }
        src = sh_s[lo] + (q - sh_r[lo]);
      } else {
        int64_t lo = 0, hi = np - 1;
        while (lo < hi) {
          const int64_t mid = (lo + hi + 1) >> 1;
          if (rowptr_out[mid] <= q) lo = mid; else hi = mid - 1;
        }
        src = sstart[lo] + (q - rowptr_out[lo]);
      }
      col[q] = __ldcs(&oc[src]);
      w[q] = __ldcs(&ow[src]);
    }
    __syncthreads();
  }
}

template <class... A>
int32_t cub_scan_excl(cudaStream_t s, A... a) {
  size_t tb = 0;
  LV_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, a..., s));
  void* tmp = nullptr;
  LV_TRY(dmalloc(&tmp, tb, s));
  LV_CUDA(cub::DeviceScan::ExclusiveSum(tmp, tb, a..., s));
  LV_CUB();
  dfree(tmp, s);
  return LOUVAIN_OK;
}

}  // namespace

namespace {
struct CTrace {
  bool on = getenv("LV_TRACE") != nullptr;
  std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
  void mark(cudaStream_t s, const char* what) {
    if (!on) return;
    cudaStreamSynchronize(s);
    const auto t1 = std::chrono::steady_clock::now();
    fprintf(stderr, "[lv]    contract %-10s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(t1 - t0).count());
    t0 = t1;
  }
};
}  // namespace

int32_t level_contract_fast(Handle& h, Level& L, Level& out, int32_t* d_map, int parity) {
  cudaStream_t s = h.stream;
  CTrace tr;
  const int64_t n = L.n, nnz = L.nnz;
  if (n == 0 || nnz == 0) return level_contract(h, L, out, d_map, parity);
  out = Level();
  out.W = L.W;
  // 1. newID, map, next degrees
  int32_t *flag = nullptr, *newID = nullptr, *iota = nullptr;
  LV_TRY(dalloc(&flag, n, s));
  LV_TRY(dalloc(&newID, n, s));
  LV_TRY(dalloc(&iota, n, s));
  k_flags<<<grid_for(n, 256), 256, 0, s>>>(L.size, n, flag);
  LV_LAUNCHED();
  LV_TRY(cub_scan_excl(s, flag, newID, n));
  int32_t last[2];
  LV_CUDA(cudaMemcpyAsync(&last[0], newID + n - 1, 4, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaMemcpyAsync(&last[1], flag + n - 1, 4, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaStreamSynchronize(s));
  const int64_t np = (int64_t)last[0] + last[1];
  k_map_iota<<<grid_for(n, 256), 256, 0, s>>>(L.ca, newID, n, d_map, iota);
  LV_LAUNCHED();
  out.n = np;
  LV_TRY(level_alloc_scratch(h, out, parity));
  k_kdeg<<<grid_for(n, 256), 256, 0, s>>>(L.ca, L.size, newID, n, out.k);
  LV_LAUNCHED();
  out.k_ready = true;
  dfree(flag, s);
  dfree(newID, s);
  tr.mark(s, "newid");
  int nb = 1;
  while (nb < 31 && (1ll << nb) < np) ++nb;
  // 2. members grouped by new vertex
  int32_t *skey = nullptr, *vorder = nullptr;
  LV_TRY(dalloc(&skey, n, s));
  LV_TRY(dalloc(&vorder, n, s));
  {
    size_t tb = 0;
    LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, d_map, skey, iota, vorder, n, 0, nb, s));
    void* tmp = nullptr;
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, d_map, skey, iota, vorder, n, 0, nb, s));
    LV_CUB();
    dfree(tmp, s);
  }
  dfree(iota, s);
  int64_t *mdeg = nullptr, *gpos = nullptr, *rfirst = nullptr;
  LV_TRY(dalloc(&mdeg, n + 1, s));
  LV_TRY(dalloc(&gpos, n + 1, s));
  LV_TRY(dalloc(&rfirst, np + 1, s));
  k_group_meta<<<grid_for(n + 1, 256), 256, 0, s>>>(skey, vorder, n, L.rowptr, mdeg, rfirst);
  LV_LAUNCHED();
  LV_TRY(cub_scan_excl(s, mdeg, gpos, n + 1));
  dfree(mdeg, s);
  dfree(skey, s);
  tr.mark(s, "group");
  // 3. grouped copy
  const bool weighted = L.w != nullptr;
  int32_t* gc = nullptr;
  uint32_t* gw = nullptr;
  {
    void* p0 = nullptr;
    LV_TRY(scratch_get(h, SC_GC, 4 * (size_t)nnz, &p0));
    gc = static_cast<int32_t*>(p0);
    if (weighted) {
      LV_TRY(scratch_get(h, SC_GW, 4 * (size_t)nnz, &p0));
      gw = static_cast<uint32_t*>(p0);
    }
  }
  {
    const int64_t* tr = nullptr;
    LV_TRY(tile_starts(h, gpos, 0, n, 0, nnz, kCTile, &tr));
    k_group_copy<<<grid_for((nnz + kCTile - 1) / kCTile, 1, 148 * 8), 256, 0, s>>>(vorder, gpos, n, L.rowptr, L.col,
                                                                                      L.w, d_map, tr, gc, gw);
  }
  LV_LAUNCHED();
  dfree(vorder, s);
  tr.mark(s, "copy");
  // segment bounds and classes
  int64_t *sstart = nullptr, *send_ = nullptr;
  uint8_t *scls = nullptr, *scls2 = nullptr;
  int32_t *rid = nullptr, *rows = nullptr;
  LV_TRY(dalloc(&sstart, np + 1, s));
  LV_TRY(dalloc(&scls, np, s));
  LV_TRY(dalloc(&scls2, np, s));
  LV_TRY(dalloc(&rid, np, s));
  LV_TRY(dalloc(&rows, np, s));
  unsigned long long* hist = nullptr;
  LV_TRY(dalloc(&hist, 4, s));
  LV_CUDA(cudaMemsetAsync(hist, 0, 32, s));
  k_seg_bounds<<<grid_for(np, 256), 256, 0, s>>>(rfirst, gpos, np, n, sstart, scls, rid, hist);
  LV_LAUNCHED();
  unsigned long long hh[4];
  LV_CUDA(cudaMemcpyAsync(hh, hist, 32, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaMemcpyAsync(sstart + np, gpos + n, 8, cudaMemcpyDeviceToDevice, s));
  send_ = sstart + 1;
  dfree(rfirst, s);
  dfree(gpos, s);
  {
    size_t tb = 0;
    LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, scls, scls2, rid, rows, np, 0, 2, s));
    void* tmp = nullptr;
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, scls, scls2, rid, rows, np, 0, 2, s));  // 4 classes
    LV_CUB();
    dfree(tmp, s);
  }
  LV_CUDA(cudaStreamSynchronize(s));
  dfree(hist, s);
  const int64_t nsmall = (int64_t)hh[0], nwarp = (int64_t)hh[1], nmid = (int64_t)hh[2], nbig = (int64_t)hh[3];
  dfree(scls, s);
  dfree(scls2, s);
  dfree(rid, s);
  tr.mark(s, "classes");
  // 4. merge
  int32_t* oc = nullptr;
  uint32_t* ow = nullptr;
  int64_t* cnt = nullptr;
  {
    void* p0 = nullptr;
    LV_TRY(scratch_get(h, SC_OC, 4 * (size_t)nnz, &p0));
    oc = static_cast<int32_t*>(p0);
    LV_TRY(scratch_get(h, SC_OW, 4 * (size_t)nnz, &p0));
    ow = static_cast<uint32_t*>(p0);
  }
  LV_TRY(dalloc(&cnt, np + 1, s));
  LV_CUDA(cudaMemsetAsync(cnt, 0, 8 * (np + 1), s));
  if (nsmall > 0) {
    k_merge_small<<<grid_for(nsmall, 8, 148 * 16), 256, 0, s>>>(rows, nsmall, sstart, send_, gc, gw, oc, ow, cnt);
    LV_LAUNCHED();
  }
  if (nwarp > 0) {
    k_merge_warp<<<grid_for(nwarp, 4, 148 * 12), 128, 0, s>>>(rows + nsmall, nwarp, sstart, send_, gc, gw, oc, ow, cnt);
    LV_LAUNCHED();
  }
  if (nmid > 0) {
    static bool attr = false;
    if (!attr) {
      LV_CUDA(cudaFuncSetAttribute(k_merge_mid, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * kMidSlots));
      attr = true;
    }
    k_merge_mid<<<grid_for(nmid, 1, 148), 512, 8 * kMidSlots, s>>>(rows + nsmall + nwarp, nmid, sstart, send_, gc, gw,
                                                                    oc, ow, cnt);
    LV_LAUNCHED();
  }
  tr.mark(s, "merge-sm");
  static const bool big_sort = getenv("LV_BIG_SORT") && getenv("LV_BIG_SORT")[0] == '1';
  if (nbig > 0 && !big_sort) {
    const int32_t* brows = rows + nsmall + nwarp + nmid;
    std::vector<int32_t> hb(nbig);
    LV_CUDA(cudaMemcpyAsync(hb.data(), brows, 4 * nbig, cudaMemcpyDeviceToHost, s));
    std::vector<int64_t> hs(np + 1);
    LV_CUDA(cudaMemcpyAsync(hs.data(), sstart, 8 * (np + 1), cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    // waves of segments whose tables fit kBigWaveSlots (a larger segment gets a wave of its own)
    std::vector<BigSeg> segs(nbig);
    std::vector<BigItem> ins, ext;
    std::vector<int64_t> ins_off{0}, ext_off{0};
    int64_t acc = 0, maxslots = 0, big_entries = 0;
    for (int64_t k = 0; k < nbig; ++k) {
      const int32_t r = hb[k];
      const int64_t len = hs[r + 1] - hs[r];
      big_entries += len;
      const int64_t cap = ((2 * std::min<int64_t>(len, np) + 3) / 4) * 4;
      if (acc > 0 && acc + cap > kBigWaveSlots) {
        ins_off.push_back((int64_t)ins.size());
        ext_off.push_back((int64_t)ext.size());
        acc = 0;
      }
      segs[k] = BigSeg{hs[r], acc, cap, r, 0};
      for (int64_t e = 0; e < len; e += kBigChunk) ins.push_back(BigItem{(int32_t)k, 0, e, std::min(len, e + kBigChunk)});
      for (int64_t e = 0; e < cap; e += kBigChunk) ext.push_back(BigItem{(int32_t)k, 0, e, std::min(cap, e + kBigChunk)});
      acc += cap;
      maxslots = std::max(maxslots, acc);
    }
    ins_off.push_back((int64_t)ins.size());
    ext_off.push_back((int64_t)ext.size());
    const int64_t nwaves = (int64_t)ins_off.size() - 1;
    if (tr.on)
      fprintf(stderr, "[lv]    contract segments: small %lld warp %lld mid %lld big %lld (big entries %lld of %lld, "
              "%lld waves)\n", (long long)nsmall, (long long)nwarp, (long long)nmid, (long long)nbig,
              (long long)big_entries, (long long)nnz, (long long)nwaves);
    BigSeg* dsegs = nullptr;
    BigItem *dins = nullptr, *dext = nullptr;
    LV_TRY(dalloc(&dsegs, nbig, s));
    LV_TRY(dalloc(&dins, ins.size(), s));
    LV_TRY(dalloc(&dext, ext.size(), s));
    LV_CUDA(cudaMemcpyAsync(dsegs, segs.data(), sizeof(BigSeg) * nbig, cudaMemcpyHostToDevice, s));
    LV_CUDA(cudaMemcpyAsync(dins, ins.data(), sizeof(BigItem) * ins.size(), cudaMemcpyHostToDevice, s));
    LV_CUDA(cudaMemcpyAsync(dext, ext.data(), sizeof(BigItem) * ext.size(), cudaMemcpyHostToDevice, s));
    unsigned long long* T = nullptr;
    {
      void* p0 = nullptr;
      LV_TRY(scratch_get(h, SC_K1, 8 * (size_t)maxslots, &p0));
      T = static_cast<unsigned long long*>(p0);
    }
    k_fill_empty<<<grid_for(maxslots, 256, 148 * 8), 256, 0, s>>>(T, maxslots);
    LV_LAUNCHED();
    for (int64_t wv = 0; wv < nwaves; ++wv) {
      const int64_t i0 = ins_off[wv], i1 = ins_off[wv + 1], x0 = ext_off[wv], x1 = ext_off[wv + 1];
      k_big_insert<<<grid_for(i1 - i0, 1, 148 * 8), 256, 0, s>>>(dins + i0, i1 - i0, dsegs, gc, gw, T);
      LV_LAUNCHED();
      k_big_extract<<<grid_for(x1 - x0, 1, 148 * 8), 256, 0, s>>>(dext + x0, x1 - x0, dsegs, T, oc, ow, cnt);
      LV_LAUNCHED();
    }
    LV_CUDA(cudaGetLastError());
    dfree(dsegs, s);
    dfree(dins, s);
    dfree(dext, s);
    LV_CUDA(cudaStreamSynchronize(s));  // host vectors die here
  } else if (nbig > 0) {  // LV_BIG_SORT=1: radix sort of (segment rank, neighbour) keys + reduce-by-key
    const int32_t* brows = rows + nsmall + nwarp + nmid;
    // offsets of big segments in the key array (their lengths, host-side: nbig is small)
    std::vector<int32_t> hb(nbig);
    LV_CUDA(cudaMemcpyAsync(hb.data(), brows, 4 * nbig, cudaMemcpyDeviceToHost, s));
    std::vector<int64_t> hs(np + 1);
    LV_CUDA(cudaMemcpyAsync(hs.data(), sstart, 8 * (np + 1), cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    std::vector<int64_t> boff(nbig + 1, 0);
    for (int64_t k = 0; k < nbig; ++k) boff[k + 1] = boff[k] + (hs[hb[k] + 1] - hs[hb[k]]);
    const int64_t m = boff[nbig];
    if (tr.on)
      fprintf(stderr, "[lv]    contract segments: small %lld warp %lld mid %lld big %lld (big entries %lld of %lld)\n",
              (long long)nsmall, (long long)nwarp, (long long)nmid, (long long)nbig, (long long)m, (long long)nnz);
    int64_t* dboff = nullptr;
    LV_TRY(dalloc(&dboff, nbig + 1, s));
    LV_CUDA(cudaMemcpyAsync(dboff, boff.data(), 8 * (nbig + 1), cudaMemcpyHostToDevice, s));
    int kb = 1;
    while (kb < 40 && (1ll << kb) < nbig) ++kb;
    unsigned long long *k0 = nullptr, *k1 = nullptr;
    uint32_t *v0 = nullptr, *v1 = nullptr;
    {
      void* p0 = nullptr;
      LV_TRY(scratch_get(h, SC_STAGE, 8 * (size_t)m, &p0));  // the level's stage is dead during contraction
      k0 = static_cast<unsigned long long*>(p0);
      LV_TRY(scratch_get(h, SC_K1, 8 * (size_t)m, &p0));
      k1 = static_cast<unsigned long long*>(p0);
      LV_TRY(scratch_get(h, SC_V0, 4 * (size_t)m, &p0));
      v0 = static_cast<uint32_t*>(p0);
      LV_TRY(scratch_get(h, SC_V1, 4 * (size_t)m, &p0));
      v1 = static_cast<uint32_t*>(p0);
    }
    k_big_keys<<<grid_for(m, 256, 148 * 16), 256, 0, s>>>(brows, nbig, sstart, dboff, gc, gw, nb, k0, v0);
    LV_LAUNCHED();
    cub::DoubleBuffer<unsigned long long> kbuf(k0, k1);
    cub::DoubleBuffer<uint32_t> vbuf(v0, v1);
    size_t tb = 0;
    LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, kbuf, vbuf, m, 0, nb + kb, s));
    void* tmp = nullptr;
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, kbuf, vbuf, m, 0, nb + kb, s));
    LV_CUB();
    dfree(tmp, s);
    int64_t* dnum = reinterpret_cast<int64_t*>(&h.ctl->bad);
    tb = 0;
    LV_CUDA(cub::DeviceReduce::ReduceByKey(nullptr, tb, kbuf.Current(), kbuf.Alternate(), vbuf.Current(),
                                           vbuf.Alternate(), dnum, cub::Sum(), m, s));
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceReduce::ReduceByKey(tmp, tb, kbuf.Current(), kbuf.Alternate(), vbuf.Current(),
                                           vbuf.Alternate(), dnum, cub::Sum(), m, s));
    LV_CUB();
    dfree(tmp, s);
    int64_t nruns = 0;
    LV_CUDA(cudaMemcpyAsync(&nruns, dnum, 8, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    int64_t* first_run = nullptr;
    LV_TRY(dalloc(&first_run, nbig, s));
    k_big_first<<<grid_for(nruns, 256), 256, 0, s>>>(kbuf.Alternate(), nruns, nb, first_run);
    LV_LAUNCHED();
    k_big_place<<<grid_for(nruns, 256), 256, 0, s>>>(kbuf.Alternate(), vbuf.Alternate(), nruns, nb, brows, sstart,
                                                      first_run, oc, ow, cnt);
    LV_LAUNCHED();
    dfree(first_run, s);
    dfree(dboff, s);
  }
  tr.mark(s, "merge-big");
  dfree(rows, s);
  // 5. rowptr' and compaction
  auto lvl = [&](int a, size_t bytes, void** o) { return scratch_get(h, SC_LVL0 + 2 * a + parity, bytes, o); };
  LV_TRY(lvl(LA_ROWPTR, 8 * (size_t)(np + 1), (void**)&out.rowptr));
  LV_TRY(cub_scan_excl(s, cnt, out.rowptr, np + 1));
  int64_t m2 = 0;
  LV_CUDA(cudaMemcpyAsync(&m2, out.rowptr + np, 8, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaStreamSynchronize(s));
  out.nnz = m2;
  LV_TRY(lvl(LA_COL, 4 * (size_t)std::max<int64_t>(m2, 1), (void**)&out.col));
  LV_TRY(lvl(LA_W, 4 * (size_t)std::max<int64_t>(m2, 1), (void**)&out.w));
  if (m2 > 0) {
    const int64_t* tr = nullptr;
    LV_TRY(tile_starts(h, out.rowptr, 0, np, 0, m2, kCTile, &tr));
    k_compact<<<grid_for((m2 + kCTile - 1) / kCTile, 1, 148 * 8), 256, 0, s>>>(sstart, out.rowptr, np, oc, ow, tr,
                                                                                out.col, out.w);
  }
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  dfree(cnt, s);
  dfree(sstart, s);
  tr.mark(s, "compact");
  return LOUVAIN_OK;
}

}  // namespace lv
