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
#include <thrust/iterator/transform_iterator.h>
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
// segment classes: 0 small (<= 32), 1..2 warp ([33,128] with 256-slot tables,
// [129,kWarpMax] with 1024), 3..6 CTA tiers with tables sized to the tier
// ([513,1024), [1024,2048), [2048,4096), [4096,kMidMax]), 7 big
constexpr int kSegClasses = 8;
constexpr int kMidTierCap[4] = {2048, 4096, 8192, kMidSlots};
constexpr int kMidTierThr[4] = {128, 256, 512, 512};

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
                             uint8_t* scls, int32_t* rid, unsigned long long* hist, int64_t c_lo, int64_t c_hi) {
  __shared__ unsigned long long sh[kSegClasses];
  if (threadIdx.x < kSegClasses) sh[threadIdx.x] = 0;
  __syncthreads();
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < np; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = gpos[rfirst[r]], e = gpos[(r + 1 < np) ? rfirst[r + 1] : n];
    sstart[r] = b;
    if (r < c_lo || r >= c_hi) continue;  // merged by another rank (sharded contraction)
    const int64_t len = e - b;
    const int c = len <= 32 ? 0 : len <= 128 ? 1 : len <= kWarpMax ? 2 : len < 1024 ? 3 : len < 2048 ? 4
                : len < 4096 ? 5 : len <= kMidMax ? 6 : 7;
    scls[r] = (uint8_t)c;
    rid[r] = (int32_t)r;
    atomicAdd(&sh[c], 1ull);
  }
  __syncthreads();
  if (threadIdx.x < kSegClasses && sh[threadIdx.x]) atomicAdd(&hist[threadIdx.x], sh[threadIdx.x]);
}

// Sharded contraction (distributed handle): new vertices [cut[r], cut[r+1]) are merged by
// rank r, cut[r] = first new vertex whose grouped segment starts at >= r * nnz / world.
__global__ void k_seg_split(const int64_t* __restrict__ rfirst, const int64_t* __restrict__ gpos, int64_t np,
                            int64_t nnz, int world, int64_t* cut) {
  const int r = threadIdx.x;
  if (r > world) return;
  if (r == 0 || r == world) {
    cut[r] = r == 0 ? 0 : np;
    return;
  }
  const int64_t target = (int64_t)((__int128)r * nnz / world);
  int64_t lo = 0, hi = np;  // lower_bound over segment starts gpos[rfirst[c]]
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (gpos[rfirst[mid]] < target) lo = mid + 1; else hi = mid;
  }
  cut[r] = lo;
}

// Step 3: every member row copied in source order -- rows read sequentially, each
// row's entries written to its member's slot of the grouped layout (dbase[u] =
// gpos[rank of u]); the only random access per entry is the map[col] gather.
__global__ void k_dest_base(const int32_t* __restrict__ vorder, const int64_t* __restrict__ gpos, int64_t n,
                            int64_t* dbase) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dbase[vorder[i]] = gpos[i];
}

#ifndef LV_DH_CONTRACT  // compile-time A/B: double hashing in the power-of-two contraction tables
#define LV_DH_CONTRACT 1
#endif
#ifndef LV_DH_POW2  // compile-time A/B: merge / hub-task tables rounded up to powers of two + double hashing
#define LV_DH_POW2 1
#endif
constexpr int kSTile = 4096;  // CSR entries per scatter-copy tile
constexpr int kSRows = 1024;  // rows staged per tile (else per-entry search in global memory)
template <bool RANGE>  // RANGE: sharded contraction, only rows whose new vertex is in [c_lo, c_hi)
__global__ void __launch_bounds__(256) k_scatter_copy(const int64_t* __restrict__ rowptr, int64_t n,
                                                      const int32_t* __restrict__ col,
                                                      const uint32_t* __restrict__ w,
                                                      const int32_t* __restrict__ map,
                                                      const int64_t* __restrict__ dbase, int64_t nnz,
                                                      const int64_t* __restrict__ tr, int32_t* gc, uint32_t* gw,
                                                      int32_t c_lo, int32_t c_hi) {
  __shared__ int64_t sh_rp[kSRows + 1];
  __shared__ int64_t sh_db[kSRows];
  __shared__ int32_t sh_mine[RANGE ? kSRows : 1];  // the row's new vertex is in this rank's range
  __shared__ int64_t sh_u0;
  __shared__ int sh_nr;
  const int64_t ntiles = (nnz + kSTile - 1) / kSTile;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t e0 = tile * kSTile, e1 = min(nnz, e0 + kSTile);
    if (threadIdx.x == 0) {
      const int64_t u0 = tr[tile], u1 = tr[tile + 1];
      sh_u0 = u0;
      sh_nr = (u1 - u0 + 1 <= kSRows) ? (int)(u1 - u0 + 1) : -1;
    }
    __syncthreads();
    const int64_t u0 = sh_u0;
    const int nr = sh_nr;
    for (int r = threadIdx.x; r < nr; r += blockDim.x) {
      sh_rp[r] = rowptr[u0 + r];
      sh_db[r] = dbase[u0 + r];
      if (RANGE && u0 + r < n) {
        const int32_t c = map[u0 + r];
        sh_mine[r] = c >= c_lo && c < c_hi;
      }
    }
    __syncthreads();
    // warp spans of 128 entries (lane + 32 q): one binary search per lane, then a
    // forward walk (the next entry of a lane is 32 further, mostly in the same row)
    const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int64_t span = e0 + (int64_t)wl * 32 * kSpanQ; span < e1; span += (int64_t)nw * 32 * kSpanQ) {
      int32_t jj[kSpanQ];
      int64_t dd[kSpanQ];
      int lo = 0;
      if (nr > 0 && span + lane < e1) {
        int hi = nr - 1;  // largest r with sh_rp[r] <= e
        const int64_t e = span + lane;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (sh_rp[mid] <= e) lo = mid; else hi = mid - 1;
        }
      }
#pragma unroll
      for (int q = 0; q < kSpanQ; ++q) {
        const int64_t e = span + lane + 32 * q;
        jj[q] = -1;
        dd[q] = 0;
        if (e < e1) {
          if (nr > 0) {
            while (lo + 1 < nr && sh_rp[lo + 1] <= e) ++lo;
            dd[q] = sh_db[lo] + (e - sh_rp[lo]);
            if (RANGE && !sh_mine[lo]) continue;  // another rank merges this row's community
          } else {
            int64_t a = 0, b = n - 1;
            while (a < b) {
              const int64_t mid = (a + b + 1) >> 1;
              if (rowptr[mid] <= e) a = mid; else b = mid - 1;
            }
            dd[q] = dbase[a] + (e - rowptr[a]);
            if (RANGE) {
              const int32_t c = map[a];
              if (c < c_lo || c >= c_hi) continue;
            }
          }
          jj[q] = __ldcs(&col[e]);
        }
      }
      int32_t mm[kSpanQ];
#pragma unroll
      for (int q = 0; q < kSpanQ; ++q) mm[q] = jj[q] >= 0 ? __ldg(&map[jj[q]]) : 0;
#pragma unroll
      for (int q = 0; q < kSpanQ; ++q) {
        const int64_t e = span + lane + 32 * q;
        if (e < e1 && jj[q] >= 0) {
          gc[dd[q]] = mm[q];
          if (gw) gw[dd[q]] = w ? __ldcs(&w[e]) : 1u;
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
// One entry t of the segment at gc/gw + b into a smem table (all 32 lanes of the warp
// call it; t >= len idles): when adjacent entries repeat a neighbour, the warp's copies of
// each neighbour are summed first (group_sum: one table atomic per neighbour and warp --
// the members of a community mostly point at a few communities; same-slot atomics serialise).
__device__ __forceinline__ void merge_insert(unsigned long long* T, uint32_t cap, const int32_t* __restrict__ gc,
                                             const uint32_t* __restrict__ gw, int64_t b, int64_t t, int64_t len) {
  const int lane = threadIdx.x & 31;
  const bool has = t < len;
  const int32_t c = has ? gc[b + t] : (int32_t)(0x80000000u | (unsigned)lane);
  uint32_t x = has ? (gw ? gw[b + t] : 1u) : 0u;
  unsigned m = 1u << lane;
  if (__any_sync(kFull, c == __shfl_xor_sync(kFull, c, 1))) group_sum((uint32_t)c, x, m);  // adaptive
  if (!has || lane != __ffs(m) - 1) return;
  const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
  uint32_t h = hash_slot(c, cap);
  for (;;) {
    const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
    if (old == kEmpty) break;
    if ((old >> 32) == (unsigned long long)(uint32_t)c) {
      atomicAdd(&T[h], (unsigned long long)x);
      break;
    }
#if LV_DH_POW2
    h = probe_next(h, cap, probe_step(c));
#else
    h = (h + 1 == cap) ? 0 : h + 1;
#endif
  }
}

template <int SLOTS>
__global__ void __launch_bounds__(128) k_merge_warp(const int32_t* __restrict__ rows, int64_t nr,
                                                    const int64_t* __restrict__ sstart,
                                                    const int64_t* __restrict__ send_, const int32_t* __restrict__ gc,
                                                    const uint32_t* __restrict__ gw, int32_t* oc, uint32_t* ow,
                                                    int64_t* cnt) {
  __shared__ unsigned long long tab[4][SLOTS];  // 4 warps x SLOTS x 8 B
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  unsigned long long* T = tab[wl];
  for (int t = lane; t < SLOTS; t += 32) T[t] = kEmpty;
  __syncwarp();
  const int64_t warps = (int64_t)gridDim.x * 4;
  for (int64_t k = (int64_t)blockIdx.x * 4 + wl; k < nr; k += warps) {
    const int32_t r = rows[k];
    const int64_t b = sstart[r], len = send_[r] - b;
#if LV_DH_POW2
    const uint32_t cap = pow2_at_least((uint32_t)(2 * len), SLOTS);
#else
    const uint32_t cap = (uint32_t)(2 * len);
#endif
    for (int64_t t0 = 0; t0 < len; t0 += 32) merge_insert(T, cap, gc, gw, b, t0 + lane, len);
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
                                                   int64_t* cnt, int capmax) {
  extern __shared__ unsigned long long T[];  // capmax slots (dynamic)
  __shared__ unsigned ncnt;
  for (int t = threadIdx.x; t < capmax; t += blockDim.x) T[t] = kEmpty;
  if (threadIdx.x == 0) ncnt = 0;
  __syncthreads();
  for (int64_t k = blockIdx.x; k < nr; k += gridDim.x) {
    const int32_t r = rows[k];
    const int64_t b = sstart[r], len = send_[r] - b;
#if LV_DH_POW2
    const uint32_t cap = (2 * len < (int64_t)capmax) ? pow2_at_least((uint32_t)(2 * len), (uint32_t)capmax)
                                                     : (uint32_t)capmax;
#else
    const uint32_t cap = (uint32_t)((2 * len < (int64_t)capmax) ? 2 * len : (int64_t)capmax);
#endif
    for (int64_t tb = threadIdx.x & ~31; tb < len; tb += blockDim.x)  // warp-uniform trips
      merge_insert(T, cap, gc, gw, b, tb + (threadIdx.x & 31), len);
    __syncthreads();
    // distinct keys appended with one shared atomic per warp and pass (not per key:
    // a single counter serialised every key of the CTA)
    const int lane = threadIdx.x & 31;
    for (uint32_t t0 = threadIdx.x - lane; t0 < cap; t0 += blockDim.x) {
      const uint32_t t = t0 + lane;
      const unsigned long long x = t < cap ? T[t] : kEmpty;
      const bool has = x != kEmpty;
      const unsigned m = __ballot_sync(kFull, has);
      if (!m) continue;
      unsigned base = 0;
      if (lane == 0) base = atomicAdd(&ncnt, (unsigned)__popc(m));
      base = __shfl_sync(kFull, base, 0);
      if (has) {
        T[t] = kEmpty;
        const unsigned pos = base + __popc(m & ((1u << lane) - 1u));
        oc[b + pos] = (int32_t)(x >> 32);
        ow[b + pos] = (uint32_t)x;
      }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      cnt[r] = ncnt;
      ncnt = 0;
    }
    __syncthreads();
  }
}


__global__ void k_big_place32(const uint32_t* __restrict__ ukeys, const uint32_t* __restrict__ sums,
                              const int64_t* __restrict__ dnum, int nb, const int32_t* __restrict__ rows,
                              const int64_t* __restrict__ sstart, int32_t* oc, uint32_t* ow, int64_t* cnt) {
  const int64_t nruns = *dnum;
  const uint32_t mask = (nb >= 32) ? 0xFFFFFFFFu : ((1u << nb) - 1u);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nruns; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t k = ukeys[i] >> nb;
    // first run of segment k: binary search back over the sorted run keys
    int64_t lo = 0, hi = i;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if ((ukeys[mid] >> nb) < k) lo = mid + 1; else hi = mid;
    }
    const int32_t r = rows[k];
    const int64_t local = i - lo;
    oc[sstart[r] + local] = (int32_t)(ukeys[i] & mask);
    ow[sstart[r] + local] = sums[i];
    if (i == nruns - 1 || (ukeys[i + 1] >> nb) != k) cnt[r] = local + 1;
  }
}

// Step 4d: big segments.  keys = (rank of segment among big ones) << nb | neighbour
// (k_big_keys_t below), one 64-bit radix sort, reduce-by-key, then placement.
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



// Combiner for the big segments when their keys are 32-bit (few new vertices: the
// contracted graph is small and the big segments repeat the same neighbours many
// times -- C5 level 2: 1.7e9 entries -> 3.6e6 distinct).  Each CTA folds a chunk
// of kCombChunk (key, weight) pairs in a shared-memory table (one slot {key:32 |
// sum:32}); a pair whose probe sequence passes kCombProbes slots is passed through
// unchanged.  The output (distinct pairs of every chunk + pass-throughs) has the
// same sums per key as the input, so the radix sort + reduce-by-key that follow
// give the same result on far fewer elements.
constexpr int kCombSlots = 16384;
constexpr int kCombChunk = 65536;
constexpr int kCombProbes = 32;
template <int SLOTS, int BITS, int CHUNK, int THREADS>
__global__ void __launch_bounds__(THREADS) k_big_combine(const uint32_t* __restrict__ keys,
                                                         const uint32_t* __restrict__ vals, int64_t m,
                                                         uint32_t* __restrict__ okeys, uint32_t* __restrict__ ovals,
                                                         unsigned long long* ocount) {
  extern __shared__ unsigned long long T[];  // SLOTS
  __shared__ unsigned wcnt[32];
  __shared__ unsigned long long sh_base;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int t = threadIdx.x; t < SLOTS; t += blockDim.x) T[t] = kEmpty;
  __syncthreads();
  const int64_t nch = (m + CHUNK - 1) / CHUNK;
  for (int64_t ch = blockIdx.x; ch < nch; ch += gridDim.x) {
    const int64_t e0 = ch * CHUNK, e1 = min(m, e0 + CHUNK);
    for (int64_t eb = e0 + threadIdx.x; eb - threadIdx.x < e1; eb += 4 * (int64_t)blockDim.x) {
      uint32_t k[4], v[4];
      bool pass[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t e = eb + (int64_t)q * blockDim.x;
        pass[q] = false;
        k[q] = 0xFFFFFFFFu;
        v[q] = 0;
        if (e < e1) {
          k[q] = __ldcs(&keys[e]);
          v[q] = __ldcs(&vals[e]);
        }
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {  // equal keys of a warp merged first (hot neighbours)
        const unsigned mm = __match_any_sync(kFull, k[q]);
        v[q] = __reduce_add_sync(mm, v[q]);
        if (lane != __ffs(mm) - 1) k[q] = 0xFFFFFFFFu;
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (k[q] == 0xFFFFFFFFu) continue;
        const unsigned long long kx = ((unsigned long long)k[q] << 32) | v[q];
        uint32_t h = (k[q] * 2654435761u) >> (32 - BITS);
        int pr = 0;
        for (; pr < kCombProbes; ++pr) {
          const unsigned long long old = atomicCAS(&T[h], kEmpty, kx);
          if (old == kEmpty) break;
          if ((uint32_t)(old >> 32) == k[q]) {
            atomicAdd(&T[h], (unsigned long long)v[q]);
            break;
          }
#if LV_DH_CONTRACT
          h = (h + probe_step((int32_t)k[q])) & (SLOTS - 1);
#else
          h = (h + 1) & (SLOTS - 1);
#endif
        }
        pass[q] = pr == kCombProbes;
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {  // pass-throughs: warp-aggregated global append
        const unsigned mk = __ballot_sync(kFull, pass[q]);
        if (!mk) continue;
        unsigned long long b = 0;
        if (lane == __ffs(mk) - 1) b = atomicAdd(ocount, (unsigned long long)__popc(mk));
        b = __shfl_sync(kFull, b, __ffs(mk) - 1);
        if (pass[q]) {
          const unsigned long long o = b + __popc(mk & ((1u << lane) - 1u));
          okeys[o] = k[q];
          ovals[o] = v[q];
        }
      }
    }
    __syncthreads();
    // emit the distinct pairs: per-warp counts -> one global atomic per CTA
    constexpr int kPer = SLOTS / THREADS;  // slots per thread (contiguous per warp)
    const int s0 = wid * 32 * kPer;
    unsigned mine = 0;
    for (int u = 0; u < kPer; ++u) mine += T[s0 + u * 32 + lane] != kEmpty;
    unsigned wsum = mine;
    for (int o = 16; o >= 1; o >>= 1) wsum += __shfl_xor_sync(kFull, wsum, o);
    if (lane == 0) wcnt[wid] = wsum;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned tot = 0;
      for (int w = 0; w < THREADS / 32; ++w) {
        const unsigned c = wcnt[w];
        wcnt[w] = tot;
        tot += c;
      }
      sh_base = tot ? atomicAdd(ocount, (unsigned long long)tot) : 0ull;
    }
    __syncthreads();
    unsigned long long o = sh_base + wcnt[wid];
    for (int u = 0; u < kPer; ++u) {
      const int t = s0 + u * 32 + lane;
      const unsigned long long x = T[t];
      const bool has = x != kEmpty;
      const unsigned mk = __ballot_sync(kFull, has);
      if (has) {
        const unsigned long long oo = o + __popc(mk & ((1u << lane) - 1u));
        okeys[oo] = (uint32_t)(x >> 32);
        ovals[oo] = (uint32_t)x;
        T[t] = kEmpty;
      }
      o += __popc(mk);
    }
    __syncthreads();
  }
}

// Tiled key build: tile plan btr gives the first big segment of every
// kBigTile-entry tile; the tile's segment offsets are staged in smem.
constexpr int kBigTile = 8192;
constexpr int kBigTileSegs = 256;
template <typename K>
__global__ void __launch_bounds__(256) k_big_keys_t(const int32_t* __restrict__ rows, int64_t nbig,
                                                    const int64_t* __restrict__ sstart,
                                                    const int64_t* __restrict__ boff, const int64_t* __restrict__ btr,
                                                    int64_t m, const int32_t* __restrict__ gc,
                                                    const uint32_t* __restrict__ gw, int nb,
                                                    K* __restrict__ keys, uint32_t* __restrict__ vals,
                                                    int wbits = 0) {
  __shared__ int64_t sh_b[kBigTileSegs + 1];
  __shared__ int64_t sh_src[kBigTileSegs];
  const int64_t ntiles = (m + kBigTile - 1) / kBigTile;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t t0 = tile * kBigTile, t1 = min(m, t0 + kBigTile);
    const int64_t k0 = btr[tile], k1 = btr[tile + 1];
    const int ns = (k1 - k0 + 1 <= kBigTileSegs) ? (int)(k1 - k0 + 1) : -1;
    __syncthreads();
    for (int r = threadIdx.x; r < ns; r += blockDim.x) {
      sh_b[r] = boff[k0 + r];
      sh_src[r] = sstart[rows[k0 + r]];
    }
    __syncthreads();
    for (int64_t t = t0 + threadIdx.x; t < t1; t += blockDim.x) {
      int64_t k, src;
      if (ns > 0) {
        int lo = 0, hi = ns - 1;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (sh_b[mid] <= t) lo = mid; else hi = mid - 1;
        }
        k = k0 + lo;
        src = sh_src[lo] + (t - sh_b[lo]);
      } else {
        int64_t lo = k0, hi = min(k1, nbig - 1);
        while (lo < hi) {
          const int64_t mid = (lo + hi + 1) >> 1;
          if (boff[mid] <= t) lo = mid; else hi = mid - 1;
        }
        k = lo;
        src = sstart[rows[lo]] + (t - boff[lo]);
      }
      const K key = (nb < 0) ? (K)(uint32_t)__ldcs(&gc[src]) : (((K)k << nb) | (K)(uint32_t)__ldcs(&gc[src]));
      const uint32_t wv = gw ? __ldcs(&gw[src]) : 1u;
      if (wbits > 0) keys[t] = (key << wbits) | (K)wv;  // weight in the low bits: keys-only sort
      else {
        keys[t] = key;
        vals[t] = wv;
      }
    }
  }
}

// Step 4d (default for big segments whose keys do not fit the 32-bit combiner):
// mergeCommunity by label partitions instead of a sort.  Big segment k of
// length L_k is split into P_k = ceil(L_k / kBigPE) partitions by part_of(neighbour,
// P_k): every copy of a neighbour lands in the same partition, so merging each
// partition on its own gives exactly the merged row.  Histogram and scatter run
// edge-parallel over the big entries (the tile plan of k_big_keys_t); the 32 entries
// of a warp fall into few partitions (P_k is small for most big segments), so one
// global atomic per warp and partition run.  Then one CTA per partition folds its
// entries in a shared-memory table and appends the distinct (neighbour, sum) pairs to
// the segment's output range from a claim list (no table scan).  Expected distinct
// neighbours per partition <= kBigPE in a table of 2 * kBigPE slots; a table that
// fills up raises *overflow and the level redoes its big segments with the sort path
// (deterministic either way).
#ifndef LV_BIGPE  // compile-time A/B (tools/ab_build.py --define)
#define LV_BIGPE 4096
#endif
constexpr int kBigPE = LV_BIGPE;
constexpr int kBigPSlots = 2 * LV_BIGPE;

__global__ void k_bigp_sizes(const int32_t* __restrict__ rows, int64_t nbig, const int64_t* __restrict__ sstart,
                             int64_t* len, int64_t* nparts) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k <= nbig; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t l = (k < nbig) ? sstart[rows[k] + 1] - sstart[rows[k]] : 0;
    len[k] = l;
    nparts[k] = (l + kBigPE - 1) / kBigPE;
  }
}

template <bool SCATTER>
__global__ void __launch_bounds__(256) k_bigp_pass(const int32_t* __restrict__ rows, int64_t nbig,
                                                   const int64_t* __restrict__ sstart,
                                                   const int64_t* __restrict__ boff, const int64_t* __restrict__ btr,
                                                   int64_t m, const int32_t* __restrict__ gc,
                                                   const uint32_t* __restrict__ gw, const int64_t* __restrict__ pbase,
                                                   unsigned long long* __restrict__ pcnt, int32_t* __restrict__ pc,
                                                   uint32_t* __restrict__ pw) {
  __shared__ int64_t sh_b[kBigTileSegs + 1];
  __shared__ int64_t sh_src[kBigTileSegs];
  __shared__ int64_t sh_pb[kBigTileSegs + 1];
  const int lane = threadIdx.x & 31;
  const int64_t ntiles = (m + kBigTile - 1) / kBigTile;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t t0 = tile * kBigTile, t1 = min(m, t0 + kBigTile);
    const int64_t k0 = btr[tile], k1 = btr[tile + 1];
    const int ns = (k1 - k0 + 1 <= kBigTileSegs) ? (int)(k1 - k0 + 1) : -1;
    __syncthreads();
    for (int r = threadIdx.x; r < ns; r += blockDim.x) {
      sh_b[r] = boff[k0 + r];
      sh_src[r] = sstart[rows[k0 + r]];
      sh_pb[r] = pbase[k0 + r];
    }
    if (ns > 0 && threadIdx.x == 0) sh_pb[ns] = pbase[min(k0 + ns, nbig)];
    __syncthreads();
    for (int64_t tb = t0 + threadIdx.x - lane; tb < t1; tb += blockDim.x) {  // warp-uniform trips
      const int64_t t = tb + lane;
      const bool active = t < t1;
      uint32_t gb = 0xFFFFFFFFu;
      int32_t c = 0;
      uint32_t x = 1u;
      if (active) {
        int64_t src, p0, p1;
        if (ns > 0) {
          int lo = 0, hi = ns - 1;
          while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (sh_b[mid] <= t) lo = mid; else hi = mid - 1;
          }
          src = sh_src[lo] + (t - sh_b[lo]);
          p0 = sh_pb[lo];
          p1 = sh_pb[lo + 1];
        } else {
          int64_t lo = k0, hi = min(k1, nbig - 1);
          while (lo < hi) {
            const int64_t mid = (lo + hi + 1) >> 1;
            if (boff[mid] <= t) lo = mid; else hi = mid - 1;
          }
          src = sstart[rows[lo]] + (t - boff[lo]);
          p0 = pbase[lo];
          p1 = pbase[lo + 1];
        }
        c = __ldcs(&gc[src]);
        if (SCATTER && gw) x = __ldcs(&gw[src]);
        gb = (uint32_t)p0 + part_of(c, (uint32_t)(p1 - p0));
      }
      const unsigned mm = __match_any_sync(kFull, gb);
      const int leader = __ffs(mm) - 1;
      if (!SCATTER) {
        if (active && lane == leader) atomicAdd(&pcnt[gb], (unsigned long long)__popc(mm));
      } else {
        unsigned long long b = 0;
        if (active && lane == leader) b = atomicAdd(&pcnt[gb], (unsigned long long)__popc(mm));
        b = __shfl_sync(kFull, b, leader);
        if (active) {
          const unsigned long long dst = b + __popc(mm & ((1u << lane) - 1u));
          __stcs(&pc[dst], c);
          if (gw) __stcs(&pw[dst], x);
        }
      }
    }
  }
}

// One CTA per partition (persistent): fold, then append the distinct pairs.
__global__ void __launch_bounds__(1024) k_bigp_merge(const int64_t* __restrict__ poff, int64_t nparts,
                                                     const int64_t* __restrict__ pbase, int64_t nbig,
                                                     const int32_t* __restrict__ rows,
                                                     const int64_t* __restrict__ sstart,
                                                     const int32_t* __restrict__ pc, const uint32_t* __restrict__ pw,
                                                     int32_t* oc, uint32_t* ow, int64_t* cnt,
                                                     unsigned long long* overflow, uint32_t capmax) {
  extern __shared__ unsigned long long T[];                            // kBigPSlots slots
  uint16_t* claim = reinterpret_cast<uint16_t*>(T + kBigPSlots);      // claimed slots, in claim order
  __shared__ unsigned ncl;
  __shared__ long long sh_base;
  __shared__ int32_t sh_r;
  const int lane = threadIdx.x & 31;
  for (int t = threadIdx.x; t < kBigPSlots; t += blockDim.x) T[t] = kEmpty;
  for (int64_t g = blockIdx.x; g < nparts; g += gridDim.x) {
    const int64_t q0 = poff[g], q1 = poff[g + 1];
    const int64_t len = q1 - q0;
    if (len == 0) continue;  // uniform across the CTA
    uint32_t cap = 64;
    while (cap < capmax && (int64_t)cap < 2 * len) cap <<= 1;
    if (threadIdx.x == 0) {
      int64_t lo = 0, hi = nbig - 1;  // segment of partition g: last k with pbase[k] <= g
      while (lo < hi) {
        const int64_t mid = (lo + hi + 1) >> 1;
        if (pbase[mid] <= g) lo = mid; else hi = mid - 1;
      }
      sh_r = rows[lo];
      ncl = 0;
    }
    __syncthreads();
    for (int64_t tb = q0 + threadIdx.x - lane; tb < q1; tb += 4 * (int64_t)blockDim.x) {  // warp-uniform trips
      int32_t cc[4];
      uint32_t xx[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t t = tb + lane + (int64_t)u * blockDim.x;
        const bool has = t < q1;
        cc[u] = has ? __ldcs(&pc[t]) : (int32_t)(0x80000000u | (unsigned)lane);
        xx[u] = has ? (pw ? __ldcs(&pw[t]) : 1u) : 0u;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const bool has = cc[u] >= 0;
        unsigned mm = 1u << lane;
        uint32_t x = xx[u];
        if (__any_sync(kFull, cc[u] == __shfl_xor_sync(kFull, cc[u], 1))) {  // adaptive merge of repeats
          mm = __match_any_sync(kFull, cc[u]);
          x = __reduce_add_sync(mm, xx[u]);
        }
        uint32_t h = 0xFFFFFFFFu;
        if (has && lane == __ffs(mm) - 1) {
          const unsigned long long key = ((unsigned long long)(uint32_t)cc[u]) << 32;
          h = hash_slot(cc[u], cap);
          for (uint32_t probes = 0;; ++probes) {
            if (probes >= cap) {
              atomicExch(overflow, 1ull);
              h = 0xFFFFFFFFu;
              break;
            }
            const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
            if (old == kEmpty) break;  // claimed: h goes on the claim list
            if ((old >> 32) == (unsigned long long)(uint32_t)cc[u]) {
              atomicAdd(&T[h], (unsigned long long)x);
              h = 0xFFFFFFFFu;
              break;
            }
#if LV_DH_CONTRACT
            h = probe_next(h, cap, probe_step(cc[u]));
#else
            h = (h + 1 == cap) ? 0 : h + 1;
#endif
          }
        }
        const unsigned cm = __ballot_sync(kFull, h != 0xFFFFFFFFu);
        if (cm) {
          unsigned b = 0;
          if (lane == __ffs(cm) - 1) b = atomicAdd(&ncl, (unsigned)__popc(cm));
          b = __shfl_sync(kFull, b, __ffs(cm) - 1);
          if (h != 0xFFFFFFFFu) claim[b + __popc(cm & ((1u << lane) - 1u))] = (uint16_t)h;
        }
      }
    }
    __syncthreads();
    const unsigned nd = ncl;
    if (threadIdx.x == 0) sh_base = (long long)atomicAdd((unsigned long long*)&cnt[sh_r], (unsigned long long)nd);
    __syncthreads();
    const int64_t b = sstart[sh_r] + sh_base;
    for (unsigned i = threadIdx.x; i < nd; i += blockDim.x) {
      const uint32_t s = claim[i];
      const unsigned long long x = T[s];
      T[s] = kEmpty;
      oc[b + i] = (int32_t)(x >> 32);
      ow[b + i] = (uint32_t)x;
    }
    __syncthreads();
  }
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
    // warp spans of 128 entries (lane + 32 u), 4 in flight per lane: one binary search
    // per lane, then a forward walk over the tile's rows
    const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int64_t span = q0 + (int64_t)wl * 128; span < q1; span += (int64_t)nw * 128) {
      int32_t cc[4];
      uint32_t ww[4];
      int lo = 0;
      if (nr > 0 && span + lane < q1) {
        int hi = nr - 1;
        const int64_t q = span + lane;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (sh_r[mid] <= q) lo = mid; else hi = mid - 1;
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t q = span + lane + 32 * u;
        if (q >= q1) continue;
        int64_t src;
        if (nr > 0) {
          while (lo + 1 < nr && sh_r[lo + 1] <= q) ++lo;
          src = sh_s[lo] + (q - sh_r[lo]);
        } else {
          int64_t a = 0, b = np - 1;
          while (a < b) {
            const int64_t mid = (a + b + 1) >> 1;
            if (rowptr_out[mid] <= q) a = mid; else b = mid - 1;
          }
          src = sstart[a] + (q - rowptr_out[a]);
        }
        cc[u] = __ldcs(&oc[src]);
        ww[u] = __ldcs(&ow[src]);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t q = span + lane + 32 * u;
        if (q >= q1) continue;
        col[q] = cc[u];
        w[q] = ww[u];
      }
    }
    __syncthreads();
  }
}

// LV_BIG_SORT=1: big segments always by the radix-sort path (the partition path's
// fallback; parity-tested as an alternative path)
bool big_sort_forced() {
  static const bool f = [] {
    const char* e = getenv("LV_BIG_SORT");
    return e && e[0] == '1';
  }();
  return f;
}

// LV_BIGP_SLOTS=s (power of 2 < kBigPSlots): smaller partition tables, so that tests
// can drive the overflow -> sort fallback
uint32_t bigp_capmax() {
  static const uint32_t c = [] {
    const char* e = getenv("LV_BIGP_SLOTS");
    const long v = e ? atol(e) : 0;
    return (v >= 64 && v < kBigPSlots && (v & (v - 1)) == 0) ? (uint32_t)v : (uint32_t)kBigPSlots;
  }();
  return c;
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
  // sharded contraction: this rank merges the new vertices [c_lo, c_hi) only (the
  // steps before are O(n) and replicated); the rows are all-gathered at the end
  int64_t c_lo = 0, c_hi = np;
  std::vector<int64_t> cuts;
  if (h.dist && h.dist->world > 1) {
    const int world = h.dist->world;
    int64_t* dcut = nullptr;
    LV_TRY(dalloc(&dcut, world + 1, s));
    k_seg_split<<<1, 1024, 0, s>>>(rfirst, gpos, np, nnz, world, dcut);
    LV_LAUNCHED();
    cuts.resize(world + 1);
    LV_CUDA(cudaMemcpyAsync(cuts.data(), dcut, 8 * (world + 1), cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    dfree(dcut, s);
    for (int r = 1; r <= world; ++r) cuts[r] = std::max(cuts[r], cuts[r - 1]);
    c_lo = cuts[h.dist->rank];
    c_hi = cuts[h.dist->rank + 1];
  }
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
  {  // source order
    int64_t* dbase = nullptr;
    LV_TRY(dalloc(&dbase, n, s));
    k_dest_base<<<grid_for(n, 256), 256, 0, s>>>(vorder, gpos, n, dbase);
    LV_LAUNCHED();
    const int64_t* tr = nullptr;
    LV_TRY(tile_starts(h, L.rowptr, 0, n, 0, nnz, kSTile, &tr));
    const unsigned g = grid_for((nnz + kSTile - 1) / kSTile, 1, 148 * 8);
    if (cuts.empty())
      k_scatter_copy<false><<<g, 256, 0, s>>>(L.rowptr, n, L.col, L.w, d_map, dbase, nnz, tr, gc, gw, 0, 0);
    else
      k_scatter_copy<true><<<g, 256, 0, s>>>(L.rowptr, n, L.col, L.w, d_map, dbase, nnz, tr, gc, gw, (int32_t)c_lo,
                                             (int32_t)c_hi);
    LV_LAUNCHED();
    dfree(dbase, s);
  }
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
  LV_TRY(dalloc(&hist, kSegClasses, s));
  LV_CUDA(cudaMemsetAsync(hist, 0, 8 * kSegClasses, s));
  k_seg_bounds<<<grid_for(np, 256), 256, 0, s>>>(rfirst, gpos, np, n, sstart, scls, rid, hist, c_lo, c_hi);
  LV_LAUNCHED();
  unsigned long long hh[kSegClasses];
  LV_CUDA(cudaMemcpyAsync(hh, hist, 8 * kSegClasses, cudaMemcpyDeviceToHost, s));
  LV_CUDA(cudaMemcpyAsync(sstart + np, gpos + n, 8, cudaMemcpyDeviceToDevice, s));
  send_ = sstart + 1;
  dfree(rfirst, s);
  dfree(gpos, s);
  {
    size_t tb = 0;
    const int64_t nown = c_hi - c_lo;  // own segments only (all of them on one GPU)
    LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, scls + c_lo, scls2, rid + c_lo, rows, nown, 0, 3, s));
    void* tmp = nullptr;
    LV_TRY(dmalloc(&tmp, tb, s));
    LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, scls + c_lo, scls2, rid + c_lo, rows, nown, 0, 3, s));  // kSegClasses classes
    LV_CUB();
    dfree(tmp, s);
  }
  LV_CUDA(cudaStreamSynchronize(s));
  dfree(hist, s);
  const int64_t nsmall = (int64_t)hh[0], nwarp = (int64_t)(hh[1] + hh[2]),
                nmid = (int64_t)(hh[3] + hh[4] + hh[5] + hh[6]), nbig = (int64_t)hh[7];
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
  // small / warp / mid merges on the side stream, concurrent with the big-segment
  // waves on the main stream (independent segments, disjoint outputs)
  cudaStream_t ms = tr.on ? s : h.side;
  if (ms != s) {
    LV_CUDA(cudaEventRecord(h.ev_fork, s));
    LV_CUDA(cudaStreamWaitEvent(ms, h.ev_fork, 0));
  }
  if (nsmall > 0) {
    k_merge_small<<<grid_for(nsmall, 8, 148 * 16), 256, 0, ms>>>(rows, nsmall, sstart, send_, gc, gw, oc, ow, cnt);
    LV_LAUNCHED();
  }
  tr.mark(s, "merge-small");
  if (hh[1] > 0) {
    k_merge_warp<256><<<grid_for((int64_t)hh[1], 4, 148 * 16), 128, 0, ms>>>(rows + nsmall, (int64_t)hh[1], sstart,
                                                                              send_, gc, gw, oc, ow, cnt);
    LV_LAUNCHED();
  }
  if (hh[2] > 0) {
    k_merge_warp<kWarpSlots><<<grid_for((int64_t)hh[2], 4, 148 * 12), 128, 0, ms>>>(
        rows + nsmall + (int64_t)hh[1], (int64_t)hh[2], sstart, send_, gc, gw, oc, ow, cnt);
    LV_LAUNCHED();
  }
  tr.mark(s, "merge-warp");
  if (nmid > 0) {
    static bool attr = false;
    static int resident[4] = {0, 0, 0, 0};
    if (!attr) {
      LV_CUDA(cudaFuncSetAttribute(k_merge_mid, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * kMidSlots));
      attr = true;
    }
    int64_t off = nsmall + nwarp;
    for (int t = 0; t < 4; ++t) {  // CTA tiers, tables sized to the tier (more segments in flight per SM)
      const int64_t cntt = (int64_t)hh[3 + t];
      if (cntt > 0) {
        const size_t sm = 8 * (size_t)kMidTierCap[t];
        if (resident[t] == 0) {
          int nb = 0;
          LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_merge_mid, kMidTierThr[t], sm));
          resident[t] = std::max(nb, 1);
        }
        k_merge_mid<<<grid_for(cntt, 1, 148 * resident[t]), kMidTierThr[t], sm, ms>>>(
            rows + off, cntt, sstart, send_, gc, gw, oc, ow, cnt, kMidTierCap[t]);
        LV_LAUNCHED();
      }
      off += cntt;
    }
  }
  tr.mark(s, "merge-mid");
  if (nbig > 0) {  // one radix sort of 64-bit (segment rank, neighbour) keys + reduce-by-key
    const int32_t* brows = rows + nsmall + nwarp + nmid;
    // offsets of the big segments in the key array: lengths + scan on the device
    int64_t *dboff = nullptr, *dpb = nullptr;
    LV_TRY(dalloc(&dboff, nbig + 1, s));
    LV_TRY(dalloc(&dpb, nbig + 1, s));
    k_bigp_sizes<<<grid_for(nbig + 1, 256), 256, 0, s>>>(brows, nbig, sstart, dboff, dpb);
    LV_LAUNCHED();
    LV_TRY(cub_scan_excl(s, dboff, dboff, nbig + 1));
    LV_TRY(cub_scan_excl(s, dpb, dpb, nbig + 1));
    int64_t mp[2] = {0, 0};
    LV_CUDA(cudaMemcpyAsync(&mp[0], dboff + nbig, 8, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaMemcpyAsync(&mp[1], dpb + nbig, 8, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    int64_t m = mp[0];
    const int64_t nparts = mp[1];
    if (tr.on)
      fprintf(stderr, "[lv]    contract segments: small %lld warp %lld mid %lld big %lld (big entries %lld of %lld)\n",
              (long long)nsmall, (long long)nwarp, (long long)nmid, (long long)nbig, (long long)m, (long long)nnz);
    int kb = 1;
    while (kb < 40 && (1ll << kb) < nbig) ++kb;
    const bool key_ok = nb + kb <= 32 && (((uint64_t)(nbig - 1) << nb) | (uint64_t)(np - 1)) < 0xFFFFFFFFull;
    const bool comb = key_ok && m >= 64 * np;
    bool sorted_path = comb || big_sort_forced();
    if (!sorted_path) {  // label partitions (k_bigp_*)
      int32_t* pc = nullptr;
      uint32_t* pw = nullptr;
      {
        void* p0 = nullptr;
        LV_TRY(scratch_get(h, SC_K1, 8 * (size_t)m, &p0));  // the level's stage / key buffers are dead here
        pc = static_cast<int32_t*>(p0);
        pw = weighted ? reinterpret_cast<uint32_t*>(pc + m) : nullptr;
      }
      unsigned long long* pcnt = nullptr;
      LV_TRY(dalloc(&pcnt, nparts + 1, s));
      LV_CUDA(cudaMemsetAsync(pcnt, 0, 8 * (nparts + 1), s));
      const int64_t* btr = nullptr;
      LV_TRY(tile_starts(h, dboff, 0, nbig, 0, m, kBigTile, &btr));
      const unsigned g = grid_for((m + kBigTile - 1) / kBigTile, 1, 148 * 8);
      k_bigp_pass<false><<<g, 256, 0, s>>>(brows, nbig, sstart, dboff, btr, m, gc, gw, dpb, pcnt, nullptr, nullptr);
      LV_LAUNCHED();
      int64_t* poff = reinterpret_cast<int64_t*>(pcnt);
      LV_TRY(cub_scan_excl(s, poff, poff, nparts + 1));
      unsigned long long* pcur = nullptr;
      LV_TRY(dalloc(&pcur, nparts + 1, s));
      LV_CUDA(cudaMemcpyAsync(pcur, poff, 8 * (nparts + 1), cudaMemcpyDeviceToDevice, s));
      k_bigp_pass<true><<<g, 256, 0, s>>>(brows, nbig, sstart, dboff, btr, m, gc, gw, dpb, pcur, pc, pw);
      LV_LAUNCHED();
      dfree(pcur, s);
      tr.mark(s, "big-part");
      static int resident = 0;
      if (resident == 0) {
        LV_CUDA(cudaFuncSetAttribute(k_bigp_merge, cudaFuncAttributeMaxDynamicSharedMemorySize, 10 * kBigPSlots));
        int nbk = 0;
        LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nbk, k_bigp_merge, 1024, 10 * kBigPSlots));
        resident = std::max(nbk, 1);
      }
      unsigned long long* ovf = &h.ctl->overflow;
      k_bigp_merge<<<grid_for(nparts, 1, 148 * resident), 1024, 10 * kBigPSlots, s>>>(
          poff, nparts, dpb, nbig, brows, sstart, pc, pw, oc, ow, cnt, ovf, bigp_capmax());
      LV_LAUNCHED();
      unsigned long long o = 0;
      LV_CUDA(cudaMemcpyAsync(&o, ovf, 8, cudaMemcpyDeviceToHost, s));
      LV_CUDA(cudaStreamSynchronize(s));
      dfree(pcnt, s);
      tr.mark(s, "big-merge");
      if (o) {  // a partition table filled up: redo the big segments with the sort path
        LV_CUDA(cudaMemsetAsync(ovf, 0, 8, s));
        if (tr.on) fprintf(stderr, "[lv]    contract big partitions overflowed: sort path\n");
        sorted_path = true;
      }
    }
    if (!sorted_path) {
      dfree(dboff, s);
    } else if (nb + kb <= 32) {  // 32-bit keys: 8 instead of 12 bytes per element and pass
      uint32_t *k0 = nullptr, *k1 = nullptr, *v0 = nullptr, *v1 = nullptr;
      {
        void* p0 = nullptr;
        LV_TRY(scratch_get(h, SC_STAGE, 8 * (size_t)m, &p0));  // the level's stage is dead during contraction
        k0 = static_cast<uint32_t*>(p0);
        k1 = k0 + m;
        LV_TRY(scratch_get(h, SC_K1, 8 * (size_t)m, &p0));
        v0 = static_cast<uint32_t*>(p0);
        v1 = v0 + m;
      }
      // combiner: worthwhile when the big segments repeat neighbours (few new
      // vertices per big entry); 0xFFFFFFFF must not be a real key (table marker, key_ok)
      {
        const int64_t* btr = nullptr;
        LV_TRY(tile_starts(h, dboff, 0, nbig, 0, m, kBigTile, &btr));
        k_big_keys_t<uint32_t><<<grid_for((m + kBigTile - 1) / kBigTile, 1, 148 * 8), 256, 0, s>>>(
            brows, nbig, sstart, dboff, btr, m, gc, gw, nb, k0, v0);
        LV_LAUNCHED();
      }
      tr.mark(s, "big-keys");
      cub::DoubleBuffer<uint32_t> kq(k0, k1), vq(v0, v1);
      if (comb) {
        static bool cattr = false;
        if (!cattr) {
          LV_CUDA(cudaFuncSetAttribute(k_big_combine<kCombSlots, 14, kCombChunk, 1024>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * kCombSlots));
          cattr = true;
        }
        unsigned long long* dcnt = reinterpret_cast<unsigned long long*>(&h.ctl->bad);
        LV_CUDA(cudaMemsetAsync(dcnt, 0, 8, s));
        k_big_combine<kCombSlots, 14, kCombChunk, 1024><<<grid_for((m + kCombChunk - 1) / kCombChunk, 1, 148), 1024,
                                                          8 * kCombSlots, s>>>(k0, v0, m, k1, v1, dcnt);
        LV_LAUNCHED();
        unsigned long long m2 = 0;
        LV_CUDA(cudaMemcpyAsync(&m2, dcnt, 8, cudaMemcpyDeviceToHost, s));
        LV_CUDA(cudaStreamSynchronize(s));
        if (tr.on) fprintf(stderr, "[lv]    contract combine: %lld -> %llu entries\n", (long long)m, m2);
        m = (int64_t)m2;
        kq = cub::DoubleBuffer<uint32_t>(k1, k0);
        vq = cub::DoubleBuffer<uint32_t>(v1, v0);
        tr.mark(s, "big-combine");
      }
      size_t tb = 0;
      LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, kq, vq, m, 0, nb + kb, s));
      void* tmp = nullptr;
      LV_TRY(dmalloc(&tmp, tb, s));
      LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, kq, vq, m, 0, nb + kb, s));
      LV_CUB();
      dfree(tmp, s);
      tr.mark(s, "big-sort");
      int64_t* dnum = reinterpret_cast<int64_t*>(&h.ctl->bad);
      tb = 0;
      LV_CUDA(cub::DeviceReduce::ReduceByKey(nullptr, tb, kq.Current(), kq.Alternate(), vq.Current(), vq.Alternate(),
                                             dnum, cub::Sum(), m, s));
      LV_TRY(dmalloc(&tmp, tb, s));
      LV_CUDA(cub::DeviceReduce::ReduceByKey(tmp, tb, kq.Current(), kq.Alternate(), vq.Current(), vq.Alternate(),
                                             dnum, cub::Sum(), m, s));
      LV_CUB();
      dfree(tmp, s);
      tr.mark(s, "big-reduce");
      k_big_place32<<<grid_for(m, 256, 148 * 16), 256, 0, s>>>(kq.Alternate(), vq.Alternate(), dnum, nb, brows, sstart,
                                                               oc, ow, cnt);
      LV_LAUNCHED();
      dfree(dboff, s);
      LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, s));
    } else {
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
      {
        const int64_t* btr = nullptr;
        LV_TRY(tile_starts(h, dboff, 0, nbig, 0, m, kBigTile, &btr));
        k_big_keys_t<<<grid_for((m + kBigTile - 1) / kBigTile, 1, 148 * 8), 256, 0, s>>>(brows, nbig, sstart, dboff, btr,
                                                                                        m, gc, gw, nb, k0, v0);
        LV_LAUNCHED();
      }
      tr.mark(s, "big-keys");
      cub::DoubleBuffer<unsigned long long> kbuf(k0, k1);
      cub::DoubleBuffer<uint32_t> vbuf(v0, v1);
      size_t tb = 0;
      LV_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, kbuf, vbuf, m, 0, nb + kb, s));
      void* tmp = nullptr;
      LV_TRY(dmalloc(&tmp, tb, s));
      LV_CUDA(cub::DeviceRadixSort::SortPairs(tmp, tb, kbuf, vbuf, m, 0, nb + kb, s));
      LV_CUB();
      dfree(tmp, s);
      tr.mark(s, "big-sort");
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
      tr.mark(s, "big-reduce");
      int64_t* first_run = nullptr;
      LV_TRY(dalloc(&first_run, nbig, s));
      k_big_first<<<grid_for(nruns, 256), 256, 0, s>>>(kbuf.Alternate(), nruns, nb, first_run);
      LV_LAUNCHED();
      k_big_place<<<grid_for(nruns, 256), 256, 0, s>>>(kbuf.Alternate(), vbuf.Alternate(), nruns, nb, brows, sstart,
                                                        first_run, oc, ow, cnt);
      LV_LAUNCHED();
      dfree(first_run, s);
      dfree(dboff, s);
      LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, s));
    }
    tr.mark(s, "big-place");
    dfree(dpb, s);
  }
  if (ms != s) {
    LV_CUDA(cudaEventRecord(h.ev_join, ms));
    LV_CUDA(cudaStreamWaitEvent(s, h.ev_join, 0));
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
  if (cuts.empty()) {
    out.nnz = m2;
    LV_TRY(lvl(LA_COL, 4 * (size_t)std::max<int64_t>(m2, 1), (void**)&out.col));
    LV_TRY(lvl(LA_W, 4 * (size_t)std::max<int64_t>(m2, 1), (void**)&out.w));
    if (m2 > 0) {
      const int64_t* tr = nullptr;
      LV_TRY(tile_starts(h, out.rowptr, 0, np, 0, m2, kCTile, &tr));
      k_compact<<<grid_for((m2 + kCTile - 1) / kCTile, 1, 148 * 8), 256, 0, s>>>(sstart, out.rowptr, np, oc, ow, tr,
                                                                                  out.col, out.w);
      LV_LAUNCHED();
    }
  } else {
    // sharded: this rank's rows [c_lo, c_hi) hold m2 entries (the others' counts are 0 here);
    // compact them, then all-gather the row lengths and the rows into the replicated CSR'
    const int world = h.dist->world;
    int32_t* col_own = nullptr;
    uint32_t* w_own = nullptr;
    LV_TRY(dalloc(&col_own, std::max<int64_t>(m2, 1), s));
    LV_TRY(dalloc(&w_own, std::max<int64_t>(m2, 1), s));
    if (m2 > 0) {
      const int64_t* tr = nullptr;
      LV_TRY(tile_starts(h, out.rowptr, 0, np, 0, m2, kCTile, &tr));
      k_compact<<<grid_for((m2 + kCTile - 1) / kCTile, 1, 148 * 8), 256, 0, s>>>(sstart, out.rowptr, np, oc, ow, tr,
                                                                                  col_own, w_own);
      LV_LAUNCHED();
    }
    std::vector<int64_t> nrow(world), drow(world);
    for (int r = 0; r < world; ++r) {
      nrow[r] = cuts[r + 1] - cuts[r];
      drow[r] = cuts[r];
    }
    int64_t* cnt_all = nullptr;
    LV_TRY(dalloc(&cnt_all, np + 1, s));
    LV_CUDA(cudaMemsetAsync(cnt_all + np, 0, 8, s));
    LV_TRY(dist_allgatherv(h, cnt + c_lo, cnt_all, nrow, drow, 8));
    LV_TRY(cub_scan_excl(s, cnt_all, out.rowptr, np + 1));
    std::vector<int64_t> rp_cut(world + 1);
    for (int r = 0; r <= world; ++r)
      LV_CUDA(cudaMemcpyAsync(&rp_cut[r], out.rowptr + cuts[r], 8, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    const int64_t total = rp_cut[world];
    out.nnz = total;
    LV_TRY(lvl(LA_COL, 4 * (size_t)std::max<int64_t>(total, 1), (void**)&out.col));
    LV_TRY(lvl(LA_W, 4 * (size_t)std::max<int64_t>(total, 1), (void**)&out.w));
    std::vector<int64_t> ne(world), de(world);
    for (int r = 0; r < world; ++r) {
      ne[r] = rp_cut[r + 1] - rp_cut[r];
      de[r] = rp_cut[r];
    }
    LV_TRY(dist_allgatherv(h, col_own, out.col, ne, de, 4));
    LV_TRY(dist_allgatherv(h, w_own, out.w, ne, de, 4));
    dfree(cnt_all, s);
    dfree(col_own, s);
    dfree(w_own, s);
  }
  LV_CUDA(cudaGetLastError());
  dfree(cnt, s);
  dfree(sstart, s);
  tr.mark(s, "compact");
  return LOUVAIN_OK;
}

}  // namespace lv
