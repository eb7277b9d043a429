// lv_device.cuh -- device helpers shared by the sweep and level kernels.
#pragma once
#include <stdint.h>

namespace lv {

constexpr unsigned kFull = 0xFFFFFFFFu;
constexpr unsigned long long kEmpty = ~0ull;  // slot label field 0xFFFFFFFF never a valid label

// A candidate move: gain score s = W*e - k*a (Eq. 2 integer form, R4), label c.
// Order: larger s first, then lower label.
struct Cand {
  long long s;
  int c;
};
__device__ __forceinline__ Cand cand_none() { return Cand{(long long)0x8000000000000000ull, 0x7FFFFFFF}; }
__device__ __forceinline__ bool better(long long s1, int c1, long long s2, int c2) {
  return s1 > s2 || (s1 == s2 && c1 < c2);
}

// Slot of label c in a table of `cap` slots (any cap >= 1): multiplicative hash.
__device__ __forceinline__ uint32_t hash_slot(int32_t c, uint32_t cap) {
  return (uint32_t)(((unsigned long long)((uint32_t)c * 2654435761u) * cap) >> 32);
}

// Open-addressing insert of (c, x) into 64-bit slots {label:32 | e:32}:
// one CAS claims an empty slot with the value already in it; a slot already
// holding c gets an atomic add on its low word (e <= W < 2^32, no carry).
// Exact per-label sums regardless of order (R25).
__device__ __forceinline__ void table_add(unsigned long long* T, uint32_t cap, int32_t c, uint32_t x) {
  const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
  uint32_t h = hash_slot(c, cap);
  for (;;) {
    unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
    if (old == kEmpty) return;
    if ((old >> 32) == (unsigned long long)(uint32_t)c) {
      atomicAdd(&T[h], (unsigned long long)x);
      return;
    }
    h = (h + 1 == cap) ? 0 : h + 1;
  }
}

// Sums x over the lanes holding the same key (all 32 lanes call it; idle lanes need keys of
// their own): m = the lane's group, the group's lowest lane gets the sum in x.  (The
// hardware serialises REDUX over the distinct group masks; a bounded loop of full-warp
// reductions measured slower: DESIGN 13.)
__device__ __forceinline__ void group_sum(uint32_t key, uint32_t& x, unsigned& m) {
  m = __match_any_sync(kFull, key);
  x = __reduce_add_sync(m, x);
}

// Probe sequence of the open-addressing tables: double hashing (an odd step from a multiplier
// independent of hash_slot's) on power-of-two tables -- no primary clusters, so the longest
// chain in a warp's divergent probe loop shortens -- linear otherwise.
__device__ __forceinline__ uint32_t probe_step(int32_t c) { return (((uint32_t)c * 0x85EBCA6Bu) >> 17) | 1u; }
__device__ __forceinline__ uint32_t probe_next(uint32_t h, uint32_t cap, uint32_t step) {
  return ((cap & (cap - 1)) == 0) ? ((h + step) & (cap - 1)) : ((h + 1 == cap) ? 0 : h + 1);
}
// Smallest power of two >= x (x >= 1), capped at lim (a power of two).
__device__ __forceinline__ uint32_t pow2_at_least(uint32_t x, uint32_t lim) {
  uint32_t p = 1;
  while (p < x && p < lim) p <<= 1;
  return p;
}

// Partition of label c among P label-partitioned tasks: fmix32 (independent of
// hash_slot's multiplier) scaled to [0, P).
__device__ __forceinline__ uint32_t part_of(int32_t c, uint32_t P) {
  uint32_t h = (uint32_t)c;  // fmix32 (independent of hash_slot's multiplier)
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return (uint32_t)(((unsigned long long)h * P) >> 32);
}

// Whole-warp version with the warp reduction unit (REDUX): max of the high word
// (signed), max of the low word among those lanes (unsigned) -- together the
// int64 max -- then the lowest label among the lanes holding it, and the
// sum.  3 + 1 single-instruction reductions instead of a 5-step butterfly of
// 64-bit shuffles and compares.  Every lane gets the result.
__device__ __forceinline__ void warp_reduce(long long& s, int& c, unsigned& eown) {
  const int hi = (int)((unsigned long long)s >> 32);
  const unsigned lo = (unsigned)(unsigned long long)s;
  const int mhi = __reduce_max_sync(kFull, hi);
  const unsigned mlo = __reduce_max_sync(kFull, hi == mhi ? lo : 0u);
  const long long ms = (long long)(((unsigned long long)(unsigned)mhi << 32) | mlo);
  const int mc = __reduce_min_sync(kFull, s == ms ? c : 0x7FFFFFFF);
  eown = __reduce_add_sync(kFull, eown);
  s = ms;
  c = mc;
}

// xor-butterfly reduction over aligned groups of G lanes: best candidate + sum.
template <int G>
__device__ __forceinline__ void group_reduce(long long& s, int& c, unsigned& eown) {
  if constexpr (G == 32) {
    warp_reduce(s, c, eown);
  } else {
#pragma unroll
    for (int off = G / 2; off >= 1; off >>= 1) {
      long long s2 = __shfl_xor_sync(kFull, s, off);
      int c2 = __shfl_xor_sync(kFull, c, off);
      unsigned e2 = __shfl_xor_sync(kFull, eown, off);
      if (better(s2, c2, s, c)) { s = s2; c = c2; }
      eown += e2;
    }
  }
}

// Block-wide version; result valid in thread 0.  `sh` needs 32 entries each.
__device__ __forceinline__ void block_reduce(long long& s, int& c, unsigned& eown, long long* sh_s, int* sh_c,
                                             unsigned* sh_e) {
  group_reduce<32>(s, c, eown);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  if (lane == 0) { sh_s[wid] = s; sh_c[wid] = c; sh_e[wid] = eown; }
  __syncthreads();
  if (wid == 0) {
    if (lane < nw) { s = sh_s[lane]; c = sh_c[lane]; eown = sh_e[lane]; }
    else { Cand z = cand_none(); s = z.s; c = z.c; eown = 0; }
    group_reduce<32>(s, c, eown);
  }
}

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) x += __shfl_xor_sync(kFull, x, off);
  return x;
}

// Largest u in [0, n] with rowptr[u] <= e (the source row of CSR entry e).
__device__ __forceinline__ int64_t row_of(const int64_t* rowptr, int64_t n, int64_t e) {
  int64_t lo = 0, hi = n;  // invariant rowptr[lo] <= e < rowptr[hi+1] ...
  while (lo < hi) {
    int64_t mid = (lo + hi + 1) >> 1;
    if (rowptr[mid] <= e) lo = mid; else hi = mid - 1;
  }
  return lo;
}

}  // namespace lv
