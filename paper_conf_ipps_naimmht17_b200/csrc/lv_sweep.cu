// lv_sweep.cu -- the modularity-optimisation sweep (computeMove, Alg. 2,
// PAPER.md P:214-236) for one degree bucket, B200 (sm_100a) kernels.
//
// Every vertex i of the bucket reads the bucket-start snapshot (C, a, size)
// and produces its target community (Alg. 1 l.6-7):
//   e_c    = sum of w_ij over j in N(i)\{i} with C[j] = c         (R3, R5)
//   s_c    = W*e_c - k_i*a_c                 for every c != C(i)  (Eq. 2, R4)
//   s_stay = W*e_own - k_i*(a_own - k_i)
//   best   = argmax s_c, ties -> lowest label                     (R7)
//   move iff s_best > s_stay (strictly, R6) and not vetoed by the
//   singleton rule (R8/R9).
// Moves are appended to a move log; commit is a separate kernel (lv_level.cu)
// because the whole bucket must decide before any C/a changes.
//
// Memory design (the sweep is bound by random gathers):
//  * col / w are streamed with evict-first loads (__ldcs) so they do not push
//    the gathered vertex records out of L2;
//  * a neighbour j is gathered as ONE 8-byte record ca[j] = {C[j], a[j]}; when
//    j represents its own community (C[j] == j, e.g. every vertex at the first
//    sweep of a level) a[C[j]] comes with it and the candidate's a_c needs no
//    second gather;
//  * edge loops are unrolled 4x so each thread has 4 independent gathers in flight.
//
// Kernel families (edge-level parallelism, redesigned for
// sm_100a; SURVEY 2.3 K1-K4 counterparts):
//   sweep_small<G>  deg <= 32: G = 4/8/16/32 lanes per vertex, one edge per
//                   lane, labels merged in registers with __match_any_sync +
//                   __reduce_add_sync (no shared memory).
//   sweep_warp<CAP> deg <= 340: a warp per vertex, per-warp smem hash table.
//   sweep_cta       deg < 12288: a CTA per vertex (persistent loop), smem table.
//   sweep_part      deg >= 12288: label-partitioned CTA tasks over the staged
//                   entries, pre-scattered into partition order.
//   hub_coop        deg > 50 M (more than kPartMaxP partitions): a cooperative
//                   kernel pipelines waves of hubs (insert chunks -> table scan
//                   chunks -> decision) across grid.sync() phases, the global
//                   tables living in a 2-segment ring small enough for L2.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <string>
#include <algorithm>
#include <cstdlib>

#include <cub/cub.cuh>
#include <thrust/iterator/counting_iterator.h>

#include "lv_device.cuh"
#include "lv_internal.cuh"

namespace cg = cooperative_groups;

namespace lv {
static bool trace_on();  // LV_TRACE=2 (per-class / per-step timing, diagnostics only)
namespace {

constexpr uint32_t kUnknownA = 0xFFFFFFFFu;  // a_c < W <= 3,037,000,499 < 2^32 - 1

struct SweepArgs {
  const int64_t* rowptr;
  const int32_t* col;
  const uint32_t* w;
  const uint32_t* k;
  const uint2* ca;
  const int32_t* size;
  long long W;
  int rule;
  int32_t* mv_v;
  int32_t* mv_new;
  unsigned long long* logn;
};

struct __align__(16) Partial {
  long long s;
  int c;
  unsigned eown;
};

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Warp-aggregated append to the move log.  Must be called by all 32 lanes.
__device__ __forceinline__ void log_moves(bool mv, int32_t v, int32_t t, const SweepArgs& A) {
  unsigned m = __ballot_sync(kFull, mv);
  if (m == 0) return;
  const int lane = threadIdx.x & 31;
  const int leader = __ffs(m) - 1;
  unsigned long long base = 0;
  if (lane == leader) base = atomicAdd(A.logn, (unsigned long long)__popc(m));
  base = __shfl_sync(kFull, base, leader);
  if (mv) {
    unsigned long long pos = base + __popc(m & lanemask_lt());
    A.mv_v[pos] = v;
    A.mv_new[pos] = t;
  }
}

// Candidate c (!= own) with accumulated weight e and total a_c: fold into (s, cb).
__device__ __forceinline__ void consider(int32_t c, uint32_t e, uint32_t ac, int32_t own, bool own_single,
                                         uint32_t ki, const SweepArgs& A, long long& s, int& cb) {
  if (A.rule == 2 && own_single && c > own && __ldg(&A.size[c]) == 1) return;  // R8 'filter' reading
  const long long sc = A.W * (long long)e - (long long)ki * (long long)ac;
  if (better(sc, c, s, cb)) { s = sc; cb = c; }
}

// Stay test and singleton veto.
__device__ __forceinline__ int32_t finish(long long s, int cb, uint32_t eown, int32_t own, uint32_t a_own,
                                          uint32_t ki, const SweepArgs& A) {
  if (cb == 0x7FFFFFFF) return own;
  const long long sstay = A.W * (long long)eown - (long long)ki * ((long long)a_own - (long long)ki);
  if (s <= sstay) return own;
  if (A.rule == 1 && cb > own && __ldg(&A.size[own]) == 1 && __ldg(&A.size[cb]) == 1) return own;  // R8 veto
  return cb;
}

// ------------------------------------------------------------ deg <= 32
template <int G, bool UNIT>
__global__ void __launch_bounds__(256) sweep_small(const int32_t* __restrict__ verts, int64_t nv, SweepArgs A) {
  const int lane = threadIdx.x & 31;
  const int sub = lane & (G - 1);
  const unsigned gmask = (G == 32) ? kFull : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  const int64_t wid = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  for (int64_t base = wid * (32 / G); base < nv; base += warps * (32 / G)) {
    const int64_t vi = base + lane / G;
    const bool active = vi < nv;
    int32_t v = 0, own = -1, deg = 0;
    int64_t rb = 0;
    uint32_t ki = 0;
    if (active) {
      v = __ldg(&verts[vi]);
      rb = __ldg(&A.rowptr[v]);
      deg = (int32_t)(__ldg(&A.rowptr[v + 1]) - rb);
      own = (int32_t)__ldg(&A.ca[v]).x;
      ki = __ldg(&A.k[v]);
    }
    const bool has = sub < deg;
    const int32_t j = has ? __ldcs(&A.col[rb + sub]) : -1;
    const uint32_t we = UNIT ? 1u : (has ? __ldcs(&A.w[rb + sub]) : 0u);
    const bool valid = has && j != v;  // R3: the self-loop does not count in e
    uint2 rec = make_uint2(0, 0);
    if (valid) rec = __ldg(&A.ca[j]);
    const int32_t c = valid ? (int32_t)rec.x : (int32_t)(0x80000000u | (unsigned)lane);
    const unsigned m = __match_any_sync(kFull, c) & gmask;
    const uint32_t e = UNIT ? (uint32_t)__popc(m) : __reduce_add_sync(m, we);
    // a lane whose neighbour represents the label (j == c) already holds a_c
    const unsigned rep = __ballot_sync(kFull, valid && j == c) & m;
    const uint32_t a_rep = __shfl_sync(kFull, rec.y, rep ? __ffs(rep) - 1 : lane);
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    if (valid && lane == __ffs(m) - 1) {
      if (c == own) {
        eown = e;
      } else {
        const uint32_t ac = rep ? a_rep : __ldg(&A.ca[c]).y;
        consider(c, e, ac, own, A.rule == 2 && __ldg(&A.size[own]) == 1, ki, A, s, cb);
      }
    }
    group_reduce<G>(s, cb, eown);
    int32_t t = own;
    if (active && sub == 0 && cb != 0x7FFFFFFF) t = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
    log_moves(active && sub == 0 && t != own, v, t, A);
  }
}

// Table scan shared by the warp and CTA kernels: slots [t0, cap) step `stride`.
// Clears every visited slot for the next vertex.  4 slots per pass so the a_c
// gathers of labels without a representative in the row overlap.
template <bool GLOBAL = false>
__device__ __forceinline__ void scan_table(unsigned long long* T, uint32_t* TA, uint32_t cap, uint32_t t0,
                                           uint32_t stride, int32_t own, bool own_single, uint32_t ki,
                                           const SweepArgs& A, long long& s, int& cb, unsigned& eown) {
  for (uint32_t base = t0; base < cap; base += 4 * stride) {
    unsigned long long x[4];
    uint32_t ac[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint32_t t = base + q * stride;
      x[q] = kEmpty;
      ac[q] = kUnknownA;
      if (t < cap) {
        x[q] = GLOBAL ? __ldcg(&T[t]) : T[t];  // global tables: L2 (atomics live there), never a stale L1 line
        if (x[q] != kEmpty) {
          ac[q] = GLOBAL ? __ldcg(&TA[t]) : TA[t];
          if (GLOBAL) {
            __stcg(&T[t], kEmpty);
            __stcg(&TA[t], kUnknownA);
          } else {
            T[t] = kEmpty;
            TA[t] = kUnknownA;
          }
        }
      }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (x[q] != kEmpty && ac[q] == kUnknownA && (int32_t)(x[q] >> 32) != own)
        ac[q] = __ldg(&A.ca[(int32_t)(x[q] >> 32)]).y;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (x[q] == kEmpty) continue;
      const int32_t c = (int32_t)(x[q] >> 32);
      const uint32_t e = (uint32_t)x[q];
      if (c == own) eown = e;
      else consider(c, e, ac[q], own, own_single, ki, A, s, cb);
    }
  }
}

// Sequential insert into a shared-memory table (CAS latency is short there):
// one CAS claims an empty slot with the value already in it; a slot already
// holding c gets an atomic add on its low word (e <= W < 2^32, no carry).
__device__ __forceinline__ uint32_t table_insert(unsigned long long* T, uint32_t cap, int32_t c, uint32_t x) {
  const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
  uint32_t h = hash_slot(c, cap);
  for (;;) {
    const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
    if (old == kEmpty) return h;
    if ((old >> 32) == (unsigned long long)(uint32_t)c) {
      atomicAdd(&T[h], (unsigned long long)x);
      return h;
    }
    h = (h + 1 == cap) ? 0 : h + 1;
  }
}

// Global-memory (hub) variant: the table is split into 4-slot buckets (32 B,
// one sector).  Each round reads a thread's bucket with two 16-byte L2 loads,
// adds into the slot holding c, or CASes the first empty slot; a failed CAS
// re-reads the same bucket, a full bucket moves to the next.  Slots only go
// EMPTY -> key once, and a key is only claimed at the first empty slot of its
// probe sequence, so no label is ever inserted twice.  One L2 round trip per
// insert at load factor <= 1/2 instead of ~(1 + 1/(1-a)^2)/2 dependent CASes.
__device__ __forceinline__ void gtable_insert4(unsigned long long* T, uint32_t* TA, uint32_t cap, const int32_t c[4],
                                               const uint32_t x[4], bool todo[4], const uint32_t arep[4]) {
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
    int tgt[4];
    bool found[4];
    unsigned long long old[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      tgt[q] = -1;
      found[q] = false;
      old[q] = 0;
      if (!todo[q]) continue;
#pragma unroll
      for (int u = 3; u >= 0; --u) {
        if (k[q][u] == kEmpty) tgt[q] = u;  // first empty slot
      }
#pragma unroll
      for (int u = 3; u >= 0; --u) {
        if (k[q][u] != kEmpty && (k[q][u] >> 32) == (unsigned long long)(uint32_t)c[q]) {
          tgt[q] = u;
          found[q] = true;
        }
      }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (todo[q] && !found[q] && tgt[q] >= 0)
        old[q] = atomicCAS(&T[b[q] + tgt[q]], kEmpty, (((unsigned long long)(uint32_t)c[q]) << 32) | x[q]);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (!todo[q]) continue;
      if (found[q]) {
        atomicAdd(&T[b[q] + tgt[q]], (unsigned long long)x[q]);
      } else if (tgt[q] >= 0) {
        if (old[q] != kEmpty) {
          if ((old[q] >> 32) != (unsigned long long)(uint32_t)c[q]) continue;  // lost the race: re-read bucket
          atomicAdd(&T[b[q] + tgt[q]], (unsigned long long)x[q]);
        }
      } else {
        b[q] = (b[q] + 4 >= cap) ? 0u : b[q] + 4;  // bucket full
        continue;
      }
      if (arep[q] != kUnknownA) TA[b[q] + tgt[q]] = arep[q];
      todo[q] = false;
    }
  }
}

// Phase 1 of the two-phase sweep (edge-parallel gather): for every neighbour
// slot of the bucket's table-based vertices, stage[soff[i] + t] = the packed
// record of the t-th neighbour of bin_vertices[i] as {label, a_c if that
// neighbour represents its label else kUnknownA}, or {kSelf, 0} for the
// self-loop (R3).  Flat over the bucket's edges in 4096-entry tiles (the tile's
// vertices are staged in smem and found by binary search), 4 gathers in flight
// per thread -- the random gathers run at the memory system's throughput
// instead of inside per-vertex latency chains.
constexpr uint32_t kSelf = 0xFFFFFFFFu;
constexpr int kStageTile = 4096;
constexpr int kStageRows = 256;

__global__ void __launch_bounds__(256) k_stage(const int32_t* __restrict__ bv, const int64_t* __restrict__ soff,
                                               int64_t pos0, int64_t pos1, const int64_t* __restrict__ tr,
                                               const int64_t* __restrict__ rowptr,
                                               const int32_t* __restrict__ col, const uint2* __restrict__ ca,
                                               uint2* __restrict__ stage, bool cs_store, bool full_a) {
  __shared__ int64_t sh_so[kStageRows + 1];
  __shared__ int64_t sh_rb[kStageRows];
  __shared__ int32_t sh_v[kStageRows];
  __shared__ int64_t sh_i0;
  __shared__ int sh_nr;
  const int64_t s0 = soff[pos0], s1 = soff[pos1];
  const int64_t ntiles = (s1 - s0 + kStageTile - 1) / kStageTile;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t t0 = s0 + tile * kStageTile, t1 = min(s1, t0 + kStageTile);
    if (threadIdx.x == 0) {  // tile plan: positions tr[tile] .. tr[tile + 1] cover the tile
      const int64_t i0 = tr[tile], i1 = tr[tile + 1];
      sh_i0 = i0;
      sh_nr = (i1 - i0 + 1 <= kStageRows) ? (int)(i1 - i0 + 1) : -1;
    }
    __syncthreads();
    const int64_t i0 = sh_i0;
    const int nr = sh_nr;
    for (int r = threadIdx.x; r < nr; r += blockDim.x) {
      const int32_t v = bv[i0 + r];
      sh_v[r] = v;
      sh_so[r] = soff[i0 + r];
      sh_rb[r] = rowptr[v];
    }
    __syncthreads();
    for (int64_t base = t0 + threadIdx.x; base < t1; base += 4 * (int64_t)blockDim.x) {
      int32_t jj[4], vv[4];
      uint2 rr[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + (int64_t)q * blockDim.x;
        jj[q] = -1;
        vv[q] = -1;
        if (t < t1) {
          int64_t e;
          if (nr > 0) {
            int lo = 0, hi = nr - 1;
            while (lo < hi) {
              const int mid = (lo + hi + 1) >> 1;
              if (sh_so[mid] <= t) lo = mid; else hi = mid - 1;
            }
            vv[q] = sh_v[lo];
            e = sh_rb[lo] + (t - sh_so[lo]);
          } else {
            int64_t lo = pos0, hi = pos1 - 1;
            while (lo < hi) {
              const int64_t mid = (lo + hi + 1) >> 1;
              if (soff[mid] <= t) lo = mid; else hi = mid - 1;
            }
            vv[q] = bv[lo];
            e = rowptr[vv[q]] + (t - soff[lo]);
          }
          jj[q] = __ldcs(&col[e]);
        }
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) rr[q] = (jj[q] >= 0 && jj[q] != vv[q]) ? __ldg(&ca[jj[q]]) : make_uint2(kSelf, 0);
      if (full_a) {  // a_c of labels whose neighbour is not their representative: a second gather
#pragma unroll       // here (edge-parallel, latency hidden) instead of in the table scans
        for (int q = 0; q < 4; ++q)
          if (jj[q] >= 0 && jj[q] != vv[q] && rr[q].x != (uint32_t)jj[q]) rr[q].y = __ldg(&ca[rr[q].x]).y;
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + (int64_t)q * blockDim.x;
        // evict-first store: the stage streams through L2 once and must not
        // displace the gathered records (LV_STAGE_WB=1: plain write-back store)
        const uint2 val = (jj[q] == vv[q]) ? make_uint2(kSelf, 0u)
                                           : make_uint2(rr[q].x, (full_a || rr[q].x == (uint32_t)jj[q]) ? rr[q].y
                                                                                                        : kUnknownA);
        if (t < t1) {
          if (cs_store) __stcs(&stage[t], val);
          else stage[t] = val;
        }
      }
    }
    __syncthreads();
  }
}

// Warp-chunked variant of phase 1 (LV_STAGE_W=1): every warp takes chunks of
// kStageChunk staged entries on its own -- no CTA barriers.  Lane r holds the
// descriptor (entry offset, row start, vertex) of the r-th row touching the
// chunk (tile plan at chunk granularity); a lane finds the row of each of its
// entries by a 5-step shuffle search, and keeps 8 gathers in flight.  A chunk
// touching more than 32 rows (rows shorter than 32 entries on average) falls
// back to a binary search over soff.
constexpr int kStageChunk = 1024;
__global__ void __launch_bounds__(256) k_stage_w(const int32_t* __restrict__ bv, const int64_t* __restrict__ soff,
                                                 int64_t pos0, int64_t pos1, int64_t s0, int64_t s1,
                                                 const int64_t* __restrict__ tr, const int64_t* __restrict__ rowptr,
                                                 const int32_t* __restrict__ col, const uint2* __restrict__ ca,
                                                 uint2* __restrict__ stage) {
  const int lane = threadIdx.x & 31;
  const int64_t nchunks = (s1 - s0 + kStageChunk - 1) / kStageChunk;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t ch = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); ch < nchunks; ch += warps) {
    const int64_t t0 = s0 + ch * kStageChunk, t1 = min(s1, t0 + kStageChunk);
    const int64_t i0 = tr[ch], i1 = tr[ch + 1];
    const int nr = (int)((i1 - i0 + 1 < 33) ? i1 - i0 + 1 : 33);
    const bool fits = i1 - i0 + 1 <= 32;
    // lane r: row i0 + r
    int64_t my_so = INT64_MAX, my_rb = 0;
    int32_t my_v = -1;
    if (fits && lane < nr && i0 + lane < pos1) {
      my_v = bv[i0 + lane];
      my_so = soff[i0 + lane];
      my_rb = rowptr[my_v];
    }
    for (int64_t b0 = t0; b0 < t1; b0 += 8 * 32) {  // warp-uniform trips (shuffles below)
      const int64_t base = b0 + lane;
      int32_t jj[8], vv[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int64_t t = base + 32 * q;
        int64_t e = 0;
        vv[q] = -1;
        jj[q] = -1;
        if (fits) {
          int lo = 0;  // largest r with so_r <= t (all lanes take part in the shuffles)
#pragma unroll
          for (int step = 16; step >= 1; step >>= 1) {
            const int64_t so_mid = __shfl_sync(kFull, my_so, lo + step);
            if (lo + step < nr && so_mid <= t) lo += step;
          }
          const int64_t so_r = __shfl_sync(kFull, my_so, lo);
          const int64_t rb_r = __shfl_sync(kFull, my_rb, lo);
          const int32_t v_r = __shfl_sync(kFull, my_v, lo);
          if (t < t1) {
            vv[q] = v_r;
            e = rb_r + (t - so_r);
          }
        } else if (t < t1) {
          int64_t lo = pos0, hi = pos1 - 1;
          while (lo < hi) {
            const int64_t mid = (lo + hi + 1) >> 1;
            if (soff[mid] <= t) lo = mid; else hi = mid - 1;
          }
          vv[q] = bv[lo];
          e = rowptr[vv[q]] + (t - soff[lo]);
        }
        if (t < t1) jj[q] = __ldcs(&col[e]);
      }
      uint2 rr[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) rr[q] = (jj[q] >= 0 && jj[q] != vv[q]) ? __ldg(&ca[jj[q]]) : make_uint2(kSelf, 0);
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int64_t t = base + 32 * q;
        if (t < t1)
          __stcs(&stage[t], (jj[q] == vv[q]) ? make_uint2(kSelf, 0u)
                                             : make_uint2(rr[q].x, rr[q].x == (uint32_t)jj[q] ? rr[q].y : kUnknownA));
      }
    }
  }
}

// Phase 2 insert: entries [t0, deg) step `stride` of one vertex's staged
// neighbours S (and weights Wt), 4 per pass, no random loads.  With AGG,
// labels are first merged across the warp (__match_any_sync, weights summed
// with __reduce_add_sync): a label shared by many neighbours costs one table
// atomic per warp.  The trip count is uniform across each warp.
template <bool UNIT, bool AGG, bool GLOBAL = false>
__device__ __forceinline__ void insert_staged(unsigned long long* T, uint32_t* TA, uint32_t cap,
                                              const uint2* __restrict__ S, const uint32_t* __restrict__ Wt,
                                              int64_t deg, int64_t t0, int64_t stride) {
  const int lane = threadIdx.x & 31;
  const int64_t t_warp0 = t0 - lane;
  for (int64_t base = 0; base + t_warp0 < deg; base += 4 * stride) {
    uint2 rr[4];
    uint32_t ww[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int64_t t = base + t0 + q * stride;
      rr[q] = (t < deg) ? __ldcs(&S[t]) : make_uint2(kSelf, 0u);
      ww[q] = UNIT ? 1u : ((t < deg) ? __ldcs(&Wt[t]) : 0u);
    }
    int32_t c[4];
    uint32_t x[4], arep[4];
    bool todo[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const bool valid = rr[q].x != kSelf;
      c[q] = valid ? (int32_t)rr[q].x : (int32_t)(0x80000000u | (unsigned)lane);
      // (adaptive merging here measured 2-3x slower on the warp kernels of C5: the
      // smem tables of these small rows tolerate same-slot atomics better than
      // __match_any_sync costs; only the hub paths merge adaptively)
      if (AGG) {
        const unsigned m = __match_any_sync(kFull, c[q]);
        x[q] = UNIT ? (uint32_t)__popc(m) : __reduce_add_sync(m, ww[q]);
        const unsigned rep = __ballot_sync(kFull, valid && rr[q].y != kUnknownA) & m;
        const uint32_t a_rep = __shfl_sync(kFull, rr[q].y, rep ? __ffs(rep) - 1 : lane);
        todo[q] = valid && lane == __ffs(m) - 1;
        arep[q] = rep ? a_rep : kUnknownA;
      } else {
        x[q] = ww[q];
        todo[q] = valid;
        arep[q] = rr[q].y;
      }
    }
    if (GLOBAL) {
      gtable_insert4(T, TA, cap, c, x, todo, arep);
    } else {
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (!todo[q]) continue;
        const uint32_t hq = table_insert(T, cap, c[q], x[q]);
        if (arep[q] != kUnknownA) TA[hq] = arep[q];
      }
    }
  }
}

// ------------------------------------------------------------ warp per vertex
template <int CAP, int WARPS, bool UNIT, bool AGG>
__global__ void __launch_bounds__(32 * WARPS) sweep_warp(const int32_t* __restrict__ verts,
                                                         const int64_t* __restrict__ soff, int64_t nv,
                                                         const uint2* __restrict__ stage, SweepArgs A) {
  __shared__ unsigned long long tab[WARPS][CAP];
  __shared__ uint32_t taba[WARPS][CAP];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  unsigned long long* T = tab[wl];
  uint32_t* TA = taba[wl];
  for (int t = lane; t < CAP; t += 32) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  __syncwarp();
  const int64_t warps = (int64_t)gridDim.x * WARPS;
  for (int64_t vi = (int64_t)blockIdx.x * WARPS + wl; vi < nv; vi += warps) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&A.rowptr[v]);
    const int64_t deg = __ldg(&A.rowptr[v + 1]) - rb;
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    insert_staged<UNIT, AGG>(T, TA, CAP, stage + __ldg(&soff[vi]), UNIT ? nullptr : A.w + rb, deg, lane, 32);
    __syncwarp();
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_table(T, TA, CAP, lane, 32, own, own_single, ki, A, s, cb, eown);
    group_reduce<32>(s, cb, eown);
    int32_t tgt = own;
    if (lane == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
    log_moves(lane == 0 && tgt != own, v, tgt, A);
    __syncwarp();
  }
}

// ------------------------------------------------------------ CTA per vertex (default)
template <bool UNIT, bool AGG>
__global__ void __launch_bounds__(1024) sweep_cta(const int32_t* __restrict__ verts, const int64_t* __restrict__ soff,
                                                  int64_t nv, const uint2* __restrict__ stage, SweepArgs A,
                                                  int capmax, int fnum) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + capmax);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  for (int t = threadIdx.x; t < capmax; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  __syncthreads();
  for (int64_t vi = blockIdx.x; vi < nv; vi += gridDim.x) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&A.rowptr[v]);
    const int64_t deg = __ldg(&A.rowptr[v + 1]) - rb;
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    // table of deg * (1 + fnum/8) slots (fnum = 8: load 1/2), at most capmax
    const int64_t want = deg + ((deg * fnum) >> 3) + 1;
    const uint32_t cap = (uint32_t)(want < (int64_t)capmax ? want : (int64_t)capmax);
    insert_staged<UNIT, AGG>(T, TA, cap, stage + __ldg(&soff[vi]), UNIT ? nullptr : A.w + rb, deg, threadIdx.x,
                             blockDim.x);
    __syncthreads();
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_table(T, TA, cap, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x < 32) {
      int32_t tgt = own;
      if (threadIdx.x == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
      log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
}


// ------------------------------------------------------------ claimed-slot lists (default)
// The thread whose CAS claims an empty slot appends the slot index to the
// table's list (warp-aggregated, one shared atomic per warp and pass), so the
// scan visits exactly the distinct labels with full warps instead of every
// slot of the table (ncu, C5 sweep 1: the slot scan of the warp / CTA kernels
// ran at 10-20 active lanes per instruction and was ~45% of their instructions).
// The four inserts of a pass share one retry loop (independent CASes in flight
// instead of four divergent probe loops).
template <bool UNIT>
__device__ __forceinline__ void insert_list(unsigned long long* T, uint32_t* TA, uint32_t cap,
                                            const uint2* __restrict__ S, const uint32_t* __restrict__ Wt,
                                            int64_t deg, int64_t t0, int64_t stride, uint16_t* Lst, int* nL) {
  const int lane = threadIdx.x & 31;
  const int64_t t_warp0 = t0 - lane;
  for (int64_t base = 0; base + t_warp0 < deg; base += 4 * stride) {  // trip count uniform across the warp
    uint2 rr[4];
    uint32_t ww[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int64_t t = base + t0 + q * stride;
      rr[q] = (t < deg) ? __ldcs(&S[t]) : make_uint2(kSelf, 0u);
      ww[q] = UNIT ? 1u : ((t < deg) ? __ldcs(&Wt[t]) : 0u);
    }
    uint32_t h[4];
    bool todo[4], claimed[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      todo[q] = rr[q].x != kSelf;
      claimed[q] = false;
      h[q] = todo[q] ? hash_slot((int32_t)rr[q].x, cap) : 0u;
    }
    while (todo[0] || todo[1] || todo[2] || todo[3]) {
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (!todo[q]) continue;
        const unsigned long long kx = ((unsigned long long)rr[q].x << 32) | ww[q];
        const unsigned long long old = atomicCAS(&T[h[q]], kEmpty, kx);
        if (old == kEmpty) {
          claimed[q] = true;
          todo[q] = false;
        } else if ((uint32_t)(old >> 32) == rr[q].x) {
          atomicAdd(&T[h[q]], (unsigned long long)ww[q]);
          todo[q] = false;
        } else {
          h[q] = (h[q] + 1 == cap) ? 0u : h[q] + 1;
        }
      }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (rr[q].x != kSelf && rr[q].y != kUnknownA) TA[h[q]] = rr[q].y;
    unsigned m[4];
    int tot = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      m[q] = __ballot_sync(kFull, claimed[q]);
      tot += __popc(m[q]);
    }
    if (tot) {
      int b0 = 0;
      if (lane == 0) b0 = atomicAdd(nL, tot);
      b0 = __shfl_sync(kFull, b0, 0);
      const unsigned lt = lanemask_lt();
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (claimed[q]) Lst[b0 + __popc(m[q] & lt)] = (uint16_t)h[q];
        b0 += __popc(m[q]);
      }
    }
  }
}

// Scan of the claimed slots (entries [t0, nl) step `stride` of the list); clears
// each visited slot for the next vertex.
__device__ __forceinline__ void scan_list(unsigned long long* T, uint32_t* TA, const uint16_t* Lst, int nl, int t0,
                                          int stride, int32_t own, bool own_single, uint32_t ki, const SweepArgs& A,
                                          long long& s, int& cb, unsigned& eown) {
  for (int base = t0; base < nl; base += 4 * stride) {
    unsigned long long x[4];
    uint32_t ac[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int t = base + q * stride;
      x[q] = kEmpty;
      ac[q] = kUnknownA;
      if (t < nl) {
        const uint32_t sl = Lst[t];
        x[q] = T[sl];
        ac[q] = TA[sl];
        T[sl] = kEmpty;
        TA[sl] = kUnknownA;
      }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (x[q] != kEmpty && ac[q] == kUnknownA && (int32_t)(x[q] >> 32) != own)
        ac[q] = __ldg(&A.ca[(int32_t)(x[q] >> 32)]).y;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (x[q] == kEmpty) continue;
      const int32_t c = (int32_t)(x[q] >> 32);
      const uint32_t e = (uint32_t)x[q];
      if (c == own) eown = e;
      else consider(c, e, ac[q], own, own_single, ki, A, s, cb);
    }
  }
}

template <int CAP, int LCAP, int WARPS, bool UNIT>
__global__ void __launch_bounds__(32 * WARPS) sweep_warp_l(const int32_t* __restrict__ verts,
                                                           const int64_t* __restrict__ soff, int64_t nv,
                                                           const uint2* __restrict__ stage, SweepArgs A) {
  __shared__ unsigned long long tab[WARPS][CAP];
  __shared__ uint32_t taba[WARPS][CAP];
  __shared__ uint16_t lst[WARPS][LCAP];
  __shared__ int nls[WARPS];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  unsigned long long* T = tab[wl];
  uint32_t* TA = taba[wl];
  for (int t = lane; t < CAP; t += 32) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  if (lane == 0) nls[wl] = 0;
  __syncwarp();
  const int64_t warps = (int64_t)gridDim.x * WARPS;
  for (int64_t vi = (int64_t)blockIdx.x * WARPS + wl; vi < nv; vi += warps) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&A.rowptr[v]);
    const int64_t deg = __ldg(&A.rowptr[v + 1]) - rb;
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    insert_list<UNIT>(T, TA, CAP, stage + __ldg(&soff[vi]), UNIT ? nullptr : A.w + rb, deg, lane, 32, lst[wl],
                      &nls[wl]);
    __syncwarp();
    const int nl = nls[wl];
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_list(T, TA, lst[wl], nl, lane, 32, own, own_single, ki, A, s, cb, eown);
    group_reduce<32>(s, cb, eown);
    int32_t tgt = own;
    if (lane == 0) {
      tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
      nls[wl] = 0;
    }
    log_moves(lane == 0 && tgt != own, v, tgt, A);
    __syncwarp();
  }
}

// CTA per vertex with a claimed-slot list; dynamic smem = capmax slots (12 B)
// + lcap list entries (2 B).
template <bool UNIT>
__global__ void __launch_bounds__(1024) sweep_cta_l(const int32_t* __restrict__ verts,
                                                    const int64_t* __restrict__ soff, int64_t nv,
                                                    const uint2* __restrict__ stage, SweepArgs A, int capmax) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + capmax);
  uint16_t* Lst = reinterpret_cast<uint16_t*>(TA + capmax);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  __shared__ int sh_n;
  for (int t = threadIdx.x; t < capmax; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  if (threadIdx.x == 0) sh_n = 0;
  __syncthreads();
  for (int64_t vi = blockIdx.x; vi < nv; vi += gridDim.x) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&A.rowptr[v]);
    const int64_t deg = __ldg(&A.rowptr[v + 1]) - rb;
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    const uint32_t cap = (uint32_t)((2 * deg < (int64_t)capmax) ? 2 * deg : (int64_t)capmax);
    insert_list<UNIT>(T, TA, cap, stage + __ldg(&soff[vi]), UNIT ? nullptr : A.w + rb, deg, threadIdx.x, blockDim.x,
                      Lst, &sh_n);
    __syncthreads();
    const int nl = sh_n;
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_list(T, TA, Lst, nl, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);  // its barrier orders every read of sh_n before the reset
    if (threadIdx.x < 32) {
      int32_t tgt = own;
      if (threadIdx.x == 0) {
        tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
        sh_n = 0;
      }
      log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
}


// ------------------------------------------------------------ CTA per vertex, pipelined (LV_CTA_PIPE=1)
// Persistent CTAs, one vertex at a time, software-pipelined so the per-vertex
// chain of dependent global loads is off the critical path: while the CTA
// hashes vertex j, lanes of warp 0 already load the bin entry of vertex j+2 and
// the row bounds / record / degree of vertex j+1 (results parked in registers and
// stored to shared memory at the end of the iteration), and a_own / size_own of
// vertex j for its decision.  Moves go to a shared buffer flushed with one
// atomic per kLogBuf moves.
constexpr int kLogBuf = 128;

__device__ __forceinline__ void flush_moves(int32_t* buf_v, int32_t* buf_t, int n, const SweepArgs& A) {
  // warp 0, all lanes
  const int lane = threadIdx.x & 31;
  unsigned long long base = 0;
  if (lane == 0 && n) base = atomicAdd(A.logn, (unsigned long long)n);
  base = __shfl_sync(kFull, base, 0);
  for (int i = lane; i < n; i += 32) {
    A.mv_v[base + i] = buf_v[i];
    A.mv_new[base + i] = buf_t[i];
  }
}

template <bool UNIT, bool AGG>
__global__ void __launch_bounds__(1024) sweep_cta_pipe(const int32_t* __restrict__ verts, const int64_t* __restrict__ soff,
                                                  int64_t nv, const uint2* __restrict__ stage, SweepArgs A,
                                                  int capmax) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + capmax);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  // header of the current vertex (j) and the bin entry of the next one (j+1)
  __shared__ int64_t h_rb, h_deg, h_so;
  __shared__ int32_t h_v, h_own, h_vnext;
  __shared__ uint32_t h_ki;
  __shared__ int32_t buf_v[kLogBuf], buf_t[kLogBuf];
  __shared__ int nbuf;
  const int lane = threadIdx.x & 31;
  const int64_t G = gridDim.x;
  for (int t = threadIdx.x; t < capmax; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  if (threadIdx.x == 0) {  // prologue: header of vertex 0, bin entry of vertex 1
    nbuf = 0;
    const int64_t vi = blockIdx.x;
    if (vi < nv) {
      const int32_t v = verts[vi];
      h_v = v;
      h_rb = A.rowptr[v];
      h_deg = A.rowptr[v + 1] - h_rb;
      h_so = soff[vi];
      h_own = (int32_t)A.ca[v].x;
      h_ki = A.k[v];
    }
    h_vnext = (vi + G < nv) ? verts[vi + G] : -1;
  }
  __syncthreads();
  for (int64_t vi = blockIdx.x; vi < nv; vi += G) {
    const int32_t v = h_v, own = h_own, vn = h_vnext;
    const int64_t rb = h_rb, deg = h_deg, so = h_so;
    const uint32_t ki = h_ki;
    // warp 0 issues the loads of the next vertices now and consumes them at the end
    int64_t pf = 0;
    if (threadIdx.x < 32) {
      if (lane == 0 && vi + 2 * G < nv) pf = verts[vi + 2 * G];
      if (vn >= 0) {
        if (lane == 1) pf = A.rowptr[vn];
        if (lane == 2) pf = A.rowptr[vn + 1];
        if (lane == 3) pf = soff[vi + G];
        if (lane == 4) pf = (int64_t)A.ca[vn].x;
        if (lane == 5) pf = (int64_t)A.k[vn];
      }
      if (lane == 6) pf = (int64_t)A.ca[own].y;
      if (lane == 7) pf = (int64_t)A.size[own];
    }
    const uint32_t cap = (uint32_t)((2 * deg < (int64_t)capmax) ? 2 * deg : (int64_t)capmax);
    insert_staged<UNIT, AGG>(T, TA, cap, stage + so, UNIT ? nullptr : A.w + rb, deg, threadIdx.x, blockDim.x);
    __syncthreads();
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_table(T, TA, cap, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x < 32) {
      const uint32_t a_own = (uint32_t)__shfl_sync(kFull, pf, 6);
      const int32_t size_own = (int32_t)__shfl_sync(kFull, pf, 7);
      if (threadIdx.x == 0 && cb != 0x7FFFFFFF) {
        int32_t tgt = own;
        const long long sstay = A.W * (long long)eown - (long long)ki * ((long long)a_own - (long long)ki);
        if (s > sstay) {
          tgt = cb;
          if (A.rule == 1 && cb > own && size_own == 1 && __ldg(&A.size[cb]) == 1) tgt = own;  // R8 veto
        }
        if (tgt != own) {
          buf_v[nbuf] = v;
          buf_t[nbuf] = tgt;
          ++nbuf;
        }
      }
      __syncwarp();
      if (nbuf == kLogBuf) {
        flush_moves(buf_v, buf_t, kLogBuf, A);
        __syncwarp();
        if (lane == 0) nbuf = 0;
      }
      // park the prefetched header of vertex j+1 and the bin entry of vertex j+2
      if (lane == 0) h_vnext = (vi + 2 * G < nv) ? (int32_t)pf : -1;
      if (vn >= 0) {
        if (lane == 0) h_v = vn;
        if (lane == 1) h_rb = pf;
        if (lane == 2) h_deg = pf;  // rowptr[v+1]; minus rb below
        if (lane == 3) h_so = pf;
        if (lane == 4) h_own = (int32_t)pf;
        if (lane == 5) h_ki = (uint32_t)pf;
      }
      __syncwarp();
      if (lane == 0 && vn >= 0) h_deg -= h_rb;
    }
    __syncthreads();
  }
  if (threadIdx.x < 32) {
    __syncwarp();
    const int n = nbuf;
    flush_moves(buf_v, buf_t, n, A);
  }
}

// ------------------------------------------------------------ batched vertices
// Table-based vertices of degree <= kBatchMaxDeg (33..1023 with the paper's
// bounds): a CTA takes a batch of consecutive bin positions (total weight
// bounded by the batch plan) and works on all of them at once, so the per-vertex
// latency chains (row bounds, records, finish) overlap instead of serialising:
//   1. batch metadata into smem (vertex, row start, entry offset);
//   2. edge-parallel over the batch's staged entries: insert into the vertex's
//      own region of the table (2*deg slots at offset 2*x0);
//   3. each vertex's region is scanned by a group of G warps (G = 16 / nv
//      rounded down to a power of two), partials to smem;
//   4. a warp per vertex reduces its partials and decides (stay test, veto).
// The records come from the staging array (k_stage gathered them edge-parallel
// at full occupancy; gathering here, inside the batch's latency chain, measured
// 3x slower on C5).
template <bool UNIT>
__global__ void __launch_bounds__(512, 2) sweep_batch(const int32_t* __restrict__ bv,
                                                    const int64_t* __restrict__ soff,
                                                    const int32_t* __restrict__ bstart, int64_t nbatch,
                                                    const uint2* __restrict__ stage, SweepArgs A) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + kBatchSlots);
  __shared__ int32_t s_v[kBatchMaxVerts];
  __shared__ int64_t s_rb[kBatchMaxVerts];
  __shared__ int32_t s_x[kBatchMaxVerts + 1];
  __shared__ Partial s_part[16];
  __shared__ int s_nv;
  constexpr int NW = 16;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int t = threadIdx.x; t < kBatchSlots; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  for (int64_t b = blockIdx.x; b < nbatch; b += gridDim.x) {
    // 1. metadata
    const int32_t p0 = __ldg(&bstart[b]), p1 = __ldg(&bstart[b + 1]);
    const int nv = p1 - p0;
    const int64_t base = __ldg(&soff[p0]);
    for (int r = threadIdx.x; r <= nv; r += blockDim.x) {
      s_x[r] = (int32_t)(__ldg(&soff[p0 + r]) - base);
      if (r < nv) {
        const int32_t v = __ldg(&bv[p0 + r]);
        s_v[r] = v;
        s_rb[r] = __ldg(&A.rowptr[v]);
      }
    }
    if (threadIdx.x == 0) s_nv = nv;
    __syncthreads();
    const int E = s_x[nv];
    // 2. inserts from the staged records (coalesced), 4 entries per thread per pass
    const uint2* S = stage + base;
    for (int x0 = threadIdx.x; x0 < E; x0 += 4 * blockDim.x) {
      uint2 rec[4];
      uint32_t ww[4];
      int rr[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int x = x0 + q * blockDim.x;
        rec[q] = (x < E) ? __ldcs(&S[x]) : make_uint2(kSelf, 0u);
        rr[q] = 0;
        ww[q] = 1u;
        if (x < E) {
          int lo = 0, hi = nv - 1;  // largest r with s_x[r] <= x
          while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (s_x[mid] <= x) lo = mid; else hi = mid - 1;
          }
          rr[q] = lo;
          if (!UNIT) ww[q] = __ldcs(&A.w[s_rb[lo] + (x - s_x[lo])]);
        }
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        if (rec[q].x == kSelf) continue;  // padding or the self-loop (R3)
        const int r = rr[q];
        const uint32_t off = 2u * (uint32_t)s_x[r];
        const uint32_t cap = 2u * (uint32_t)(s_x[r + 1] - s_x[r]);
        const uint32_t hq = table_insert(T + off, cap, (int32_t)rec[q].x, ww[q]);
        if (rec[q].y != kUnknownA) TA[off + hq] = rec[q].y;  // the neighbour represents its label: a_c known
      }
    }
    __syncthreads();
    // 3. scan: vertex r by warps [r*G, r*G + G) (nv <= 16), else warp-strided vertices
    int G = 1;
    while (G * 2 * nv <= NW) G *= 2;
    const int gw = warp % G;  // warp index inside its group
    for (int r = warp / G; r < nv; r += NW / G) {
      const int32_t v = s_v[r];
      const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
      const uint32_t ki = __ldg(&A.k[v]);
      const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
      const uint32_t off = 2u * (uint32_t)s_x[r];
      const uint32_t cap = 2u * (uint32_t)(s_x[r + 1] - s_x[r]);
      long long sc = (long long)0x8000000000000000ull;
      int cb = 0x7FFFFFFF;
      unsigned eown = 0;
      scan_table(T + off, TA + off, cap, (uint32_t)(gw * 32 + lane), (uint32_t)(32 * G), own, own_single, ki, A, sc,
                 cb, eown);
      group_reduce<32>(sc, cb, eown);
      if (G == 1) {
        int32_t tgt = own;
        if (lane == 0 && cb != 0x7FFFFFFF) tgt = finish(sc, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
        log_moves(lane == 0 && tgt != own, v, tgt, A);
      } else if (lane == 0) {
        s_part[warp] = Partial{sc, cb, eown};
      }
    }
    if (G > 1) {
      __syncthreads();
      // 4. a warp per vertex reduces its G partials
      if (warp < nv) {
        const int r = warp;
        long long sc = (long long)0x8000000000000000ull;
        int cb = 0x7FFFFFFF;
        unsigned eown = 0;
        if (lane < G) {
          const Partial pp = s_part[r * G + lane];
          sc = pp.s;
          cb = pp.c;
          eown = pp.eown;
        }
        group_reduce<32>(sc, cb, eown);
        const int32_t v = s_v[r];
        const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
        int32_t tgt = own;
        if (lane == 0 && cb != 0x7FFFFFFF) tgt = finish(sc, cb, eown, own, __ldg(&A.ca[own]).y, __ldg(&A.k[v]), A);
        log_moves(lane == 0 && tgt != own, v, tgt, A);
      }
    }
    __syncthreads();
  }
}

__global__ void k_batch_flags(const int64_t* __restrict__ soff, int64_t p0, int64_t p1, int64_t s0, int64_t bw,
                              uint8_t* flag) {
  for (int64_t i = p0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < p1; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t wi = (soff[i] - s0 + kBatchVertexWeight * (i - p0)) / bw;
    const int64_t wp = (i == p0) ? -1 : (soff[i - 1] - s0 + kBatchVertexWeight * (i - 1 - p0)) / bw;
    flag[i - p0] = (wi != wp) ? 1 : 0;
  }
}

// ------------------------------------------------------------ label-partitioned CTAs
// deg >= 12288: vertex v gets P = ceil(deg / kPartLabels) independent CTA tasks;
// task p owns the labels c with part_of(c, P) == p, so a partition sees
// ~deg/P distinct labels whatever the degree.  The staged entries are first
// scattered into partition order (k_part_hist / k_part_scan / k_part_scatter),
// so each task reads only its own share; the CTA that finishes v's last task
// reduces the P partials and decides.  No clusters, grid syncs or global hash
// tables.  A table that would pass 7/8 load sets DevCtl::overflow and the
// library reports an error (the expected load is <= 3/8).

// Pre-partitioning of the staged entries of the plan's vertices (every sweep,
// after k_stage): histogram of partition sizes per chunk -> per-vertex scan into
// poff / cursors -> scatter into S2 (and the weights into W2) in partition order.
// Labels of a warp are merged per partition with __match_any_sync so a hot
// partition costs one shared atomic per warp.
__global__ void __launch_bounds__(1024) k_part_hist(const PartChunk* __restrict__ chunks, int64_t c0, int64_t c1,
                                                    const int32_t* __restrict__ vert_pos,
                                                    const int32_t* __restrict__ vert_P,
                                                    const int64_t* __restrict__ vert_pbase,
                                                    const int64_t* __restrict__ soff, const uint2* __restrict__ stage,
                                                    int64_t* poff) {
  __shared__ uint32_t hist[kPartMaxP];
  for (int64_t ci = c0 + blockIdx.x; ci < c1; ci += gridDim.x) {
    const PartChunk ch = chunks[ci];
    const uint32_t P = (uint32_t)vert_P[ch.vi];
    const uint2* S = stage + soff[vert_pos[ch.vi]];
    for (uint32_t q = threadIdx.x; q < P; q += blockDim.x) hist[q] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    for (int64_t t0 = ch.begin + (threadIdx.x - lane); t0 < ch.end; t0 += blockDim.x) {  // warp-uniform trips
      const int64_t t = t0 + lane;
      const uint32_t lab = (t < ch.end) ? __ldcs(&S[t]).x : kSelf;
      const uint32_t q = (lab != kSelf) ? part_of((int32_t)lab, P) : 0xFFFFFFFFu;
      const unsigned m = __match_any_sync(kFull, q);
      if (q != 0xFFFFFFFFu && lane == __ffs(m) - 1) atomicAdd(&hist[q], (uint32_t)__popc(m));
    }
    __syncthreads();
    int64_t* cnt = poff + vert_pbase[ch.vi] + 1;
    for (uint32_t q = threadIdx.x; q < P; q += blockDim.x)
      if (hist[q]) atomicAdd(reinterpret_cast<unsigned long long*>(&cnt[q]), (unsigned long long)hist[q]);
    __syncthreads();
  }
}

// One warp per plan vertex: poff[pb + q] = segment start + sum of earlier counts,
// cursors of the scatter initialised to the partition starts.
__global__ void k_part_scan(int64_t v0, int64_t v1, const int32_t* __restrict__ vert_pos,
                            const int32_t* __restrict__ vert_P, const int64_t* __restrict__ vert_pbase,
                            const int32_t* __restrict__ vert_first, const int64_t* __restrict__ soff, int64_t* poff,
                            unsigned long long* pcur) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t vi = v0 + (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); vi < v1; vi += warps) {
    const int32_t P = vert_P[vi];
    const int64_t pb = vert_pbase[vi];
    const int64_t f = vert_first[vi];
    long long run = soff[vert_pos[vi]];
    for (int32_t q0 = 0; q0 < P; q0 += 32) {
      const int32_t q = q0 + lane;
      const long long c = (q < P) ? poff[pb + 1 + q] : 0;
      long long x = c;  // inclusive warp scan
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const long long y = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += y;
      }
      if (q < P) {
        const long long start = run + x - c;
        poff[pb + q] = start;
        pcur[f + q] = (unsigned long long)start;
      }
      run += __shfl_sync(kFull, x, 31);
    }
    if (lane == 0) poff[pb + P] = run;
  }
}

template <bool UNIT>
__global__ void __launch_bounds__(1024) k_part_scatter(const PartChunk* __restrict__ chunks, int64_t c0, int64_t c1,
                                                       const int32_t* __restrict__ vert_pos,
                                                       const int32_t* __restrict__ vert_P,
                                                       const int32_t* __restrict__ vert_first,
                                                       const int32_t* __restrict__ bv,
                                                       const int64_t* __restrict__ soff,
                                                       const uint2* __restrict__ stage, unsigned long long* pcur,
                                                       uint2* S2, uint32_t* W2, SweepArgs A) {
  __shared__ uint32_t hist[kPartMaxP];
  constexpr uint32_t kSeg = 1024;  // partitions reserved per round (the chunk is re-read when P > kSeg)
  __shared__ unsigned long long base[kSeg];
  for (int64_t ci = c0 + blockIdx.x; ci < c1; ci += gridDim.x) {
    const PartChunk ch = chunks[ci];
    const uint32_t P = (uint32_t)vert_P[ch.vi];
    const int32_t pos = vert_pos[ch.vi];
    const uint2* S = stage + soff[pos];
    const uint32_t* Wt = UNIT ? nullptr : A.w + A.rowptr[bv[pos]];
    unsigned long long* cur = pcur + vert_first[ch.vi];
    const int lane = threadIdx.x & 31;
    // the chunk's partition sizes
    for (uint32_t q = threadIdx.x; q < P; q += blockDim.x) hist[q] = 0;
    __syncthreads();
    for (int64_t t0 = ch.begin + (threadIdx.x - lane); t0 < ch.end; t0 += blockDim.x) {
      const int64_t t = t0 + lane;
      const uint32_t lab = (t < ch.end) ? __ldcs(&S[t]).x : kSelf;
      const uint32_t q = (lab != kSelf) ? part_of((int32_t)lab, P) : 0xFFFFFFFFu;
      const unsigned m = __match_any_sync(kFull, q);
      if (q != 0xFFFFFFFFu && lane == __ffs(m) - 1) atomicAdd(&hist[q], (uint32_t)__popc(m));
    }
    __syncthreads();
    // reserve the chunk's ranges, then scatter with local cursors (P in rounds of kSeg)
    for (uint32_t h0 = 0; h0 < P; h0 += kSeg) {
      const uint32_t h1 = min(P, h0 + kSeg);
      for (uint32_t q = h0 + threadIdx.x; q < h1; q += blockDim.x)
        base[q - h0] = hist[q] ? atomicAdd(&cur[q], (unsigned long long)hist[q]) : 0ull;
      __syncthreads();
      for (int64_t t0 = ch.begin + (threadIdx.x - lane); t0 < ch.end; t0 += blockDim.x) {
        const int64_t t = t0 + lane;
        const uint2 rec = (t < ch.end) ? __ldcs(&S[t]) : make_uint2(kSelf, 0u);
        uint32_t q = (rec.x != kSelf) ? part_of((int32_t)rec.x, P) : 0xFFFFFFFFu;
        if (q < h0 || q >= h1) q = 0xFFFFFFFFu;
        const unsigned m = __match_any_sync(kFull, q);
        unsigned long long b = 0;
        const int leader = __ffs(m) - 1;
        if (q != 0xFFFFFFFFu && lane == leader) b = atomicAdd(&base[q - h0], (unsigned long long)__popc(m));
        b = __shfl_sync(m, b, leader);
        if (q != 0xFFFFFFFFu) {
          const unsigned long long dst = b + __popc(m & lanemask_lt());
          __stcs(&S2[dst], rec);
          if (!UNIT) __stcs(&W2[dst], __ldcs(&Wt[t]));
        }
      }
      __syncthreads();
    }
  }
}

// Shared-memory insert of one partition's entries (warp-uniform trips; equal
// labels of a warp merged first with __match_any_sync, so the hot labels of later
// sweeps cost one shared atomic per warp).  Returns, in every lane, how many new
// slots this thread's warp claimed (only counted when `count`).
template <bool UNIT, bool AGG>
__device__ __forceinline__ unsigned part_insert(unsigned long long* T, uint32_t* TA, uint32_t cap,
                                                const uint2* __restrict__ S, const uint32_t* __restrict__ Wt,
                                                int64_t q0, int64_t q1, bool count) {
  const int lane = threadIdx.x & 31;
  unsigned claims = 0;
  for (int64_t base = q0 + (threadIdx.x - lane); base < q1; base += 4 * (int64_t)blockDim.x) {
    uint2 rr[4];
    uint32_t ww[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int64_t t = base + lane + (int64_t)u * blockDim.x;
      rr[u] = (t < q1) ? __ldcs(&S[t]) : make_uint2(kSelf, 0u);
      ww[u] = (t < q1) ? (UNIT ? 1u : __ldcs(&Wt[t])) : 0u;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      unsigned m = 1u << lane, rep = (rr[u].y != kUnknownA) ? m : 0u;
      uint32_t x = ww[u], a_rep = rr[u].y;
      const uint32_t key_u = (rr[u].x != kSelf) ? rr[u].x : (0x80000000u | (unsigned)lane);
      if (AGG || __any_sync(kFull, key_u == __shfl_xor_sync(kFull, key_u, 1))) {  // adaptive merge
        m = __match_any_sync(kFull, rr[u].x);
        x = __reduce_add_sync(m, ww[u]);
        rep = __ballot_sync(kFull, rr[u].y != kUnknownA) & m;
        a_rep = __shfl_sync(kFull, rr[u].y, rep ? __ffs(rep) - 1 : lane);
      }
      bool claimed = false;
      if (rr[u].x != kSelf && lane == __ffs(m) - 1) {
        const int32_t c = (int32_t)rr[u].x;
        const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
        uint32_t hq = hash_slot(c, cap);
        for (uint32_t probes = 0;; ++probes) {
          const unsigned long long old = atomicCAS(&T[hq], kEmpty, key | x);
          if (old == kEmpty) { claimed = true; break; }
          if ((old >> 32) == (unsigned long long)(uint32_t)c) {
            atomicAdd(&T[hq], (unsigned long long)x);
            break;
          }
          hq = (hq + 1 == cap) ? 0 : hq + 1;
          if (probes >= cap) { hq = 0xFFFFFFFFu; break; }  // full table (only possible when counting)
        }
        if (rep && hq != 0xFFFFFFFFu) TA[hq] = a_rep;
      }
      if (count) claims += __popc(__ballot_sync(kFull, claimed));
    }
  }
  return claims;
}

// Streaming variant for vertices with P <= kStreamMaxP (the default for them):
// task p streams all of v's staged labels (an L2-resident segment, read P times)
// and keeps only the labels with part_of(c, P) == p; each warp compacts its
// matching entries into a shared queue (ballot + popc) and inserts 32 at a time.
// Measured faster than pre-partitioning at C5 level 0 (15 vs 24 ms), slower for
// the giant hubs of the contracted levels, which take the pre-partitioned tasks.
template <bool UNIT>
__global__ void __launch_bounds__(1024) sweep_part_stream(const int32_t* __restrict__ task_vpos,
                                                  const int32_t* __restrict__ task_p, int64_t t_begin, int64_t t_end,
                                                  const int32_t* __restrict__ vert_pos,
                                                  const int32_t* __restrict__ vert_P,
                                                  const int32_t* __restrict__ vert_first, int32_t* done,
                                                  Partial* part, unsigned long long* overflow,
                                                  const int32_t* __restrict__ bv, const int64_t* __restrict__ soff,
                                                  const uint2* __restrict__ stage, SweepArgs A) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + kPartSlots);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  __shared__ int is_last;
  __shared__ unsigned claimed;
  __shared__ uint2 qbuf[32][64];
  __shared__ uint32_t qwt[32][64];
  for (int t = threadIdx.x; t < kPartSlots; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  if (threadIdx.x == 0) claimed = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  for (int64_t task = t_begin + blockIdx.x; task < t_end; task += gridDim.x) {
    const int32_t vi = task_vpos[task];
    const uint32_t p = (uint32_t)task_p[task];
    const int32_t pos = vert_pos[vi];
    const uint32_t P = (uint32_t)vert_P[vi];
    const int32_t v = __ldg(&bv[pos]);
    const int64_t sb = __ldg(&soff[pos]), deg = __ldg(&soff[pos + 1]) - sb;
    const uint2* S = stage + sb;
    const uint32_t* Wt = UNIT ? nullptr : A.w + __ldg(&A.rowptr[v]);
    // table sized to the task: ~2x its expected labels (deg / P) + slack, so the
    // scan visits ~2 slots per label instead of all kPartSlots (C5 level 0: the
    // full-table scans were most of this kernel's work)
    const uint32_t cap = (uint32_t)min((int64_t)kPartSlots, 2 * ((deg + P - 1) / P) + 512);
    const unsigned limit = cap / 8 * 7;
    // Only ~1/P of the streamed entries belong to this task: each warp compacts
    // the matching entries into a shared queue (ballot + popc) and inserts them
    // 32 at a time, so the insert code runs with full warps.
    uint2* Q = qbuf[threadIdx.x >> 5];
    uint32_t* QW = qwt[threadIdx.x >> 5];
    int qn = 0;  // warp-uniform queue length
    auto insert_one = [&](uint2 e, uint32_t x) {
      const int32_t c = (int32_t)e.x;
      const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
      uint32_t h = hash_slot(c, cap);
      for (;;) {
        const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
        if (old == kEmpty) {
          if (atomicAdd(&claimed, 1u) >= limit) atomicAdd(overflow, 1ull);
          break;
        }
        if ((old >> 32) == (unsigned long long)(uint32_t)c) {
          atomicAdd(&T[h], (unsigned long long)x);
          break;
        }
        h = (h + 1 == cap) ? 0 : h + 1;
        if (claimed >= cap - 1) {
          atomicAdd(overflow, 1ull);
          break;
        }
      }
      if (e.y != kUnknownA) TA[h] = e.y;
    };
    // a full warp inserts its 32 queued entries (lanes >= n idle); equal labels are
    // merged first when adjacent lanes share one (hot labels of later sweeps)
    auto insert_warp = [&](uint2 e, uint32_t x, bool valid) {
      const uint32_t key = valid ? e.x : (0x80000000u | (unsigned)lane);
      if (__any_sync(kFull, key == __shfl_xor_sync(kFull, key, 1))) {
        const unsigned m = __match_any_sync(kFull, key);
        const uint32_t sx = __reduce_add_sync(m, x);
        const unsigned rep = __ballot_sync(kFull, valid && e.y != kUnknownA) & m;
        const uint32_t a_rep = __shfl_sync(kFull, e.y, rep ? __ffs(rep) - 1 : lane);
        if (valid && lane == __ffs(m) - 1) insert_one(make_uint2(e.x, rep ? a_rep : kUnknownA), sx);
      } else if (valid) {
        insert_one(e, x);
      }
    };
    for (int64_t base = 0; base + (int64_t)(threadIdx.x - lane) < deg; base += 4 * (int64_t)blockDim.x) {
      uint2 rr[4];
      uint32_t ww[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + threadIdx.x + (int64_t)q * blockDim.x;
        rr[q] = (t < deg) ? __ldcg(&S[t]) : make_uint2(kSelf, 0u);
        ww[q] = UNIT ? 1u : ((t < deg) ? __ldcg(&Wt[t]) : 0u);
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const bool valid = rr[q].x != kSelf && part_of((int32_t)rr[q].x, P) == p;
        const unsigned m = __ballot_sync(kFull, valid);
        if (valid) {
          const int slot = qn + __popc(m & lanemask_lt());
          Q[slot] = rr[q];
          QW[slot] = ww[q];
        }
        qn += __popc(m);
        if (qn >= 32) {
          __syncwarp();
          insert_warp(Q[lane], QW[lane], true);
          const uint2 mv = (lane < qn - 32) ? Q[32 + lane] : make_uint2(0, 0);
          const uint32_t mw = (lane < qn - 32) ? QW[32 + lane] : 0u;
          __syncwarp();
          if (lane < qn - 32) {
            Q[lane] = mv;
            QW[lane] = mw;
          }
          qn -= 32;
          __syncwarp();
        }
      }
    }
    __syncwarp();
    insert_warp(lane < qn ? Q[lane] : make_uint2(0u, kUnknownA), lane < qn ? QW[lane] : 0u, lane < qn);
    __syncthreads();
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_table(T, TA, cap, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x == 0) {
      part[task] = Partial{s, cb, eown};
      __threadfence();
      is_last = (atomicAdd(&done[vi], 1) == (int)P - 1);
      claimed = 0;
    }
    __syncthreads();
    if (is_last && threadIdx.x < 32) {
      __threadfence();
      s = (long long)0x8000000000000000ull;
      cb = 0x7FFFFFFF;
      eown = 0;
      const int32_t f = vert_first[vi];
      for (uint32_t q = threadIdx.x; q < P; q += 32) {
        const longlong2 raw = __ldcg(reinterpret_cast<const longlong2*>(&part[f + q]));
        const long long ps = raw.x;
        const int pc = (int)(raw.y & 0xFFFFFFFFll);
        const unsigned pe = (unsigned)((unsigned long long)raw.y >> 32);
        if (better(ps, pc, s, cb)) { s = ps; cb = pc; }
        eown += pe;
      }
      group_reduce<32>(s, cb, eown);
      int32_t tgt = own;
      if (threadIdx.x == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
      log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
}


// Hub vertices of the label-partitioned path (the streaming ones, deg >= kSub5Min)
// with a per-CTA table in global memory instead of P label partitions: each CTA
// takes the next vertex (dynamic, the plan lists them by degree, descending),
// inserts its staged labels once into a 2*deg-slot region of its own (4-slot
// buckets, gtable_insert4: one L2 round trip per insert), scans and clears it.
// The live regions of all CTAs (~148 x 2 x deg x 12 B) stay in L2.  Replaces the
// P-fold streaming of sweep_part_stream (ncu, C5 level 0: 8.6e9 instructions,
// issue-bound) -- but measured 4x slower (see gtab_on); off by default.
template <bool UNIT, bool AGG>
__global__ void __launch_bounds__(512) sweep_gtab(const int32_t* __restrict__ vert_pos, int64_t v_begin,
                                                  int64_t v_end, unsigned* next, const int32_t* __restrict__ bv,
                                                  const int64_t* __restrict__ soff, const uint2* __restrict__ stage,
                                                  SweepArgs A, unsigned long long* gT, uint32_t* gTA,
                                                  int64_t region) {
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  __shared__ int64_t sh_vi;
  unsigned long long* T = gT + (int64_t)blockIdx.x * region;
  uint32_t* TA = gTA + (int64_t)blockIdx.x * region;
  for (;;) {
    if (threadIdx.x == 0) sh_vi = v_begin + (int64_t)atomicAdd(next, 1u);
    __syncthreads();
    const int64_t vi = sh_vi;
    if (vi >= v_end) break;
    const int32_t pos = vert_pos[vi];
    const int32_t v = __ldg(&bv[pos]);
    const int64_t sb = __ldg(&soff[pos]), deg = __ldg(&soff[pos + 1]) - sb;
    const uint32_t cap = (uint32_t)(((2 * deg + 3) / 4) * 4);
    insert_staged<UNIT, AGG, true>(T, TA, cap, stage + sb, UNIT ? nullptr : A.w + __ldg(&A.rowptr[v]), deg,
                                   threadIdx.x, blockDim.x);
    __syncthreads();
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_table<true>(T, TA, cap, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x < 32) {
      int32_t tgt = own;
      if (threadIdx.x == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
      log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
}

// Cluster variant of the streaming tasks (LV_CLU=1, experiment): a cluster of kCluCS CTAs
// takes kCluCS consecutive partitions p0 .. p0+kCluCS-1 of one vertex.  Every
// CTA streams 1/kCluCS of the vertex's staged labels and inserts each label of
// those partitions into the table of the CTA that owns it, through distributed
// shared memory (one remote CAS per distinct label), so the vertex's list is read
// ceil(P / kCluCS) times instead of P times.  After a cluster barrier each CTA
// scans its own table exactly like sweep_part_stream and the CTA finishing v's
// last partition reduces the partials.
constexpr int kCluCS = 8;
template <bool UNIT>
__global__ void __launch_bounds__(1024, 1) sweep_part_clu(const int32_t* __restrict__ grp_vi,
                                                          const int32_t* __restrict__ grp_p0, int64_t g_begin,
                                                          int64_t g_end, const int32_t* __restrict__ vert_pos,
                                                          const int32_t* __restrict__ vert_P,
                                                          const int32_t* __restrict__ vert_first, int32_t* done,
                                                          Partial* part, unsigned long long* overflow,
                                                          const int32_t* __restrict__ bv,
                                                          const int64_t* __restrict__ soff,
                                                          const uint2* __restrict__ stage, SweepArgs A) {
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  const unsigned rank = cl.block_rank();
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + kPartSlots);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  __shared__ int is_last;
  for (int t = threadIdx.x; t < kPartSlots; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  cl.sync();  // every table of the cluster is initialised before remote inserts
  const int lane = threadIdx.x & 31;
  const int64_t ncl = gridDim.x / kCluCS, cid = blockIdx.x / kCluCS;
  for (int64_t g = g_begin + cid; g < g_end; g += ncl) {
    const int32_t vi = grp_vi[g];
    const uint32_t p0 = (uint32_t)grp_p0[g];
    const int32_t pos = vert_pos[vi];
    const uint32_t P = (uint32_t)vert_P[vi];
    const int32_t v = __ldg(&bv[pos]);
    const int64_t sb = __ldg(&soff[pos]), deg = __ldg(&soff[pos + 1]) - sb;
    // table size of this group: 2x the expected labels per partition + slack
    const uint32_t cap = (uint32_t)min((int64_t)kPartSlots, 2 * ((deg + P - 1) / P) + 512);
    const uint2* S = stage + sb;
    const uint32_t* Wt = UNIT ? nullptr : A.w + __ldg(&A.rowptr[v]);
    const int64_t lo = deg * rank / kCluCS, hi = deg * (rank + 1) / kCluCS;
    for (int64_t base = lo; base + (int64_t)(threadIdx.x - lane) < hi; base += 4 * (int64_t)blockDim.x) {
      uint2 rr[4];
      uint32_t ww[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int64_t t = base + threadIdx.x + (int64_t)q * blockDim.x;
        rr[q] = (t < hi) ? __ldcg(&S[t]) : make_uint2(kSelf, 0u);
        ww[q] = UNIT ? 1u : ((t < hi) ? __ldcg(&Wt[t]) : 0u);
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t d = (rr[q].x != kSelf) ? part_of((int32_t)rr[q].x, P) - p0 : 0xFFFFFFFFu;
        bool keep = d < (uint32_t)kCluCS;
        uint32_t x = ww[q], arep = rr[q].y;
        // equal labels of a warp are merged first when adjacent lanes share one
        const uint32_t key = keep ? rr[q].x : (0x80000000u | (unsigned)lane);
        if (__any_sync(kFull, key == __shfl_xor_sync(kFull, key, 1))) {
          const unsigned m = __match_any_sync(kFull, key);
          x = __reduce_add_sync(m, x);
          const unsigned rep = __ballot_sync(kFull, keep && rr[q].y != kUnknownA) & m;
          arep = __shfl_sync(kFull, rr[q].y, rep ? __ffs(rep) - 1 : lane);
          if (!rep) arep = kUnknownA;
          keep = keep && lane == __ffs(m) - 1;
        }
        if (!keep) continue;
        unsigned long long* Tr = cl.map_shared_rank(T, d);
        const unsigned long long kx = ((unsigned long long)rr[q].x << 32) | x;
        uint32_t h = hash_slot((int32_t)rr[q].x, cap);
        uint32_t probes = 0;
        for (;;) {
          const unsigned long long old = atomicCAS(&Tr[h], kEmpty, kx);
          if (old == kEmpty) break;
          if ((uint32_t)(old >> 32) == rr[q].x) {
            atomicAdd(&Tr[h], (unsigned long long)x);
            break;
          }
          h = (h + 1 == cap) ? 0u : h + 1;
          if (++probes >= cap) {  // table full: cannot happen at the planned load; reported as an error
            atomicAdd(overflow, 1ull);
            break;
          }
        }
        if (arep != kUnknownA) cl.map_shared_rank(TA, d)[h] = arep;
      }
    }
    cl.sync();  // all inserts into every table of the cluster are done
    const uint32_t p = p0 + rank;
    if (p < P) {
      const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
      const uint32_t ki = __ldg(&A.k[v]);
      const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
      long long s = (long long)0x8000000000000000ull;
      int cb = 0x7FFFFFFF;
      unsigned eown = 0;
      scan_table(T, TA, cap, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);
      block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
      const int32_t f = vert_first[vi];
      if (threadIdx.x == 0) {
        part[f + p] = Partial{s, cb, eown};
        __threadfence();
        is_last = (atomicAdd(&done[vi], 1) == (int)P - 1);
      }
      __syncthreads();
      if (is_last && threadIdx.x < 32) {
        __threadfence();
        s = (long long)0x8000000000000000ull;
        cb = 0x7FFFFFFF;
        eown = 0;
        for (uint32_t q = threadIdx.x; q < P; q += 32) {
          const longlong2 raw = __ldcg(reinterpret_cast<const longlong2*>(&part[f + q]));
          const long long ps = raw.x;
          const int pc = (int)(raw.y & 0xFFFFFFFFll);
          const unsigned pe = (unsigned)((unsigned long long)raw.y >> 32);
          if (better(ps, pc, s, cb)) { s = ps; cb = pc; }
          eown += pe;
        }
        group_reduce<32>(s, cb, eown);
        int32_t tgt = own;
        if (threadIdx.x == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
        log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
      }
    }
    cl.sync();  // every table is scanned (and cleared) before the next group's inserts
  }
}

// Task (v, p) of the plan: inserts the partition's pre-scattered entries
// (S2[poff[p] .. poff[p+1])) into a smem table of 2 * n_p slots (n_p = entries >=
// distinct labels: load <= 1/2, no overflow possible) -- or kPartSlots with a
// distinct-label count when the partition is larger (passing 7/8 load sets
// DevCtl::overflow; expected load <= 3/8) -- scans it, and the CTA finishing v's
// last task reduces the P partials and decides.  (Measured on C5: one CTA walking
// all partitions of a vertex was 20% slower than independent tasks.)
template <bool UNIT, bool AGG>
__global__ void __launch_bounds__(1024) sweep_part(const int32_t* __restrict__ task_vpos,
                                                  const int32_t* __restrict__ task_p, int64_t t_begin, int64_t t_end,
                                                  const int32_t* __restrict__ vert_pos,
                                                  const int32_t* __restrict__ vert_P,
                                                  const int32_t* __restrict__ vert_first,
                                                  const int64_t* __restrict__ vert_pbase,
                                                  const int64_t* __restrict__ poff, int32_t* done, Partial* part,
                                                  unsigned long long* overflow, const int32_t* __restrict__ bv,
                                                  const uint2* __restrict__ S2, const uint32_t* __restrict__ W2,
                                                  SweepArgs A) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + kPartSlots);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  __shared__ int is_last;
  __shared__ unsigned claimed;
  for (int t = threadIdx.x; t < kPartSlots; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  if (threadIdx.x == 0) claimed = 0;
  __syncthreads();
  const unsigned limit = (unsigned)(kPartSlots / 8 * 7);
  for (int64_t task = t_begin + blockIdx.x; task < t_end; task += gridDim.x) {
    const int32_t vi = task_vpos[task];
    const int32_t p = task_p[task];
    const int32_t pos = vert_pos[vi];
    const uint32_t P = (uint32_t)vert_P[vi];
    const int32_t v = __ldg(&bv[pos]);
    const int64_t pb = vert_pbase[vi];
    const int64_t q0 = poff[pb + p], q1 = poff[pb + p + 1];
    const int64_t n_p = q1 - q0;
    const bool big = 2 * n_p > kPartSlots;
    const uint32_t cap = big ? (uint32_t)kPartSlots : (uint32_t)(n_p > 0 ? 2 * n_p : 1);
    const unsigned cl = part_insert<UNIT, AGG>(T, TA, cap, S2, UNIT ? nullptr : W2, q0, q1, big);
    if (big && (threadIdx.x & 31) == 0 && cl) atomicAdd(&claimed, cl);
    __syncthreads();
    if (big && threadIdx.x == 0) {
      if (claimed > limit) atomicAdd(overflow, 1ull);
      claimed = 0;
    }
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    scan_table(T, TA, cap, threadIdx.x, blockDim.x, own, own_single, ki, A, s, cb, eown);  // clears the slots
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x == 0) {
      part[task] = Partial{s, cb, eown};
      __threadfence();
      is_last = (atomicAdd(&done[vi], 1) == (int)P - 1);
    }
    __syncthreads();
    if (is_last && threadIdx.x < 32) {
      __threadfence();
      s = (long long)0x8000000000000000ull;
      cb = 0x7FFFFFFF;
      eown = 0;
      const int32_t f = vert_first[vi];
      for (uint32_t q = threadIdx.x; q < P; q += 32) {
        const longlong2 raw = __ldcg(reinterpret_cast<const longlong2*>(&part[f + q]));
        const long long ps = raw.x;
        const int pc = (int)(raw.y & 0xFFFFFFFFll);
        const unsigned pe = (unsigned)((unsigned long long)raw.y >> 32);
        if (better(ps, pc, s, cb)) { s = ps; cb = pc; }
        eown += pe;
      }
      group_reduce<32>(s, cb, eown);
      int32_t tgt = own;
      if (threadIdx.x == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
      log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------ hubs
// Cooperative kernel over the level's hub plan (lv_internal.cuh HubPlan).
// Phase p: inserts of wave p (ring segment p % 2), table scans of wave p-1
// (segment (p-1) % 2, left clean for wave p+1), decisions of wave p-2 (one
// warp per hub reducing its scan partials).  grid.sync() between phases orders
// everything; all CTAs are co-resident (cooperative launch).
template <bool UNIT>
__global__ void __launch_bounds__(512) hub_coop(const HubItem* __restrict__ ins, const int64_t* __restrict__ ins_off,
                                                const HubItem* __restrict__ scans,
                                                const int64_t* __restrict__ scan_off,
                                                const int64_t* __restrict__ wave_hub,
                                                const HubInfo* __restrict__ info, int64_t nwaves, int64_t seg,
                                                unsigned long long* ring, uint32_t* ring_a, Partial* part,
                                                const uint2* __restrict__ stage, SweepArgs A) {
  cg::grid_group grid = cg::this_grid();
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  const int wpb = blockDim.x >> 5;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int64_t p = 0; p < nwaves + 2; ++p) {
    const int64_t nI = (p < nwaves) ? ins_off[p + 1] - ins_off[p] : 0;
    const int64_t nS = (p >= 1 && p - 1 < nwaves) ? scan_off[p] - scan_off[p - 1] : 0;
    const int64_t nFh = (p >= 2) ? wave_hub[p - 1] - wave_hub[p - 2] : 0;
    const int64_t nF = (nFh + wpb - 1) / wpb;
    for (int64_t it = blockIdx.x; it < nI + nS + nF; it += gridDim.x) {
      if (it < nI) {
        const HubItem item = ins[ins_off[p] + it];
        const HubInfo hi = info[item.hub];
        unsigned long long* T = ring + (p & 1) * seg + hi.off;
        uint32_t* TA = ring_a + (p & 1) * seg + hi.off;
        insert_staged<UNIT, true, true>(T, TA, (uint32_t)hi.cap, stage + hi.sbase + item.begin,
                                        UNIT ? nullptr : A.w + item.begin, item.end - item.begin, threadIdx.x,
                                        blockDim.x);
      } else if (it < nI + nS) {
        const int64_t q = scan_off[p - 1] + (it - nI);
        const HubItem item = scans[q];
        const HubInfo hi = info[item.hub];
        unsigned long long* T = ring + ((p - 1) & 1) * seg + hi.off;
        uint32_t* TA = ring_a + ((p - 1) & 1) * seg + hi.off;
        const int32_t own = (int32_t)__ldg(&A.ca[hi.v]).x;
        const uint32_t ki = __ldg(&A.k[hi.v]);
        const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
        long long s = (long long)0x8000000000000000ull;
        int cb = 0x7FFFFFFF;
        unsigned eown = 0;
        for (int64_t base = item.begin + threadIdx.x; base < item.end; base += 4 * (int64_t)blockDim.x) {
          unsigned long long x[4];
          uint32_t ac[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int64_t t = base + (int64_t)u * blockDim.x;
            x[u] = kEmpty;
            ac[u] = kUnknownA;
            if (t < item.end) {
              x[u] = __ldcg(&T[t]);
              if (x[u] != kEmpty) {
                ac[u] = __ldcg(&TA[t]);
                T[t] = kEmpty;  // clean for wave p+1, which reuses this segment
                TA[t] = kUnknownA;
              }
            }
          }
#pragma unroll
          for (int u = 0; u < 4; ++u)
            if (x[u] != kEmpty && ac[u] == kUnknownA && (int32_t)(x[u] >> 32) != own)
              ac[u] = __ldg(&A.ca[(int32_t)(x[u] >> 32)]).y;
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            if (x[u] == kEmpty) continue;
            const int32_t c = (int32_t)(x[u] >> 32);
            const uint32_t e = (uint32_t)x[u];
            if (c == own) eown = e;
            else consider(c, e, ac[u], own, own_single, ki, A, s, cb);
          }
        }
        block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
        if (threadIdx.x == 0) part[q] = Partial{s, cb, eown};
        __syncthreads();
      } else {
        const int64_t hub = wave_hub[p - 2] + (it - nI - nS) * wpb + warp;
        if (hub < wave_hub[p - 1]) {  // warp-uniform
          const HubInfo hi = info[hub];
          long long s = (long long)0x8000000000000000ull;
          int cb = 0x7FFFFFFF;
          unsigned eown = 0;
          for (int q = lane; q < hi.nscan; q += 32) {
            const Partial pp = part[hi.scan_first + q];
            if (better(pp.s, pp.c, s, cb)) { s = pp.s; cb = pp.c; }
            eown += pp.eown;
          }
          group_reduce<32>(s, cb, eown);
          const int32_t own = (int32_t)__ldg(&A.ca[hi.v]).x;
          int32_t tgt = own;
          if (lane == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, __ldg(&A.k[hi.v]), A);
          log_moves(lane == 0 && tgt != own, hi.v, tgt, A);
        }
      }
    }
    grid.sync();
  }
}

template <class K>
int32_t set_smem(K kernel, size_t bytes) {
  LV_CUDA(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes));
  return LOUVAIN_OK;
}

template <bool UNIT>
int32_t launch_hub(Handle& h, Level& L, const SweepArgs& A, const uint2* stage, int bucket) {
  HubPlan& P = L.hub;
  const int64_t w0 = P.bucket_wave[bucket - 1], w1 = P.bucket_wave[bucket];
  if (w1 <= w0) return LOUVAIN_OK;
  if (!P.grid) {
    int per_sm = 0, nsm = 0;
    LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, hub_coop<UNIT>, 512, 0));
    LV_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, h.device));
    P.grid = std::max(1, per_sm) * nsm;  // cooperative launch: every CTA co-resident
  }
  const HubItem* a0 = P.ins;
  const int64_t* a1 = P.ins_off + w0;  // the bucket's waves only (wave parity is relative: the ring is clean)
  const HubItem* a2 = P.scans;
  const int64_t* a3 = P.scan_off + w0;
  const int64_t* a4 = P.wave_hub + w0;
  const HubInfo* a5 = P.info;
  int64_t a6 = w1 - w0, a7 = P.seg;
  unsigned long long* a8 = P.ring;
  uint32_t* a9 = P.ring_a;
  Partial* a10 = (Partial*)P.partial;
  const uint2* a11 = stage;
  SweepArgs a12 = A;
  void* args[] = {&a0, &a1, &a2, &a3, &a4, &a5, &a6, &a7, &a8, &a9, &a10, &a11, &a12};
  LV_CUDA(cudaLaunchCooperativeKernel((void*)hub_coop<UNIT>, P.grid, 512, args, 0, h.stream));
  LV_LAUNCHED();
  return LOUVAIN_OK;
}

// LV_GTAB=1: per-CTA global tables instead of the single-CTA streaming partition
// tasks.  Measured 4x slower on C5 (level 0: 28.3 -> 111.7 ms per 2 sweeps, with or
// without warp label merging): L2 atomic round trips per label cost far more than
// the P-fold L2 streaming they replace.  Kept as an experiment (parity-tested).
static bool gtab_on() {
  static const bool on = getenv("LV_GTAB") && getenv("LV_GTAB")[0] == '1';
  return on;
}
// Per-CTA global hash regions for sweep_gtab (grow-only, kept clean: every scan
// clears what it visited), plus the dynamic vertex counter.
static int32_t gtab_get(Handle& h, int64_t slots, unsigned long long** T, uint32_t** TA, unsigned** next) {
  void* p = nullptr;
  LV_TRY(scratch_get(h, SC_GTAB, 12 * (size_t)slots + 256, &p));
  size_t have = 0;
  LV_TRY(scratch_size(h, SC_GTAB, &have));
  const int64_t cap_slots = (int64_t)((have - 256) / 12);
  unsigned long long* t = static_cast<unsigned long long*>(p);
  if (h.scratch.gtab_init != p || h.scratch.gtab_init_bytes != have) {  // new or grown: every slot empty once

    LV_CUDA(cudaMemsetAsync(t, 0xFF, 8 * (size_t)cap_slots, h.stream));             // kEmpty
    LV_CUDA(cudaMemsetAsync(t + cap_slots, 0xFF, 4 * (size_t)cap_slots, h.stream));  // kUnknownA
    h.scratch.gtab_init = p;
    h.scratch.gtab_init_bytes = have;
  }
  *T = t;
  *TA = reinterpret_cast<uint32_t*>(t + cap_slots);
  *next = reinterpret_cast<unsigned*>(reinterpret_cast<char*>(p) + 12 * (size_t)cap_slots);
  return LOUVAIN_OK;
}

// LV_CLU=1: cluster (DSMEM) streaming groups instead of single-CTA streaming tasks.
// Measured 2.4x slower on C5 (level 0: 30.7 -> 72.5 ms per 2 sweeps; level 1:
// 14.9 -> 36.9 ms): one remote CAS round trip per label costs more than the
// redundant L2 streaming it saves.  Kept as an experiment (parity-tested).
static bool clu_on() {
  static const bool on = getenv("LV_CLU") && getenv("LV_CLU")[0] == '1';
  return on;
}

// The label-partitioned path of one bucket.  Plan vertices are ordered by degree
// (descending); those with P > kStreamMaxP form a prefix and take the
// pre-partitioned pipeline (histogram -> scan -> scatter -> tasks), the rest
// the streaming tasks.  The partitioned stage lives in contraction-only scratch.
template <bool UNIT, bool AGG>
void launch_part_tasks(Handle& h, Level& L, const SweepArgs& A, int64_t t0, int64_t t1, uint2* S2, uint32_t* W2) {
  PartPlan& Q = L.part;
  sweep_part<UNIT, AGG><<<grid_for(t1 - t0, 1, 148), 1024, 12 * (size_t)kPartSlots, h.stream>>>(
      Q.task_vpos, Q.task_p, t0, t1, Q.vert_pos, Q.vert_P, Q.vert_first, Q.vert_pbase, Q.poff, Q.done,
      (Partial*)Q.partial, &h.ctl->overflow, L.bin_vertices, S2, W2, A);
  LV_LAUNCHED();
}

int32_t launch_part(Handle& h, Level& L, const SweepArgs& A, int bucket, bool unit) {
  PartPlan& Q = L.part;
  const int64_t t0 = Q.bucket_task[bucket - 1], t1 = Q.bucket_task[bucket];
  const int64_t v0 = Q.bucket_vert[bucket - 1], v1 = Q.bucket_vert[bucket];
  const int64_t c0 = Q.bucket_chunk[bucket - 1], c1 = Q.bucket_chunk[bucket];
  const int64_t vs = Q.bucket_vsplit[bucket - 1], ts = Q.bucket_tsplit[bucket - 1];
  if (t1 <= t0) return LOUVAIN_OK;
  cudaStream_t s = h.stream;
  static bool attr = false;
  if (!attr) {
    LV_TRY(set_smem(sweep_part<true, false>, 12 * (size_t)kPartSlots));
    LV_TRY(set_smem(sweep_part<false, false>, 12 * (size_t)kPartSlots));
    LV_TRY(set_smem(sweep_part<true, true>, 12 * (size_t)kPartSlots));
    LV_TRY(set_smem(sweep_part<false, true>, 12 * (size_t)kPartSlots));
    LV_TRY(set_smem(sweep_part_stream<true>, 12 * (size_t)kPartSlots));
    LV_TRY(set_smem(sweep_part_stream<false>, 12 * (size_t)kPartSlots));
    attr = true;
  }
  auto mark = [&](const char* what) {
    if (!trace_on()) return;
    static auto last = std::chrono::steady_clock::now();
    cudaStreamSynchronize(s);
    const auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "[lv]          part %-8s %8.3f ms\n", what, std::chrono::duration<double, std::milli>(now - last).count());
    last = now;
  };
  mark("setup");
  LV_CUDA(cudaMemsetAsync(Q.done + v0, 0, sizeof(int32_t) * (v1 - v0), s));
  const uint2* stage = L.stage;
  if (ts > t0) {  // pre-partitioned prefix: vertices [v0, vs), tasks [t0, ts), chunks [c0, c1)
    void *p2 = nullptr, *pw = nullptr;
    LV_TRY(scratch_get(h, SC_K1, 8 * (size_t)std::max<int64_t>(L.nnz, 1), &p2));
    if (!unit) LV_TRY(scratch_get(h, SC_V0, 4 * (size_t)std::max<int64_t>(L.nnz, 1), &pw));
    uint2* S2 = static_cast<uint2*>(p2);
    uint32_t* W2 = static_cast<uint32_t*>(pw);
    int64_t pb0 = 0, pb1 = Q.npoff;
    if (v0 > 0) LV_CUDA(cudaMemcpyAsync(&pb0, Q.vert_pbase + v0, 8, cudaMemcpyDeviceToHost, s));
    if (vs < Q.nverts) LV_CUDA(cudaMemcpyAsync(&pb1, Q.vert_pbase + vs, 8, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    LV_CUDA(cudaMemsetAsync(Q.poff + pb0, 0, 8 * (size_t)(pb1 - pb0), s));
    k_part_hist<<<grid_for(c1 - c0, 1, 148 * 2), 1024, 0, s>>>(Q.chunks, c0, c1, Q.vert_pos, Q.vert_P, Q.vert_pbase,
                                                                L.soff, stage, Q.poff);
    LV_LAUNCHED();
    mark("hist");
    k_part_scan<<<grid_for(vs - v0, 8, 148 * 4), 256, 0, s>>>(v0, vs, Q.vert_pos, Q.vert_P, Q.vert_pbase, Q.vert_first,
                                                               L.soff, Q.poff, Q.pcur);
    LV_LAUNCHED();
    mark("scan");
    static const char* agg_env = getenv("LV_PART_AGG");
    const bool agg = agg_env ? agg_env[0] == '1' : !unit;  // merging pays off once labels concentrate
    if (unit) {
      k_part_scatter<true><<<grid_for(c1 - c0, 1, 148 * 2), 1024, 0, s>>>(Q.chunks, c0, c1, Q.vert_pos, Q.vert_P,
                                                                          Q.vert_first, L.bin_vertices, L.soff, stage,
                                                                          Q.pcur, S2, W2, A);
      LV_LAUNCHED();
      mark("scatter");
      if (agg) launch_part_tasks<true, true>(h, L, A, t0, ts, S2, W2);
      else launch_part_tasks<true, false>(h, L, A, t0, ts, S2, W2);
    } else {
      k_part_scatter<false><<<grid_for(c1 - c0, 1, 148 * 2), 1024, 0, s>>>(Q.chunks, c0, c1, Q.vert_pos, Q.vert_P,
                                                                           Q.vert_first, L.bin_vertices, L.soff, stage,
                                                                           Q.pcur, S2, W2, A);
      LV_LAUNCHED();
      mark("scatter");
      if (agg) launch_part_tasks<false, true>(h, L, A, t0, ts, S2, W2);
      else launch_part_tasks<false, false>(h, L, A, t0, ts, S2, W2);
    }
    mark("pre-tasks");
  }
  const int64_t g0 = Q.bucket_grp[bucket - 1], g1 = Q.bucket_grp[bucket];
  if (t1 > ts && gtab_on()) {  // streaming vertices [vs, v1): per-CTA global tables (LV_GTAB=1)
    int64_t maxdeg = 0;  // the plan lists vertices by degree, descending: the first is the largest
    {
      int32_t pos = 0;
      int64_t so[2] = {0, 0};
      LV_CUDA(cudaMemcpyAsync(&pos, Q.vert_pos + vs, 4, cudaMemcpyDeviceToHost, s));
      LV_CUDA(cudaStreamSynchronize(s));
      LV_CUDA(cudaMemcpyAsync(so, L.soff + pos, 16, cudaMemcpyDeviceToHost, s));
      LV_CUDA(cudaStreamSynchronize(s));
      maxdeg = so[1] - so[0];
    }
    const int64_t region = ((2 * maxdeg + 3) / 4) * 4;
    static int resident = 0;
    if (resident == 0) {
      int nb = 0;
      LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sweep_gtab<true, false>, 512, 0));
      resident = std::max(nb, 1);
    }
    const int64_t nblk = std::min<int64_t>(148 * resident, v1 - vs);
    unsigned long long* gT = nullptr;
    uint32_t* gTA = nullptr;
    unsigned* next = nullptr;
    LV_TRY(gtab_get(h, nblk * region, &gT, &gTA, &next));
    LV_CUDA(cudaMemsetAsync(next, 0, 4, s));
    static const char* ge = getenv("LV_GTAB_AGG");
    const bool gagg = ge ? ge[0] == '1' : !unit;
    if (unit) {
      if (gagg) sweep_gtab<true, true><<<(unsigned)nblk, 512, 0, s>>>(Q.vert_pos, vs, v1, next, L.bin_vertices, L.soff, stage, A, gT, gTA, region);
      else sweep_gtab<true, false><<<(unsigned)nblk, 512, 0, s>>>(Q.vert_pos, vs, v1, next, L.bin_vertices, L.soff, stage, A, gT, gTA, region);
    } else {
      if (gagg) sweep_gtab<false, true><<<(unsigned)nblk, 512, 0, s>>>(Q.vert_pos, vs, v1, next, L.bin_vertices, L.soff, stage, A, gT, gTA, region);
      else sweep_gtab<false, false><<<(unsigned)nblk, 512, 0, s>>>(Q.vert_pos, vs, v1, next, L.bin_vertices, L.soff, stage, A, gT, gTA, region);
    }
    LV_LAUNCHED();
    mark("stream");
  } else if (t1 > ts && clu_on() && g1 > g0) {  // streaming tasks, cluster variant (LV_CLU=1)
    static bool cattr = false;
    if (!cattr) {
      LV_TRY(set_smem(sweep_part_clu<true>, 12 * (size_t)kPartSlots));
      LV_TRY(set_smem(sweep_part_clu<false>, 12 * (size_t)kPartSlots));
      cattr = true;
    }
    static_assert(kCluCS == kCluGroup, "cluster size must match the plan's group size");
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(1024, 1, 1);
    cfg.dynamicSmemBytes = 12 * (size_t)kPartSlots;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = kCluCS;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    static int max_clu = 0;  // co-resident clusters (GPC packing decides, not 148 / kCluCS)
    if (max_clu == 0) {
      cfg.gridDim = dim3(148 / kCluCS * kCluCS, 1, 1);
      int nc = 0;
      LV_CUDA(cudaOccupancyMaxActiveClusters(&nc, sweep_part_clu<true>, &cfg));
      max_clu = std::max(nc, 1);
    }
    const int64_t nclu = std::min<int64_t>(g1 - g0, max_clu);
    cfg.gridDim = dim3((unsigned)(nclu * kCluCS), 1, 1);
    if (unit)
      LV_CUDA(cudaLaunchKernelEx(&cfg, sweep_part_clu<true>, (const int32_t*)Q.grp_vi, (const int32_t*)Q.grp_p0, g0, g1,
                                 (const int32_t*)Q.vert_pos, (const int32_t*)Q.vert_P, (const int32_t*)Q.vert_first,
                                 Q.done, (Partial*)Q.partial, &h.ctl->overflow, (const int32_t*)L.bin_vertices,
                                 (const int64_t*)L.soff, stage, A));
    else
      LV_CUDA(cudaLaunchKernelEx(&cfg, sweep_part_clu<false>, (const int32_t*)Q.grp_vi, (const int32_t*)Q.grp_p0, g0,
                                 g1, (const int32_t*)Q.vert_pos, (const int32_t*)Q.vert_P,
                                 (const int32_t*)Q.vert_first, Q.done, (Partial*)Q.partial, &h.ctl->overflow,
                                 (const int32_t*)L.bin_vertices, (const int64_t*)L.soff, stage, A));
    LV_LAUNCHED();
    mark("stream");
  } else if (t1 > ts) {  // streaming tasks
    if (unit)
      sweep_part_stream<true><<<grid_for(t1 - ts, 1, 148 * 2), 1024, 12 * (size_t)kPartSlots, s>>>(
          Q.task_vpos, Q.task_p, ts, t1, Q.vert_pos, Q.vert_P, Q.vert_first, Q.done, (Partial*)Q.partial,
          &h.ctl->overflow, L.bin_vertices, L.soff, stage, A);
    else
      sweep_part_stream<false><<<grid_for(t1 - ts, 1, 148 * 2), 1024, 12 * (size_t)kPartSlots, s>>>(
          Q.task_vpos, Q.task_p, ts, t1, Q.vert_pos, Q.vert_P, Q.vert_first, Q.done, (Partial*)Q.partial,
          &h.ctl->overflow, L.bin_vertices, L.soff, stage, A);
    LV_LAUNCHED();
    mark("stream");
  }
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

bool batch_on(const Level& L, int bucket) {
  return L.batch.bstart && L.batch.off[bucket] - L.batch.off[bucket - 1] > 1;
}

// Claimed-slot lists pay where the table is much larger than the distinct count:
// the fixed 512-slot warp tables of bucket 6 (C5 level 0: 10.2 -> 6.3 ms per 2
// sweeps).  The CTA tables are sized 2*deg, where the list measured slower
// (b7 [1024,2048): 12.5 -> 19.4 ms), and so was the 128-slot warp table of bucket 5.
// LV_LIST=0 turns it off; LV_LIST_CTA=1 turns it on for the CTA tiers (A/B only).
static bool use_list() {
  static const bool on = !(getenv("LV_LIST") && getenv("LV_LIST")[0] == '0');
  return on;
}
static bool list_cta() {
  static const bool on = getenv("LV_LIST_CTA") && getenv("LV_LIST_CTA")[0] == '1';
  return on;
}
static bool pipe_on() {
  static const bool on = getenv("LV_CTA_PIPE") && getenv("LV_CTA_PIPE")[0] == '1';
  return on;
}
// largest degree of CTA tier `sub` (lv_internal.cuh)
static int64_t max_deg_of_tier(int sub) {
  static const int64_t ub[5] = {kSub1Min - 1, kSub2Min - 1, kSub3Min - 1, kSub4Min - 1, kSub5Min - 1};
  return ub[sub];
}

template <bool UNIT, bool AGG>
int32_t dispatch_class(Handle& h, Level& L, const SweepArgs& A, int bucket, int sub, int64_t max_deg) {
  const int64_t off = L.class_off[kSubPerBucket * bucket + sub];
  const int64_t nv = L.class_off[kSubPerBucket * bucket + sub + 1] - off;
  if (nv <= 0) return LOUVAIN_OK;
  const int32_t* verts = L.bin_vertices + off;
  const int64_t* soff = L.soff + off;
  const uint2* stage = L.stage;
  cudaStream_t s = h.stream;
  if (sub == 0 && max_deg <= 32) {
    const int G = max_deg <= 4 ? 4 : max_deg <= 8 ? 8 : max_deg <= 16 ? 16 : 32;
    const unsigned grid = grid_for(nv, 8 * (32 / G), 148 * 8);
    switch (G) {
      case 4: sweep_small<4, UNIT><<<grid, 256, 0, s>>>(verts, nv, A); break;
      case 8: sweep_small<8, UNIT><<<grid, 256, 0, s>>>(verts, nv, A); break;
      case 16: sweep_small<16, UNIT><<<grid, 256, 0, s>>>(verts, nv, A); break;
      default: sweep_small<32, UNIT><<<grid, 256, 0, s>>>(verts, nv, A); break;
    }
    LV_LAUNCHED();
  } else if (sub == 0 && batch_on(L, bucket)) {
    static bool battr = false;
    if (!battr) {
      LV_TRY(set_smem(sweep_batch<true>, 12 * (size_t)kBatchSlots));
      LV_TRY(set_smem(sweep_batch<false>, 12 * (size_t)kBatchSlots));
      battr = true;
    }
    const int64_t b0 = L.batch.off[bucket - 1], nb = L.batch.off[bucket] - b0 - 1;  // minus the sentinel
    sweep_batch<UNIT><<<grid_for(nb, 1, 148 * 2), 512, 12 * (size_t)kBatchSlots, s>>>(L.bin_vertices, L.soff,
                                                                                    L.batch.bstart + b0, nb, stage, A);
    LV_LAUNCHED();
  } else if (sub == 0 && max_deg > 84 && max_deg <= 340 && use_list()) {
    sweep_warp_l<512, 352, 4, UNIT><<<grid_for(nv, 4, 148 * 8), 128, 0, s>>>(verts, soff, nv, stage, A);
    LV_LAUNCHED();
  } else if (sub == 0 && max_deg <= 84) {
    sweep_warp<128, 8, UNIT, AGG><<<grid_for(nv, 8, 148 * 8), 256, 0, s>>>(verts, soff, nv, stage, A);
    LV_LAUNCHED();
  } else if (sub == 0 && max_deg <= 340) {
    sweep_warp<512, 4, UNIT, AGG><<<grid_for(nv, 4, 148 * 12), 128, 0, s>>>(verts, soff, nv, stage, A);
    LV_LAUNCHED();
  } else if (sub >= kSubPart) {
    if (sub == kSubPart) LV_TRY(launch_part(h, L, A, bucket, UNIT));  // one pipeline covers sub-classes kSubPart..
    if (sub == kSubHub && L.hub.nh > 0) LV_TRY(launch_hub<UNIT>(h, L, A, stage, bucket));  // giants (P > kPartMaxP)
  } else {
    static const int* caps = kCapT;
    static const int* threads = kThrT;
    static const int* per_sm = kPerSmT;
    const size_t smem = 12 * (size_t)caps[sub];
    static bool attr_done = false;
    if (!attr_done) {
      LV_TRY(set_smem(sweep_cta<true, false>, 12 * (size_t)kCapMax));
      LV_TRY(set_smem(sweep_cta<false, false>, 12 * (size_t)kCapMax));
      LV_TRY(set_smem(sweep_cta<true, true>, 12 * (size_t)kCapMax));
      LV_TRY(set_smem(sweep_cta<false, true>, 12 * (size_t)kCapMax));
      attr_done = true;
    }
    if (list_cta()) {  // claimed-slot list variant (LV_LIST_CTA=1; measured slower on C5, tables are 2*deg here)
      static int resident[5] = {0, 0, 0, 0, 0};
      const int capl = std::min(caps[sub], 16384);
      const int lcap = (int)std::min<int64_t>(capl, max_deg_of_tier(sub));
      const size_t lsmem = 12 * (size_t)capl + 2 * (size_t)((lcap + 7) & ~7);
      static bool lattr = false;
      if (!lattr) {
        LV_TRY(set_smem(sweep_cta_l<true>, 12 * (size_t)16384 + 2 * 12288));
        LV_TRY(set_smem(sweep_cta_l<false>, 12 * (size_t)16384 + 2 * 12288));
        lattr = true;
      }
      if (resident[sub] == 0) {
        int nb = 0;
        LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sweep_cta_l<UNIT>, threads[sub], lsmem));
        resident[sub] = std::max(nb, 1);
      }
      const unsigned lgrid = grid_for(nv, 1, 148 * resident[sub]);
      sweep_cta_l<UNIT><<<lgrid, threads[sub], lsmem, s>>>(verts, soff, nv, stage, A, capl);
      LV_LAUNCHED();
      LV_CUDA(cudaGetLastError());
      return LOUVAIN_OK;
    }
    static const int fnum = [] {  // table size factor 1 + fnum/8 (LV_CAP_F, A/B only)
      const char* e = getenv("LV_CAP_F");
      const int x = e ? atoi(e) : 0;
      return (x >= 2 && x <= 24) ? x : 8;
    }();
    if (!pipe_on()) {
      static int resident[5] = {0, 0, 0, 0, 0};
      const int64_t md = max_deg_of_tier(sub);
      const int capt = (int)std::min<int64_t>(caps[sub], ((md + ((md * fnum) >> 3) + 1 + 31) / 32) * 32);
      if (resident[sub] == 0) {
        int nb = 0;
        LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, sweep_cta<UNIT, AGG>, threads[sub], 12 * (size_t)capt));
        resident[sub] = std::max(nb, 1);
      }
      sweep_cta<UNIT, AGG><<<grid_for(nv, 1, 148 * resident[sub]), threads[sub], 12 * (size_t)capt, s>>>(
          verts, soff, nv, stage, A, capt, fnum);
      LV_LAUNCHED();
      LV_CUDA(cudaGetLastError());
      return LOUVAIN_OK;
    }
    const unsigned grid = grid_for(nv, 1, 148 * per_sm[sub]);
    static const bool pipe = getenv("LV_CTA_PIPE") && getenv("LV_CTA_PIPE")[0] == '1';
    if (pipe) {
      static bool pattr = false;
      if (!pattr) {
        LV_TRY(set_smem(sweep_cta_pipe<true, false>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_pipe<false, false>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_pipe<true, true>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_pipe<false, true>, 12 * (size_t)kCapMax));
        pattr = true;
      }
      sweep_cta_pipe<UNIT, AGG><<<grid, threads[sub], smem, s>>>(verts, soff, nv, stage, A, caps[sub]);
    }
    LV_LAUNCHED();
  }
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

}  // namespace

size_t hub_partial_bytes() { return sizeof(Partial); }

void batch_free(BatchPlan& B, cudaStream_t s) {
  dfree(B.bstart, s);
  B = BatchPlan();
}

// Batch plan (see kBatchSlots): for every bucket whose sub-class 0 is table-based
// (bound > 32), positions where floor((soff[i] - soff[p0] + 32 (i - p0)) / bw)
// changes start a batch; bw keeps every batch's entries <= kBatchSlots / 2.
// Experimental, off by default (LV_BATCH=1): on C5 it measured 2x slower than the
// warp / CTA kernels it replaces (per-batch phases serialise the per-vertex loads).
int32_t build_batch_plan(Handle& h, Level& L, const louvain_params_t& p) {
  cudaStream_t s = h.stream;
  batch_free(L.batch, s);
  static const bool on = getenv("LV_BATCH") && getenv("LV_BATCH")[0] == '1';
  if (!on || L.n == 0) return LOUVAIN_OK;
  BatchPlan& B = L.batch;
  int64_t total = 0;
  for (int b = 1; b <= 7; ++b) {
    const int c = kSubPerBucket * b;
    total += L.class_off[c + 1] - L.class_off[c] + 1;
  }
  LV_TRY(dalloc(&B.bstart, total + 1, s));
  uint8_t* flag = nullptr;
  LV_TRY(dalloc(&flag, std::max<int64_t>(L.n, 1), s));
  int64_t* d_num = reinterpret_cast<int64_t*>(&h.ctl->bad);
  int64_t pos = 0;
  B.off[0] = 0;
  for (int b = 1; b <= 7; ++b) {
    const int c = kSubPerBucket * b;
    const int64_t p0 = L.class_off[c], p1 = L.class_off[c + 1];
    const int64_t hi = (b <= 6) ? p.deg_bounds[b - 1] : INT64_MAX;
    const int64_t max_deg = std::min<int64_t>(hi, kSub1Min - 1);
    if (p1 > p0 && max_deg > 32 && max_deg <= kBatchMaxDeg) {
      const int64_t bw = kBatchSlots / 2 - (max_deg + kBatchVertexWeight);
      k_batch_flags<<<grid_for(p1 - p0, 256), 256, 0, s>>>(L.soff, p0, p1, L.class_soff[c], bw, flag);
      LV_LAUNCHED();
      thrust::counting_iterator<int32_t> it((int32_t)p0);
      size_t tb = 0;
      LV_CUDA(cub::DeviceSelect::Flagged(nullptr, tb, it, flag, B.bstart + pos, d_num, p1 - p0, s));
      void* tmp = nullptr;
      LV_TRY(dmalloc(&tmp, tb, s));
      LV_CUDA(cub::DeviceSelect::Flagged(tmp, tb, it, flag, B.bstart + pos, d_num, p1 - p0, s));
      LV_CUB();
      dfree(tmp, s);
      int64_t cnt = 0;
      LV_CUDA(cudaMemcpyAsync(&cnt, d_num, 8, cudaMemcpyDeviceToHost, s));
      LV_CUDA(cudaStreamSynchronize(s));
      const int32_t end = (int32_t)p1;
      LV_CUDA(cudaMemcpyAsync(B.bstart + pos + cnt, &end, 4, cudaMemcpyHostToDevice, s));
      LV_CUDA(cudaStreamSynchronize(s));  // `end` is a host stack value
      pos += cnt + 1;
    }
    B.off[b] = pos;
  }
  dfree(flag, s);
  LV_CUDA(cudaMemsetAsync(&h.ctl->bad, 0, 8, s));
  return LOUVAIN_OK;
}

// LV_TRACE=2: per-class timing (synchronises the stream; diagnostics only)
static bool trace_on() {
  static const bool on = getenv("LV_TRACE") && std::string(getenv("LV_TRACE")) == "2";
  return on;
}
static void trace_step(Handle& h, Level& L, int bucket, int sub, int64_t pos0, int64_t pos1) {
  static auto last = std::chrono::steady_clock::now();
  cudaStreamSynchronize(h.stream);
  auto now = std::chrono::steady_clock::now();
  const double ms = std::chrono::duration<double, std::milli>(now - last).count();
  last = now;
  if (pos1 <= pos0) return;
  int64_t e[2] = {0, 0};
  cudaMemcpy(&e[0], L.soff + pos0, 8, cudaMemcpyDeviceToHost);
  cudaMemcpy(&e[1], L.soff + pos1, 8, cudaMemcpyDeviceToHost);
  last = std::chrono::steady_clock::now();
  fprintf(stderr, "[lv]        b%d %-5s nv=%-9ld edges=%-11ld %8.3f ms %7.2f Gedge/s\n", bucket,
          sub < 0 ? "stage" : (std::string("sub") + char('0' + sub)).c_str(), (long)(pos1 - pos0),
          (long)(e[1] - e[0]), ms, ms > 0 ? (e[1] - e[0]) / ms / 1e6 : 0.0);
}

// LV_STAGE_A=1: the stage carries a_c for every label (see k_stage), A/B
static bool stage_full_a() {
  static const bool on = getenv("LV_STAGE_A") && getenv("LV_STAGE_A")[0] == '1';
  return on;
}

int32_t launch_stage(Handle& h, Level& L, int64_t pos0, int64_t pos1, int64_t s0, int64_t s1) {
  if (s1 <= s0) return LOUVAIN_OK;
  static const bool wb = getenv("LV_STAGE_WB") && getenv("LV_STAGE_WB")[0] == '1';
  static const bool tiled = !(getenv("LV_STAGE_W") && getenv("LV_STAGE_W")[0] == '1');
  const int64_t* tr = nullptr;
  if (tiled || wb) {  // CTA-tiled variant (default)
    LV_TRY(tile_starts(h, L.soff, pos0, pos1, s0, s1, kStageTile, &tr));
    k_stage<<<grid_for((s1 - s0 + kStageTile - 1) / kStageTile, 1, 148 * 8), 256, 0, h.stream>>>(
        L.bin_vertices, L.soff, pos0, pos1, tr, L.rowptr, L.col, L.ca, L.stage, !wb, stage_full_a());
  } else {
    LV_TRY(tile_starts(h, L.soff, pos0, pos1, s0, s1, kStageChunk, &tr));
    k_stage_w<<<grid_for((s1 - s0 + kStageChunk - 1) / kStageChunk, 8, 148 * 8), 256, 0, h.stream>>>(
        L.bin_vertices, L.soff, pos0, pos1, s0, s1, tr, L.rowptr, L.col, L.ca, L.stage);
  }
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

// All kernels of bucket `bucket` (1..7).  Bucket b's degree range is
// (bounds[b-2], bounds[b-1]] with bounds[-1] = 0 and bounds[6] = inf.
int32_t launch_sweep_bucket(Handle& h, Level& L, const louvain_params_t& p, int bucket) {
  SweepArgs A;
  A.rowptr = L.rowptr;
  A.col = L.col;
  A.w = L.w;
  A.k = L.k;
  A.ca = L.ca;
  A.size = L.size;
  A.W = (long long)L.W;
  A.rule = p.singleton_rule;
  A.mv_v = L.mv_v;
  A.mv_new = L.mv_new;
  A.logn = &h.ctl->logn;
  const int64_t hi = (bucket <= 6) ? p.deg_bounds[bucket - 1] : INT64_MAX;
  static const char* agg_env = getenv("LV_AGG");  // diagnostics: LV_AGG=1 forces warp label merging on
  const bool agg = agg_env && agg_env[0] == '1';
  auto dispatch = [&](int sub) -> int32_t {
    const int64_t max_deg = (sub == 0) ? std::min<int64_t>(hi, kSub1Min - 1) : hi;
    // warp-level label merging (__match_any_sync before the table insert) is
    // off: measured slower at every level and sweep of C5 (profiles/README.md)
    if (L.w) {
      if (agg) LV_TRY((dispatch_class<false, true>(h, L, A, bucket, sub, max_deg)));
      else LV_TRY((dispatch_class<false, false>(h, L, A, bucket, sub, max_deg)));
    } else {
      if (agg) LV_TRY((dispatch_class<true, true>(h, L, A, bucket, sub, max_deg)));
      else LV_TRY((dispatch_class<true, false>(h, L, A, bucket, sub, max_deg)));
    }
    if (trace_on())
      trace_step(h, L, bucket, sub, L.class_off[kSubPerBucket * bucket + sub],
                 L.class_off[kSubPerBucket * bucket + sub + 1]);
    return LOUVAIN_OK;
  };
  // phase 1: gather the records of every neighbour of the bucket's table-based vertices
  const bool sub0_small = std::min<int64_t>(hi, kSub1Min - 1) <= 32;
  const int c0 = kSubPerBucket * bucket + (sub0_small ? 1 : 0), c1 = kSubPerBucket * (bucket + 1);
  const int cp = kSubPerBucket * bucket + kSubPart;  // first label-partitioned class
  const int64_t pos0 = L.class_off[c0], pos1 = L.class_off[c1], posp = L.class_off[cp];
  // The label-partitioned hub classes (issue-bound) run on the side stream,
  // concurrently with the staging (memory-bound) and the CTA tiers of the rest of
  // the bucket: both read only the bucket-start snapshot and append to the move
  // log; the commit waits for both.  LV_OVERLAP=0 serialises.
  static const bool overlap_env = !(getenv("LV_OVERLAP") && getenv("LV_OVERLAP")[0] == '0');
  const bool overlap = overlap_env && !trace_on() && posp < pos1 && posp > pos0 && L.hub.nh == 0;
  if (overlap) {
    LV_TRY(launch_stage(h, L, posp, pos1, L.class_soff[cp], L.class_soff[c1]));
    LV_CUDA(cudaEventRecord(h.ev_fork, h.stream));
    LV_CUDA(cudaStreamWaitEvent(h.side, h.ev_fork, 0));
    cudaStream_t main_s = h.stream;
    h.stream = h.side;
    int32_t rc = LOUVAIN_OK;
    for (int sub = kSubPart; sub < kSubPerBucket && rc == LOUVAIN_OK; ++sub) rc = dispatch(sub);
    h.stream = main_s;
    LV_TRY(rc);
    LV_CUDA(cudaEventRecord(h.ev_join, h.side));
    LV_TRY(launch_stage(h, L, pos0, posp, L.class_soff[c0], L.class_soff[cp]));
    for (int sub = 0; sub < kSubPart; ++sub) LV_TRY(dispatch(sub));
    LV_CUDA(cudaStreamWaitEvent(h.stream, h.ev_join, 0));
    return LOUVAIN_OK;
  }
  if (pos1 > pos0) LV_TRY(launch_stage(h, L, pos0, pos1, L.class_soff[c0], L.class_soff[c1]));
  if (trace_on()) trace_step(h, L, bucket, -1, pos0, pos1);
  for (int sub = 0; sub < kSubPerBucket; ++sub) LV_TRY(dispatch(sub));
  return LOUVAIN_OK;
}

}  // namespace lv
