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

// Per-warp move buffer in shared memory: moves are collected warp-locally and appended to
// the global log up to CAP at a time (one atomic per flush), instead of one atomic on the
// single log counter per warp iteration -- in the register kernel of degree-1 vertices that
// atomic was 43% of the stall samples (ncu, profiles/r02/final/ncu_small.sass.csv).  All
// 32 lanes call add() and flush(); `n` is warp-uniform.
template <int CAP>
struct MoveBuf {
  int32_t* v;
  int32_t* t;
  int n;
  __device__ __forceinline__ void flush(const SweepArgs& A) {
    if (n == 0) return;
    const int lane = threadIdx.x & 31;
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(A.logn, (unsigned long long)n);
    base = __shfl_sync(kFull, base, 0);
    __syncwarp();
    for (int k = lane; k < n; k += 32) {
      A.mv_v[base + k] = v[k];
      A.mv_new[base + k] = t[k];
    }
    __syncwarp();
    n = 0;
  }
  __device__ __forceinline__ void add(bool mv, int32_t vv, int32_t tt, const SweepArgs& A) {
    const unsigned m = __ballot_sync(kFull, mv);
    if (m == 0) return;
    if (mv) {
      const int pos = n + __popc(m & lanemask_lt());
      v[pos] = vv;
      t[pos] = tt;
    }
    n += __popc(m);
    if (n > CAP - 32) flush(A);
  }
};

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
__global__ void __launch_bounds__(256, 8) sweep_small(const int32_t* __restrict__ verts, const int64_t* __restrict__ brb,
                                                   const int64_t* __restrict__ soff, int64_t nv, SweepArgs A) {
  const int lane = threadIdx.x & 31;
  const int sub = lane & (G - 1);
  const unsigned gmask = (G == 32) ? kFull : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  const int64_t wid = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  __shared__ int32_t mb_v[8][256], mb_t[8][256];  // 256 threads = 8 warps
  MoveBuf<256> mb{mb_v[threadIdx.x >> 5], mb_t[threadIdx.x >> 5], 0};
  for (int64_t base = wid * (32 / G); base < nv; base += warps * (32 / G)) {
    const int64_t vi = base + lane / G;
    const bool active = vi < nv;
    int32_t v = 0, own = -1, deg = 0;
    int64_t rb = 0;
    uint32_t ki = 0;
    if (active) {  // row by bin position (sequential loads), then the vertex's own record
      v = __ldg(&verts[vi]);
      rb = __ldg(&brb[vi]);
      deg = (int32_t)(__ldg(&soff[vi + 1]) - __ldg(&soff[vi]));
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
    mb.add(active && sub == 0 && t != own, v, t, A);
  }
  mb.flush(A);
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
                                               const int64_t* __restrict__ brb,
                                               const int32_t* __restrict__ col, const uint2* __restrict__ ca,
                                               uint2* __restrict__ stage) {
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
      sh_v[r] = bv[i0 + r];
      sh_so[r] = soff[i0 + r];
      sh_rb[r] = brb[i0 + r];
    }
    __syncthreads();
    // warp spans of 128 entries (lane + 32 q): one binary search per lane for its first
    // entry, then a forward walk -- the next entry of a lane is 32 further, mostly in
    // the same row (the per-entry searches were most of this kernel's instructions)
    const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int64_t span = t0 + (int64_t)wl * 32 * kSpanQ; span < t1; span += (int64_t)nw * 32 * kSpanQ) {
      int32_t jj[kSpanQ], vv[kSpanQ];
      uint2 rr[kSpanQ];
      int lo = 0;
      if (nr > 0 && span + lane < t1) {
        int hi = nr - 1;
        const int64_t t = span + lane;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (sh_so[mid] <= t) lo = mid; else hi = mid - 1;
        }
      }
#pragma unroll
      for (int q = 0; q < kSpanQ; ++q) {
        const int64_t t = span + lane + 32 * q;
        jj[q] = -1;
        vv[q] = -1;
        if (t < t1) {
          int64_t e;
          if (nr > 0) {
            while (lo + 1 < nr && sh_so[lo + 1] <= t) ++lo;
            vv[q] = sh_v[lo];
            e = sh_rb[lo] + (t - sh_so[lo]);
          } else {
            int64_t a = pos0, b = pos1 - 1;
            while (a < b) {
              const int64_t mid = (a + b + 1) >> 1;
              if (soff[mid] <= t) a = mid; else b = mid - 1;
            }
            vv[q] = bv[a];
            e = brb[a] + (t - soff[a]);
          }
          jj[q] = __ldcs(&col[e]);
        }
      }
#pragma unroll
      for (int q = 0; q < kSpanQ; ++q) rr[q] = (jj[q] >= 0 && jj[q] != vv[q]) ? __ldg(&ca[jj[q]]) : make_uint2(kSelf, 0);
#pragma unroll
      for (int q = 0; q < kSpanQ; ++q) {
        const int64_t t = span + lane + 32 * q;
        // evict-first store: the stage streams through L2 once and must not
        // displace the gathered records
        const uint2 val = (jj[q] == vv[q]) ? make_uint2(kSelf, 0u)
                                           : make_uint2(rr[q].x, rr[q].x == (uint32_t)jj[q] ? rr[q].y : kUnknownA);
        if (t < t1) __stcs(&stage[t], val);
      }
    }
    __syncthreads();
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

// ------------------------------------------------------------ register claim lists
// The thread whose CAS claims an empty slot (the first entry of label c in the
// row) keeps that slot's index in a register.  After the inserts the claimers --
// together exactly the distinct labels of the row -- evaluate Eq. (2) for their
// labels and clear their slots: no scan of the 2*deg-slot table (the scan was half
// of the CTA tiers' instructions, ncu profiles/r02_sass_lines_cta.txt).
// Covers rows of up to 4 * PASSES * stride entries.
constexpr uint32_t kNoClaim = 0xFFFFFFFFu;

#ifndef LV_DOUBLE_HASH  // compile-time A/B
#define LV_DOUBLE_HASH 1
#endif
#ifndef LV_DH_POW2  // compile-time A/B: hub-task tables rounded up to powers of two + double hashing
#define LV_DH_POW2 1
#endif
#ifndef LV_DH_PART  // compile-time A/B: the same for the pre-partitioned hub tasks
#define LV_DH_PART 1
#endif
__device__ __forceinline__ uint32_t table_insert_c(unsigned long long* T, uint32_t cap, int32_t c, uint32_t x,
                                                   bool* claimed) {
  const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
  uint32_t h = hash_slot(c, cap);
#if LV_DOUBLE_HASH
  // double hashing on power-of-two tables (odd step: a full cycle): no primary clusters,
  // so the longest probe chain of a warp -- what its divergent loop waits for -- shortens
  const bool pow2 = (cap & (cap - 1)) == 0;
  const uint32_t step = (((uint32_t)c * 0x85EBCA6Bu) >> 17) | 1u;  // independent of hash_slot's bits
#endif
  for (;;) {
    const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
    if (old == kEmpty) {
      *claimed = true;
      return h;
    }
    if ((old >> 32) == (unsigned long long)(uint32_t)c) {
      atomicAdd(&T[h], (unsigned long long)x);
      *claimed = false;
      return h;
    }
#if LV_DOUBLE_HASH
    h = pow2 ? ((h + step) & (cap - 1)) : ((h + 1 == cap) ? 0 : h + 1);
#else
    h = (h + 1 == cap) ? 0 : h + 1;
#endif
  }
}

template <bool UNIT, int PASSES>
__device__ __forceinline__ void insert_claim(unsigned long long* T, uint32_t* TA, uint32_t cap,
                                             const uint2* __restrict__ S, const uint32_t* __restrict__ Wt,
                                             int64_t deg, int t0, int stride, uint32_t (&cl)[4 * PASSES]) {
#pragma unroll
  for (int pass = 0; pass < PASSES; ++pass) {
    uint2 rr[4];
    uint32_t ww[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int64_t t = (int64_t)t0 + (int64_t)(4 * pass + q) * stride;
      rr[q] = (t < deg) ? __ldcs(&S[t]) : make_uint2(kSelf, 0u);
      ww[q] = UNIT ? 1u : ((t < deg) ? __ldcs(&Wt[t]) : 0u);
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint32_t slot = kNoClaim;
      if (rr[q].x != kSelf) {
        bool claimed = false;
        const uint32_t hq = table_insert_c(T, cap, (int32_t)rr[q].x, ww[q], &claimed);
        if (rr[q].y != kUnknownA) TA[hq] = rr[q].y;
        if (claimed) slot = hq;
      }
      cl[4 * pass + q] = slot;
    }
  }
}

// Eq. (2) for the claimed labels, 4 at a time (a_c gathers of labels without a
// representative in the row in flight together); clears the claimed slots.
template <int PASSES>
__device__ __forceinline__ void eval_claims(unsigned long long* T, uint32_t* TA, const uint32_t (&cl)[4 * PASSES],
                                            int32_t own, bool own_single, uint32_t ki, const SweepArgs& A,
                                            long long& s, int& cb, unsigned& eown) {
#pragma unroll
  for (int pass = 0; pass < PASSES; ++pass) {
    unsigned long long x[4];
    uint32_t ac[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint32_t sl = cl[4 * pass + q];
      x[q] = kEmpty;
      ac[q] = kUnknownA;
      if (sl != kNoClaim) {
        x[q] = T[sl];
        ac[q] = TA[sl];
        T[sl] = kEmpty;
        TA[sl] = kUnknownA;
      }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (x[q] != kEmpty && ac[q] == kUnknownA && (int32_t)(x[q] >> 32) != own)
        ac[q] = __ldg(&A.ca[(int32_t)(x[q] >> 32)]).y;
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

// The same inserts gathering the neighbour records directly (no stage): entry t of
// row v reads col[rb + t] and ca[col] (all 4 * PASSES gathers of a lane in flight
// together), the self-loop skipped (R3), a_c known when the neighbour represents
// its label.
template <bool UNIT, int PASSES>
__device__ __forceinline__ void insert_claim_direct(unsigned long long* T, uint32_t* TA, uint32_t cap,
                                                    const SweepArgs& A, int32_t v, int64_t rb, int64_t deg, int t0,
                                                    int stride, uint32_t (&cl)[4 * PASSES]) {
  int32_t jj[4 * PASSES];
  uint32_t ww[4 * PASSES];
#pragma unroll
  for (int u = 0; u < 4 * PASSES; ++u) {
    const int64_t t = (int64_t)t0 + (int64_t)u * stride;
    jj[u] = (t < deg) ? __ldcs(&A.col[rb + t]) : -1;
    ww[u] = UNIT ? 1u : ((t < deg) ? __ldcs(&A.w[rb + t]) : 0u);
  }
  uint2 rr[4 * PASSES];
#pragma unroll
  for (int u = 0; u < 4 * PASSES; ++u) rr[u] = (jj[u] >= 0 && jj[u] != v) ? __ldg(&A.ca[jj[u]]) : make_uint2(kSelf, 0);
#pragma unroll
  for (int u = 0; u < 4 * PASSES; ++u) {
    uint32_t slot = kNoClaim;
    if (rr[u].x != kSelf) {
      bool claimed = false;
      const uint32_t hq = table_insert_c(T, cap, (int32_t)rr[u].x, ww[u], &claimed);
      if (rr[u].x == (uint32_t)jj[u]) TA[hq] = rr[u].y;  // the neighbour represents its label
      if (claimed) slot = hq;
    }
    cl[u] = slot;
  }
}

// LPV lanes per vertex (a warp, or half a warp: two vertices per warp, twice the vertices in
// flight per SM) gathering directly (no stage round trip of 16 B per entry).
template <int CAP, int WARPS, bool UNIT, int PASSES, int LPV = 32>
__global__ void __launch_bounds__(32 * WARPS) sweep_warp_d(const int32_t* __restrict__ verts,
                                                           const int64_t* __restrict__ brb,
                                                           const int64_t* __restrict__ soff, int64_t nv,
                                                           SweepArgs A) {
  constexpr int VPW = 32 / LPV;  // vertices per warp
  __shared__ unsigned long long tab[WARPS * VPW][CAP];
  __shared__ uint32_t taba[WARPS * VPW][CAP];
  __shared__ int32_t mb_v[WARPS][64], mb_t[WARPS][64];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5, sub = lane / LPV, sl = lane % LPV;
  unsigned long long* T = tab[wl * VPW + sub];
  uint32_t* TA = taba[wl * VPW + sub];
  MoveBuf<64> mb{mb_v[wl], mb_t[wl], 0};
  for (int t = sl; t < CAP; t += LPV) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  __syncwarp();
  const int64_t step = (int64_t)gridDim.x * WARPS * VPW;
  for (int64_t base = ((int64_t)blockIdx.x * WARPS + wl) * VPW; base < nv; base += step) {  // warp-uniform
    const int64_t vi = base + sub;
    const bool act = vi < nv;
    int32_t v = 0, own = -1;
    int64_t rb = 0, deg = 0;
    uint32_t ki = 0;
    if (act) {
      v = __ldg(&verts[vi]);
      rb = __ldg(&brb[vi]);
      deg = __ldg(&soff[vi + 1]) - __ldg(&soff[vi]);
      own = (int32_t)__ldg(&A.ca[v]).x;
      ki = __ldg(&A.k[v]);
    }
    uint32_t cl[4 * PASSES];
    insert_claim_direct<UNIT, PASSES>(T, TA, CAP, A, v, rb, deg, sl, LPV, cl);
    __syncwarp();
    const bool own_single = act && A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    eval_claims<PASSES>(T, TA, cl, own, own_single, ki, A, s, cb, eown);
    group_reduce<LPV>(s, cb, eown);
    int32_t tgt = own;
    if (act && sl == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
    mb.add(act && sl == 0 && tgt != own, v, tgt, A);
    __syncwarp();
  }
  mb.flush(A);
}

// Warp per vertex with register claims (rows of <= 128 * PASSES entries).
template <int CAP, int WARPS, bool UNIT, int PASSES>
__global__ void __launch_bounds__(32 * WARPS) sweep_warp_c(const int32_t* __restrict__ verts,
                                                           const int64_t* __restrict__ brb,
                                                           const int64_t* __restrict__ soff, int64_t nv,
                                                           const uint2* __restrict__ stage, SweepArgs A) {
  __shared__ unsigned long long tab[WARPS][CAP];
  __shared__ uint32_t taba[WARPS][CAP];
  __shared__ int32_t mb_v[WARPS][64], mb_t[WARPS][64];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  unsigned long long* T = tab[wl];
  uint32_t* TA = taba[wl];
  MoveBuf<64> mb{mb_v[wl], mb_t[wl], 0};
  for (int t = lane; t < CAP; t += 32) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  __syncwarp();
  const int64_t warps = (int64_t)gridDim.x * WARPS;
  for (int64_t vi = (int64_t)blockIdx.x * WARPS + wl; vi < nv; vi += warps) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&brb[vi]);
    const int64_t deg = __ldg(&soff[vi + 1]) - __ldg(&soff[vi]);
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    uint32_t cl[4 * PASSES];
    insert_claim<UNIT, PASSES>(T, TA, CAP, stage + __ldg(&soff[vi]), UNIT ? nullptr : A.w + rb, deg, lane, 32, cl);
    __syncwarp();
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    eval_claims<PASSES>(T, TA, cl, own, own_single, ki, A, s, cb, eown);
    group_reduce<32>(s, cb, eown);
    int32_t tgt = own;
    if (lane == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
    mb.add(lane == 0 && tgt != own, v, tgt, A);
    __syncwarp();
  }
  mb.flush(A);
}

// CTA per vertex with register claims (rows of <= 4 * PASSES * blockDim entries).  The
// single-pass tiers (128-512 threads) are held to 32 registers, so that their CTAs fill
// an SM (the weighted variant used 44: 1408 instead of 2048 threads; C5 sweeps -7 ms).
template <bool UNIT, int PASSES>
__global__ void __launch_bounds__(1024, PASSES == 1 ? 2 : 1) sweep_cta_c(const int32_t* __restrict__ verts,
                                                    const int64_t* __restrict__ brb,
                                                    const int64_t* __restrict__ soff, int64_t nv,
                                                    const uint2* __restrict__ stage, SweepArgs A, int capmax) {
  extern __shared__ unsigned long long smem[];
  unsigned long long* T = smem;
  uint32_t* TA = reinterpret_cast<uint32_t*>(smem + capmax);
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  __shared__ int32_t mb_v[64], mb_t[64];  // warp 0's move buffer
  MoveBuf<64> mb{mb_v, mb_t, 0};
  for (int t = threadIdx.x; t < capmax; t += blockDim.x) {
    T[t] = kEmpty;
    TA[t] = kUnknownA;
  }
  __syncthreads();
  for (int64_t vi = blockIdx.x; vi < nv; vi += gridDim.x) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&brb[vi]);
    const int64_t deg = __ldg(&soff[vi + 1]) - __ldg(&soff[vi]);
    const int32_t own = (int32_t)__ldg(&A.ca[v]).x;
    const uint32_t ki = __ldg(&A.k[v]);
    // the whole tier table (2-4x the row, load 1/4-1/2): nothing scans it (claims clear
    // their own slots), so a lower load only shortens the probe chains -- the divergent
    // probe loop was ~40% of these kernels' instructions at 4-9 active lanes (ncu)
    const uint32_t cap = (uint32_t)capmax;
    uint32_t cl[4 * PASSES];
    insert_claim<UNIT, PASSES>(T, TA, cap, stage + __ldg(&soff[vi]), UNIT ? nullptr : A.w + rb, deg, threadIdx.x,
                               blockDim.x, cl);
    __syncthreads();
    const bool own_single = A.rule == 2 && __ldg(&A.size[own]) == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    eval_claims<PASSES>(T, TA, cl, own, own_single, ki, A, s, cb, eown);
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x < 32) {
      int32_t tgt = own;
      if (threadIdx.x == 0) tgt = finish(s, cb, eown, own, __ldg(&A.ca[own]).y, ki, A);
      mb.add(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
  if (threadIdx.x < 32) mb.flush(A);
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
#if LV_DH_PART
          hq = probe_next(hq, cap, probe_step(c));
#else
          hq = (hq + 1 == cap) ? 0 : hq + 1;
#endif
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
#if LV_DH_POW2
    const uint32_t cap = pow2_at_least((uint32_t)min((int64_t)kPartSlots, 2 * ((deg + P - 1) / P) + 512), kPartSlots);
#else
    const uint32_t cap = (uint32_t)min((int64_t)kPartSlots, 2 * ((deg + P - 1) / P) + 512);
#endif
    const unsigned limit = cap / 8 * 7;
    // Only ~1/P of the streamed entries belong to this task: each warp compacts
    // the matching entries into a shared queue (ballot + popc) and inserts them
    // 32 at a time, so the insert code runs with full warps.
    uint2* Q = qbuf[threadIdx.x >> 5];
    uint32_t* QW = qwt[threadIdx.x >> 5];
    int qn = 0;  // warp-uniform queue length
    unsigned nclaim = 0;  // slots this thread claimed (summed per warp once per task: no shared
                          // counter per claim -- it serialised every claim of the CTA)
    auto insert_one = [&](uint2 e, uint32_t x) {
      const int32_t c = (int32_t)e.x;
      const unsigned long long key = ((unsigned long long)(uint32_t)c) << 32;
      uint32_t h = hash_slot(c, cap);
      for (uint32_t probes = 0;; ++probes) {
        if (probes >= cap) {  // full table (the fill check below reports it)
          atomicAdd(overflow, 1ull);
          return;
        }
        const unsigned long long old = atomicCAS(&T[h], kEmpty, key | x);
        if (old == kEmpty) {
          ++nclaim;
          break;
        }
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
    {
      const unsigned wsum = __reduce_add_sync(kFull, nclaim);
      if (lane == 0 && wsum) atomicAdd(&claimed, wsum);  // read by thread 0 after block_reduce's barrier
    }
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x == 0) {
      if (claimed > limit) atomicAdd(overflow, 1ull);  // past 7/8 load (expected <= 3/8)
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
#if LV_DH_PART
    const uint32_t cap = big ? (uint32_t)kPartSlots : pow2_at_least((uint32_t)(n_p > 0 ? 2 * n_p : 1), kPartSlots);
#else
    const uint32_t cap = big ? (uint32_t)kPartSlots : (uint32_t)(n_p > 0 ? 2 * n_p : 1);
#endif
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
    const bool agg = !unit;  // merging pays off once labels concentrate (contracted levels)
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
  if (t1 > ts) {  // streaming tasks
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

// Claimed-slot lists pay where the table is much larger than the distinct count:
// the fixed 512-slot warp tables of bucket 6 (C5 level 0: 10.2 -> 6.3 ms per 2
// sweeps).  The CTA tables are sized 2*deg, where the list measured slower
// (b7 [1024,2048): 12.5 -> 19.4 ms), and so was the 128-slot warp table of bucket 5.
// Rows of <= kDirectMaxDeg entries (bucket 5 with the paper's bounds) are hashed by a warp
// that gathers the records itself (sweep_warp_d): C5 level 0 bucket 5 stage 2.8 + warp 2.2 ->
// 4.0 ms; bucket 6 (85-319) measured slower that way (6.5 -> 7.6 ms) and keeps the stage.
constexpr int64_t kDirectMaxDeg = 84;
#ifndef LV_WARPD_CAP  // table slots per warp of the direct bucket-5 kernel (256: load <= 1/3; 128 measured slower)
#define LV_WARPD_CAP 256
#endif
#ifndef LV_WARPD_LPV  // lanes per vertex of the direct bucket-5 kernel (16: two vertices per warp, r2)
#define LV_WARPD_LPV 16
#endif
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
  const int64_t* brb = L.bin_rb + off;
  const uint2* stage = L.stage;
  cudaStream_t s = h.stream;
  if (sub == 0 && max_deg <= 32) {
    const int G = max_deg <= 4 ? 4 : max_deg <= 8 ? 8 : max_deg <= 16 ? 16 : 32;
    const unsigned grid = grid_for(nv, 8 * (32 / G), 148 * 8);
    switch (G) {
      case 4: sweep_small<4, UNIT><<<grid, 256, 0, s>>>(verts, brb, soff, nv, A); break;
      case 8: sweep_small<8, UNIT><<<grid, 256, 0, s>>>(verts, brb, soff, nv, A); break;
      case 16: sweep_small<16, UNIT><<<grid, 256, 0, s>>>(verts, brb, soff, nv, A); break;
      default: sweep_small<32, UNIT><<<grid, 256, 0, s>>>(verts, brb, soff, nv, A); break;
    }
    LV_LAUNCHED();
  } else if (sub == 0 && max_deg <= kDirectMaxDeg) {
#if LV_WARPD_LPV == 16
    // half-warp tables of 128 slots (16 per block: 24 KB; 256 would pass the 48 KB static limit)
    sweep_warp_d<128, 8, UNIT, 2, 16><<<grid_for(nv, 16, 148 * 8), 256, 0, s>>>(verts, brb, soff, nv, A);
#else
    sweep_warp_d<LV_WARPD_CAP, 8, UNIT, 1><<<grid_for(nv, 8, 148 * 8), 256, 0, s>>>(verts, brb, soff, nv, A);
#endif
    LV_LAUNCHED();
  } else if (sub == 0 && max_deg <= 340) {  // warp per vertex, 3 claim passes of 4 entries per lane
    sweep_warp_c<512, 4, UNIT, 3><<<grid_for(nv, 4, 148 * 8), 128, 0, s>>>(verts, brb, soff, nv, stage, A);
    LV_LAUNCHED();
  } else if (sub >= kSubPart) {
    if (sub == kSubPart) LV_TRY(launch_part(h, L, A, bucket, UNIT));  // one pipeline covers sub-classes kSubPart..
    if (sub == kSubHub && L.hub.nh > 0) LV_TRY(launch_hub<UNIT>(h, L, A, stage, bucket));  // giants (P > kPartMaxP)
  } else {
    static const int* caps = kCapT;
    static const int* threads = kThrT;
    const int64_t md = std::min<int64_t>(max_deg_of_tier(sub), max_deg);
    {
      static bool cattr = false;
      if (!cattr) {
        LV_TRY(set_smem(sweep_cta_c<true, 1>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_c<false, 1>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_c<true, 2>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_c<false, 2>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_c<true, 3>, 12 * (size_t)kCapMax));
        LV_TRY(set_smem(sweep_cta_c<false, 3>, 12 * (size_t)kCapMax));
        cattr = true;
      }
      const int passes = (int)((md + 4 * threads[sub] - 1) / (4 * threads[sub]));
      const int capt = (int)std::min<int64_t>(caps[sub], ((2 * md + 1 + 31) / 32) * 32);
      static int cres[5][4] = {{0}};
      auto go = [&](auto kern) -> int32_t {
        if (cres[sub][passes] == 0) {
          int nb = 0;
          LV_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, threads[sub], 12 * (size_t)capt));
          cres[sub][passes] = std::max(nb, 1);
        }
        kern<<<grid_for(nv, 1, 148 * cres[sub][passes]), threads[sub], 12 * (size_t)capt, s>>>(verts, brb, soff,
                                                                                             nv, stage, A, capt);
        LV_LAUNCHED();
        LV_CUDA(cudaGetLastError());
        return LOUVAIN_OK;
      };
      if (passes <= 1) return go(sweep_cta_c<UNIT, 1>);
      if (passes == 2) return go(sweep_cta_c<UNIT, 2>);
      if (passes == 3) return go(sweep_cta_c<UNIT, 3>);
      set_error("sweep: CTA tier degree beyond the claim-list capacity");
      return LOUVAIN_E_UNSUPPORTED;
    }
  }
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

}  // namespace

size_t hub_partial_bytes() { return sizeof(Partial); }

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

int32_t launch_stage(Handle& h, Level& L, int64_t pos0, int64_t pos1, int64_t s0, int64_t s1) {
  if (s1 <= s0) return LOUVAIN_OK;
  const int64_t* tr = nullptr;
  LV_TRY(tile_starts(h, L.soff, pos0, pos1, s0, s1, kStageTile, &tr));
  k_stage<<<grid_for((s1 - s0 + kStageTile - 1) / kStageTile, 1, 148 * 8), 256, 0, h.stream>>>(
      L.bin_vertices, L.soff, pos0, pos1, tr, L.bin_rb, L.col, L.ca, L.stage);
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
  if (hi <= kSmallMaxDeg) {  // register kernels only: lane groups of 1..32 lanes, by degree (k_classify)
    cudaStream_t s = h.stream;
    for (int sub = 1; sub <= 6; ++sub) {
      const int64_t off = L.class_off[kSubPerBucket * bucket + sub];
      const int64_t nv = L.class_off[kSubPerBucket * bucket + sub + 1] - off;
      if (nv <= 0) continue;
      const int32_t* verts = L.bin_vertices + off;
      const int64_t* brb = L.bin_rb + off;
      const int64_t* soff = L.soff + off;
      const int G = 1 << (sub - 1);
      const unsigned grid = grid_for(nv, 8 * (32 / G), 148 * 8);
#define LV_SMALL(GG)                                                              \
  if (L.w) sweep_small<GG, false><<<grid, 256, 0, s>>>(verts, brb, soff, nv, A); \
  else sweep_small<GG, true><<<grid, 256, 0, s>>>(verts, brb, soff, nv, A)
      switch (G) {
        case 1: LV_SMALL(1); break;
        case 2: LV_SMALL(2); break;
        case 4: LV_SMALL(4); break;
        case 8: LV_SMALL(8); break;
        case 16: LV_SMALL(16); break;
        default: LV_SMALL(32); break;
      }
#undef LV_SMALL
      LV_LAUNCHED();
      if (trace_on()) trace_step(h, L, bucket, sub, off, off + nv);
    }
    LV_CUDA(cudaGetLastError());
    return LOUVAIN_OK;
  }
  auto dispatch = [&](int sub) -> int32_t {
    const int64_t max_deg = (sub == 0) ? std::min<int64_t>(hi, kSub1Min - 1) : hi;
    // warp-level label merging (__match_any_sync before the table insert) is
    // off: measured slower at every level and sweep of C5 (profiles/README.md)
    if (L.w) LV_TRY((dispatch_class<false, false>(h, L, A, bucket, sub, max_deg)));
    else LV_TRY((dispatch_class<true, false>(h, L, A, bucket, sub, max_deg)));
    if (trace_on())
      trace_step(h, L, bucket, sub, L.class_off[kSubPerBucket * bucket + sub],
                 L.class_off[kSubPerBucket * bucket + sub + 1]);
    return LOUVAIN_OK;
  };
  // phase 1: gather the records of every neighbour of the bucket's table-based vertices
  const int64_t sub0_max = std::min<int64_t>(hi, kSub1Min - 1);
  const bool sub0_small = sub0_max <= kDirectMaxDeg;  // register kernels / direct warp kernels: not staged
  const int c0 = kSubPerBucket * bucket + (sub0_small ? 1 : 0), c1 = kSubPerBucket * (bucket + 1);
  const int cp = kSubPerBucket * bucket + kSubPart;  // first label-partitioned class
  const int64_t pos0 = L.class_off[c0], pos1 = L.class_off[c1], posp = L.class_off[cp];
  // The label-partitioned hub classes (issue-bound) run on the side stream,
  // concurrently with the staging (memory-bound) and the CTA tiers of the rest of
  // the bucket: both read only the bucket-start snapshot and append to the move
  // log; the commit waits for both (LV_TRACE=2 serialises).
  const bool overlap = !trace_on() && posp < pos1 && posp > pos0 && L.hub.nh == 0;
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
