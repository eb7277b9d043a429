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
// Kernel families (edge-level parallelism, redesigned for
// sm_100a; SURVEY 2.3 K1-K4 counterparts):
//   sweep_small<G>  deg <= 32: G = 4/8/16/32 lanes per vertex, one edge per
//                   lane, duplicate labels merged in registers with
//                   __match_any_sync + __reduce_add_sync (no shared memory).
//   sweep_warp<CAP> deg <= 340: a warp per vertex, per-warp smem hash table
//                   of CAP 64-bit {label|e} slots (single-CAS insert).
//   sweep_cta       deg < 12288: a CTA per vertex (persistent loop), smem
//                   table of min(CAPMAX, 2*deg) slots (64 KB / 128 KB).
//   hub_*           deg >= 12288: one vertex split over many CTAs (chunks of
//                   8192 edges) inserting into a global-memory table, then a
//                   chunked table scan and a per-hub final reduction.
#include <cuda_runtime.h>

#include <algorithm>

#include "lv_device.cuh"
#include "lv_internal.cuh"

namespace lv {
namespace {

struct SweepArgs {
  const int64_t* rowptr;
  const int32_t* col;
  const uint32_t* w;
  const uint32_t* k;
  const int32_t* C;
  const uint32_t* a;
  const int32_t* size;
  long long W;
  int rule;
  int32_t* mv_v;
  int32_t* mv_new;
  unsigned long long* logn;
};

struct Partial {
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

// Candidate c (!= own) with accumulated weight e: fold into (s, cb).
__device__ __forceinline__ void consider(int32_t c, uint32_t e, int32_t own, bool own_single, uint32_t ki,
                                         const SweepArgs& A, long long& s, int& cb) {
  if (A.rule == 2 && own_single && c > own && A.size[c] == 1) return;  // R8 'filter' reading
  long long sc = A.W * (long long)e - (long long)ki * (long long)A.a[c];
  if (better(sc, c, s, cb)) { s = sc; cb = c; }
}

// Stay test and singleton veto.
__device__ __forceinline__ int32_t finish(long long s, int cb, uint32_t eown, int32_t own, uint32_t ki,
                                          const SweepArgs& A) {
  if (cb == 0x7FFFFFFF) return own;
  long long sstay = A.W * (long long)eown - (long long)ki * ((long long)A.a[own] - (long long)ki);
  if (s <= sstay) return own;
  if (A.rule == 1 && cb > own && A.size[own] == 1 && A.size[cb] == 1) return own;  // R8 veto
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
      own = A.C[v];
      ki = __ldg(&A.k[v]);
    }
    const bool has = sub < deg;
    int32_t j = has ? __ldg(&A.col[rb + sub]) : -1;
    uint32_t we = UNIT ? 1u : (has ? __ldg(&A.w[rb + sub]) : 0u);
    const bool valid = has && j != v;  // R3: the self-loop does not count in e
    const int32_t c = valid ? A.C[j] : (int32_t)(0x80000000u | (unsigned)lane);
    const unsigned m = __match_any_sync(kFull, c) & gmask;
    const uint32_t e = UNIT ? (uint32_t)__popc(m) : __reduce_add_sync(m, we);
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    if (valid && lane == __ffs(m) - 1) {
      if (c == own) eown = e;
      else consider(c, e, own, A.rule == 2 && active && A.size[own] == 1, ki, A, s, cb);
    }
    group_reduce<G>(s, cb, eown);
    int32_t t = own;
    if (active && sub == 0) t = finish(s, cb, eown, own, ki, A);
    log_moves(active && sub == 0 && t != own, v, t, A);
  }
}

// ------------------------------------------------------------ warp per vertex
template <int CAP, bool UNIT>
__global__ void __launch_bounds__(256) sweep_warp(const int32_t* __restrict__ verts, int64_t nv, SweepArgs A) {
  __shared__ unsigned long long tab[8][CAP];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  unsigned long long* T = tab[wl];
  for (int t = lane; t < CAP; t += 32) T[t] = kEmpty;
  __syncwarp();
  const int64_t warps = (int64_t)gridDim.x * 8;
  for (int64_t vi = (int64_t)blockIdx.x * 8 + wl; vi < nv; vi += warps) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&A.rowptr[v]);
    const int32_t deg = (int32_t)(__ldg(&A.rowptr[v + 1]) - rb);
    const int32_t own = A.C[v];
    const uint32_t ki = __ldg(&A.k[v]);
    for (int32_t t = lane; t < deg; t += 32) {
      const int32_t j = __ldg(&A.col[rb + t]);
      if (j == v) continue;
      table_add(T, CAP, A.C[j], UNIT ? 1u : __ldg(&A.w[rb + t]));
    }
    __syncwarp();
    const bool own_single = A.rule == 2 && A.size[own] == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    for (int t = lane; t < CAP; t += 32) {
      const unsigned long long x = T[t];
      if (x == kEmpty) continue;
      T[t] = kEmpty;
      const int32_t c = (int32_t)(x >> 32);
      const uint32_t e = (uint32_t)x;
      if (c == own) eown = e;
      else consider(c, e, own, own_single, ki, A, s, cb);
    }
    group_reduce<32>(s, cb, eown);
    const int32_t tgt = (lane == 0) ? finish(s, cb, eown, own, ki, A) : own;
    log_moves(lane == 0 && tgt != own, v, tgt, A);
    __syncwarp();
  }
}

// ------------------------------------------------------------ CTA per vertex
template <bool UNIT>
__global__ void __launch_bounds__(1024) sweep_cta(const int32_t* __restrict__ verts, int64_t nv, SweepArgs A, int capmax) {
  extern __shared__ unsigned long long T[];
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  for (int t = threadIdx.x; t < capmax; t += blockDim.x) T[t] = kEmpty;
  __syncthreads();
  for (int64_t vi = blockIdx.x; vi < nv; vi += gridDim.x) {
    const int32_t v = __ldg(&verts[vi]);
    const int64_t rb = __ldg(&A.rowptr[v]);
    const int64_t deg = __ldg(&A.rowptr[v + 1]) - rb;
    const int32_t own = A.C[v];
    const uint32_t ki = __ldg(&A.k[v]);
    const uint32_t cap = (uint32_t)((2 * deg < (int64_t)capmax) ? 2 * deg : (int64_t)capmax);
    for (int64_t t = threadIdx.x; t < deg; t += blockDim.x) {
      const int32_t j = __ldg(&A.col[rb + t]);
      if (j == v) continue;
      table_add(T, cap, A.C[j], UNIT ? 1u : __ldg(&A.w[rb + t]));
    }
    __syncthreads();
    const bool own_single = A.rule == 2 && A.size[own] == 1;
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    for (uint32_t t = threadIdx.x; t < cap; t += blockDim.x) {
      const unsigned long long x = T[t];
      if (x == kEmpty) continue;
      T[t] = kEmpty;
      const int32_t c = (int32_t)(x >> 32);
      const uint32_t e = (uint32_t)x;
      if (c == own) eown = e;
      else consider(c, e, own, own_single, ki, A, s, cb);
    }
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x < 32) {
      const int32_t tgt = (threadIdx.x == 0) ? finish(s, cb, eown, own, ki, A) : own;
      log_moves(threadIdx.x == 0 && tgt != own, v, tgt, A);
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------ hubs
template <bool UNIT>
__global__ void __launch_bounds__(512) hub_insert(const int64_t* __restrict__ chunk, int64_t nchunks,
                                                  const int32_t* __restrict__ hub_v,
                                                  const int64_t* __restrict__ tab_off,
                                                  const int64_t* __restrict__ tab_cap,
                                                  unsigned long long* table, SweepArgs A) {
  for (int64_t q = blockIdx.x; q < nchunks; q += gridDim.x) {
    const int64_t hidx = chunk[3 * q], eb = chunk[3 * q + 1], ee = chunk[3 * q + 2];
    const int32_t v = hub_v[hidx];
    unsigned long long* T = table + tab_off[hidx];
    const uint32_t cap = (uint32_t)tab_cap[hidx];
    for (int64_t e = eb + threadIdx.x; e < ee; e += blockDim.x) {
      const int32_t j = __ldg(&A.col[e]);
      if (j == v) continue;
      table_add(T, cap, A.C[j], UNIT ? 1u : __ldg(&A.w[e]));
    }
  }
}

__global__ void __launch_bounds__(512) hub_scan(const int64_t* __restrict__ scan, int64_t nscan,
                                                const int32_t* __restrict__ hub_v,
                                                const int64_t* __restrict__ tab_off, unsigned long long* table,
                                                Partial* part, SweepArgs A) {
  __shared__ long long sh_s[32];
  __shared__ int sh_c[32];
  __shared__ unsigned sh_e[32];
  for (int64_t q = blockIdx.x; q < nscan; q += gridDim.x) {
    const int64_t hidx = scan[3 * q], sb = scan[3 * q + 1], se = scan[3 * q + 2];
    const int32_t v = hub_v[hidx];
    const int32_t own = A.C[v];
    const uint32_t ki = A.k[v];
    const bool own_single = A.rule == 2 && A.size[own] == 1;
    unsigned long long* T = table + tab_off[hidx];
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    for (int64_t t = sb + threadIdx.x; t < se; t += blockDim.x) {
      const unsigned long long x = T[t];
      if (x == kEmpty) continue;
      T[t] = kEmpty;  // leave the table clean for the next sweep
      const int32_t c = (int32_t)(x >> 32);
      const uint32_t e = (uint32_t)x;
      if (c == own) eown = e;
      else consider(c, e, own, own_single, ki, A, s, cb);
    }
    block_reduce(s, cb, eown, sh_s, sh_c, sh_e);
    if (threadIdx.x == 0) part[q] = Partial{s, cb, eown};
    __syncthreads();
  }
}

__global__ void hub_final(int64_t nh, const int64_t* __restrict__ scan_first, const Partial* __restrict__ part,
                          const int32_t* __restrict__ hub_v, SweepArgs A) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t hidx = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); hidx < nh; hidx += warps) {
    long long s = (long long)0x8000000000000000ull;
    int cb = 0x7FFFFFFF;
    unsigned eown = 0;
    for (int64_t q = scan_first[hidx] + lane; q < scan_first[hidx + 1]; q += 32) {
      Partial p = part[q];
      if (better(p.s, p.c, s, cb)) { s = p.s; cb = p.c; }
      eown += p.eown;
    }
    group_reduce<32>(s, cb, eown);
    const int32_t v = hub_v[hidx];
    const int32_t own = A.C[v];
    const int32_t tgt = (lane == 0) ? finish(s, cb, eown, own, A.k[v], A) : own;
    log_moves(lane == 0 && tgt != own, v, tgt, A);
  }
}

template <bool UNIT>
int32_t dispatch_class(Handle& h, Level& L, const SweepArgs& A, int bucket, int sub, int64_t max_deg) {
  const int64_t off = L.class_off[4 * bucket + sub];
  const int64_t nv = L.class_off[4 * bucket + sub + 1] - off;
  if (nv <= 0) return LOUVAIN_OK;
  const int32_t* verts = L.bin_vertices + off;
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
  } else if (sub == 0 && max_deg <= 84) {
    sweep_warp<128, UNIT><<<grid_for(nv, 8, 148 * 8), 256, 0, s>>>(verts, nv, A);
    LV_LAUNCHED();
  } else if (sub == 0 && max_deg <= 340) {
    sweep_warp<512, UNIT><<<grid_for(nv, 8, 148 * 6), 256, 0, s>>>(verts, nv, A);
    LV_LAUNCHED();
  } else if (sub <= 1) {
    const int cap = (sub == 0) ? kCtaSmallCap : kCtaLargeCap;
    const int threads = (sub == 0) ? 256 : 1024;
    const size_t smem = sizeof(unsigned long long) * (size_t)cap;
    static bool attr_set[2][2] = {{false, false}, {false, false}};
    if (!attr_set[UNIT][sub]) {
      LV_CUDA(cudaFuncSetAttribute(sweep_cta<UNIT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kCtaLargeCap * 8));
      attr_set[UNIT][sub] = true;
    }
    const unsigned grid = grid_for(nv, 1, 148 * (sub == 0 ? 3 : 1));
    sweep_cta<UNIT><<<grid, threads, smem, s>>>(verts, nv, A, cap);
    LV_LAUNCHED();
  } else {
    HubPlan& P = L.hub;
    if (P.nh > 0) {
      hub_insert<UNIT><<<grid_for(P.nchunks, 1, 148 * 4), 512, 0, s>>>(P.chunk, P.nchunks, P.hub_v, P.tab_off,
                                                                       P.tab_cap, P.table, A);
      LV_LAUNCHED();
      hub_scan<<<grid_for(P.nscan, 1, 148 * 4), 512, 0, s>>>(P.scan, P.nscan, P.hub_v, P.tab_off, P.table,
                                                             (Partial*)P.partial, A);
      LV_LAUNCHED();
      hub_final<<<grid_for(P.nh, 8), 256, 0, s>>>(P.nh, P.scan_first, (const Partial*)P.partial, P.hub_v, A);
      LV_LAUNCHED();
    }
  }
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

}  // namespace

size_t hub_partial_bytes() { return sizeof(Partial); }

// All kernels of bucket `bucket` (1..7).  Bucket b's degree range is
// (bounds[b-2], bounds[b-1]] with bounds[-1] = 0 and bounds[6] = inf.
int32_t launch_sweep_bucket(Handle& h, Level& L, const louvain_params_t& p, int bucket) {
  SweepArgs A;
  A.rowptr = L.rowptr;
  A.col = L.col;
  A.w = L.w;
  A.k = L.k;
  A.C = L.C;
  A.a = L.a;
  A.size = L.size;
  A.W = (long long)L.W;
  A.rule = p.singleton_rule;
  A.mv_v = L.mv_v;
  A.mv_new = L.mv_new;
  A.logn = &h.ctl->logn;
  const int64_t hi = (bucket <= 6) ? p.deg_bounds[bucket - 1] : INT64_MAX;
  for (int sub = 0; sub < 3; ++sub) {
    int64_t max_deg = hi;
    if (sub == 0) max_deg = std::min<int64_t>(hi, kCtaLargeMin - 1);
    if (L.w) LV_TRY(dispatch_class<false>(h, L, A, bucket, sub, max_deg));
    else LV_TRY(dispatch_class<true>(h, L, A, bucket, sub, max_deg));
  }
  return LOUVAIN_OK;
}

}  // namespace lv
