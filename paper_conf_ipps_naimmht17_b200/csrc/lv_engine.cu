// lv_engine.cu -- C-ABI (include/louvain.h) and the level driver of the GPU
// Louvain hot path: one sweep = Alg. 1's repeat body, the phase
// loop with the threshold schedule (R13-R15), the multilevel loop
// (R16) and label composition (R22).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <tuple>
#include <vector>

#include "lv_internal.cuh"

#define LV_API extern "C" __attribute__((visibility("default")))

namespace lv {

static thread_local std::string g_err;
long long g_launches = 0, g_cub_calls = 0;
void set_error(const std::string& msg) { g_err = msg; }

int32_t cuda_fail(cudaError_t e, const char* what, const char* file, int line) {
  g_err = std::string(what) + ": " + cudaGetErrorString(e) + " (" + file + ":" + std::to_string(line) + ")";
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    return LOUVAIN_E_NOMEM;
  }
  return LOUVAIN_E_CUDA;
}

// Stream-ordered allocations come from a library-private memory pool per device
// (never the device's default pool, which other libraries in the process share):
// it keeps freed blocks (release threshold = max) so per-level temporaries do not
// go back to the driver between levels, and it is trimmed when an allocation fails.
namespace {
std::mutex g_pool_mu;
cudaMemPool_t g_pools[64] = {};
cudaMemPool_t lib_pool(int dev) {
  if (dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (!g_pools[dev]) {
    cudaMemPoolProps pr = {};
    pr.allocType = cudaMemAllocationTypePinned;
    pr.handleTypes = cudaMemHandleTypeNone;
    pr.location.type = cudaMemLocationTypeDevice;
    pr.location.id = dev;
    cudaMemPool_t p = nullptr;
    if (cudaMemPoolCreate(&p, &pr) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
    g_pools[dev] = p;
  }
  return g_pools[dev];
}

// Process-wide cache of the scratch buffers of destroyed handles, so a new handle
// on the same device (e.g. every end-to-end louvain_create_csr + louvain_run)
// reuses device memory instead of paying tens of GB of cudaMalloc again.  Bounded:
// one handle's set per device (scratch_free).  Released on any allocation failure, by
// louvain_release_cache(), or never filled with LV_SCRATCH_CACHE=0.
std::mutex g_cache_mu;
std::vector<std::tuple<int, void*, size_t, int>> g_cache;  // (device, ptr, bytes, scratch slot)
bool cache_on() {
  static const bool on = !(getenv("LV_SCRATCH_CACHE") && getenv("LV_SCRATCH_CACHE")[0] == '0');
  return on;
}
// A buffer that served the same scratch slot before is preferred (handles of one graph
// ask every slot for the same size, so each buffer goes back to its own role), else the
// smallest cached buffer that is large enough.
void* cache_take(int dev, int slot, size_t bytes, size_t* got) {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  int best = -1;
  for (int pass = 0; pass < 2 && best < 0; ++pass) {
    for (int i = 0; i < (int)g_cache.size(); ++i) {
      const auto& c = g_cache[i];
      if (std::get<0>(c) == dev && std::get<2>(c) >= bytes && (pass == 1 || std::get<3>(c) == slot) &&
          (best < 0 || std::get<2>(c) < std::get<2>(g_cache[best])))
        best = i;
    }
  }
  if (best < 0) return nullptr;
  void* p = std::get<1>(g_cache[best]);
  *got = std::get<2>(g_cache[best]);
  g_cache.erase(g_cache.begin() + best);
  return p;
}
void cache_release_locked(int dev) {
  for (auto it = g_cache.begin(); it != g_cache.end();) {
    if (dev < 0 || std::get<0>(*it) == dev) {
      int cur = -1;
      cudaGetDevice(&cur);
      if (cur != std::get<0>(*it)) cudaSetDevice(std::get<0>(*it));
      cudaFree(std::get<1>(*it));
      if (cur >= 0 && cur != std::get<0>(*it)) cudaSetDevice(cur);
      it = g_cache.erase(it);
    } else {
      ++it;
    }
  }
}
void cache_release(int dev) {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  cache_release_locked(dev);
}
// Give memory back after an allocation failure: the scratch cache and the idle
// blocks of the library pool (after the stream's queued frees have run).
void reclaim(int dev, cudaStream_t s) {
  cudaGetLastError();
  cache_release(dev);
  if (cudaMemPool_t p = lib_pool(dev)) {
    if (s) cudaStreamSynchronize(s);
    cudaMemPoolTrimTo(p, 0);
  }
  cudaGetLastError();
}
}  // namespace

int32_t dmalloc(void** p, size_t bytes, cudaStream_t s) {
  *p = nullptr;
  int dev = 0;
  cudaGetDevice(&dev);
  cudaMemPool_t pool = lib_pool(dev);
  auto alloc = [&]() {
    return pool ? cudaMallocFromPoolAsync(p, bytes ? bytes : 1, pool, s) : cudaMallocAsync(p, bytes ? bytes : 1, s);
  };
  cudaError_t e = alloc();
  if (e != cudaSuccess) {  // retry once after giving cached / pooled memory back
    reclaim(dev, s);
    e = alloc();
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    *p = nullptr;
    g_err = "device allocation of " + std::to_string(bytes) + " bytes failed: " + cudaGetErrorString(e);
    return LOUVAIN_E_NOMEM;
  }
  return LOUVAIN_OK;
}

void dfree(void* p, cudaStream_t s) {
  if (p) cudaFreeAsync(p, s);
}

int32_t scratch_size(Handle& h, int slot, size_t* bytes) {
  *bytes = h.scratch.bytes[slot];
  return LOUVAIN_OK;
}

int32_t scratch_get(Handle& h, int slot, size_t bytes, void** out) {
  Scratch& S = h.scratch;
  if (S.bytes[slot] < bytes) {
    if (S.p[slot]) {
      cudaStreamSynchronize(h.stream);  // the old buffer may still be in use by queued work
      cudaFree(S.p[slot]);
      S.p[slot] = nullptr;
      S.bytes[slot] = 0;
    }
    size_t got = 0;
    void* c = cache_on() ? cache_take(h.device, slot, bytes, &got) : nullptr;
    if (c) {
      S.p[slot] = c;
      S.bytes[slot] = got;
    } else {
      const size_t want = bytes + bytes / 8;  // headroom: later levels are usually smaller
      cudaError_t e = cudaMalloc(&S.p[slot], want);
      if (e != cudaSuccess) {  // give cached buffers and pooled stream-ordered memory back, retry once
        reclaim(h.device, h.stream);
        e = cudaMalloc(&S.p[slot], want);
      }
      if (e != cudaSuccess) {
        cudaGetLastError();
        S.p[slot] = nullptr;
        g_err = "scratch allocation of " + std::to_string(want) + " bytes failed: " + cudaGetErrorString(e);
        return LOUVAIN_E_NOMEM;
      }
      S.bytes[slot] = want;
    }
  }
  *out = S.p[slot];
  return LOUVAIN_OK;
}

// Bounded: the cache holds one handle's set per device -- a destroy first frees what an
// earlier handle left unused, then caches its own buffers.  With slot-keyed reuse the next
// handle of the same graph takes every buffer back, so in the end-to-end loop of create /
// run / destroy nothing is left over and a destroy frees nothing.
void scratch_free(Handle& h) {
  std::lock_guard<std::mutex> lk(g_cache_mu);
  if (cache_on()) cache_release_locked(h.device);
  for (int i = 0; i < SC_COUNT; ++i) {
    if (h.scratch.p[i]) {
      if (cache_on()) g_cache.emplace_back(h.device, h.scratch.p[i], h.scratch.bytes[i], i);
      else cudaFree(h.scratch.p[i]);
    }
    h.scratch.p[i] = nullptr;
    h.scratch.bytes[i] = 0;
  }
}

// Control blocks (device DevCtl + its pinned host mirror) of destroyed handles, reused by the
// next handles: a cudaFree / cudaFreeHost per destroy synchronised the device and cost up
// to 0.66 s inside the end-to-end step (LV_TRACE destroy timing).
std::mutex g_ctl_mu;
std::vector<std::tuple<int, DevCtl*, DevCtl*>> g_ctl_free;
bool ctl_take(int dev, DevCtl** d, DevCtl** hh) {
  std::lock_guard<std::mutex> lk(g_ctl_mu);
  for (auto it = g_ctl_free.begin(); it != g_ctl_free.end(); ++it)
    if (std::get<0>(*it) == dev) {
      *d = std::get<1>(*it);
      *hh = std::get<2>(*it);
      g_ctl_free.erase(it);
      return true;
    }
  return false;
}
void ctl_give(int dev, DevCtl* d, DevCtl* hh) {
  std::lock_guard<std::mutex> lk(g_ctl_mu);
  g_ctl_free.emplace_back(dev, d, hh);
}
void ctl_release_all() {
  std::lock_guard<std::mutex> lk(g_ctl_mu);
  for (auto& c : g_ctl_free) {
    int cur = -1;
    cudaGetDevice(&cur);
    cudaSetDevice(std::get<0>(c));
    cudaFree(std::get<1>(c));
    cudaFreeHost(std::get<2>(c));
    if (cur >= 0) cudaSetDevice(cur);
  }
  g_ctl_free.clear();
}

void release_cache_all() {
  ctl_release_all();
  cache_release(-1);
  for (int d = 0; d < 64; ++d) {
    cudaMemPool_t p = nullptr;
    {
      std::lock_guard<std::mutex> lk(g_pool_mu);
      p = g_pools[d];
    }
    if (p) cudaMemPoolTrimTo(p, 0);
  }
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

namespace {

__global__ void k_fill_u32(uint32_t* p, int64_t n, uint32_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}
__global__ void k_iota(int32_t* p, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = (int32_t)i;
}

int32_t check_params(const louvain_params_t& p) {
  if (p.mode != LOUVAIN_MODE_BIN_SYNC && p.mode != LOUVAIN_MODE_RELAXED) {
    set_error("params.mode must be BIN_SYNC (0) or RELAXED (1)");
    return LOUVAIN_E_INVALID_ARG;
  }
  if (p.singleton_rule < 0 || p.singleton_rule > 2) {
    set_error("params.singleton_rule must be 0, 1 or 2");
    return LOUVAIN_E_INVALID_ARG;
  }
  if (p.th_bin_exp < 0 || p.th_bin_exp > 18 || p.th_final_exp < 0 || p.th_final_exp > 18) {
    set_error("threshold exponents must be in [0, 18]");
    return LOUVAIN_E_INVALID_ARG;
  }
  for (int t = 0; t < 6; ++t) {
    if (p.deg_bounds[t] < 1 || (t > 0 && p.deg_bounds[t] <= p.deg_bounds[t - 1])) {
      set_error("deg_bounds must be positive and strictly increasing");
      return LOUVAIN_E_INVALID_ARG;
    }
  }
  return LOUVAIN_OK;
}

int32_t init_handle(Handle& h, void* stream) {
  LV_CUDA(cudaGetDevice(&h.device));
  if (stream) {
    h.stream = (cudaStream_t)stream;
    h.own_stream = false;
  } else {
    LV_CUDA(cudaStreamCreateWithFlags(&h.stream, cudaStreamNonBlocking));
    h.own_stream = true;
  }
  if (!ctl_take(h.device, &h.ctl, &h.h_ctl)) {
    LV_CUDA(cudaMalloc(&h.ctl, sizeof(DevCtl)));
    LV_CUDA(cudaMallocHost(&h.h_ctl, sizeof(DevCtl)));
  }
  LV_CUDA(cudaMemset(h.ctl, 0, sizeof(DevCtl)));
  for (auto& e : h.ev) LV_CUDA(cudaEventCreate(&e));
  LV_CUDA(cudaStreamCreateWithFlags(&h.side, cudaStreamNonBlocking));
  LV_CUDA(cudaEventCreateWithFlags(&h.ev_fork, cudaEventDisableTiming));
  LV_CUDA(cudaEventCreateWithFlags(&h.ev_join, cudaEventDisableTiming));

  return LOUVAIN_OK;
}

void destroy_handle(Handle& h) {
  // LV_TRACE: where a destroy's time goes (diagnostics only)
  static const bool tr = getenv("LV_TRACE") != nullptr;
  auto t0 = std::chrono::steady_clock::now();
  auto mark = [&](const char* what) {
    if (!tr) return;
    const auto t1 = std::chrono::steady_clock::now();
    fprintf(stderr, "[lv] destroy %-12s %8.3f ms\n", what, std::chrono::duration<double, std::milli>(t1 - t0).count());
    t0 = t1;
  };
  cudaSetDevice(h.device);
  dist_free(h);
  if (h.stream) {
    dfree(h.dl_big, h.stream);
    dfree(h.dl_mid, h.stream);
  }
  if (h.stream) {
    level_free(h.lv, h.stream);
    cudaStreamSynchronize(h.stream);
  }
  mark("level");
  if (tr) {
    size_t mine = 0, cached = 0;
    for (int i = 0; i < SC_COUNT; ++i) mine += h.scratch.bytes[i];
    {
      std::lock_guard<std::mutex> lk(g_cache_mu);
      for (const auto& c : g_cache) cached += std::get<2>(c);
    }
    fprintf(stderr, "[lv] destroy scratch %.2f GB, cache before %.2f GB\n", mine / 1e9, cached / 1e9);
  }
  scratch_free(h);
  mark("scratch");
  if (h.ctl) ctl_give(h.device, h.ctl, h.h_ctl);  // kept for the next handle (no cudaFree:
  h.ctl = nullptr;                                  // it synchronised the device for up to
  h.h_ctl = nullptr;                                // 0.66 s per destroy, LV_TRACE)
  mark("ctl");
  for (auto& e : h.ev)
    if (e) cudaEventDestroy(e);
  if (h.side) {
    cudaStreamSynchronize(h.side);
    cudaStreamDestroy(h.side);
  }
  if (h.ev_fork) cudaEventDestroy(h.ev_fork);
  if (h.ev_join) cudaEventDestroy(h.ev_join);

  if (h.own_stream && h.stream) cudaStreamDestroy(h.stream);
}

// Every call first makes the handle's device current and refuses poisoned handles.
struct DeviceScope {
  int prev = -1;
  explicit DeviceScope(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceScope() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

int32_t guard(louvain_graph_t g) {
  if (!g) {
    set_error("null handle");
    return LOUVAIN_E_INVALID_ARG;
  }
  if (g->h.poisoned) {
    set_error("handle poisoned by an earlier sticky CUDA error");
    return LOUVAIN_E_STATE;
  }
  return LOUVAIN_OK;
}

int32_t finish_call(Handle& h, int32_t rc) {
  if (rc == LOUVAIN_E_CUDA) {
    cudaError_t e = cudaPeekAtLastError();
    if (e == cudaErrorIllegalAddress || e == cudaErrorLaunchFailure || e == cudaErrorIllegalInstruction ||
        e == cudaErrorMisalignedAddress || e == cudaErrorHardwareStackError)
      h.poisoned = true;
  }
  return rc;
}

bool bucket_nonempty(const Level& L, int b) {
  return L.class_off[kSubPerBucket * (b + 1)] > L.class_off[kSubPerBucket * b];
}
// On a distributed handle every rank runs the same sequence of commits and
// exchanges: a bucket counts if any rank owns one of its vertices.
bool bucket_active(const Handle& h, const Level& L, int b) {
  return h.dist ? h.dist->cap[b] > 0 : bucket_nonempty(L, b);
}

// One sweep body: for each non-empty bucket 1..7 its sweep kernels, then its
// commit (BIN_SYNC) -- or a single commit at the end (RELAXED).
int32_t sweep_body(Handle& h, Level& L, const louvain_params_t& p) {
  static const bool trace = getenv("LV_TRACE") && std::string(getenv("LV_TRACE")) == "2";
  LV_CUDA(cudaMemsetAsync(h.ctl, 0, offsetof(DevCtl, L), h.stream));  // logn + bounds
  int commits = 0;
  for (int b = 1; b <= 7; ++b) {
    if (!bucket_active(h, L, b)) continue;
    auto t0 = std::chrono::steady_clock::now();
    LV_TRY(launch_sweep_bucket(h, L, p, b));
    auto t1 = std::chrono::steady_clock::now();
    if (p.mode == LOUVAIN_MODE_BIN_SYNC) {
      // every rank's bucket-b moves: all-gathered, or written into every replica by the
      // peer-memory commit itself (LOUVAIN_DIST_P2P)
      if (h.dist && !dist_p2p(h)) LV_TRY(dist_exchange(h, L, commits, b));
      LV_TRY(launch_commit(h, L, commits++));
    }
    if (trace) {
      cudaStreamSynchronize(h.stream);
      auto t2 = std::chrono::steady_clock::now();
      fprintf(stderr, "[lv]      bucket %d: enqueue %.3f ms, done %.3f ms (n=%ld)\n", b,
              std::chrono::duration<double, std::milli>(t1 - t0).count(),
              std::chrono::duration<double, std::milli>(t2 - t0).count(),
              (long)(L.class_off[kSubPerBucket * (b + 1)] - L.class_off[kSubPerBucket * b]));
    }
  }
  if (p.mode == LOUVAIN_MODE_RELAXED) {
    if (h.dist && !dist_p2p(h)) LV_TRY(dist_exchange(h, L, 0, 0));
    LV_TRY(launch_commit(h, L, commits++));
  }
  ++L.sweeps_done;
  return LOUVAIN_OK;
}

using i128 = __int128;

// LV_TRACE=1: per-level phase timeline on stderr (host wall clock after a stream sync)
struct Trace {
  bool on = getenv("LV_TRACE") != nullptr;
  std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
  void mark(cudaStream_t s, const char* what, int level) {
    if (!on) return;
    cudaStreamSynchronize(s);
    const auto t1 = std::chrono::steady_clock::now();
    fprintf(stderr, "[lv] level %d %-12s %9.3f ms\n", level, what,
            std::chrono::duration<double, std::milli>(t1 - t0).count());
    t0 = t1;
  }
};

i128 pow10_i128(int p) {
  i128 r = 1;
  for (int t = 0; t < p; ++t) r *= 10;
  return r;
}

// (num_new - num_old) / W^2 < 10^-p, in exact integers (R13)
bool below_threshold(int64_t num_new, int64_t num_old, uint64_t W, int p) {
  i128 d = (i128)num_new - (i128)num_old;
  return d * pow10_i128(p) < (i128)W * (i128)W;
}

int64_t qnum_of(uint64_t L, uint64_t S, uint64_t W) { return (int64_t)((i128)L * (i128)W - (i128)S); }

void fill_q(louvain_qnum_t* q, uint64_t L, uint64_t S, uint64_t W) {
  if (!q) return;
  q->L = L;
  q->S_lo = S;
  q->S_hi = 0;
  q->W = W;
  q->q = W ? (double)qnum_of(L, S, W) / ((double)W * (double)W) : 0.0;
}

int32_t copy_out(void* dst, const void* src, size_t bytes, cudaStream_t s) {
  if (!dst || !bytes) return LOUVAIN_OK;
  LV_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDefault, s));
  return LOUVAIN_OK;
}

float elapsed(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0.f;
  cudaEventElapsedTime(&ms, a, b);
  return ms;
}

// Eq. (1) parts of the level's own partition; on a distributed handle each rank
// sums the entries of its rows and L is all-reduced (S from the replicated a_c).
int32_t modularity_parts(Handle& h, Level& L, bool singletons, uint64_t* Lout, uint64_t* Sout) {
  if (!h.dist) return level_modularity(h, L, nullptr, Lout, Sout, singletons);
  LV_TRY(launch_modularity(h, L, nullptr, singletons));
  LV_TRY(dist_allreduce(h, &h.ctl->L, 1));
  LV_CUDA(cudaMemcpyAsync(h.h_ctl, h.ctl, sizeof(DevCtl), cudaMemcpyDeviceToHost, h.stream));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  *Lout = h.h_ctl->L;
  *Sout = h.h_ctl->S;
  return LOUVAIN_OK;
}

// The multilevel driver (SURVEY 8(c) listing; oracle/louvain_oracle.c orc_louvain
// is the independent CPU transcription of the same control flow).
int32_t run_impl(Handle& h, const louvain_params_t& p, int32_t* labels_out, louvain_qnum_t* q_final,
                 louvain_stats_t* st) {
  cudaStream_t s = h.stream;
  Level& L0 = h.lv;
  const int64_t n0 = L0.n;
  const uint64_t W = L0.W;
  louvain_stats_t local;
  std::memset(&local, 0, sizeof local);
  auto t_begin = std::chrono::steady_clock::now();
  const long long launches0 = g_launches, cub0 = g_cub_calls;
  // Every device resource of the run is owned by `R`, so each return path
  // (errors included) frees it and leaves no dangling pointer in the handle.
  struct RunRes {
    Handle& h;
    int32_t* lab = nullptr;  // original vertex -> current community (R22)
    uint2* pcn = nullptr;    // {label at the sweep start, label now} (delta pass of Eq. (1))
    int32_t* map = nullptr;  // contraction map of the current level
    Level owned;             // current contracted level (levels >= 1)
    bool has_owned = false;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    explicit RunRes(Handle& hh) : h(hh) {}
    ~RunRes() {
      h.pcn = nullptr;
      dfree(lab, h.stream);
      dfree(pcn, h.stream);
      dfree(map, h.stream);
      if (has_owned) level_free(owned, h.stream);
      if (e0) cudaEventDestroy(e0);
      if (e1) cudaEventDestroy(e1);
    }
  } R(h);
  LV_TRY(dalloc(&R.lab, n0, s));
  int32_t* const lab = R.lab;
  // labels at each sweep start, for the delta pass of Eq. (1) (LV_MOD_DELTA=0: full passes only)
  static const bool mod_delta = !(getenv("LV_MOD_DELTA") && getenv("LV_MOD_DELTA")[0] == '0');
  if (mod_delta && !dist_p2p(h)) LV_TRY(dalloc(&R.pcn, std::max<int64_t>(n0, 1), s));
  // peer-memory commits write the snapshot's "label now" of every rank: the shared block
  uint2* const pcn = (mod_delta && dist_p2p(h)) ? static_cast<uint2*>(h.dist->pcn_block) : R.pcn;
  LV_CUDA(cudaEventCreate(&R.e0));
  LV_CUDA(cudaEventCreate(&R.e1));
  cudaEvent_t e_lvl0 = R.e0, e_lvl1 = R.e1;
  if (n0) { k_iota<<<grid_for(n0, 256), 256, 0, s>>>(lab, n0); LV_LAUNCHED(); }
  // level 0 starts from singletons; a full run owns every vertex.  The
  // degree binning (a2) is redone by every run -- nothing of a previous run is
  // reused, so a timed run includes every step of the path.
  if (!h.dist) L0.own_hi = -1;  // a distributed handle keeps its rows (set per level below)
  L0.bins_valid = false;
  if (n0) LV_TRY(level_set_labels(h, L0, nullptr));
  uint64_t Lq = 0, Sq = 0;  // exact parts of the current level's kept partition
  Level* cur = &L0;
  Trace tr;
  if (W > 0) {
    for (int level = 0;; ++level) {
      if ((p.max_levels > 0 && level >= p.max_levels) || level >= LOUVAIN_MAX_LEVELS) break;
      cudaEventRecord(e_lvl0, s);
      Level& L = *cur;
      const int pexp = (L.n > p.size_limit) ? p.th_bin_exp : p.th_final_exp;  // P:330, R14
      tr.mark(s, "start", level);
      if (h.dist) LV_TRY(dist_set_level_range(h, L, level));
      LV_TRY(level_binning(h, L, p));
      if (h.dist) LV_TRY(dist_after_binning(h, L));
      tr.mark(s, "binning", level);
      // level start: singletons.  Level 0 evaluates Eq. (1); a contracted level
      // starts exactly where the previous one ended (contraction preserves L and
      // S, R18 -- pinned by the oracle tests and the parity suite).
      if (level == 0) LV_TRY(modularity_parts(h, L, /*singletons=*/true, &Lq, &Sq));
      const int64_t num_start = qnum_of(Lq, Sq, W);
      int64_t num_prev = num_start;
      int64_t moved_level = 0;
      int32_t sweeps = 0;
      auto sweep_once = [&]() -> int32_t {
        LV_CUDA(cudaEventRecord(h.ev[0], s));
        if (mod_delta) LV_TRY(launch_snapshot(h, L));
        // peer-memory commits: no rank may write into a replica before its owner has taken
        // the sweep's snapshot (and finished the previous level's setup)
        if (dist_p2p(h)) LV_TRY(dist_barrier(h));
        LV_TRY(sweep_body(h, L, p));
        LV_CUDA(cudaEventRecord(h.ev[1], s));
        tr.mark(s, "sweep", level);
        if (mod_delta) LV_TRY(launch_modularity_delta(h, L));
        else LV_TRY(launch_modularity(h, L, nullptr));
        if (h.dist) {  // the ranks' parts: overflow flags and L change (delta pass) / L (full pass)
          LV_TRY(dist_allreduce(h, &h.ctl->overflow, 2));
          if (!mod_delta) LV_TRY(dist_allreduce(h, &h.ctl->L, 1));
          LV_TRY(dist_total_moved(h));
        }
        LV_CUDA(cudaEventRecord(h.ev[2], s));
        tr.mark(s, "modularity", level);
        return LOUVAIN_OK;
      };
      for (;;) {
        if (p.max_sweeps > 0 && sweeps >= p.max_sweeps) break;
        h.pcn = pcn;
        LV_TRY(sweep_once());
        LV_CUDA(cudaMemcpyAsync(h.h_ctl, h.ctl, sizeof(DevCtl), cudaMemcpyDeviceToHost, s));
        LV_CUDA(cudaStreamSynchronize(s));
        const float t_sw = elapsed(h.ev[0], h.ev[1]);
        local.t_sweep_ms_total += t_sw;
        local.t_modularity_ms_total += elapsed(h.ev[1], h.ev[2]);
        // moves of the sweep (every rank's: peer-memory commits log only this rank's own)
        const int64_t moved = h.dist ? (int64_t)h.h_ctl->gmoved : (int64_t)h.h_ctl->logn;
        if (level == 0 && sweeps == 0) {
          local.t_sweep_ms_first = t_sw;
          local.moved_first = moved;
        }
        if (level == 0 && sweeps < 32) local.t_sweep_ms_level0[sweeps] = t_sw;
        local.edges_swept += L.nnz;
        ++sweeps;
        if (h.h_ctl->overflow) {
          set_error("partitioned hash table overflow (sweep_part); please report");
          return LOUVAIN_E_CUDA;
        }
        // Eq. (1) numerator of the swept partition: delta pass (L_before + dL, exact
        // modular arithmetic) or full pass
        const uint64_t L_after = (mod_delta && delta_chosen(*h.h_ctl, L.nnz)) ? Lq + h.h_ctl->dL : h.h_ctl->L;
        const int64_t num = qnum_of(L_after, h.h_ctl->S, W);
        if (tr.on)
          fprintf(stderr, "[lv] level %d sweep %d: moved %llu, moved entries %s%.4f of nnz, %s pass\n", level, sweeps,
                  h.h_ctl->logn, delta_div() > 1 ? "" : "(not summed, gate off) ",
                  L.nnz ? (double)h.h_ctl->mdeg / (double)L.nnz : 0.0,
                  (mod_delta && delta_chosen(*h.h_ctl, L.nnz)) ? "delta" : "full");
        if (p.revert_on_decrease && num < num_prev) {  // R15
          LV_TRY(launch_revert(h, L));
          break;
        }
        Lq = L_after;
        Sq = h.h_ctl->S;
        moved_level += moved;
        if (moved == 0 || below_threshold(num, num_prev, W, pexp)) break;  // Alg. 1 l.12, R13
        num_prev = num;
      }
      const int64_t num_end = qnum_of(Lq, Sq, W);  // the partition kept at the end of the phase
      cudaEventRecord(e_lvl1, s);
      local.n[level] = L.n;
      local.nnz[level] = L.nnz;
      local.sweeps_per_level[level] = sweeps;
      local.moved_per_level[level] = moved_level;
      local.num_start[level] = num_start;
      local.num_end[level] = num_end;
      local.levels = level + 1;
      local.sweeps += sweeps;
      LV_CUDA(cudaEventSynchronize(e_lvl1));
      local.t_opt_ms[level] = elapsed(e_lvl0, e_lvl1);
      if (moved_level == 0 || below_threshold(num_end, num_start, W, p.th_final_exp)) {  // R16
        LV_TRY(compose_labels_ca(h, lab, n0, L.ca));
        break;
      }
      // aggregation phase (Alg. 3)
      cudaEventRecord(e_lvl0, s);
      Level next;  // scratch-backed (parity buffers); its plans are freed with it below
      LV_TRY(dalloc(&R.map, L.n, s));
      int32_t* const map = R.map;
      tr.mark(s, "pre-contract", level);
      // mergeCommunity-style grouping + hashing (default, NEXT-1) or the canonical sort-based one (LV_CONTRACT=sort)
      static const bool hash_contract = !(getenv("LV_CONTRACT") && std::string(getenv("LV_CONTRACT")) == "sort");
      if (hash_contract) LV_TRY(level_contract_fast(h, L, next, map, (level + 1) & 1));
      else LV_TRY(level_contract(h, L, next, map, (level + 1) & 1));
      tr.mark(s, "contract", level);
      LV_TRY(compose_labels(h, lab, n0, map));
      dfree(R.map, s);
      R.map = nullptr;
      LV_TRY(level_setup(h, next));
      tr.mark(s, "setup", level);
      cudaEventRecord(e_lvl1, s);
      LV_CUDA(cudaEventSynchronize(e_lvl1));
      local.t_agg_ms[level] = elapsed(e_lvl0, e_lvl1);
      if (R.has_owned) level_free(R.owned, s);
      R.owned = next;
      R.has_owned = true;
      cur = &R.owned;
    }
  }
  // the handle's partition becomes the final one; (Lq, Sq) are the exact parts of
  // the last level's kept partition, equal to those of `lab` on the input graph
  bool final_set = false;
  if (R.has_owned && R.owned.n <= kFinalHistMax) {  // totals from the last level, sizes by an smem histogram
    LV_TRY(level_set_final(h, L0, lab, R.owned.ca, R.owned.n));
    final_set = true;
  }
  if (R.has_owned) {
    level_free(R.owned, s);
    R.has_owned = false;
  }
  if (!final_set) LV_TRY(level_set_labels(h, L0, lab));
  LV_TRY(copy_out(labels_out, lab, sizeof(int32_t) * (size_t)n0, s));
  LV_CUDA(cudaStreamSynchronize(s));
  fill_q(&local.q, Lq, Sq, W);
  local.t_total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_begin).count();
  local.kernel_launches = g_launches - launches0;
  local.cub_calls = g_cub_calls - cub0;
  if (q_final) *q_final = local.q;
  if (st) *st = local;
  return LOUVAIN_OK;
}

// Stage caller input (host or device) as device memory: returns a device pointer
// (the caller's own if it is already device memory and borrow is allowed).
template <class T>
int32_t stage(const T* src, int64_t count, bool borrow, cudaStream_t s, T** dst, bool* owned) {
  *owned = false;
  if (!src) { *dst = nullptr; return LOUVAIN_OK; }
  if (borrow && is_device_ptr(src)) {
    *dst = const_cast<T*>(src);
    return LOUVAIN_OK;
  }
  LV_TRY(dalloc(dst, count, s));
  LV_CUDA(cudaMemcpyAsync(*dst, src, sizeof(T) * (size_t)count, cudaMemcpyDefault, s));
  *owned = true;
  return LOUVAIN_OK;
}

}  // namespace
}  // namespace lv

using namespace lv;

LV_API void louvain_params_default(louvain_params_t* p) {
  if (!p) return;
  std::memset(p, 0, sizeof *p);
  p->mode = LOUVAIN_MODE_BIN_SYNC;
  p->singleton_rule = 1;
  p->revert_on_decrease = 1;
  p->th_bin_exp = 2;
  p->th_final_exp = 6;
  p->size_limit = 100000;
  const int64_t b[6] = {4, 8, 16, 32, 84, 319};
  std::memcpy(p->deg_bounds, b, sizeof b);
  p->max_sweeps = 0;
  p->max_levels = 0;
}

LV_API const char* louvain_last_error(void) { return g_err.c_str(); }
LV_API int32_t louvain_release_cache(void) {
  release_cache_all();
  cudaGetLastError();
  return LOUVAIN_OK;
}
LV_API void louvain_launch_counts(int64_t* kernel_launches, int64_t* cub_calls) {
  if (kernel_launches) *kernel_launches = g_launches;
  if (cub_calls) *cub_calls = g_cub_calls;
}

LV_API int32_t louvain_create_csr(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                                  uint32_t flags, void* cuda_stream, louvain_graph_t* out) {
  g_err.clear();
  if (!out || n < 0 || nnz < 0 || !rowptr || (nnz > 0 && !col) || n > INT32_MAX - 1) {
    set_error("louvain_create_csr: null/negative argument or n >= 2^31 - 1");
    return LOUVAIN_E_INVALID_ARG;
  }
  *out = nullptr;
  const bool validate = flags & LOUVAIN_VALIDATE;
  const bool borrow = flags & LOUVAIN_BORROW;
  // Host-side validation before any device work (works without a GPU for host inputs).
  const bool host_in = !is_device_ptr(rowptr);
  if (host_in) {
    LV_TRY(validate_csr_host(n, nnz, rowptr, col, w, validate, nullptr));
  } else if (validate) {
    std::vector<int64_t> r(n + 1);
    std::vector<int32_t> c(nnz);
    std::vector<uint32_t> ww(w ? nnz : 0);
    LV_CUDA(cudaMemcpy(r.data(), rowptr, 8 * (n + 1), cudaMemcpyDefault));
    if (nnz) LV_CUDA(cudaMemcpy(c.data(), col, 4 * nnz, cudaMemcpyDefault));
    if (w && nnz) LV_CUDA(cudaMemcpy(ww.data(), w, 4 * nnz, cudaMemcpyDefault));
    LV_TRY(validate_csr_host(n, nnz, r.data(), c.data(), w ? ww.data() : nullptr, true, nullptr));
  }
  louvain_graph_s* g = new louvain_graph_s();
  Handle& h = g->h;
  int32_t rc = init_handle(h, cuda_stream);
  if (rc != LOUVAIN_OK) {
    destroy_handle(h);
    delete g;
    return rc;
  }
  Level& L = h.lv;
  L.n = n;
  L.nnz = nnz;
  // LOUVAIN_BORROW: use device inputs in place only if every given array is device memory
  const bool all_dev = is_device_ptr(rowptr) && (nnz == 0 || is_device_ptr(col)) && (!w || is_device_ptr(w));
  const bool use_in_place = borrow && all_dev;
  bool o1 = false, o2 = false, o3 = false;
  rc = stage(rowptr, n + 1, use_in_place, h.stream, &L.rowptr, &o1);
  if (rc == LOUVAIN_OK && nnz) rc = stage(col, nnz, use_in_place, h.stream, &L.col, &o2);
  if (rc == LOUVAIN_OK && w && nnz) rc = stage(w, nnz, use_in_place, h.stream, &L.w, &o3);
  L.owns_csr = !use_in_place;
  if (rc == LOUVAIN_OK && !L.col) rc = dalloc(&L.col, 1, h.stream);
  if (rc == LOUVAIN_OK) rc = level_alloc_state(L, h.stream);
  if (rc == LOUVAIN_OK) rc = level_setup(h, L);
  if (rc == LOUVAIN_OK) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "cudaStreamSynchronize", __FILE__, __LINE__);
  }
  if (rc != LOUVAIN_OK) {
    destroy_handle(h);
    delete g;
    return rc;
  }
  *out = g;
  return LOUVAIN_OK;
}

namespace lv {
int32_t create_from_device(int64_t n, int64_t nnz, int64_t* rowptr, int32_t* col, uint32_t* w, void* cuda_stream,
                           louvain_graph_t* out) {
  *out = nullptr;
  louvain_graph_s* g = new louvain_graph_s();
  Handle& h = g->h;
  int32_t rc = init_handle(h, cuda_stream);
  Level& L = h.lv;
  L.n = n;
  L.nnz = nnz;
  L.rowptr = rowptr;
  L.col = col;
  L.w = w;
  L.owns_csr = true;  // freed with the handle (or below, on failure)
  if (rc == LOUVAIN_OK) rc = level_alloc_state(L, h.stream);
  if (rc == LOUVAIN_OK) rc = level_setup(h, L);
  if (rc == LOUVAIN_OK) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "cudaStreamSynchronize", __FILE__, __LINE__);
  }
  if (rc != LOUVAIN_OK) {
    if (!h.stream) {  // init failed before the stream existed: free the arrays directly
      dfree(rowptr, nullptr);
      dfree(col, nullptr);
      dfree(w, nullptr);
      L.rowptr = nullptr;
      L.col = nullptr;
      L.w = nullptr;
    }
    destroy_handle(h);
    delete g;
    return rc;
  }
  *out = g;
  return LOUVAIN_OK;
}
}  // namespace lv

LV_API int32_t louvain_destroy(louvain_graph_t g) {
  if (!g) return LOUVAIN_OK;
  destroy_handle(g->h);
  delete g;
  return LOUVAIN_OK;
}

LV_API int32_t louvain_get_info(louvain_graph_t g, int64_t* n, int64_t* nnz, uint64_t* W) {
  LV_TRY(guard(g));
  if (n) *n = g->h.lv.n;
  if (nnz) *nnz = g->h.lv.nnz;
  if (W) *W = g->h.lv.W;
  return LOUVAIN_OK;
}

LV_API int32_t louvain_get_csr(louvain_graph_t g, int64_t* rowptr, int32_t* col, uint32_t* w) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  int32_t rc = copy_out(rowptr, L.rowptr, 8 * (size_t)(L.n + 1), h.stream);
  if (!rc) rc = copy_out(col, L.col, 4 * (size_t)L.nnz, h.stream);
  if (!rc && w && L.nnz) {
    if (L.w) {
      rc = copy_out(w, L.w, 4 * (size_t)L.nnz, h.stream);
    } else if (is_device_ptr(w)) {
      k_fill_u32<<<grid_for(L.nnz, 256), 256, 0, h.stream>>>(w, L.nnz, 1u);
      LV_LAUNCHED();
    } else {
      cudaStreamSynchronize(h.stream);
      for (int64_t e = 0; e < L.nnz; ++e) w[e] = 1u;
    }
  }
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "sync", __FILE__, __LINE__);
  }
  return finish_call(h, rc);
}

LV_API int32_t louvain_set_labels(louvain_graph_t g, const int32_t* labels) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  int32_t rc = LOUVAIN_OK;
  if (!labels) {
    rc = level_set_labels(h, L, nullptr);
  } else {
    int32_t* d = nullptr;
    bool owned = false;
    rc = stage(labels, L.n, false, h.stream, &d, &owned);
    if (!rc) rc = level_set_labels(h, L, d);
    if (owned) dfree(d, h.stream);
  }
  return finish_call(h, rc);
}

LV_API int32_t louvain_get_labels(louvain_graph_t g, int32_t* labels_out) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  if (!labels_out && h.lv.n) { set_error("null labels_out"); return LOUVAIN_E_INVALID_ARG; }
  int32_t* tmp = nullptr;
  int32_t rc = dalloc(&tmp, h.lv.n, h.stream);
  if (!rc) rc = level_get_labels(h, h.lv, tmp);
  if (!rc) rc = copy_out(labels_out, tmp, 4 * (size_t)h.lv.n, h.stream);
  dfree(tmp, h.stream);
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "sync", __FILE__, __LINE__);
  }
  return finish_call(h, rc);
}

LV_API int32_t louvain_get_totals(louvain_graph_t g, uint32_t* a_out, int32_t* size_out) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  uint32_t* tmp = nullptr;
  int32_t rc = dalloc(&tmp, h.lv.n, h.stream);
  if (!rc) rc = level_get_a(h, h.lv, tmp);
  if (!rc) rc = copy_out(a_out, tmp, 4 * (size_t)h.lv.n, h.stream);
  dfree(tmp, h.stream);
  if (!rc) rc = copy_out(size_out, h.lv.size, 4 * (size_t)h.lv.n, h.stream);
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "sync", __FILE__, __LINE__);
  }
  return finish_call(h, rc);
}

LV_API int32_t louvain_sweep(louvain_graph_t g, const louvain_params_t* p, int64_t* moved, louvain_qnum_t* q_after) {
  LV_TRY(guard(g));
  louvain_params_t pp;
  if (p) pp = *p; else louvain_params_default(&pp);
  LV_TRY(check_params(pp));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  int32_t rc = level_binning(h, L, pp);
  if (!rc && h.dist) rc = dist_after_binning(h, L);
  if (!rc) rc = sweep_body(h, L, pp);
  if (!rc && q_after) rc = launch_modularity(h, L, nullptr);
  if (!rc && q_after && h.dist) rc = dist_allreduce(h, &h.ctl->L, 1);
  if (!rc && h.dist) rc = dist_allreduce(h, &h.ctl->overflow, 1);
  if (!rc && h.dist) rc = dist_total_moved(h);
  if (!rc) {
    cudaError_t e = cudaMemcpyAsync(h.h_ctl, h.ctl, sizeof(DevCtl), cudaMemcpyDeviceToHost, h.stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "sweep", __FILE__, __LINE__);
  }
  if (!rc && h.h_ctl->overflow) {
    set_error("partitioned hash table overflow (sweep_part); please report");
    rc = LOUVAIN_E_CUDA;
  }
  if (!rc) {
    if (moved) *moved = (int64_t)(h.dist ? h.h_ctl->gmoved : h.h_ctl->logn);
    if (q_after) fill_q(q_after, h.h_ctl->L, h.h_ctl->S, L.W);
  }
  return finish_call(h, rc);
}

LV_API int32_t louvain_modularity(louvain_graph_t g, const int32_t* labels, louvain_qnum_t* q) {
  LV_TRY(guard(g));
  if (!q) { set_error("null q"); return LOUVAIN_E_INVALID_ARG; }
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  int32_t* d = nullptr;
  bool owned = false;
  int32_t rc = LOUVAIN_OK;
  if (labels) rc = stage(labels, L.n, false, h.stream, &d, &owned);
  uint64_t Lq = 0, Sq = 0;
  if (!rc) rc = level_modularity(h, L, d, &Lq, &Sq);
  if (owned) dfree(d, h.stream);
  if (!rc) fill_q(q, Lq, Sq, L.W);
  return finish_call(h, rc);
}

LV_API int32_t louvain_aggregate(louvain_graph_t g, louvain_graph_t* next, int32_t* map_out) {
  LV_TRY(guard(g));
  if (!next) { set_error("null next"); return LOUVAIN_E_INVALID_ARG; }
  Handle& h = g->h;
  DeviceScope ds(h.device);
  louvain_graph_s* ng = new louvain_graph_s();
  // a library-owned stream dies with its handle, so the child gets its own
  int32_t rc = init_handle(ng->h, h.own_stream ? nullptr : (void*)h.stream);
  int32_t* map = nullptr;
  if (!rc) rc = dalloc(&map, h.lv.n, h.stream);
  if (!rc) rc = level_contract(h, h.lv, ng->h.lv, map);
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "aggregate", __FILE__, __LINE__);
  }
  if (!rc) rc = level_setup(ng->h, ng->h.lv);
  if (!rc) rc = copy_out(map_out, map, 4 * (size_t)h.lv.n, h.stream);
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "aggregate", __FILE__, __LINE__);
  }
  dfree(map, h.stream);
  if (rc) {
    destroy_handle(ng->h);
    delete ng;
    return finish_call(h, rc);
  }
  *next = ng;
  return LOUVAIN_OK;
}

LV_API int32_t louvain_run(louvain_graph_t g, const louvain_params_t* p, int32_t* labels_out, louvain_qnum_t* q_final,
                           louvain_stats_t* stats) {
  LV_TRY(guard(g));
  louvain_params_t pp;
  if (p) pp = *p; else louvain_params_default(&pp);
  LV_TRY(check_params(pp));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  return finish_call(h, run_impl(h, pp, labels_out, q_final, stats));
}

LV_API int32_t louvain_set_owned_range(louvain_graph_t g, int64_t v_begin, int64_t v_end) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  if (v_begin < 0 || v_end < v_begin || v_end > L.n) {
    set_error("owned range must satisfy 0 <= v_begin <= v_end <= n");
    return LOUVAIN_E_INVALID_ARG;
  }
  int64_t e[2] = {0, 0};
  LV_CUDA(cudaMemcpy(&e[0], L.rowptr + v_begin, 8, cudaMemcpyDeviceToHost));
  LV_CUDA(cudaMemcpy(&e[1], L.rowptr + v_end, 8, cudaMemcpyDeviceToHost));
  L.own_lo = v_begin;
  L.own_hi = v_end;
  L.own_e0 = e[0];
  L.own_e1 = e[1];
  L.bins_valid = false;  // bucket lists hold the owned vertices only
  return LOUVAIN_OK;
}

LV_API int32_t louvain_begin_sweep(louvain_graph_t g) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  if (L.log_committed > 0) ++L.sweeps_done;
  L.log_committed = 0;
  ++L.stamp_id;
  return finish_call(h, set_ctl_u64(h, &h.ctl->logn, 0));
}

LV_API int32_t louvain_decide_bucket(louvain_graph_t g, const louvain_params_t* p, int32_t bucket, int32_t* moves_out,
                                     int64_t cap, int64_t* count) {
  LV_TRY(guard(g));
  if (bucket < 1 || bucket > 7 || !count || cap < 0 || (cap > 0 && !moves_out)) {
    set_error("louvain_decide_bucket: bucket in 1..7, count and moves_out required");
    return LOUVAIN_E_INVALID_ARG;
  }
  louvain_params_t pp;
  if (p) pp = *p; else louvain_params_default(&pp);
  LV_TRY(check_params(pp));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  const int64_t c0 = L.log_committed;
  int32_t rc = level_binning(h, L, pp);
  if (!rc) rc = set_ctl_u64(h, &h.ctl->logn, (unsigned long long)c0);
  if (!rc && bucket_nonempty(L, bucket)) rc = launch_sweep_bucket(h, L, pp, bucket);
  unsigned long long c1 = c0;
  if (!rc) {
    cudaError_t e = cudaMemcpyAsync(&c1, &h.ctl->logn, 8, cudaMemcpyDeviceToHost, h.stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "decide_bucket", __FILE__, __LINE__);
  }
  const int64_t cnt = (int64_t)c1 - c0;
  if (!rc && cnt > cap) {
    set_error("louvain_decide_bucket: moves_out capacity too small");
    rc = LOUVAIN_E_INVALID_ARG;
  }
  if (!rc && cnt > 0) {
    int32_t* tmp = nullptr;
    rc = dalloc(&tmp, 2 * cnt, h.stream);
    if (!rc) rc = pack_moves(h, L, c0, cnt, tmp);
    if (!rc) rc = copy_out(moves_out, tmp, 8 * (size_t)cnt, h.stream);
    dfree(tmp, h.stream);
  }
  if (!rc) rc = set_ctl_u64(h, &h.ctl->logn, (unsigned long long)c0);  // nothing committed yet
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "decide_bucket", __FILE__, __LINE__);
  }
  if (!rc) *count = cnt;
  return finish_call(h, rc);
}

LV_API int32_t louvain_commit_moves(louvain_graph_t g, const int32_t* moves, int64_t count) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  Level& L = h.lv;
  if (count < 0 || (count > 0 && !moves) || L.log_committed + count > L.n) {
    set_error("louvain_commit_moves: bad count (each vertex moves at most once per sweep)");
    return LOUVAIN_E_INVALID_ARG;
  }
  DeviceScope ds(h.device);
  const int64_t c0 = L.log_committed;
  int32_t rc = LOUVAIN_OK;
  if (count > 0) {
    int32_t* d = nullptr;
    bool owned = false;
    rc = stage(moves, 2 * count, false, h.stream, &d, &owned);
    if (!rc) rc = unpack_moves(h, L, c0, count, d);
    if (owned) dfree(d, h.stream);
    if (!rc) rc = set_ctl_u64(h, &h.ctl->bounds[0], (unsigned long long)c0);
    if (!rc) rc = set_ctl_u64(h, &h.ctl->logn, (unsigned long long)(c0 + count));
    if (!rc) rc = launch_commit(h, L, 0);
    if (!rc) {
      cudaError_t e = cudaStreamSynchronize(h.stream);
      if (e != cudaSuccess) rc = cuda_fail(e, "commit_moves", __FILE__, __LINE__);
    }
  }
  if (!rc) L.log_committed = c0 + count;
  return finish_call(h, rc);
}

LV_API int32_t louvain_revert_sweep(louvain_graph_t g) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  int32_t rc = set_ctl_u64(h, &h.ctl->logn, (unsigned long long)L.log_committed);
  if (!rc) rc = launch_revert(h, L);
  if (!rc) rc = set_ctl_u64(h, &h.ctl->logn, 0);
  if (!rc) {
    cudaError_t e = cudaStreamSynchronize(h.stream);
    if (e != cudaSuccess) rc = cuda_fail(e, "revert", __FILE__, __LINE__);
  }
  if (!rc) L.log_committed = 0;
  return finish_call(h, rc);
}

namespace lv {
namespace abi_kernels {
__global__ void k_compose_ext(int32_t* lab, int64_t n0, const int32_t* map) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n0; i += (int64_t)gridDim.x * blockDim.x)
    lab[i] = map[lab[i]];
}
}  // namespace abi_kernels
}  // namespace lv

LV_API int32_t louvain_compose_labels(int32_t* lab, int64_t n0, const int32_t* map, void* cuda_stream) {
  if (n0 < 0 || (n0 > 0 && (!lab || !map))) {
    set_error("louvain_compose_labels: null pointer");
    return LOUVAIN_E_INVALID_ARG;
  }
  if (n0 == 0) return LOUVAIN_OK;
  if (!is_device_ptr(lab) || !is_device_ptr(map)) {
    set_error("louvain_compose_labels: lab and map must be device pointers");
    return LOUVAIN_E_INVALID_ARG;
  }
  lv::abi_kernels::k_compose_ext<<<grid_for(n0, 256), 256, 0, (cudaStream_t)cuda_stream>>>(lab, n0, map);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  LV_CUDA(cudaStreamSynchronize((cudaStream_t)cuda_stream));
  return LOUVAIN_OK;
}

LV_API int32_t louvain_modularity_owned(louvain_graph_t g, uint64_t* L_owned, uint64_t* S, uint64_t* W) {
  LV_TRY(guard(g));
  Handle& h = g->h;
  DeviceScope ds(h.device);
  Level& L = h.lv;
  uint64_t Lq = 0, Sq = 0;
  int32_t rc = level_modularity(h, L, nullptr, &Lq, &Sq);
  if (!rc) {
    if (L_owned) *L_owned = Lq;
    if (S) *S = Sq;
    if (W) *W = L.W;
  }
  return finish_call(h, rc);
}
