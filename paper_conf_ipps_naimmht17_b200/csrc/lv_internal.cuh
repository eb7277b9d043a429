// lv_internal.cuh -- private declarations of liblouvain.so (B200, sm_100a).
//
// Device layout of one level (SURVEY 8 "Device layout at every level"):
//   rowptr int64[n+1], col int32[nnz], w uint32[nnz] (absent at unit weight),
//   k uint32[n], C int32[n], a uint32[n], size int32[n], W uint64,
//   bin_vertices int32[n] sorted by dispatch class, move log (v, new, old) int32[n].
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "louvain.h"

namespace lv {

constexpr uint64_t kWGuard = 3037000499ULL;  // W^2 < 2^63 (R4)

// ------------------------------------------------------------------ errors
void set_error(const std::string& msg);
int32_t cuda_fail(cudaError_t e, const char* what, const char* file, int line);

#define LV_CUDA(call)                                                     \
  do {                                                                    \
    cudaError_t e_ = (call);                                              \
    if (e_ != cudaSuccess) return lv::cuda_fail(e_, #call, __FILE__, __LINE__); \
  } while (0)
#define LV_TRY(expr)            \
  do {                          \
    int32_t rc_ = (expr);       \
    if (rc_ != LOUVAIN_OK) return rc_; \
  } while (0)

// ------------------------------------------------------------------ dispatch classes
// Vertices are sorted once per level by class = 4*bucket + sub, bucket in 0..7
// (0 = degree 0, never moves; 1..7 = the paper's buckets) and sub the
// kernel family inside the bucket (by degree): 0 register/warp/CTA-small,
// 1 CTA-large, 2 hub (multi-CTA, global hash).
constexpr int kNumClasses = 32;
constexpr int64_t kCtaLargeMin = 4096;   // deg >= this: 1024-thread CTA, 128 KB table
constexpr int64_t kHubMin = 12288;       // deg >= this: multi-CTA global hash
constexpr int kCtaSmallCap = 8192;       // slots (64 KB)
constexpr int kCtaLargeCap = 16384;      // slots (128 KB)
constexpr int64_t kHubChunkEdges = 8192; // edges per hub insert chunk
constexpr int64_t kHubScanSlots = 8192;  // slots per hub scan chunk

struct DevCtl {
  unsigned long long logn;       // move-log entries appended in this sweep
  unsigned long long bounds[9];  // log offset at the start of bucket b's commit
  unsigned long long L, S;       // modularity parts
  unsigned long long bad;        // validation flag
};

struct HubPlan {
  int64_t nh = 0;
  int64_t nchunks = 0, nscan = 0;
  int32_t* hub_v = nullptr;         // [nh]
  int64_t* tab_off = nullptr;       // [nh]
  int64_t* tab_cap = nullptr;       // [nh]
  int64_t* chunk = nullptr;         // [3*nchunks]: hub, e_begin, e_end
  int64_t* scan = nullptr;          // [3*nscan]: hub, slot_begin, slot_end
  int64_t* scan_first = nullptr;    // [nh+1]: first scan chunk of each hub
  unsigned long long* table = nullptr;  // sum tab_cap slots (EMPTY-initialised)
  int64_t table_slots = 0;
  void* partial = nullptr;          // [nscan] Partial
};

struct Level {
  int64_t n = 0, nnz = 0;
  uint64_t W = 0;
  int64_t* rowptr = nullptr;
  int32_t* col = nullptr;
  uint32_t* w = nullptr;  // nullptr = unit weights (level 0 of every config, R20)
  bool owns_csr = true;
  uint32_t* k = nullptr;
  int32_t* C = nullptr;
  uint32_t* a = nullptr;
  int32_t* size = nullptr;
  // move log of the current sweep (v, new, old) -- also the revert record (R15)
  int32_t* mv_v = nullptr;
  int32_t* mv_new = nullptr;
  int32_t* mv_old = nullptr;
  // binning (valid for bins_bounds)
  bool bins_valid = false;
  int64_t bins_bounds[6] = {0, 0, 0, 0, 0, 0};
  int32_t* bin_vertices = nullptr;
  int64_t class_off[kNumClasses + 1] = {0};
  HubPlan hub;
};

struct Handle {
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  bool poisoned = false;
  Level lv;
  DevCtl* ctl = nullptr;     // device
  DevCtl* h_ctl = nullptr;   // pinned host mirror
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  // distributed (nullptr when single GPU)
  void* dist = nullptr;
};

// ------------------------------------------------------------------ launch accounting
// Every explicit <<<>>> launch is followed by LV_LAUNCHED(); every device-wide
// CUB call (scan / radix sort / reduce) by LV_CUB().  Reported in louvain_stats_t.
extern long long g_launches, g_cub_calls;
#define LV_LAUNCHED() (++lv::g_launches)
#define LV_CUB() (++lv::g_cub_calls)

// ------------------------------------------------------------------ memory helpers
int32_t dmalloc(void** p, size_t bytes, cudaStream_t s);
void dfree(void* p, cudaStream_t s);
template <class T>
int32_t dalloc(T** p, size_t count, cudaStream_t s) {
  return dmalloc(reinterpret_cast<void**>(p), sizeof(T) * (count ? count : 1), s);
}
bool is_device_ptr(const void* p);

// ------------------------------------------------------------------ level ops (lv_level.cu)
int32_t level_alloc_state(Level& L, cudaStream_t s);
void level_free(Level& L, cudaStream_t s);
int32_t level_setup(Handle& h, Level& L);  // k, W, singleton partition (Alg. 1 l.2)
int32_t level_set_labels(Handle& h, Level& L, const int32_t* d_labels);  // C given, recompute a/size
int32_t level_binning(Handle& h, Level& L, const louvain_params_t& p);  // classes + hub plan
int32_t level_modularity(Handle& h, Level& L, const int32_t* d_C, uint64_t* Lout, uint64_t* Sout);
int32_t launch_modularity(Handle& h, Level& L, const int32_t* d_C);  // async: ctl->L, ctl->S
int32_t launch_commit(Handle& h, Level& L, int bucket);
int32_t launch_revert(Handle& h, Level& L);
int32_t level_contract(Handle& h, Level& L, Level& out, int32_t* d_map);  // Alg. 3
int32_t compose_labels(Handle& h, int32_t* lab, int64_t n0, const int32_t* map);  // lab[i] = map[lab[i]]
int32_t validate_csr_host(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                          bool full, uint64_t* W);

// ------------------------------------------------------------------ sweep (lv_sweep.cu)
int32_t launch_sweep_bucket(Handle& h, Level& L, const louvain_params_t& p, int bucket);

// ------------------------------------------------------------------ launch geometry
inline unsigned grid_for(int64_t items, int per_block, int max_blocks = 148 * 16) {
  int64_t b = (items + per_block - 1) / per_block;
  if (b > max_blocks) b = max_blocks;
  if (b < 1) b = 1;
  return (unsigned)b;
}

}  // namespace lv

struct louvain_graph_s {
  lv::Handle h;
};
