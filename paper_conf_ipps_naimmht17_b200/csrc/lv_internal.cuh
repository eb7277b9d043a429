// lv_internal.cuh -- private declarations of liblouvain.so (B200, sm_100a).
//
// Device layout of one level (SURVEY 8 "Device layout at every level"):
//   rowptr int64[n+1], col int32[nnz], w uint32[nnz] (absent at unit weight),
//   k uint32[n], ca uint2[n] = {C[v], a[v]} packed so one 8-byte gather of a
//   neighbour brings both its label and (when it represents its community) a_c,
//   size int32[n], W uint64,
//   bin_vertices int32[n] sorted by dispatch class, move log (v, new, old) int32[n].
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <memory>
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
// Vertices are sorted once per level by class = 8*bucket + sub, bucket in 0..7
// (0 = degree 0, never moves; 1..7 = the paper's buckets) and sub the
// kernel family inside the bucket, by degree:
//   sub 0: deg < 512    (register / warp / 128-thread CTA kernels, by bucket bound)
//   sub 1..4: CTA per vertex, table of <= kCap[sub] slots sized to the tier's
//             degree range so that small tiers keep more vertices in flight per SM:
//             [512,1024) 256 thr, [1024,2048) 512, [2048,4096) 512, [4096,12288) 1024
//   sub 5..7: >= 12288      label-partitioned CTA tasks (P = ceil(deg/kPartLabels) smem tables,
//                           the staged entries pre-partitioned); sub 7 (>= 393216) with
//                           P > kPartMaxP only: hub, cooperative grid, global table ring
constexpr int kSubPerBucket = 8;
constexpr int kNumClasses = 8 * kSubPerBucket;
constexpr int kSubPart = 5, kSubHub = 7;  // first partitioned sub-class, hub sub-class
constexpr int64_t kSub1Min = 512, kSub2Min = 1024, kSub3Min = 2048, kSub4Min = 4096, kSub5Min = 12288,
                  kSub6Min = 32768, kHubMin = 393216;
#ifndef LV_TIER4_SLOTS  // compile-time A/B (16384: a power of two, double hashing)
#define LV_TIER4_SLOTS 16384
#endif
constexpr int kCapT[5] = {2048, 4096, 8192, 16384, LV_TIER4_SLOTS};  // max smem table slots (12 B each) of sub 0..4
constexpr int kThrT[5] = {128, 256, 512, 512, 1024};  // (tier 3 with 1024: slower at level 2, DESIGN 13)
constexpr int kPerSmT[5] = {16, 8, 4, 2, 1};
constexpr int kCapMax = 18432;
// Buckets whose degree bound is <= kSmallMaxDeg (1-4 with the paper's bounds) run the
// register kernels; their sub-class is 1 + ceil(log2 deg) (1..6): lane groups of 1,
// 2, 4, ..., 32 lanes per vertex.
constexpr int64_t kSmallMaxDeg = 32;
__host__ __device__ inline int small_sub_of_degree(int64_t d) {
  int s = 1;
  while (s < 6 && (int64_t(1) << (s - 1)) < d) ++s;
  return s;
}
__host__ __device__ inline int sub_of_degree(int64_t d) {
  return d < kSub1Min ? 0 : d < kSub2Min ? 1 : d < kSub3Min ? 2 : d < kSub4Min ? 3 : d < kSub5Min ? 4
       : d < kSub6Min ? 5 : d < kHubMin ? 6 : 7;
}

constexpr int64_t kHubChunkEdges = 2048;  // edges per hub insert item
constexpr int64_t kHubScanSlots = 4096;   // slots per hub scan item
constexpr int64_t kHubWaveSlots = 3 << 19;  // table slots per wave (12 B each; ring = 2 segments)

struct DevCtl {
  unsigned long long logn;       // move-log entries appended in this sweep
  unsigned long long bounds[9];  // log offset at the start of bucket b's commit
  unsigned long long mdeg;       // sum of the degrees of the vertices moved in this sweep
  unsigned long long L, S;       // modularity parts
  unsigned long long bad;        // validation flag
  unsigned long long overflow;   // a partitioned hash table filled up (must stay 0)
  unsigned long long dL;         // delta pass: L_after - L_before (two's complement)
  unsigned long long nbig;       // delta pass: moved vertices left to the block kernel
  unsigned long long nmid;       // delta pass: moved vertices left to the warp kernel
  unsigned long long ddiv;       // delta pass chosen iff mdeg * ddiv <= nnz
  unsigned long long gmoved;     // distributed peer-memory commits: moves of all ranks in this sweep
};

// Hub work plan (one per level).  Hubs are grouped into waves whose tables fit
// one segment of a 2-segment ring (wave k uses segment k % 2).  A cooperative
// kernel runs phases separated by grid.sync(): phase p inserts the edges of
// wave p, scans the tables of wave p-1 and takes the decisions of wave p-2, so
// every dependency is enforced by a barrier (no spinning, no tickets) and at
// most two waves' tables are live -- small enough to stay in L2.
struct HubItem {
  int32_t hub;
  int32_t pad;
  int64_t begin, end;  // insert: edge range; scan: slot range of the hub's table
};
struct HubInfo {
  int32_t v;           // vertex id
  int32_t nscan;       // scan items of this hub
  int64_t off, cap;    // table region within its wave's ring segment
  int64_t scan_first;  // index of its first scan item (= its first partial)
  int64_t sbase;       // stage index of edge e of the hub = sbase + e
};
struct HubPlan {
  int64_t nh = 0, nwaves = 0, nins = 0, nscan = 0, seg = 0;
  HubItem* ins = nullptr;        // insert items, wave-major
  HubItem* scans = nullptr;      // scan items, wave-major (index = partial slot)
  int64_t* ins_off = nullptr;    // [nwaves+1]
  int64_t* scan_off = nullptr;   // [nwaves+1]
  int64_t* wave_hub = nullptr;   // [nwaves+1] first hub of each wave
  HubInfo* info = nullptr;       // [nh]
  unsigned long long* ring = nullptr;  // 2 * seg slots {label|e}, EMPTY-initialised
  uint32_t* ring_a = nullptr;          // a_c when known (0xFFFFFFFF = unknown)
  void* partial = nullptr;             // [nscan]
  int grid = 0;                        // co-resident CTAs of the cooperative kernel
  int64_t bucket_wave[9] = {0};        // waves of bucket b: [bucket_wave[b-1], bucket_wave[b])
};

// Label-partitioned plan for vertices of degree >= kSub5Min: vertex v gets
// P_v = ceil(deg / kPartLabels) CTA tasks; task p owns the labels c with
// part_of(c, P_v) == p.  Each sweep the vertex's staged entries are first
// scattered into partition order (histogram -> per-vertex scan -> scatter, in
// chunks of kPartChunk entries), so task p reads only its own share and keeps
// it in one shared-memory table.  Vertices with P_v > kPartMaxP (deg > 50 M)
// go to the cooperative hub kernel instead.
#ifndef LV_PART_LABELS  // compile-time A/B
#define LV_PART_LABELS 12288
#endif
constexpr int64_t kPartLabels = LV_PART_LABELS;  // expected labels per task (table load ~3/4 with double hashing, overflow check at 7/8; r1: 6144 / 8192 / 10240 / 12288 -> 28.3 / 22.2 / 21.4 / 21.0 ms at level 0; r2 12288 vs 10240: run -1.7 ms)
constexpr int kPartSlots = 16384;      // smem table slots per task (12 B each: 192 KB)
constexpr int kPartMaxP = 8192;        // partitions per vertex (smem histogram of a chunk)
constexpr int64_t kPartChunk = 32768;  // staged entries per histogram / scatter item
struct PartChunk {
  int32_t vi;  // plan vertex
  int32_t pad;
  int64_t begin, end;  // entries of the vertex's staged segment
};
struct PartPlan {
  int64_t ntasks = 0, nverts = 0, nchunks = 0, npoff = 0;
  int32_t* task_vpos = nullptr;   // [ntasks] index into the plan's vertex list
  int32_t* task_p = nullptr;      // [ntasks] partition index
  int32_t* vert_pos = nullptr;    // [nverts] bin position of the vertex
  int32_t* vert_P = nullptr;      // [nverts] partitions of the vertex
  int32_t* vert_first = nullptr;  // [nverts] first task (= first partial)
  int64_t* vert_pbase = nullptr;  // [nverts] first poff index (sum of (P+1) of earlier vertices)
  int32_t* done = nullptr;        // [nverts] tasks finished (reset every sweep)
  void* partial = nullptr;        // [ntasks] Partial
  int64_t* poff = nullptr;        // [npoff] partition starts in the partitioned stage (+ end)
  unsigned long long* pcur = nullptr;  // [ntasks] scatter cursors
  PartChunk* chunks = nullptr;    // [nchunks]
  int64_t bucket_task[9] = {0};   // tasks of bucket b: [bucket_task[b-1], bucket_task[b])
  int64_t bucket_vert[9] = {0};   // plan vertices of bucket b
  int64_t bucket_chunk[9] = {0};  // chunks of bucket b (pre-partitioned vertices only)
  int64_t bucket_vsplit[8] = {0};  // bucket b's vertices [bucket_vert[b-1], vsplit) are pre-partitioned,
  int64_t bucket_tsplit[8] = {0};  // tasks [bucket_task[b-1], tsplit); the rest stream (P <= kStreamMaxP)
};
#ifndef LV_SPAN_Q  // compile-time A/B (tools/ab_build.py -D)
#define LV_SPAN_Q 4
#endif
constexpr int kSpanQ = LV_SPAN_Q;  // entries per lane in flight in the warp-span tile kernels
constexpr int64_t kStreamMaxP = 16;  // (4 at level 0, 1 at the weighted levels: measured no better, DESIGN 13)

struct Level {
  int64_t n = 0, nnz = 0;
  uint64_t W = 0;
  int64_t* rowptr = nullptr;
  int32_t* col = nullptr;
  uint32_t* w = nullptr;  // nullptr = unit weights (level 0 of every config, R20)
  bool owns_csr = true;
  bool scratch_backed = false;  // all arrays live in the handle's scratch (level of a run)
  int parity = 0;
  bool k_ready = false;  // k already holds the degrees (contracted level: community totals)
  uint32_t* k = nullptr;
  uint2* ca = nullptr;  // {C[v], a[v]}
  int32_t* C = nullptr;  // copy of C[v] (4-byte label gathers of the modularity pass)
  int32_t* size = nullptr;
  // move log of the current sweep (v, new, old) -- also the revert record (R15)
  int32_t* mv_v = nullptr;
  int32_t* mv_new = nullptr;
  int32_t* mv_old = nullptr;
  int32_t* mv_stamp = nullptr;  // sharded ABI only: sweep id of each vertex's last committed move
  int32_t stamp_id = 0;         // incremented by every louvain_begin_sweep
  // distributed handle with peer-memory commits: ca / size / C live in the replica set
  // `rep_set` of DistCtx (IPC-exported memory every rank writes into); not freed here
  int rep_set = -1;
  bool state_external = false;
  int32_t sweeps_done = 0;  // sweeps since the partition was last reset to singletons
  // sharded sweeps: owned vertex range (decisions, L) and its edge range
  int64_t own_lo = 0, own_hi = -1;  // own_hi < 0: all vertices
  int64_t own_e0 = 0, own_e1 = -1;
  int64_t log_committed = 0;        // entries of the sweep's move log already committed
  // binning (valid for bins_bounds)
  bool bins_valid = false;
  int64_t bins_bounds[6] = {0, 0, 0, 0, 0, 0};
  int64_t bins_bounds_pending[6] = {0, 0, 0, 0, 0, 0};  // bounds of the binning being built (plans)
  int32_t* bin_vertices = nullptr;
  int64_t class_off[kNumClasses + 1] = {0};
  int64_t class_soff[kNumClasses + 1] = {0};  // soff[class_off[c]] (host copy)
  // gather staging (two-phase sweep): soff[i] = sum of degrees of bin_vertices[0..i),
  // stage[soff[i] + t] = {label, a_c or 0xFFFFFFFF} of the t-th neighbour of bin_vertices[i]
  int64_t* soff = nullptr;
  uint2* stage = nullptr;
  // bin_rb[i] = rowptr[bin_vertices[i]] (with soff: a vertex's row from two sequential
  // loads by bin position, not the dependent bin_vertices -> rowptr round trips)
  int64_t* bin_rb = nullptr;
  HubPlan hub;
  PartPlan part;
};

// Grow-only scratch buffers owned by a handle (cudaMalloc'ed once, reused by
// every level and every run): avoids multi-GB stream-ordered allocations
// churning the memory pool between levels.
enum ScratchSlot {
  SC_STAGE = 0, SC_GC, SC_GW, SC_OC, SC_OW, SC_K1, SC_V0, SC_V1, SC_TMP, SC_TILES,
  // arrays of a contracted level inside louvain_run, double-buffered by level parity
  SC_LVL0, SC_LVL_END = SC_LVL0 + 2 * 13, SC_COUNT = SC_LVL_END
};
enum LevelArray { LA_ROWPTR = 0, LA_COL, LA_W, LA_K, LA_CA, LA_SIZE, LA_MVV, LA_MVN, LA_MVO, LA_BIN, LA_SOFF, LA_C, LA_BINRB };
struct Scratch {
  void* p[SC_COUNT] = {nullptr};
  size_t bytes[SC_COUNT] = {0};
};

struct Handle {
  int device = 0;
  Scratch scratch;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  bool poisoned = false;
  Level lv;
  DevCtl* ctl = nullptr;     // device
  DevCtl* h_ctl = nullptr;   // pinned host mirror
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  // side stream for independent kernels inside one phase (fork/join through events)
  cudaStream_t side = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  // louvain_run only: {label at the sweep start, label after} per vertex; the
  // commit writes .y of every moved vertex (delta pass of Eq. (1))
  uint2* pcn = nullptr;
  // delta pass of Eq. (1): lists of long moved rows (grow-only, reused by every sweep so a
  // captured sweep graph allocates nothing)
  int32_t* dl_big = nullptr;
  int32_t* dl_mid = nullptr;
  size_t dl_big_n = 0, dl_mid_n = 0;
  // distributed handle (louvain_create_csr_dist*): nullptr on one GPU
  struct DistCtx* dist = nullptr;
};

// ------------------------------------------------------------------ multi-GPU (lv_dist.cu)
struct Comm;
constexpr int kMaxWorld = 64;
// Every rank's replica of one set of partition-state arrays (device-resident table).
struct PeerPtrs {
  uint2* ca[kMaxWorld];
  int32_t* size[kMaxWorld];
  int32_t* C[kMaxWorld];
  uint2* pcn[kMaxWorld];
};
struct DistCtx {
  Comm* comm = nullptr;
  int rank = 0, world = 1;
  std::vector<int64_t> vlo0;   // level-0 row ranges of all ranks (world + 1)
  int64_t cap[8] = {0};        // exchange capacity per commit group: max over ranks of owned
                               // vertices of bucket b (b = 1..7), of all buckets (0, RELAXED)
  int32_t* sbuf = nullptr;     // (v, new) pairs, 2 * max cap
  int32_t* rbuf = nullptr;     // world * that
  size_t sbuf_n = 0, rbuf_n = 0;
  // LOUVAIN_DIST_P2P: the commit kernel writes every move into every rank's replica
  // through peer memory (CUDA IPC mappings: NVLink P2P across GPUs, the same memory for
  // ranks sharing one GPU) and a barrier ends each bucket -- no all-gather of moves.
  // Replica sets: 0 = the handle's level 0, 1 / 2 = contracted levels of even / odd depth.
  bool p2p = false;
  int64_t rep_n = 0;                 // capacity (vertices) of every replica array
  void* rep_block[3] = {nullptr, nullptr, nullptr};  // ca | size | C, cudaMalloc'ed (IPC)
  void* pcn_block = nullptr;         // uint2[rep_n], cudaMalloc'ed (IPC)
  std::vector<void*> opened;         // peers' blocks mapped into this process
  PeerPtrs* d_peers[3] = {nullptr, nullptr, nullptr};  // device tables, one per set
  unsigned long long* d_bar = nullptr;  // barrier operand
  ~DistCtx();
};
int32_t dist_set_level_range(Handle& h, Level& L, int level);  // own range of this rank at this level
int32_t dist_after_binning(Handle& h, Level& L);                // exchange capacities of the level
int32_t dist_exchange(Handle& h, Level& L, int commit_idx, int group);  // all ranks' moves into the log
int32_t dist_allreduce(Handle& h, unsigned long long* dev, size_t count);  // in-place sum (no-op on 1 GPU)
// recv[displ[r] .. + cnt[r]) <- rank r's send (units of elem bytes; device buffers, handle's stream)
int32_t dist_allgatherv(Handle& h, const void* send, void* recv, const std::vector<int64_t>& cnt,
                        const std::vector<int64_t>& displ, size_t elem);
void dist_free(Handle& h);
inline bool dist_p2p(const Handle& h) { return h.dist && h.dist->p2p; }
int32_t dist_barrier(Handle& h);                                // all ranks' preceding work done
int32_t dist_bind_state(Handle& h, Level& L, int set);          // L.ca / size / C -> replica set
int32_t dist_commit_p2p(Handle& h, Level& L, int bucket);       // commit own moves into every replica
int32_t dist_revert_p2p(Handle& h, Level& L);                   // undo own moves in every replica
int32_t dist_total_moved(Handle& h);                            // ctl->gmoved = sum over ranks of logn

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
int32_t scratch_get(Handle& h, int slot, size_t bytes, void** out);  // grow-only per-handle buffer
int32_t scratch_size(Handle& h, int slot, size_t* bytes);  // current size of a scratch buffer
void scratch_free(Handle& h);

// ------------------------------------------------------------------ level ops (lv_level.cu)
int32_t level_alloc_state(Level& L, cudaStream_t s);
int32_t level_alloc_scratch(Handle& h, Level& L, int parity);  // state arrays from scratch slots
void level_free(Level& L, cudaStream_t s);
int32_t level_setup(Handle& h, Level& L);  // k, W, singleton partition (Alg. 1 l.2)
int32_t level_set_labels(Handle& h, Level& L, const int32_t* d_labels);  // C given (nullptr = iota), recompute a/size
// end of louvain_run: labels in [0, n_last) of the last level (state ca_last); n_last <= kFinalHistMax
constexpr int64_t kFinalHistMax = 49152;  // size histogram in shared memory (4 B per label)
int32_t level_set_final(Handle& h, Level& L, const int32_t* d_labels, const uint2* ca_last, int64_t n_last);
int32_t level_get_labels(Handle& h, Level& L, int32_t* d_out);          // C -> d_out (device)
int32_t level_get_a(Handle& h, Level& L, uint32_t* d_out);              // a -> d_out (device)
int32_t level_binning(Handle& h, Level& L, const louvain_params_t& p);  // classes + hub plan
// d_C == nullptr: the level's own partition (maintained a_c); else external labels
// singletons: the caller guarantees C is the singleton partition (no label gathers)
int32_t level_modularity(Handle& h, Level& L, const int32_t* d_C, uint64_t* Lout, uint64_t* Sout,
                         bool singletons = false);
int32_t launch_modularity(Handle& h, Level& L, const int32_t* d_C, bool singletons = false);  // async: ctl->L, ctl->S
// Eq. (1) after a sweep from the sweep's move log (async).  h.pcn[v] = {label at
// the sweep start, label now}.  If the moved vertices hold <= nnz/ddiv entries:
// ctl->dL = L_after - L_before (delta pass), else ctl->L = L_after (full pass);
// ctl->S either way.  The host tells which from ctl->mdeg (delta_chosen).
int32_t launch_snapshot(Handle& h, Level& L);  // h.pcn[v] = {C[v], C[v]}
unsigned long long delta_div();                 // LV_DELTA_DIV (default 1)
int32_t launch_modularity_delta(Handle& h, Level& L);
__host__ __device__ __forceinline__ bool delta_chosen(const DevCtl& c, int64_t nnz) { return c.mdeg * c.ddiv <= (unsigned long long)nnz; }
int32_t launch_commit(Handle& h, Level& L, int bucket);
int32_t set_ctl_u64(Handle& h, unsigned long long* dst, unsigned long long v);
int32_t pack_moves(Handle& h, Level& L, int64_t c0, int64_t cnt, int32_t* out);          // log -> (v,new) pairs
int32_t unpack_moves(Handle& h, Level& L, int64_t c0, int64_t cnt, const int32_t* in);   // (v,new) pairs -> log
int32_t launch_revert(Handle& h, Level& L);
// Alg. 3, canonical (rows sorted); parity >= 0: arrays from the handle's scratch (inside louvain_run)
int32_t level_contract(Handle& h, Level& L, Level& out, int32_t* d_map, int parity = -1);
int32_t level_contract_fast(Handle& h, Level& L, Level& out, int32_t* d_map, int parity);  // Alg. 3, rows unsorted
int32_t compose_labels(Handle& h, int32_t* lab, int64_t n0, const int32_t* map);  // lab[i] = map[lab[i]]
// Tile plan of an edge-centric kernel over the entries [base, end) of rows [lo, hi) with
// prefix offsets offs (offs[hi] >= end): out[t] = the row holding entry min(base + t*T, end - 1),
// t = 0..ntiles (ntiles = ceil((end - base) / T)).  One binary search per tile, all in
// parallel, instead of a serial search by one thread at the start of every tile.
int32_t tile_starts(Handle& h, const int64_t* offs, int64_t lo, int64_t hi, int64_t base, int64_t end, int64_t T,
                    const int64_t** out);
int32_t compose_labels_ca(Handle& h, int32_t* lab, int64_t n0, const uint2* ca);   // lab[i] = C[lab[i]]
size_t hub_partial_bytes();
// Handle over device CSR arrays it takes ownership of (freed on failure too).
int32_t create_from_device(int64_t n, int64_t nnz, int64_t* rowptr, int32_t* col, uint32_t* w, void* cuda_stream,
                           louvain_graph_t* out);
int32_t validate_csr_host(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                          bool full, uint64_t* W);

// ------------------------------------------------------------------ sweep (lv_sweep.cu)
int32_t launch_sweep_bucket(Handle& h, Level& L, const louvain_params_t& p, int bucket);
// phase 1 gather for bin positions [pos0,pos1), staged entries [s0,s1)
int32_t launch_stage(Handle& h, Level& L, int64_t pos0, int64_t pos1, int64_t s0, int64_t s1);
int32_t build_part_plan(Handle& h, Level& L);

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
