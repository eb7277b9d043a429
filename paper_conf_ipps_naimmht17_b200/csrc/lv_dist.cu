// lv_dist.cu -- the vertex-sharded multi-GPU path, inside the
// library: one process per GPU, one distributed handle per rank.
//
// Why it shards: inside a degree bucket every computeMove reads the same
// bucket-start snapshot (Alg. 1 l.6-7), so the bucket's
// vertices are independent units; the commit (Alg. 1 l.8-11) is the
// only cross-vertex dependency.  Design:
//   * every rank holds the level graph (replicated; C5 = 8.9 GB, ~5% of HBM) and a
//     replica of the partition state (C, a_c, size_c);
//   * rank r decides only the vertices of its edge-balanced range [v_r, v_{r+1})
//     (the caller's rows at level 0, rowptr[v_r] ~ r*nnz/P at later levels);
//   * after each bucket, every rank's moves are all-gathered (one collective of
//     (v, new) pairs, padded to the largest owned bucket share, which every rank
//     knows from the per-level bucket counts) and every rank commits ALL of them
//     with the same exact integer updates, so the replicas stay bit-identical and
//     no a_c all-reduce is needed;
//   * Eq. (1) after a sweep: the delta pass runs over the moved rows the rank owns
//     and the partial L change is all-reduced (one uint64); S = sum a_c^2 comes
//     from the replicated a_c;
//   * contraction (Alg. 3) is sharded by new vertex: the O(n) steps (renumbering,
//     member grouping) run on every rank, then rank r copies and merges only the
//     member rows of the new vertices [c_r, c_{r+1}) (balanced by merged-row
//     length, lv_contract.cu k_seg_split) and the ranks' rows are all-gathered
//     into the replicated CSR' of the next level.
// Transports: NCCL (ncclAllGather / ncclAllReduce / grouped ncclBroadcast on the
// handle's stream; libnccl is loaded at run time, the unique id is bootstrapped by
// the caller, e.g. torch.distributed) or host callbacks (tests: gloo, or several
// ranks sharing one GPU, which NCCL does not allow).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "lv_device.cuh"
#include "lv_internal.cuh"

#if defined(LOUVAIN_HAVE_NCCL_HEADERS)
#include <nccl.h>
#endif

namespace lv {

// ------------------------------------------------------------------ transports
struct Comm {
  int rank = 0, world = 1;
  virtual ~Comm() {}
  // device buffers; recv holds world * bytes, rank-major
  virtual int32_t allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) = 0;
  // in-place sum of `count` uint64 values (device buffer)
  virtual int32_t allreduce_u64(unsigned long long* buf, size_t count, cudaStream_t s) = 0;
  // recv[displ[r] .. displ[r] + cnt[r]) <- rank r's send (elem-byte units), device buffers
  virtual int32_t allgatherv(const void* send, void* recv, const std::vector<int64_t>& cnt,
                             const std::vector<int64_t>& displ, size_t elem, cudaStream_t s) = 0;
};

#if defined(LOUVAIN_HAVE_NCCL_HEADERS)
namespace {
struct NcclApi {
  bool ok = false;
  std::string err;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
// The process's libnccl (torch loads its own libnccl.so.2 first; dlopen by soname
// returns that copy), else the system one.
const NcclApi& nccl() {
  static NcclApi api = [] {
    NcclApi a;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      a.err = std::string("cannot load libnccl.so.2: ") + dlerror();
      return a;
    }
    auto sym = [&](const char* name) { return dlsym(h, name); };
    a.GetUniqueId = (decltype(a.GetUniqueId))sym("ncclGetUniqueId");
    a.CommInitRank = (decltype(a.CommInitRank))sym("ncclCommInitRank");
    a.CommDestroy = (decltype(a.CommDestroy))sym("ncclCommDestroy");
    a.AllGather = (decltype(a.AllGather))sym("ncclAllGather");
    a.AllReduce = (decltype(a.AllReduce))sym("ncclAllReduce");
    a.Broadcast = (decltype(a.Broadcast))sym("ncclBroadcast");
    a.GroupStart = (decltype(a.GroupStart))sym("ncclGroupStart");
    a.GroupEnd = (decltype(a.GroupEnd))sym("ncclGroupEnd");
    a.GetErrorString = (decltype(a.GetErrorString))sym("ncclGetErrorString");
    a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.AllGather && a.AllReduce && a.Broadcast &&
           a.GroupStart && a.GroupEnd && a.GetErrorString;
    if (!a.ok) a.err = "libnccl lacks a required symbol";
    return a;
  }();
  return api;
}

int32_t nccl_fail(ncclResult_t r, const char* what) {
  set_error(std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "NCCL error"));
  return LOUVAIN_E_NCCL;
}
#define LV_NCCL(call)                                      \
  do {                                                     \
    ncclResult_t r_ = (call);                              \
    if (r_ != ncclSuccess) return nccl_fail(r_, #call);    \
  } while (0)

struct NcclComm final : Comm {
  ncclComm_t comm = nullptr;
  ~NcclComm() override {
    if (comm) nccl().CommDestroy(comm);
  }
  int32_t allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
    LV_NCCL(nccl().AllGather(send, recv, bytes, ncclUint8, comm, s));
    return LOUVAIN_OK;
  }
  int32_t allreduce_u64(unsigned long long* buf, size_t count, cudaStream_t s) override {
    LV_NCCL(nccl().AllReduce(buf, buf, count, ncclUint64, ncclSum, comm, s));
    return LOUVAIN_OK;
  }
  int32_t allgatherv(const void* send, void* recv, const std::vector<int64_t>& cnt, const std::vector<int64_t>& displ,
                     size_t elem, cudaStream_t s) override {
    LV_NCCL(nccl().GroupStart());
    for (int r = 0; r < world; ++r) {
      if (cnt[r] == 0) continue;
      char* dst = static_cast<char*>(recv) + displ[r] * elem;
      ncclResult_t rr = nccl().Broadcast(r == rank ? send : dst, dst, (size_t)cnt[r] * elem, ncclUint8, r, comm, s);
      if (rr != ncclSuccess) {
        nccl().GroupEnd();
        return nccl_fail(rr, "ncclBroadcast");
      }
    }
    LV_NCCL(nccl().GroupEnd());
    return LOUVAIN_OK;
  }
};
}  // namespace
#endif

namespace {
// Host callbacks (louvain_host_comm_t): device data is staged through pinned
// host memory around each call.
struct HostComm final : Comm {
  louvain_host_comm_t cb{};
  void* hbuf = nullptr;
  size_t hcap = 0;
  ~HostComm() override {
    if (hbuf) cudaFreeHost(hbuf);
  }
  int32_t host(size_t bytes, char** out) {
    if (hcap < bytes) {
      if (hbuf) cudaFreeHost(hbuf);
      hbuf = nullptr;
      hcap = 0;
      LV_CUDA(cudaMallocHost(&hbuf, bytes));
      hcap = bytes;
    }
    *out = static_cast<char*>(hbuf);
    return LOUVAIN_OK;
  }
  int32_t allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
    char* hb = nullptr;
    LV_TRY(host(bytes * (size_t)(world + 1), &hb));
    char* hs = hb + bytes * (size_t)world;
    if (bytes) LV_CUDA(cudaMemcpyAsync(hs, send, bytes, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    if (cb.allgather(cb.user, hs, hb, (int64_t)bytes) != 0) {
      set_error("host all-gather callback failed");
      return LOUVAIN_E_NCCL;
    }
    if (bytes) LV_CUDA(cudaMemcpyAsync(recv, hb, bytes * (size_t)world, cudaMemcpyHostToDevice, s));
    LV_CUDA(cudaStreamSynchronize(s));  // hb is reused by the next call
    return LOUVAIN_OK;
  }
  int32_t allreduce_u64(unsigned long long* buf, size_t count, cudaStream_t s) override {
    char* hb = nullptr;
    LV_TRY(host(8 * count, &hb));
    LV_CUDA(cudaMemcpyAsync(hb, buf, 8 * count, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    if (cb.allreduce_u64(cb.user, reinterpret_cast<uint64_t*>(hb), (int64_t)count) != 0) {
      set_error("host all-reduce callback failed");
      return LOUVAIN_E_NCCL;
    }
    LV_CUDA(cudaMemcpyAsync(buf, hb, 8 * count, cudaMemcpyHostToDevice, s));
    LV_CUDA(cudaStreamSynchronize(s));
    return LOUVAIN_OK;
  }
  int32_t allgatherv(const void* send, void* recv, const std::vector<int64_t>& cnt, const std::vector<int64_t>& displ,
                     size_t elem, cudaStream_t s) override {
    const int64_t mx = *std::max_element(cnt.begin(), cnt.end());
    const size_t bytes = (size_t)mx * elem;
    if (bytes == 0) return LOUVAIN_OK;
    char* hb = nullptr;
    LV_TRY(host(bytes * (size_t)(world + 1), &hb));
    char* hs = hb + bytes * (size_t)world;
    std::memset(hs, 0, bytes);
    if (cnt[rank]) LV_CUDA(cudaMemcpyAsync(hs, send, (size_t)cnt[rank] * elem, cudaMemcpyDeviceToHost, s));
    LV_CUDA(cudaStreamSynchronize(s));
    if (cb.allgather(cb.user, hs, hb, (int64_t)bytes) != 0) {
      set_error("host all-gather callback failed");
      return LOUVAIN_E_NCCL;
    }
    for (int r = 0; r < world; ++r)
      if (cnt[r])
        LV_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + displ[r] * elem, hb + bytes * (size_t)r,
                                (size_t)cnt[r] * elem, cudaMemcpyHostToDevice, s));
    LV_CUDA(cudaStreamSynchronize(s));
    return LOUVAIN_OK;
  }
};

// ------------------------------------------------------------------ kernels
// This rank's moves of one commit group, log [bounds[idx], logn), as (v, new)
// pairs padded with (-1, -1) to the group's common capacity.
__global__ void k_dist_pack(const DevCtl* ctl, int idx, const int32_t* __restrict__ mv_v,
                            const int32_t* __restrict__ mv_new, int64_t cap, int32_t* __restrict__ send) {
  const int64_t start = (int64_t)ctl->bounds[idx], cnt = (int64_t)ctl->logn - start;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x) {
    const bool has = i < cnt;
    send[2 * i] = has ? mv_v[start + i] : -1;
    send[2 * i + 1] = has ? mv_new[start + i] : -1;
  }
}
__global__ void k_dist_rewind(DevCtl* ctl, int idx) { ctl->logn = ctl->bounds[idx]; }
// Every rank's moves (rank-major, padded) appended to the local move log; the
// commit that follows applies all of them (integer updates: order-independent).
__global__ void k_dist_append(DevCtl* ctl, const int32_t* __restrict__ recv, int64_t total, int32_t* mv_v,
                              int32_t* mv_new) {
  const int lane = threadIdx.x & 31;
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + (threadIdx.x - lane); b < total;
       b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = b + lane;
    const int32_t v = i < total ? recv[2 * i] : -1;
    const bool has = v >= 0;
    const unsigned m = __ballot_sync(kFull, has);
    if (!m) continue;
    unsigned long long base = 0;
    if (lane == __ffs(m) - 1) base = atomicAdd(&ctl->logn, (unsigned long long)__popc(m));
    base = __shfl_sync(kFull, base, __ffs(m) - 1);
    if (has) {
      const unsigned long long p = base + __popc(m & ((1u << lane) - 1u));
      mv_v[p] = v;
      mv_new[p] = recv[2 * i + 1];
    }
  }
}
// Edge-balanced split: out[r] = first row u with rowptr[u] >= r*nnz/world (r = 1..world-1).
__global__ void k_dist_split(const int64_t* __restrict__ rowptr, int64_t n, int world, int64_t* out) {
  const int r = threadIdx.x;
  if (r > world) return;
  if (r == 0) { out[0] = 0; return; }
  if (r == world) { out[world] = n; return; }
  const int64_t nnz = rowptr[n], target = (int64_t)((__int128)r * nnz / world);
  int64_t lo = 0, hi = n;  // lower_bound
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (rowptr[mid] < target) lo = mid + 1; else hi = mid;
  }
  out[r] = lo;
}
__global__ void k_dist_shift_rowptr(int64_t* rowptr, int64_t v0, int64_t v1, int64_t add) {
  for (int64_t i = v0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < v1; i += (int64_t)gridDim.x * blockDim.x)
    rowptr[i] += add;
}
// Peer-memory commit of this rank's moves of one commit group (log [bounds[idx],
// logn)): the commit of Alg. 1 l.8-11 (C[i] = newComm[i], exact integer a_c /
// size_c deltas) applied to EVERY rank's replica -- the exchange is part of the
// commit (remote stores and atomics over NVLink, or the same memory for ranks
// sharing a GPU), so no move list crosses the interconnect and no all-gather runs.
__global__ void k_commit_p2p(DevCtl* ctl, int idx, const int32_t* __restrict__ mv_v,
                             const int32_t* __restrict__ mv_new, int32_t* __restrict__ mv_old,
                             const PeerPtrs* __restrict__ pp, int world, int rank, const uint32_t* __restrict__ k,
                             bool with_pcn) {
  const unsigned long long start = ctl->bounds[idx];
  const unsigned long long end = *(volatile unsigned long long*)&ctl->logn;
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->bounds[idx + 1] = end;
  const int32_t* Cl = pp->C[rank];
  for (unsigned long long p = start + blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; p < end;
       p += (unsigned long long)gridDim.x * blockDim.x) {
    const int32_t i = mv_v[p], t = mv_new[p];
    const int32_t old = Cl[i];  // i is this rank's vertex: no other rank writes C[i]
    mv_old[p] = old;
    const uint32_t ki = k[i];
    for (int q = 0; q < world; ++q) {
      uint32_t* w32 = reinterpret_cast<uint32_t*>(pp->ca[q]);
      w32[2 * (int64_t)i] = (uint32_t)t;
      pp->C[q][i] = t;
      if (with_pcn) pp->pcn[q][i].y = (uint32_t)t;
      atomicSub(&w32[2 * (int64_t)old + 1], ki);
      atomicAdd(&w32[2 * (int64_t)t + 1], ki);
      atomicSub(&pp->size[q][old], 1);
      atomicAdd(&pp->size[q][t], 1);
    }
  }
  __threadfence_system();  // the stores reach every replica before the barrier
}
// R15 for peer-memory commits: every rank undoes its own moves in every replica.
__global__ void k_revert_p2p(const DevCtl* ctl, const int32_t* __restrict__ mv_v, const int32_t* __restrict__ mv_new,
                             const int32_t* __restrict__ mv_old, const PeerPtrs* __restrict__ pp, int world,
                             const uint32_t* __restrict__ k) {
  const unsigned long long end = ctl->logn;
  for (unsigned long long p = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; p < end;
       p += (unsigned long long)gridDim.x * blockDim.x) {
    const int32_t i = mv_v[p], t = mv_new[p], old = mv_old[p];
    const uint32_t ki = k[i];
    for (int q = 0; q < world; ++q) {
      uint32_t* w32 = reinterpret_cast<uint32_t*>(pp->ca[q]);
      w32[2 * (int64_t)i] = (uint32_t)old;
      pp->C[q][i] = old;
      atomicSub(&w32[2 * (int64_t)t + 1], ki);
      atomicAdd(&w32[2 * (int64_t)old + 1], ki);
      atomicSub(&pp->size[q][t], 1);
      atomicAdd(&pp->size[q][old], 1);
    }
  }
  __threadfence_system();
}
__global__ void k_copy_u64(const unsigned long long* src, unsigned long long* dst) { *dst = *src; }
}  // namespace

// ------------------------------------------------------------------ context
DistCtx::~DistCtx() {
  for (void* p : opened) cudaIpcCloseMemHandle(p);
  for (void* p : rep_block)
    if (p) cudaFree(p);
  if (pcn_block) cudaFree(pcn_block);
  for (PeerPtrs* p : d_peers)
    if (p) cudaFree(p);
  if (d_bar) cudaFree(d_bar);
  delete comm;
}

int32_t dist_barrier(Handle& h) {
  // a one-word all-reduce: it completes on a rank only after every rank's preceding
  // stream work (the commit kernels and their system-scope fences) has completed
  return h.dist->comm->allreduce_u64(h.dist->d_bar, 1, h.stream);
}

int32_t dist_total_moved(Handle& h) {
  k_copy_u64<<<1, 1, 0, h.stream>>>(&h.ctl->logn, &h.ctl->gmoved);
  LV_LAUNCHED();
  if (!dist_p2p(h)) return LOUVAIN_OK;  // the all-gathered log already holds every rank's moves
  return h.dist->comm->allreduce_u64(&h.ctl->gmoved, 1, h.stream);
}

int32_t dist_bind_state(Handle& h, Level& L, int set) {
  DistCtx& D = *h.dist;
  if (L.n > D.rep_n) {
    set_error("distributed handle: level larger than the replica capacity");
    return LOUVAIN_E_STATE;
  }
  char* b = static_cast<char*>(D.rep_block[set]);
  L.ca = reinterpret_cast<uint2*>(b);
  L.size = reinterpret_cast<int32_t*>(b + 8 * (size_t)D.rep_n);
  L.C = reinterpret_cast<int32_t*>(b + 12 * (size_t)D.rep_n);
  L.rep_set = set;
  L.state_external = true;
  return LOUVAIN_OK;
}

int32_t dist_commit_p2p(Handle& h, Level& L, int bucket) {
  DistCtx& D = *h.dist;
  // every rank has decided the bucket against the same snapshot before any rank
  // writes into another's replica (Alg. 1 l.6-9: the commit follows all decisions)
  LV_TRY(dist_barrier(h));
  k_commit_p2p<<<148 * 4, 256, 0, h.stream>>>(h.ctl, bucket, L.mv_v, L.mv_new, L.mv_old, D.d_peers[L.rep_set],
                                             D.world, D.rank, L.k, h.pcn != nullptr);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return dist_barrier(h);
}

int32_t dist_revert_p2p(Handle& h, Level& L) {
  DistCtx& D = *h.dist;
  LV_TRY(dist_barrier(h));
  k_revert_p2p<<<148 * 4, 256, 0, h.stream>>>(h.ctl, L.mv_v, L.mv_new, L.mv_old, D.d_peers[L.rep_set], D.world, L.k);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return dist_barrier(h);
}

// Allocate the IPC-exportable replica sets and the delta-pass snapshot, exchange the
// IPC handles through the transport and map every peer's blocks.
static int32_t setup_p2p(Handle& h, int64_t n) {
  DistCtx& D = *h.dist;
  if (D.world > kMaxWorld) {
    set_error("LOUVAIN_DIST_P2P: at most 64 ranks");
    return LOUVAIN_E_UNSUPPORTED;
  }
  D.p2p = true;
  D.rep_n = std::max<int64_t>(n, 1);
  const size_t sb = 16 * (size_t)D.rep_n;
  for (auto& b : D.rep_block) LV_CUDA(cudaMalloc(&b, sb));
  LV_CUDA(cudaMalloc(&D.pcn_block, 8 * (size_t)D.rep_n));
  LV_CUDA(cudaMalloc(&D.d_bar, 8));
  LV_CUDA(cudaMemset(D.d_bar, 0, 8));
  constexpr int kBlocks = 4;
  cudaIpcMemHandle_t mine[kBlocks];
  void* blocks[kBlocks] = {D.rep_block[0], D.rep_block[1], D.rep_block[2], D.pcn_block};
  for (int b = 0; b < kBlocks; ++b) LV_CUDA(cudaIpcGetMemHandle(&mine[b], blocks[b]));
  char *dsend = nullptr, *drecv = nullptr;
  LV_TRY(dmalloc((void**)&dsend, sizeof mine, h.stream));
  LV_TRY(dmalloc((void**)&drecv, sizeof mine * D.world, h.stream));
  LV_CUDA(cudaMemcpyAsync(dsend, mine, sizeof mine, cudaMemcpyHostToDevice, h.stream));
  LV_TRY(D.comm->allgather(dsend, drecv, sizeof mine, h.stream));
  std::vector<cudaIpcMemHandle_t> all((size_t)kBlocks * D.world);
  LV_CUDA(cudaMemcpyAsync(all.data(), drecv, sizeof mine * D.world, cudaMemcpyDeviceToHost, h.stream));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  dfree(dsend, h.stream);
  dfree(drecv, h.stream);
  PeerPtrs hp[3];
  std::memset(hp, 0, sizeof hp);
  for (int q = 0; q < D.world; ++q) {
    void* base[kBlocks];
    for (int b = 0; b < kBlocks; ++b) {
      if (q == D.rank) {
        base[b] = blocks[b];
      } else {
        void* p = nullptr;
        LV_CUDA(cudaIpcOpenMemHandle(&p, all[(size_t)q * kBlocks + b], cudaIpcMemLazyEnablePeerAccess));
        D.opened.push_back(p);
        base[b] = p;
      }
    }
    for (int s = 0; s < 3; ++s) {
      char* c = static_cast<char*>(base[s]);
      hp[s].ca[q] = reinterpret_cast<uint2*>(c);
      hp[s].size[q] = reinterpret_cast<int32_t*>(c + 8 * (size_t)D.rep_n);
      hp[s].C[q] = reinterpret_cast<int32_t*>(c + 12 * (size_t)D.rep_n);
      hp[s].pcn[q] = static_cast<uint2*>(base[3]);
    }
  }
  for (int s = 0; s < 3; ++s) {
    LV_CUDA(cudaMalloc(&D.d_peers[s], sizeof(PeerPtrs)));
    LV_CUDA(cudaMemcpy(D.d_peers[s], &hp[s], sizeof(PeerPtrs), cudaMemcpyHostToDevice));
  }
  // level 0 of the handle lives in replica set 0 (its state is re-initialised there)
  Level& L = h.lv;
  dfree(L.ca, h.stream);
  dfree(L.size, h.stream);
  dfree(L.C, h.stream);
  LV_TRY(dist_bind_state(h, L, 0));
  L.k_ready = false;
  LV_TRY(level_setup(h, L));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  return dist_barrier(h);
}

int32_t dist_allreduce(Handle& h, unsigned long long* dev, size_t count) {
  if (!h.dist) return LOUVAIN_OK;
  return h.dist->comm->allreduce_u64(dev, count, h.stream);
}

int32_t dist_allgatherv(Handle& h, const void* send, void* recv, const std::vector<int64_t>& cnt,
                        const std::vector<int64_t>& displ, size_t elem) {
  return h.dist->comm->allgatherv(send, recv, cnt, displ, elem, h.stream);
}

static int32_t set_range(Level& L, int64_t lo, int64_t hi) {
  if (L.own_hi == hi && L.own_lo == lo) return LOUVAIN_OK;
  int64_t e[2] = {0, 0};
  LV_CUDA(cudaMemcpy(&e[0], L.rowptr + lo, 8, cudaMemcpyDeviceToHost));
  LV_CUDA(cudaMemcpy(&e[1], L.rowptr + hi, 8, cudaMemcpyDeviceToHost));
  L.own_lo = lo;
  L.own_hi = hi;
  L.own_e0 = e[0];
  L.own_e1 = e[1];
  L.bins_valid = false;
  return LOUVAIN_OK;
}

int32_t dist_set_level_range(Handle& h, Level& L, int level) {
  DistCtx& D = *h.dist;
  if (level == 0) return set_range(L, D.vlo0[D.rank], D.vlo0[D.rank + 1]);
  int64_t* d = nullptr;
  LV_TRY(dalloc(&d, D.world + 1, h.stream));
  k_dist_split<<<1, 1024, 0, h.stream>>>(L.rowptr, L.n, D.world, d);
  LV_LAUNCHED();
  std::vector<int64_t> v(D.world + 1);
  LV_CUDA(cudaMemcpyAsync(v.data(), d, 8 * (D.world + 1), cudaMemcpyDeviceToHost, h.stream));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  dfree(d, h.stream);
  for (int r = 1; r <= D.world; ++r) v[r] = std::max(v[r], v[r - 1]);
  return set_range(L, v[D.rank], v[D.rank + 1]);
}

// After the level's binning: the owned bucket sizes of every rank, so each
// bucket's exchange has a capacity all ranks agree on without a per-bucket sync.
int32_t dist_after_binning(Handle& h, Level& L) {
  DistCtx& D = *h.dist;
  int64_t mine[8];
  mine[0] = 0;
  for (int b = 1; b <= 7; ++b) {
    mine[b] = L.class_off[kSubPerBucket * (b + 1)] - L.class_off[kSubPerBucket * b];
    mine[0] += mine[b];
  }
  int64_t *ds = nullptr, *dr = nullptr;
  LV_TRY(dalloc(&ds, 8, h.stream));
  LV_TRY(dalloc(&dr, 8 * (size_t)D.world, h.stream));
  LV_CUDA(cudaMemcpyAsync(ds, mine, sizeof mine, cudaMemcpyHostToDevice, h.stream));
  LV_TRY(D.comm->allgather(ds, dr, sizeof mine, h.stream));
  std::vector<int64_t> all(8 * (size_t)D.world);
  LV_CUDA(cudaMemcpyAsync(all.data(), dr, 64 * (size_t)D.world, cudaMemcpyDeviceToHost, h.stream));
  LV_CUDA(cudaStreamSynchronize(h.stream));
  dfree(ds, h.stream);
  dfree(dr, h.stream);
  int64_t mx = 0;
  for (int g = 0; g < 8; ++g) {
    D.cap[g] = 0;
    for (int r = 0; r < D.world; ++r) D.cap[g] = std::max(D.cap[g], all[8 * (size_t)r + g]);
    mx = std::max(mx, D.cap[g]);
  }
  const size_t need_s = 2 * (size_t)std::max<int64_t>(mx, 1), need_r = need_s * (size_t)D.world;
  if (D.sbuf_n < need_s) {
    dfree(D.sbuf, h.stream);
    LV_TRY(dalloc(&D.sbuf, need_s, h.stream));
    D.sbuf_n = need_s;
  }
  if (D.rbuf_n < need_r) {
    dfree(D.rbuf, h.stream);
    LV_TRY(dalloc(&D.rbuf, need_r, h.stream));
    D.rbuf_n = need_r;
  }
  return LOUVAIN_OK;
}

// The exchange of one commit group (bucket b under BIN_SYNC, group 0 = the whole
// sweep under RELAXED), between this rank's decisions and the commit.
int32_t dist_exchange(Handle& h, Level& L, int commit_idx, int group) {
  DistCtx& D = *h.dist;
  const int64_t cap = D.cap[group];
  if (cap == 0) return LOUVAIN_OK;
  cudaStream_t s = h.stream;
  k_dist_pack<<<grid_for(cap, 256), 256, 0, s>>>(h.ctl, commit_idx, L.mv_v, L.mv_new, cap, D.sbuf);
  LV_LAUNCHED();
  k_dist_rewind<<<1, 1, 0, s>>>(h.ctl, commit_idx);
  LV_LAUNCHED();
  LV_TRY(D.comm->allgather(D.sbuf, D.rbuf, 8 * (size_t)cap, s));
  const int64_t total = cap * D.world;
  k_dist_append<<<grid_for(total, 256), 256, 0, s>>>(h.ctl, D.rbuf, total, L.mv_v, L.mv_new);
  LV_LAUNCHED();
  LV_CUDA(cudaGetLastError());
  return LOUVAIN_OK;
}

void dist_free(Handle& h) {
  if (!h.dist) return;
  dfree(h.dist->sbuf, h.stream);
  dfree(h.dist->rbuf, h.stream);
  delete h.dist;
  h.dist = nullptr;
}

// Assemble the replicated level-0 CSR from every rank's rows and build the handle.
int32_t create_dist(Comm* comm, int64_t n, int64_t v_begin, int64_t v_end, const int64_t* rowptr_local,
                    const int32_t* col_local, const uint32_t* w_local, uint32_t flags, void* cuda_stream,
                    louvain_graph_t* out) {
  std::unique_ptr<Comm> cp(comm);
  const int world = comm->world, rank = comm->rank;
  *out = nullptr;
  if (n < 0 || v_begin < 0 || v_end < v_begin || v_end > n || !rowptr_local || n > INT32_MAX - 1) {
    set_error("louvain_create_csr_dist: need 0 <= v_begin <= v_end <= n < 2^31 - 1 and rowptr_local");
    return LOUVAIN_E_INVALID_ARG;
  }
  cudaStream_t s0 = cuda_stream ? (cudaStream_t)cuda_stream : nullptr;
  const int64_t rows = v_end - v_begin;
  int64_t r0 = 0, nnz_local = 0;
  LV_CUDA(cudaMemcpy(&r0, rowptr_local, 8, cudaMemcpyDefault));
  LV_CUDA(cudaMemcpy(&nnz_local, rowptr_local + rows, 8, cudaMemcpyDefault));
  if (r0 != 0 || nnz_local < 0 || (nnz_local > 0 && !col_local)) {
    set_error("louvain_create_csr_dist: rowptr_local must start at 0; col_local required");
    return LOUVAIN_E_INVALID_ARG;
  }
  // metadata of every rank: (v_begin, v_end, nnz_local, n, weighted)
  int64_t meta[5] = {v_begin, v_end, nnz_local, n, w_local ? 1 : 0};
  int64_t *dm = nullptr, *dall = nullptr;
  LV_TRY(dmalloc((void**)&dm, sizeof meta, s0));
  LV_TRY(dmalloc((void**)&dall, sizeof meta * world, s0));
  LV_CUDA(cudaMemcpyAsync(dm, meta, sizeof meta, cudaMemcpyHostToDevice, s0));
  LV_TRY(comm->allgather(dm, dall, sizeof meta, s0));
  std::vector<int64_t> all(5 * (size_t)world);
  LV_CUDA(cudaMemcpyAsync(all.data(), dall, sizeof meta * world, cudaMemcpyDeviceToHost, s0));
  LV_CUDA(cudaStreamSynchronize(s0));
  dfree(dm, s0);
  dfree(dall, s0);
  std::vector<int64_t> vlo(world + 1), cnt_v(world), cnt_e(world), dv(world), de(world);
  bool ok = true;
  int64_t e_off = 0;
  for (int r = 0; r < world; ++r) {
    const int64_t* m = &all[5 * (size_t)r];
    ok = ok && m[3] == n && m[4] == meta[4] && m[0] == (r == 0 ? 0 : all[5 * (size_t)(r - 1) + 1]);
    vlo[r] = m[0];
    cnt_v[r] = m[1] - m[0];
    cnt_e[r] = m[2];
    dv[r] = m[0];
    de[r] = e_off;
    e_off += m[2];
  }
  vlo[world] = all[5 * (size_t)(world - 1) + 1];
  ok = ok && vlo[world] == n;
  if (!ok) {
    set_error("louvain_create_csr_dist: ranks' rows must be contiguous in rank order, cover [0, n), "
              "agree on n and on weights");
    return LOUVAIN_E_INVALID_ARG;
  }
  const int64_t nnz = e_off;
  // local pieces as device memory
  int64_t* drow_l = nullptr;
  int32_t* dcol_l = nullptr;
  uint32_t* dw_l = nullptr;
  LV_TRY(dalloc(&drow_l, rows + 1, s0));
  LV_CUDA(cudaMemcpyAsync(drow_l, rowptr_local, 8 * (size_t)(rows + 1), cudaMemcpyDefault, s0));
  LV_TRY(dalloc(&dcol_l, std::max<int64_t>(nnz_local, 1), s0));
  if (nnz_local) LV_CUDA(cudaMemcpyAsync(dcol_l, col_local, 4 * (size_t)nnz_local, cudaMemcpyDefault, s0));
  if (w_local) {
    LV_TRY(dalloc(&dw_l, std::max<int64_t>(nnz_local, 1), s0));
    if (nnz_local) LV_CUDA(cudaMemcpyAsync(dw_l, w_local, 4 * (size_t)nnz_local, cudaMemcpyDefault, s0));
  }
  // replicated CSR
  int64_t* rowptr = nullptr;
  int32_t* col = nullptr;
  uint32_t* w = nullptr;
  LV_TRY(dalloc(&rowptr, n + 1, s0));
  LV_TRY(dalloc(&col, std::max<int64_t>(nnz, 1), s0));
  if (w_local) LV_TRY(dalloc(&w, std::max<int64_t>(nnz, 1), s0));
  LV_TRY(comm->allgatherv(drow_l, rowptr, cnt_v, dv, 8, s0));
  LV_TRY(comm->allgatherv(dcol_l, col, cnt_e, de, 4, s0));
  if (w_local) LV_TRY(comm->allgatherv(dw_l, w, cnt_e, de, 4, s0));
  for (int r = 0; r < world; ++r)
    if (cnt_v[r] && de[r]) {
      k_dist_shift_rowptr<<<grid_for(cnt_v[r], 256), 256, 0, s0>>>(rowptr, vlo[r], vlo[r + 1], de[r]);
      LV_LAUNCHED();
    }
  LV_CUDA(cudaMemcpyAsync(rowptr + n, &nnz, 8, cudaMemcpyHostToDevice, s0));
  LV_CUDA(cudaStreamSynchronize(s0));  // &nnz is a host stack value
  dfree(drow_l, s0);
  dfree(dcol_l, s0);
  dfree(dw_l, s0);
  if (flags & LOUVAIN_VALIDATE) {
    std::vector<int64_t> hr(n + 1);
    std::vector<int32_t> hc(nnz);
    std::vector<uint32_t> hw(w ? nnz : 0);
    LV_CUDA(cudaMemcpy(hr.data(), rowptr, 8 * (n + 1), cudaMemcpyDeviceToHost));
    if (nnz) LV_CUDA(cudaMemcpy(hc.data(), col, 4 * nnz, cudaMemcpyDeviceToHost));
    if (w && nnz) LV_CUDA(cudaMemcpy(hw.data(), w, 4 * nnz, cudaMemcpyDeviceToHost));
    int32_t rc = validate_csr_host(n, nnz, hr.data(), hc.data(), w ? hw.data() : nullptr, true, nullptr);
    if (rc) {
      dfree(rowptr, s0); dfree(col, s0); dfree(w, s0);
      cudaStreamSynchronize(s0);
      return rc;
    }
  }
  louvain_graph_t g = nullptr;
  int32_t rc = create_from_device(n, nnz, rowptr, col, w, cuda_stream, &g);
  if (rc) return rc;  // create_from_device took ownership of the arrays
  Handle& h = g->h;
  h.dist = new DistCtx();
  h.dist->comm = cp.release();
  h.dist->rank = rank;
  h.dist->world = world;
  h.dist->vlo0 = vlo;
  rc = set_range(h.lv, vlo[rank], vlo[rank + 1]);
  if (!rc && (flags & LOUVAIN_DIST_P2P)) rc = setup_p2p(h, n);
  if (rc) {
    louvain_destroy(g);
    return rc;
  }
  *out = g;
  return LOUVAIN_OK;
}

}  // namespace lv

using namespace lv;
#define LV_API extern "C" __attribute__((visibility("default")))

LV_API int32_t louvain_dist_unique_id(uint8_t id[128]) {
  if (!id) {
    set_error("null id");
    return LOUVAIN_E_INVALID_ARG;
  }
#if defined(LOUVAIN_HAVE_NCCL_HEADERS)
  static_assert(sizeof(ncclUniqueId) == 128, "NCCL unique id size");
  if (!nccl().ok) {
    set_error(nccl().err);
    return LOUVAIN_E_UNSUPPORTED;
  }
  ncclUniqueId u;
  LV_NCCL(nccl().GetUniqueId(&u));
  std::memcpy(id, &u, 128);
  return LOUVAIN_OK;
#else
  set_error("built without NCCL headers");
  return LOUVAIN_E_UNSUPPORTED;
#endif
}

LV_API int32_t louvain_create_csr_dist(int64_t n, int64_t v_begin, int64_t v_end, const int64_t* rowptr_local,
                                       const int32_t* col_local, const uint32_t* w_local, uint32_t flags,
                                       int32_t rank, int32_t world, const uint8_t id[128], void* cuda_stream,
                                       louvain_graph_t* out) {
  if (!out || !id || world < 1 || rank < 0 || rank >= world) {
    set_error("louvain_create_csr_dist: out, id and 0 <= rank < world required");
    return LOUVAIN_E_INVALID_ARG;
  }
#if defined(LOUVAIN_HAVE_NCCL_HEADERS)
  if (!nccl().ok) {
    set_error(nccl().err);
    return LOUVAIN_E_UNSUPPORTED;
  }
  NcclComm* c = new NcclComm();
  c->rank = rank;
  c->world = world;
  ncclUniqueId u;
  std::memcpy(&u, id, 128);
  ncclResult_t r = nccl().CommInitRank(&c->comm, world, u, rank);
  if (r != ncclSuccess) {
    delete c;
    return nccl_fail(r, "ncclCommInitRank");
  }
  return create_dist(c, n, v_begin, v_end, rowptr_local, col_local, w_local, flags, cuda_stream, out);
#else
  (void)n; (void)v_begin; (void)v_end; (void)rowptr_local; (void)col_local; (void)w_local; (void)flags;
  (void)cuda_stream;
  set_error("built without NCCL headers");
  return LOUVAIN_E_UNSUPPORTED;
#endif
}

LV_API int32_t louvain_create_csr_dist_host(int64_t n, int64_t v_begin, int64_t v_end, const int64_t* rowptr_local,
                                            const int32_t* col_local, const uint32_t* w_local, uint32_t flags,
                                            int32_t rank, int32_t world, const louvain_host_comm_t* comm,
                                            void* cuda_stream, louvain_graph_t* out) {
  if (!out || !comm || !comm->allgather || !comm->allreduce_u64 || world < 1 || rank < 0 || rank >= world) {
    set_error("louvain_create_csr_dist_host: out, both callbacks and 0 <= rank < world required");
    return LOUVAIN_E_INVALID_ARG;
  }
  HostComm* c = new HostComm();
  c->rank = rank;
  c->world = world;
  c->cb = *comm;
  return create_dist(c, n, v_begin, v_end, rowptr_local, col_local, w_local, flags, cuda_stream, out);
}

// Host-only helper (no device work): the edge-balanced split the library uses
// at levels >= 1, for callers choosing level-0 rows: bounds[r] = first row u
// with rowptr[u] >= r*nnz/world, bounds[0] = 0, bounds[world] = n.
LV_API int32_t louvain_dist_ranges(int64_t n, const int64_t* rowptr, int32_t world, int64_t* bounds) {
  if (n < 0 || !rowptr || world < 1 || !bounds) {
    set_error("louvain_dist_ranges: n >= 0, rowptr, world >= 1, bounds[world+1] required");
    return LOUVAIN_E_INVALID_ARG;
  }
  const int64_t nnz = rowptr[n];
  bounds[0] = 0;
  for (int r = 1; r < world; ++r) {
    const int64_t target = (int64_t)((__int128)r * nnz / world);
    bounds[r] = std::max<int64_t>(bounds[r - 1], std::lower_bound(rowptr, rowptr + n + 1, target) - rowptr);
    bounds[r] = std::min<int64_t>(bounds[r], n);
  }
  bounds[world] = n;
  return LOUVAIN_OK;
}
