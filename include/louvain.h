/* louvain.h -- C-ABI of the B200-native GPU Louvain hot path.
 *
 * Method: Naim, Manne, Halappanavar, Tumeo, "Community Detection on the GPU"
 * (IPDPS'17).  Citations "P:<line>" refer to /root/reference/PAPER.md (a text
 * extraction of the paper); "R<k>" to the readings of SURVEY.md 8(c), restated
 * in DESIGN.md.  Implemented by liblouvain.so (hand-written CUDA for sm_100a).
 *
 * Conventions (every function):
 *  - extern "C", returns int32_t status: LOUVAIN_OK (0) or a negative code;
 *    never throws, never exits; louvain_last_error() gives a thread-local message.
 *  - Graph input: undirected, positive integer weights, stored as
 *    CSR with BOTH directions of every non-loop edge and each self-loop ONCE
 *    (R1).  rowptr int64[n+1], col int32[nnz], w uint32[nnz] (NULL = all 1).
 *    Rows need not be sorted.  k_i = row sum, W = 2m = sum_i k_i.
 *  - Input pointers may be host or device memory (detected with
 *    cudaPointerGetAttributes); they are caller-owned, copied during the call
 *    and not retained (except with LOUVAIN_BORROW, below).
 *  - Output buffers are caller-allocated, host or device, of the stated length.
 *  - A handle owns all device memory of one level graph and its partition state
 *    (C, a_c, size_c).  It is bound to the device current at creation and to one
 *    stream (NULL -> a library-owned stream).  Calls that return scalars
 *    synchronise that stream.  A handle is not thread-safe; distinct handles are
 *    independent.
 *  - Arithmetic is exact integers (R4): e, k, a in uint32, gains
 *    s = W*e - k*a in int64, so W must be <= 3,037,000,499 (else
 *    LOUVAIN_E_OVERFLOW).  Q is reported as exact parts plus a double.
 */
#ifndef LOUVAIN_H
#define LOUVAIN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define LOUVAIN_OK 0
#define LOUVAIN_E_INVALID_ARG (-1)
#define LOUVAIN_E_INVALID_GRAPH (-2)
#define LOUVAIN_E_OVERFLOW (-3)
#define LOUVAIN_E_NOMEM (-4)
#define LOUVAIN_E_CUDA (-5)
#define LOUVAIN_E_NCCL (-6)
#define LOUVAIN_E_STATE (-7)       /* handle poisoned by a sticky CUDA error */
#define LOUVAIN_E_UNSUPPORTED (-8)

/* louvain_create_csr flags */
#define LOUVAIN_VALIDATE 1u /* full O(n + nnz) validation incl. symmetry; else O(1) checks only */
#define LOUVAIN_BORROW 2u   /* device inputs are used in place (caller keeps them alive, unmodified) */
#define LOUVAIN_DIST_P2P 4u /* distributed handles: commits write every rank's replica through peer
                               memory (CUDA IPC / NVLink P2P) + one barrier per bucket, no all-gather */

/* modes */
#define LOUVAIN_MODE_BIN_SYNC 0 /* Alg. 1: commit after each degree bucket (default) */
#define LOUVAIN_MODE_RELAXED 1  /* one commit per sweep ("relaxed") */

typedef struct louvain_graph_s* louvain_graph_t;

/* Q = (L*W - S) / W^2 (Eq. 1), exact parts; S = S_hi*2^64 + S_lo. */
typedef struct {
  uint64_t L, S_lo, S_hi, W;
  double q;
} louvain_qnum_t;

typedef struct {
  int32_t mode;               /* LOUVAIN_MODE_* */
  int32_t singleton_rule;     /* 1 veto-after-argmax (default) | 2 filter | 0 off (R8) */
  int32_t revert_on_decrease; /* 1 (default): a sweep that lowers Q is undone and ends the phase (R15) */
  int32_t th_bin_exp, th_final_exp; /* theta = 10^-exp; defaults 2, 6 */
  int64_t size_limit;         /* 100000: n > limit -> theta_bin, else theta_final */
  int64_t deg_bounds[6];      /* bucket bounds {4,8,16,32,84,319} */
  int32_t max_sweeps, max_levels; /* safety caps; 0 = unlimited */
} louvain_params_t;

#define LOUVAIN_MAX_LEVELS 256
typedef struct {
  int32_t levels, sweeps;
  int64_t n[LOUVAIN_MAX_LEVELS], nnz[LOUVAIN_MAX_LEVELS];
  int32_t sweeps_per_level[LOUVAIN_MAX_LEVELS];
  int64_t moved_per_level[LOUVAIN_MAX_LEVELS];
  int64_t num_start[LOUVAIN_MAX_LEVELS], num_end[LOUVAIN_MAX_LEVELS]; /* L*W - S per level */
  double t_opt_ms[LOUVAIN_MAX_LEVELS], t_agg_ms[LOUVAIN_MAX_LEVELS];
  double t_total_ms;
  /* measurement: sweep bodies only (buckets + commits, no modularity pass) */
  double t_sweep_ms_total;    /* all sweeps of all levels */
  double t_sweep_ms_first;    /* level 0, sweep 1 */
  double t_modularity_ms_total;
  int64_t edges_swept;        /* sum over executed sweeps of nnz of their level */
  int64_t moved_first;        /* moves of level 0, sweep 1 */
  double t_sweep_ms_level0[32]; /* each of the first 32 level-0 sweep bodies (median / phase-1 rates) */
  int64_t kernel_launches;    /* explicit kernel launches by the library during the call */
  int64_t cub_calls;          /* device-wide CUB primitives (scan/sort/reduce) during the call */
  louvain_qnum_t q;
} louvain_stats_t;

/* Fill *p with the paper's defaults (R8, R15). */
void louvain_params_default(louvain_params_t* p);

/* Create a level graph from CSR.  n >= 0, nnz >= 0, rowptr[n+1],
 * col[nnz] in [0,n), w[nnz] > 0 or NULL.  The partition starts as singletons
 * (P:164).  Errors: INVALID_ARG (null/negative), INVALID_GRAPH (validation),
 * OVERFLOW (W > 3,037,000,499), NOMEM, CUDA. */
int32_t louvain_create_csr(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                           const uint32_t* w, uint32_t flags, void* cuda_stream, louvain_graph_t* out);
/* Release a handle (NULL is a no-op). */
int32_t louvain_destroy(louvain_graph_t g);
/* n, nnz, W = 2m of the handle's graph (any output may be NULL). */
int32_t louvain_get_info(louvain_graph_t g, int64_t* n, int64_t* nnz, uint64_t* W);
/* Copy the handle's CSR out: rowptr[n+1], col[nnz], w[nnz] (any may be NULL;
 * w of a unit-weight graph is written as 1s). */
int32_t louvain_get_csr(louvain_graph_t g, int64_t* rowptr, int32_t* col, uint32_t* w);
/* Set the partition C (labels[n], each in [0,n)); NULL = singletons.  a_c and
 * size_c are recomputed. */
int32_t louvain_set_labels(louvain_graph_t g, const int32_t* labels);
/* Copy the current partition C[n]. */
int32_t louvain_get_labels(louvain_graph_t g, int32_t* labels_out);
/* Copy a_c (uint32[n]) and size_c (int32[n]) of the current partition (either may be NULL). */
int32_t louvain_get_totals(louvain_graph_t g, uint32_t* a_out, int32_t* size_out);

/* Exactly one iteration of Alg. 1's repeat body: buckets 1..7 in
 * ascending order; every vertex of a bucket runs computeMove (Alg. 2)
 * against the bucket-start state with Eq. (2) in integer form and the rules of
 * P:172 (R5-R9), then the bucket's moves are committed (C, a_c, size_c).  No
 * revert and no stop decision.  *moved = vertices that changed community;
 * q_after (may be NULL) = modularity after the sweep. */
int32_t louvain_sweep(louvain_graph_t g, const louvain_params_t* p, int64_t* moved, louvain_qnum_t* q_after);
/* Eq. (1) of `labels` (n entries; NULL = current partition), exact parts. */
int32_t louvain_modularity(louvain_graph_t g, const int32_t* labels, louvain_qnum_t* q);
/* Alg. 3 CONTRACT: communities of the current partition become the
 * vertices of *next, numbered consecutively in label order (R17); parallel
 * edges merge by summing weights and intra-community entries form the
 * self-loop (R18); rows sorted by column.  map_out[n] (may be NULL)
 * receives the new vertex of every vertex.  *next is a new handle on g's stream
 * (or on its own library stream if g's stream is library-owned). */
int32_t louvain_aggregate(louvain_graph_t g, louvain_graph_t* next, int32_t* map_out);
/* Full multilevel Louvain from singletons: phases of
 * sweeps with the threshold schedule of P:330-334 (R13-R16), contraction
 * between levels.  labels_out[n] (may be NULL): final community of every
 * vertex; q_final / stats may be NULL.  On return the handle's partition is
 * the final one. */
int32_t louvain_run(louvain_graph_t g, const louvain_params_t* p, int32_t* labels_out, louvain_qnum_t* q_final,
                    louvain_stats_t* stats);
/* Thread-local message of the last error ("" if none). */
const char* louvain_last_error(void);
/* Free the device memory the library keeps between handles: the scratch
 * buffers of the most recently destroyed handle per device (reused by the next
 * handle, buffer by buffer in the role each served; bounded to one handle's set
 * per device) and the idle blocks of the
 * library's private stream-ordered memory pool.  Never needed for correctness:
 * an allocation failure releases both and retries once. */
int32_t louvain_release_cache(void);
/* Process-wide counters of the kernels (and CUB device calls) this library has
 * launched so far, on every handle; either pointer may be NULL.  Diagnostics:
 * the difference around a call counts its launches (louvain_stats_t reports
 * the same for louvain_run). */
void louvain_launch_counts(int64_t* kernel_launches, int64_t* cub_calls);

/* ---- sharded sweep primitives (multi-GPU, one process per GPU) ----
 * Every rank holds the same level graph and a replica of the partition state.
 * Rank r owns the vertex range [v_begin, v_end): it decides only its own
 * vertices, exchanges the moves of each bucket with the other ranks (the
 * caller's collective, e.g. an NCCL all-gather through torch.distributed), and
 * every rank commits ALL moves of the bucket, so the replicas stay bit-identical
 * (integer updates, order-independent).  A single rank owning [0, n) reproduces
 * louvain_sweep exactly. */
/* Restrict decisions (and louvain_modularity_owned's L) to [v_begin, v_end). */
int32_t louvain_set_owned_range(louvain_graph_t g, int64_t v_begin, int64_t v_end);
/* Start a sweep: clears the sweep's move log (the revert record, R15). */
int32_t louvain_begin_sweep(louvain_graph_t g);
/* computeMove (Alg. 2) for the owned vertices of bucket `bucket` (1..7) against
 * the current state, without committing.  moves_out: int32 pairs (v, new),
 * capacity `cap` pairs (host or device); *count = moves written.  Bucket
 * bounds come from p->deg_bounds. */
int32_t louvain_decide_bucket(louvain_graph_t g, const louvain_params_t* p, int32_t bucket, int32_t* moves_out,
                              int64_t cap, int64_t* count);
/* Commit `count` moves (v, new) (any owner; each v at most once per sweep):
 * C, a_c, size_c updated with exact integer deltas (Alg. 1 l.8-11) and the
 * moves appended to the sweep's log. */
int32_t louvain_commit_moves(louvain_graph_t g, const int32_t* moves, int64_t count);
/* Undo every move committed since louvain_begin_sweep (R15). */
int32_t louvain_revert_sweep(louvain_graph_t g);
/* Label composition across levels (R22): lab[i] = map[lab[i]] for i < n0
 * (device pointers; runs on `cuda_stream`, NULL = default stream). */
int32_t louvain_compose_labels(int32_t* lab, int64_t n0, const int32_t* map, void* cuda_stream);
/* Eq. (1) parts of the current partition with L summed over the owned rows
 * only (the ranks' L add up to the graph's L); S and W are global. */
int32_t louvain_modularity_owned(louvain_graph_t g, uint64_t* L_owned, uint64_t* S, uint64_t* W);

/* ---- multi-GPU: the vertex-sharded run inside the library ----
 * One process per GPU, one distributed handle per rank.  Every bucket decides on
 * one snapshot (Alg. 1 l.6-7), so rank r runs computeMove (Alg. 2) for
 * its own edge-balanced vertex range only; after each bucket the ranks' moves
 * are all-gathered and every rank commits all of them to its replica of
 * (C, a_c, size_c) with the same exact integer updates (Alg. 1 l.8-11), so the
 * replicas stay bit-identical; Eq. (1) after a sweep is all-reduced (partial L
 * change of the owned moved rows).  The level graph is replicated on every rank;
 * contraction (Alg. 3) is sharded by new vertex (each rank merges the member rows
 * of its share of the communities) and the merged rows are all-gathered.
 * Every louvain_* call on a distributed handle that runs a sweep
 * (louvain_sweep, louvain_run) is COLLECTIVE over its ranks; the other calls are
 * local.  Results equal the single-GPU ones bit for bit (and oracle (b)).
 * The per-bucket primitives above must not be used on a distributed handle. */

/* Host-side transport: both callbacks get host buffers and return 0 on success.
 * allgather: every rank contributes `bytes` bytes from `send`; `recv` receives
 * world * bytes, rank-major.  allreduce_u64: in-place sum of `count` uint64
 * values over the ranks (modular).  Used with any process group (e.g. gloo), and
 * where NCCL cannot run (several ranks sharing one GPU). */
typedef struct {
  void* user;
  int32_t (*allgather)(void* user, const void* send, void* recv, int64_t bytes);
  int32_t (*allreduce_u64)(void* user, uint64_t* data, int64_t count);
} louvain_host_comm_t;

/* A new NCCL unique id (128 bytes) for louvain_create_csr_dist; call on one rank
 * and broadcast it (e.g. torch.distributed.broadcast_object_list).
 * Errors: UNSUPPORTED (libnccl.so.2 cannot be loaded), NCCL. */
int32_t louvain_dist_unique_id(uint8_t id[128]);
/* Collective over `world` ranks.  Rank `rank` passes its rows [v_begin, v_end)
 * of the n-vertex graph (the ranks' ranges contiguous in rank order and covering
 * [0, n)): rowptr_local[v_end - v_begin + 1] starting at 0, col_local (GLOBAL
 * column ids) and w_local (NULL on every rank = unit weights), host or device.
 * The handle is bound to the current device and to cuda_stream; NCCL
 * communicator from `id`.  flags: LOUVAIN_VALIDATE (the assembled graph).
 * louvain_dist_ranges gives the edge-balanced ranges the library itself uses for
 * contracted levels.  Errors: INVALID_ARG (ranges / n / weights disagree across
 * ranks), INVALID_GRAPH, OVERFLOW, NOMEM, CUDA, NCCL, UNSUPPORTED. */
int32_t louvain_create_csr_dist(int64_t n, int64_t v_begin, int64_t v_end, const int64_t* rowptr_local,
                                const int32_t* col_local, const uint32_t* w_local, uint32_t flags, int32_t rank,
                                int32_t world, const uint8_t id[128], void* cuda_stream, louvain_graph_t* out);
/* Same, with the host-side transport `comm` (copied; the callbacks and `user`
 * must stay valid for the handle's lifetime). */
int32_t louvain_create_csr_dist_host(int64_t n, int64_t v_begin, int64_t v_end, const int64_t* rowptr_local,
                                     const int32_t* col_local, const uint32_t* w_local, uint32_t flags,
                                     int32_t rank, int32_t world, const louvain_host_comm_t* comm,
                                     void* cuda_stream, louvain_graph_t* out);
/* Host-only (no device work): edge-balanced contiguous ranges of a CSR,
 * bounds[world + 1]: bounds[r] = first row u with rowptr[u] >= r*nnz/world. */
int32_t louvain_dist_ranges(int64_t n, const int64_t* rowptr, int32_t world, int64_t* bounds);

#ifdef __cplusplus
}
#endif
#endif
