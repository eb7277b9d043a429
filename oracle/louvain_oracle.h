/* louvain_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded C reference of the GPU Louvain method of
 * Naim, Manne, Halappanavar and Tumeo ("Community Detection on the GPU",
 * IPDPS'17; /root/reference/PAPER.md, cited P:<line>).  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load it.  It shares no code with the CUDA path
 * (paper_conf_ipps_naimmht17_b200/) and includes none of its headers.
 *
 * Readings of the paper (R1..R26) are those of SURVEY.md 8(c), listed in
 * DESIGN.md.  All arithmetic that decides anything is exact integer
 * arithmetic (R4); doubles are produced only for reporting Q.
 */
#ifndef LOUVAIN_ORACLE_H
#define LOUVAIN_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_BIN_SYNC = 0, ORC_RELAXED = 1, ORC_SEQ = 2, ORC_SEQ_ADAPTIVE = 3 };

typedef struct {
  int32_t mode;               /* ORC_* */
  int32_t singleton_rule;     /* 1 veto-after-argmax, 2 filter, 0 off (R8); SEQ ignores it */
  int32_t revert_on_decrease; /* R15 */
  int32_t th_bin_exp, th_final_exp; /* theta = 10^-exp */
  int64_t size_limit;         /* n > limit -> theta_bin */
  int64_t deg_bounds[6];
  int32_t max_sweeps, max_levels; /* 0 = unlimited */
} orc_params;

#define ORC_MAX_LEVELS 256
typedef struct {
  int32_t levels, sweeps;
  int64_t n[ORC_MAX_LEVELS], nnz[ORC_MAX_LEVELS];
  int32_t sweeps_per_level[ORC_MAX_LEVELS];
  int64_t moved_per_level[ORC_MAX_LEVELS];
  int64_t num_start[ORC_MAX_LEVELS], num_end[ORC_MAX_LEVELS];
  uint64_t L, S, W; /* final exact parts: Q = (L*W - S) / W^2 */
  double q;
} orc_stats;

void orc_params_default(orc_params* p);

/* Eq. (1), as exact integers: L = sum_i e_{i->C(i)} with self-loops
 * included (R2), S = sum_c a_c^2, W = 2m = sum_i k_i (R1).  Returns 0, or -3 if
 * W exceeds the int64 guard 3,037,000,499 (R4). */
int orc_modularity(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                   const int32_t* C, uint64_t* L, uint64_t* S, uint64_t* W);

/* a_c and size_c of partition C (P:78-80 a_c = sum_{i in c} k_i). */
void orc_totals(int64_t n, const int64_t* rowptr, const uint32_t* w, const int32_t* C,
                uint64_t* a, int64_t* size);

/* Alg. 2 computeMove with Eq. (2) in integer form and the rules
 * of P:172: returns the new community of vertex i given the snapshot (C, a, size). */
int32_t orc_decide(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                   const int32_t* C, const uint64_t* a, const int64_t* size, uint64_t W,
                   int64_t i, int32_t singleton_rule);
/* orc_decide for a list of vertices, all against the same snapshot. */
void orc_decide_batch(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                      const int32_t* C, const uint64_t* a, const int64_t* size, uint64_t W,
                      int32_t singleton_rule, int64_t nv, const int64_t* verts, int32_t* out);

/* One iteration of Alg. 1's repeat body: buckets 1..7 in order,
 * decisions on the bucket-start snapshot, commit after each bucket (BIN_SYNC),
 * or a single all-vertex bucket (RELAXED), or sequential immediate moves
 * (SEQ).  Updates C, a, size in place; returns the number of moves. */
int64_t orc_sweep(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                  const orc_params* p, int32_t* C, uint64_t* a, int64_t* size, uint64_t W);
/* orc_sweep that also returns D (measurement only, SURVEY 8(d) byte model): the
 * number of distinct (vertex, candidate label != own) pairs the sweep's
 * decisions evaluated, each against its own bucket-start snapshot. */
int64_t orc_sweep_counted(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                          const orc_params* p, int32_t* C, uint64_t* a, int64_t* size, uint64_t W,
                          int64_t* D_out);

/* Alg. 3 CONTRACT with R17/R18.  Outputs go to caller buffers of
 * capacity rowptr_out[n+1], col_out[nnz], w_out[nnz], map_out[n].  Returns n'. */
int64_t orc_contract(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                     const int32_t* C, int64_t* rowptr_out, int32_t* col_out, uint32_t* w_out,
                     int64_t* nnz_out, int32_t* map_out);

/* Multilevel driver (SURVEY 8(c) listing).
 * labels_out[n0] receives the final community of every input vertex. */
int orc_louvain(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                const orc_params* p, int32_t* labels_out, orc_stats* stats);

#ifdef __cplusplus
}
#endif
#endif
