/* graphgen.h -- seeded synthetic-graph generators (input module).
 *
 * This library is shared by the oracle side and the CUDA side as the ONLY
 * common code: it produces inputs (CSR graphs with unit weights) and holds
 * none of the Louvain method's arithmetic.  Every generator is a pure function
 * of its parameters and seed (counter-based Philox, gg_philox.h), and the
 * host and device builders of the same graph are bit-identical.
 *
 * Output graphs follow SURVEY.md 8(c) R1/R21/R24: symmetric CSR (each
 * undirected edge stored in both directions), rows sorted by column, no
 * self-loops, no duplicate edges, unit weights (w == NULL), isolated vertices
 * removed by an order-preserving relabel when `compact` is set.
 *
 * All functions return 0 on success, negative on error (message via
 * gg_last_error()).  Handles own their arrays (host or device memory, see
 * gg_on_device) and are released with gg_free.
 */
#ifndef GRAPHGEN_H
#define GRAPHGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct gg_graph_s* gg_graph_t;

/* Zachary karate club, 34 vertices / 78 unit edges. */
int gg_karate(gg_graph_t* out);
/* Undirected edge list -> canonical CSR (drops self-loops, merges duplicates). */
int gg_from_edges(int64_t n, int64_t m, const int32_t* u, const int32_t* v, int compact,
                  gg_graph_t* out);
/* R-MAT (A,B,C,D=1-A-B-C), `ntuples` undirected tuples, vertex space 2^scale. */
int gg_rmat_host(int scale, int64_t ntuples, uint64_t seed, double a, double b, double c,
                 int compact, gg_graph_t* out);
int gg_rmat_device(int scale, int64_t ntuples, uint64_t seed, double a, double b, double c,
                   int compact, gg_graph_t* out);
/* 3-D 7-point mesh L x L x L; ids in Morton (Z) order if morton != 0, else row-major. */
int gg_mesh3d_host(int L, int morton, gg_graph_t* out);
int gg_mesh3d_device(int L, int morton, gg_graph_t* out);
/* Random geometric graph in the unit square, radius = rfac * sqrt(ln n / n);
 * ids by row-major grid cell (side >= radius), then x. */
int gg_rgg_host(int64_t n, double rfac, uint64_t seed, int compact, gg_graph_t* out);
int gg_rgg_device(int64_t n, double rfac, uint64_t seed, int compact, gg_graph_t* out);
/* LFR-style planted partition; ground truth via gg_labels. */
int gg_lfr_host(int64_t n, double gamma, int32_t kmin, int32_t kmax, double beta, int32_t smin,
                int32_t smax, double mu, uint64_t seed, gg_graph_t* out);

int64_t gg_n(gg_graph_t g);
int64_t gg_nnz(gg_graph_t g);
int gg_on_device(gg_graph_t g);
const int64_t* gg_rowptr(gg_graph_t g);
const int32_t* gg_col(gg_graph_t g);
const int32_t* gg_labels(gg_graph_t g); /* ground-truth labels (host) or NULL */
/* Copy rowptr (n+1) and col (nnz) to caller buffers (host or device). */
int gg_copy_out(gg_graph_t g, int64_t* rowptr_dst, int32_t* col_dst);
void gg_free(gg_graph_t g);
const char* gg_last_error(void);

/* ---- graph files (graph_io.cpp): a loader for real inputs next to the generators ----
 * format: 0 = by extension (.mtx Matrix Market, .csrbin binary CSR, else edge list),
 * 1 = Matrix Market coordinate, 2 = edge list "u v [w]", 3 = .csrbin.
 * one_based (edge lists): 1, 0, or -1 = 1-based iff no id is 0.  Text inputs are
 * undirected and become R1 CSR (both directions, self-loop once, rows sorted);
 * see graph_io.cpp for weights and repeated edges. */
typedef struct gg_csr_s* gg_csr_t;
int gg_load(const char* path, int format, int one_based, gg_csr_t* out);
int gg_save_csrbin(const char* path, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                   const uint32_t* w /* NULL = unit */);
int64_t gg_csr_n(gg_csr_t g);
int64_t gg_csr_nnz(gg_csr_t g);
const int64_t* gg_csr_rowptr(gg_csr_t g);
const int32_t* gg_csr_col(gg_csr_t g);
const uint32_t* gg_csr_w(gg_csr_t g); /* NULL = unit weights */
void gg_csr_free(gg_csr_t g);
const char* gg_io_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
