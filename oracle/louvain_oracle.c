/* louvain_oracle.c -- TEST INFRASTRUCTURE ONLY (see louvain_oracle.h).
 *
 * A plain, slow, obviously-correct single-threaded C transcription of the
 * method of Naim, Manne, Halappanavar, Tumeo, "Community Detection on the
 * GPU" (IPDPS'17).  Citations P:<line> refer to /root/reference/PAPER.md;
 * R<k> refers to the readings of SURVEY.md 8(c) (listed in DESIGN.md).
 * No blocking, fusion or reordering beyond what the paper's Algorithms 1-3
 * state.  Shares no code with the CUDA path.
 *
 * Pins (tests/test_oracle_*.py): closed-form modularity (singletons, one
 * community, disjoint cliques, ring of cliques), networkx modularity on random
 * partitions, exact-rational Eq. (2) gains vs re-evaluated Eq. (1), brute force
 * over all partitions (n <= 9), contraction == P^T A P (scipy) with W and Q
 * preserved, karate values, singleton-rule micro cases, hand-computed worked
 * cases of RELAXED (star K_{1,5}: one snapshot vs bucket commits) and of the
 * (adaptive) sequential variant (path P_4 with the theta_bin schedule).  The
 * bucket/commit rules R10-R12 are "parity unpinned" by the paper (no worked
 * example); DESIGN.md records that.
 */
#include "louvain_oracle.h"

#include <stdlib.h>
#include <string.h>

#define ORC_W_GUARD 3037000499ULL /* W^2 < 2^63 (R4) */

typedef __int128 i128;

static uint64_t wt(const uint32_t* w, int64_t e) { return w ? (uint64_t)w[e] : 1u; }

void orc_params_default(orc_params* p) {
  p->mode = ORC_BIN_SYNC;
  p->singleton_rule = 1;
  p->revert_on_decrease = 1;
  p->th_bin_exp = 2;   /* t_bin = 10^-2   (P:334 garbled "102", "(10-2,10-6)") */
  p->th_final_exp = 6; /* t_final = 10^-6 */
  p->size_limit = 100000;
  p->deg_bounds[0] = 4; p->deg_bounds[1] = 8; p->deg_bounds[2] = 16;
  p->deg_bounds[3] = 32; p->deg_bounds[4] = 84; p->deg_bounds[5] = 319;
  p->max_sweeps = 0;
  p->max_levels = 0;
}

/* k_i = sum_{j in N[i]} w(i,j) including self-loops; W = sum_i k_i = 2m (R1). */
static uint64_t degrees(int64_t n, const int64_t* rowptr, const uint32_t* w, uint64_t* k) {
  uint64_t W = 0;
  for (int64_t i = 0; i < n; ++i) {
    uint64_t s = 0;
    for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e) s += wt(w, e);
    if (k) k[i] = s;
    W += s;
  }
  return W;
}

void orc_totals(int64_t n, const int64_t* rowptr, const uint32_t* w, const int32_t* C,
                uint64_t* a, int64_t* size) {
  for (int64_t c = 0; c < n; ++c) { a[c] = 0; size[c] = 0; }
  for (int64_t i = 0; i < n; ++i) {
    uint64_t ki = 0;
    for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e) ki += wt(w, e);
    a[C[i]] += ki;   /* a_c = sum_{i in c} k_i */
    size[C[i]] += 1;
  }
}

int orc_modularity(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                   const int32_t* C, uint64_t* Lout, uint64_t* Sout, uint64_t* Wout) {
  uint64_t W = degrees(n, rowptr, w, NULL);
  if (W > ORC_W_GUARD) return -3;
  /* L = sum_i e_{i->C(i)}, counting every stored entry (i,j) with C(j) = C(i),
   * self-loops included (R2). */
  uint64_t L = 0;
  for (int64_t i = 0; i < n; ++i)
    for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e)
      if (C[col[e]] == C[i]) L += wt(w, e);
  uint64_t* a = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(n > 0 ? n : 1));
  int64_t* size = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  orc_totals(n, rowptr, w, C, a, size);
  uint64_t S = 0;
  for (int64_t c = 0; c < n; ++c) S += a[c] * a[c]; /* sum_c a_c^2 */
  free(a);
  free(size);
  *Lout = L;
  *Sout = S;
  *Wout = W;
  return 0;
}

/* Q numerator: Q = (1/2m) L - S/(4m^2) = (L*W - S) / W^2 with W = 2m (Eq. 1). */
static int64_t qnum(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                    const int32_t* C) {
  uint64_t L, S, W;
  orc_modularity(n, rowptr, col, w, C, &L, &S, &W);
  return (int64_t)(L * W) - (int64_t)S;
}

/* ---------------------------------------------------------------- decide */
typedef struct {
  uint64_t* acc;     /* e_{i->c}, indexed by community label (dense; plain) */
  int32_t* touched;  /* labels with acc > 0 */
} orc_ws;

static void ws_init(orc_ws* ws, int64_t n) {
  ws->acc = (uint64_t*)calloc((size_t)(n > 0 ? n : 1), sizeof(uint64_t));
  ws->touched = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
}
static void ws_free(orc_ws* ws) { free(ws->acc); free(ws->touched); }

/* Alg. 2.  The hash table of the paper is only a way
 * to obtain e_{i->c} for every neighbouring community c; any exact per-label
 * accumulation is equivalent (R25).  Gains per Eq. (2) in the
 * integer form s_c = W*e_c - k_i*a_c, so that
 *   dQ_{i->D} = 2 (s_D - s_stay) / W^2,  s_stay = W*e_own - k_i*(a_own - k_i)
 * (R3: the self-loop is excluded from e; R5: candidates are the labels of
 * N(i)\{i} other than C(i)).  Ties -> lowest label (R7); move only on a
 * strictly positive gain (R6); singleton rule of P:148-152/P:172 (R8, R9). */
static int32_t decide_ws(orc_ws* ws, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                         const int32_t* C, const uint64_t* a, const int64_t* size, uint64_t W,
                         int64_t i, int32_t rule, int64_t* dcount) {
  int32_t own = C[i];
  uint64_t ki = 0;
  int64_t nt = 0;
  for (int64_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
    uint64_t we = wt(w, e);
    ki += we;
    int32_t j = col[e];
    if (j == i) continue; /* R3 */
    int32_t c = C[j];
    if (ws->acc[c] == 0) ws->touched[nt++] = c;
    ws->acc[c] += we;
  }
  int64_t s_stay = (int64_t)W * (int64_t)ws->acc[own] - (int64_t)ki * ((int64_t)a[own] - (int64_t)ki);
  int32_t best = -1;
  int64_t s_best = 0;
  for (int64_t t = 0; t < nt; ++t) {
    int32_t c = ws->touched[t];
    if (c == own) continue;
    if (dcount) ++*dcount; /* measurement only: distinct candidate labels */
    if (rule == 2 && size[own] == 1 && size[c] == 1 && c > own) continue; /* R8 filter */
    int64_t s = (int64_t)W * (int64_t)ws->acc[c] - (int64_t)ki * (int64_t)a[c];
    if (best < 0 || s > s_best || (s == s_best && c < best)) { best = c; s_best = s; }
  }
  for (int64_t t = 0; t < nt; ++t) ws->acc[ws->touched[t]] = 0;
  if (best < 0 || s_best <= s_stay) return own;                                   /* R6 */
  if (rule == 1 && size[own] == 1 && size[best] == 1 && best > own) return own;  /* R8 veto */
  return best;
}

int32_t orc_decide(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                   const int32_t* C, const uint64_t* a, const int64_t* size, uint64_t W,
                   int64_t i, int32_t singleton_rule) {
  orc_ws ws;
  ws_init(&ws, n);
  int32_t r = decide_ws(&ws, rowptr, col, w, C, a, size, W, i, singleton_rule, NULL);
  ws_free(&ws);
  return r;
}

void orc_decide_batch(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                      const int32_t* C, const uint64_t* a, const int64_t* size, uint64_t W,
                      int32_t singleton_rule, int64_t nv, const int64_t* verts, int32_t* out) {
  orc_ws ws;
  ws_init(&ws, n);
  for (int64_t t = 0; t < nv; ++t)
    out[t] = decide_ws(&ws, rowptr, col, w, C, a, size, W, verts[t], singleton_rule, NULL);
  ws_free(&ws);
}

/* ---------------------------------------------------------------- sweep */
/* Bucket of vertex i: smallest b with deg(i) <= bucDSize[b] (R11);
 * deg = stored row length (self-loop entry included); deg 0 -> no bucket (-1). */
static int bucket_of(const orc_params* p, int64_t deg) {
  if (deg == 0) return -1;
  for (int b = 0; b < 6; ++b)
    if (deg <= p->deg_bounds[b]) return b;
  return 6;
}

static void move_vertex(int32_t* C, uint64_t* a, int64_t* size, int64_t i, int32_t t, uint64_t ki) {
  a[C[i]] -= ki;
  size[C[i]] -= 1;
  a[t] += ki;
  size[t] += 1;
  C[i] = t;
}

int64_t orc_sweep(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                  const orc_params* p, int32_t* C, uint64_t* a, int64_t* size, uint64_t W) {
  return orc_sweep_counted(n, rowptr, col, w, p, C, a, size, W, NULL);
}

int64_t orc_sweep_counted(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                          const orc_params* p, int32_t* C, uint64_t* a, int64_t* size, uint64_t W,
                          int64_t* D_out) {
  if (D_out) *D_out = 0;
  orc_ws ws;
  ws_init(&ws, n);
  uint64_t* k = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(n > 0 ? n : 1));
  degrees(n, rowptr, w, k);
  int64_t moved = 0;
  if (p->mode == ORC_SEQ || p->mode == ORC_SEQ_ADAPTIVE) {
    /* Sequential Louvain: each vertex in turn, ascending id, immediate
     * update, no singleton rule (R23). */
    for (int64_t i = 0; i < n; ++i) {
      int32_t t = decide_ws(&ws, rowptr, col, w, C, a, size, W, i, 0, D_out);
      if (t != C[i]) { move_vertex(C, a, size, i, t, k[i]); ++moved; }
    }
  } else {
    /* Alg. 1 lines 4-11: for each bucket, computeMove on all of its
     * vertices against the same state, then C[i] = newComm[i], then a_c. */
    int nbuckets = (p->mode == ORC_RELAXED) ? 1 : 7;
    int64_t* vset = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int32_t* newComm = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    for (int b = 0; b < nbuckets; ++b) {
      int64_t nv = 0;
      for (int64_t i = 0; i < n; ++i) {
        int bi = bucket_of(p, rowptr[i + 1] - rowptr[i]);
        if (bi < 0) continue;
        if (p->mode == ORC_RELAXED || bi == b) vset[nv++] = i;
      }
      for (int64_t t = 0; t < nv; ++t)
        newComm[t] = decide_ws(&ws, rowptr, col, w, C, a, size, W, vset[t], p->singleton_rule, D_out);
      for (int64_t t = 0; t < nv; ++t) {
        int64_t i = vset[t];
        if (newComm[t] != C[i]) { move_vertex(C, a, size, i, newComm[t], k[i]); ++moved; }
      }
    }
    free(vset);
    free(newComm);
  }
  free(k);
  ws_free(&ws);
  return moved;
}

/* ---------------------------------------------------------------- contract */
static int cmp_i32(const void* x, const void* y) {
  int32_t a = *(const int32_t*)x, b = *(const int32_t*)y;
  return (a > b) - (a < b);
}

int64_t orc_contract(int64_t n, const int64_t* rowptr, const int32_t* col, const uint32_t* w,
                     const int32_t* C, int64_t* rowptr_out, int32_t* col_out, uint32_t* w_out,
                     int64_t* nnz_out, int32_t* map_out) {
  size_t nz = (size_t)(n > 0 ? n : 1);
  /* Alg. 3 lines 2-12: comSize, newID = prefix sum of [comSize > 0]
   * (consecutive numbering from zero in label order, R17). */
  int64_t* comSize = (int64_t*)calloc(nz, sizeof(int64_t));
  int32_t* newID = (int32_t*)malloc(sizeof(int32_t) * nz);
  for (int64_t i = 0; i < n; ++i) comSize[C[i]] += 1;
  int64_t np = 0;
  for (int64_t c = 0; c < n; ++c) newID[c] = comSize[c] > 0 ? (int32_t)np++ : -1;
  for (int64_t i = 0; i < n; ++i) map_out[i] = newID[C[i]];
  /* Alg. 3 lines 15-19: vertices grouped by community (com[] via vertexStart). */
  int64_t* vstart = (int64_t*)calloc((size_t)np + 1, sizeof(int64_t));
  for (int64_t i = 0; i < n; ++i) vstart[map_out[i] + 1] += 1;
  for (int64_t r = 0; r < np; ++r) vstart[r + 1] += vstart[r];
  int64_t* cursor = (int64_t*)malloc(sizeof(int64_t) * ((size_t)np + 1));
  for (int64_t r = 0; r <= np; ++r) cursor[r] = vstart[r];
  int64_t* com = (int64_t*)malloc(sizeof(int64_t) * nz);
  for (int64_t i = 0; i < n; ++i) com[cursor[map_out[i]]++] = i;
  /* mergeCommunity: all neighbours of all members of c accumulated in
   * one table keyed by the neighbour's new id; weights summed (P:118-122,
   * R18: intra-community entries become the self-loop). */
  uint64_t* acc = (uint64_t*)calloc((size_t)(np > 0 ? np : 1), sizeof(uint64_t));
  int32_t* touched = (int32_t*)malloc(sizeof(int32_t) * (size_t)(np > 0 ? np : 1));
  int64_t e_out = 0;
  rowptr_out[0] = 0;
  for (int64_t r = 0; r < np; ++r) {
    int64_t nt = 0;
    for (int64_t m = vstart[r]; m < vstart[r + 1]; ++m) {
      int64_t u = com[m];
      for (int64_t e = rowptr[u]; e < rowptr[u + 1]; ++e) {
        int32_t d = map_out[col[e]];
        if (acc[d] == 0) touched[nt++] = d;
        acc[d] += wt(w, e);
      }
    }
    qsort(touched, (size_t)nt, sizeof(int32_t), cmp_i32); /* rows sorted by column */
    for (int64_t t = 0; t < nt; ++t) {
      col_out[e_out] = touched[t];
      w_out[e_out] = (uint32_t)acc[touched[t]];
      acc[touched[t]] = 0;
      ++e_out;
    }
    rowptr_out[r + 1] = e_out;
  }
  *nnz_out = e_out;
  free(comSize); free(newID); free(vstart); free(cursor); free(com); free(acc); free(touched);
  return np;
}

/* ---------------------------------------------------------------- driver */
static i128 pow10_i128(int p) {
  i128 r = 1;
  for (int t = 0; t < p; ++t) r *= 10;
  return r;
}

/* gain test "(num_new - num_old) / W^2 < 10^-p" in exact integers (R13) */
static int below_threshold(int64_t num_new, int64_t num_old, uint64_t W, int p) {
  i128 d = (i128)num_new - (i128)num_old;
  return d * pow10_i128(p) < (i128)W * (i128)W;
}

int orc_louvain(int64_t n0, const int64_t* rowptr0, const int32_t* col0, const uint32_t* w0,
                const orc_params* p, int32_t* labels_out, orc_stats* st) {
  memset(st, 0, sizeof *st);
  uint64_t W = degrees(n0, rowptr0, w0, NULL);
  if (W > ORC_W_GUARD) return -3;
  for (int64_t v = 0; v < n0; ++v) labels_out[v] = (int32_t)v;
  st->W = W;
  if (W == 0) return 0;

  int64_t n = n0;
  const int64_t* rowptr = rowptr0;
  const int32_t* col = col0;
  const uint32_t* w = w0;
  int64_t *own_rowptr = NULL;
  int32_t *own_col = NULL;
  uint32_t *own_w = NULL;
  int seq = (p->mode == ORC_SEQ || p->mode == ORC_SEQ_ADAPTIVE);

  for (int level = 0;; ++level) {
    if ((p->max_levels > 0 && level >= p->max_levels) || level >= ORC_MAX_LEVELS) break;
    size_t nz = (size_t)(n > 0 ? n : 1);
    /* threshold schedule (R14); sequential (a) uses t_final throughout
     * unless adaptive */
    int pexp = (n > p->size_limit) ? p->th_bin_exp : p->th_final_exp;
    if (p->mode == ORC_SEQ) pexp = p->th_final_exp;
    int32_t* C = (int32_t*)malloc(sizeof(int32_t) * nz);
    int32_t* saved = (int32_t*)malloc(sizeof(int32_t) * nz);
    uint64_t* a = (uint64_t*)malloc(sizeof(uint64_t) * nz);
    int64_t* size = (int64_t*)malloc(sizeof(int64_t) * nz);
    for (int64_t i = 0; i < n; ++i) C[i] = (int32_t)i; /* C[i] = i at phase start */
    orc_totals(n, rowptr, w, C, a, size);
    int64_t num_start = qnum(n, rowptr, col, w, C);
    int64_t num_prev = num_start;
    int64_t moved_level = 0;
    int32_t sweeps = 0;
    for (;;) {
      if (p->max_sweeps > 0 && sweeps >= p->max_sweeps) break;
      memcpy(saved, C, sizeof(int32_t) * (size_t)n);
      int64_t moved = orc_sweep(n, rowptr, col, w, p, C, a, size, W);
      ++sweeps;
      int64_t num = qnum(n, rowptr, col, w, C);
      if (p->revert_on_decrease && num < num_prev) { /* R15 */
        memcpy(C, saved, sizeof(int32_t) * (size_t)n);
        orc_totals(n, rowptr, w, C, a, size);
        break;
      }
      moved_level += moved;
      if (moved == 0 || below_threshold(num, num_prev, W, pexp)) break; /* Alg. 1 l.12, R13 */
      num_prev = num;
    }
    int64_t num_end = qnum(n, rowptr, col, w, C);
    st->n[level] = n;
    st->nnz[level] = rowptr[n];
    st->sweeps_per_level[level] = sweeps;
    st->moved_per_level[level] = moved_level;
    st->num_start[level] = num_start;
    st->num_end[level] = num_end;
    st->levels = level + 1;
    st->sweeps += sweeps;
    (void)seq;
    /* outer termination (R16 uses t_final) */
    if (moved_level == 0 || below_threshold(num_end, num_start, W, p->th_final_exp)) {
      for (int64_t v = 0; v < n0; ++v) labels_out[v] = C[labels_out[v]];
      free(C); free(saved); free(a); free(size);
      break;
    }
    /* aggregation phase (Alg. 3) */
    int64_t nnz = rowptr[n];
    int64_t* nrow = (int64_t*)malloc(sizeof(int64_t) * (nz + 1));
    int32_t* ncol = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
    uint32_t* nw = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz > 0 ? nnz : 1));
    int32_t* map = (int32_t*)malloc(sizeof(int32_t) * nz);
    int64_t nnz2 = 0;
    int64_t n2 = orc_contract(n, rowptr, col, w, C, nrow, ncol, nw, &nnz2, map);
    for (int64_t v = 0; v < n0; ++v) labels_out[v] = map[labels_out[v]];
    free(map); free(C); free(saved); free(a); free(size);
    free(own_rowptr); free(own_col); free(own_w);
    own_rowptr = nrow; own_col = ncol; own_w = nw;
    n = n2; rowptr = nrow; col = ncol; w = nw;
  }
  /* final Q from the exact parts, evaluated on the input graph */
  uint64_t L, S, Wc;
  orc_modularity(n0, rowptr0, col0, w0, labels_out, &L, &S, &Wc);
  st->L = L;
  st->S = S;
  st->W = Wc;
  st->q = (double)((int64_t)(L * Wc) - (int64_t)S) / ((double)Wc * (double)Wc);
  free(own_rowptr); free(own_col); free(own_w);
  return 0;
}
