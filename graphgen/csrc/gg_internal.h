// gg_internal.h -- private declarations of the graph-generator module.
#ifndef GG_INTERNAL_H
#define GG_INTERNAL_H
#include <stdint.h>
#include <vector>
#include "gg_philox.h"

struct gg_graph_s {
  int64_t n, nnz;
  int device;        // 1 if rowptr/col are device pointers
  int64_t* rowptr;   // n + 1
  int32_t* col;      // nnz
  int32_t* labels;   // host, optional ground truth
};

void gg_set_error(const char* msg);
gg_graph_s* gg_alloc_host(int64_t n, int64_t nnz);
gg_graph_s* gg_build_csr_host(int64_t n, std::vector<uint64_t>& keys, int compact, const int32_t* labels_in);
void gg_device_free(gg_graph_s* g);
int gg_device_copy_out(gg_graph_s* g, int64_t* rowptr_dst, int32_t* col_dst);
int gg_copy_any(void* d0, const void* s0, size_t b0, void* d1, const void* s1, size_t b1);
void gg_rmat_thresholds(double a, double b, double c, uint32_t* tA, uint32_t* tAB, uint32_t* tABC);
int gg_mesh_bits(int L);
double gg_rgg_radius(int64_t n, double rfac);

#endif
