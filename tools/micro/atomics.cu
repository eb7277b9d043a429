// Micro-benchmark: random 64-bit CAS / 32-bit RED / 8-byte gathers vs table size on one GPU.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t hsh(uint64_t x) { x ^= x >> 33; x *= 0xff51afd7ed558ccdULL; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ULL; x ^= x >> 33; return (uint32_t)x; }
__global__ void k_cas(unsigned long long* T, uint64_t mask, int64_t n, int ilp) {
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 4; i < n; i += (int64_t)gridDim.x * blockDim.x * 4) {
    unsigned long long o[4];
    #pragma unroll
    for (int q = 0; q < 4; ++q) o[q] = atomicCAS(&T[hsh(i + q) & mask], ~0ull, (unsigned long long)(i + q));
    if ((o[0] & o[1] & o[2] & o[3]) == 12345) T[0] = 1;
  }
}
__global__ void k_cas1(unsigned long long* T, uint64_t mask, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    unsigned long long o = atomicCAS(&T[hsh(i) & mask], ~0ull, (unsigned long long)i);
    if (o == 12345) T[0] = 1;
  }
}
__global__ void k_red(unsigned int* T, uint64_t mask, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&T[hsh(i) & mask], 1u);
}
__global__ void k_gather(const uint2* T, uint64_t mask, int64_t n, unsigned* out) {
  unsigned acc = 0;
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 4; i < n; i += (int64_t)gridDim.x * blockDim.x * 4) {
    uint2 v[4];
    #pragma unroll
    for (int q = 0; q < 4; ++q) v[q] = __ldg(&T[hsh(i + q) & mask]);
    #pragma unroll
    for (int q = 0; q < 4; ++q) acc += v[q].x;
  }
  if (acc == 7) out[0] = acc;
}
int main() {
  const int64_t n = 1ll << 28;  // ops
  unsigned long long* T; cudaMalloc(&T, 8ull << 30);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int lg : {19, 22, 23, 24, 26, 28, 30}) {  // slots (8 B each): 4 MB .. 8 GB
    uint64_t mask = (1ull << lg) - 1;
    float ms;
    cudaMemset(T, 0xFF, 8ull << lg);
    cudaEventRecord(a); k_cas<<<148 * 16, 256>>>(T, mask, n, 4); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b); double cas4 = n / (ms * 1e6);
    cudaMemset(T, 0xFF, 8ull << lg);
    cudaEventRecord(a); k_cas1<<<148 * 16, 256>>>(T, mask, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b); double cas1 = n / (ms * 1e6);
    cudaEventRecord(a); k_red<<<148 * 16, 256>>>((unsigned*)T, (mask << 1) | 1, n); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b); double red = n / (ms * 1e6);
    cudaEventRecord(a); k_gather<<<148 * 16, 256>>>((const uint2*)T, mask, n, (unsigned*)T); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b); double gat = n / (ms * 1e6);
    printf("table %8.1f MB: CAS64 ilp4 %6.1f G/s  CAS64 ilp1 %6.1f G/s  RED32 %6.1f G/s  gather8B ilp4 %6.1f G/s\n",
           (8.0 * (1ull << lg)) / 1e6, cas4, cas1, red, gat);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
