/* gg_philox.h -- counter-based Philox4x32-10 shared by the host and device
 * graph generators (input module only; holds none of the Louvain method's
 * arithmetic).  Salmon et al., "Parallel random numbers: as easy as 1, 2, 3"
 * (SC'11): 10 rounds, multipliers 0xD2511F53 / 0xCD9E8D57, Weyl key bumps
 * 0x9E3779B9 / 0xBB67AE85.  Being a pure function of (key, counter) it gives
 * bit-identical streams on the CPU and on the GPU, which is what lets the
 * oracle and the CUDA path see the same synthetic graph.
 */
#ifndef GG_PHILOX_H
#define GG_PHILOX_H
#include <stdint.h>

#if defined(__CUDACC__)
#define GG_HD __host__ __device__ __forceinline__
#else
#define GG_HD static inline
#endif

typedef struct { uint32_t v[4]; } gg_u32x4;

GG_HD uint32_t gg_mulhi32(uint32_t a, uint32_t b) {
  return (uint32_t)(((uint64_t)a * (uint64_t)b) >> 32);
}

GG_HD gg_u32x4 gg_philox4x32_10(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                uint32_t k0, uint32_t k1) {
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0 = gg_mulhi32(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    uint32_t hi1 = gg_mulhi32(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    uint32_t n0 = hi1 ^ c1 ^ k0, n1 = lo1, n2 = hi0 ^ c3 ^ k1, n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    k0 += 0x9E3779B9u; k1 += 0xBB67AE85u;
  }
  gg_u32x4 out;
  out.v[0] = c0; out.v[1] = c1; out.v[2] = c2; out.v[3] = c3;
  return out;
}

/* Word `idx` of the stream (seed, stream, item): word idx lives in call idx/4. */
GG_HD uint32_t gg_rand_u32(uint64_t seed, uint32_t stream, uint64_t item, uint32_t idx) {
  gg_u32x4 r = gg_philox4x32_10((uint32_t)item, (uint32_t)(item >> 32), idx >> 2, stream,
                                (uint32_t)seed, (uint32_t)(seed >> 32));
  return r.v[idx & 3u];
}

/* R-MAT quadrant walk for one undirected tuple (Chakrabarti, Zhan, Faloutsos,
 * SDM'04).  Level l (0 = most significant bit) draws one 32-bit word and
 * compares it with the cumulative integer thresholds t[0] < t[1] < t[2]
 * (floor(c * 2^32) of A, A+B, A+B+C).  No id scrambling: hubs keep low ids
 * (SURVEY R24). */
GG_HD void gg_rmat_tuple(uint64_t seed, uint64_t t, int scale, uint32_t tA, uint32_t tAB,
                         uint32_t tABC, uint32_t* u, uint32_t* v) {
  uint32_t uu = 0, vv = 0;
  for (int c = 0; c * 4 < scale; ++c) {
    gg_u32x4 r = gg_philox4x32_10((uint32_t)t, (uint32_t)(t >> 32), (uint32_t)c, 0x524D4154u /* "RMAT" */,
                                  (uint32_t)seed, (uint32_t)(seed >> 32));
    for (int q = 0; q < 4; ++q) {
      int l = c * 4 + q;
      if (l >= scale) break;
      uint32_t x = r.v[q];
      uint32_t bu = (x >= tAB) ? 1u : 0u;                 /* quadrants C, D: row bit set */
      uint32_t bv = (x >= tA && x < tAB) || (x >= tABC);   /* quadrants B, D: col bit set */
      uu = (uu << 1) | bu;
      vv = (vv << 1) | bv;
    }
  }
  *u = uu; *v = vv;
}

/* Morton (Z-order) code of (x, y, z): bit b of x -> 3b, of y -> 3b+1, of z -> 3b+2. */
GG_HD uint64_t gg_morton3(uint32_t x, uint32_t y, uint32_t z, int bits) {
  uint64_t code = 0;
  for (int b = 0; b < bits; ++b) {
    code |= (uint64_t)((x >> b) & 1u) << (3 * b);
    code |= (uint64_t)((y >> b) & 1u) << (3 * b + 1);
    code |= (uint64_t)((z >> b) & 1u) << (3 * b + 2);
  }
  return code;
}

GG_HD void gg_morton3_decode(uint64_t code, int bits, uint32_t* x, uint32_t* y, uint32_t* z) {
  uint32_t xx = 0, yy = 0, zz = 0;
  for (int b = 0; b < bits; ++b) {
    xx |= (uint32_t)((code >> (3 * b)) & 1u) << b;
    yy |= (uint32_t)((code >> (3 * b + 1)) & 1u) << b;
    zz |= (uint32_t)((code >> (3 * b + 2)) & 1u) << b;
  }
  *x = xx; *y = yy; *z = zz;
}

/* uniform double in [0,1) from 53 random bits of two words */
GG_HD double gg_u01(uint32_t hi, uint32_t lo) {
  uint64_t m = (((uint64_t)hi << 32) | lo) >> 11;
  return (double)m * (1.0 / 9007199254740992.0);
}

#endif
