/* graphgen/philox.h — counter-based RNG for the SEEDED INPUT GENERATORS only.
 *
 * Philox4x32-10 (Salmon et al., "Parallel random numbers: as easy as 1, 2, 3",
 * SC'11).  This header belongs to the input-generator module: it holds none of
 * the triangle-counting method's arithmetic.  Both the CPU generator
 * (graphgen_cpu.c) and the CUDA generator (graphgen_cuda.cu) include it so that
 * the synthetic graphs they emit are bit-identical; the known-answer vectors in
 * tests/test_graphgen.py pin it.
 */
#ifndef GRAPHGEN_PHILOX_H
#define GRAPHGEN_PHILOX_H
#include <stdint.h>

#if defined(__CUDACC__)
#define GG_HD __host__ __device__ __forceinline__
#else
#define GG_HD static inline
#endif

#define GG_PHILOX_M0 0xD2511F53u
#define GG_PHILOX_M1 0xCD9E8D57u
#define GG_PHILOX_W0 0x9E3779B9u
#define GG_PHILOX_W1 0xBB67AE85u

typedef struct { uint32_t v[4]; } gg_u32x4;

GG_HD gg_u32x4 gg_philox4x32_10(gg_u32x4 c, uint32_t k0, uint32_t k1) {
  for (int r = 0; r < 10; ++r) {
    if (r) { k0 += GG_PHILOX_W0; k1 += GG_PHILOX_W1; }
    uint64_t p0 = (uint64_t)GG_PHILOX_M0 * c.v[0];
    uint64_t p1 = (uint64_t)GG_PHILOX_M1 * c.v[2];
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    gg_u32x4 o;
    o.v[0] = hi1 ^ c.v[1] ^ k0;
    o.v[1] = lo1;
    o.v[2] = hi0 ^ c.v[3] ^ k1;
    o.v[3] = lo0;
    c = o;
  }
  return c;
}

/* Draw j (j = 0,1,2,...) of sample e: Philox(key = seed, ctr = (e_lo, e_hi, j/4, tag))[j%4]. */
GG_HD uint32_t gg_draw(uint64_t seed, uint64_t e, uint32_t j, uint32_t tag) {
  gg_u32x4 c;
  c.v[0] = (uint32_t)e; c.v[1] = (uint32_t)(e >> 32); c.v[2] = j >> 2; c.v[3] = tag;
  gg_u32x4 r = gg_philox4x32_10(c, (uint32_t)seed, (uint32_t)(seed >> 32));
  return r.v[j & 3];
}

/* R-MAT / Kronecker sample e (Graph500 quadrant recursion, no per-level noise).
 * Quadrant per level from one u32 draw against integer thresholds
 * ta = floor(a*2^32), tab = floor((a+b)*2^32), tabc = floor((a+b+c)*2^32). */
GG_HD void gg_rmat_sample(uint64_t seed, uint64_t e, uint32_t scale, uint32_t ta, uint32_t tab,
                          uint32_t tabc, uint32_t *u_out, uint32_t *v_out) {
  uint32_t u = 0, v = 0;
  for (uint32_t l = 0; l < scale; ++l) {
    uint32_t r = gg_draw(seed, e, l, 0x524D4154u /* "RMAT" */);
    uint32_t bu = r >= tab;                       /* quadrants c, d */
    uint32_t bv = (r >= ta && r < tab) || r >= tabc; /* quadrants b, d */
    u = (u << 1) | bu;
    v = (v << 1) | bv;
  }
  *u_out = u; *v_out = v;
}

/* Bijective label scramble on [0, 2^scale): two rounds of odd-multiply-add and
 * xor-shift, all mod 2^scale.  Graph500 permutes labels too; without it id order
 * correlates with degree. */
GG_HD uint32_t gg_scramble(uint32_t x, uint32_t scale, uint64_t seed) {
  if (scale == 0) return 0;
  uint64_t mask = (scale >= 64) ? ~0ull : ((1ull << scale) - 1);
  uint64_t y = x;
  uint32_t sh = (scale + 1) / 2;
  uint64_t k1 = (seed * 0x9E3779B97F4A7C15ull) | 1ull;
  uint64_t k2 = seed ^ 0xD1B54A32D192ED03ull;
  y = (y * 0xBF58476D1CE4E5B9ull + k2) & mask;
  y ^= y >> sh;
  y = (y * k1 + (k2 >> 17)) & mask;
  y ^= y >> sh;
  return (uint32_t)y;
}

/* Erdos-Renyi G(n, M) sample e: u, v = floor(r * n / 2^32) (64-bit multiply-shift). */
GG_HD void gg_er_sample(uint64_t seed, uint64_t e, uint32_t n, uint32_t *u_out, uint32_t *v_out) {
  gg_u32x4 c;
  c.v[0] = (uint32_t)e; c.v[1] = (uint32_t)(e >> 32); c.v[2] = 0; c.v[3] = 0x45524452u; /* "ERDR" */
  gg_u32x4 r = gg_philox4x32_10(c, (uint32_t)seed, (uint32_t)(seed >> 32));
  *u_out = (uint32_t)(((uint64_t)r.v[0] * n) >> 32);
  *v_out = (uint32_t)(((uint64_t)r.v[1] * n) >> 32);
}

#endif
