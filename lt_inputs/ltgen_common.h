/* ltgen_common.h — the tuple recipe shared by the CPU and GPU builds of the input generator.
 * Input generation only: nothing here is part of the random-walk method (see ltgen.h). */
#ifndef LTGEN_COMMON_H
#define LTGEN_COMMON_H
#include <stdint.h>

#if defined(__CUDACC__)
#define LTGEN_HD __host__ __device__ __forceinline__
#else
#define LTGEN_HD static inline
#endif

/* splitmix64 finalizer (Steele, Lea, Flood 2014). */
LTGEN_HD uint64_t ltgen_mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

#define LTGEN_GOLDEN 0x9E3779B97F4A7C15ULL

/* Graph500 initiator as u32 thresholds: a=0.57, a+b=0.76, a+b+c=0.95 (x 2^32, floored). */
#define LTGEN_TA   2448131358u
#define LTGEN_TAB  3264175144u
#define LTGEN_TABC 4080218931u

LTGEN_HD uint64_t ltgen_key(uint64_t seed) { return ltgen_mix64(seed ^ 0x5851F42D4C957F2DULL); }

/* Seeded Feistel bijection on [0, 2^scale) (cycle-walking when scale is odd). */
LTGEN_HD uint32_t ltgen_feistel_once(uint32_t x, uint32_t half, uint64_t pkey) {
  uint32_t mask = (half >= 32) ? 0xFFFFFFFFu : ((1u << half) - 1u);
  uint32_t L = x >> half, R = x & mask;
  for (uint32_t r = 0; r < 4; ++r) {
    uint32_t F = (uint32_t)(ltgen_mix64(pkey + LTGEN_GOLDEN * (uint64_t)(r + 1) + ((uint64_t)R << 8)) & mask);
    uint32_t nL = R, nR = L ^ F;
    L = nL; R = nR;
  }
  return (L << half) | R;
}

LTGEN_HD uint32_t ltgen_permute(uint32_t x, uint32_t scale, uint64_t seed) {
  uint32_t bits = scale + (scale & 1u);
  uint32_t half = bits / 2u;
  uint64_t pkey = ltgen_mix64(seed ^ 0xD1B54A32D192ED03ULL);
  uint64_t lim = 1ULL << scale;
  do { x = ltgen_feistel_once(x, half, pkey); } while ((uint64_t)x >= lim);
  return x;
}

/* R-MAT tuple e: level L in [0, scale) decides bit (scale-1-L) of u and v. */
LTGEN_HD void ltgen_tuple_impl(uint32_t scale, uint64_t key, uint64_t seed, int permute,
                               uint64_t e, uint32_t* uo, uint32_t* vo) {
  uint32_t u = 0, v = 0;
  uint64_t word = 0;
  for (uint32_t L = 0; L < scale; ++L) {
    uint32_t r;
    if ((L & 1u) == 0) {
      word = ltgen_mix64(key + LTGEN_GOLDEN * (32ULL * e + (uint64_t)(L >> 1)));
      r = (uint32_t)(word >> 32);
    } else {
      r = (uint32_t)word;
    }
    uint32_t bu, bv;
    if (r < LTGEN_TA) { bu = 0; bv = 0; }
    else if (r < LTGEN_TAB) { bu = 0; bv = 1; }
    else if (r < LTGEN_TABC) { bu = 1; bv = 0; }
    else { bu = 1; bv = 1; }
    u = (u << 1) | bu;
    v = (v << 1) | bv;
  }
  if (permute) { u = ltgen_permute(u, scale, seed); v = ltgen_permute(v, scale, seed); }
  *uo = u; *vo = v;
}

#endif
