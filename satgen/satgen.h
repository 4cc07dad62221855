/* satgen.h -- seeded, counter-based synthetic input generator.
 *
 * This module is shared by the CUDA path's tests/bench (device fill kernel in
 * satgen.cu) and by the CPU oracle harness (host fill / row provider).  It
 * holds NONE of the summed-area-table arithmetic: it only maps a pixel
 * coordinate (seed, image, y, x) to an input value, so that both sides can
 * regenerate identical inputs without copying them.
 *
 * Generator: splitmix64 finaliser applied to an FNV-style fold of the
 * coordinate.  Value mappings:
 *   8u   uniform  : top 8 bits                       -> [0, 255]
 *   32f  uniform  : top 24 bits * 2^-24              -> [0, 1), 24-bit granular
 *   64f  uniform  : top 53 bits * 2^-53              -> [0, 1), full mantissa
 *   64f  dyadic24 : top 24 bits * 2^-24 (as double)  -> sums exact while H*W <= 2^29
 *   any  const    : the constant `value` (all-ones, all-255, ...)
 */
#ifndef SATGEN_H
#define SATGEN_H

#include <stdint.h>

#if defined(__CUDACC__)
#define SATGEN_HD __host__ __device__ __forceinline__
#else
#define SATGEN_HD static inline
#endif

enum satgen_kind { SATGEN_U8 = 0, SATGEN_F32 = 1, SATGEN_F64 = 2 };
enum satgen_mode { SATGEN_UNIFORM = 0, SATGEN_DYADIC24 = 1, SATGEN_CONST = 2 };

SATGEN_HD uint64_t satgen_mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

SATGEN_HD uint64_t satgen_bits(uint64_t seed, uint64_t img, uint64_t y, uint64_t x) {
  const uint64_t P = 0x100000001B3ULL; /* FNV-1a 64-bit prime */
  uint64_t k = 0xCBF29CE484222325ULL ^ seed;
  k = (k * P) ^ img;
  k = (k * P) ^ y;
  k = (k * P) ^ x;
  return satgen_mix64(k);
}

SATGEN_HD uint8_t satgen_u8(uint64_t seed, uint64_t img, uint64_t y, uint64_t x, int mode,
                            double value) {
  if (mode == SATGEN_CONST) return (uint8_t)value;
  return (uint8_t)(satgen_bits(seed, img, y, x) >> 56);
}

SATGEN_HD float satgen_f32(uint64_t seed, uint64_t img, uint64_t y, uint64_t x, int mode,
                           double value) {
  if (mode == SATGEN_CONST) return (float)value;
  return (float)(satgen_bits(seed, img, y, x) >> 40) * (1.0f / 16777216.0f);
}

SATGEN_HD double satgen_f64(uint64_t seed, uint64_t img, uint64_t y, uint64_t x, int mode,
                            double value) {
  if (mode == SATGEN_CONST) return value;
  uint64_t b = satgen_bits(seed, img, y, x);
  if (mode == SATGEN_DYADIC24) return (double)(b >> 40) * (1.0 / 16777216.0);
  return (double)(b >> 11) * (1.0 / 9007199254740992.0);
}

#endif /* SATGEN_H */
