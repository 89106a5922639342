/*
 * gen.c — seeded synthetic inputs shared by the tests, the oracle checks and bench.py.
 *
 * This module holds NONE of the top-K method's arithmetic: it only produces key
 * arrays. Both the CUDA path and the CPU oracle consume its output (the keys are
 * generated on the host and copied to the device), so every comparison is made on
 * bit-identical inputs.
 *
 * Distributions follow the paper's benchmark section (§5.1):
 *   "uniform distribution in the range of (0, 1], normal distribution with mean 0 and
 *    standard deviation 1, and a specially designed radix-adversarial distribution,
 *    where the first M bits of all the input elements are the same."
 * and the radix-adversarial example of PAPER.md:162-164 (§3.2): floats in
 * [1.0, 1.00049] = bit patterns [0x3F800000, 0x3F800FFF] share their first 20 bits.
 *
 * Recipe:
 *   x_i = splitmix64_mix(seed + (i + 1) * 0x9E3779B97F4A7C15), i = global element index
 *   uniform (0,1]:  u = x_i >> 32;  f = fl(fl((float)u) * 2^-32) + 2^-33   (round-to-nearest, no FMA)
 *   normal(0,1):    Box-Muller in double from u1 = hi32, u2 = lo32 (each mapped to (0,1]), rounded to f32
 *   adversarial M:  bits = (0x3F800000 & ~mask) | (u & mask), mask = 2^(32-M) - 1
 *   raw u32 / u64:  u = x_i >> 32 / x_i
 * "global index" lets a row of a batch or a shard of a split row be generated independently
 * and still equal the corresponding slice of the whole array.
 */
#include <stdint.h>
#include <math.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

static inline uint64_t draw(uint64_t seed, uint64_t i) {
  return mix64(seed + (i + 1ULL) * 0x9E3779B97F4A7C15ULL);
}

/* (0,1] from a 32-bit integer, cuRAND-style: fl(fl(u) * 2^-32) + 2^-33. volatile blocks contraction. */
static inline float u01f(uint32_t u) {
  volatile float a = (float)u;
  volatile float b = a * 2.3283064365386963e-10f; /* 2^-32, exact scaling */
  return b + 1.1641532182693481e-10f;             /* 2^-33 */
}

void gen_uniform_f32(uint64_t seed, uint64_t offset, int64_t n, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = u01f((uint32_t)(draw(seed, offset + (uint64_t)i) >> 32));
}

void gen_normal_f32(uint64_t seed, uint64_t offset, int64_t n, float* out) {
  const double two_pi = 6.283185307179586476925286766559;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    uint64_t x = draw(seed, offset + (uint64_t)i);
    double u1 = ((double)(uint32_t)(x >> 32) + 1.0) * 2.3283064365386963e-10; /* (0,1] */
    double u2 = ((double)(uint32_t)x + 0.5) * 2.3283064365386963e-10;         /* (0,1) */
    out[i] = (float)(sqrt(-2.0 * log(u1)) * cos(two_pi * u2));
  }
}

void gen_adversarial_f32(uint64_t seed, uint64_t offset, int64_t n, int m_bits, float* out) {
  uint32_t mask = (m_bits >= 32) ? 0u : (uint32_t)((1ULL << (32 - m_bits)) - 1ULL);
  uint32_t base = 0x3F800000u & ~mask;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    uint32_t u = (uint32_t)(draw(seed, offset + (uint64_t)i) >> 32);
    uint32_t b = base | (u & mask);
    memcpy(&out[i], &b, 4);
  }
}

void gen_u32(uint64_t seed, uint64_t offset, int64_t n, uint32_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = (uint32_t)(draw(seed, offset + (uint64_t)i) >> 32);
}

void gen_u64(uint64_t seed, uint64_t offset, int64_t n, uint64_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = draw(seed, offset + (uint64_t)i);
}

/* uniform (0,1] in double: ((x >> 11) + 1) * 2^-53 */
void gen_uniform_f64(uint64_t seed, uint64_t offset, int64_t n, double* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = (double)((draw(seed, offset + (uint64_t)i) >> 11) + 1ULL) * 1.1102230246251565e-16;
}

int gen_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
