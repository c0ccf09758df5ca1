/*
 * gen_rng.h — counter-based synthetic-input generator (shared by the host and the
 * device builds of gen/ ONLY).  Holds none of the method's arithmetic: it maps
 * (seed, stream, index) to bits and to fp32 values with exactly-rounded IEEE
 * operations (integer ops, one fp64 multiply, one fp64->fp32 rounding), so the
 * host (gcc, -ffp-contract=off) and the device (nvcc, explicit _rn intrinsics)
 * produce bit-identical values for any element, independently of any other.
 */
#ifndef GBDTMO_GEN_RNG_H
#define GBDTMO_GEN_RNG_H
#include <stdint.h>

#if defined(__CUDACC__)
#define GEN_HD __host__ __device__ __forceinline__
#else
#define GEN_HD static inline
#endif

/* splitmix64 finaliser (Steele, Lea, Flood 2014). */
GEN_HD uint64_t gen_mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* 64 random bits for element `index` of stream `stream` under `seed`. */
GEN_HD uint64_t gen_bits(uint64_t seed, uint64_t stream, uint64_t index) {
  return gen_mix64(gen_mix64(seed * 0xD1B54A32D192ED03ull + stream * 0x632BE59BD9B4E019ull) + index);
}

/* Approximately standard-normal fp32: Irwin-Hall sum of four 32-bit uniforms,
 * centred and scaled to unit variance: z = (S - 2^33) * 2^-32 * sqrt(3).
 * S is exact in fp64 (< 2^34); the product is one correctly-rounded fp64 multiply
 * (2^-32 * sqrt(3) is a single fp64 constant); the result is rounded once to fp32. */
GEN_HD double gen_irwin_hall_f64(uint64_t a, uint64_t b) {
  uint64_t s = (a & 0xFFFFFFFFull) + (a >> 32) + (b & 0xFFFFFFFFull) + (b >> 32);
  double c = (double)((int64_t)s - (int64_t)0x200000000ll);
#if defined(__CUDA_ARCH__)
  return __dmul_rn(c, 4.0327450436746636e-10);
#else
  return c * 4.0327450436746636e-10;    /* = sqrt(3) / 2^32 rounded to fp64 */
#endif
}

GEN_HD float gen_normal_f32(uint64_t seed, uint64_t stream, uint64_t index) {
  uint64_t a = gen_bits(seed, stream, 2 * index), b = gen_bits(seed, stream, 2 * index + 1);
#if defined(__CUDA_ARCH__)
  return __double2float_rn(gen_irwin_hall_f64(a, b));
#else
  return (float)gen_irwin_hall_f64(a, b);
#endif
}

/* MNIST-shaped pixel: 0 with probability zero_q24 / 2^24, else a uniform integer 1..255. */
GEN_HD float gen_pixel_f32(uint64_t seed, uint64_t stream, uint64_t index, uint32_t zero_q24) {
  uint64_t u = gen_bits(seed, stream, index);
  if ((uint32_t)(u >> 40) < zero_q24) return 0.0f;
  return (float)(1u + (uint32_t)((u & 0xFFFFFFFFull) % 255u));
}

/* Uniform in [0, 1) with 53 bits (host-side label/noise generation). */
GEN_HD double gen_uniform_f64(uint64_t seed, uint64_t stream, uint64_t index) {
  return (double)(gen_bits(seed, stream, index) >> 11) * 1.1102230246251565e-16;
}

enum { GEN_KIND_NORMAL = 0, GEN_KIND_PIXEL = 1 };

#endif
