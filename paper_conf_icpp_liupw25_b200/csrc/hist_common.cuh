// hist_common.cuh — helpers shared by the histogram kernels (hist.cu, small.cu).
#pragma once
#include "common.cuh"

namespace gbdtmo {

// Raw window of a row's bins: NW 8-byte words starting at the 8-aligned byte f0 & ~7.
template <int NW>
struct BinWin { uint64_t w[NW]; };

template <int KF>
struct HistRow {
  static constexpr int NW = (KF + 14) / 8;    // raw words: covers (f0 & 7) + KF <= 7 + KF bytes
  static constexpr int SW = (KF + 7) / 8;     // words after shifting byte (f0 & 7) to position 0
};

// Shift the raw window right by 8*o bits (o = f0 & 7): byte j of the result = bin of feature f0 + j.
template <int NW, int SW>
__device__ __forceinline__ void shift_window(const uint64_t (&w)[NW], int o, uint64_t (&sw)[SW]) {
  const int sh = 8 * o;
#pragma unroll
  for (int i = 0; i < SW; ++i) {
    const uint64_t lo = w[i] >> sh;
    const uint64_t hi = (i + 1 < NW && sh) ? (w[i + 1] << (64 - sh)) : 0ull;
    sw[i] = lo | hi;
  }
}

template <int SW>
__device__ __forceinline__ uint32_t byte_of(const uint64_t (&sw)[SW], int j) {   // j compile-time after unroll
  const uint64_t x = sw[j >> 3];
  const uint32_t half = ((j & 7) < 4) ? (uint32_t)x : (uint32_t)(x >> 32);
  return __byte_perm(half, 0u, 0x4440u | (uint32_t)(j & 3));                     // PRMT: one byte, zero-extended
}

// PRMT in its default mode, where a selector nibble with bit 3 set replicates the sign bit of
// the selected byte (__byte_perm ignores that bit): prmt_sx(x, 0x4410) = x & 0xFFFF,
// prmt_sx(x, 0xBB32) = x >> 16 (arithmetic).
__device__ __forceinline__ uint32_t prmt_sx(uint32_t x, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, 0, %2;" : "=r"(r) : "r"(x), "r"(sel));
  return r;
}

// Shared-memory atomic add without return (SASS ATOMS.ADD) at a 32-bit shared address.
__device__ __forceinline__ void red_shared_add(uint32_t addr, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}

template <int SW>
__device__ __forceinline__ int byte_of_rt(const uint64_t (&sw)[SW], int j) {  // j runtime (per lane)
  uint64_t x = sw[0];
#pragma unroll
  for (int i = 1; i < SW; ++i) x = (j >= 8 * i) ? sw[i] : x;
  return (int)((x >> ((j & 7) * 8)) & 0xFFu);
}

}  // namespace gbdtmo
