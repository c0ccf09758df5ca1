// Shared-memory atomic throughput vs which 128-byte lines an instruction hits (measurement only).
// 1024 128-B lines (128 KB); every mode: same ALU per atomic (IADD + AND + LEA + optional LOP).
//  0  32 lanes -> one random line, any parity
//  1  32 lanes -> one random EVEN line
//  2  32 lanes -> one random ODD line
//  3  lanes 0-15 -> words 0-15 of random line L1, 16-31 -> words 16-31 of random line L2 (any parity)
//  4  as 3, L1 and L2 both even
//  5  as 3, L1 even and L2 odd
//  6  as 0, lines restricted to lines 6r + j (r random, j = warp's feature slot 0..5): the histogram's
//     record layout (192-word records, line parity = j parity)
//  7  as 6 with the swizzle line 6r + (j ^ (r & 1))
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void __launch_bounds__(1024, 1) k(int iters, unsigned long long* cyc, unsigned* sink) {
  extern __shared__ __align__(16) uint32_t s[];
  constexpr int NL = 1024;
  for (int i = threadIdx.x; i < NL * 32; i += blockDim.x) s[i] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(s);
  uint32_t r = (warp * 37u + blockIdx.x * 11u) & (NL - 1);
  const uint32_t step = (MODE >= 3 && MODE <= 5 && lane >= 16) ? 311u : 173u;
  if (MODE >= 3 && MODE <= 5 && lane >= 16) r = (r * 5u + 77u) & (NL - 1);
  const uint32_t j = warp % 6;
  const unsigned long long c0 = clock64();
  for (int i = 0; i < iters; i += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      r = (r + step) & (NL - 1);
      uint32_t line;
      if (MODE == 0 || MODE == 3) line = r;
      else if (MODE == 1 || (MODE == 4) || (MODE == 5 && lane < 16)) line = r & ~1u;
      else if (MODE == 2 || MODE == 5) line = r | 1u;
      else if (MODE == 6) line = ((r % 170u) * 6u + j);
      else line = ((r % 170u) * 6u + (j ^ ((r % 170u) & 1u)));
      asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(base + 4u * (line * 32u + lane)), "r"((uint32_t)u + 1u)
                   : "memory");
    }
  }
  __syncthreads();
  const unsigned long long c1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
  uint32_t acc = 0;
  for (int i = threadIdx.x; i < NL * 32; i += blockDim.x) acc += s[i];
  if (acc == 0x7fffffffu) sink[0] = acc;
}

template <int MODE>
void run(int sms, unsigned long long* cyc, unsigned* sink) {
  const int smem = 1024 * 32 * 4;
  cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 40000;
  for (int rep = 0; rep < 2; ++rep) k<MODE><<<sms, 1024, smem>>>(iters, cyc, sink);
  cudaDeviceSynchronize();
  unsigned long long h[1024];
  cudaMemcpy(h, cyc, 8 * sms, cudaMemcpyDeviceToHost);
  unsigned long long mx = 0;
  for (int i = 0; i < sms; ++i) mx = h[i] > mx ? h[i] : mx;
  printf("{\"mode\": %d, \"atoms_instr_per_clk_sm\": %.4f, \"err\": \"%s\"}\n", MODE, 32.0 * iters / mx,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* cyc;
  unsigned* sink;
  cudaMalloc(&cyc, 8 * 1024);
  cudaMalloc(&sink, 4);
  run<0>(sms, cyc, sink); run<1>(sms, cyc, sink); run<2>(sms, cyc, sink); run<3>(sms, cyc, sink);
  run<4>(sms, cyc, sink); run<5>(sms, cyc, sink); run<6>(sms, cyc, sink); run<7>(sms, cyc, sink);
  return 0;
}
