// Lane-map micro-benchmark for the histogram's limb atomics (measurement only).
// Every mode does the same ALU per atomic (one IADD + one AND + one LEA from a per-warp seed), so
// differences are the shared-memory atomic unit's, not issue:
//  0  32 lanes -> 32 consecutive words of one random 32-word record          (1 line)
//  1  lanes 0-15 -> words c of random 192-word record r1, 16-31 -> words 16+c of r2 (2 lines: k_hist_smem)
//  2  32 lanes -> the 32-word slot j of one random 192-word record            (1 line, ROW1 map)
//  3  lanes 0-15 -> words c of slot j of r1, 16-31 -> words 16+c of slot j' of r2 (2 lines, different j)
//  4  as 1 but the two rows' records are the same (r2 = r1)                  (1 line)
//  5  lanes -> 32 random words (lanes = rows, one count each)                 (count atomics)
//  6  mode 1's lane map over 128 records (96 KB footprint instead of 192 KB)
//  7  mode 0's lane map over 1536 records (192 KB footprint instead of 128 KB)
//  8  mode 1's lane map over 160 records (120 KB)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o atoms_lanemap atoms_lanemap.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void __launch_bounds__(1024, 1) k(int iters, unsigned long long* cyc, unsigned* sink) {
  extern __shared__ __align__(16) uint32_t s[];
  constexpr int RW = (MODE == 0 || MODE == 7) ? 32 : 192;
  constexpr int NREC = MODE == 0 ? 1024 : MODE == 7 ? 1536 : MODE == 6 ? 128 : MODE == 8 ? 160 : 256;
  for (int i = threadIdx.x; i < NREC * RW; i += blockDim.x) s[i] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(s);
  // per-lane start offsets (computed once): the loop only advances a record index
  uint32_t r1 = (warp * 37u + blockIdx.x * 11u) % NREC, r2 = (r1 * 5u + 77u) % NREC;
  uint32_t j1 = warp % 6, j2 = (warp + 3) % 6;
  uint32_t rec = (MODE == 1 || MODE == 3 || MODE == 6 || MODE == 8) && lane >= 16 ? r2 : r1;
  uint32_t slot = MODE == 2 ? 32u * j1 : MODE == 3 ? 32u * (lane < 16 ? j1 : j2) : 0u;
  uint32_t word = MODE == 5 ? (lane * 97u) % (NREC * RW) : (uint32_t)lane;
  const uint32_t stepr = MODE == 5 ? 0u : ((lane < 16 || MODE == 4 || MODE == 0 || MODE == 2 || MODE == 7) ? 173u : 311u);
  const unsigned long long c0 = clock64();
  for (int i = 0; i < iters; i += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      if ((NREC & (NREC - 1)) == 0) rec = (rec + stepr) & (NREC - 1);
      else { rec += stepr; rec = rec >= NREC ? rec - NREC : rec; }
      if (MODE == 5) word = (word + 1237u * (u + 1)) & (NREC * RW - 1);
      const uint32_t w = MODE == 5 ? word : rec * RW + slot + word;
      asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(base + 4u * w), "r"((uint32_t)u + 1u) : "memory");
    }
  }
  __syncthreads();
  const unsigned long long c1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
  uint32_t acc = 0;
  for (int i = threadIdx.x; i < NREC * RW; i += blockDim.x) acc += s[i];
  if (acc == 0x7fffffffu) sink[0] = acc;
}

template <int MODE>
void run(int sms, unsigned long long* cyc, unsigned* sink) {
  const int smem = (MODE == 0 ? 1024 * 32 : MODE == 7 ? 1536 * 32 : MODE == 6 ? 128 * 192 : MODE == 8 ? 160 * 192 : 256 * 192) * 4;
  cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 40000;
  for (int rep = 0; rep < 2; ++rep) k<MODE><<<sms, 1024, smem>>>(iters, cyc, sink);
  cudaDeviceSynchronize();
  unsigned long long h[1024];
  cudaMemcpy(h, cyc, 8 * sms, cudaMemcpyDeviceToHost);
  unsigned long long mx = 0;
  for (int i = 0; i < sms; ++i) mx = h[i] > mx ? h[i] : mx;
  printf("{\"mode\": %d, \"lane_ops_per_clk_sm\": %.3f, \"atoms_instr_per_clk_sm\": %.4f, \"err\": \"%s\"}\n", MODE,
         1024.0 * iters / mx, 32.0 * iters / mx, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* cyc;
  unsigned* sink;
  cudaMalloc(&cyc, 8 * 1024);
  cudaMalloc(&sink, 4);
  run<0>(sms, cyc, sink); run<1>(sms, cyc, sink); run<2>(sms, cyc, sink);
  run<3>(sms, cyc, sink); run<4>(sms, cyc, sink); run<5>(sms, cyc, sink);
  run<6>(sms, cyc, sink); run<7>(sms, cyc, sink); run<8>(sms, cyc, sink);
  return 0;
}
