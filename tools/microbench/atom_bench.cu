// On-chip accumulation micro-benchmarks (sm_100a).
//
// These measure the denominators for the histogram kernel's on-chip roofline
// (DESIGN.md "Roofline"): how many accumulate-updates per SM per clock the
// shared-memory pipe sustains for the accumulator layouts the histogram
// builder can use.  Address generation is 2 integer ops per access so the loop
// is not issue-bound on it.  Not part of the product path; run via gpurun.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o atom_bench atom_bench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t;
}
struct Stat { unsigned long long cyc; unsigned long long ns; };

// All modes: a "row" (bin) index r_i = (seed + i * 0x9E3779B1) >> (32 - LOGROWS) (cheap pseudo-random),
// lanes address consecutive words of the row (lanes = channels, distinct banks).
// MODE 0: ATOMS.ADD u32 (atomicAdd, return unused)
// MODE 1: red.shared.add.u32 (PTX red)
// MODE 2: int32 plain RMW, warp-owned region, U rows in flight (LDS x U, IADD x U, STS x U)
// MODE 3: int64 plain RMW, warp-owned, U rows in flight
// MODE 4: fp32 atomicAdd (CAS loop on sm_100a)
// MODE 5: u64 atomicAdd (CAS loop)
// MODE 6: LDS.64 only (sum into register)
// MODE 7: STS.64 only
// MODE 8: ATOMS.ADD u32, all lanes of a warp on ONE word (hot-bin worst case)
// MODE 9: ATOMS.ADD u32 where lanes = rows (random row per lane, 1 channel) - small-d mapping
template <int MODE, int U>
__global__ void __launch_bounds__(1024) kbench(int iters, int logrows, int rowwords, Stat* st, int* sink) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint32_t* s32 = (uint32_t*)smem;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int words_total = (1 << logrows) * rowwords * ((MODE == 2 || MODE == 3 || MODE == 6 || MODE == 7) ? nw : 1)
                          * ((MODE == 3 || MODE == 5 || MODE == 6 || MODE == 7) ? 2 : 1);
  for (int i = threadIdx.x; i < words_total; i += blockDim.x) s32[i] = 0;
  __syncthreads();
  uint32_t seed = (blockIdx.x * 977u + warp * 131u) * 0x85EBCA6Bu;
  if (MODE == 9) seed += lane * 0x27D4EB2Fu;
  const int sh = 32 - logrows;
  unsigned long long c0 = clock64(); uint64_t t0 = gtimer();
  uint64_t acc64 = 0;
  if (MODE == 0 || MODE == 1 || MODE == 4 || MODE == 5 || MODE == 8 || MODE == 9) {
    for (int i = 0; i < iters; i += U) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        uint32_t r = (seed + (uint32_t)(i + u) * 0x9E3779B1u) >> sh;
        int a = r * rowwords + lane;
        if (MODE == 0) atomicAdd(&s32[a], (uint32_t)lane + 1u);
        if (MODE == 1) asm volatile("red.shared.add.u32 [%0], %1;" :: "r"((uint32_t)__cvta_generic_to_shared(&s32[a])), "r"(lane + 1) : "memory");
        if (MODE == 4) atomicAdd(&((float*)s32)[a], 1.5f);
        if (MODE == 5) atomicAdd(&((unsigned long long*)s32)[r * rowwords + lane], 3ull);
        if (MODE == 8) atomicAdd(&s32[r * rowwords], (uint32_t)lane + 1u);
        if (MODE == 9) atomicAdd(&s32[r * rowwords], (uint32_t)lane + 1u);
      }
    }
  } else if (MODE == 2) {
    uint32_t* reg = s32 + warp * ((1 << logrows) * rowwords);
    for (int i = 0; i < iters; i += U) {
      int a[U]; uint32_t v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) a[u] = (int)(((seed + (uint32_t)(i + u) * 0x9E3779B1u) >> sh) * rowwords + lane);
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = reg[a[u]];
#pragma unroll
      for (int u = 0; u < U; ++u) reg[a[u]] = v[u] + (uint32_t)u + 1u;
    }
  } else if (MODE == 3 || MODE == 6 || MODE == 7) {
    unsigned long long* reg = (unsigned long long*)s32 + warp * ((1 << logrows) * rowwords);
    for (int i = 0; i < iters; i += U) {
      int a[U]; unsigned long long v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) a[u] = (int)(((seed + (uint32_t)(i + u) * 0x9E3779B1u) >> sh) * rowwords + lane);
      if (MODE == 3) {
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = reg[a[u]];
#pragma unroll
        for (int u = 0; u < U; ++u) reg[a[u]] = v[u] + (unsigned long long)(u + 1);
      } else if (MODE == 6) {
#pragma unroll
        for (int u = 0; u < U; ++u) acc64 += reg[a[u]];
      } else {
#pragma unroll
        for (int u = 0; u < U; ++u) reg[a[u]] = (unsigned long long)(i + u);
      }
    }
  }
  __syncthreads();
  unsigned long long c1 = clock64(); uint64_t t1 = gtimer();
  if (threadIdx.x == 0) { st[blockIdx.x].cyc = c1 - c0; st[blockIdx.x].ns = t1 - t0; }
  uint32_t acc = (uint32_t)acc64;
  for (int i = threadIdx.x; i < words_total; i += blockDim.x) acc += s32[i];
  if (acc == 0x7fffffffu) sink[0] = acc;
}

// global REDG.ADD.64, cheap addresses, lanes = consecutive words of a random row (hist-like)
__global__ void kredg(int iters, int logrows, unsigned long long* g, Stat* st) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t seed = (blockIdx.x * 977u + warp * 131u) * 0x85EBCA6Bu;
  const int sh = 32 - logrows;
  unsigned long long c0 = clock64(); uint64_t t0 = gtimer();
  for (int i = 0; i < iters; i += 4) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      uint32_t r = (seed + (uint32_t)(i + u) * 0x9E3779B1u) >> sh;
      atomicAdd(&g[(size_t)r * 32 + lane], 1ull);
    }
  }
  __syncthreads();
  unsigned long long c1 = clock64(); uint64_t t1 = gtimer();
  if (threadIdx.x == 0) { st[blockIdx.x].cyc = c1 - c0; st[blockIdx.x].ns = t1 - t0; }
}

template <int MODE, int U>
int run(const char* name, int bps, int threads, int logrows, int rowwords, int iters, Stat* dst, int* dsink, int nsm) {
  int nw = threads / 32;
  size_t words = (size_t)(1 << logrows) * rowwords * ((MODE == 2 || MODE == 3 || MODE == 6 || MODE == 7) ? nw : 1)
                 * ((MODE == 3 || MODE == 5 || MODE == 6 || MODE == 7) ? 2 : 1);
  int smem = (int)(words * 4);
  if (smem > 227 * 1024) { printf("%-40s skipped (smem %d)\n", name, smem); return 0; }
  CK(cudaFuncSetAttribute(kbench<MODE, U>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  int grid = nsm * bps;
  kbench<MODE, U><<<grid, threads, smem>>>(iters / 8, logrows, rowwords, dst, dsink);
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kbench<MODE, U><<<grid, threads, smem>>>(iters, logrows, rowwords, dst, dsink);
  cudaEventRecord(e1);
  CK(cudaDeviceSynchronize());
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  static Stat h[148 * 64];
  CK(cudaMemcpy(h, dst, sizeof(Stat) * grid, cudaMemcpyDeviceToHost));
  double cyc = 0, ns = 0; for (int i = 0; i < grid; ++i) { cyc += h[i].cyc; ns += h[i].ns; }
  double mhz = cyc / ns * 1e3;
  double ops = (double)grid * threads * iters;
  double per_s = ops / (ms * 1e-3);
  printf("%-40s blk/SM=%d thr=%4d U=%d smem=%6d %8.3f ms %9.2f Glane-op/s clk=%5.0f MHz %6.2f lane-op/clk/SM\n",
         name, bps, threads, U, smem, ms, per_s * 1e-9, mhz, per_s / (mhz * 1e6) / nsm);
  return 0;
}

int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  printf("device %s sms=%d smemPerBlockOptin=%zu smemPerSM=%zu L2=%d\n", p.name,
         p.multiProcessorCount, p.sharedMemPerBlockOptin, p.sharedMemPerMultiprocessor, p.l2CacheSize);
  int nsm = p.multiProcessorCount;
  Stat* dst; int* dsink; CK(cudaMalloc(&dst, sizeof(Stat) * nsm * 64)); CK(cudaMalloc(&dsink, 64));
  const int it = 1 << 14;
  for (int thr : {1024}) {
    run<0, 8>("ATOMS.ADD u32 lanes=channels", 1, thr, 10, 32, it, dst, dsink, nsm);
    run<1, 8>("red.shared.add.u32 lanes=channels", 1, thr, 10, 32, it, dst, dsink, nsm);
    run<4, 8>("atomicAdd f32 smem (CAS)", 1, thr, 10, 32, it / 4, dst, dsink, nsm);
    run<5, 8>("atomicAdd u64 smem (CAS)", 1, thr, 9, 32, it / 4, dst, dsink, nsm);
    run<8, 8>("ATOMS.ADD u32 warp on one word", 1, thr, 10, 32, it / 8, dst, dsink, nsm);
    run<9, 8>("ATOMS.ADD u32 lanes=rows (rand word)", 1, thr, 14, 1, it, dst, dsink, nsm);
  }
  for (int thr : {256, 512, 1024}) {
    int lr = thr == 256 ? 6 : thr == 512 ? 5 : 4;     // keep per-warp region inside smem
    run<2, 4>("int32 plain RMW warp-owned", 1, thr, lr, 32, it, dst, dsink, nsm);
    run<2, 8>("int32 plain RMW warp-owned", 1, thr, lr, 32, it, dst, dsink, nsm);
    run<3, 4>("int64 plain RMW warp-owned", 1, thr, lr - 1, 32, it, dst, dsink, nsm);
    run<3, 8>("int64 plain RMW warp-owned", 1, thr, lr - 1, 32, it, dst, dsink, nsm);
    run<6, 8>("LDS.64 only", 1, thr, lr - 1, 32, it, dst, dsink, nsm);
    run<7, 8>("STS.64 only", 1, thr, lr - 1, 32, it, dst, dsink, nsm);
  }
  run<0, 8>("ATOMS.ADD u32 lanes=channels 2blk", 2, 512, 9, 32, it, dst, dsink, nsm);
  for (int lr : {15, 18, 21}) {
    unsigned long long* g; size_t words = (size_t(1) << lr) * 32; CK(cudaMalloc(&g, 8 * words)); cudaMemset(g, 0, 8 * words);
    int grid = nsm * 4, thr = 512, iters = 1 << 11;
    kredg<<<grid, thr>>>(iters / 8, lr, g, dst); CK(cudaDeviceSynchronize());
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0); kredg<<<grid, thr>>>(iters, lr, g, dst); cudaEventRecord(e1);
    CK(cudaDeviceSynchronize()); float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)grid * thr * iters;
    printf("REDG.ADD.64 hist-like over %6.0f MB: %8.3f ms %8.2f Gop/s\n", words * 8.0 / 1e6, ms, ops / ms * 1e-6);
    cudaFree(g);
  }
  return 0;
}
