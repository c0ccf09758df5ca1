// peaks.cu — same-run on-chip roofline denominators for bench.py.
//
// Not part of the product path: bench.py loads libgbdtmo_peaks.so with ctypes and calls
// peaks_atoms() right before its timed region, so the histogram kernel's `roofline.peak` is the
// shared-memory atomic rate measured on the same GPU, in the same process, at the same clocks.
//
// mode 0  red.shared.add.u32, lanes = 32 consecutive words of a pseudo-random 32-word record
//         (32 distinct banks): the pipe ceiling of conflict-free 32-bit shared atomics.
// mode 1  the histogram kernel's lane map (hist.cu, K = 16): lanes 0-15 add to words c of a
//         random 192-word bin record, lanes 16-31 to words 16 + c of another random record (the
//         swapped-limb row pair), i.e. the exact address pattern of one k_hist_smem instruction.
// mode 2  a row-per-instruction lane map (proposal): all 32 lanes add to the 32 words (16 lo + 16 hi
//         limbs) of ONE random 32-word feature slot of a random 192-word bin record.
// All: 1024 threads x 1 CTA per SM, ~200 KB of shared memory, U = 8 atomics in flight per
// thread; cycles from clock64 (max over CTAs), time from %globaltimer.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ void red_add(uint32_t addr, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}

template <int MODE>
__global__ void __launch_bounds__(1024, 1) k_atoms(int iters, int records, int lrec, unsigned long long* cyc,
                                                   unsigned long long* ns, unsigned* sink) {
  extern __shared__ __align__(16) uint32_t s[];
  constexpr int RW = MODE == 0 ? 32 : 192;            // words per record
  static_assert(MODE >= 0 && MODE <= 2, "mode");
  for (int i = threadIdx.x; i < records * RW; i += blockDim.x) s[i] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(s);
  uint32_t seed = (blockIdx.x * 977u + warp * 131u) * 0x85EBCA6Bu;
  const uint32_t lanew = MODE == 0 ? lane : ((lane & 15) + ((lane >> 4) << 4));
  const unsigned long long c0 = clock64();
  const uint64_t t0 = gtimer();
  for (int i = 0; i < iters; i += 8) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t h = (seed + (uint32_t)(i + u) * 0x9E3779B1u);
      // mode 1: the two half-warps take two different random records (two rows' bins)
      const uint32_t rec = MODE == 1 ? ((lane < 16 ? h : (h * 0x2545F491u)) >> lrec) : (h >> lrec);
      const uint32_t jw = MODE == 2 ? 32u * ((uint32_t)(i + u) % 6u) : 0u;
      red_add(base + 4u * (rec * RW + jw + lanew), (uint32_t)u + 1u);
    }
  }
  __syncthreads();
  const unsigned long long c1 = clock64();
  const uint64_t t1 = gtimer();
  if (threadIdx.x == 0) {
    cyc[blockIdx.x] = c1 - c0;
    ns[blockIdx.x] = t1 - t0;
  }
  uint32_t acc = 0;
  for (int i = threadIdx.x; i < records * RW; i += blockDim.x) acc += s[i];
  if (acc == 0x7fffffffu) sink[0] = acc;
}

}  // namespace

// Runs mode `mode` (0 or 1) on `device` with `iters` atomics per thread (multiple of 8) and writes
// lane_ops_per_clk_sm (32 lanes x instructions / (max CTA cycles x SMs)), lane_ops_per_s (total
// lane operations / max CTA wall time) and the effective SM clock (MHz).  Returns a cudaError_t.
extern "C" int peaks_atoms(int device, int mode, int iters, double* lane_ops_per_clk_sm, double* lane_ops_per_s,
                           double* clk_mhz) {
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(device);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  const int RW = mode == 0 ? 32 : 192;
  const int records = mode == 0 ? 1024 : 256;            // 128 KB / 192 KB, a power of two
  const int lrec = mode == 0 ? 22 : 24;                  // record = top log2(records) bits of a hash
  if (mode < 0 || mode > 2) return (int)cudaErrorInvalidValue;
  const int smem = records * RW * 4;
  unsigned long long *cyc = nullptr, *ns = nullptr;
  unsigned* sink = nullptr;
  cudaError_t e = cudaMalloc(&cyc, sizeof(unsigned long long) * sms * 2);
  if (e == cudaSuccess) e = cudaMalloc(&sink, 4);
  if (e == cudaSuccess) {
    ns = cyc + sms;
    auto kern = mode == 0 ? k_atoms<0> : mode == 1 ? k_atoms<1> : k_atoms<2>;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int rep = 0; rep < 2 && e == cudaSuccess; ++rep) {        // rep 0: warm-up
      kern<<<sms, 1024, smem>>>(iters, records, lrec, cyc, ns, sink);
      e = cudaDeviceSynchronize();
    }
  }
  if (e == cudaSuccess) {
    unsigned long long hc[1024], hn[1024];
    cudaMemcpy(hc, cyc, sizeof(unsigned long long) * sms, cudaMemcpyDeviceToHost);
    e = cudaMemcpy(hn, ns, sizeof(unsigned long long) * sms, cudaMemcpyDeviceToHost);
    unsigned long long mc = 0, mn = 0;
    for (int i = 0; i < sms; ++i) {
      mc = hc[i] > mc ? hc[i] : mc;
      mn = hn[i] > mn ? hn[i] : mn;
    }
    const double lane_ops = (double)sms * 1024.0 * iters;     // every thread: iters atomics x 1 lane
    *lane_ops_per_clk_sm = lane_ops / ((double)mc * sms);
    *lane_ops_per_s = lane_ops / ((double)mn * 1e-9);
    *clk_mhz = (double)mc / ((double)mn * 1e-3);
  }
  cudaFree(cyc);
  cudaFree(sink);
  cudaSetDevice(prev);
  return (int)e;
}
