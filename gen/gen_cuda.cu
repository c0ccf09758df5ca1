/*
 * gen_cuda.cu — device build of the synthetic-input generator (see gen_rng.h).
 * Bench-only (inputs for the large configs are generated in HBM); bit-identical to gen.c.
 */
#include <cuda_runtime.h>
#include "gen_rng.h"

__global__ void gen_matrix_kernel(uint64_t seed, uint64_t stream, int32_t kind, uint32_t zero_q24,
                                  int64_t r0, int64_t nr, int64_t c0, int64_t nc, int64_t ncols_total,
                                  float* out, int64_t ld_out) {
  int64_t total = nr * nc;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total;
       t += (int64_t)gridDim.x * blockDim.x) {
    int64_t i = t / nc, j = t - i * nc;
    uint64_t idx = (uint64_t)((r0 + i) * ncols_total + (c0 + j));
    out[i * ld_out + j] = (kind == GEN_KIND_NORMAL) ? gen_normal_f32(seed, stream, idx)
                                                    : gen_pixel_f32(seed, stream, idx, zero_q24);
  }
}

extern "C" int gen_matrix_f32_cuda(uint64_t seed, uint64_t stream, int32_t kind, uint32_t zero_q24,
                                   int64_t r0, int64_t nr, int64_t c0, int64_t nc, int64_t ncols_total,
                                   float* out, int64_t ld_out, void* cuda_stream) {
  if (nr <= 0 || nc <= 0) return 0;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  gen_matrix_kernel<<<sms * 8, 256, 0, (cudaStream_t)cuda_stream>>>(seed, stream, kind, zero_q24, r0, nr, c0, nc,
                                                                    ncols_total, out, ld_out);
  return (int)cudaGetLastError();
}
