// plan.cuh — device-side level planning: the list of histogram work chunks of a level.
// Runs inside a single CTA (blockDim.x == 256) so no host round trip is needed.
#pragma once
#include "common.cuh"

namespace gbdtmo {

constexpr int kPlanThreads = 256;

// Exclusive scan of one int per thread across a 256-thread block; returns the prefix and
// writes the block total to *total (all threads).
__device__ inline int block_excl_scan_256(int v, int* total) {
  __shared__ int warp_sums[kPlanThreads / 32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_sums[w] = x;
  __syncthreads();
  if (w == 0) {
    int s = lane < kPlanThreads / 32 ? warp_sums[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < kPlanThreads / 32) warp_sums[lane] = s;   // inclusive per warp
  }
  __syncthreads();
  int base = w > 0 ? warp_sums[w - 1] : 0;
  *total = warp_sums[kPlanThreads / 32 - 1];
  __syncthreads();
  return base + x - v;
}

// Write the build chunks of `level` into s.chunks: every node of the level with mode BUILD
// is cut into pieces of R rows, R = clamp(ceil(build_rows / target_chunks), kChunkMin, kChunkMax).
__device__ inline void plan_level_chunks(const gbdtmo_problem& p, const State& s, int level,
                                         int target_chunks, int64_t gmem_max_rows) {
  const int64_t LN = int64_t(1) << level, first = LN - 1;
  __shared__ long long sh_rows;
  __shared__ int sh_R, sh_base;
  if (threadIdx.x == 0) { sh_rows = 0; sh_base = 0; }
  __syncthreads();
  long long my = 0;
  auto is_gmem = [&](int64_t h) { return (int64_t)(s.node_end[h] - s.node_begin[h]) <= gmem_max_rows; };
  for (int64_t i = threadIdx.x; i < LN; i += blockDim.x) {
    int64_t h = first + i;
    if (s.node_mode[h] == MODE_BUILD && !is_gmem(h)) my += s.node_end[h] - s.node_begin[h];
  }
  atomicAdd((unsigned long long*)&sh_rows, (unsigned long long)my);
  __syncthreads();
  if (threadIdx.x == 0) {
    long long t = target_chunks > 0 ? target_chunks : 1;
    long long R = (sh_rows + t - 1) / t;
    if (R < kChunkMin) R = kChunkMin;
    if (R > kChunkMax) R = kChunkMax;
    sh_R = (int)R;
  }
  __syncthreads();
  const int R = sh_R;
  for (int64_t i0 = 0; i0 < LN; i0 += blockDim.x) {
    int64_t i = i0 + threadIdx.x;
    int nchunk = 0, b = 0, e = 0;
    if (i < LN) {
      int64_t h = first + i;
      if (s.node_mode[h] == MODE_BUILD && !is_gmem(h)) {
        b = s.node_begin[h]; e = s.node_end[h];
        nchunk = (e - b + R - 1) / R;
      }
    }
    int total;
    int off = block_excl_scan_256(nchunk, &total) + sh_base;
    for (int c = 0; c < nchunk; ++c) {
      int cb = b + c * R;
      int ce = cb + R < e ? cb + R : e;
      s.chunks[off + c] = make_int4((int)hist_index(p, level, i), cb, ce, nchunk == 1 ? 1 : 0);   // w = 1: sole writer
    }
    if (nchunk == 1) s.node_mode[first + i] = MODE_BUILD1;
    __syncthreads();
    if (threadIdx.x == 0) sh_base += total;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    s.misc[MISC_CHUNK_COUNT] = sh_base;
    s.misc[MISC_WORK_COUNTER] = 0;
    s.misc[MISC_CHUNK_ROWS] = R;
  }
  __syncthreads();
  // small BUILD nodes -> the global-atomic variant's list, with an exclusive row prefix
  __shared__ int sh_gn, sh_gr;
  if (threadIdx.x == 0) { sh_gn = 0; sh_gr = 0; }
  __syncthreads();
  for (int64_t i0 = 0; i0 < LN; i0 += blockDim.x) {
    const int64_t i = i0 + threadIdx.x;
    int take = 0, rows = 0, b = 0, e = 0;
    if (i < LN) {
      const int64_t h = first + i;
      if (s.node_mode[h] == MODE_BUILD && is_gmem(h)) { take = 1; b = s.node_begin[h]; e = s.node_end[h]; rows = e - b; }
    }
    int tn, tr;
    const int on = block_excl_scan_256(take, &tn);
    const int orow = block_excl_scan_256(rows, &tr);
    if (take) s.gnodes[sh_gn + on] = make_int4((int)hist_index(p, level, i), b, e, sh_gr + orow);
    __syncthreads();
    if (threadIdx.x == 0) { sh_gn += tn; sh_gr += tr; }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    s.misc[MISC_GNODE_COUNT] = sh_gn;
    s.misc[MISC_GNODE_ROWS] = sh_gr;
  }
  __syncthreads();
  // SMALL nodes (fused build + search) -> their own list
  __shared__ int sh_sn;
  if (threadIdx.x == 0) sh_sn = 0;
  __syncthreads();
  for (int64_t i0 = 0; i0 < LN; i0 += blockDim.x) {
    const int64_t i = i0 + threadIdx.x;
    int take = 0;
    if (i < LN) take = s.node_mode[first + i] == MODE_SMALL && s.node_state[first + i] == GBDTMO_NODE_ACTIVE;
    int tn;
    const int on = block_excl_scan_256(take, &tn);
    if (take) s.snodes[sh_sn + on] = make_int4((int)i, s.node_begin[first + i], s.node_end[first + i], 0);
    __syncthreads();
    if (threadIdx.x == 0) sh_sn += tn;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    s.misc[MISC_SNODE_COUNT] = sh_sn;
    s.misc[MISC_SWORK_COUNTER] = 0;
  }
}

}  // namespace gbdtmo
