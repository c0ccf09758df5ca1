// bin.cu — (a)1: per-feature quantile binning ("feature-value bin mapping",
// "cut points" PAPER.md:166, <= 256 bins PAPER.md:237, 255; exact rule = reading R14).
//
// Per tile of TC columns: transpose the column tile into order-preserving uint32 keys,
// sort every column with a stable 4-pass LSD radix sort (8-bit digits, per-(column, digit,
// tile) offsets), derive the cuts from the sorted column (distinct values if <= B of them,
// else the order statistics s[floor(j n / B)]), then bin(x) = #{cuts <= x} by bisection.
#include "common.cuh"

namespace gbdtmo {

constexpr int kBinTC = 64;          // columns per tile
constexpr int kSortTile = 4096;     // keys per radix block
constexpr int kSortThreads = 256;

__device__ __forceinline__ uint32_t f2key(float x) {
  uint32_t u = __float_as_uint(x == 0.0f ? 0.0f : x);     // -0.0 == +0.0
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float key2f(uint32_t k) {
  return __uint_as_float((k & 0x80000000u) ? (k ^ 0x80000000u) : ~k);
}

// X[i*ld + c0 + j] -> keys[j*n + i] for j < tc, through a 32x32 shared tile.
__global__ void k_bin_keys(const float* __restrict__ X, int64_t n, int64_t ld_x, int c0, int tc,
                           uint32_t* __restrict__ keys) {
  __shared__ uint32_t t[32][33];
  const int64_t i0 = (int64_t)blockIdx.x * 32;
  const int j0 = blockIdx.y * 32;
  for (int r = threadIdx.y; r < 32; r += blockDim.y) {
    const int64_t i = i0 + r;
    const int j = j0 + threadIdx.x;
    if (i < n && j < tc) t[r][threadIdx.x] = f2key(X[i * ld_x + c0 + j]);
  }
  __syncthreads();
  for (int r = threadIdx.y; r < 32; r += blockDim.y) {
    const int j = j0 + r;
    const int64_t i = i0 + threadIdx.x;
    if (i < n && j < tc) keys[(int64_t)j * n + i] = t[threadIdx.x][r];
  }
}

// counts[(col*256 + digit)*T + tile] = #keys of the tile with that digit
__global__ void __launch_bounds__(kSortThreads)
k_radix_count(const uint32_t* __restrict__ keys, int64_t n, int shift, uint32_t* __restrict__ counts, int64_t T) {
  __shared__ uint32_t hs[256];
  const int col = blockIdx.y;
  const int64_t tile = blockIdx.x;
  hs[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t* kc = keys + (int64_t)col * n;
  const int64_t beg = tile * kSortTile;
  for (int j = 0; j < kSortTile / kSortThreads; ++j) {
    const int64_t pos = beg + j * kSortThreads + threadIdx.x;
    if (pos < n) atomicAdd(&hs[(kc[pos] >> shift) & 0xFFu], 1u);
  }
  __syncthreads();
  counts[((int64_t)col * 256 + threadIdx.x) * T + tile] = hs[threadIdx.x];
}

// In-place exclusive scan of counts[col][0 .. 256*T) (digit-major, tile-minor).
__global__ void __launch_bounds__(1024) k_radix_scan(uint32_t* __restrict__ counts, int64_t T) {
  __shared__ uint32_t ws[32];
  __shared__ uint32_t carry;
  const int col = blockIdx.x;
  uint32_t* c = counts + (int64_t)col * 256 * T;
  const int64_t total = 256 * T;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t b0 = 0; b0 < total; b0 += 1024) {
    const int64_t i = b0 + threadIdx.x;
    const uint32_t v = i < total ? c[i] : 0u;
    uint32_t x = v;
    for (int o = 1; o < 32; o <<= 1) { uint32_t y = __shfl_up_sync(0xffffffffu, x, o); if (lane >= o) x += y; }
    if (lane == 31) ws[w] = x;
    __syncthreads();
    if (w == 0) {
      uint32_t s = ws[lane];
      for (int o = 1; o < 32; o <<= 1) { uint32_t y = __shfl_up_sync(0xffffffffu, s, o); if (lane >= o) s += y; }
      ws[lane] = s;
    }
    __syncthreads();
    const uint32_t base = (w ? ws[w - 1] : 0u) + carry;
    if (i < total) c[i] = base + x - v;
    __syncthreads();
    if (threadIdx.x == 0) carry += ws[31];
    __syncthreads();
  }
}

// Stable scatter: the tile is consumed in rounds of 256 consecutive keys; ranks inside a round
// come from warp match + per-(warp, digit) counts, so equal digits keep their input order.
__global__ void __launch_bounds__(kSortThreads)
k_radix_scatter(const uint32_t* __restrict__ kin, uint32_t* __restrict__ kout, int64_t n, int shift,
                const uint32_t* __restrict__ counts, int64_t T) {
  constexpr int NW = kSortThreads / 32;
  __shared__ uint32_t base[256];
  __shared__ uint32_t run[256];
  __shared__ uint32_t wcnt[NW][256];
  __shared__ uint32_t woff[NW][256];
  const int col = blockIdx.y;
  const int64_t tile = blockIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  base[threadIdx.x] = counts[((int64_t)col * 256 + threadIdx.x) * T + tile];
  run[threadIdx.x] = 0;
  for (int x = 0; x < NW; ++x) wcnt[x][threadIdx.x] = 0;
  __syncthreads();
  const uint32_t* kc = kin + (int64_t)col * n;
  uint32_t* ko = kout + (int64_t)col * n;
  const uint32_t lt = (1u << lane) - 1u;
  for (int rd = 0; rd < kSortTile / kSortThreads; ++rd) {
    const int64_t pos = tile * kSortTile + (int64_t)rd * kSortThreads + threadIdx.x;
    const bool on = pos < n;
    const uint32_t key = on ? kc[pos] : 0u;
    const int dig = on ? (int)((key >> shift) & 0xFFu) : 256;
    const uint32_t peers = __match_any_sync(0xffffffffu, dig);
    const int rank = __popc(peers & lt);
    if (on && rank == 0) wcnt[w][dig] = __popc(peers);
    __syncthreads();
    {
      const int t = threadIdx.x;
      uint32_t acc = run[t];
      for (int x = 0; x < NW; ++x) { const uint32_t cx = wcnt[x][t]; woff[x][t] = acc; acc += cx; wcnt[x][t] = 0; }
      run[t] = acc;
    }
    __syncthreads();
    if (on) ko[base[dig] + woff[w][dig] + rank] = key;
    __syncthreads();
  }
}

// One block per column of the sorted tile: cuts and nbins (reading R14).
__global__ void __launch_bounds__(1024)
k_bin_cuts(const uint32_t* __restrict__ keys, int64_t n, int B, float* __restrict__ cuts, int32_t* __restrict__ nbins) {
  __shared__ uint32_t ws[32];
  __shared__ uint32_t sh_total, carry;
  const int col = blockIdx.x;
  const uint32_t* s = keys + (int64_t)col * n;
  float* cut = cuts + (int64_t)col * (B - 1);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  // distinct count (capped: we only need to know whether it is <= B)
  uint32_t local = 0;
  for (int64_t i = 1 + threadIdx.x; i < n; i += blockDim.x) local += s[i] != s[i - 1];
  for (int o = 16; o > 0; o >>= 1) local += __shfl_xor_sync(0xffffffffu, local, o);
  if (threadIdx.x == 0) sh_total = 0;
  __syncthreads();
  if (lane == 0) atomicAdd(&sh_total, local);
  for (int j = threadIdx.x; j < B - 1; j += blockDim.x) cut[j] = __int_as_float(0x7f800000);   // +inf
  __syncthreads();
  const uint64_t distinct = (uint64_t)sh_total + 1;
  if (distinct <= (uint64_t)B) {
    // rule (i): every distinct value except the smallest, in order
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (int64_t b0 = 1; b0 < n; b0 += blockDim.x) {
      const int64_t i = b0 + threadIdx.x;
      const uint32_t f = (i < n && s[i] != s[i - 1]) ? 1u : 0u;
      uint32_t x = f;
      for (int o = 1; o < 32; o <<= 1) { uint32_t y = __shfl_up_sync(0xffffffffu, x, o); if (lane >= o) x += y; }
      if (lane == 31) ws[w] = x;
      __syncthreads();
      if (w == 0) {
        uint32_t t = ws[lane];
        for (int o = 1; o < 32; o <<= 1) { uint32_t y = __shfl_up_sync(0xffffffffu, t, o); if (lane >= o) t += y; }
        ws[lane] = t;
      }
      __syncthreads();
      const uint32_t off = carry + (w ? ws[w - 1] : 0u) + x - f;
      if (f) cut[off] = key2f(s[i]);
      __syncthreads();
      if (threadIdx.x == 0) carry += ws[31];
      __syncthreads();
    }
    if (threadIdx.x == 0) nbins[col] = (int32_t)distinct;
  } else if (threadIdx.x == 0) {
    // rule (ii): order statistics s[floor(j n / B)], deduplicated, those <= s[0] dropped
    const float s0 = key2f(s[0]);
    int k = 0;
    float last = 0.0f;
    for (int j = 1; j <= B - 1; ++j) {
      const float v = key2f(s[((int64_t)j * n) / B]);
      if (v <= s0) continue;
      if (k > 0 && v == last) continue;
      cut[k++] = v;
      last = v;
    }
    nbins[col] = k + 1;
  }
}

// bins[i*ld + c0 + j] = #{cuts_j <= X[i, c0 + j]}
__global__ void k_bin_apply(const float* __restrict__ X, int64_t n, int64_t ld_x, int c0, int tc, int B,
                            const float* __restrict__ cuts, const int32_t* __restrict__ nbins,
                            uint8_t* __restrict__ bins, int64_t ld_bins) {
  extern __shared__ float sc[];          // [tc][B-1]
  __shared__ int nb[kBinTC];
  for (int e = threadIdx.x; e < tc * (B - 1); e += blockDim.x) sc[e] = cuts[(int64_t)c0 * (B - 1) + e];
  for (int j = threadIdx.x; j < tc; j += blockDim.x) nb[j] = nbins[c0 + j];
  __syncthreads();
  const int64_t total = n * tc;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / tc;
    const int j = (int)(e - i * tc);
    const float x = X[i * ld_x + c0 + j];
    const float* c = sc + j * (B - 1);
    int lo = 0, hi = nb[j] - 1;
    while (lo < hi) { const int mid = (lo + hi) >> 1; if (c[mid] <= x) lo = mid + 1; else hi = mid; }
    bins[i * ld_bins + c0 + j] = (uint8_t)lo;
  }
}

inline int64_t sort_tiles(int64_t n) { return (n + kSortTile - 1) / kSortTile; }

// dflt[f] = most frequent bin of feature f (ties: smallest).  One block per 8 features (one
// aligned 8-byte load per row), per-feature shared counters.
__global__ void __launch_bounds__(256) k_default_bins(const uint8_t* __restrict__ bins, int64_t n, int m, int64_t ld,
                                                      int B, int64_t min_count, int32_t* __restrict__ dflt) {
  __shared__ uint32_t c[8][256];
  for (int i = threadIdx.x; i < 8 * 256; i += blockDim.x) (&c[0][0])[i] = 0;
  __syncthreads();
  const int f0 = blockIdx.x * 8;
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
    const uint64_t w = *reinterpret_cast<const uint64_t*>(bins + i * ld + f0);
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (f0 + j < m) atomicAdd(&c[j][(w >> (8 * j)) & 0xFF], 1u);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;   // warp j -> feature f0 + j
  if (f0 + warp < m) {
    uint32_t best = 0;
    int bb = 0;
    for (int b = lane; b < B; b += 32) {
      const uint32_t v = c[warp][b];
      if (v > best) { best = v; bb = b; }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const uint32_t ov = __shfl_xor_sync(0xffffffffu, best, o);
      const int ob = __shfl_xor_sync(0xffffffffu, bb, o);
      if (ov > best || (ov == best && ob < bb)) { best = ov; bb = ob; }
    }
    if (lane == 0) dflt[f0 + warp] = ((int64_t)best >= min_count) ? bb : -1;
  }
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" size_t gbdtmo_bin_workspace_bytes(int64_t n, int32_t m, int32_t B) {
  (void)B;
  const int64_t tc = m < kBinTC ? m : kBinTC;
  return (size_t)(2 * tc * n * 4 + tc * 256 * sort_tiles(n) * 4 + 1024);
}

extern "C" gbdtmo_status gbdtmo_bin(gbdtmo_ctx c, const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t B,
                                    uint8_t* bins, int64_t ld_bins, float* cuts, int32_t* nbins, void* ws,
                                    size_t ws_bytes) {
  Ctx* ctx = (Ctx*)c;
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(X && bins && cuts && nbins && ws, "null pointer");
  GB_CHECK_ARG(n >= 1 && n < (int64_t(1) << 31) && m >= 1, "bad n or m");
  GB_CHECK_ARG(ld_x >= m && ld_bins >= m, "bad leading dimension");
  if (B > 256) { ctx->err = "gbdtmo_bin: B > 256 unsupported (bins are uint8)"; return GBDTMO_EUNSUPPORTED; }
  GB_CHECK_ARG(B >= 2, "B < 2");
  if (ws_bytes < gbdtmo_bin_workspace_bytes(n, m, B)) { ctx->err = "gbdtmo_bin: workspace too small"; return GBDTMO_ENOMEM; }
  const int64_t tcmax = m < kBinTC ? m : kBinTC;
  const int64_t T = sort_tiles(n);
  uint32_t* ka = (uint32_t*)ws;
  uint32_t* kb = ka + tcmax * n;
  uint32_t* counts = kb + tcmax * n;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_bin_apply, cudaFuncAttributeMaxDynamicSharedMemorySize, kBinTC * 255 * 4);
    attr = true;
  }
  for (int c0 = 0; c0 < m; c0 += kBinTC) {
    const int tc = (int)(m - c0 < kBinTC ? m - c0 : kBinTC);
    GB_LAUNCH(k_bin_keys, dim3((unsigned)((n + 31) / 32), (unsigned)((tc + 31) / 32)), dim3(32, 8), 0, X, n, ld_x, c0, tc, ka);
    uint32_t* kin = ka;
    uint32_t* kout = kb;
    for (int pass = 0; pass < 4; ++pass) {
      GB_LAUNCH(k_radix_count, dim3((unsigned)T, (unsigned)tc), kSortThreads, 0, kin, n, 8 * pass, counts, T);
      GB_LAUNCH(k_radix_scan, (unsigned)tc, 1024, 0, counts, T);
      GB_LAUNCH(k_radix_scatter, dim3((unsigned)T, (unsigned)tc), kSortThreads, 0, kin, kout, n, 8 * pass, counts, T);
      uint32_t* t = kin; kin = kout; kout = t;
    }
    GB_LAUNCH(k_bin_cuts, (unsigned)tc, 1024, 0, kin, n, B, cuts + (int64_t)c0 * (B - 1), nbins + c0);
    GB_LAUNCH(k_bin_apply, ctx->num_sms * 4, 256, (size_t)tc * (B - 1) * 4, X, n, ld_x, c0, tc, B, cuts, nbins, bins, ld_bins);
  }
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_default_bins(gbdtmo_ctx c, const uint8_t* bins, int64_t n, int32_t m, int64_t ld_bins,
                                             int32_t B, int64_t min_count, int32_t* dflt) {
  Ctx* ctx = (Ctx*)c;
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(bins && dflt, "null pointer");
  GB_CHECK_ARG(n >= 1 && m >= 1 && ld_bins >= m && ld_bins % 8 == 0 && B >= 2 && B <= 256, "bad shape");
  GB_CHECK_ARG(((uintptr_t)bins & 7) == 0, "bins must be 8-byte aligned");
  GB_LAUNCH(k_default_bins, (unsigned)((m + 7) / 8), 256, 0, bins, n, m, ld_bins, B, min_count, dflt);
  return GBDTMO_OK;
}
