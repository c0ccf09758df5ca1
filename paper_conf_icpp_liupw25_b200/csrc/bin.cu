// bin.cu — (a)1: per-feature quantile binning ("feature-value bin mapping",
// "cut points" PAPER.md:166, <= 256 bins PAPER.md:237, 255; exact rule = reading R14).
//
// Per tile of TC columns: transpose the column tile into order-preserving uint32 keys, find
// per column either its distinct values (if <= B of them) or the order statistics
// s[floor(j n / B)] by exact most-significant-digit selection (8 counting passes of 4 bits, no
// key is moved: the column is never sorted), then bin(x) = #{cuts <= x} by bisection.
#include "common.cuh"

namespace gbdtmo {

constexpr int kBinTC = 64;          // columns per tile

__device__ __forceinline__ uint32_t f2key(float x) {
  uint32_t u = __float_as_uint(x == 0.0f ? 0.0f : x);     // -0.0 == +0.0
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float key2f(uint32_t k) {
  return __uint_as_float((k & 0x80000000u) ? (k ^ 0x80000000u) : ~k);
}

// X[i*ld + c0 + j] -> keys[j*ldk + i] for j < tc, through a 32x32 shared tile.
__global__ void k_bin_keys(const float* __restrict__ X, int64_t n, int64_t ld_x, int c0, int tc,
                           uint32_t* __restrict__ keys, int64_t ldk) {
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
    if (i < n && j < tc) keys[(int64_t)j * ldk + i] = t[threadIdx.x][r];
  }
}

// ---- exact selection of the order statistics by most-significant-digit refinement.
//
// Per column, a sorted list A of at most 256 key prefixes, each with the rank of its first key
// (base), is refined 4 bits per pass over 8 passes.  A pass counts, for every key whose prefix is
// in A, the next digit (k_sel_count); k_sel_refine then keeps either every non-empty longer
// prefix while there are at most B of them ("few" mode: at the end they are the distinct values,
// rule (i)) or only the prefixes holding one of the ranks 0, floor(j n / B) ("targets" mode: at
// the end each is the key at that rank, rule (ii)).  Only counters are written: no keys move.
constexpr int kSelDigits = 16;                 // 4-bit digits
constexpr int kSelMax = 256;                   // prefixes tracked per column (>= B)
constexpr int kSelRows = 32768;                // keys per count block
constexpr int kSelHist = kSelMax * kSelDigits; // counters per column

struct SelMeta {
  int an;      // entries in A
  int mode;    // 0: few (all non-empty prefixes), 1: targets
  int pad[2];
};

__global__ void k_sel_init(int tc, SelMeta* __restrict__ meta, uint32_t* __restrict__ pre, uint32_t* __restrict__ base,
                           uint32_t* __restrict__ ghist) {
  const int col = blockIdx.x;
  if (threadIdx.x == 0) {
    meta[col].an = 1; meta[col].mode = 0;
    pre[col * kSelMax] = 0; base[col * kSelMax] = 0;
  }
  for (int e = threadIdx.x; e < kSelHist; e += blockDim.x) ghist[(int64_t)col * kSelHist + e] = 0;
}

// One counting pass.  pbits = 0: the first pass, counters by the key's top 12 bits (as if A held
// all 256 8-bit prefixes, 16 digits each).  pbits >= 12: counters of the next 4-bit digit per
// prefix in A; keys whose prefix is not in A are skipped.  Lookup: a 4096-entry table on the
// prefix's top 12 bits gives (first entry, entries) of A sharing them, so keys outside A cost one
// load and the rest a short search.  kout != null: the keys found in A (the only keys later
// passes can match) are compacted within the block's own slice of kout, their number written to
// cnt_out[col][block]; cnt_in != null: the block reads only that many keys of its slice.  Each thread
// takes 8 consecutive keys per step with two 16-byte loads; a warp whose lanes all hit one
// counter (constant or skewed columns) adds once.
__global__ void __launch_bounds__(256)
k_sel_count(const uint32_t* __restrict__ kin, const int32_t* __restrict__ cnt_in, int64_t n, int64_t ldk, int pbits,
            const SelMeta* __restrict__ meta, const uint32_t* __restrict__ pre, uint32_t* __restrict__ ghist,
            uint32_t* __restrict__ kout, int32_t* __restrict__ cnt_out) {
  __shared__ uint32_t sp[kSelMax];
  __shared__ uint32_t h[kSelHist];
  __shared__ uint32_t tab[4096];                 // (first << 16) | count, by top-12 bits of the prefix
  __shared__ int sh_out;
  const int col = blockIdx.y;
  const int64_t slot = (int64_t)col * gridDim.x + blockIdx.x;
  const int64_t beg = (int64_t)blockIdx.x * kSelRows;
  const int64_t end = cnt_in ? beg + cnt_in[slot] : (beg + kSelRows < n ? beg + kSelRows : n);
  if (end <= beg) {
    if (cnt_out && threadIdx.x == 0) cnt_out[slot] = 0;
    return;
  }
  if (threadIdx.x == 0) sh_out = 0;
  const int an = pbits ? meta[col].an : kSelMax;
  const int dshift = 28 - pbits;
  for (int e = threadIdx.x; e < an * kSelDigits; e += blockDim.x) h[e] = 0;
  if (pbits) {
    for (int i = threadIdx.x; i < an; i += blockDim.x) sp[i] = pre[col * kSelMax + i];
    for (int e = threadIdx.x; e < 4096; e += blockDim.x) tab[e] = 0;
    __syncthreads();
    for (int i = threadIdx.x; i < an; i += blockDim.x) {     // A is sorted: runs of equal top bits
      const uint32_t t = sp[i] >> (pbits - 12);
      if (i == 0 || (sp[i - 1] >> (pbits - 12)) != t) {
        int k = i + 1;
        while (k < an && (sp[k] >> (pbits - 12)) == t) ++k;
        tab[t] = ((uint32_t)i << 16) | (uint32_t)(k - i);
      }
    }
  }
  __syncthreads();
  const uint32_t* kc = kin + (int64_t)col * ldk;
  uint32_t* ko = kout ? kout + (int64_t)col * ldk : nullptr;
  const int lane = threadIdx.x & 31;
  for (int64_t i0 = beg + 8 * threadIdx.x; i0 - 8 * threadIdx.x < end; i0 += 8 * blockDim.x) {
    uint32_t k8[8];
    if (i0 + 8 <= end) {
      const uint4 a = __ldg(reinterpret_cast<const uint4*>(kc + i0));
      const uint4 b = __ldg(reinterpret_cast<const uint4*>(kc + i0 + 4));
      k8[0] = a.x; k8[1] = a.y; k8[2] = a.z; k8[3] = a.w; k8[4] = b.x; k8[5] = b.y; k8[6] = b.z; k8[7] = b.w;
    } else {
#pragma unroll
      for (int u = 0; u < 8; ++u) k8[u] = (i0 + u < end) ? kc[i0 + u] : 0u;
    }
    int ev[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      int e = -1;
      if (i0 + u < end) {
        const uint32_t key = k8[u];
        if (!pbits) {
          e = (int)(key >> 20);
        } else {
          const uint32_t kp = key >> (32 - pbits);
          const uint32_t te = tab[kp >> (pbits - 12)];
          int lo = (int)(te >> 16), cnt = (int)(te & 0xFFFFu);
          while (cnt > 1) {                                   // last entry <= kp within the run
            const int half = cnt >> 1;
            if (sp[lo + half] <= kp) lo += half;
            cnt -= half;
          }
          if (cnt && sp[lo] == kp) e = lo * kSelDigits + (int)((key >> dshift) & 15u);
        }
      }
      ev[u] = e;
      // lanes sharing lane 0's counter (a dominant value) add once; the others add their own
      const int e0 = __shfl_sync(0xffffffffu, e, 0);
      const unsigned same = __ballot_sync(0xffffffffu, e == e0);
      if (e == e0) {
        if (lane == 0 && e0 >= 0) atomicAdd(&h[e0], (uint32_t)__popc(same));
      } else if (e >= 0) {
        atomicAdd(&h[e], 1u);
      }
    }
    if (ko) {                                                 // compact the matched keys: one warp scan per 8 keys
      int mine = 0;
#pragma unroll
      for (int u = 0; u < 8; ++u) mine += ev[u] >= 0;
      int x = mine;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) { const int y = __shfl_up_sync(0xffffffffu, x, o); if (lane >= o) x += y; }
      int wbase = 0;
      if (lane == 31 && x) wbase = atomicAdd(&sh_out, x);
      wbase = __shfl_sync(0xffffffffu, wbase, 31) + x - mine;
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (ev[u] >= 0) ko[beg + wbase++] = k8[u];
    }
  }
  __syncthreads();
  if (cnt_out && threadIdx.x == 0) cnt_out[slot] = sh_out;
  uint32_t* gh = ghist + (int64_t)col * kSelHist;
  for (int e = threadIdx.x; e < an * kSelDigits; e += blockDim.x)
    if (h[e]) atomicAdd(&gh[e], h[e]);
}

__device__ __forceinline__ uint32_t sel_rank(int j, int64_t n, int B) { return (uint32_t)(((int64_t)j * n) / B); }

// one block of kSelMax threads per column: the next prefix list (and re-zeroed counters)
__global__ void __launch_bounds__(kSelMax)
k_sel_refine(int64_t n, int B, int first, SelMeta* __restrict__ meta, uint32_t* __restrict__ pre,
             uint32_t* __restrict__ base, uint32_t* __restrict__ ghist) {
  __shared__ uint32_t ws[kSelMax / 32];
  __shared__ int sh_total;
  const int col = blockIdx.x, t = threadIdx.x;
  const int lane = t & 31, w = t >> 5;
  const int an = first ? kSelMax : meta[col].an, mode = meta[col].mode;
  uint32_t c[kSelDigits];
  uint32_t p0 = 0, b0 = 0, tot = 0;
  uint32_t* gh = ghist + (int64_t)col * kSelHist;
  if (t < an) {
    p0 = first ? (uint32_t)t : pre[col * kSelMax + t];        // first pass: A = all 8-bit prefixes
    b0 = first ? 0u : base[col * kSelMax + t];
#pragma unroll
    for (int d = 0; d < kSelDigits; ++d) { c[d] = gh[t * kSelDigits + d]; gh[t * kSelDigits + d] = 0; tot += c[d]; }
  } else {
#pragma unroll
    for (int d = 0; d < kSelDigits; ++d) c[d] = 0;
  }
  // block exclusive scan helper (kSelMax threads)
  auto scan = [&](uint32_t v) -> uint32_t {
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) { const uint32_t y = __shfl_up_sync(0xffffffffu, x, o); if (lane >= o) x += y; }
    if (lane == 31) ws[w] = x;
    __syncthreads();
    if (t == 0) {
      uint32_t acc = 0;
      for (int k = 0; k < kSelMax / 32; ++k) { const uint32_t q = ws[k]; ws[k] = acc; acc += q; }
      sh_total = (int)acc;
    }
    __syncthreads();
    const uint32_t r = ws[w] + x - v;
    __syncthreads();
    return r;
  };
  if (first) b0 = scan(tot);
  uint32_t nzmask = 0;
#pragma unroll
  for (int d = 0; d < kSelDigits; ++d) nzmask |= (c[d] ? 1u : 0u) << d;
  uint32_t off = scan((uint32_t)__popc(nzmask));
  const int N = sh_total;
  uint32_t keep = nzmask;
  int new_mode = mode;
  if (mode == 1 || N > B) {
    new_mode = 1;                                  // keep the prefixes holding a target rank
    keep = 0;
    if (t < an && tot) {
      const uint32_t lo = b0, hi = b0 + tot;       // ranks [lo, hi)
      int j = (int)(((int64_t)lo * B) / n);
      while (j > 0 && sel_rank(j, n, B) >= lo) --j;
      while (j < B && sel_rank(j, n, B) < lo) ++j;
      for (; j < B && sel_rank(j, n, B) < hi; ++j) {
        const uint32_t r = sel_rank(j, n, B) - lo;
        uint32_t acc = 0;
        int d = 0;
        while (acc + c[d] <= r) { acc += c[d]; ++d; }
        keep |= 1u << d;
      }
    }
    off = scan((uint32_t)__popc(keep));
  }
  const int total = sh_total;
  if (t < an) {
    uint32_t acc = b0, k = off;
#pragma unroll
    for (int d = 0; d < kSelDigits; ++d) {
      if ((keep >> d) & 1u) {
        pre[col * kSelMax + k] = (p0 << 4) | (uint32_t)d;
        base[col * kSelMax + k] = acc;
        ++k;
      }
      acc += c[d];
    }
  }
  if (t == 0) { meta[col].an = total; meta[col].mode = new_mode; }
}

// cuts and nbins from the final (full-key) list (reading R14)
__global__ void k_sel_cuts(int64_t n, int B, const SelMeta* __restrict__ meta, const uint32_t* __restrict__ pre,
                           const uint32_t* __restrict__ base, float* __restrict__ cuts, int32_t* __restrict__ nbins) {
  const int col = blockIdx.x;
  float* cut = cuts + (int64_t)col * (B - 1);
  for (int j = threadIdx.x; j < B - 1; j += blockDim.x) cut[j] = __int_as_float(0x7f800000);   // +inf
  __syncthreads();
  if (threadIdx.x) return;
  const int an = meta[col].an;
  const uint32_t* P = pre + col * kSelMax;
  const uint32_t* R = base + col * kSelMax;
  if (meta[col].mode == 0) {                       // rule (i): every distinct value but the smallest
    for (int k = 1; k < an; ++k) cut[k - 1] = key2f(P[k]);
    nbins[col] = an;
    return;
  }
  // rule (ii): s[floor(j n / B)], j = 1..B-1, deduplicated, those <= s[0] dropped
  const uint32_t s0 = P[0];
  int k = 0, e = 0;
  uint32_t last = 0;
  for (int j = 1; j <= B - 1; ++j) {
    const uint32_t r = sel_rank(j, n, B);
    while (e + 1 < an && R[e + 1] <= r) ++e;      // last entry starting at or before rank r
    const uint32_t v = P[e];
    if (v <= s0) continue;
    if (k > 0 && v == last) continue;
    cut[k++] = key2f(v);
    last = v;
  }
  nbins[col] = k + 1;
}

// bins[i*ld + c0 + j] = #{cuts_j <= X[i, c0 + j]}: lanes over the tile's columns, rows strided.
// 1024-thread blocks (two per SM share the 64-column cut table's 65 KB each) and 4 rows per
// thread keep enough loads in flight: the kernel is bound by the latency of X.
constexpr int kApplyThreads = 1024;
__global__ void __launch_bounds__(kApplyThreads)
k_bin_apply(const float* __restrict__ X, int64_t n, int64_t ld_x, int c0, int tc, int B,
            const float* __restrict__ cuts, const int32_t* __restrict__ nbins, uint8_t* __restrict__ bins,
            int64_t ld_bins) {
  extern __shared__ float sc[];          // [tc][B-1]
  __shared__ int nc[kBinTC];
  for (int e = threadIdx.x; e < tc * (B - 1); e += blockDim.x) sc[e] = cuts[(int64_t)c0 * (B - 1) + e];
  for (int j = threadIdx.x; j < tc; j += blockDim.x) nc[j] = nbins[c0 + j] - 1;
  __syncthreads();
  const int j = threadIdx.x % kBinTC, r0 = threadIdx.x / kBinTC;
  constexpr int RPB = kApplyThreads / kBinTC;   // rows per block iteration
  if (j >= tc) return;
  const float* c = sc + j * (B - 1);
  const int ncut = nc[j];
  constexpr int U = 4;                   // rows per thread per step (loads issued first)
  const int64_t step = (int64_t)gridDim.x * RPB;
  for (int64_t i = (int64_t)blockIdx.x * RPB + r0; i < n; i += U * step) {
    float x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = (i + u * step < n) ? __ldg(&X[(i + u * step) * ld_x + c0 + j]) : 0.0f;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      int lo = 0;                        // #cuts <= x (ncut <= 255)
#pragma unroll
      for (int st = 128; st > 0; st >>= 1)
        if (lo + st <= ncut && c[lo + st - 1] <= x[u]) lo += st;
      if (i + u * step < n) bins[(i + u * step) * ld_bins + c0 + j] = (uint8_t)lo;
    }
  }
}

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

// ---- CSC input (values, row indices, column pointers; absent entries are 0)

// keys of the tile's stored values, column by column (ka[j*ldk + i], i < nnz_j); per column the
// number of implicit zeros, and per (column, block) the number of stored keys the block reads
__global__ void k_csc_keys(const float* __restrict__ values, const int64_t* __restrict__ col_ptr, int64_t n, int c0,
                           uint32_t* __restrict__ keys, int64_t ldk, int32_t* __restrict__ zeros,
                           int32_t* __restrict__ cnt0, int row_blocks) {
  const int j = blockIdx.y;
  const int64_t p0 = col_ptr[c0 + j], nz = col_ptr[c0 + j + 1] - p0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nz; i += (int64_t)gridDim.x * blockDim.x)
    keys[(int64_t)j * ldk + i] = f2key(values[p0 + i]);
  if (blockIdx.x == 0) {
    if (threadIdx.x == 0) zeros[j] = (int32_t)(n - nz);
    for (int b = threadIdx.x; b < row_blocks; b += blockDim.x) {
      const int64_t left = nz - (int64_t)b * kSelRows;
      cnt0[(int64_t)j * row_blocks + b] = (int32_t)(left <= 0 ? 0 : (left < kSelRows ? left : kSelRows));
    }
  }
}

// the implicit zeros of each column join the counters of this pass (if their prefix is in A)
__global__ void k_sel_zeros(int tc, int pbits, const int32_t* __restrict__ zeros, const SelMeta* __restrict__ meta,
                            const uint32_t* __restrict__ pre, uint32_t* __restrict__ ghist) {
  const int col = blockIdx.x * blockDim.x + threadIdx.x;
  if (col >= tc || zeros[col] <= 0) return;
  const uint32_t key0 = f2key(0.0f);
  int e = -1;
  if (!pbits) {
    e = (int)(key0 >> 20);
  } else {
    const uint32_t kp = key0 >> (32 - pbits);
    const int an = meta[col].an;
    for (int i = 0; i < an; ++i)
      if (pre[col * kSelMax + i] == kp) { e = i * kSelDigits + (int)((key0 >> (28 - pbits)) & 15u); break; }
  }
  if (e >= 0) ghist[(int64_t)col * kSelHist + e] += (uint32_t)zeros[col];
}

// bins of a CSC column tile: every row gets bin(0) of its column, then the stored values theirs
__global__ void k_csc_zero_bins(int64_t n, int c0, int tc, int B, const float* __restrict__ cuts,
                                const int32_t* __restrict__ nbins, uint8_t* __restrict__ bins, int64_t ld_bins) {
  __shared__ uint8_t zb[kBinTC];
  for (int j = threadIdx.x; j < tc; j += blockDim.x) {
    const float* c = cuts + (int64_t)(c0 + j) * (B - 1);
    const int nc = nbins[c0 + j] - 1;
    int k = 0;
    while (k < nc && c[k] <= 0.0f) ++k;
    zb[j] = (uint8_t)k;
  }
  __syncthreads();
  const int64_t total = n * tc;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / tc;
    const int j = (int)(e - i * tc);
    bins[i * ld_bins + c0 + j] = zb[j];
  }
}

__global__ void __launch_bounds__(256)
k_csc_apply(const float* __restrict__ values, const int32_t* __restrict__ row_idx, const int64_t* __restrict__ col_ptr,
            int c0, int B, const float* __restrict__ cuts, const int32_t* __restrict__ nbins,
            uint8_t* __restrict__ bins, int64_t ld_bins) {
  __shared__ float c[256];
  const int j = blockIdx.y;
  for (int k = threadIdx.x; k < B - 1; k += blockDim.x) c[k] = cuts[(int64_t)(c0 + j) * (B - 1) + k];
  __syncthreads();
  const int ncut = nbins[c0 + j] - 1;
  const int64_t p0 = col_ptr[c0 + j], p1 = col_ptr[c0 + j + 1];
  for (int64_t p = p0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < p1; p += (int64_t)gridDim.x * blockDim.x) {
    const float x = values[p];
    int lo = 0;
#pragma unroll
    for (int st = 128; st > 0; st >>= 1)
      if (lo + st <= ncut && c[lo + st - 1] <= x) lo += st;
    bins[(int64_t)row_idx[p] * ld_bins + c0 + j] = (uint8_t)lo;
  }
}

struct SelWs {
  int64_t ldk;
  unsigned row_blocks;
  uint32_t *ka, *kb, *pre, *base, *ghist;
  SelMeta* meta;
  int32_t *cnt_a, *cnt_b, *cnt_0, *zeros;
};

// workspace: keys, compacted keys [tc][ldk] u32 | meta [tc] | prefixes, bases [tc][kSelMax] u32 |
// counters [tc][kSelHist] u32 | kept-key counts 3 x [tc][row blocks] i32 | implicit zeros [tc] i32
static size_t sel_ws_bytes(int64_t n, int32_t m) {
  const int64_t tc = m < kBinTC ? m : kBinTC;
  const int64_t rb = (n + kSelRows - 1) / kSelRows;
  return (size_t)(2 * tc * ((n + 3) / 4 * 4) * 4 + tc * (int64_t)sizeof(SelMeta) + 2 * tc * kSelMax * 4 +
                  tc * kSelHist * 4 + 3 * tc * rb * 4 + tc * 4 + 1024);
}

static SelWs sel_ws(void* ws, int64_t n, int32_t m) {
  SelWs w;
  const int64_t tcmax = m < kBinTC ? m : kBinTC;
  w.ldk = (n + 3) / 4 * 4;                                 // 16-byte aligned key columns
  w.row_blocks = (unsigned)((n + kSelRows - 1) / kSelRows);
  w.ka = (uint32_t*)ws;
  w.kb = w.ka + tcmax * w.ldk;
  w.meta = (SelMeta*)(w.kb + tcmax * w.ldk);
  w.pre = (uint32_t*)(w.meta + tcmax);
  w.base = w.pre + tcmax * kSelMax;
  w.ghist = w.base + tcmax * kSelMax;
  w.cnt_a = (int32_t*)(w.ghist + tcmax * kSelHist);       // kept keys per (column, block)
  w.cnt_b = w.cnt_a + tcmax * w.row_blocks;
  w.cnt_0 = w.cnt_b + tcmax * w.row_blocks;               // CSC: stored keys per (column, block)
  w.zeros = w.cnt_0 + tcmax * w.row_blocks;
  return w;
}

// cuts and nbins of a column tile whose keys are in w.ka.  csc: w.cnt_0 / w.zeros describe the
// stored keys and the implicit zeros of each column.
static gbdtmo_status run_selection(Ctx* ctx, const SelWs& w, int64_t n, int tc, int B, bool csc, float* cuts, int32_t* nbins) {
  GB_LAUNCH(k_sel_init, (unsigned)tc, 256, 0, tc, w.meta, w.pre, w.base, w.ghist);
  // prefix bits before each pass: 0 (12-bit digit), then 12, 16, 20, 24, 28 (4-bit digits);
  // from 16 bits on, the matched keys are compacted and only they are read by the next pass
  const int pb[6] = {0, 12, 16, 20, 24, 28};
  for (int k = 0; k < 6; ++k) {
    const bool rd_c = pb[k] >= 20, wr_c = pb[k] >= 16 && pb[k] <= 24;
    const uint32_t* kin = (pb[k] == 20 || pb[k] == 28) ? w.kb : w.ka;
    uint32_t* kout = wr_c ? (pb[k] == 20 ? w.ka : w.kb) : nullptr;
    const int32_t* cin = rd_c ? ((pb[k] == 24) ? w.cnt_b : w.cnt_a) : (csc ? w.cnt_0 : nullptr);
    int32_t* cout = wr_c ? ((pb[k] == 20) ? w.cnt_b : w.cnt_a) : nullptr;
    GB_LAUNCH(k_sel_count, dim3(w.row_blocks, (unsigned)tc), 256, 0, kin, cin, n, w.ldk, pb[k], w.meta, w.pre, w.ghist,
              kout, cout);
    if (csc) GB_LAUNCH(k_sel_zeros, (unsigned)((tc + 63) / 64), 64, 0, tc, pb[k], w.zeros, w.meta, w.pre, w.ghist);
    GB_LAUNCH(k_sel_refine, (unsigned)tc, kSelMax, 0, n, B, (int)(pb[k] == 0), w.meta, w.pre, w.base, w.ghist);
  }
  GB_LAUNCH(k_sel_cuts, (unsigned)tc, 256, 0, n, B, w.meta, w.pre, w.base, cuts, nbins);
  return GBDTMO_OK;
}

void ctx_release_streams(Ctx* ctx) {
  if (!ctx->copy_stream) return;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(ctx->device);
  cudaStreamSynchronize(ctx->copy_stream);
  for (int i = 0; i < 2; ++i) {
    if (ctx->strip_ready[i]) cudaEventDestroy(ctx->strip_ready[i]);
    if (ctx->strip_free[i]) cudaEventDestroy(ctx->strip_free[i]);
    ctx->strip_ready[i] = ctx->strip_free[i] = nullptr;
  }
  cudaStreamDestroy(ctx->copy_stream);
  ctx->copy_stream = nullptr;
  cudaGetLastError();
  cudaSetDevice(prev);
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" size_t gbdtmo_bin_host_workspace_bytes(int64_t n, int32_t m, int32_t B, int32_t strip) {
  const int64_t sw = strip < m ? strip : m;
  const size_t stage = (size_t)(align_up((size_t)n * sw * 4, 256));
  return 2 * stage + sel_ws_bytes(n, (int32_t)sw);
}

extern "C" size_t gbdtmo_bin_workspace_bytes(int64_t n, int32_t m, int32_t B) {
  (void)B;
  return sel_ws_bytes(n, m);
}

extern "C" gbdtmo_status gbdtmo_bin(gbdtmo_ctx c, const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t B,
                                    uint8_t* bins, int64_t ld_bins, float* cuts, int32_t* nbins, void* ws,
                                    size_t ws_bytes) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(X && bins && cuts && nbins && ws, "null pointer");
  GB_CHECK_ARG(((uintptr_t)ws & 15) == 0, "ws must be 16-byte aligned");
  GB_CHECK_ARG(n >= 1 && n < (int64_t(1) << 31) && m >= 1, "bad n or m");
  GB_CHECK_ARG(ld_x >= m && ld_bins >= m, "bad leading dimension");
  if (B > 256) { ctx->err = "gbdtmo_bin: B > 256 unsupported (bins are uint8)"; return GBDTMO_EUNSUPPORTED; }
  GB_CHECK_ARG(B >= 2, "B < 2");
  if (ws_bytes < gbdtmo_bin_workspace_bytes(n, m, B)) { ctx->err = "gbdtmo_bin: workspace too small"; return GBDTMO_ENOMEM; }
  const SelWs w = sel_ws(ws, n, m);
  static unsigned long long attr_mask = 0;
  smem_optin_once(ctx, k_bin_apply, attr_mask, kBinTC * 255 * 4);
  for (int c0 = 0; c0 < m; c0 += kBinTC) {
    const int tc = (int)(m - c0 < kBinTC ? m - c0 : kBinTC);
    GB_LAUNCH(k_bin_keys, dim3((unsigned)((n + 31) / 32), (unsigned)((tc + 31) / 32)), dim3(32, 8), 0, X, n, ld_x, c0,
              tc, w.ka, w.ldk);
    const gbdtmo_status st = run_selection(ctx, w, n, tc, B, false, cuts + (int64_t)c0 * (B - 1), nbins + c0);
    if (st != GBDTMO_OK) return st;
    GB_LAUNCH(k_bin_apply, ctx->num_sms * 2, kApplyThreads, (size_t)tc * (B - 1) * 4, X, n, ld_x, c0, tc, B, cuts,
              nbins, bins, ld_bins);
  }
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_bin_host(gbdtmo_ctx c, const float* X_host, int64_t n, int32_t m, int64_t ld_x,
                                         int32_t B, uint8_t* bins, int64_t ld_bins, float* cuts, int32_t* nbins,
                                         void* ws, size_t ws_bytes, int32_t strip) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(X_host && bins && cuts && nbins && ws, "null pointer");
  GB_CHECK_ARG(((uintptr_t)ws & 255) == 0, "ws must be 256-byte aligned");
  GB_CHECK_ARG(n >= 1 && n < (int64_t(1) << 31) && m >= 1 && strip >= 1, "bad n, m or strip");
  GB_CHECK_ARG(ld_x >= m && ld_bins >= m, "bad leading dimension");
  if (B > 256) { ctx->err = "gbdtmo_bin_host: B > 256 unsupported (bins are uint8)"; return GBDTMO_EUNSUPPORTED; }
  GB_CHECK_ARG(B >= 2, "B < 2");
  if (ws_bytes < gbdtmo_bin_host_workspace_bytes(n, m, B, strip)) {
    ctx->err = "gbdtmo_bin_host: workspace too small";
    return GBDTMO_ENOMEM;
  }
  if (!ctx->copy_stream) {
    if (cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking) != cudaSuccess) {
      ctx->err = std::string("gbdtmo_bin_host: ") + cudaGetErrorString(cudaGetLastError());
      ctx->copy_stream = nullptr;
      return GBDTMO_ECUDA;
    }
    for (int i = 0; i < 2; ++i) {
      cudaEventCreateWithFlags(&ctx->strip_ready[i], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&ctx->strip_free[i], cudaEventDisableTiming);
    }
  }
  const int32_t sw = strip < m ? strip : m;
  const size_t stage = align_up((size_t)n * sw * 4, 256);
  float* buf[2] = {reinterpret_cast<float*>(ws), reinterpret_cast<float*>((char*)ws + stage)};
  void* bws = (char*)ws + 2 * stage;
  const size_t bws_bytes = ws_bytes - 2 * stage;
  // column strips: strip k is copied (copy stream) into buf[k % 2] while strip k - 1 is binned (the
  // context's stream); binning is per column, so a strip's bins, cuts and nbins are final
  for (int32_t k = 0, f0 = 0; f0 < m; ++k, f0 += sw) {
    const int32_t w = m - f0 < sw ? m - f0 : sw;
    const int j = k & 1;
    if (k >= 2) cudaStreamWaitEvent(ctx->copy_stream, ctx->strip_free[j], 0);   // strip k-2 binned
    cudaMemcpy2DAsync(buf[j], (size_t)w * 4, X_host + f0, (size_t)ld_x * 4, (size_t)w * 4, (size_t)n,
                      cudaMemcpyHostToDevice, ctx->copy_stream);
    cudaEventRecord(ctx->strip_ready[j], ctx->copy_stream);
    cudaStreamWaitEvent(ctx->stream, ctx->strip_ready[j], 0);
    GB_CHECK_LAUNCH();
    const gbdtmo_status st = gbdtmo_bin(c, buf[j], n, w, w, B, bins + f0, ld_bins, cuts + (int64_t)f0 * (B - 1),
                                        nbins + f0, bws, bws_bytes);
    if (st != GBDTMO_OK) return st;
    cudaEventRecord(ctx->strip_free[j], ctx->stream);
  }
  GB_CHECK_LAUNCH();
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_bin_csc(gbdtmo_ctx c, const float* values, const int32_t* row_idx,
                                        const int64_t* col_ptr, const int64_t* col_ptr_host, int64_t n, int32_t m,
                                        int32_t B, uint8_t* bins, int64_t ld_bins, float* cuts, int32_t* nbins,
                                        void* ws, size_t ws_bytes) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(col_ptr && col_ptr_host && bins && cuts && nbins && ws, "null pointer");
  GB_CHECK_ARG(((uintptr_t)ws & 15) == 0, "ws must be 16-byte aligned");
  GB_CHECK_ARG(n >= 1 && n < (int64_t(1) << 31) && m >= 1, "bad n or m");
  GB_CHECK_ARG(ld_bins >= m, "bad leading dimension");
  if (B > 256) { ctx->err = "gbdtmo_bin_csc: B > 256 unsupported (bins are uint8)"; return GBDTMO_EUNSUPPORTED; }
  GB_CHECK_ARG(B >= 2, "B < 2");
  GB_CHECK_ARG(col_ptr_host[0] == 0, "col_ptr[0] must be 0");
  for (int32_t j = 0; j < m; ++j)
    GB_CHECK_ARG(col_ptr_host[j + 1] >= col_ptr_host[j] && col_ptr_host[j + 1] - col_ptr_host[j] <= n,
                 "col_ptr must be non-decreasing with at most n entries per column");
  GB_CHECK_ARG(col_ptr_host[m] == 0 || (values && row_idx), "null values / row_idx");
  if (ws_bytes < gbdtmo_bin_workspace_bytes(n, m, B)) { ctx->err = "gbdtmo_bin_csc: workspace too small"; return GBDTMO_ENOMEM; }
  const SelWs w = sel_ws(ws, n, m);
  for (int c0 = 0; c0 < m; c0 += kBinTC) {
    const int tc = (int)(m - c0 < kBinTC ? m - c0 : kBinTC);
    int64_t maxnz = 1;
    for (int j = 0; j < tc; ++j) {
      const int64_t nz = col_ptr_host[c0 + j + 1] - col_ptr_host[c0 + j];
      maxnz = nz > maxnz ? nz : maxnz;
    }
    const unsigned gx = (unsigned)((maxnz + 255) / 256 < 1024 ? (maxnz + 255) / 256 : 1024);
    GB_LAUNCH(k_csc_keys, dim3(gx, (unsigned)tc), 256, 0, values, col_ptr, n, c0, w.ka, w.ldk, w.zeros, w.cnt_0,
              (int)w.row_blocks);
    const gbdtmo_status st = run_selection(ctx, w, n, tc, B, true, cuts + (int64_t)c0 * (B - 1), nbins + c0);
    if (st != GBDTMO_OK) return st;
    GB_LAUNCH(k_csc_zero_bins, ctx->num_sms * 4, 256, 0, n, c0, tc, B, cuts, nbins, bins, ld_bins);
    GB_LAUNCH(k_csc_apply, dim3(gx, (unsigned)tc), 256, 0, values, row_idx, col_ptr, c0, B, cuts, nbins, bins, ld_bins);
  }
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_default_bins(gbdtmo_ctx c, const uint8_t* bins, int64_t n, int32_t m, int64_t ld_bins,
                                             int32_t B, int64_t min_count, int32_t* dflt) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(bins && dflt, "null pointer");
  GB_CHECK_ARG(n >= 1 && m >= 1 && ld_bins >= m && ld_bins % 8 == 0 && B >= 2 && B <= 256, "bad shape");
  GB_CHECK_ARG(((uintptr_t)bins & 7) == 0, "bins must be 8-byte aligned");
  GB_LAUNCH(k_default_bins, (unsigned)((m + 7) / 8), 256, 0, bins, n, m, ld_bins, B, min_count, dflt);
  return GBDTMO_OK;
}
